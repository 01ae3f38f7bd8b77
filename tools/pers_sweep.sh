#!/bin/bash
mkdir -p gpurun_out
run() {  # tag so args env...
  tag=$1; so=$2; args=$3; shift 3
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    env "$@" DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e $args > gpurun_out/${PFX}_${tag}_$c.json 2> gpurun_out/${PFX}_${tag}_$c.err
  done
}
run np vsos/np.so "" X=1
run pers vsos/pers.so "" X=1
for U in 16 32 128; do CONFIGS="c2 c4 c5" run persu$U vsos/pers.so "--unit-blocks $U" X=1; done
CONFIGS="c3 c3h" run persu512 vsos/pers.so "--unit-blocks 512" X=1
