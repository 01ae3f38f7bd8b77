#!/bin/bash
mkdir -p gpurun_out
run() {  # tag so args env...
  tag=$1; so=$2; args=$3; shift 3
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    env "$@" DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e $args > gpurun_out/${PFX}_${tag}_$c.json 2> gpurun_out/${PFX}_${tag}_$c.err
  done
}
for v in np b8a3 b16a3 b8a4 b8a3s3 b8a3s6; do run $v vsos/$v.so "" X=1; done
CONFIGS="c2 c4" run b8a3u32 vsos/b8a3.so "--unit-blocks 32" X=1
CONFIGS="c2 c4 c5" run b8a3u128 vsos/b8a3.so "--unit-blocks 128" X=1
