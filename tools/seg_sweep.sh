#!/bin/bash
mkdir -p gpurun_out
run() {  # tag args env...
  tag=$1; args=$2; shift 2
  for c in ${CONFIGS:-c3 c5}; do
    env "$@" timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e $args > gpurun_out/${PFX}_${tag}_$c.json 2> gpurun_out/${PFX}_${tag}_$c.err
  done
}
run seg8 "" X=1
run seg4 "" DTC_PAD_SEG=4
run seg8sl2 "" DTC_PAD_SL=2
CONFIGS="c3 c3h c5" run seg8u512 "--unit-blocks 512" X=1
CONFIGS="c2 c3h c4" run base "" X=1
