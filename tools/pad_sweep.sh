#!/bin/bash
mkdir -p gpurun_out
run() {  # tag so env...
  tag=$1; so=$2; shift 2
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    env "$@" DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/pd_${tag}_$c.json 2> gpurun_out/pd_${tag}_$c.err
  done
}
run ldg vsos/ldg.so X=1
run pad vsos/pad.so X=1
run pads8 vsos/pad_s8.so X=1
run pads16 vsos/pad_s16.so X=1
CONFIGS="c3 c5" run padsl4 vsos/pad.so DTC_PAD_SL=4
CONFIGS="c3 c3h c5" run padsl1 vsos/pad.so DTC_PAD_SL=1
