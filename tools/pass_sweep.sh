#!/bin/bash
# direct-path pass-width sweep (DTC_PASS_WS) + ldg baseline -> gpurun_out/ps_<tag>_<cfg>.json
mkdir -p gpurun_out
run() {  # tag so env...
  tag=$1; so=$2; shift 2
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    env "$@" DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/ps_${tag}_$c.json 2> gpurun_out/ps_${tag}_$c.err
  done
}
run ldg vsos/ldg.so X=1
run dir_auto vsos/dir96.so X=1
run dir_p1 vsos/dir96.so DTC_PASS_WS=1
run dir_p2 vsos/dir96.so DTC_PASS_WS=2
run dir_p99 vsos/dir96.so DTC_PASS_WS=99
