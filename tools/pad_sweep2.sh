#!/bin/bash
mkdir -p gpurun_out
run() {  # tag so args env...
  tag=$1; so=$2; args=$3; shift 3
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    env "$@" DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e $args > gpurun_out/pe_${tag}_$c.json 2> gpurun_out/pe_${tag}_$c.err
  done
}
for k in 3 4 6 8 10; do run s$k vsos/pad_s$k.so "" X=1; done
for U in 16 64 128; do CONFIGS="c2 c4" run s6u$U vsos/pad_s6.so "--unit-blocks $U" X=1; CONFIGS="c2 c4" run s4u$U vsos/pad_s4.so "--unit-blocks $U" X=1; done
CONFIGS="c3 c5" run s4sl4 vsos/pad_s4.so "" DTC_PAD_SL=4
CONFIGS="c3 c5" run s3sl4 vsos/pad_s3.so "" DTC_PAD_SL=4
