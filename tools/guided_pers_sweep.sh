#!/bin/bash
# Persistent launch x guided F4 tail (units of U/2 over the last ~half wave) x unit size.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c4 c3h}; do
  for m in ${MODES:-"0,0,0" "1,32,1" "1,0,1" "1,16,1" "0,32,1"}; do
    IFS=, read p u g <<< "$m"
    DTC_PAD_PERS=$p timeout 300 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cusparse --no-cpu --no-e2e --graphconv 0 --tca 0 --unit-blocks $u --guided $g > gpurun_out/g_p${p}_u${u}_g${g}_$c.json 2> gpurun_out/g_p${p}_u${u}_g${g}_$c.err
  done
done
