#!/bin/bash
# F4 unit-size sweep for the TMA (pad) path -> gpurun_out/pu_u<U>_<cfg>.json
mkdir -p gpurun_out
for U in ${US:-32 48 64 96 128 192 256 384 512}; do
  for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
    DTC_LIBRARY=$PWD/${SO:-vsos/pad_s4.so} timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e --unit-blocks $U > gpurun_out/pu_u${U}_$c.json 2> gpurun_out/pu_u${U}_$c.err
  done
done
