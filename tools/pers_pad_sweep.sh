#!/bin/bash
# Persistent padded-row launch (DTC_PAD_PERS=1) vs one CTA per unit, and unit sizes, per config.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
  for p in 0 1; do
    for U in ${UNITS:-0 16 32}; do
      DTC_PAD_PERS=$p timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e --unit-blocks $U > gpurun_out/pp${p}_u${U}_$c.json 2> gpurun_out/pp${p}_u${U}_$c.err
    done
  done
done
