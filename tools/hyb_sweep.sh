#!/bin/bash
# Hybrid gather experiment (DTC_PAD_HYB=1) vs the default pad path, same box, bench lines per config.
mkdir -p gpurun_out
for c in c2 c3 c3h c4 c5; do
  for h in 0 1; do
    DTC_PAD_HYB=$h timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/hyb${h}_$c.json 2> gpurun_out/hyb${h}_$c.err
  done
done
