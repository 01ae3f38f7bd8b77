#!/bin/bash
# Dual-engine gather: every k-th block by cp.async (DTC_PAD_LSU=k), 0 = TMA only.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
  for k in ${KS:-0 4 3 2}; do
    DTC_PAD_LSU=$k timeout 300 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cusparse --no-cpu --no-e2e --graphconv 0 --tca 0 > gpurun_out/lsu${k}_$c.json 2> gpurun_out/lsu${k}_$c.err
  done
done
