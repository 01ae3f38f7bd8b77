#!/bin/bash
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c4 c3h}; do for U in ${US:-12 16 24 32 48 64 96 128 256}; do
  timeout 300 python bench.py --config $c --unit-blocks $U --steps 15 --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/us_${c}_U$U.json 2>/dev/null
done; done
