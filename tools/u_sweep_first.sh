#!/bin/bash
# c2 unit size sweep with first-batch side records on (gpurun_out/us_*)
mkdir -p gpurun_out
for rep in 1 2; do
  for u in 16 24 32 48; do
    timeout 600 python bench.py --config c2 --unit-blocks $u --steps 200 --warmup 10 --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 > gpurun_out/us_c2_${u}_$rep.json 2>/dev/null
  done
done
for u in 32 48 64; do
  timeout 600 python bench.py --config c4 --unit-blocks $u --steps 30 --warmup 5 --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 > gpurun_out/us_c4_${u}_1.json 2>/dev/null
done
