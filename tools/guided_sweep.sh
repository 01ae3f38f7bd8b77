#!/bin/bash
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c4 c3 c5 c3h}; do for G in 0 -1; do
  timeout 300 python bench.py --config $c --guided $G --steps 20 --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/gs_${c}_G$G.json 2>/dev/null
done; done
