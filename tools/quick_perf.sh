#!/bin/bash
# quick perf sweep on the GPU box: dtc only, one JSON per config -> gpurun_out/qp_<cfg>.json
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3 c3h c4 c5 c1}; do
  timeout 600 python bench.py --config $c --steps ${STEPS:-30} --warmup 5 --no-cusparse --no-cpu --no-e2e $EXTRA > gpurun_out/qp_$c.json 2> gpurun_out/qp_$c.err
done
