#!/bin/bash
mkdir -p gpurun_out
for k in 1 2; do python tools/dbg_coop.py c2 256 2>&1 | head -2; python tools/dbg_coop.py c4 256 2>&1 | head -2; done > gpurun_out/g6_dbg.txt
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/g6_pytest.log 2>&1
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
$B --legs c2,c3h,c4:64,c4:128,c4:256,c5 > gpurun_out/g6_bench.json 2>/dev/null
