#!/bin/bash
# NEXT-2 A/B on one box: 16-row ME-TCF vs 32-row windows, every TF32 workload, two reps; then tests
mkdir -p gpurun_out; out=gpurun_out/ab_tall.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
for rep in 1 2; do
  for wr in 16 32; do
    $B --window-rows $wr --legs c2,c4:64,c4:128,c4:256,c5 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
rows=[(d['config']['workload'][:3],d['config']['N'],d['value'],d['config'].get('num_tc_blocks'),d.get('clocks',{}).get('sm_mhz'))]
rows+=[(l['config'],l['N'],l['value'],l['num_tc_blocks'],l['clocks']['sm_mhz']) for l in d['legs']]
for r in rows: print('wr=$wr', *r)
" >> $out
  done
done
cat $out
timeout 1800 python -m pytest tests/test_gpu_paths.py tests/test_gpu_format.py -m gpu -x -q -p no:cacheprovider > gpurun_out/tall_pytest.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_spmm.py -m gpu -x -q -p no:cacheprovider -k "tall" > gpurun_out/tall_pytest2.log 2>&1
