#!/bin/bash
mkdir -p gpurun_out; out=gpurun_out/ab_tall2.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
run() {
  lab=$1; shift
  env "$@" | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
rows=[(d['config']['workload'][:3],d['config']['N'],d['value'],d.get('clocks',{}).get('sm_mhz'))]
rows+=[(l['config'],l['N'],l['value'],l['clocks']['sm_mhz']) for l in d['legs']]
for r in rows: print('$lab', *r)
" >> $out
}
for rep in 1 2; do
  run auto16 $B --legs c2,c3h,c4:64,c4:128,c4:256,c5 2>/dev/null
  run tall32 $B --window-rows 32 --legs c2,c4:64,c4:128,c4:256,c5 2>/dev/null
done
cat $out
timeout 1800 python -m pytest tests/test_gpu_paths.py tests/test_gpu_format.py tests/test_gpu_spmm.py -m gpu -x -q -p no:cacheprovider -k "not full_size or tall" > gpurun_out/tall2_pytest.log 2>&1
tail -8 gpurun_out/tall2_pytest.log
