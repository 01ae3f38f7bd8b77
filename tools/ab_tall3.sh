#!/bin/bash
mkdir -p gpurun_out; out=gpurun_out/ab_tall3.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
run() {
  lab=$1; shift
  env "$@" | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
rows=[(d['config']['workload'][:3],d['config']['N'],d['value'],d['config'].get('num_tc_blocks'),d.get('clocks',{}).get('sm_mhz'))]
rows+=[(l['config'],l['N'],l['value'],l['num_tc_blocks'],l['clocks']['sm_mhz']) for l in d['legs']]
for r in rows: print('$lab', *r)
" >> $out
}
for rep in 1 2; do
  run w16 $B --legs c2,c4:64,c4:128,c4:256,c5 2>/dev/null
  run w32 $B --window-rows 32 --legs c2,c4:64,c4:128,c4:256,c5 2>/dev/null
done
cat $out
