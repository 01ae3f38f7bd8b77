#!/bin/bash
# F4 plan A/B on one box: fixed rule vs the B200 Selector, every BASELINE workload, two reps
mkdir -p gpurun_out; out=gpurun_out/ab_sel.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
for rep in 1 2; do
  for sel in 0 1; do
    $B --selector $sel --legs c2,c3h,c4:64,c4:128,c4:256,c5 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
rows=[(d['config']['workload'][:3],d['config']['N'],d['value'],d['config'].get('unit_blocks'),d.get('clocks',{}).get('sm_mhz'))]
rows+=[(l['config'],l['N'],l['value'],l['unit_blocks'],l['clocks']['sm_mhz']) for l in d['legs']]
for r in rows: print('sel=$sel', *r)
" >> $out
  done
done
cat $out
