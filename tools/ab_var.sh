#!/bin/bash
# A/B of build variants (build_variants/<name>/libdtc.so) on one box; VARS and LEGS from the env
mkdir -p gpurun_out; out=gpurun_out/ab_var.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
run() {
  lab=$1; shift
  timeout 400 env "$@" | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
rows=[(d['config']['workload'][:3],d['config']['N'],d['value'],d.get('clocks',{}).get('sm_mhz'))]
rows+=[(l['config'],l['N'],l['value'],l['clocks']['sm_mhz']) for l in d['legs']]
for r in rows: print('$lab', *r)
" >> $out
}
for rep in 1 2; do
  for v in default ${VARS}; do
    if [ $v = default ]; then L=""; else L="DTC_LIBRARY=$PWD/${VDIR:-vbuild}/$v/libdtc.so"; fi
    run $v $L $B --legs ${LEGS:-c2,c4:128,c4:256,c5} 2>/dev/null
  done
done
cat $out
