#!/bin/bash
mkdir -p gpurun_out; out=gpurun_out/ab_na.txt; : > $out
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
for v in na3 na2 na4 coop0; do
  for k in 1 2; do
    if [ $v = na3 ]; then L=""; else L="DTC_LIBRARY=$PWD/build_variants/$v/libdtc.so"; fi
    env $L python tools/dbg_coop.py c2 256 2>&1 | head -2 | sed "s/^/$v /" >> gpurun_out/ab_na_dbg.txt
    env $L python tools/dbg_coop.py c5 512 2>&1 | head -2 | sed "s/^/$v /" >> gpurun_out/ab_na_dbg.txt
  done
done
for rep in 1 2; do
  run na3 $B --legs c3h,c4:256,c5 2>/dev/null
  run na2 DTC_LIBRARY=$PWD/build_variants/na2/libdtc.so $B --legs c3h,c4:256,c5 2>/dev/null
  run na4 DTC_LIBRARY=$PWD/build_variants/na4/libdtc.so $B --legs c3h,c4:256,c5 2>/dev/null
  run coop0 DTC_LIBRARY=$PWD/build_variants/coop0/libdtc.so $B --legs c3h,c4:256,c5 2>/dev/null
done
cat $out
