#!/bin/bash
# F4 unit size (and persistent launch) sweep of the default kernel on one box: GFLOP/s per
# (config, N, U); U=0 is the auto rule (auto_unit_blocks).  CFGS="c2 c3:256 c4:128" UNITS="0 16 32 64"
mkdir -p gpurun_out; out=gpurun_out/unit_sweep.txt; : > $out
B="python bench.py --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --legs none --steps 30 --warmup 5"
for cn in ${CFGS:-c2 c3 c4:64 c4:128 c5}; do
  c=${cn%%:*}; n=0; [ "$c" != "$cn" ] && n=${cn##*:}
  for U in ${UNITS:-0 16 24 32 48 64 128 256}; do
    for P in 0 ${PERS:-}; do
      timeout 400 $B --config $c --n $n --unit-blocks $U --persistent $P 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); c=d['config']
print('$c', c['N'], 'U=%s' % c.get('unit_blocks'), 'units=%s' % c.get('num_units'), 'pers=$P', d['value'], d.get('clocks',{}).get('sm_mhz'))
" >> $out
    done
  done
done
cat $out
