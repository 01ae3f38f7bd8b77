#!/bin/bash
# A/B of library variants on one box: r01 tree vs current (+ build variants via DTC_LIBRARY)
mkdir -p gpurun_out
out=gpurun_out/ab.txt; : > $out
NEW="python bench.py --legs none --ncu off --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
OLD="python bench.py --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 --steps 30 --warmup 5"
for rep in 1 2; do
 for c in ${CFGS:-c4 c3h c2}; do
  v=$(cd build_variants/r01 && $OLD --config $c 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['clocks']['sm_mhz'])"); echo "$c r01 $v" >> $out
  v=$($NEW --config $c 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['clocks']['sm_mhz'])"); echo "$c new $v" >> $out
  for var in ${VARS:-nopairs lbmin}; do
   v=$(DTC_LIBRARY=$PWD/build_variants/$var/libdtc.so $NEW --config $c 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['clocks']['sm_mhz'])"); echo "$c $var $v" >> $out
  done
 done
done
cat $out
