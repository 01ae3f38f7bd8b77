#!/bin/bash
# DTC_HOST_ZC=0/1 (C stored straight into pinned host memory) x chunk counts: e2e (gpurun_out/zc_*)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spmm.py -k "host_api" -q -p no:cacheprovider > gpurun_out/zc_pytest.log 2>&1
for cfg in c2 c3 c4 c5; do
  for z in 0 1; do
    DTC_HOST_ZC=$z timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/zc_${cfg}_${z}_d.json 2>/dev/null
  done
done
for c in 1 2 4; do
  DTC_HOST_ZC=1 DTC_HOST_CHUNKS=$c timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/zc_c2_1_$c.json 2>/dev/null
done
