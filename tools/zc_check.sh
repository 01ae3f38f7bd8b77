#!/bin/bash
# zero-copy C auto rule: host-API tests + e2e on every config (gpurun_out/zk_*)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spmm.py -k "host_api" -q -p no:cacheprovider > gpurun_out/zk_pytest.log 2>&1
for cfg in c3h c3 c2; do
  timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/zk_${cfg}.json 2>/dev/null
done
DTC_HOST_ZC=0 timeout 600 python bench.py --config c3h --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/zk_c3h_off.json 2>/dev/null
