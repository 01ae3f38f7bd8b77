#!/bin/bash
# e2e (dtc_spmm_host) vs DTC_HOST_CHUNKS on c2 and c5-sized calls; outputs gpurun_out/hc_*.json
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_spmm.py -k "host_api" -q -p no:cacheprovider > gpurun_out/hc_pytest.log 2>&1
for cfg in c2 c3 c5; do
  for c in 1 2 4 8; do
    DTC_HOST_CHUNKS=$c timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 \
      > gpurun_out/hc_${cfg}_$c.json 2> gpurun_out/hc_${cfg}_$c.err
  done
done
