#!/bin/bash
# dtc_spmm_host default chunk rule: host-API parity tests + e2e on every config (gpurun_out/hk_*)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spmm.py -k "host_api" -q -p no:cacheprovider > gpurun_out/hk_pytest.log 2>&1
for c in c2 c3 c3h c4 c5; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/hk_$c.json 2> gpurun_out/hk_$c.err
done
