#!/bin/bash
# DTC_PAD_FIRST=0/1 (first-batch side records): parity tests + kernel GFLOP/s per config (gpurun_out/fs_*)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_paths.py tests/test_gpu_spmm.py -q -p no:cacheprovider -x > gpurun_out/fs_pytest.log 2>&1
for rep in 1 2; do
  for f in 0 1; do
    DTC_PAD_FIRST=$f timeout 600 python bench.py --config c2 --steps 200 --warmup 10 --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 > gpurun_out/fs_c2_${f}_$rep.json 2>/dev/null
  done
done
for c in c3 c4 c5; do
  for f in 0 1; do
    DTC_PAD_FIRST=$f timeout 600 python bench.py --config $c --steps 30 --warmup 5 --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 > gpurun_out/fs_${c}_${f}_1.json 2>/dev/null
  done
done
DTC_PAD_FIRST=1 timeout 300 python tools/trace_cta.py c2 > gpurun_out/fs_trace_c2.txt 2>&1
