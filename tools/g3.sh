#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_paths.py tests/test_gpu_spmm.py -m gpu -x -q -p no:cacheprovider -k "not full_size" > gpurun_out/g3_pytest.log 2>&1
timeout 600 python bench.py --legs c2 --no-cpu --no-cusparse --no-e2e --tca 0 --graphconv 0 > gpurun_out/g3_bench.json 2> gpurun_out/g3_bench.err
echo done
