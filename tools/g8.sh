#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_spmm.py tests/test_gpu_format.py tests/test_gpu_paths.py -m gpu -q -p no:cacheprovider -x -k "not full_size" > gpurun_out/g8_pytest.log 2>&1
timeout 900 python bench.py --no-cpu > gpurun_out/g8_bench.json 2> gpurun_out/g8_bench.err
