#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_gcn.py tests/test_gpu_format.py -m gpu -x -q -p no:cacheprovider > gpurun_out/g5_pytest.log 2>&1
echo done
