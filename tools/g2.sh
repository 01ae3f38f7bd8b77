#!/bin/bash
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/g2_bench.json 2> gpurun_out/g2_bench.err
timeout 3000 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/g2_pytest.log 2>&1
echo done
