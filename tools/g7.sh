#!/bin/bash
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/g7_pytest.log 2>&1
timeout 300 python tools/trace_cta.py c2 > gpurun_out/g7_trace_c2.txt 2>&1
timeout 300 python tools/trace_cta.py c2 --persistent 1 > gpurun_out/g7_trace_pers_c2.txt 2>&1
timeout 900 python bench.py > gpurun_out/g7_bench.json 2> gpurun_out/g7_bench.err
