#!/bin/bash
mkdir -p gpurun_out
timeout 3300 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/g4_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/g4_pytest.log
echo done
