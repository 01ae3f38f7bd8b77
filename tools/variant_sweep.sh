#!/bin/bash
# sweep build variants (${VDIR:-vsos}/*.so) over configs -> gpurun_out/vs_<variant>_<cfg>.json
# each variant first runs a parity subset (gpurun_out/vs_<variant>_parity.txt)
mkdir -p gpurun_out
for so in ${VDIR:-vsos}/*.so; do
  v=$(basename $so .so)
  DTC_LIBRARY=$PWD/$so timeout 300 python -m pytest tests/test_gpu_spmm.py -q -x -p no:cacheprovider -k "p2_integer or split or random_tolerance or p6" 2>&1 | tail -1 > gpurun_out/vs_${v}_parity.txt
  for c in ${CONFIGS:-c2 c3 c3h c5}; do
    DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cusparse --no-cpu --no-e2e > gpurun_out/vs_${v}_$c.json 2> gpurun_out/vs_${v}_$c.err
  done
done
