#!/bin/bash
# Compare library build variants (DTC_LIBRARY=<so>) on the default path, per config.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3 c4 c5}; do
  for so in ${SOS:-paper_conf_asplos_fan0024_b200/libdtc.so}; do
    tag=$(basename $so .so)
    DTC_LIBRARY=$PWD/$so timeout 300 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cusparse --no-cpu --no-e2e --graphconv 0 --tca 0 > gpurun_out/so_${tag}_$c.json 2> gpurun_out/so_${tag}_$c.err
  done
done
