#!/bin/bash
# TMA element size (8 vs 4 bytes) x launch mode x unit size on the padded-row path.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3h c4}; do
  for te in 8 4; do
    for pu in "0 0" "0 32" "1 32" "1 0"; do
      set -- $pu
      DTC_PAD_TE=$te DTC_PAD_PERS=$1 timeout 300 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cusparse --no-cpu --no-e2e --graphconv 0 --unit-blocks $2 > gpurun_out/te${te}_p$1_u$2_$c.json 2> gpurun_out/te${te}_p$1_u$2_$c.err
    done
  done
done
