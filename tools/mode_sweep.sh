#!/bin/bash
# Launch mode (one CTA per unit vs persistent) x F4 unit size on the padded-row path, per config.
mkdir -p gpurun_out
for c in ${CONFIGS:-c2 c3 c3h c4 c5}; do
  for pu in ${MODES:-"0,0" "0,32" "1,0" "1,32"}; do
    p=${pu%,*}; u=${pu#*,}
    DTC_PAD_PERS=$p timeout 300 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cusparse --no-cpu --no-e2e --graphconv 0 --unit-blocks $u > gpurun_out/m_p${p}_u${u}_$c.json 2> gpurun_out/m_p${p}_u${u}_$c.err
  done
done
