#!/bin/bash
# ncu --set full of the dominant kernel for each config in CFGS (default: every bench workload),
# summaries into gpurun_out/fe_ncu_<cfg>.txt (tools/ncu_summary.py) and raw CSVs.
mkdir -p gpurun_out /tmp/ncu
for cn in ${CFGS:-c3 c2 c3h c4 c5}; do
  c=${cn%%:*}; n=0; [ "$c" != "$cn" ] && n=${cn##*:}; tag=${cn/:/_}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -f -o /tmp/ncu/p_$tag \
    python bench.py --config $c --n $n --steps 3 --warmup 3 --minimal > gpurun_out/fe_ncu_$tag.log 2>&1
  python tools/ncu_summary.py /tmp/ncu/p_$tag.ncu-rep > gpurun_out/fe_ncu_$tag.txt 2>&1
  ncu -i /tmp/ncu/p_$tag.ncu-rep --page raw --csv > gpurun_out/fe_raw_$tag.csv 2>/dev/null
done
