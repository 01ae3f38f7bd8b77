mkdir -p gpurun_out /tmp/ncu
timeout 900 python bench.py > gpurun_out/fe_bench.json 2> gpurun_out/fe_bench.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/fe_bench_reference.json 2> gpurun_out/fe_bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fe_launches_default.csv python bench.py --steps 5 --warmup 3 --no-cpu --ncu off --legs none --tca 0 --graphconv 0 --no-e2e --no-cusparse > /dev/null 2>&1
for c in c3 c5; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -f -o /tmp/ncu/fe_prof_$c python bench.py --config $c --steps 3 --warmup 3 --minimal > gpurun_out/fe_ncu_$c.log 2>&1
  python tools/ncu_summary.py /tmp/ncu/fe_prof_$c.ncu-rep > gpurun_out/fe_ncu_$c.txt 2>&1
  ncu -i /tmp/ncu/fe_prof_$c.ncu-rep --page raw --csv > gpurun_out/fe_raw_$c.csv 2>/dev/null
  timeout 300 python tools/trace_cta.py $c > gpurun_out/fe_trace_$c.txt 2>&1
done
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fe_smoke.txt 2>&1
