#!/bin/bash
# Everything the round's evidence needs, in one GPU call (outputs in gpurun_out/ev_*).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/ev_smi.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/ev_smi.txt
git log -1 --format=%H > gpurun_out/ev_commit.txt 2>/dev/null
timeout 900 python bench.py > gpurun_out/ev_bench_default.json 2> gpurun_out/ev_bench_default.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/ev_bench_reference.json 2> gpurun_out/ev_bench_reference.err
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/ev_pytest_gpu.log 2>&1
# launch list of the default bench command (device times per launch; shares, not absolutes)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_default.csv python bench.py --steps 5 --warmup 3 --no-cpu --ncu off --legs none --tca 0 --graphconv 0 --no-e2e --no-cusparse > /dev/null 2>&1
mkdir -p /tmp/ncu
for c in c3 c2 c3h c4 c5; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -f -o /tmp/ncu/ev_prof_$c python bench.py --config $c --steps 3 --warmup 3 --minimal > gpurun_out/ev_ncu_$c.log 2>&1
  python tools/ncu_summary.py /tmp/ncu/ev_prof_$c.ncu-rep > gpurun_out/ev_ncu_$c.txt 2>&1
  ncu -i /tmp/ncu/ev_prof_$c.ncu-rep --page raw --csv > gpurun_out/ev_raw_$c.csv 2>/dev/null
  timeout 300 python tools/trace_cta.py $c > gpurun_out/ev_trace_$c.txt 2>&1
  timeout 300 python tools/trace_cta.py $c --persistent 1 > gpurun_out/ev_trace_pers_$c.txt 2>&1
done
ncu -i /tmp/ncu/ev_prof_c3.ncu-rep --page source --csv > gpurun_out/ev_source_c3.csv 2>/dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ev_smoke.txt 2>&1
du -sh gpurun_out
find gpurun_out -size +16M -print -delete
