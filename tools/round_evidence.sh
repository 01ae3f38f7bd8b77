#!/bin/bash
# Everything the round's evidence needs, in one GPU call (outputs in gpurun_out/ev_*).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/ev_smi.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/ev_smi.txt
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/ev_pytest_gpu.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_smoke.py > gpurun_out/ev_sanitize_$tool.log 2>&1; echo "rc=$?" >> gpurun_out/ev_sanitize_$tool.log
done
timeout 900 python bench.py > gpurun_out/ev_bench_default.json 2> gpurun_out/ev_bench_default.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ev_bench_reference.json 2> gpurun_out/ev_bench_reference.err
for c in c3 c3h c4 c5; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 5 --no-cpu > gpurun_out/ev_bench_$c.json 2> gpurun_out/ev_bench_$c.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_c2.csv python bench.py --steps 5 --warmup 3 --no-cpu > /dev/null 2>&1
# full ncu captures stay on the box (/tmp, tens of MB each); only text/CSV summaries come back
mkdir -p /tmp/ncu
for c in c2 c3 c3h c4 c5; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1 -f -o /tmp/ncu/ev_prof_$c python bench.py --config $c --steps 3 --warmup 3 --minimal > gpurun_out/ev_ncu_$c.log 2>&1
  python tools/ncu_summary.py /tmp/ncu/ev_prof_$c.ncu-rep > gpurun_out/ev_ncu_$c.txt 2>&1
  ncu -i /tmp/ncu/ev_prof_$c.ncu-rep --page raw --csv > gpurun_out/ev_raw_$c.csv 2>/dev/null
  timeout 300 python tools/trace_cta.py $c > gpurun_out/ev_trace_$c.txt 2>&1
done
ncu -i /tmp/ncu/ev_prof_c2.ncu-rep --page source --csv > gpurun_out/ev_source_c2.csv 2>/dev/null
du -sh gpurun_out
find gpurun_out -size +16M -print -delete
