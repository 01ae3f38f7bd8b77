mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/g1_smi.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/g1_smi.txt
for c in c2 c3 c3h c4 c5; do
  timeout 300 python bench.py --config $c --steps 30 --warmup 5 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/g1_bench_$c.json 2> gpurun_out/g1_bench_$c.err
done
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/g1_pytest.log 2>&1
echo done
