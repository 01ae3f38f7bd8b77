#!/bin/bash
# Post-change validation: GPU suite, smoke, default bench line, e2e on c3/c5 (gpurun_out/fc_*)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/fc_pytest_gpu.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/fc_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/fc_bench_default.json 2> gpurun_out/fc_bench_default.err
for c in c3 c3h c4 c5; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 5 --no-cpu --no-cusparse --tca 0 --graphconv 0 > gpurun_out/fc_bench_$c.json 2> gpurun_out/fc_bench_$c.err
done
