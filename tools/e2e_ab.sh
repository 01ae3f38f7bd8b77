mkdir -p gpurun_out; : > gpurun_out/e2e_ab.txt
for r in 1 2; do for v in default base; do
  if [ $v = default ]; then L=""; else L="DTC_LIBRARY=$PWD/vbuild/base/libdtc.so"; fi
  env $L timeout 400 python bench.py --legs none --no-cpu --no-cusparse --ncu off --tca 0 --graphconv 0 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); e=d['e2e']; s=d['e2e_sync']
print('$v', d['value'], 'e2e', e['value'], e['ms_per_step'], 'sync', s['value'], s['ms_per_step'])" >> gpurun_out/e2e_ab.txt
done; done
timeout 900 python -m pytest tests/test_gpu_spmm.py -m gpu -q -k "split_windows or misaligned_c" >> gpurun_out/e2e_ab.txt 2>&1
cat gpurun_out/e2e_ab.txt
