timeout 900 python -m pytest tests/test_gpu_bench_configs.py -x -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g24_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/g24_tests.log
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g24_chain32.json 2>&1
python tools/lc_chain.py --batch 1 --autotune > gpurun_out/g24_chain1.json 2>&1
python - <<'PY'
import json
for f in ('gpurun_out/g24_chain32.json','gpurun_out/g24_chain1.json'):
    a=json.load(open(f)); print(f, a['overlap'], round(sum(k['us'] for k in a['per_kernel']),1), round(sum(k['roof_us'] for k in a['per_kernel']),1))
    for k in a['per_kernel'][:3]: print('  ', k['name'], round(k['us'],1), round(k['roof_us'],1), k.get('bn'))
PY
