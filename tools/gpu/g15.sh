timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -x -q -m gpu --timeout 300 -p no:cacheprovider > gpurun_out/g15_tests.log 2>&1; echo "tests rc=$?"; tail -15 gpurun_out/g15_tests.log
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g15_chain.json 2>&1
python -c "
import json; a=json.load(open('gpurun_out/g15_chain.json')); print(a['overlap'], sum(k['us'] for k in a['per_kernel']), sum(k['roof_us'] for k in a['per_kernel']))
for k in a['per_kernel']:
  if 'conv2' in k['name']: print('%-22s %7.1f roof %6.1f bn %s tiles %s'%(k['name'], k['us'], k['roof_us'], k.get('bn'), k.get('tiles')))"
