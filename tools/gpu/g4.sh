timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -x -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g4_tests.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/g4_tests.log
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g4_chain_tma.json 2>&1
TACKER_EPI_TMA=0 python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g4_chain_notma.json 2>&1
python - <<'PY'
import json
a=json.load(open('gpurun_out/g4_chain_tma.json')); b=json.load(open('gpurun_out/g4_chain_notma.json'))
print('tma', a['overlap'], 'no', b['overlap'])
for x,y in zip(a['per_kernel'], b['per_kernel']): print('%-22s %7.1f %7.1f roof %6.1f bn %s'%(x['name'], x['us'], y['us'], x['roof_us'], x.get('bn')))
PY
