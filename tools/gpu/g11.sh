timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -x -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g11_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/g11_tests.log
for f in 0 3 5; do TACKER_LC_DBG=$f python tools/lc_breakdown.py layer1.0.conv1 layer1.0.conv2 layer1.0.conv3 layer2.1.conv2 layer3.1.conv2 layer4.1.conv2; done
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g11_chain.json 2>&1
python -c "
import json; a=json.load(open('gpurun_out/g11_chain.json')); print(a['overlap'], sum(k['us'] for k in a['per_kernel']), sum(k['roof_us'] for k in a['per_kernel']))
for k in a['per_kernel']: print('%-22s %7.1f roof %6.1f bn %s'%(k['name'], k['us'], k['roof_us'], k.get('bn')))" | head -20
