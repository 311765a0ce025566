timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -x -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g7_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/g7_tests.log
for bn in 64 128 256; do
for f in 0 1 6; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn $bn layer1.0.conv1 layer1.0.conv2 layer1.0.conv3 layer2.1.conv2 layer3.1.conv2 layer3.1.conv1 layer4.1.conv2; done
done
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g7_chain.json 2>&1
python -c "
import json; a=json.load(open('gpurun_out/g7_chain.json')); print(a['overlap'], sum(k['us'] for k in a['per_kernel']), sum(k['roof_us'] for k in a['per_kernel']))"
