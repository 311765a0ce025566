timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 300 -p no:cacheprovider -k "halo or conv" > gpurun_out/g17_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/g17_tests.log
for f in 0 3 5 6; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn 64 layer1.0.conv2 layer2.1.conv2 layer3.1.conv2; done
for f in 0 3 5; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn 128 layer2.1.conv2 layer3.1.conv2; done
