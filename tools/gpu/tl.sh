mkdir -p gpurun_out/tl
TACKER_LC_DBG=8 timeout 300 python tools/lc_timeline.py --bn 128 layer1.0.conv3 > gpurun_out/tl/l1c3.txt 2>&1
TACKER_LC_DBG=8 timeout 300 python tools/lc_timeline.py --bn 128 layer3.1.conv1 > gpurun_out/tl/l3c1.txt 2>&1
TACKER_LC_DBG=8 timeout 300 python tools/lc_timeline.py --bn 128 layer2.1.conv2 > gpurun_out/tl/l2c2.txt 2>&1
