for f in 0 1 3 5 6; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn 64 layer1.0.conv2 layer2.1.conv2 layer3.1.conv2; done
for f in 0 1 3 5 6; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn 128 layer1.0.conv2 layer2.1.conv2 layer3.1.conv2; done
TACKER_LC_DBG=8 python tools/lc_timeline.py --bn 64 --ctas 0,100 layer1.0.conv2
TACKER_LC_DBG=13 python tools/lc_timeline.py --bn 64 --ctas 0 layer1.0.conv2
TACKER_LC_DBG=11 python tools/lc_timeline.py --bn 64 --ctas 0 layer1.0.conv2
