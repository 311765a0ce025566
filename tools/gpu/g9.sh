export TACKER_LC_DBG=8
python tools/lc_timeline.py --bn 64 layer1.0.conv2
python tools/lc_timeline.py --bn 256 layer1.0.conv3
export TACKER_LC_DBG=14
python tools/lc_timeline.py --bn 64 layer1.0.conv2
python tools/lc_timeline.py --bn 256 layer1.0.conv3
export TACKER_LC_DBG=13
python tools/lc_timeline.py --bn 64 layer1.0.conv2
