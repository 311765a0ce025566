for bn in 64 128 256; do
for f in 0 1 2 4 3 5 6; do TACKER_LC_DBG=$f python tools/lc_breakdown.py --bn $bn layer1.0.conv1 layer1.0.conv2 layer1.0.conv3 layer2.1.conv2 layer3.1.conv2 layer3.1.conv1 layer4.1.conv2; done
done
