set -x
ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "target/" -k regex:fused_kernel -c 2 -o gpurun_out/lc_l1c2 python tools/lc_one.py --reps 1 layer1.0.conv2 layer1.0.conv3 > gpurun_out/g3_ncu.log 2>&1
tail -3 gpurun_out/g3_ncu.log
