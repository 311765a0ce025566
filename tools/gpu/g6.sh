ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "target/" -k regex:fused_kernel -c 1 -o gpurun_out/l1c3_bn256 python tools/lc_one.py --bn 256 --reps 1 layer1.0.conv3 > gpurun_out/g6_ncu.log 2>&1
tail -2 gpurun_out/g6_ncu.log
