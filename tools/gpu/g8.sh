TACKER_LC_DBG=6 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "target/" -k regex:fused_kernel -c 1 -o gpurun_out/l1c3_epi python tools/lc_one.py --bn 256 --reps 1 layer1.0.conv3 > gpurun_out/g8_ncu.log 2>&1
tail -2 gpurun_out/g8_ncu.log
