mkdir -p gpurun_out/ncumode
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_kernel --launch-skip 2 -c 1 -f -o gpurun_out/ncumode/l1c3_mode python tools/lc_one.py --bn 128 --reps 3 layer1.0.conv3 > gpurun_out/ncumode/l1c3.log 2>&1
TACKER_LC_MODE_KERNELS=0 timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_kernel --launch-skip 2 -c 1 -f -o gpurun_out/ncumode/l1c3_any python tools/lc_one.py --bn 128 --reps 3 layer1.0.conv3 > gpurun_out/ncumode/l1c3_any.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_kernel --launch-skip 2 -c 1 -f -o gpurun_out/ncumode/l2c2_mode python tools/lc_one.py --bn 128 --reps 3 layer2.1.conv2 > gpurun_out/ncumode/l2c2.log 2>&1
