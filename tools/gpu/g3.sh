set -x
ncu --set full --clock-control none --import-source on -k regex:fused_kernel -c 2 -o gpurun_out/lc_l1c2 python tools/lc_one.py --reps 1 layer1.0.conv2 layer1.0.conv3 > gpurun_out/g3_ncu.log 2>&1
ls -la gpurun_out/
python tools/lc_chain.py --batch 32 --autotune > gpurun_out/g3_chain_b32.json 2>gpurun_out/g3_chain.err
tail -c 300 gpurun_out/g3_chain_b32.json
