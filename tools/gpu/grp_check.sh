mkdir -p gpurun_out/grp
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_large.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/grp/tests.txt
for g in 1 2; do
  TACKER_EPI_GROUPS=$g timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/grp/g$g.json 2>&1
done
TACKER_EPI_GROUPS=2 timeout 600 python tools/lc_chain.py --batch 1 --autotune --reps 10 > gpurun_out/grp/b1_g2.json 2>&1
TACKER_EPI_GROUPS=1 timeout 600 python tools/lc_chain.py --batch 1 --autotune --reps 10 > gpurun_out/grp/b1_g1.json 2>&1
