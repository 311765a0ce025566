mkdir -p gpurun_out/epi
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/epi/tests.txt
for b in 2 4; do
  TACKER_EPI_BUFS=$b timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/epi/b$b.json 2>&1
done
TACKER_LC_DBG=16 timeout 300 python tools/lc_gaps.py --batch 32 > gpurun_out/epi/gaps.json 2>&1
