mkdir -p gpurun_out/bias
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/bias/tests.txt
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/bias/res1.json 2>&1
TACKER_BIAS_RES=0 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/bias/res0.json 2>&1
TACKER_LC_DBG=7 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/bias/dbg7.json 2>&1
