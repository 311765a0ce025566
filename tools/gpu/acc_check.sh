mkdir -p gpurun_out/acc
TACKER_ACC=4 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/acc/tests.txt
for a in 2 4; do TACKER_ACC=$a timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/acc/a$a.json 2>&1; done
TACKER_ACC=4 TACKER_LC_DBG=7 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/acc/a4_dbg7.json 2>&1
