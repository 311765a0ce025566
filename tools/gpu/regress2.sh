D=gpurun_out/reg2
mkdir -p $D
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -2 > $D/tests.txt
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > $D/base.json 2>&1
(cd ab_old && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > ../$D/old.json 2>&1)
