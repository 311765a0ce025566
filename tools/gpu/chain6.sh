D=gpurun_out/chain6
mkdir -p $D
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_manager.py -m gpu -x -q 2>&1 | tail -2 > $D/tests.txt
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/head.json 2>&1
TACKER_KPS=1 TACKER_KPS64=1 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/kps1.json 2>&1
TACKER_KPS64=2 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/kps64_2.json 2>&1
(cd ab_old && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/old.json 2>&1)
timeout 600 python tools/lc_chain.py --batch 1 --autotune --reps 20 > $D/b1.json 2>&1
