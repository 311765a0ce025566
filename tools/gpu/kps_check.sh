mkdir -p gpurun_out/kps
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/kps/tests.txt
TACKER_KPS_MAXBN=128 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 >> gpurun_out/kps/tests.txt
for cfg in "1 64" "2 64" "2 128"; do set -- $cfg
  TACKER_KPS=$1 TACKER_KPS_MAXBN=$2 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/kps/k$1_$2.json 2>&1
done
