D=gpurun_out/burst
mkdir -p $D
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "conv or gemm" 2>&1 | tail -2 > $D/tests.txt
for b in 0 1 2 0 1 2; do TACKER_FIRST_BURST=$b timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/b$b.json.$RANDOM 2>&1; done
TACKER_FIRST_BURST=1 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "conv or gemm" 2>&1 | tail -2 >> $D/tests.txt
