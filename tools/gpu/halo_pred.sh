mkdir -p gpurun_out/halo gpurun_out/pred
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/halo/tests.txt
for h in 0 1; do TACKER_HALO_BRES=$h timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/halo/h$h.json 2>&1; done
timeout 1500 python tools/predictor_sweep.py --out gpurun_out/pred/predictor_sweep_r02b.json > gpurun_out/pred/summary.json 2> gpurun_out/pred/err.txt
