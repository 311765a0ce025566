mkdir -p gpurun_out/pred
timeout 1500 python tools/predictor_sweep.py --out gpurun_out/pred/predictor_sweep_r02b.json > gpurun_out/pred/summary.json 2> gpurun_out/pred/err.txt
