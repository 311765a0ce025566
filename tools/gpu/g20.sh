timeout 1500 python -m pytest tests -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g20_all.log 2>&1; echo "all rc=$?"; tail -4 gpurun_out/g20_all.log
timeout 1800 python tools/predictor_sweep.py --out gpurun_out/predictor_sweep_r02.json > gpurun_out/g20_sweep.log 2>&1; echo "sweep rc=$?"; tail -2 gpurun_out/g20_sweep.log
timeout 900 python bench.py --steps 5 --warmup 3 --seeds 1 --no-extra --no-cpu > gpurun_out/g20_bench.json 2> gpurun_out/g20_bench.err; echo "bench rc=$?"; tail -c 400 gpurun_out/g20_bench.json; tail -3 gpurun_out/g20_bench.err
