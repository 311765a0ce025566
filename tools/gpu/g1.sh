set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_manager.py -x -q -m gpu > gpurun_out/g1_new.log 2>&1; echo "new rc=$?"
tail -5 gpurun_out/g1_new.log
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/g1_all.log 2>&1; echo "all rc=$?"
tail -5 gpurun_out/g1_all.log
timeout 1500 python bench.py --steps 20 --warmup 5 --seeds 1 > gpurun_out/g1_bench.json 2> gpurun_out/g1_bench.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/g1_bench.json; tail -20 gpurun_out/g1_bench.err
