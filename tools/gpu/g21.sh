timeout 900 python -m pytest tests/test_gpu_manager.py -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g21_mgr.log 2>&1; echo "mgr rc=$?"; tail -2 gpurun_out/g21_mgr.log
timeout 1800 python tools/predictor_sweep.py --out gpurun_out/predictor_sweep_r02.json > gpurun_out/g21_sweep.log 2>&1; echo "sweep rc=$?"; tail -1 gpurun_out/g21_sweep.log
