D=gpurun_out/fmode
mkdir -p $D
python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py tests/test_gpu_bench_configs.py tests/test_gpu_manager.py -m gpu -x -q 2>&1 | tail -2 > $D/tests.txt
for m in 1 0; do
  TACKER_LC_MODE_KERNELS=$m timeout 600 python tools/fig20.py > $D/fig20_m$m.jsonl 2> /dev/null
  TACKER_LC_MODE_KERNELS=$m timeout 600 python tools/fuse_sweep.py --batch 32 --convs 1,2,3,10,11 --ws 24 --be mriq,stencil,lbm,cp > $D/sweep_m$m.jsonl 2>&1
done
