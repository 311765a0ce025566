mkdir -p gpurun_out/v2
python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -m gpu -x -q 2>&1 | tail -5 > gpurun_out/v2/tests.txt
for r in 1 0; do TACKER_RICH=$r timeout 600 python tools/fuse_sweep.py --convs 5,20,40 --ws 4,8,16,24 --be fft,stencil,lbm,mriq,mrifhd,cp > gpurun_out/v2/sweep_rich$r.jsonl 2>&1; done
