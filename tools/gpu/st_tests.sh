mkdir -p gpurun_out/stt
python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py tests/test_gpu_bench_configs.py -m gpu -q -k "stencil or STENCIL or fused" 2>&1 | tail -3 > gpurun_out/stt/tests.txt
timeout 300 python tools/be_table.py stencil > gpurun_out/stt/be.json 2>&1
timeout 600 python tools/fuse_sweep.py --convs 5,20,40 --ws 16,20,24 --be stencil > gpurun_out/stt/sweep.jsonl 2>&1
