mkdir -p gpurun_out/rf
python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/rf/tests.txt
for r in 0 8; do TACKER_RASTER=$r timeout 300 python tools/table1.py > gpurun_out/rf/table1_r$r.json 2>&1; done
for st in 4 2; do TACKER_FUSED_STAGES=$st timeout 600 python tools/fuse_sweep.py --convs 5,40 --ws 16,24 --be stencil,mriq,lbm,fft > gpurun_out/rf/fst$st.jsonl 2>&1; done
