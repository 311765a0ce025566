mkdir -p gpurun_out/fst
for st in 4 2; do TACKER_FUSED_STAGES=$st timeout 600 python tools/fuse_sweep.py --convs 5,20,40 --ws 16,24 --be stencil,mriq,lbm,fft > gpurun_out/fst/s$st.jsonl 2>&1; done
