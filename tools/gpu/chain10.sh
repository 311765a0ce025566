D=gpurun_out/chain11
mkdir -p $D
python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_large.py -m gpu -x -q 2>&1 | tail -2 > $D/tests.txt
for i in 1 2; do
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/head$i.json 2>&1
(cd ab_prev && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/prev$i.json 2>&1)
done
timeout 600 python tools/fuse_sweep.py --batch 32 --convs 1,2,3,10,11 --ws 24 --be mriq,stencil,lbm,cp > $D/sweep_head.jsonl 2>&1
(cd ab_prev && timeout 600 python tools/fuse_sweep.py --batch 32 --convs 1,2,3,10,11 --ws 24 --be mriq,stencil,lbm,cp > ../$D/sweep_prev.jsonl 2>&1)
