D=gpurun_out/atab
mkdir -p $D
for i in 1 2; do
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/auto$i.json 2>&1
timeout 600 python tools/lc_chain.py --batch 32 --reps 20 > $D/default$i.json 2>&1
done
