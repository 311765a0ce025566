D=gpurun_out/chain7
mkdir -p $D
for i in 1 2; do
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/head$i.json 2>&1
TACKER_KPS64=2 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/kps64_2_$i.json 2>&1
(cd ab_prev && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/prev$i.json 2>&1)
done
