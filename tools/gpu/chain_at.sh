D=gpurun_out/chainat
mkdir -p $D
for i in 1 2; do
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/auto$i.json 2>&1
timeout 600 python tools/lc_chain.py --batch 32 --autotune --chain-autotune --reps 20 > $D/chain$i.json 2>&1
done
timeout 600 python tools/lc_chain.py --batch 1 --autotune --reps 20 > $D/b1_auto.json 2>&1
timeout 600 python tools/lc_chain.py --batch 1 --autotune --chain-autotune --reps 20 > $D/b1_chain.json 2>&1
