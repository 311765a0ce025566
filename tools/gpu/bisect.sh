D=gpurun_out/bisect
mkdir -p $D
for v in old 4110086 1eede18 ca73d22; do (cd ab_$v && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/$v.json 2>&1); done
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/head.json 2>&1
(cd ab_old && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/old2.json 2>&1)
