# same-box A/B: this tree vs the round-2 head at session start (ab_old/, commit 60cf5af)
D=gpurun_out/ab
mkdir -p $D
A="--steps 30 --warmup 5 --seeds 1 --no-extra --no-cpu"
timeout 900 python bench.py $A > $D/new1.json 2> $D/new1.err
(cd ab_old && timeout 900 python bench.py $A > ../$D/old.json 2> ../$D/old.err)
timeout 900 python bench.py $A > $D/new2.json 2> $D/new2.err
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > $D/lc_new.json 2>&1
(cd ab_old && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 20 > ../$D/lc_old.json 2>&1)
