D=gpurun_out/reg
mkdir -p $D
timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > $D/base.json 2>&1
TACKER_LIB=$PWD/variants/lib_solo6.so timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > $D/solo6.json 2>&1
TACKER_BIAS_RES=0 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > $D/nobias.json 2>&1
TACKER_HALO_BRES=0 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > $D/nohbres.json 2>&1
(cd ab_old && timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > ../$D/old.json 2>&1)
