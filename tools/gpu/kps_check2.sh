mkdir -p gpurun_out/kps2
for cfg in "1 64 0" "2 128 0" "2 256 0" "2 128 4" "2 128 3"; do set -- $cfg
  TACKER_KPS=$1 TACKER_KPS_MAXBN=$2 TACKER_KPS64=$3 timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/kps2/k$1_$2_$3.json 2>&1
done
