# LC b32 query decomposition: per-kernel back-to-back times with parts of the pipeline disabled
# (TACKER_LC_DBG bits: 1 = epilogue drains without math/stores, 2 = no MMAs, 4 = no TMA loads)
mkdir -p gpurun_out/lcd
for d in 0 7 3 4 1; do
  TACKER_LC_DBG=$d timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/lcd/dbg$d.json 2> gpurun_out/lcd/dbg$d.err
done
