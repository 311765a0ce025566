# LC b32 query decomposition: per-kernel back-to-back times with parts of the pipeline disabled
# (TACKER_LC_DBG bits: 1 = epilogue drains without math/stores, 2 = no MMAs, 4 = no TMA loads).
# The switches exist only in a -DTK_LC_DIAG=1 build (production kernels carry no diagnostics).
mkdir -p gpurun_out/lcd variants
python -m paper_conf_hpca_zhaocczlllg22_b200.build --out $PWD/variants/lib_diag.so -DTK_LC_DIAG=1 > /dev/null
for d in 0 7 3 4 1; do
  TACKER_LIB=$PWD/variants/lib_diag.so TACKER_LC_DBG=$d timeout 600 python tools/lc_chain.py --batch 32 --autotune --reps 10 > gpurun_out/lcd/dbg$d.json 2> gpurun_out/lcd/dbg$d.err
done
