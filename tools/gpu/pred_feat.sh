D=gpurun_out/predfeat
mkdir -p $D
timeout 1500 python tools/predictor_sweep.py --features blocks --out $D/sweep_blocks.json > $D/blocks_summary.json 2> $D/err.txt
