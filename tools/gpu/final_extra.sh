D=gpurun_out/extra
mkdir -p $D
timeout 1500 python tools/predictor_sweep.py --out $D/predictor_sweep_final.json > $D/pred_summary.json 2> $D/pred_err.txt
timeout 900 python tools/fig20.py > $D/fig20.jsonl 2> $D/fig20.err
timeout 600 python tools/be_table.py > $D/be_table.json 2>&1
