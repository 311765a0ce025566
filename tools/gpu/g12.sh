timeout 1500 python -m pytest tests -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/g12_all.log 2>&1; echo "all rc=$?"; tail -4 gpurun_out/g12_all.log
timeout 900 python bench.py --steps 20 --warmup 5 --seeds 1 --no-extra --no-cpu > gpurun_out/g12_k20.json 2> gpurun_out/g12_k20.err; echo "k20 rc=$?"
timeout 1200 python bench.py --steps 100 --warmup 5 --seeds 1 --no-extra --no-cpu > gpurun_out/g12_k100.json 2> gpurun_out/g12_k100.err; echo "k100 rc=$?"
python - <<'PY'
import json
for f in ('gpurun_out/g12_k20.json','gpurun_out/g12_k100.json'):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, 'ERR', e); continue
    print(f, round(d['value'],1), round(d['be_norm_thpt'],4), round(d['lc_p99_ms'],2), d['queries_in_window'], d['service_ms'], d['improvement_vs_baymax_same_rule_eq10_normalised'], d['tacker_paper_vs_baymax_eq10_normalised'], d['roofline']['frac'])
PY
