timeout 900 python tools/qos_tail.py --queries 10000 --policy baymax 2>&1 | tail -5
timeout 1200 python bench.py --steps 100 --warmup 5 --seeds 1 --no-extra --no-cpu > gpurun_out/g14_k100.json 2> gpurun_out/g14_k100.err; echo "k100 rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 --seeds 1 --no-extra --no-cpu > gpurun_out/g14_k20.json 2> gpurun_out/g14_k20.err; echo "k20 rc=$?"
python - <<'PY'
import json
for f in ('gpurun_out/g14_k20.json','gpurun_out/g14_k100.json'):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, 'ERR', e); continue
    print(f, round(d['value'],1), round(d['be_norm_thpt'],4), 'p99', round(d['lc_p99_ms'],2), d['violations'], d['queries_in_window'], 'peak', d['lambda_peak_load'], d['improvement_vs_baymax_same_rule_eq10_normalised'], d['tacker_paper_vs_baymax_eq10_normalised'])
    for a,v in d['arms'].items(): print('   ', a, {k:v.get(k) for k in ('be_kernels_per_s','be_norm_thpt','lc_p50_ms','lc_p99_ms','violations','fused','reordered')})
PY
