tail -1 gpurun_out/$1 | timeout 20 python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['rows']
import statistics as s
for k in ('stencil','mriq'):
  rr=[x for x in r if x['be'].startswith(k)]
  print(k, 'be_orig', round(s.mean(x['t_be'] for x in rr)*1e3,1), 'fused', round(s.mean(x['t_fused'] for x in rr)*1e3,1), 'seq', round(s.mean(x['seq'] for x in rr)*1e3,1))
"
