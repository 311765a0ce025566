timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 300 -p no:cacheprovider > gpurun_out/g26_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/g26_tests.log
python tools/fig20.py 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print(d['pair'], d['warp_split'], round(d['T_TC_ms'],4), round(d['T_CD_ms'],4), 'fused', round(d['fused_ms'],4), 'seq', round(d['sequential_ms'],4), {k: round(v,3) for k,v in d['overlap_eq11'].items() if v is not None})
"
