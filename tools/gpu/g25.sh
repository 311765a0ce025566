mkdir -p gpurun_out/r02
timeout 1500 python -m pytest tests -q -m gpu --timeout 600 -p no:cacheprovider > gpurun_out/r02/gpu_tests.log 2>&1; echo "gpu tests rc=$?"; tail -2 gpurun_out/r02/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02/smoke.log
S=$(date +%s); timeout 2400 python bench.py > gpurun_out/r02/bench_default.json 2> gpurun_out/r02/bench_default.err; echo "bench default rc=$? wall $(( $(date +%s) - S )) s"
S=$(date +%s); timeout 2400 python bench.py --steps 20 --warmup 5 > gpurun_out/r02/bench_k20.json 2> gpurun_out/r02/bench_k20.err; echo "bench k20 rc=$? wall $(( $(date +%s) - S )) s"
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02/bench_reference.json 2>&1; echo "ref rc=$?"
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" -c 3000 --csv --log-file gpurun_out/r02/launches_timed.csv python bench.py --steps 2 --warmup 3 --seeds 1 --no-extra --no-cpu > gpurun_out/r02/ncu_bench.log 2>&1; echo "ncu launches rc=$?"
