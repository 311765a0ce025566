mkdir -p gpurun_out/r01c
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r01c/gpu_tests.log 2>&1; echo "pytest_rc=$?" >> gpurun_out/r01c/gpu_tests.log
timeout 900 python bench.py > gpurun_out/r01c/bench.json 2> gpurun_out/r01c/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv --log-file gpurun_out/r01c/launches_timed.csv python bench.py --steps 40 --warmup 3 --no-extra --no-cpu > gpurun_out/r01c/bench_under_ncu.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fused_kernel -c 12 -o gpurun_out/r01c/targets python tools/ncu_targets.py --next3 > gpurun_out/r01c/ncu_targets.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01c/smoke.log 2>&1
tail -2 gpurun_out/r01c/gpu_tests.log; tail -1 gpurun_out/r01c/smoke.log; tail -2 gpurun_out/r01c/ncu_targets.log; ls -la gpurun_out/r01c
timeout 600 ncu --metrics "pmsampling:TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed,pmsampling:TPC.TriageCompute.sm__pipe_fma_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed,pmsampling:SM_A.TriageCompute.sm__inst_executed_pipe_xu_realtime.avg.pct_of_peak_sustained_elapsed" --clock-control none -k regex:"fused_kernel|be_original" -c 4 -o gpurun_out/r01c/pm python tools/pm_targets.py > gpurun_out/r01c/pm.log 2>&1
