D=gpurun_out/head_final4
mkdir -p $D
timeout 1500 python -m pytest tests -m gpu -q > $D/gpu_tests.log 2>&1; echo "pytest_rc=$?" >> $D/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1
timeout 1500 python bench.py > $D/bench_default.json 2> $D/bench_default.err
timeout 900 python bench.py --steps 20 --warmup 5 > $D/bench_k20.json 2> $D/bench_k20.err
timeout 600 python tools/lc_chain.py --batch 32 --autotune --chain-autotune --reps 20 > $D/lc_chain_b32.json 2>&1
timeout 600 python tools/lc_chain.py --batch 1 --autotune --chain-autotune --reps 20 > $D/lc_chain_b1.json 2>&1
