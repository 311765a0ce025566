# round-2b final capture: default bench (K = 100), reference arm, launch list of the timed region,
# per-launch DRAM traffic of one b32 LC query, ncu --set full of the dominant LC conv class
D=gpurun_out/r02c_final
mkdir -p $D
timeout 1500 python bench.py > $D/bench_default.json 2> $D/bench_default.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $D/bench_reference.json 2> $D/bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv --log-file $D/launches_timed.csv python bench.py --steps 2 --warmup 3 --no-extra --no-cpu --seeds 1 > $D/bench_under_ncu.log 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "query/" -k regex:fused_kernel -c 53 --csv --log-file $D/lc_b32_dram.csv python tools/lc_query.py 32 1 1 > $D/lc_dram.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include "query/" -k regex:fused_kernel -c 8 -f -o $D/lc_b32_full python tools/lc_query.py 32 1 1 > $D/lc_full.log 2>&1
gzip -f $D/launches_timed.csv
