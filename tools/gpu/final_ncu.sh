# launch list of the timed region and per-launch LC DRAM bytes on the final head
D=gpurun_out/final_ncu
mkdir -p $D
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv --log-file $D/launches_timed.csv python bench.py --steps 2 --warmup 3 --no-extra --no-cpu --seeds 1 > $D/bench_under_ncu.log 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "query/" -k regex:fused_kernel -c 53 --csv --log-file $D/lc_b32_dram.csv python tools/lc_query.py 32 1 1 > $D/lc_dram.log 2>&1
gzip -f $D/launches_timed.csv
