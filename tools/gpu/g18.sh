timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -x -q -m gpu --timeout 300 -p no:cacheprovider -k "cutcp or CUTCP" > gpurun_out/g18_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/g18_tests.log
python tools/be_table.py 2>&1 | tail -2
NAMES=$(python -c "import sys; sys.path.insert(0,'.'); import synth; print(' '.join(c.name if c.name!='conv1' else 'conv1.gemm' for c in synth.resnet50_convs(32)))")
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv --nvtx --nvtx-include "target/" --log-file gpurun_out/lc_traffic.csv python tools/lc_one.py --reps 1 $NAMES > gpurun_out/g18_ncu.log 2>&1
tail -2 gpurun_out/g18_ncu.log; wc -l gpurun_out/lc_traffic.csv
