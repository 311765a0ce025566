mkdir -p gpurun_out/gaps
TACKER_LC_DBG=16 timeout 300 python tools/lc_gaps.py --batch 32 > gpurun_out/gaps/b32.json 2> gpurun_out/gaps/b32.err
TACKER_LC_DBG=16 timeout 300 python tools/lc_gaps.py --batch 32 --overlap 0 > gpurun_out/gaps/b32_serial.json 2>> gpurun_out/gaps/b32.err
TACKER_LC_DBG=16 timeout 300 python tools/lc_gaps.py --batch 1 > gpurun_out/gaps/b1.json 2>> gpurun_out/gaps/b32.err
