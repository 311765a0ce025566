mkdir -p gpurun_out/ncube
timeout 600 ncu --set full --import-source on --clock-control none -k regex:be_original_kernel --launch-skip 1 -c 2 -f -o gpurun_out/ncube/stencil_mriq python tools/be_launch.py stencil,mriq 2 > gpurun_out/ncube/log.txt 2>&1
