for r in 0 1; do for bn in 0 64 128 256; do for nm in layer2.0.conv2 layer1.0.conv3; do
  timeout 60 python tools/gpu/diag_residual.py $nm $bn $r > /tmp/o.txt 2>&1; echo "$nm bn=$bn res=$r rc=$?"; tail -2 /tmp/o.txt
done; done; done
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 -p no:cacheprovider --deselect "tests/test_gpu_bench_configs.py::test_b32_conv_residual_epilogue_vs_oracle" > gpurun_out/g2_all.log 2>&1; echo "all rc=$?"
tail -30 gpurun_out/g2_all.log
