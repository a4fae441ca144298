mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -m gpu -q --timeout 120 -x -k "partition" > gpurun_out/gpu_part.log 2>&1
WG_DISABLE_TC=1 timeout 600 python -m pytest tests/test_gpu_conv_lin.py -q --timeout 120 > gpurun_out/gpu_lin_simt.log 2>&1
timeout 600 python -m pytest tests/test_gpu_conv_lin.py -q --timeout 120 > gpurun_out/gpu_lin_tc.log 2>&1
tail -3 gpurun_out/gpu_part.log gpurun_out/gpu_lin_simt.log gpurun_out/gpu_lin_tc.log
