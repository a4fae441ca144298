mkdir -p gpurun_out/r2f
O=gpurun_out/r2f
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_conv_lstm.py tests/test_gpu_stack.py -m gpu -q > $O/tests.log 2>&1; echo rc=$? >> $O/tests.log
