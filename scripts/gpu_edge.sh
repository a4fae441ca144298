#!/bin/bash
# Degenerate-input parity tests (+ the three conv test modules they reuse)
mkdir -p gpurun_out/edge
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/edge/build.log 2>&1 || { tail -30 gpurun_out/edge/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_edge_cases.py -m gpu -q --timeout 300 > gpurun_out/edge/edge.log 2>&1
echo "edge exit $?"; tail -n 30 gpurun_out/edge/edge.log
timeout 900 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_conv_gat.py tests/test_gpu_conv_rgcn.py -m gpu -q --timeout 300 > gpurun_out/edge/conv.log 2>&1
echo "conv exit $?"; tail -n 3 gpurun_out/edge/conv.log
