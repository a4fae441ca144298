#!/bin/bash
# stack + gat tests, then bench all configs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_stack.py tests/test_gpu_conv_gat.py -x -q > gpurun_out/pytest_stack.log 2>&1
echo "pytest exit $?"; tail -5 gpurun_out/pytest_stack.log
STEPS=10 bash scripts/bench_all.sh
