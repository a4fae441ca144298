#!/bin/bash
# full GPU test suite (+ smoke)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/gpu_all.log 2>&1
echo "pytest exit $?"; tail -n 15 gpurun_out/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -n 3
