#!/bin/bash
# quick GPU check of selected tests: bash scripts/gpu_quick.sh <pytest -k expr>
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -k "$1" > gpurun_out/quick.log 2>&1
tail -40 gpurun_out/quick.log
