#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/gpu_all.log 2>&1
echo "pytest exit $?"; tail -n 3 gpurun_out/gpu_all.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_agg -s 6 -c 2 -o gpurun_out/c5_agg -f \
  python bench.py --config C5 --rank-slice 8 --steps 1 --warmup 1 --no-graph > gpurun_out/c5_agg.log 2>&1
echo "ncu exit $?"
python scripts/ncu_summary.py gpurun_out/c5_agg.ncu-rep > gpurun_out/c5_agg.txt
