#!/bin/bash
# tests matching $1, then ordered launch lists of C2 GAT and C4 SAGE (one epoch each)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "$1" > gpurun_out/quick.log 2>&1
echo "pytest exit $?"; tail -n 4 gpurun_out/quick.log
for cm in "C2 gat" "C4 sage"; do
  set -- $cm
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$1_$2.csv \
    python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-cpu --no-e2e > /dev/null 2>&1
  python scripts/launch_seq.py gpurun_out/launches_$1_$2.csv 60
done
