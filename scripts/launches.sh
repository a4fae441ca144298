#!/bin/bash
# per-kernel launch list (cold, serialized) for configs: bash scripts/launches.sh "C3 rgcn" "C2 gat"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for cm in "$@"; do
  set -- $cm
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control ${CACHE:-all} --csv --log-file gpurun_out/launches_$1_$2.csv \
    python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-cpu --no-e2e > /dev/null 2> gpurun_out/launches_$1_$2.err
  echo "$1 $2 exit $?"
done
