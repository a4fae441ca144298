#!/bin/bash
# Bench every config/model combination (one GPU); JSON lines to gpurun_out/bench_<cfg>_<model>.json
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin" "C4 sage"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --steps ${STEPS:-10} --warmup 3 ${EXTRA} \
     > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"; tail -c 600 gpurun_out/bench_$1_$2.json
done
