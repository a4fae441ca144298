#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/pytest_all.log 2>&1
echo "pytest exit $?"; tail -15 gpurun_out/pytest_all.log
for cm in "C2 gat" "C3 rgcn" "C1 gcn"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"; tail -3 gpurun_out/bench_$1_$2.err
done
