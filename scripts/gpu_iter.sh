#!/bin/bash
# quick iteration: tests matching $1, bench lines for the remaining "CFG model" args, C3 launch order
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
K="$1"; shift
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -k "$K" > gpurun_out/quick.log 2>&1
  echo "pytest exit $?"; tail -n 4 gpurun_out/quick.log
fi
for cm in "$@"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --steps ${STEPS:-10} --warmup 3 --no-cpu ${EXTRA} > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"; python scripts/show_bench.py gpurun_out/bench_$1_$2.json
done
if [ -n "$SEQ" ]; then
  set -- $SEQ
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$1_$2.csv \
    python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-cpu --no-e2e > /dev/null 2>&1
  python scripts/launch_seq.py gpurun_out/launches_$1_$2.csv ${SEQN:-45}
fi
