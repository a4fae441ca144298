#!/bin/bash
# bash scripts/gpu_cfg.sh "<pytest -k expr or ''>" "C2 gat" "C3 rgcn" ...   (tests, then bench lines)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
K="$1"; shift
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 -k "$K" > gpurun_out/quick.log 2>&1
  echo "pytest exit $?"; tail -n 12 gpurun_out/quick.log
fi
for cm in "$@"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --steps ${STEPS:-10} --warmup 3 --no-cpu ${EXTRA} > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"; tail -n 3 gpurun_out/bench_$1_$2.err
done
