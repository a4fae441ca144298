#!/bin/bash
# Full check: build, all GPU tests, smoke, default bench, every config bench line.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt 2>&1
nproc > gpurun_out/nproc.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/gpu_all.log 2>&1
echo "pytest exit $?"; tail -n 15 gpurun_out/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -n 3 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo "default exit $?"; tail -c 400 gpurun_out/bench_default.json
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --no-cpu > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"
done
