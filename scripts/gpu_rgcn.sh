#!/bin/bash
# RGCN iteration: tests, C3 bench line, ordered launch list
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "rgcn or RGCN" > gpurun_out/quick.log 2>&1
echo "pytest exit $?"; tail -n 5 gpurun_out/quick.log
timeout 600 python bench.py --config C3 --model rgcn --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_C3_rgcn.json 2> gpurun_out/bench_C3_rgcn.err
python scripts/show_bench.py gpurun_out/bench_C3_rgcn.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C3_rgcn.csv \
    python bench.py --config C3 --model rgcn --steps 1 --warmup 1 --no-cpu --no-e2e > /dev/null 2>&1
python scripts/launch_seq.py gpurun_out/launches_C3_rgcn.csv 45
