#!/bin/bash
# Session-3 check at HEAD: full GPU tests + smoke, then every bench config.
mkdir -p gpurun_out
bash scripts/gpu_tests.sh
STEPS=10 bash scripts/bench_all.sh 2>&1 | grep -E "exit"
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
tail -c 1500 gpurun_out/bench_default.json
