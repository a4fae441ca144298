#!/bin/bash
# One GPU session: build, tests, bench, ncu launch list + full capture of the
# gather/segment-reduce kernel.  Usage: bash scripts/gpu_round.sh [tests|bench|ncu|all]
mode=${1:-all}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [[ $mode == tests || $mode == all ]]; then
  timeout 900 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/gputest.log 2>&1
  tail -15 gpurun_out/gputest.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
fi
if [[ $mode == bench || $mode == all ]]; then
  timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
  tail -c 3000 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
fi
if [[ $mode == ncu || $mode == all ]]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_run.log 2>&1
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_agg -s 6 -c 3 -o gpurun_out/prof_agg -f \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_run.log 2>&1
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gemm_nt_p -s 4 -c 3 -o gpurun_out/prof_gemm -f \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_gemm_run.log 2>&1
  ls -la gpurun_out/*.ncu-rep
fi
if [[ $mode == ncuagg ]]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_agg_cp -s 5 -c 1 -o gpurun_out/prof_agg1 -f \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_agg1.log 2>&1
  ls -la gpurun_out/prof_agg1.ncu-rep
fi
if [[ $mode == ncugemm ]]; then
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_gemm_nt_p|k_tc_gemm" -s 4 -c 6 -o gpurun_out/prof_gemm -f \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_gemm_run.log 2>&1
  ls -la gpurun_out/prof_gemm.ncu-rep
fi
