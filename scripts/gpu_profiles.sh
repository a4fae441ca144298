#!/bin/bash
# Round evidence: default bench line, all-config bench lines, ncu launch list of
# the default command, ncu --set full of the dominant kernels (C4 SAGE).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo "default exit $?"
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 > gpurun_out/bench_$1_$2.json 2> gpurun_out/bench_$1_$2.err
  echo "$1 $2 exit $?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_default.csv \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_run.log 2>&1
echo "launch list exit $?"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_agg_cp|k_gemm_nt_p|k_tc_gemm" -s 20 -c 12 \
  -o gpurun_out/prof_c4 -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/prof_c4.log 2>&1
echo "ncu full exit $?"
ls -la gpurun_out/*.ncu-rep
