#!/bin/bash
# Session-3 round evidence: GPU tests + smoke, bench lines for every config
# (default C4 SAGE with the oracle baseline, C5 rank slice, the reference arm),
# ncu launch lists and --set full captures of the dominant kernel classes.
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > $O/gpu_tests.log 2>&1
echo "pytest exit $?"; tail -n 3 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -n 2 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "default exit $?"
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --no-cpu > $O/bench_$1_$2.json 2> $O/bench_$1_$2.err
  echo "$1 $2 exit $?"
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference exit $?"
timeout 1200 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/bench_C5_slice.json 2> $O/bench_C5_slice.err; echo "C5 slice exit $?"
for f in $O/bench_*.json; do python scripts/show_bench.py $f | head -1; done
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
for cm in "C4 sage" "C3 rgcn" "C2 gat" "C4 gin"; do
  set -- $cm
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$1_$2.csv \
    $B --config $1 --model $2 > /dev/null 2> $O/launches_$1_$2.err
  echo "launches $1 $2 exit $?"
done
full() {  # config model regex count name
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$3" -c $4 -o $O/$5 -f \
    $B --config $1 --model $2 > $O/$5.log 2>&1
  echo "full $5 exit $?"
  ncu -i $O/$5.ncu-rep --page raw --csv > $O/$5_raw.csv 2>/dev/null
  python scripts/ncu_summary.py $O/$5.ncu-rep > $O/$5.txt 2>&1
  rm -f $O/$5.ncu-rep
}
full C4 sage "k_agg_cp" 5 full_C4_sage_agg
full C3 rgcn "k_agg" 9 full_C3_rgcn_agg
full C2 gat "k_gat" 14 full_C2_gat
ls -la $O | tail -40
