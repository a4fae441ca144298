#!/bin/bash
# Copy the session-3 evidence run (gpurun_out/final) into profiles/r01/session3/final
O=gpurun_out/final; P=profiles/r01/session3/final
mkdir -p $P
cp $O/bench_*.json $O/gpu_tests.log $O/smoke.log $O/gpu.txt $P/ 2>/dev/null
for f in $O/launches_*.csv; do
  b=$(basename $f .csv); cp $f $P/
  python scripts/launch_table.py $f 30 > $P/${b/launches/launch_table}.txt
done
cp $O/full_*.txt $P/ 2>/dev/null
for f in $O/full_*_raw.csv; do gzip -c $f > $P/$(basename $f).gz; done
python scripts/ncu_traffic.py $O/full_C4_sage_agg_raw.csv C4:sage:gather_reduce "k_agg" "session 3, one epoch's 5 launches"
python scripts/ncu_traffic.py $O/full_C3_rgcn_agg_raw.csv C3:rgcn:gather_reduce "k_agg" "session 3, one epoch's 9 launches"
for f in $P/bench_*.json; do python scripts/show_bench.py $f | head -1; done
