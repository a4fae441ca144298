#!/bin/bash
# smoke + every bench line at HEAD (no ncu): gpurun_out/bench_head
O=gpurun_out/bench_head; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -n 1 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "default exit $?"
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --no-cpu > $O/bench_$1_$2.json 2> $O/bench_$1_$2.err
  echo "$1 $2 exit $?"
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference exit $?"
timeout 1200 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/bench_C5_slice.json 2> $O/bench_C5_slice.err; echo "C5 slice exit $?"
for f in $O/bench_*.json; do python scripts/show_bench.py $f | head -1; done
