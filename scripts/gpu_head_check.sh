#!/bin/bash
# Full GPU suite + smoke + default bench line at HEAD: gpurun_out/head
O=gpurun_out/head; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 > $O/gpu_tests.log 2>&1
echo "pytest exit $?"; tail -n 2 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; tail -n 1 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "default exit $?"
python scripts/show_bench.py $O/bench_default.json | head -1
