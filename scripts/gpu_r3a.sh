#!/bin/bash
# Validate HEAD: full GPU suite + C2 / C3 / C4 benches
O=gpurun_out/r3a
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3.json 2> $O/c3.err
timeout 600 $B --config C2 --model gat > $O/c2.json 2> $O/c2.err
timeout 600 $B > $O/c4.json 2> $O/c4.err
tail -3 $O/tests.log
