#!/bin/bash
O=gpurun_out/r3d
mkdir -p $O
timeout 120 ./scripts/mma_probe > $O/mma_probe.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_conv_gat.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
timeout 600 python bench.py --no-cpu --no-e2e --config C2 --model gat > $O/c2.json 2> $O/c2.err
cat $O/mma_probe.txt; tail -2 $O/tests.log
