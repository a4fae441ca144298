#!/bin/bash
# A/B of the round-3 changes: targeted GPU tests + C1..C4 benches
O=gpurun_out/r3c
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_stack.py tests/test_gpu_conv_gat.py tests/test_gpu_conv_rgcn.py tests/test_gpu_conv_lin.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3.json 2> $O/c3.err
timeout 600 $B --config C2 --model gat > $O/c2.json 2> $O/c2.err
timeout 600 $B --config C1 --model gcn > $O/c1.json 2> $O/c1.err
timeout 600 $B > $O/c4.json 2> $O/c4.err
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 600 ncu --metrics $M --clock-control none --csv --log-file $O/launches_C2.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph --config C2 --model gat > /dev/null 2> $O/l2.err
tail -3 $O/tests.log
