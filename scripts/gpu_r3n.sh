#!/bin/bash
# C5 rank-slice launch list (what is in its 8 ms "misc" class) + wide-row softmax-xent
O=gpurun_out/r3n
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_stack.py -m gpu -q -x -k "xent" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 1500 ncu --metrics $M --clock-control none --csv --log-file $O/launches_C5.csv python bench.py --config C5 --rank-slice 8 --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph > /dev/null 2> $O/l5.err
timeout 1200 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 --no-cpu --no-e2e > $O/c5.json 2> $O/c5.err
tail -2 $O/tests.log
