#!/bin/bash
# softmax-xent rows in flight (raw vectors, 4 CTAs / SM): tests + ncu time of k_xent_vec (C4 47 classes bf16, C2 40 fp32)
O=gpurun_out/r3l
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_stack.py -m gpu -q -x -k "xent or adam or training" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 600 ncu --metrics $M --clock-control none --csv -k regex:"k_xent" --log-file $O/xent_c4.csv $B > /dev/null 2> $O/x4.err
timeout 600 ncu --metrics $M --clock-control none --csv -k regex:"k_xent" --log-file $O/xent_c2.csv $B --config C2 --model gat > /dev/null 2> $O/x2.err
timeout 600 python bench.py --no-cpu --no-e2e > $O/c4.json 2> $O/c4.err
tail -2 $O/tests.log
