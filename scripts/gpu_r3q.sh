#!/bin/bash
# k_colsum at 4 CTAs / SM (64 registers): tests + ncu times on C4 / C5 slice + benches
O=gpurun_out/r3q
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_stack.py tests/test_gpu_conv_gat.py tests/test_gpu_conv_rgcn.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 600 ncu --metrics $M --clock-control none --csv -k regex:"k_colsum" --log-file $O/colsum_c4.csv $B > /dev/null 2> $O/c4n.err
timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"k_colsum" --log-file $O/colsum_c5.csv $B --config C5 --rank-slice 8 > /dev/null 2> $O/c5n.err
timeout 600 python bench.py --no-cpu --no-e2e > $O/c4.json 2> $O/c4.err
tail -2 $O/tests.log
