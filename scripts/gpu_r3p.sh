#!/bin/bash
# NT persistent: direct stores for a chunk straddling the D / D2 split (C5's 32-wide [Y|S]); wide xent
O=gpurun_out/r3p
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_stack.py tests/test_gpu_edge_cases.py tests/test_gpu_fullsize.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
timeout 1200 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 --no-cpu --no-e2e > $O/c5.json 2> $O/c5.err
timeout 600 python bench.py --no-cpu --no-e2e > $O/c4.json 2> $O/c4.err
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_c5.csv python bench.py --config C5 --rank-slice 8 --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph > /dev/null 2> $O/g5.err
tail -2 $O/tests.log
