#!/bin/bash
O=gpurun_out/r2s
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__throughput.avg.pct_of_peak_sustained_elapsed
timeout 600 python bench.py --no-cpu --no-e2e --config C3 --model rgcn > $O/c3.json 2> $O/c3b.err
timeout 1200 ncu --metrics $M --clock-control none --csv -k regex:"k_xg|k_agg|k_tc" --log-file $O/c3.csv $B --config C3 --model rgcn > /dev/null 2> $O/c3.err
timeout 1500 python -m pytest tests/test_gpu_conv_rgcn.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
tail -3 $O/tests.log
