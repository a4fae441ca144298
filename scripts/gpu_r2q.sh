#!/bin/bash
# C3 RGCN and C2 GAT launch lists with DRAM bytes and L2 hit rate (one epoch after warm-up)
O=gpurun_out/r2q
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__throughput.avg.pct_of_peak_sustained_elapsed
timeout 1200 ncu --metrics $M --clock-control none --csv --log-file $O/c3.csv $B --config C3 --model rgcn > /dev/null 2> $O/c3.err
timeout 1200 ncu --metrics $M --clock-control none --csv --log-file $O/c2.csv $B --config C2 --model gat > /dev/null 2> $O/c2.err
