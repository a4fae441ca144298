#!/bin/bash
# C3 / C2 launch lists + full ncu of the C3 grouped TN GEMM and Y GEMM
O=gpurun_out/r3b
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed
timeout 900 ncu --metrics $M --clock-control none --csv --log-file $O/launches_C3.csv $B --config C3 --model rgcn > /dev/null 2> $O/l3.err
timeout 900 ncu --metrics $M --clock-control none --csv --log-file $O/launches_C2.csv $B --config C2 --model gat > /dev/null 2> $O/l2.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_tc_gemm" -c 2 -o $O/full_C3_tn -f $B --config C3 --model rgcn > $O/full_C3_tn.log 2>&1
ncu -i $O/full_C3_tn.ncu-rep --page details --csv > $O/full_C3_tn_details.csv 2>/dev/null
ncu -i $O/full_C3_tn.ncu-rep --page source --csv > $O/full_C3_tn_source.csv 2>/dev/null
ls -la $O
