#!/bin/bash
# fp32 TN with separate lo buffers: tests + C3 / C2 / C4 benches + ncu of the TN launches
O=gpurun_out/r2t
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_rgcn.py tests/test_gpu_conv_lin.py tests/test_gpu_conv_gat.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3.json 2> $O/c3.err
timeout 600 $B --config C2 --model gat > $O/c2.json 2> $O/c2.err
timeout 600 $B > $O/c4.json 2> $O/c4.err
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed
timeout 1200 ncu --metrics $M --clock-control none --csv -k regex:"k_tc|k_gemm" --log-file $O/c3.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph --config C3 --model rgcn > /dev/null 2> $O/c3n.err
tail -3 $O/tests.log
