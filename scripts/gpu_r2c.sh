# L2::64B row copies: C4 SAGE / GIN bench + per-launch DRAM bytes of the gathers; C5 slice (compute only)
mkdir -p gpurun_out/r2c
O=gpurun_out/r2c
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu > $O/bench_c4_sage.json 2> $O/bench_c4_sage.err
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --model gin > $O/bench_c4_gin.json 2> $O/bench_c4_gin.err
timeout 900 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/bench_c5.json 2> $O/bench_c5.err
timeout 900 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 --emulate-xchg > $O/bench_c5_x.json 2> $O/bench_c5_x.err
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:"k_agg" --log-file $O/agg_C4_sage.csv $B > /dev/null 2> $O/agg_C4_sage.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_agg" -c 12 --log-file $O/agg_C5.csv $B --config C5 --rank-slice 8 > /dev/null 2> $O/agg_C5.err
