mkdir -p gpurun_out/r2j
O=gpurun_out/r2j
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_conv_gat.py tests/test_gpu_conv_lin.py tests/test_gpu_edge_cases.py -m gpu -q > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
timeout 900 python bench.py --config C2 --model gat --steps 20 --warmup 5 --no-cpu > $O/bench_c2.json 2> $O/bench_c2.err
WG_GAT_HALF=0 timeout 900 python bench.py --config C2 --model gat --steps 20 --warmup 5 --no-cpu --no-e2e > $O/bench_c2_nohalf.json 2> $O/bench_c2_nohalf.err
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu > $O/bench_c4.json 2> $O/bench_c4.err
timeout 1500 compute-sanitizer --tool synccheck --error-exitcode 9 python scripts/sanitize_cases.py > $O/san_synccheck.log 2>&1; echo "synccheck rc=$?" >> $O/san_rc.txt
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed.sum --clock-control none --csv -k regex:"k_gat|k_agg" --log-file $O/gat_C2.csv $B --config C2 --model gat > /dev/null 2> $O/gat_C2.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:"k_agg" --log-file $O/agg_C4.csv $B > /dev/null 2> $O/agg_C4.err
