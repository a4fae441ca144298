mkdir -p gpurun_out/r2k
O=gpurun_out/r2k
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_stack.py tests/test_gpu_conv_lstm.py tests/test_gpu_edge_cases.py tests/test_gpu_conv_gat.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
for b in 1 0; do
WG_NT_BRES=$b timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e > $O/bench_c4_bres$b.json 2> $O/bench_c4_bres$b.err
WG_NT_BRES=$b timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e --model gin > $O/bench_c4gin_bres$b.json 2> $O/bench_c4gin_bres$b.err
done
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed
timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_C4_sage.csv $B > /dev/null 2> $O/gemm.err
