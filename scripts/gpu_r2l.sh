mkdir -p gpurun_out/r2l
O=gpurun_out/r2l
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_stack.py tests/test_gpu_fullsize.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e --model gin > $O/bench_c4gin.json 2> $O/bench_c4gin.err
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_C4_sage.csv $B > /dev/null 2> $O/gemm.err
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_agg_cp" -s 2 -c 1 -o $O/full_L3 -f $B > $O/full_L3.log 2>&1
ncu -i $O/full_L3.ncu-rep --page source --csv > $O/full_L3_source.csv 2>/dev/null
ncu -i $O/full_L3.ncu-rep --page raw --csv > $O/full_L3_raw.csv 2>/dev/null
rm -f $O/full_L3.ncu-rep
