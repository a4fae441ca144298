#!/bin/bash
# Round-2 final evidence (session 4 final code): GPU tests + smoke, bench lines for every config, rank slices,
# the reference arm, ncu launch list + full capture of the dominant kernel,
# tensor-pipe metrics of the GEMM classes (compute-sanitizer is closed on the pool).
O=gpurun_out/final_r2e
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > $O/gpu_tests.log 2>&1; echo "pytest rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
for cm in "C1 gcn" "C2 gat" "C3 rgcn" "C4 gin"; do
  set -- $cm
  timeout 900 python bench.py --config $1 --model $2 --no-cpu > $O/bench_$1_$2.json 2> $O/bench_$1_$2.err
done

timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err
timeout 1200 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/bench_C5_slice.json 2> $O/bench_C5_slice.err
timeout 900 python bench.py --rank-slice 8 --steps 10 --warmup 3 > $O/bench_C4_slice8.json 2> $O/bench_C4_slice8.err
timeout 900 python bench.py --rank-slice 8 --steps 10 --warmup 3 --emulate-xchg > $O/bench_C4_slice8_x.json 2> $O/bench_C4_slice8_x.err
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_C4_sage.csv $B > /dev/null 2> $O/launches_C4_sage.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_C4_sage.csv $B > /dev/null 2> $O/gemm_C4.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_C3_rgcn.csv $B --config C3 --model rgcn > /dev/null 2> $O/gemm_C3.err
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_agg_cp" -c 5 -o $O/full_C4_sage_agg -f $B > $O/full_C4_sage_agg.log 2>&1
ncu -i $O/full_C4_sage_agg.ncu-rep --page raw --csv > $O/full_C4_sage_agg_raw.csv 2>/dev/null
python scripts/ncu_summary.py $O/full_C4_sage_agg.ncu-rep > $O/full_C4_sage_agg.txt 2>&1
rm -f $O/full_C4_sage_agg.ncu-rep


ls -la $O | tail -40
