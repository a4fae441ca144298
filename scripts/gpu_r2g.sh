# measurement extras: TF32 peak, tensor-pipe utilisation of the GEMM classes, sanitizers
mkdir -p gpurun_out/r2g
O=gpurun_out/r2g
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
python scripts/tf32_peak.py $O/tf32_peak.json > $O/tf32.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_tc.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
for cm in "C4 sage" "C4 gin" "C3 rgcn" "C2 gat" "C1 gcn"; do
  set -- $cm
  timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"gemm" --log-file $O/gemm_$1_$2.csv $B --config $1 --model $2 > /dev/null 2> $O/gemm_$1_$2.err
done
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_cases.py > $O/san_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/san_rc.txt
done
