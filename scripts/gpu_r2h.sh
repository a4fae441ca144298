# full GPU suite + sanitizers (all kernel families) + NT GEMM BN experiment + outlier breakdown + strategy search
mkdir -p gpurun_out/r2h
O=gpurun_out/r2h
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q --durations=20 > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
for bn in 256 128; do
  WG_NT_BNMAX=$bn timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > $O/bench_c4_bn$bn.json 2> $O/bench_c4_bn$bn.err
done
timeout 1500 python scripts/outlier_breakdown.py > $O/outlier_breakdown.md 2> $O/outlier_breakdown.err
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --tune --tune-cache $O/tune_cache.json > $O/bench_c4_tune.json 2> $O/bench_c4_tune.err
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_cases.py > $O/san_$tool.log 2>&1
  echo "$tool rc=$?" >> $O/san_rc.txt
done
