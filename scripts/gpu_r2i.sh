mkdir -p gpurun_out/r2i
O=gpurun_out/r2i
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 python bench.py --config C2 --model gat --steps 20 --warmup 5 --no-cpu > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --config C4 --model gin --steps 20 --warmup 5 --no-cpu > $O/bench_c4gin.json 2> $O/bench_c4gin.err
timeout 2400 python -m pytest tests -m gpu -q -x > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 1500 python scripts/outlier_breakdown.py > $O/outlier_breakdown.md 2> $O/outlier_breakdown.err
bash scripts/hidden_sweep.sh
timeout 1500 compute-sanitizer --tool synccheck --error-exitcode 9 python scripts/sanitize_cases.py > $O/san_synccheck.log 2>&1; echo "synccheck rc=$?" >> $O/san_rc.txt
