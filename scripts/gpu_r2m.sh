mkdir -p gpurun_out/r2m
O=gpurun_out/r2m
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for v in 0 1 2 3; do
WG_GAT_HALF=$v timeout 600 python bench.py --config C2 --model gat --steps 20 --warmup 5 --no-cpu --no-e2e > $O/c2_half$v.json 2> $O/c2_half$v.err
done
WG_GAT_HALF=2 timeout 900 python -m pytest tests/test_gpu_conv_gat.py -m gpu -q > $O/tests_half2.log 2>&1; echo "rc=$?" >> $O/tests_half2.log
