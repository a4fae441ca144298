mkdir -p gpurun_out/r2e
O=gpurun_out/r2e
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_stack.py tests/test_gpu_gpart.py -m gpu -q > $O/tests.log 2>&1; echo rc=$? >> $O/tests.log
for P in 2 4 8; do
timeout 600 python bench.py --rank-slice $P --steps 10 --warmup 3 > $O/c4_slice$P.json 2> $O/c4_slice$P.err
timeout 600 python bench.py --rank-slice $P --steps 10 --warmup 3 --emulate-xchg > $O/c4_slice${P}_x.json 2> $O/c4_slice${P}_x.err
done
WG_XCHG_CHUNK_BYTES=0 timeout 600 python bench.py --rank-slice 8 --steps 10 --warmup 3 --emulate-xchg > $O/c4_slice8_x_nochunk.json 2> $O/c4_slice8_x_nochunk.err
timeout 600 python bench.py --config C3 --rank-slice 4 --steps 5 --warmup 3 > $O/c3_slice4.json 2> $O/c3_slice4.err
