#!/bin/bash
# hot-row L2 policy A/B: C4 SAGE / GIN, C5 slice, C3; GPU tests of the gather paths
O=gpurun_out/r2n
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for h in 0 196608 65536 393216; do
  WG_HOT_ROWS=$h timeout 600 python bench.py --no-cpu --no-e2e > $O/c4_h$h.json 2> $O/c4_h$h.err
done
WG_HOT_ROWS=0 timeout 600 python bench.py --no-cpu --no-e2e --config C4 --model gin > $O/c4gin_h0.json 2> $O/c4gin_h0.err
timeout 600 python bench.py --no-cpu --no-e2e --config C4 --model gin > $O/c4gin.json 2> $O/c4gin.err
WG_HOT_ROWS=0 timeout 900 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 --no-cpu --no-e2e > $O/c5_h0.json 2> $O/c5_h0.err
timeout 900 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 --no-cpu --no-e2e > $O/c5.json 2> $O/c5.err
timeout 1200 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_fullsize.py tests/test_gpu_stack.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
tail -3 $O/tests.log
