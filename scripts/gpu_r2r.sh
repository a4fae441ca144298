#!/bin/bash
# source-ordered X_g copy + one-wave TN splits: C3 / C4 / C2 benches, RGCN + TN tests
O=gpurun_out/r2r
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3.json 2> $O/c3.err
timeout 600 $B > $O/c4.json 2> $O/c4.err
timeout 600 $B --config C2 --model gat > $O/c2.json 2> $O/c2.err
timeout 1500 python -m pytest tests/test_gpu_conv_rgcn.py tests/test_gpu_fullsize.py tests/test_gpu_conv_lin.py tests/test_gpu_gemm.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
tail -3 $O/tests.log
