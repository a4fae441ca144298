#!/bin/bash
# TN M-fold (fp32, M <= 64): parity tests + C3 / C1 A/B (WG_TN_FOLD=0 restores 3 MMAs per k-step)
O=gpurun_out/r3i
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_rgcn.py tests/test_gpu_conv_lin.py tests/test_gpu_conv_lstm.py tests/test_gpu_stack.py tests/test_gpu_edge_cases.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3_fold.json 2> $O/c3_fold.err
WG_TN_FOLD=0 timeout 600 $B --config C3 --model rgcn > $O/c3_nofold.json 2> $O/c3_nofold.err
timeout 600 $B --config C3 --model rgcn > $O/c3_fold2.json 2> $O/c3_fold2.err
timeout 600 $B --config C1 --model gcn > $O/c1.json 2> $O/c1.err
tail -3 $O/tests.log
