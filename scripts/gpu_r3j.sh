#!/bin/bash
# GAT logits fused into the G GEMM epilogue + RGCN layer-2 shape test
O=gpurun_out/r3j
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_gat.py tests/test_gpu_conv_rgcn.py tests/test_gpu_fullsize.py -m gpu -q -x -k "gat or rgcn" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C2 --model gat > $O/c2.json 2> $O/c2.err
timeout 600 $B --config C2 --model gat > $O/c2b.json 2> $O/c2b.err
tail -3 $O/tests.log
