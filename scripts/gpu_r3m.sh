#!/bin/bash
# NT bfold (fp32, BN <= 64, pre-split weights): RGCN parity + C3 A/B (WG_NT_BFOLD=0 restores 3 MMAs / k-step)
O=gpurun_out/r3m
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_conv_rgcn.py tests/test_gpu_fullsize.py -m gpu -q -x -k "rgcn" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C3 --model rgcn > $O/c3_bfold.json 2> $O/c3_bfold.err
WG_NT_BFOLD=0 timeout 600 $B --config C3 --model rgcn > $O/c3_nobfold.json 2> $O/c3_nobfold.err
timeout 600 $B --config C3 --model rgcn > $O/c3_bfold2.json 2> $O/c3_bfold2.err
WG_NT_BFOLD=0 timeout 600 $B --config C3 --model rgcn > $O/c3_nobfold2.json 2> $O/c3_nobfold2.err
tail -3 $O/tests.log
