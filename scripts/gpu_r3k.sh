#!/bin/bash
# fp32 persistent NT GEMM: BN 128 (3 stages of raw + lo twin) vs BN 64 (4 stages) on C2 / C1
O=gpurun_out/r3k
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B --config C2 --model gat > $O/c2_bn128.json 2> $O/c2_bn128.err
WG_NT_BNMAX=64 timeout 600 $B --config C2 --model gat > $O/c2_bn64.json 2> $O/c2_bn64.err
timeout 600 $B --config C2 --model gat > $O/c2_bn128b.json 2> $O/c2_bn128b.err
WG_NT_BNMAX=64 timeout 600 $B --config C2 --model gat > $O/c2_bn64b.json 2> $O/c2_bn64b.err
