#!/bin/bash
# EXPERIMENT: what bounds the grouped 3xTF32 TN GEMM (C3 dW_r): converters off / 1 MMA per k-step
O=gpurun_out/r3e
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for x in 0 1 2 3; do
  WG_TN_EXP=$x timeout 600 python bench.py --no-cpu --no-e2e --steps 5 --config C3 --model rgcn > $O/c3_exp$x.json 2> $O/c3_exp$x.err
done
grep -h -o '"tc_gemm_tn": {[^}]*}' $O/*.json
