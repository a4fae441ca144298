#!/bin/bash
# GAT C2 occupancy / rows-in-flight sweep (WG_GAT_V selects the fwd2 / bwd_src3 instantiation)
O=gpurun_out/r3g
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for v in 0 1 2 3 4; do
  WG_GAT_V=$v timeout 600 python bench.py --no-cpu --no-e2e --config C2 --model gat > $O/c2_v$v.json 2> $O/c2_v$v.err
done
WG_GAT_V=0 timeout 600 python bench.py --no-cpu --no-e2e --config C2 --model gat > $O/c2_v0b.json 2> $O/c2_v0b.err
