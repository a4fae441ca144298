#!/bin/bash
# GAT row-chunk length sweep on C2 (WG_GAT_CHUNK)
O=gpurun_out/r3r
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for c in 256 128 512 1024 2048 256; do
  WG_GAT_CHUNK=$c timeout 600 python bench.py --no-cpu --no-e2e --config C2 --model gat > $O/c2_$c.json 2> $O/c2_$c.err
  cp $O/c2_$c.json $O/c2_${c}_$(date +%s%N).json
done
WG_GAT_CHUNK=1024 timeout 900 python -m pytest tests/test_gpu_conv_gat.py -m gpu -q -x > $O/tests_1024.log 2>&1; echo "rc=$?" >> $O/tests_1024.log
