#!/bin/bash
# A/B the gather-reduce kernel variants on the C4 bench (WG_AGG_CFG / WG_AGG_V2)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for v in "0" "1" "2"; do
  WG_AGG_CFG=$v timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_cfg$v.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/bench_cfg$v.json').read().strip().splitlines()[-1]); print('cfg $v', round(d['ms_per_step'],2), round(d['kernels']['gather_reduce']['ms_per_step'],2), round(d['roofline']['frac'],3))"
done
