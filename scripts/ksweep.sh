#!/bin/bash
# measured sweep of the gTask edge limit E_max (the paper's
# K sweeps, Fig 18) -- bench lines per (config, model, E_max)
mkdir -p gpurun_out/ksweep
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
IFS=',' read -ra LIST <<< "${CMS:-C4 sage,C3 rgcn}"   # CMS: comma-separated "config model" pairs
for cm in "${LIST[@]}"; do
  set -- $cm
  for t in ${TS:-128}; do
    for k in ${KS:-1024 4096 16384 65536}; do
      tag=$k; [ "$t" != 128 ] && tag=T${t}_$k
      timeout 600 python bench.py --config $1 --model $2 --steps 5 --warmup 3 --no-cpu --no-e2e --emax $k --tile $t \
        > gpurun_out/ksweep/$1_$2_$tag.json 2> gpurun_out/ksweep/$1_$2_$tag.err
      echo "$1 $2 T=$t E_max=$k exit $?"
    done
  done
done
python scripts/ksweep_table.py gpurun_out/ksweep/*.json
