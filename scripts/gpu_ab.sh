#!/bin/bash
# A/B of env settings on one bench config: bash scripts/gpu_ab.sh "C4 sage" "WG_NT_BNMAX=256" "WG_NT_BNMAX=128" ...
mkdir -p gpurun_out/ab
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
cm="$1"; shift
set -- $cm "$@"
cfg=$1; model=$2; shift 2
for envs in "$@"; do
  tag=$(echo "$envs" | tr ' =' '__')
  env $envs timeout 600 python bench.py --config $cfg --model $model --steps 10 --warmup 3 --no-cpu ${EXTRA} \
    > gpurun_out/ab/${cfg}_${model}_$tag.json 2> gpurun_out/ab/${cfg}_${model}_$tag.err
  echo "== $envs"; python scripts/show_bench.py gpurun_out/ab/${cfg}_${model}_$tag.json | head -6
done
