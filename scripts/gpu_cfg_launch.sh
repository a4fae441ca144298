#!/bin/bash
# tests (-k expr), bench lines and an ncu launch list of each config:
# bash scripts/gpu_cfg_launch.sh "<pytest -k expr or ''>" "C2 gat" ...
bash scripts/gpu_cfg.sh "$@"
shift
for cm in "$@"; do
  set -- $cm
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$1_$2.csv \
    python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-cpu --no-e2e > /dev/null 2> gpurun_out/launches_$1_$2.err
  echo "launches $1 $2 exit $?"
done
