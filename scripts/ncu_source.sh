#!/bin/bash
# One kernel launch under ncu --set full with source/SASS stall sampling; exports
# the raw + source pages as CSV (the .ncu-rep stays on the box unless small).
# bash scripts/ncu_source.sh <config> <model> <kernel regex> <skip> <name>
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$3" -s $4 -c 1 -o gpurun_out/$5 -f \
  python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph > gpurun_out/$5.log 2>&1
echo "ncu exit $?"
ncu -i gpurun_out/$5.ncu-rep --page raw --csv > gpurun_out/$5_raw.csv 2>/dev/null
ncu -i gpurun_out/$5.ncu-rep --page source --csv --print-source sass > gpurun_out/$5_sass.csv 2>/dev/null
ls -la gpurun_out/$5*
