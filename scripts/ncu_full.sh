#!/bin/bash
# ncu --set full capture: bash scripts/ncu_full.sh <config> <model> <kernel regex> <skip> <count> <name>
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$3" -s $4 -c $5 -o gpurun_out/$6 -f \
  python bench.py --config $1 --model $2 --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/$6.log 2>&1
echo "ncu exit $?"; tail -n 3 gpurun_out/$6.log; ls -la gpurun_out/$6.ncu-rep
