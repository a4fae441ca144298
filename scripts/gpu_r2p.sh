#!/bin/bash
# L2 hit rate of the register gather with / without hot-row flags (C4 SAGE)
O=gpurun_out/r2p
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph"
M=gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum
for h in 0 196608; do
  WG_AGG_V2=1 WG_HOT_ROWS=$h timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"k_agg" -c 5 --log-file $O/v2_h$h.csv $B > /dev/null 2> $O/v2_h$h.err
done
timeout 900 ncu --metrics $M --clock-control none --csv -k regex:"k_agg" -c 5 --log-file $O/cp.csv $B > /dev/null 2> $O/cp.err
cd scripts && timeout 300 ncu --metrics $M --csv -c 12 --log-file ../$O/probe.csv ./l2_probe > /dev/null 2>&1
