#!/bin/bash
# Round evidence (session 2): ncu launch lists (cold, serialised) of one epoch per
# config, and --set full captures of one epoch's launches of each config's
# dominant kernel class (traffic for bench.py's roofline.traffic).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu"
for cm in "C4 sage" "C3 rgcn" "C2 gat" "C4 gin"; do
  set -- $cm
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$1_$2.csv \
    $B --config $1 --model $2 > /dev/null 2> gpurun_out/launches_$1_$2.err
  echo "launches $1 $2 exit $?"
done
full() {  # config model regex count name
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$3" -c $4 -o gpurun_out/$5 -f \
    $B --config $1 --model $2 > gpurun_out/$5.log 2>&1
  echo "full $5 exit $?"
  ncu -i gpurun_out/$5.ncu-rep --page raw --csv > gpurun_out/$5_raw.csv 2>/dev/null
  python scripts/ncu_summary.py gpurun_out/$5.ncu-rep > gpurun_out/$5.txt 2>&1
  rm -f gpurun_out/$5.ncu-rep   # gpurun copies back <= 64 MiB
}
full C4 sage "k_agg_cp" 5 full_C4_sage_agg
full C4 sage "k_gemm_nt_p|k_tc_gemm" 11 full_C4_sage_gemm
full C3 rgcn "k_agg" 9 full_C3_rgcn_agg
full C2 gat "k_gat" 12 full_C2_gat
ls -la gpurun_out/; rm -rf gpurun_out/*.ncu-rep
