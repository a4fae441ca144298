#!/bin/bash
# ncu --set full of the C2 fp32 NT GEMM (G = x W, 169K x 128 -> 256)
O=gpurun_out/r3h
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-graph --config C2 --model gat"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_gemm_nt_p" -s 3 -c 1 -o $O/nt_c2 -f $B > $O/nt_c2.log 2>&1
ncu -i $O/nt_c2.ncu-rep --page details --csv > $O/nt_c2_details.csv 2>/dev/null
ncu -i $O/nt_c2.ncu-rep --page raw --csv > $O/nt_c2_raw.csv 2>/dev/null
ncu -i $O/nt_c2.ncu-rep --page source --csv > $O/nt_c2_source.csv 2>/dev/null
tail -3 $O/nt_c2.log
