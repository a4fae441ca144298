#!/bin/bash
# ncu --set full of C3 RGCN epoch-2 GEMMs (fwd Y/EDGE/self) and gather-reduce launches
bash scripts/ncu_full.sh C3 rgcn "k_gemm_nt_p" 8 4 c3_gemm
bash scripts/ncu_full.sh C3 rgcn "k_agg_cp" 9 9 c3_agg
python scripts/ncu_summary.py gpurun_out/c3_gemm.ncu-rep > gpurun_out/c3_gemm.txt
python scripts/ncu_summary.py gpurun_out/c3_agg.ncu-rep > gpurun_out/c3_agg.txt
