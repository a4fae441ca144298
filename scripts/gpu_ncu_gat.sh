#!/bin/bash
# ncu --set full: C2 GAT forward / backward edge kernels (epoch 2), C4 SAGE NT GEMMs (epoch 2)
bash scripts/ncu_full.sh C2 gat "k_gat_fwd2|k_gat_bwd_src3" 6 3 c2_gat
python scripts/ncu_summary.py gpurun_out/c2_gat.ncu-rep > gpurun_out/c2_gat.txt
bash scripts/ncu_full.sh C4 sage "k_gemm_nt_p" 4 4 c4_nt
python scripts/ncu_summary.py gpurun_out/c4_nt.ncu-rep > gpurun_out/c4_nt.txt
