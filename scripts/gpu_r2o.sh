#!/bin/bash
# register gather (k_agg) with hot-row L2 policy vs the cp.async ring
O=gpurun_out/r2o
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B > $O/c4_cp.json 2> $O/c4_cp.err
WG_AGG_V2=1 timeout 600 $B > $O/c4_v2u4.json 2> $O/c4_v2u4.err
WG_AGG_V2=1 WG_AGG_U=8 timeout 600 $B > $O/c4_v2u8.json 2> $O/c4_v2u8.err
WG_AGG_V2=1 WG_HOT_ROWS=0 timeout 600 $B > $O/c4_v2u4_h0.json 2> $O/c4_v2u4_h0.err
WG_AGG_V2=1 WG_HOT_ROWS=393216 timeout 600 $B > $O/c4_v2u4_h393k.json 2> $O/c4_v2u4_h393k.err
WG_AGG_V2=1 WG_AGG_NARROW=1 timeout 900 $B --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/c5_v2.json 2> $O/c5_v2.err
WG_AGG_V2=1 WG_AGG_U=8 WG_AGG_NARROW=1 timeout 900 $B --config C5 --rank-slice 8 --steps 5 --warmup 3 > $O/c5_v2u8.json 2> $O/c5_v2u8.err
WG_AGG_V2=1 timeout 600 $B --config C3 --model rgcn > $O/c3_v2.json 2> $O/c3_v2.err
WG_AGG_V2=1 WG_AGG_U=8 timeout 1200 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_fullsize.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
tail -3 $O/tests.log
