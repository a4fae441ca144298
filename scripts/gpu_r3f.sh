#!/bin/bash
# A/B: L2 persistence window on the gathers (WG_L2_PERSIST_MB=0 disables)
O=gpurun_out/r3f
mkdir -p $O
python - > $O/attrs.txt 2>&1 <<'PY'
from cuda.bindings import runtime as rt
for a in ["cudaDevAttrMaxPersistingL2CacheSize", "cudaDevAttrMaxAccessPolicyWindowSize", "cudaDevAttrL2CacheSize"]:
    print(a, rt.cudaDeviceGetAttribute(getattr(rt.cudaDeviceAttr, a), 0))
PY
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
B="python bench.py --no-cpu --no-e2e"
timeout 600 $B > $O/c4_on.json 2> $O/c4_on.err
WG_L2_PERSIST_MB=0 timeout 600 $B > $O/c4_off.json 2> $O/c4_off.err
WG_L2_PERSIST_MB=40 timeout 600 $B > $O/c4_40.json 2> $O/c4_40.err
timeout 600 $B --model gin > $O/c4gin_on.json 2> $O/c4gin_on.err
timeout 1200 python -m pytest tests/test_gpu_conv_lin.py tests/test_gpu_stack.py tests/test_gpu_fullsize.py -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
cat $O/attrs.txt; tail -2 $O/tests.log
