#!/bin/bash
# Edge-case tests one process each (a sticky CUDA error must not hide the others) + sanitizer on E=0
mkdir -p gpurun_out/edge2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/edge2/build.log 2>&1 || { tail -30 gpurun_out/edge2/build.log; exit 1; }
python -m pytest tests/test_gpu_edge_cases.py --collect-only -q 2>/dev/null | grep '::' > gpurun_out/edge2/ids.txt
while read id; do
  timeout 300 python -m pytest "$id" -m gpu -q -x > gpurun_out/edge2/one.log 2>&1
  rc=$?; echo "$rc $id" | tee -a gpurun_out/edge2/summary.txt
  [ $rc -ne 0 ] && { echo "=== $id"; grep -E "^E " gpurun_out/edge2/one.log | head -4; } >> gpurun_out/edge2/errors.txt
done < gpurun_out/edge2/ids.txt
CUDA_LAUNCH_BLOCKING=1 timeout 600 compute-sanitizer --print-limit 5 python -m pytest "tests/test_gpu_edge_cases.py::test_no_edges_lin[dtype0-gcn]" -q -x > gpurun_out/edge2/san_gcn.log 2>&1
grep -m 20 -E "Invalid|at 0x|by thread|Address|k_[a-z_]+" gpurun_out/edge2/san_gcn.log | head -30
CUDA_LAUNCH_BLOCKING=1 timeout 600 compute-sanitizer --print-limit 5 python -m pytest "tests/test_gpu_edge_cases.py::test_star_lin[0-star_in-gcn]" -q -x > gpurun_out/edge2/san_star.log 2>&1
grep -m 20 -E "Invalid|at 0x|by thread|Address|k_[a-z_]+" gpurun_out/edge2/san_star.log | head -30
