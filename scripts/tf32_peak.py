"""Measured TF32 tensor-core peak (torch.matmul fp32 with TF32 allowed,
8192^3, best of 10, CUDA events) -- the roofline denominator of the 3xTF32
GEMMs (three TF32 MMAs per fp32 product: effective peak = TF32 / 3)."""
import json
import sys

import torch

torch.backends.cuda.matmul.allow_tf32 = True
n = 8192
a = torch.randn(n, n, device="cuda")
b = torch.randn(n, n, device="cuda")
best = 1e9
for _ in range(12):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    torch.matmul(a, b)
    e1.record()
    torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
tf = 2 * n ** 3 / (best / 1e3) / 1e12
out = {"tf32_tflops": tf, "three_tf32_effective_tflops": tf / 3, "how": "torch.matmul fp32 allow_tf32 8192^3, best of 12",
       "gpu": torch.cuda.get_device_name()}
json.dump(out, open(sys.argv[1], "w"), indent=1)
print(out)
