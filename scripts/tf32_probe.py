"""Print fp32 layer errors vs the oracle (3xTF32 accuracy probe, A/B of
WG_TF32_NOHI): python scripts/tf32_probe.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from tests.test_gpu_conv_rgcn import run  # noqa: E402

for kw in (dict(policy="vertex", fi=128, fo=64, R=8, V=6000, E=60000, seed=1),
           dict(policy="edge", fi=64, fo=64, R=8, V=6000, E=60000, seed=2, self_loop=True)):
    e, _ = run(torch.float32, **kw)
    print(os.environ.get("WG_TF32_NOHI", "0"), kw["policy"], kw["fi"], {k: f"{v:.2e}" for k, v in e.items()})
