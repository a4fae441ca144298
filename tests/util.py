"""Shared test helpers: run the CUDA path through the C-ABI binding and the
oracle on the same seeded inputs, compare with the Q15 metric."""
import numpy as np
import torch

TOL = {torch.float32: 1e-4, torch.bfloat16: 2e-2}


def rel_err(got, ref):
    """Q15: max_i |g_i - o_i| / max(max_i |o_i|, 1e-30)."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    if ref.size == 0:
        return 0.0
    return float(np.abs(got - ref).max() / max(np.abs(ref).max(), 1e-30))


def q(t, dtype):
    """Round an fp32 tensor to the conv dtype (RNE) and return float64 numpy (exact)."""
    return t.to(dtype).to(torch.float64).cpu().numpy()


def f64(t):
    return t.to(torch.float64).cpu().numpy()
