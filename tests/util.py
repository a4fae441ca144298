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


# ---------------------------------------------------------------------------
# ReLU decisions (DESIGN.md §2 "Kink band").  Every mask the oracle applies is
# its own, [pre > 0] on its fp64 pre-activation.  The kernel decides on its own
# rounded pre-activation, which may differ from the oracle's only where
# |pre| is below the rounding-error bound of the kernel's arithmetic path:
#   |pre_gpu - pre| <= K * u * mag,   mag = the same computation on |inputs|
# (every value the kernel stores on the way is rounded once to the conv dtype,
# unit roundoff u; fp32 accumulation error is << u at these depths; the fp32
# path is 3xTF32, ~2^-21 per product).  Elements inside that band are the kink
# band: the test input dy is chosen so that no compared value depends on the
# decision there (dy = 0 on band elements of an output ReLU; dy rows projected
# orthogonal to the W2 rows of band elements of GIN's inner ReLU), and outside
# the band the kernel's decisions must EQUAL the oracle's.
U_BAND = {torch.float32: 2.0 ** -19, torch.bfloat16: 2.0 ** -8}
K_BAND = 2.0


def kink_band(pre, mag, dtype, exact=False):
    """Elements where the kernel's ReLU decision may legitimately differ
    (empty when the inputs make every kernel operation exact: small integers)."""
    pre = np.asarray(pre, dtype=np.float64)
    if exact:
        return np.zeros(pre.shape, bool)
    if mag is None:                        # no |input| propagation available: global scale
        mag = np.full_like(pre, np.abs(pre).max() if pre.size else 0.0)
    return np.abs(pre) < K_BAND * U_BAND[dtype] * np.asarray(mag, dtype=np.float64)


def relu_dy(dy, pre, band):
    """dy zeroed on the kink band, and the oracle's dT = dy * [pre > 0]."""
    dy = np.where(band, 0.0, np.asarray(dy, dtype=np.float64))
    return dy, dy * (np.asarray(pre) > 0)


def assert_mask_agrees(y_gpu, pre, band, what="ReLU"):
    """Outside the kink band the kernel's decision [y_gpu > 0] equals [pre > 0]."""
    got = np.asarray(y_gpu) > 0
    ref = np.asarray(pre) > 0
    bad = (got != ref) & ~band
    assert not bad.any(), f"{what}: {int(bad.sum())} decisions differ outside the kink band " \
                          f"(first at {np.argwhere(bad)[:3].tolist()})"


def gin_inner_safe_dy(dy, a, band_a, W2, free=None):
    """Project each row of dy (on its free coordinates) orthogonal to the rows
    W2[j, :] of that row's inner kink-band elements j, so that
    dh[v, j] = dy[v] . W2[j] = 0 there: the inner ReLU decision at (v, j)
    then does not change any gradient.  free: [V x fo] bool, coordinates dy
    may use (default all)."""
    dy = np.array(dy, dtype=np.float64)
    for v in np.nonzero(band_a.any(1))[0]:
        J = np.nonzero(band_a[v])[0]
        S = np.nonzero(free[v])[0] if free is not None else np.arange(dy.shape[1])
        if len(S) == 0:
            continue
        A = W2[np.ix_(J, S)]
        g = dy[v, S]
        coef, *_ = np.linalg.lstsq(A.T, g, rcond=None)   # SVD: stable for near-square A
        dy[v, S] = g - A.T @ coef
    return dy


def gin_mags(z, a, W1, b1, W2, b2):
    """First-order error magnitudes of GIN's two pre-activations on the
    kernel's path: a = z W1 + b1 is computed from z rounded once to the conv
    dtype (mag_a = |z| |W1| + |b1|); y = h W2 + b2 from h = ReLU(a) rounded
    once, h inheriting a's error (mag_y = (|h| + mag_a) |W2| + |b2|).  (The
    oracle run on |x| would bound z by sum |x|, which for a hub row is
    orders of magnitude above |z| and the actual rounding.)"""
    mag_a = np.abs(z) @ np.abs(W1) + np.abs(b1)
    mag_y = (np.maximum(a, 0) + mag_a) @ np.abs(W2) + np.abs(b2)
    return mag_a, mag_y
