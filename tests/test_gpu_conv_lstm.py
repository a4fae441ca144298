"""SAGE-LSTM (the paper's fifth model) forward + backward
through the C ABI == the oracle (fp64 BPTT per vertex, pinned against
torch.nn.LSTM in tests/test_oracle_lstm.py).  The degree-ordered prefix
batching (uniq(dst-degree) = min & uniq(dst) = K gTasks) must
give the per-vertex sequential result: fp32 (3xTF32) within 1e-4."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import assert_mask_agrees, f64, kink_band, rel_err, relu_dy

pytestmark = pytest.mark.gpu


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def run(V, E, fi, fo, seed, alpha=0.7, relu=False, need_dx=True, edges=None):
    m = wg()
    src, dst = edges if edges is not None else synth.make_graph(V, E, seed=seed, alpha=alpha)[:2]
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V)
    conv = m.Conv(g, "sage_lstm", fi, fo, dtype=torch.float32, fuse_relu=relu, need_dx=need_dx)
    params = m.init_params("sage_lstm", fi, fo, seed=seed)
    gen = torch.Generator(device="cuda").manual_seed(seed)
    params = {k: v + 0.05 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    x = torch.from_numpy(synth.make_features(V, fi, seed=seed + 1))
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    P = {k: f64(v) for k, v in params.items()}
    pre = oracle.sage_lstm_forward(src, dst, V, f64(x), P["W_self"], P["W"], P["bias"], P["Wih"], P["Whh"], P["bl"])
    dy = synth.normal((V, fo), seed=seed + 2, std=0.2).astype(np.float64)
    yo = pre
    if relu:
        band = kink_band(pre, None, torch.float32)
        assert_mask_agrees(f64(y), pre, band)
        dy, _ = relu_dy(dy, pre, band)
        yo = np.maximum(pre, 0)
    dyt = torch.from_numpy(dy).float()
    dx, grads = conv.backward_raw(m.pad_to(dyt.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dT = f64(dyt) * (pre > 0) if relu else f64(dyt)
    go = oracle.sage_lstm_backward(src, dst, V, f64(x), P["W_self"], P["W"], P["Wih"], P["Whh"], P["bl"], dT)
    errs = {"y": rel_err(f64(y), yo)}
    if need_dx:
        errs["dx"] = rel_err(f64(dx), go[0])
    for k, ref in zip(("W_self", "W", "bias", "Wih", "Whh", "bl"), go[1:]):
        errs["d" + k] = rel_err(f64(grads[k]), ref)
    return errs, conv


@pytest.mark.parametrize("fi,fo", [(16, 8), (32, 24), (64, 40)])
def test_sage_lstm_parity(fi, fo):
    errs, _ = run(800, 6000, fi, fo, seed=fi)
    assert max(errs.values()) <= 1e-4, errs


def test_sage_lstm_relu_isolated_split_rows():
    # isolated vertices (V beyond the edges' range) and a small E_max (SPLIT rows on the transposed gather)
    m = wg()
    V, E = 2000, 9000
    src, dst, _ = synth.make_graph(1500, E, seed=7, alpha=0.85)
    errs, conv = run(V, E, 24, 16, seed=8, relu=True, edges=(src, dst))
    assert max(errs.values()) <= 1e-4, errs


def test_sage_lstm_need_dx_false_and_unsupported():
    errs, _ = run(500, 3000, 16, 16, seed=11, need_dx=False)
    assert max(errs.values()) <= 1e-4, errs
    m = wg()
    src, dst, _ = synth.make_graph(100, 500, seed=1)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=100)
    with pytest.raises(m.WGError):
        m.Conv(g, "sage_lstm", 16, 16, dtype=torch.bfloat16)
