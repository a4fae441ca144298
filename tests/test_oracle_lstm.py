"""SAGE-LSTM oracle (reading Q26) pinned by torch.nn.LSTM in
fp64 (a library routine run per vertex on its neighbour sequence in edge-id
order) and by autograd through it; special cases: an isolated vertex has
h_N = 0; a one-neighbour vertex has the closed form h = s(z_o) tanh(s(z_i) tanh(z_g))."""
import numpy as np
import pytest
import torch

import oracle
import synth


def lstm_ref(src, dst, V, x, Ws, Wn, b, Wih, Whh, bl):
    fi = x.shape[1]
    t = {k: torch.tensor(v, requires_grad=True) for k, v in
         dict(x=x, Ws=Ws, Wn=Wn, b=b, Wih=Wih, Whh=Whh, bl=bl).items()}
    cell = torch.nn.LSTM(fi, fi, batch_first=True).double()
    hs = []
    for v in range(V):
        eids = np.nonzero(dst == v)[0]              # edge-id order
        if len(eids) == 0:
            hs.append(torch.zeros(fi, dtype=torch.float64))
            continue
        seq = t["x"][torch.from_numpy(src[eids].astype(np.int64))][None]
        _, (h, _) = torch.func.functional_call(
            cell, {"weight_ih_l0": t["Wih"].T, "weight_hh_l0": t["Whh"].T, "bias_ih_l0": t["bl"],
                   "bias_hh_l0": torch.zeros_like(t["bl"])}, (seq,))
        hs.append(h[0, 0])
    hN = torch.stack(hs)
    y = t["b"] + t["x"] @ t["Ws"] + hN @ t["Wn"]
    return t, y, hN


@pytest.mark.parametrize("seed", [0, 1])
def test_lstm_forward_backward_vs_torch(seed):
    V, E, fi, fo = 30, 120, 5, 4
    src, dst, _ = synth.make_graph(V, E, seed=seed + 40, alpha=0.7)
    r = np.random.default_rng(seed)
    x = r.standard_normal((V, fi))
    Ws, Wn, b = r.standard_normal((fi, fo)) * 0.5, r.standard_normal((fi, fo)) * 0.5, r.standard_normal(fo)
    Wih, Whh, bl = r.standard_normal((fi, 4 * fi)) * 0.5, r.standard_normal((fi, 4 * fi)) * 0.5, r.standard_normal(4 * fi)
    t, y, hN = lstm_ref(src, dst, V, x, Ws, Wn, b, Wih, Whh, bl)
    yo, ho = oracle.sage_lstm_forward(src, dst, V, x, Ws, Wn, b, Wih, Whh, bl, return_h=True)
    np.testing.assert_allclose(yo, y.detach().numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(ho, hN.detach().numpy(), rtol=1e-11, atol=1e-11)
    dy = r.standard_normal((V, fo))
    y.backward(torch.tensor(dy))
    got = oracle.sage_lstm_backward(src, dst, V, x, Ws, Wn, Wih, Whh, bl, dy)
    for g, k in zip(got, ("x", "Ws", "Wn", "b", "Wih", "Whh", "bl")):
        np.testing.assert_allclose(g, t[k].grad.numpy(), rtol=1e-10, atol=1e-10, err_msg=k)
    # dy supported on a row subset: exact gradients of that dy
    rows = np.array([0, 5, 9, 17])
    dyz = np.zeros_like(dy)
    dyz[rows] = dy[rows]
    full = oracle.sage_lstm_backward(src, dst, V, x, Ws, Wn, Wih, Whh, bl, dyz)
    part = oracle.sage_lstm_backward(src, dst, V, x, Ws, Wn, Wih, Whh, bl, dy, dy_rows=rows)
    for a, c in zip(full, part):
        np.testing.assert_allclose(a, c, rtol=1e-12, atol=1e-12)


def test_lstm_special_cases():
    fi = 3
    r = np.random.default_rng(5)
    Wih, Whh, bl = r.standard_normal((fi, 4 * fi)), r.standard_normal((fi, 4 * fi)), r.standard_normal(4 * fi)
    x = r.standard_normal((3, fi))
    src, dst = np.array([1], np.int32), np.array([0], np.int32)   # vertex 0: one neighbour; 1, 2 isolated
    y, h = oracle.sage_lstm_forward(src, dst, 3, x, np.zeros((fi, fi)), np.eye(fi), None, Wih, Whh, bl, return_h=True)
    z = x[1] @ Wih + bl
    s = lambda a: 1 / (1 + np.exp(-a))   # noqa: E731
    hc = s(z[3 * fi:]) * np.tanh(s(z[:fi]) * np.tanh(z[2 * fi:3 * fi]))
    np.testing.assert_allclose(h[0], hc, rtol=1e-13)
    np.testing.assert_allclose(y[0], hc, rtol=1e-13)
    assert (h[1:] == 0).all() and (y[1:] == 0).all()
