"""Pins for the oracle's convolutions (forward and backward).

Each oracle function (per-edge message loops, oracle/wg_oracle.c) is checked
against something other than itself:

* closed forms on the paper's worked example (Eq. (1), Fig 5a);
* the dense-adjacency matrix form of each model on graphs with <= 64 vertices
  (numpy, with multi-edge multiplicities), i.e. a different formulation;
* torch.autograd (float64) through that dense form for every backward;
* exactness on small-integer inputs (int64 dense arithmetic);
* special cases that reduce to another model or to a plain mean;
* central finite differences for the non-linear GAT softmax.
"""
import numpy as np
import pytest
import torch

import oracle
import synth


def dense_adj(src, dst, V, et=None, r=None):
    A = np.zeros((V, V))
    for s, d, t in zip(src, dst, et if et is not None else [0] * len(src)):
        if r is None or t == r:
            A[d, s] += 1
    return A


def tgraph(seed, V=40, E=260, R=1):
    src, dst, et = synth.small_graph(V, E, seed=seed, R=R, alpha=0.4)
    return src, dst, et


# ------------------------------------------------------------ worked example
def test_closed_forms(worked_example):
    ex = worked_example
    src, dst, et = np.array(ex["src"]), np.array(ex["dst"]), np.array(ex["etype"])
    cf = ex["closed_forms"]
    x = np.array(cf["x"], float)[:, None]
    y = oracle.gcn_forward(src, dst, 5, x, np.ones((1, 1)), norm="none")
    assert y[:, 0].tolist() == cf["gcn_W1"]
    W = np.array([[[1.0]], [[10.0]]])
    y = oracle.rgcn_forward(src, dst, et, 5, x, W, norm="none")
    assert y[:, 0].tolist() == cf["rgcn_Wa1_Wb10"]
    y = oracle.sage_forward(src, dst, 5, x, np.zeros((1, 1)), np.ones((1, 1)))
    # per-edge messages (1/3)*x rounds in fp64: exact up to one ulp-scale error
    np.testing.assert_allclose(y[:, 0], cf["sage_mean_Ws0_Wn1"], rtol=0, atol=1e-14)
    dx, _, _ = oracle.gcn_backward(src, dst, 5, x, np.ones((1, 1)), np.ones((5, 1)), norm="none")
    assert dx[:, 0].tolist() == cf["gcn_backward_dy1_W1_dx"]
    # GAT with a_l = a_r = 0 is the plain mean (alpha = 1/deg): same as SAGE-mean here
    y = oracle.gat_forward(src, dst, 5, x, np.ones((1, 1)), np.zeros((1, 1)), np.zeros((1, 1)), heads=1)
    assert np.allclose(y[:, 0], cf["sage_mean_Ws0_Wn1"], rtol=0, atol=1e-15)


# ------------------------------------------------------------------- GCN
@pytest.mark.parametrize("norm", ["none", "right", "both"])
def test_gcn_dense(norm):
    src, dst, _ = tgraph(1)
    V, fi, fo = 40, 7, 5
    x = synth.normal((V, fi), seed=1).astype(float)
    W = synth.normal((fi, fo), seed=2).astype(float)
    b = synth.normal((fo,), seed=3).astype(float)
    A = dense_adj(src, dst, V)
    din = np.maximum(A.sum(1), 1)
    dout = np.maximum(A.sum(0), 1)
    if norm == "both":
        Ah = A / np.sqrt(din)[:, None] / np.sqrt(dout)[None, :]
    elif norm == "right":
        Ah = A / din[:, None]
    else:
        Ah = A
    y = oracle.gcn_forward(src, dst, V, x, W, b, norm=norm)
    np.testing.assert_allclose(y, Ah @ x @ W + b, rtol=1e-12, atol=1e-12)
    # backward vs torch.autograd on the dense form
    dy = synth.normal((V, fo), seed=4).astype(float)
    tx = torch.tensor(x, requires_grad=True)
    tW = torch.tensor(W, requires_grad=True)
    tb = torch.tensor(b, requires_grad=True)
    (torch.tensor(Ah) @ tx @ tW + tb).backward(torch.tensor(dy))
    dx, dW, db = oracle.gcn_backward(src, dst, V, x, W, dy, norm=norm)
    np.testing.assert_allclose(dx, tx.grad.numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(dW, tW.grad.numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(db, tb.grad.numpy(), rtol=1e-11, atol=1e-11)


def test_gcn_rows_subset():
    src, dst, _ = tgraph(2)
    x = synth.normal((40, 6), seed=1).astype(float)
    W = synth.normal((6, 3), seed=2).astype(float)
    full = oracle.gcn_forward(src, dst, 40, x, W)
    rows = [0, 5, 17, 39]
    part = oracle.gcn_forward(src, dst, 40, x, W, rows=rows)
    np.testing.assert_array_equal(part[rows], full[rows])


# ------------------------------------------------------------------ SAGE
def test_sage_dense():
    src, dst, _ = tgraph(3)
    V, fi, fo = 40, 6, 4
    x = synth.normal((V, fi), seed=5).astype(float)
    Ws = synth.normal((fi, fo), seed=6).astype(float)
    Wn = synth.normal((fi, fo), seed=7).astype(float)
    b = synth.normal((fo,), seed=8).astype(float)
    A = dense_adj(src, dst, V)
    M = A / np.maximum(A.sum(1), 1)[:, None]
    y = oracle.sage_forward(src, dst, V, x, Ws, Wn, b)
    np.testing.assert_allclose(y, x @ Ws + M @ x @ Wn + b, rtol=1e-12, atol=1e-12)
    dy = synth.normal((V, fo), seed=9).astype(float)
    t = [torch.tensor(a, requires_grad=True) for a in (x, Ws, Wn, b)]
    (t[0] @ t[1] + torch.tensor(M) @ t[0] @ t[2] + t[3]).backward(torch.tensor(dy))
    got = oracle.sage_backward(src, dst, V, x, Ws, Wn, dy)
    for g, tt in zip(got, t):
        np.testing.assert_allclose(g, tt.grad.numpy(), rtol=1e-11, atol=1e-11)


def test_sage_special_case_mean():
    # W_s = 0, W_n = I: pure mean aggregation
    src, dst, _ = tgraph(4)
    x = synth.normal((40, 3), seed=1).astype(float)
    y = oracle.sage_forward(src, dst, 40, x, np.zeros((3, 3)), np.eye(3))
    for v in range(40):
        nb = src[dst == v]
        exp = x[nb].mean(0) if len(nb) else np.zeros(3)
        np.testing.assert_allclose(y[v], exp, rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------- GIN
@pytest.mark.parametrize("eps", [0.0, 0.25])
def test_gin_dense(eps):
    src, dst, _ = tgraph(5)
    V, fi, fo = 40, 5, 6
    x = synth.normal((V, fi), seed=10).astype(float)
    W1 = synth.normal((fi, fo), seed=11).astype(float)
    b1 = synth.normal((fo,), seed=12).astype(float)
    W2 = synth.normal((fo, fo), seed=13).astype(float)
    b2 = synth.normal((fo,), seed=14).astype(float)
    A = dense_adj(src, dst, V)
    z = (1 + eps) * x + A @ x
    ref = np.maximum(z @ W1 + b1, 0) @ W2 + b2
    np.testing.assert_allclose(oracle.gin_forward(src, dst, V, x, W1, b1, W2, b2, eps), ref, rtol=1e-12, atol=1e-12)
    dy = synth.normal((V, fo), seed=15).astype(float)
    t = [torch.tensor(a, requires_grad=True) for a in (x, W1, b1, W2, b2)]
    zz = (1 + eps) * t[0] + torch.tensor(A) @ t[0]
    (torch.relu(zz @ t[1] + t[2]) @ t[3] + t[4]).backward(torch.tensor(dy))
    got = oracle.gin_backward(src, dst, V, x, W1, b1, W2, dy, eps)
    for g, tt in zip(got, t):
        np.testing.assert_allclose(g, tt.grad.numpy(), rtol=1e-11, atol=1e-11)


def test_gin_rows_za_and_dy_rows():
    """Row-restricted forward == full forward on those rows; z and the
    pre-activation a are the dense z = (1+eps)x + A x, a = z W1 + b1; the
    dy_rows backward equals autograd with dy zeroed outside the rows (dx for
    every vertex)."""
    src, dst, _ = tgraph(8)
    V, fi, fo, eps = 40, 5, 6, 0.5
    x = synth.normal((V, fi), seed=20).astype(float)
    W1 = synth.normal((fi, fo), seed=21).astype(float)
    b1 = synth.normal((fo,), seed=22).astype(float)
    W2 = synth.normal((fo, fo), seed=23).astype(float)
    b2 = synth.normal((fo,), seed=24).astype(float)
    A = dense_adj(src, dst, V)
    rows = np.array([0, 3, 7, 11, 39])
    y, z, a = oracle.gin_forward(src, dst, V, x, W1, b1, W2, b2, eps, rows=rows, return_za=True)
    zr = (1 + eps) * x + A @ x
    np.testing.assert_allclose(z[rows], zr[rows], rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(a[rows], (zr @ W1 + b1)[rows], rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(y[rows], (np.maximum(zr @ W1 + b1, 0) @ W2 + b2)[rows], rtol=1e-12, atol=1e-12)
    dy = synth.normal((V, fo), seed=25).astype(float)
    dyz = np.zeros_like(dy)
    dyz[rows] = dy[rows]
    t = [torch.tensor(v, requires_grad=True) for v in (x, W1, b1, W2, b2)]
    zz = (1 + eps) * t[0] + torch.tensor(A) @ t[0]
    (torch.relu(zz @ t[1] + t[2]) @ t[3] + t[4]).backward(torch.tensor(dyz))
    got = oracle.gin_backward(src, dst, V, x, W1, b1, W2, dy, eps, dy_rows=rows)
    for g, tt in zip(got, t):
        np.testing.assert_allclose(g, tt.grad.numpy(), rtol=1e-11, atol=1e-11)


def test_gin_relu_derivative_at_zero():
    """Integer inputs with pre-activations exactly 0: ReLU'(0) = 0 (Q8 / SURVEY
    c3), as torch.relu's backward."""
    src, dst, _ = tgraph(9)
    V, fi, fo = 40, 3, 4
    x = synth.small_ints((V, fi), seed=30).astype(float)
    W1 = synth.small_ints((fi, fo), seed=31).astype(float)
    b1 = np.zeros(fo)
    W2 = synth.small_ints((fo, fo), seed=32).astype(float)
    _, _, a = oracle.gin_forward(src, dst, V, x, W1, b1, W2, np.zeros(fo), return_za=True)
    assert (a == 0).any()          # the kink is hit exactly
    dy = synth.small_ints((V, fo), seed=33).astype(float)
    A = dense_adj(src, dst, V)
    t = [torch.tensor(v, requires_grad=True) for v in (x, W1, b1, W2)]
    zz = t[0] + torch.tensor(A) @ t[0]
    (torch.relu(zz @ t[1] + t[2]) @ t[3]).backward(torch.tensor(dy))
    got = oracle.gin_backward(src, dst, V, x, W1, b1, W2, dy)
    for g, tt in zip((got[0], got[1], got[2], got[3]), t):
        np.testing.assert_array_equal(g, tt.grad.numpy())


def test_gin_special_case_neighbour_sum():
    # eps = -1, W1 = W2 = I, b = 0, x >= 0: pure neighbour sum
    src, dst, _ = tgraph(6)
    x = synth.make_features(40, 4, seed=3, dist="uniform01").astype(float)
    y = oracle.gin_forward(src, dst, 40, x, np.eye(4), np.zeros(4), np.eye(4), np.zeros(4), eps=-1.0)
    np.testing.assert_allclose(y, dense_adj(src, dst, 40) @ x, rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------ RGCN
@pytest.mark.parametrize("norm,self_loop,bias", [("none", False, False), ("right", True, True)])
def test_rgcn_dense(norm, self_loop, bias):
    R = 3
    src, dst, et = tgraph(7, R=R)
    V, fi, fo = 40, 4, 5
    x = synth.normal((V, fi), seed=16).astype(float)
    W = synth.normal((R, fi, fo), seed=17).astype(float)
    W0 = synth.normal((fi, fo), seed=18).astype(float) if self_loop else None
    b = synth.normal((fo,), seed=19).astype(float) if bias else None
    ref = np.zeros((V, fo))
    As = []
    for r in range(R):
        Ar = dense_adj(src, dst, V, et, r)
        if norm == "right":
            Ar = Ar / np.maximum(Ar.sum(1), 1)[:, None]
        As.append(Ar)
        ref += Ar @ x @ W[r]
    if self_loop:
        ref += x @ W0
    if bias:
        ref += b
    y = oracle.rgcn_forward(src, dst, et, V, x, W, W0, b, norm=norm)
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)
    dy = synth.normal((V, fo), seed=20).astype(float)
    tx, tW = torch.tensor(x, requires_grad=True), torch.tensor(W, requires_grad=True)
    out = sum(torch.tensor(As[r]) @ tx @ tW[r] for r in range(R))
    tW0 = None
    if self_loop:
        tW0 = torch.tensor(W0, requires_grad=True)
        out = out + tx @ tW0
    out.backward(torch.tensor(dy))
    dx, dW, dW0, db = oracle.rgcn_backward(src, dst, et, V, x, W, dy, W0, norm=norm)
    np.testing.assert_allclose(dx, tx.grad.numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(dW, tW.grad.numpy(), rtol=1e-11, atol=1e-11)
    if self_loop:
        np.testing.assert_allclose(dW0, tW0.grad.numpy(), rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(db, dy.sum(0), rtol=1e-12, atol=1e-12)


def test_rgcn_single_relation_is_gcn_none():
    src, dst, _ = tgraph(8)
    x = synth.normal((40, 5), seed=1).astype(float)
    W = synth.normal((5, 3), seed=2).astype(float)
    a = oracle.rgcn_forward(src, dst, None, 40, x, W[None])
    b = oracle.gcn_forward(src, dst, 40, x, W, norm="none")
    np.testing.assert_array_equal(a, b)


# ------------------------------------------------------------------- GAT
def dense_gat(A, x, W, al, ar, b, H, concat, slope=0.2, lib=np):
    fo = W.shape[1] // H
    outs = []
    for k in range(H):
        g = x @ W[:, k * fo:(k + 1) * fo]
        el, er = g @ al[k], g @ ar[k]
        t = er[:, None] + el[None, :]
        l = lib.where(t > 0, t, slope * t)
        mask = A > 0
        lm = lib.where(mask, l, lib.full_like(l, -1e300))
        m = lm.max(1, keepdims=True) if lib is np else lm.max(1, keepdim=True).values
        w = A * lib.exp(lm - m)
        den = w.sum(1, keepdims=True) if lib is np else w.sum(1, keepdim=True)
        den = lib.where(den > 0, den, lib.ones_like(den))
        outs.append((w / den) @ g)
    y = lib.concatenate(outs, 1) if (concat and lib is np) else (torch.cat(outs, 1) if concat else sum(outs) / H)
    return y + b


@pytest.mark.parametrize("H,concat", [(1, True), (3, True), (2, False)])
def test_gat_dense(H, concat):
    src, dst, _ = tgraph(9)
    V, fi, fo = 40, 5, 4
    x = synth.normal((V, fi), seed=21).astype(float)
    W = synth.normal((fi, H * fo), seed=22).astype(float)
    al = synth.normal((H, fo), seed=23).astype(float)
    ar = synth.normal((H, fo), seed=24).astype(float)
    FO = H * fo if concat else fo
    b = synth.normal((FO,), seed=25).astype(float)
    A = dense_adj(src, dst, V)
    y = oracle.gat_forward(src, dst, V, x, W, al, ar, b, heads=H, concat=concat)
    np.testing.assert_allclose(y, dense_gat(A, x, W, al, ar, b, H, concat), rtol=1e-11, atol=1e-11)
    dy = synth.normal((V, FO), seed=26).astype(float)
    t = [torch.tensor(a, requires_grad=True) for a in (x, W, al, ar, b)]
    dense_gat(torch.tensor(A), *t, H, concat, lib=torch).backward(torch.tensor(dy))
    got = oracle.gat_backward(src, dst, V, x, W, al, ar, dy, heads=H, concat=concat)
    for g, tt in zip(got, t):
        np.testing.assert_allclose(g, tt.grad.numpy(), rtol=1e-10, atol=1e-10)


def test_gat_finite_difference():
    src, dst, _ = tgraph(10, V=20, E=90)
    V, fi, fo, H = 20, 3, 2, 2
    x = synth.normal((V, fi), seed=30).astype(float)
    W = synth.normal((fi, H * fo), seed=31).astype(float)
    al = synth.normal((H, fo), seed=32).astype(float)
    ar = synth.normal((H, fo), seed=33).astype(float)
    dy = synth.normal((V, H * fo), seed=34).astype(float)
    _, dW, dal, _, _ = oracle.gat_backward(src, dst, V, x, W, al, ar, dy, heads=H)
    h = 1e-6
    for (i, j) in [(0, 0), (2, 3), (1, 2)]:
        Wp, Wm = W.copy(), W.copy()
        Wp[i, j] += h
        Wm[i, j] -= h
        fd = ((oracle.gat_forward(src, dst, V, x, Wp, al, ar, heads=H) * dy).sum()
              - (oracle.gat_forward(src, dst, V, x, Wm, al, ar, heads=H) * dy).sum()) / (2 * h)
        assert abs(fd - dW[i, j]) < 1e-6 * max(1, abs(fd))
    alp, alm = al.copy(), al.copy()
    alp[1, 0] += h
    alm[1, 0] -= h
    fd = ((oracle.gat_forward(src, dst, V, x, W, alp, ar, heads=H) * dy).sum()
          - (oracle.gat_forward(src, dst, V, x, W, alm, ar, heads=H) * dy).sum()) / (2 * h)
    assert abs(fd - dal[1, 0]) < 1e-6 * max(1, abs(fd))


# ------------------------------------------------------ integer exactness
def test_integer_exactness():
    src, dst, et = tgraph(11, R=2)
    V = 40
    x = synth.small_ints((V, 6), seed=1)
    W = synth.small_ints((6, 4), seed=2)
    A = dense_adj(src, dst, V).astype(np.int64)
    y = oracle.gcn_forward(src, dst, V, x, W, norm="none")
    exact = A @ x.astype(np.int64) @ W.astype(np.int64)
    assert (y == exact).all()
    Wr = synth.small_ints((2, 6, 4), seed=3)
    y = oracle.rgcn_forward(src, dst, et, V, x, Wr)
    exact = sum(dense_adj(src, dst, V, et, r).astype(np.int64) @ x.astype(np.int64) @ Wr[r].astype(np.int64)
                for r in range(2))
    assert (y == exact).all()


def test_dw_probe_matches_backward():
    src, dst, _ = tgraph(12)
    V, fi, fo = 40, 5, 3
    x = synth.normal((V, fi), seed=40).astype(float)
    W = synth.normal((fi, fo), seed=41).astype(float)
    dy = synth.normal((V, fo), seed=42).astype(float)
    u = synth.normal((fi,), seed=43).astype(float)
    v = synth.normal((fo,), seed=44).astype(float)
    _, dW, _ = oracle.gcn_backward(src, dst, V, x, W, dy, norm="none")
    assert abs(oracle.dw_probe(src, dst, x, dy, u, v) - u @ dW @ v) < 1e-10


# ------------------------------------------------------- degenerate graphs
def test_no_edges_closed_forms():
    # E = 0: every neighbourhood is empty, so each model reduces to its
    # per-vertex terms (Eq. (1) with an empty sum)
    V, fi, fo, R, H = 12, 5, 4, 3, 2
    e = np.zeros(0, np.int32)
    x = synth.normal((V, fi), seed=40).astype(float)
    W = synth.normal((fi, fo), seed=41).astype(float)
    W2 = synth.normal((fo, fo), seed=42).astype(float)
    b = synth.normal((fo,), seed=43).astype(float)
    b2 = synth.normal((fo,), seed=44).astype(float)
    for norm in ("none", "right", "both"):
        np.testing.assert_array_equal(oracle.gcn_forward(e, e, V, x, W, b, norm=norm), np.tile(b, (V, 1)))
    np.testing.assert_allclose(oracle.sage_forward(e, e, V, x, W, W, b),
                               x @ W + b, rtol=1e-13, atol=1e-13)
    np.testing.assert_allclose(oracle.gin_forward(e, e, V, x, W, b, W2, b2, 0.5),
                               np.maximum(1.5 * x @ W + b, 0) @ W2 + b2, rtol=1e-13, atol=1e-13)
    Wr = synth.normal((R, fi, fo), seed=45).astype(float)
    np.testing.assert_allclose(oracle.rgcn_forward(e, e, e, V, x, Wr, W, b), x @ W + b, rtol=1e-13, atol=1e-13)
    Wg = synth.normal((fi, H * fo), seed=46).astype(float)
    al, ar = synth.normal((H, fo), seed=47).astype(float), synth.normal((H, fo), seed=48).astype(float)
    bg = synth.normal((H * fo,), seed=49).astype(float)
    np.testing.assert_array_equal(oracle.gat_forward(e, e, V, x, Wg, al, ar, bg, heads=H), np.tile(bg, (V, 1)))
    # neighbour-path weight gradients vanish
    dy = synth.normal((V, fo), seed=50).astype(float)
    assert not np.any(oracle.gcn_backward(e, e, V, x, W, dy, norm="both")[1])
    assert not np.any(oracle.sage_backward(e, e, V, x, W, W, dy)[2])
    assert not np.any(oracle.rgcn_backward(e, e, e, V, x, Wr, dy, W)[1])


def test_gat_equal_logits_attention_gradient_vanishes():
    # every in-neighbourhood is copies of one source: each softmax is over
    # equal logits, y does not depend on a_l / a_r, so da_l = da_r = 0
    V, fi, fo, H = 20, 4, 3, 2
    src = np.zeros(90, np.int32)
    dst = synth.make_graph(V, 90, seed=3)[1]
    x = synth.normal((V, fi), seed=51).astype(float)
    W = synth.normal((fi, H * fo), seed=52).astype(float)
    al, ar = synth.normal((H, fo), seed=53).astype(float), synth.normal((H, fo), seed=54).astype(float)
    dy = synth.normal((V, H * fo), seed=55).astype(float)
    y = oracle.gat_forward(src, dst, V, x, W, al, ar, heads=H)
    has = np.bincount(dst, minlength=V) > 0
    np.testing.assert_allclose(y[has], np.tile(x[0] @ W, (has.sum(), 1)), rtol=1e-13, atol=1e-13)
    dx, dW, dal, dar, _ = oracle.gat_backward(src, dst, V, x, W, al, ar, dy, heads=H)
    assert np.abs(dal).max() < 1e-12 * np.abs(dW).max() and np.abs(dar).max() < 1e-12 * np.abs(dW).max()
