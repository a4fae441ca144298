"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same synthetic recipe, graph, plans and kernels).

Outputs the oracle can compute one by one are compared on sampled rows (random
rows + every SPLIT row + the highest-degree rows); weight gradients on
sampled entries dW[i, j] = sum_e c_e x[s_e, i] dy[d_e, j] (the definition,
contracted: oracle.dw_probe on single columns); the partition on sampled
destination tiles (a gTask never spans tiles, so a tile's tables are the
oracle's tables for that tile's in-edges)."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import f64, q

pytestmark = pytest.mark.gpu

RNG = np.random.default_rng(2024)


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def sampled_err(got, ref, rows):
    a, b = got[rows], ref[rows]
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))


def sample_rows(deg, E_max, n=2000):
    V = deg.shape[0]
    rows = set(RNG.choice(V, size=min(n, V), replace=False).tolist())
    rows |= set(np.nonzero(deg > E_max)[0].tolist())
    rows |= set(np.argsort(deg)[-50:].tolist())
    return np.array(sorted(rows))


def entry_probe(src, dst, coef, x, dy, i, j):
    return oracle.dw_probe(src, dst, x[:, i:i + 1], dy[:, j:j + 1], np.ones(1), np.ones(1), coef)


@pytest.fixture(scope="module")
def c4():
    import bench
    c = synth.CONFIGS["C4"]
    src, dst, _, x, labels = bench.make_inputs(c, "sage")
    m = wg()
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    return c, src, dst, g


def test_c4_partition_sampled_tiles(c4):
    c, src, dst, g = c4
    perm, tasks, _ = g.export()
    T = g.T
    tiles = RNG.choice(-(-c.V // T), size=40, replace=False)
    tiles = np.concatenate([tiles, [int(np.argmax(np.bincount(dst, minlength=c.V))) // T]])
    key_tile = dst // T
    for t in tiles:
        eids = np.nonzero(key_tile == t)[0]                   # in generation (edge id) order
        p_o, t_o = oracle.partition(dst[eids], src[eids], T=T, E_max=g.E_max)
        sel = tasks["tile"] == t
        tk = tasks[sel]
        off = tk["e_begin"][0] if len(tk) else 0
        np.testing.assert_array_equal(perm[off:off + len(eids)], eids[p_o])
        for k in ("type", "d_lo", "d_hi", "flags", "n_uniq_src"):
            np.testing.assert_array_equal(tk[k], t_o[k])
        np.testing.assert_array_equal(tk["e_begin"] - off, t_o["e_begin"])
        np.testing.assert_array_equal(tk["e_end"] - off, t_o["e_end"])


@pytest.mark.parametrize("layer", [0, 1, 2])
def test_c4_sage_layer_sampled(c4, layer):
    c, src, dst, g = c4
    m = wg()
    fi, fo = c.dims[layer], c.dims[layer + 1]
    relu = layer < 2
    dt = torch.bfloat16
    conv = m.Conv(g, "sage", fi, fo, dtype=dt, fuse_relu=relu, need_dx=True)
    params = m.init_params("sage", fi, fo, seed=layer)
    gen = torch.Generator(device="cuda").manual_seed(layer)
    params = {k: v + 0.05 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=500 + layer)).to(dt)
    dy = torch.from_numpy(synth.normal((c.V, fo), seed=600 + layer, std=0.05)).to(dt)
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    W = {k: q(v, dt) for k, v in params.items()}
    xo, yg = f64(x), f64(y)
    deg = np.bincount(dst, minlength=c.V)
    rows = sample_rows(deg, g.E_max)
    yo = oracle.sage_forward(src, dst, c.V, xo, W["W_self"], W["W"], W["bias"], rows=rows)
    if relu:
        yo = np.maximum(yo, 0)
    assert sampled_err(yg, yo, rows) <= 2e-2
    dyo = f64(dy) * (yg > 0) if relu else f64(dy)
    outdeg = np.bincount(src, minlength=c.V)
    rows_t = sample_rows(outdeg, g.E_max)
    dxo, _, _, _ = oracle.sage_backward(src, dst, c.V, xo, W["W_self"], W["W"], dyo, rows=rows_t, grads=False)
    assert sampled_err(f64(dx), dxo, rows_t) <= 2e-2
    coef = 1.0 / np.maximum(deg[dst], 1)
    idx = np.arange(c.V, dtype=np.int32)
    gWn, gWs = f64(grads["W"]), f64(grads["W_self"])
    errs = []
    for (i, j) in [(0, 0), (fi - 1, fo - 1), (fi // 2, fo // 3), (3 % fi, (7 * fo) // 8)]:
        on = entry_probe(src, dst, coef, xo, dyo, i, j)
        os_ = entry_probe(idx, idx, None, xo, dyo, i, j)
        errs.append((abs(gWn[i, j] - on), abs(on), abs(gWs[i, j] - os_), abs(os_)))
    scale_n = max(np.abs(gWn).max(), 1e-30)
    scale_s = max(np.abs(gWs).max(), 1e-30)
    assert all(a / scale_n <= 2e-2 and c_ / scale_s <= 2e-2 for a, _, c_, _ in errs), errs
    db = f64(grads["bias"])
    np.testing.assert_allclose(db, dyo.sum(0), rtol=0, atol=2e-2 * max(1e-30, np.abs(dyo.sum(0)).max()))


def test_c1_gcn_full_exact():
    c = synth.CONFIGS["C1"]
    m = wg()
    src, dst, _ = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha, symmetric=True)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    x = torch.from_numpy(synth.make_features(c.V, c.dims[0], seed=c.seed * 16 + 2, dist="bernoulli", p=c.xp))
    for layer in range(2):
        fi, fo = c.dims[layer], c.dims[layer + 1]
        conv = m.Conv(g, "gcn", fi, fo, dtype=torch.float32, fuse_relu=layer == 0)
        params = m.init_params("gcn", fi, fo, seed=layer)
        xd = m.pad_to(x.cuda())
        y, saved = conv.forward_raw(xd, params)
        dy = torch.from_numpy(synth.normal((c.V, fo), seed=layer, std=0.3))
        dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
        torch.cuda.synchronize()
        Wo, bo = f64(params["W"]), f64(params["bias"])
        yo = oracle.gcn_forward(src, dst, c.V, f64(x), Wo, bo)
        dyo = f64(dy)
        if layer == 0:
            yo = np.maximum(yo, 0)
            dyo = dyo * (f64(y) > 0)
        dxo, dWo, dbo = oracle.gcn_backward(src, dst, c.V, f64(x), Wo, dyo)
        for a, b in ((f64(y), yo), (f64(dx), dxo), (f64(grads["W"]), dWo), (f64(grads["bias"]), dbo)):
            assert np.abs(a - b).max() / max(np.abs(b).max(), 1e-30) <= 1e-4
        x = y.detach().cpu().float()


def test_c2_gat_layer1_full():
    c = synth.CONFIGS["C2"]
    m = wg()
    src, dst, _ = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    H, fi, fo = c.heads, c.dims[0], c.dims[1]
    conv = m.Conv(g, "gat", fi, fo, dtype=torch.float32, heads=H, concat=True, fuse_relu=True)
    params = m.init_params("gat", fi, fo, heads=H, seed=1)
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=c.seed * 16 + 2))
    dy = torch.from_numpy(synth.normal((c.V, H * fo), seed=3, std=0.1))
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    P = {k: f64(v) for k, v in params.items()}
    yo = np.maximum(oracle.gat_forward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], P["bias"], heads=H), 0)
    dyo = f64(dy) * (f64(y) > 0)
    dxo, dWo, dal, dar, dbo = oracle.gat_backward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], dyo, heads=H)
    for a, b in ((f64(y), yo), (f64(dx), dxo), (f64(grads["W"]), dWo), (f64(grads["attn_l"]), dal),
                 (f64(grads["attn_r"]), dar), (f64(grads["bias"]), dbo)):
        assert np.abs(a - b).max() / max(np.abs(b).max(), 1e-30) <= 1e-4


def test_c3_rgcn_layer1_sampled():
    c = synth.CONFIGS["C3"]
    m = wg()
    src, dst, et = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha, R=c.R, zipf_s=c.zipf_s)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V,
                etype=torch.from_numpy(et).cuda(), num_types=c.R)
    fi, fo = c.dims[0], c.dims[1]
    conv = m.Conv(g, "rgcn", fi, fo, dtype=torch.float32, fuse_relu=True, bias=True)
    params = m.init_params("rgcn", fi, fo, R=c.R, bias=True, seed=2)
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=c.seed * 16 + 2))
    dy = torch.from_numpy(synth.normal((c.V, fo), seed=4, std=0.1))
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    W, b = f64(params["W"]), f64(params["bias"])
    deg = np.bincount(dst, minlength=c.V)
    rows = sample_rows(deg, g.E_max, 1000)
    yo = np.maximum(oracle.rgcn_forward(src, dst, et, c.V, f64(x), W, None, b, rows=rows), 0)
    assert sampled_err(f64(y), yo, rows) <= 1e-4
    dyo = f64(dy) * (f64(y) > 0)
    rows_t = sample_rows(np.bincount(src, minlength=c.V), g.E_max, 1000)
    dxo, _, _, _ = oracle.rgcn_backward(src, dst, et, c.V, f64(x), W, dyo, rows=rows_t, grads=False)
    assert sampled_err(f64(dx), dxo, rows_t) <= 1e-4
    gW = f64(grads["W"])
    scale = np.abs(gW).max()
    xo = f64(x)
    for r in (0, 1, 5, c.R - 1):
        sel = et == r
        for (i, j) in [(0, 0), (fi - 1, fo - 1), (17, 33)]:
            ref = entry_probe(src[sel], dst[sel], None, xo, dyo, i, j)
            assert abs(gW[r, i, j] - ref) <= 1e-4 * scale, (r, i, j, gW[r, i, j], ref)


def test_c5_rank_slice_layer1_sampled():
    """C5 (111 M V, 1.6 B E) at full size, in the launch configuration bench.py
    --rank-slice 8 times: rank 0's block of the 8-way 1-D partition (its in- and
    out-edges only).  Layer-1 SAGE forward of owned rows is exact on the slice
    (every in-edge of an owned row is present, degrees of owned rows are
    global), so sampled rows are compared with the oracle on their induced
    in-neighbourhood.  The EDGE plan gathers the replicated input table
    itself; the VERTEX plan would gather Y = x W rows that other ranks own
    (filled by the all-gather a single process does not run)."""
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import partition_1d
    c = synth.CONFIGS["C5"]
    m = wg()
    block, bounds = partition_1d(c.V, 8)
    vb, ve = bounds[0]
    src, dst = synth.make_graph_slice(c.V, c.E, vb, ve, seed=c.seed * 16, alpha=c.alpha)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V, v_begin=vb, v_end=ve)
    dt = torch.bfloat16
    fi, fo = c.dims[0], c.dims[1]
    x = m.padded(c.V, fi, dt)
    gen = torch.Generator(device="cuda").manual_seed(5)
    for r0 in range(0, c.V, 1 << 22):
        r1 = min(c.V, r0 + (1 << 22))
        x[r0:r1].copy_(torch.randn((r1 - r0, fi), generator=gen, device="cuda"))
    conv = m.Conv(g, "sage", fi, fo, dtype=dt, fuse_relu=True, need_dx=False, policy="edge")
    params = m.init_params("sage", fi, fo, seed=7)
    y, saved = conv.forward_raw(x, params)
    torch.cuda.synchronize()
    own = (dst >= vb) & (dst < ve)
    s_own, d_own = src[own], dst[own]
    deg = np.bincount(d_own - vb, minlength=ve - vb)
    rows = set((RNG.choice(ve - vb, size=1000, replace=False) + vb).tolist())
    rows |= set((np.argsort(deg)[-20:] + vb).tolist())
    rows = np.array(sorted(rows))
    sel = np.isin(d_own, rows)
    s_r, d_r = s_own[sel], d_own[sel]
    U = np.unique(np.concatenate([rows, s_r]))
    remap = lambda a: np.searchsorted(U, a).astype(np.int32)  # noqa: E731
    xs = f64(x[torch.from_numpy(U).cuda()])
    W = {k: q(v, dt) for k, v in params.items()}
    yo = np.maximum(oracle.sage_forward(remap(s_r), remap(d_r), len(U), xs, W["W_self"], W["W"], W["bias"],
                                        rows=remap(rows)), 0)
    yg = f64(y)[rows - vb]
    ref = yo[remap(rows)]
    err = np.abs(yg - ref).max() / max(np.abs(ref).max(), 1e-30)
    assert err <= 2e-2, err
