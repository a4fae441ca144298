"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same synthetic recipe, graph, plans and kernels).

Outputs the oracle can compute one by one are compared on sampled rows;
weight gradients on sampled entries dW[i, j] = sum_e c_e x[s_e, i] dT[d_e, j]
(the definition, contracted: oracle.dw_probe on single columns); the
partition on sampled destination tiles (a gTask never spans tiles, so a
tile's tables are the oracle's tables for that tile's in-edges).

ReLU decisions (DESIGN.md §2 "Kink band").  Every mask the oracle applies is
its own fp64 decision.  At full size the oracle computes pre-activations only
for sampled rows, so a layer with a fused ReLU is driven by a dy SUPPORTED on
a sampled destination set D (dy = 0 elsewhere): every dT row that can reach a
compared value is one whose ReLU the oracle decided, and outside the kink band
the kernel's decisions on D must equal the oracle's.  Layers without a ReLU
keep a dense dy."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import (assert_mask_agrees, f64, gin_inner_safe_dy, gin_mags, kink_band, q, relu_dy)

pytestmark = pytest.mark.gpu

RNG = np.random.default_rng(2024)


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def sampled_err(got, ref, rows):
    a, b = got[rows], ref[rows]
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))


def sample_rows(deg, E_max, n=2000, top=50, pool=None):
    """Random rows (from `pool` if given) + every SPLIT row + the `top`
    highest-degree rows."""
    V = deg.shape[0]
    base = np.arange(V) if pool is None else np.asarray(pool)
    rows = set(RNG.choice(base, size=min(n, len(base)), replace=False).tolist())
    rows |= set(np.nonzero(deg > E_max)[0].tolist())
    rows |= set(np.argsort(deg)[-top:].tolist())
    return np.array(sorted(rows))


def entry_probe(src, dst, coef, x, dy, i, j):
    return oracle.dw_probe(src, dst, x[:, i:i + 1], dy[:, j:j + 1], np.ones(1), np.ones(1), coef)


def supported_dy(V, F, rows, seed, std):
    """N(0, std) on `rows`, zero elsewhere (float64 [V x F])."""
    dy = np.zeros((V, F))
    dy[rows] = synth.normal((len(rows), F), seed=seed, std=std)
    return dy


def sources_into(src, dst, D, n, extra_V=0, extra=0):
    """A sample of the sources of edges into D (+ `extra` random rows of [0, extra_V))."""
    into = np.isin(dst, D)
    s = np.unique(src[into])
    rows = set(RNG.choice(s, size=min(n, len(s)), replace=False).tolist())
    if extra:
        rows |= set(RNG.choice(extra_V, size=extra, replace=False).tolist())
    return np.array(sorted(rows)), into


def to_dev(m, a, dtype):
    return m.pad_to(torch.from_numpy(np.ascontiguousarray(a)).to(dtype).cuda())


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


def _probe_errs(src, dst, coef, xo, dT, gW, pairs, self_rows=None, gWs=None):
    """dW entries (and W_self entries over self_rows) vs the contracted definition."""
    errs = []
    sc_n = max(np.abs(gW).max(), 1e-30)
    for (i, j) in pairs:
        on = entry_probe(src, dst, coef, xo, dT, i, j)
        errs.append(abs(gW[i, j] - on) / sc_n)
        if gWs is not None:
            idx = self_rows.astype(np.int32)
            os_ = entry_probe(idx, idx, None, xo, dT, i, j)
            errs.append(abs(gWs[i, j] - os_) / max(np.abs(gWs).max(), 1e-30))
    return errs


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
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    W = {k: q(v, dt) for k, v in params.items()}
    xo, yg = f64(x), f64(y)
    deg = np.bincount(dst, minlength=c.V)
    D = sample_rows(deg, g.E_max, n=2000, top=10)
    pre = oracle.sage_forward(src, dst, c.V, xo, W["W_self"], W["W"], W["bias"], rows=D)
    yo = np.maximum(pre, 0) if relu else pre
    assert sampled_err(yg, yo, D) <= 2e-2
    if relu:   # dy supported on D, zero on D's kink band; the kernel's decisions on D must be the oracle's
        Wa = {k: np.abs(v) for k, v in W.items()}
        mag = oracle.sage_forward(src, dst, c.V, np.abs(xo), Wa["W_self"], Wa["W"], Wa["bias"], rows=D)
        band = kink_band(pre[D], mag[D], dt)
        assert_mask_agrees(yg[D], pre[D], band)
        dy_np = supported_dy(c.V, fo, D, 600 + layer, 0.05)
        dy_np[D], _ = relu_dy(dy_np[D], pre[D], band)
    else:
        dy_np = f64(torch.from_numpy(synth.normal((c.V, fo), seed=600 + layer, std=0.05)))
    dy = torch.from_numpy(dy_np).to(dt)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dT = f64(dy)
    if relu:
        dT[D] *= pre[D] > 0
        rows_t, into = sources_into(src, dst, D, 1500, c.V, 300)
    else:
        rows_t = sample_rows(np.bincount(src, minlength=c.V), g.E_max, n=2000, top=10)
        into = np.ones(src.shape[0], bool)
    dxo, _, _, _ = oracle.sage_backward(src, dst, c.V, xo, W["W_self"], W["W"], dT, rows=rows_t, grads=False)
    assert sampled_err(f64(dx), dxo, rows_t) <= 2e-2
    coef = 1.0 / np.maximum(deg[dst[into]], 1)
    self_rows = D if relu else np.arange(c.V)
    pairs = [(0, 0), (fi - 1, fo - 1), (fi // 2, fo // 3), (3 % fi, (7 * fo) // 8)]
    errs = _probe_errs(src[into], dst[into], coef, xo, dT, f64(grads["W"]), pairs, self_rows, f64(grads["W_self"]))
    assert max(errs) <= 2e-2, errs
    db = f64(grads["bias"])
    np.testing.assert_allclose(db, dT.sum(0), rtol=0, atol=2e-2 * max(1e-30, np.abs(dT.sum(0)).max()))


@pytest.mark.parametrize("layer", [0, 1, 2])
def test_c4_gin_layer_sampled(c4, layer):
    """C4 GIN (100 -> 256 -> 256 -> 47, bf16) at full size, the plans bench.py
    --model gin runs.  dy is supported on a sampled destination set D, which
    makes the oracle's gradients exact for EVERY vertex (gin_backward with
    dy_rows = D): dx is compared on all rows with a non-zero oracle dx plus
    random zero rows, dW1 / db1 / dW2 / db2 in full.  Both ReLUs (the inner
    one of the MLP and the fused output ReLU of the hidden layers) are decided
    by the oracle; dy is zero on the output kink band and projected orthogonal
    to the W2 rows of inner kink-band elements (tests/util.py)."""
    c, src, dst, g = c4
    m = wg()
    fi, fo = c.dims[layer], c.dims[layer + 1]
    relu = layer < 2
    dt = torch.bfloat16
    conv = m.Conv(g, "gin", fi, fo, dtype=dt, fuse_relu=relu, need_dx=True)
    params = m.init_params("gin", fi, fo, seed=10 + layer)
    gen = torch.Generator(device="cuda").manual_seed(10 + layer)
    params = {k: v + 0.05 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=520 + layer)).to(dt)
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    W = {k: q(v, dt) for k, v in params.items()}
    xo = f64(x)
    deg = np.bincount(dst, minlength=c.V)
    D = sample_rows(deg, g.E_max, n=3000, top=10)
    pre, z, a = oracle.gin_forward(src, dst, c.V, xo, W["W"], W["bias"], W["W2"], W["b2"], rows=D, return_za=True)
    mag_a, mag = np.zeros_like(a), np.zeros_like(pre)
    mag_a[D], mag[D] = gin_mags(z[D], a[D], W["W"], W["bias"], W["W2"], W["b2"])
    Dd = torch.from_numpy(D).cuda()
    yg = f64(y[Dd])
    yo = np.maximum(pre[D], 0) if relu else pre[D]
    assert np.abs(yg - yo).max() / np.abs(yo).max() <= 2e-2
    band_a = kink_band(a[D], mag_a[D], dt)
    assert_mask_agrees(f64(conv.buffer_view(saved, "h", c.V, fo)[Dd]), a[D], band_a, "GIN inner ReLU")
    dyD = synth.normal((len(D), fo), seed=620 + layer, std=0.05).astype(np.float64)
    free = None
    if relu:
        band = kink_band(pre[D], mag[D], dt)
        assert_mask_agrees(yg, pre[D], band, "output ReLU")
        dyD, _ = relu_dy(dyD, pre[D], band)
        free = (pre[D] > 0) & ~band
    dyD = gin_inner_safe_dy(dyD, a[D], band_a, W["W2"], free)
    dy_np = np.zeros((c.V, fo))
    dy_np[D] = dyD
    dy = torch.from_numpy(dy_np).to(dt)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dT = np.zeros((c.V, fo))
    dT[D] = f64(dy[D]) * ((pre[D] > 0) if relu else 1.0)
    dxo, dW1, db1, dW2, db2 = oracle.gin_backward(src, dst, c.V, xo, W["W"], W["bias"], W["W2"], dT, dy_rows=D)
    nz = np.unique(np.concatenate([D, src[np.isin(dst, D)]]))
    rows = np.union1d(nz, RNG.choice(c.V, size=3000, replace=False))
    dxg = f64(dx[torch.from_numpy(rows).cuda()])
    errs = {"dx": np.abs(dxg - dxo[rows]).max() / np.abs(dxo[rows]).max()}
    for k, ref in (("W", dW1), ("bias", db1), ("W2", dW2), ("b2", db2)):
        errs["d" + k] = np.abs(f64(grads[k]) - ref).max() / max(np.abs(ref).max(), 1e-30)
    assert max(errs.values()) <= 2e-2, errs


def test_c1_gcn_full_exact():
    c = synth.CONFIGS["C1"]
    m = wg()
    src, dst, _ = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha, symmetric=True)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    x = torch.from_numpy(synth.make_features(c.V, c.dims[0], seed=c.seed * 16 + 2, dist="bernoulli", p=c.xp))
    for layer in range(2):
        fi, fo = c.dims[layer], c.dims[layer + 1]
        relu = layer == 0
        conv = m.Conv(g, "gcn", fi, fo, dtype=torch.float32, fuse_relu=relu)
        params = m.init_params("gcn", fi, fo, seed=layer)
        xd = m.pad_to(x.cuda())
        y, saved = conv.forward_raw(xd, params)
        torch.cuda.synchronize()
        Wo, bo = f64(params["W"]), f64(params["bias"])
        pre = oracle.gcn_forward(src, dst, c.V, f64(x), Wo, bo)
        dyo = f64(torch.from_numpy(synth.normal((c.V, fo), seed=layer, std=0.3)))
        yo = pre
        if relu:
            mag = oracle.gcn_forward(src, dst, c.V, np.abs(f64(x)), np.abs(Wo), np.abs(bo))
            band = kink_band(pre, mag, torch.float32)
            assert_mask_agrees(f64(y), pre, band)
            dyo, _ = relu_dy(dyo, pre, band)
            yo = np.maximum(pre, 0)
        dy = torch.from_numpy(dyo).float()
        dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
        torch.cuda.synchronize()
        dT = f64(dy) * (pre > 0) if relu else f64(dy)
        dxo, dWo, dbo = oracle.gcn_backward(src, dst, c.V, f64(x), Wo, dT)
        for a, b in ((f64(y), yo), (f64(dx), dxo), (f64(grads["W"]), dWo), (f64(grads["bias"]), dbo)):
            assert np.abs(a - b).max() / max(np.abs(b).max(), 1e-30) <= 1e-4
        x = y.detach().cpu().float()


def _c2():
    c = synth.CONFIGS["C2"]
    src, dst, _ = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha)
    return c, src, dst


def test_c2_gat_layer1_full():
    c, src, dst = _c2()
    m = wg()
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    H, fi, fo = c.heads, c.dims[0], c.dims[1]
    conv = m.Conv(g, "gat", fi, fo, dtype=torch.float32, heads=H, concat=True, fuse_relu=True)
    params = m.init_params("gat", fi, fo, heads=H, seed=1)
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=c.seed * 16 + 2))
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    P = {k: f64(v) for k, v in params.items()}
    pre = oracle.gat_forward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], P["bias"], heads=H)
    band = kink_band(pre, None, torch.float32)
    assert_mask_agrees(f64(y), pre, band)
    dy_np, _ = relu_dy(f64(torch.from_numpy(synth.normal((c.V, H * fo), seed=3, std=0.1))), pre, band)
    dy = torch.from_numpy(dy_np).float()
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dyo = f64(dy) * (pre > 0)
    dxo, dWo, dal, dar, dbo = oracle.gat_backward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], dyo, heads=H)
    for a, b in ((f64(y), np.maximum(pre, 0)), (f64(dx), dxo), (f64(grads["W"]), dWo), (f64(grads["attn_l"]), dal),
                 (f64(grads["attn_r"]), dar), (f64(grads["bias"]), dbo)):
        assert np.abs(a - b).max() / max(np.abs(b).max(), 1e-30) <= 1e-4


def test_c2_gat_last_layer_full():
    """C2's last layer at full size: 4 heads x 40 classes AVERAGED (Q6), input
    the concatenated 4 x 64 hidden width, no ReLU, fp32."""
    c, src, dst = _c2()
    m = wg()
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V)
    H, fi, fo = c.heads, c.heads * c.dims[2], c.dims[3]
    conv = m.Conv(g, "gat", fi, fo, dtype=torch.float32, heads=H, concat=False, fuse_relu=False)
    params = m.init_params("gat", fi, fo, heads=H, concat=False, seed=3)
    gen = torch.Generator(device="cuda").manual_seed(3)
    params = {k: v + 0.1 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    x = torch.from_numpy(synth.make_features(c.V, fi, seed=c.seed * 16 + 7))
    dy = torch.from_numpy(synth.normal((c.V, fo), seed=8, std=0.1))
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    P = {k: f64(v) for k, v in params.items()}
    yo = oracle.gat_forward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], P["bias"], heads=H,
                            concat=False)
    dxo, dWo, dal, dar, dbo = oracle.gat_backward(src, dst, c.V, f64(x), P["W"], P["attn_l"], P["attn_r"], f64(dy),
                                                  heads=H, concat=False)
    errs = {}
    for k, a, b in (("y", f64(y), yo), ("dx", f64(dx), dxo), ("dW", f64(grads["W"]), dWo),
                    ("da_l", f64(grads["attn_l"]), dal), ("da_r", f64(grads["attn_r"]), dar),
                    ("db", f64(grads["bias"]), dbo)):
        errs[k] = np.abs(a - b).max() / max(np.abs(b).max(), 1e-30)
    assert max(errs.values()) <= 1e-4, errs


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
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    W, b = f64(params["W"]), f64(params["bias"])
    xo = f64(x)
    deg = np.bincount(dst, minlength=c.V)
    D = sample_rows(deg, g.E_max, 1000, top=10)
    pre = oracle.rgcn_forward(src, dst, et, c.V, xo, W, None, b, rows=D)
    mag = oracle.rgcn_forward(src, dst, et, c.V, np.abs(xo), np.abs(W), None, np.abs(b), rows=D)
    assert sampled_err(f64(y), np.maximum(pre, 0), D) <= 1e-4
    band = kink_band(pre[D], mag[D], torch.float32)
    assert_mask_agrees(f64(y)[D], pre[D], band)
    dy_np = supported_dy(c.V, fo, D, 4, 0.1)
    dy_np[D], _ = relu_dy(dy_np[D], pre[D], band)
    dy = torch.from_numpy(dy_np).float()
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dT = f64(dy)
    dT[D] *= pre[D] > 0
    rows_t, into = sources_into(src, dst, D, 800, c.V, 200)
    dxo, _, _, _ = oracle.rgcn_backward(src, dst, et, c.V, xo, W, dT, rows=rows_t, grads=False)
    assert sampled_err(f64(dx), dxo, rows_t) <= 1e-4
    gW = f64(grads["W"])
    scale = np.abs(gW).max()
    s_in, d_in, t_in = src[into], dst[into], et[into]
    for r in (0, 1, 5, c.R - 1):
        sel = t_in == r
        for (i, j) in [(0, 0), (fi - 1, fo - 1), (17, 33)]:
            ref = entry_probe(s_in[sel], d_in[sel], None, xo, dT, i, j)
            assert abs(gW[r, i, j] - ref) <= 1e-4 * scale, (r, i, j, gW[r, i, j], ref)
    np.testing.assert_allclose(f64(grads["bias"]), dT.sum(0), rtol=0, atol=1e-4 * np.abs(dT.sum(0)).max())


# ------------------------------------------------------------------ C5
@pytest.fixture(scope="module")
def c5slice():
    """Rank 0's slice of C5's 8-way 1-D partition (its in- and out-edges), the
    graph bench.py --rank-slice 8 builds."""
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    c = synth.CONFIGS["C5"]
    m = wg()
    block, bounds = equal_blocks(c.V, 8)
    vb, ve = bounds[0]
    src, dst = synth.make_graph_slice(c.V, c.E, vb, ve, seed=c.seed * 16, alpha=c.alpha)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V, v_begin=vb, v_end=ve)
    return c, src, dst, g, block, bounds


def _induced(src, dst, rows):
    """Edges into `rows` (all of them: degrees stay global), vertices relabelled."""
    sel = np.isin(dst, rows)
    s_r, d_r = src[sel], dst[sel]
    U = np.unique(np.concatenate([rows, s_r]))
    remap = lambda a: np.searchsorted(U, a).astype(np.int32)  # noqa: E731
    return U, remap, remap(s_r), remap(d_r)


def _randn_table(m, V, F, dt, seed):
    t = m.padded(V, F, dt)
    gen = torch.Generator(device="cuda").manual_seed(seed)
    for r0 in range(0, V, 1 << 22):
        r1 = min(V, r0 + (1 << 22))
        t[r0:r1].copy_(torch.randn((r1 - r0, F), generator=gen, device="cuda"))
    return t


def test_c5_rank_slice_layer1_sampled(c5slice):
    """C5 (111 M V, 1.6 B E) at full size, in the launch configuration bench.py
    --rank-slice 8 times: rank 0's block of the 8-way 1-D partition (its in- and
    out-edges only).  Layer-1 SAGE forward of owned rows is exact on the slice
    (every in-edge of an owned row is present, degrees of owned rows are
    global), so sampled rows are compared with the oracle on their induced
    in-neighbourhood.  The EDGE plan gathers the replicated input table
    itself."""
    c, src, dst, g, block, bounds = c5slice
    m = wg()
    vb, ve = bounds[0]
    dt = torch.bfloat16
    fi, fo = c.dims[0], c.dims[1]
    x = _randn_table(m, c.V, fi, dt, 5)
    conv = m.Conv(g, "sage", fi, fo, dtype=dt, fuse_relu=True, need_dx=False, policy="edge")
    params = m.init_params("sage", fi, fo, seed=7)
    y, saved = conv.forward_raw(x, params)
    torch.cuda.synchronize()
    own = (dst >= vb) & (dst < ve)
    deg = np.bincount(dst[own] - vb, minlength=ve - vb)
    rows = set((RNG.choice(ve - vb, size=1000, replace=False) + vb).tolist())
    rows |= set((np.argsort(deg)[-20:] + vb).tolist())
    rows = np.array(sorted(rows))
    U, remap, s_r, d_r = _induced(src[own], dst[own], rows)
    xs = f64(x[torch.from_numpy(U).cuda()])
    W = {k: q(v, dt) for k, v in params.items()}
    yo = np.maximum(oracle.sage_forward(s_r, d_r, len(U), xs, W["W_self"], W["W"], W["bias"], rows=remap(rows)), 0)
    yg = f64(y)[rows - vb]
    ref = yo[remap(rows)]
    err = np.abs(yg - ref).max() / max(np.abs(ref).max(), 1e-30)
    assert err <= 2e-2, err
    del x, y, saved, conv
    torch.cuda.empty_cache()


def test_c5_rank_slice_vertex_layer_fwd_bwd(c5slice):
    """C5 layer 2 (SAGE 32 -> 32, fused ReLU, bf16) on rank 0's slice with the
    VERTEX plan and both exchange tables, forward AND backward.
    Forward: every other rank's PRE phase (Y = x W_n for its rows, written into
    the shared exchange table) is run by the library itself on an edgeless
    graph owning that rank's rows -- a forward PRE reads no edges -- so the
    table rank 0's POST gathers holds exactly what the all-gather would bring.
    Backward: dy is supported on a sampled set D of rank 0's own rows, so the
    other ranks' dT rows are zero and so are their rows of the backward
    exchange table; rank 0's PRE writes its rows, its POST runs the transposed
    gather over its out-edges.  Compared with the oracle on induced
    neighbourhoods: y on D, dx on owned sources of edges into D, and rank 0's
    local weight gradients (its share of the all-reduce) on probed entries."""
    c, src, dst, g, block, bounds = c5slice
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import _capi as C
    vb, ve = bounds[0]
    dt = torch.bfloat16
    fi, fo = c.dims[1], c.dims[2]
    Vtab = block * 8
    x = _randn_table(m, Vtab, fi, dt, 11)
    params = m.init_params("sage", fi, fo, seed=12)
    gen = torch.Generator(device="cuda").manual_seed(12)
    params = {k: v + 0.05 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    xf = m.padded(Vtab, m.pitch(fo, dt), dt)
    # the other ranks' PRE phases (edgeless graphs owning their rows)
    empty = torch.zeros(0, dtype=torch.int32, device="cuda")
    for p in range(1, 8):
        b0, b1 = bounds[p]
        if b0 >= b1:
            continue
        gq = m.Graph(empty, empty, num_vertices=c.V, v_begin=b0, v_end=b1)
        cq = m.Conv(gq, "sage", fi, fo, dtype=dt, fuse_relu=True, policy="vertex")
        yq = m.padded(b1 - b0, fo, dt)
        cq.forward_raw(x, params, y=yq, phase=C.PHASE_PRE, xchg=xf)
        torch.cuda.synchronize()
        cq.close(); gq.close()
        del cq, gq, yq
    conv = m.Conv(g, "sage", fi, fo, dtype=dt, fuse_relu=True, need_dx=True, policy="vertex")
    assert conv.n_vertex_tasks > 0 and conv.bwd_path == 1
    y = m.padded(ve - vb, fo, dt)
    saved = conv.new_saved()
    conv.forward_raw(x, params, y=y, saved=saved, phase=C.PHASE_PRE, xchg=xf)
    conv.forward_raw(x, params, y=y, saved=saved, phase=C.PHASE_POST, xchg=xf)
    torch.cuda.synchronize()
    del xf
    own = (dst >= vb) & (dst < ve)
    s_own, d_own = src[own], dst[own]
    deg = np.bincount(d_own - vb, minlength=ve - vb)
    D = set((RNG.choice(ve - vb, size=1500, replace=False) + vb).tolist())
    D |= set((np.argsort(deg)[-5:] + vb).tolist())
    D = np.array(sorted(D))
    U, remap, s_r, d_r = _induced(s_own, d_own, D)
    xs = f64(x[torch.from_numpy(U).cuda()])
    W = {k: q(v, dt) for k, v in params.items()}
    Wa = {k: np.abs(v) for k, v in W.items()}
    Dl = remap(D)
    pre = oracle.sage_forward(s_r, d_r, len(U), xs, W["W_self"], W["W"], W["bias"], rows=Dl)[Dl]
    mag = oracle.sage_forward(s_r, d_r, len(U), np.abs(xs), Wa["W_self"], Wa["W"], Wa["bias"], rows=Dl)[Dl]
    yg = f64(y)[D - vb]
    assert np.abs(yg - np.maximum(pre, 0)).max() / np.abs(np.maximum(pre, 0)).max() <= 2e-2
    band = kink_band(pre, mag, dt)
    assert_mask_agrees(yg, pre, band)
    dyD, _ = relu_dy(synth.normal((len(D), fo), seed=13, std=0.05).astype(np.float64), pre, band)
    dy = m.padded(ve - vb, fo, dt)
    dy[torch.from_numpy(D - vb).cuda()] = torch.from_numpy(dyD).to(dt).cuda()
    xb = m.padded(Vtab, m.pitch(fo, dt), dt)          # other ranks' rows: their dT is zero
    dx = m.padded(ve - vb, fi, dt)
    grads = {k: torch.zeros_like(v) for k, v in params.items()}
    for ph in (C.PHASE_PRE, C.PHASE_POST):
        conv.backward_raw(dy, x, y, saved, params, dx=dx, phase=ph, xchg=xb, grads=grads)
    torch.cuda.synchronize()
    dTD = f64(dy[torch.from_numpy(D - vb).cuda()]) * (pre > 0)
    # oracle: edges into D (all of them -- global degrees of D), dT on D only
    dT_U = np.zeros((len(U), fo))
    dT_U[Dl] = dTD
    ownsrc = U[(U >= vb) & (U < ve)]
    rows_t = np.array(sorted(set(RNG.choice(ownsrc, size=min(1500, len(ownsrc)), replace=False).tolist())))
    dxo, _, _, _ = oracle.sage_backward(s_r, d_r, len(U), xs, W["W_self"], W["W"], dT_U, rows=remap(rows_t),
                                        grads=False)
    dxg = f64(dx[torch.from_numpy(rows_t - vb).cuda()])
    ref = dxo[remap(rows_t)]
    assert np.abs(dxg - ref).max() / np.abs(ref).max() <= 2e-2
    # rank 0's local weight gradients (G path: dW_n = x_own^T G_own over its out-edges)
    sel = (U[s_r] >= vb) & (U[s_r] < ve)
    degD = np.bincount(d_r, minlength=len(U))
    coef = 1.0 / np.maximum(degD[d_r[sel]], 1)
    pairs = [(0, 0), (fi - 1, fo - 1), (fi // 2, fo // 3)]
    errs = _probe_errs(s_r[sel], d_r[sel], coef, xs, dT_U, f64(grads["W"]), pairs, Dl, f64(grads["W_self"]))
    assert max(errs) <= 2e-2, errs
    np.testing.assert_allclose(f64(grads["bias"]), dTD.sum(0), rtol=0, atol=2e-2 * np.abs(dTD.sum(0)).max())
