"""GAT forward + backward through the C ABI == oracle (fp64).

Covers concatenated (hidden) and averaged (last) heads, one and several
heads, ReLU fusion, rows longer than the online-softmax chunk (flash-style
merge of split rows) and isolated vertices."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import TOL, assert_mask_agrees, f64, kink_band, q, rel_err, relu_dy

pytestmark = pytest.mark.gpu


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def run(dtype, H, concat, V=1200, E=15000, fi=24, fo=16, relu=False, seed=0, alpha=0.8, edges=None,
        zero_attn=False):
    m = wg()
    src, dst = edges if edges is not None else synth.make_graph(V, E, seed=seed, alpha=alpha)[:2]
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V)
    conv = m.Conv(g, "gat", fi, fo, dtype=dtype, heads=H, concat=concat, fuse_relu=relu)
    params = m.init_params("gat", fi, fo, heads=H, concat=concat, seed=seed)
    gen = torch.Generator(device="cuda").manual_seed(seed)
    params = {k: v + 0.3 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
    FO = H * fo if concat else fo
    x = torch.from_numpy(synth.make_features(V, fi, seed=seed + 1)).to(dtype)
    dy = torch.from_numpy(synth.normal((V, FO), seed=seed + 2, std=0.3)).to(dtype)
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    W = q(params["W"], dtype)
    al, ar, b = f64(params["attn_l"]), f64(params["attn_r"]), f64(params["bias"])
    yo = oracle.gat_forward(src, dst, V, f64(x), W, al, ar, b, heads=H, concat=concat)
    dyo = f64(dy)
    if relu:   # the oracle's own ReLU decision; dy = 0 on the kink band (tests/util.py)
        band = kink_band(yo, None, dtype)
        assert_mask_agrees(f64(y), yo, band)
        dy_np, dyo = relu_dy(dyo, yo, band)
        dy = torch.from_numpy(dy_np).to(dtype)
        dyo = f64(dy) * (yo > 0)
        yo = np.maximum(yo, 0)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dxo, dWo, dalo, daro, dbo = oracle.gat_backward(src, dst, V, f64(x), W, al, ar, dyo, heads=H, concat=concat)
    errs = {"y": rel_err(f64(y), yo), "dx": rel_err(f64(dx), dxo), "dW": rel_err(f64(grads["W"]), dWo),
            "da_l": rel_err(f64(grads["attn_l"]), dalo), "da_r": rel_err(f64(grads["attn_r"]), daro),
            "db": rel_err(f64(grads["bias"]), dbo)}
    if zero_attn:   # da_l = da_r = 0 exactly (every softmax is over equal logits): rounding noise vs dW's scale
        sc = max(np.abs(dWo).max(), 1e-30)
        errs["da_l"] = float(np.abs(f64(grads["attn_l"]) - dalo).max() / sc)
        errs["da_r"] = float(np.abs(f64(grads["attn_r"]) - daro).max() / sc)
    return errs, g


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("H,concat", [(1, True), (4, True), (4, False), (2, False)])
def test_gat_parity(dtype, H, concat):
    errs, g = run(dtype, H, concat)
    assert g.max_in_degree > 256      # exercises the chunk split + flash merge
    tol = TOL[dtype]
    assert all(v <= tol for v in errs.values()), str(errs)


def test_gat_relu_and_isolated():
    errs, _ = run(torch.float32, 4, True, V=3000, E=5000, relu=True, seed=5, alpha=0.3)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


def test_gat_c2_shape_sampled():
    """C2 layer shape (128 -> 4 x 64, ogbn-arxiv-like skew) at reduced V."""
    errs, _ = run(torch.float32, 4, True, V=6000, E=42000, fi=128, fo=64, seed=7, alpha=0.7)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


def test_gat_needs_full_graph():
    """GAT plans on a graph owning only a row block: WG_ERR_UNSUPPORTED (include/wg.h;
    the 1-D partition covers GCN / SAGE / GIN / RGCN)."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200._capi import WGError
    src, dst, _ = synth.make_graph(1000, 8000, seed=3)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=1000, v_begin=128,
                v_end=512)
    with pytest.raises(WGError, match="unsupported"):
        m.Conv(g, "gat", 16, 8, heads=2)


@pytest.mark.parametrize("H,fo", [(3, 16), (8, 8), (12, 8), (16, 8), (5, 24)])
@pytest.mark.parametrize("concat", [True, False])
def test_gat_head_counts(H, fo, concat):
    # head counts off the specialised kernels' {1, 2, 4, 8} (generic logits /
    # der / source-major passes) and above the fused forward's 8-head limit
    for dtype in (torch.float32, torch.bfloat16):
        errs, _ = run(dtype, H, concat, V=700, E=7000, fi=20, fo=fo, seed=H)
        bad = {k: v for k, v in errs.items() if not v <= TOL[dtype]}
        assert not bad, f"H={H} fo={fo} {dtype}: {errs}"


@pytest.mark.parametrize("dtype,fo", [(torch.float32, 7), (torch.bfloat16, 4)])
def test_gat_unaligned_head_width_is_rejected(dtype, fo):
    # per-head rows narrower than / not a multiple of 16 bytes are refused
    # loudly (WG_ERR_UNSUPPORTED, include/wg.h), never computed approximately
    m = wg()
    with pytest.raises(m.WGError, match="unsupported"):
        run(dtype, 4, True, V=300, E=2000, fi=16, fo=fo)
