"""GCN / SAGE / GIN forward + backward through the C ABI == oracle (fp64).

Tolerances (BASELINE north_star, Q15 metric): fp32 <= 1e-4, bf16 <= 2e-2;
small-integer fp32 inputs: bit-exact.  Every plan policy must give the same
result (T2 indexing swapping is an equivalence, "equivalent
results" P:L1819-1821).  Sizes span several 128-row tiles with a ragged tail;
small E_max values force SPLIT chunks (degree-aware splitting)."""
import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import (TOL, assert_mask_agrees, f64, gin_inner_safe_dy, gin_mags, kink_band, q, rel_err,
                        relu_dy)

pytestmark = pytest.mark.gpu


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def make_inputs(V, E, fi, fo, dtype, seed, alpha=0.6, ints=False, edges=None):
    src, dst = edges if edges is not None else synth.make_graph(V, E, seed=seed, alpha=alpha)[:2]
    if ints:
        x = torch.from_numpy(synth.small_ints((V, fi), seed=seed + 1))
        dy = torch.from_numpy(synth.small_ints((V, fo), seed=seed + 2))
    else:
        x = torch.from_numpy(synth.make_features(V, fi, seed=seed + 1))
        dy = torch.from_numpy(synth.normal((V, fo), seed=seed + 2, std=1.0 / np.sqrt(fo)))
    return src, dst, x.to(dtype), dy.to(dtype)


def oracle_fwd(model, src, dst, V, xo, Wq, norm, eps=0.0):
    """Oracle forward (before any output ReLU); GIN also returns its inner
    pre-activation a = z W1 + b1."""
    if model == "gcn":
        return oracle.gcn_forward(src, dst, V, xo, Wq["W"], Wq.get("bias"), norm=norm), None
    if model == "sage":
        return oracle.sage_forward(src, dst, V, xo, Wq["W_self"], Wq["W"], Wq.get("bias")), None
    if model == "gin":
        y, _, a = oracle.gin_forward(src, dst, V, xo, Wq["W"], Wq["bias"], Wq["W2"], Wq["b2"], eps, return_za=True)
        return y, a
    raise ValueError(model)


def oracle_bwd(model, src, dst, V, xo, Wq, dT, norm, eps=0.0):
    if model == "gcn":
        dx, dW, db = oracle.gcn_backward(src, dst, V, xo, Wq["W"], dT, norm=norm)
        return dx, {"W": dW, "bias": db}
    if model == "sage":
        dx, dWs, dWn, db = oracle.sage_backward(src, dst, V, xo, Wq["W_self"], Wq["W"], dT)
        return dx, {"W": dWn, "W_self": dWs, "bias": db}
    if model == "gin":
        dx, dW1, db1, dW2, db2 = oracle.gin_backward(src, dst, V, xo, Wq["W"], Wq["bias"], Wq["W2"], dT, eps)
        return dx, {"W": dW1, "bias": db1, "W2": dW2, "b2": db2}
    raise ValueError(model)


def oracle_dy(model, src, dst, V, xo, Wq, dy, dtype, norm, fuse_relu, y_gpu=None, h_gpu=None, exact=False):
    """Oracle forward + the kink-band-safe dy (tests/util.py): returns
    (pre, dy_in for the kernel, dT for the oracle backward).  y_gpu / h_gpu
    (optional) are checked to take the oracle's ReLU decisions outside the band."""
    Wabs = {k: np.abs(v) for k, v in Wq.items()}
    if model == "gin":
        pre, z, a = oracle.gin_forward(src, dst, V, xo, Wq["W"], Wq["bias"], Wq["W2"], Wq["b2"], return_za=True)
        mag_a, mag = gin_mags(z, a, Wq["W"], Wq["bias"], Wq["W2"], Wq["b2"])
    else:
        pre = oracle_fwd(model, src, dst, V, xo, Wq, norm)[0]
        mag = oracle_fwd(model, src, dst, V, np.abs(xo), Wabs, norm)[0]
    dy = np.asarray(dy, dtype=np.float64)
    free = None
    if fuse_relu:
        band = kink_band(pre, mag, dtype, exact)
        if y_gpu is not None:
            assert_mask_agrees(y_gpu, pre, band, "output ReLU")
        dy, _ = relu_dy(dy, pre, band)
        free = (pre > 0) & ~band
    if model == "gin":
        band_a = kink_band(a, mag_a, dtype, exact)
        if h_gpu is not None:
            assert_mask_agrees(h_gpu, a, band_a, "GIN inner ReLU")
        dy = gin_inner_safe_dy(dy, a, band_a, Wq["W2"], free)
    dy_in = torch.from_numpy(dy).to(dtype)
    dT = f64(dy_in) * (pre > 0) if fuse_relu else f64(dy_in)
    return pre, dy_in, dT


def run(model, dtype=torch.float32, policy="auto", V=900, E=12000, fi=37, fo=20, T=128, E_max=0, fuse_relu=False,
        norm="both", seed=0, ints=False, need_dx=True, alpha=0.6, edges=None):
    m = wg()
    src, dst, x, dy = make_inputs(V, E, fi, fo, dtype, seed, alpha=alpha, ints=ints, edges=edges)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V, tile_rows=T,
                max_task_edges=E_max)
    conv = m.Conv(g, model, fi, fo, dtype=dtype, policy=policy, seed=seed, fuse_relu=fuse_relu, norm=norm,
                  need_dx=need_dx)
    params = m.init_params(model, fi, fo, seed=seed)
    if ints:
        params = {k: torch.from_numpy(synth.small_ints(tuple(v.shape), seed=seed + 7 + i)).cuda()
                  for i, (k, v) in enumerate(params.items())}
    else:
        gen = torch.Generator(device="cuda").manual_seed(seed)   # non-zero biases, seeded
        params = {k: (v + 0.1 * torch.randn(v.shape, generator=gen, device=v.device)) for k, v in params.items()}
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    yg = f64(y)
    Wq = {k: q(v, dtype) for k, v in params.items()}
    xo = f64(x)
    hg = f64(conv.buffer_view(saved, "h", V, fo)) if model == "gin" else None
    pre, dy_in, dT = oracle_dy(model, src, dst, V, xo, Wq, f64(dy), dtype, norm, fuse_relu, y_gpu=yg, h_gpu=hg,
                                exact=ints)
    dx, grads = conv.backward_raw(m.pad_to(dy_in.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dxo, go = oracle_bwd(model, src, dst, V, xo, Wq, dT, norm)
    yo = np.maximum(pre, 0) if fuse_relu else pre
    return dict(conv=conv, y=(yg, yo), dx=(f64(dx) if need_dx else None, dxo),
                grads={k: (f64(grads[k]), go[k]) for k in go if k in grads})


def check(res, dtype, exact=False):
    tol = 0.0 if exact else TOL[dtype]
    errs = {"y": rel_err(*res["y"])}
    if res["dx"][0] is not None:
        errs["dx"] = rel_err(*res["dx"])
    for k, (a, b) in res["grads"].items():
        errs["d" + k] = rel_err(a, b)
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, f"errors {errs} (tol {tol})"
    return errs


@pytest.mark.parametrize("model", ["gcn", "sage", "gin"])
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("policy", ["auto", "edge", "vertex", "random"])
def test_plan_invariance(model, dtype, policy):
    res = run(model, dtype, policy)
    check(res, dtype)


@pytest.mark.parametrize("model", ["gcn", "sage", "gin"])
@pytest.mark.parametrize("policy", ["edge", "vertex"])
def test_split_rows_and_relu(model, policy):
    # E_max = 64 forces SPLIT chunks on the hubs; fused ReLU in the epilogue
    res = run(model, torch.float32, policy, V=1500, E=30000, E_max=64, fuse_relu=True, alpha=0.8, seed=3)
    assert res["conv"].n_split_rows > 0
    check(res, torch.float32)


@pytest.mark.parametrize("model,norm", [("gcn", "none"), ("gin", "none")])
@pytest.mark.parametrize("policy", ["edge", "vertex", "random"])
def test_integer_inputs_bit_exact(model, norm, policy):
    res = run(model, torch.float32, policy, V=600, E=5000, fi=12, fo=8, ints=True, norm=norm, seed=5, alpha=0.3)
    check(res, torch.float32, exact=True)


@pytest.mark.parametrize("fi,fo", [(1, 1), (3, 5), (100, 47), (256, 256), (300, 129)])
def test_widths(fi, fo):
    for dtype in (torch.float32, torch.bfloat16):
        check(run("sage", dtype, "auto", V=700, E=6000, fi=fi, fo=fo, seed=fi), dtype)


@pytest.mark.parametrize("fi,fo", [(32, 32), (96, 40), (32, 172)])
@pytest.mark.parametrize("policy", ["vertex", "edge"])
def test_split_outputs_off_chunk_grid(fi, fo, policy):
    """SAGE's split GEMM outputs ([Y | S] forward, [dAgg | dX_s] backward) whose
    split falls inside a 128-byte output chunk (bf16 widths not multiples of
    64: C5's 32-wide layers) -- the straddling chunk is stored from registers."""
    check(run("sage", torch.bfloat16, policy, V=900, E=9000, fi=fi, fo=fo, seed=fi + fo, fuse_relu=True),
          torch.bfloat16)


def test_need_dx_false_and_norms():
    for norm in ("none", "right", "both"):
        check(run("gcn", torch.float32, "edge", norm=norm, need_dx=False), torch.float32)


def test_isolated_vertices_and_tiny_tiles():
    # vertices beyond the edge range are isolated; T = 16 gives many tiles
    res = run("gin", torch.float32, "random", V=2000, E=800, T=16, seed=9, alpha=0.2)
    check(res, torch.float32)


def test_deterministic():
    a = run("sage", torch.bfloat16, "edge", seed=4)
    b = run("sage", torch.bfloat16, "edge", seed=4)
    np.testing.assert_array_equal(a["y"][0], b["y"][0])
    np.testing.assert_array_equal(a["dx"][0], b["dx"][0])
    for k in a["grads"]:
        np.testing.assert_array_equal(a["grads"][k][0], b["grads"][k][0])


def test_autograd_module():
    m = wg()
    V, E, fi, fo = 500, 4000, 16, 8
    src, dst, x, _ = make_inputs(V, E, fi, fo, torch.float32, 21)
    g = m.Graph(src, dst, num_vertices=V)
    conv = m.Conv(g, "gcn", fi, fo, dtype=torch.float32)
    params = {k: v.requires_grad_() for k, v in m.init_params("gcn", fi, fo, seed=1).items()}
    xd = x.cuda().requires_grad_()
    y = conv(xd, params)
    (y.float() ** 2).sum().backward()
    assert xd.grad is not None and params["W"].grad is not None
    yo = oracle.gcn_forward(src, dst, V, f64(x), f64(params["W"].detach()), f64(params["bias"].detach()))
    assert rel_err(f64(y.detach()), yo) < 1e-4


def test_overfill_cluster_path_deterministic():
    """Rows longer than E_max run on the thread-block-cluster kernel (DSMEM
    merge in rank order): bitwise-equal reruns, and the partial + combine path
    (WG_HEAVY=0, read once per process) gives the same result within fp32."""
    a = run("sage", torch.float32, "edge", V=1500, E=30000, E_max=64, fuse_relu=True, alpha=0.8, seed=3)
    b = run("sage", torch.float32, "edge", V=1500, E=30000, E_max=64, fuse_relu=True, alpha=0.8, seed=3)
    assert a["conv"].n_split_rows > 0
    np.testing.assert_array_equal(a["y"][0], b["y"][0])
    np.testing.assert_array_equal(a["dx"][0], b["dx"][0])
    import os
    import subprocess
    import sys
    code = ("from tests.test_gpu_conv_lin import run, check\n"
            "import torch\n"
            "for m in ('gcn', 'sage', 'gin'):\n"
            "    for pol in ('edge', 'vertex'):\n"
            "        r = run(m, torch.float32, pol, V=1500, E=30000, E_max=64, fuse_relu=True, alpha=0.8, seed=3)\n"
            "        assert r['conv'].n_split_rows > 0\n"
            "        check(r, torch.float32)\n"
            "print('ok')\n")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], cwd=root, capture_output=True, text=True, timeout=600,
                       env=dict(os.environ, WG_HEAVY="0", WG_UNDERFILL="0"))
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]
