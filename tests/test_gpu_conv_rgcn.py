"""RGCN (Eq. (1)) forward + backward through the C ABI == oracle.

Every per-gTask plan policy (EDGE = (dst, relation) segment sums, VERTEX =
gTask-local unique-source transforms, mixed) must give the same result;
small-integer inputs are bit-exact; SPLIT chunks (small E_max) are merged."""
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


def run(dtype=torch.float32, policy="auto", norm="none", self_loop=False, bias=False, R=5, V=1500, E=20000, fi=24,
        fo=16, E_max=0, seed=0, ints=False, relu=False, alpha=0.6, edges=None):
    m = wg()
    src, dst, et = edges if edges is not None else synth.make_graph(V, E, seed=seed, alpha=alpha, R=R)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V,
                etype=None if et is None else torch.from_numpy(et).cuda(), num_types=R, max_task_edges=E_max)
    conv = m.Conv(g, "rgcn", fi, fo, dtype=dtype, policy=policy, seed=seed, norm=norm, self_loop=self_loop,
                  bias=bias, fuse_relu=relu)
    params = m.init_params("rgcn", fi, fo, R=R, self_loop=self_loop, bias=bias, seed=seed)
    if ints:
        params = {k: torch.from_numpy(synth.small_ints(tuple(v.shape), seed=seed + 3 + i)).cuda()
                  for i, (k, v) in enumerate(params.items())}
        x = torch.from_numpy(synth.small_ints((V, fi), seed=seed + 1)).to(dtype)
        dy = torch.from_numpy(synth.small_ints((V, fo), seed=seed + 2)).to(dtype)
    else:
        gen = torch.Generator(device="cuda").manual_seed(seed)
        params = {k: v + 0.1 * torch.randn(v.shape, generator=gen, device="cuda") for k, v in params.items()}
        x = torch.from_numpy(synth.make_features(V, fi, seed=seed + 1)).to(dtype)
        dy = torch.from_numpy(synth.normal((V, fo), seed=seed + 2, std=0.25)).to(dtype)
    xd = m.pad_to(x.cuda())
    y, saved = conv.forward_raw(xd, params)
    torch.cuda.synchronize()
    Wq = {k: q(v, dtype) for k, v in params.items()}
    yo = oracle.rgcn_forward(src, dst, et, V, f64(x), Wq["W"], Wq.get("W_self"), Wq.get("bias"), norm=norm)
    dyo = f64(dy)
    if relu:   # the oracle's own ReLU decision; dy = 0 on the kink band (tests/util.py)
        Wa = {k: np.abs(v) for k, v in Wq.items()}
        mag = oracle.rgcn_forward(src, dst, et, V, np.abs(f64(x)), Wa["W"], Wa.get("W_self"), Wa.get("bias"),
                                  norm=norm)
        band = kink_band(yo, mag, dtype, exact=ints)
        assert_mask_agrees(f64(y), yo, band)
        dy_np, _ = relu_dy(dyo, yo, band)
        dy = torch.from_numpy(dy_np).to(dtype)
        dyo = f64(dy) * (yo > 0)
        yo = np.maximum(yo, 0)
    dx, grads = conv.backward_raw(m.pad_to(dy.cuda()), xd, y, saved, params)
    torch.cuda.synchronize()
    dxo, dWo, dW0o, dbo = oracle.rgcn_backward(src, dst, et, V, f64(x), Wq["W"], dyo, Wq.get("W_self"), norm=norm)
    errs = {"y": rel_err(f64(y), yo), "dx": rel_err(f64(dx), dxo), "dW": rel_err(f64(grads["W"]), dWo)}
    if self_loop:
        errs["dW0"] = rel_err(f64(grads["W_self"]), dW0o)
    if bias:
        errs["db"] = rel_err(f64(grads["bias"]), dbo)
    return errs, conv


@pytest.mark.parametrize("policy", ["auto", "edge", "vertex", "random"])
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_rgcn_plan_invariance(policy, dtype):
    errs, conv = run(dtype, policy)
    if policy == "random":
        assert conv.n_edge_tasks > 0 and conv.n_vertex_tasks > 0
    assert all(v <= TOL[dtype] for v in errs.values()), str(errs)


@pytest.mark.parametrize("policy", ["edge", "vertex"])
def test_rgcn_norm_selfloop_bias_relu_split(policy):
    errs, conv = run(torch.float32, policy, norm="right", self_loop=True, bias=True, relu=True, E_max=16, seed=3,
                     alpha=0.8)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


@pytest.mark.parametrize("policy", ["edge", "vertex", "random"])
def test_rgcn_integer_bit_exact(policy):
    errs, _ = run(torch.float32, policy, ints=True, self_loop=True, seed=5, V=800, E=6000, fi=8, fo=8, alpha=0.3)
    assert all(v == 0.0 for v in errs.values()), str(errs)


def test_rgcn_single_relation():
    errs, _ = run(torch.float32, "auto", R=1, seed=7)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


def test_rgcn_c3_shape_sampled():
    """C3 layer shape (128 -> 64, R = 128 Zipf relations) at reduced V / E."""
    errs, _ = run(torch.float32, "auto", R=128, V=20000, E=220000, fi=128, fo=64, seed=9, alpha=0.5)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


def test_rgcn_c3_layer2_shape_sampled():
    """C3 second-layer shape (64 -> 64, R = 128): the fp32 weight gradient runs the
    TN M fold (A_lo in the MMA's rows 64..127) with two real A chunks."""
    errs, _ = run(torch.float32, "auto", R=128, V=20000, E=220000, fi=64, fo=64, seed=11, alpha=0.5, relu=True)
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


@pytest.mark.parametrize("policy", ["edge", "vertex", "auto"])
@pytest.mark.parametrize("P", [2, 3])
def test_rgcn_1d_partition_phases_match_oracle(policy, P):
    """1-D multi-GPU layer simulated on one GPU: P row blocks,
    forward reads every row of x, backward PRE writes each block's dT rows into
    one exchange table, POST runs the transposed gather over the block's
    out-edges; the blocks' y / dx rows and the summed weight gradients equal
    the oracle (global 1/|N_v^r| coefficients, SPLIT rows via a small E_max)."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    V, E, fi, fo, R = 3000, 40000, 24, 16, 6
    dtype = torch.float32
    src, dst, et = synth.make_graph(V, E, seed=41, alpha=0.7, R=R)
    x = torch.from_numpy(synth.make_features(V, fi, seed=42))
    dy = torch.from_numpy(synth.normal((V, fo), seed=43, std=0.25))
    params = m.init_params("rgcn", fi, fo, R=R, self_loop=True, bias=True, seed=4)
    ts, td, tt = (torch.from_numpy(a).cuda() for a in (src, dst, et))
    block, bounds = equal_blocks(V, P)
    Vt = block * P
    xt = m.padded(Vt, fi, dtype)
    xt[:V] = x.cuda()
    yt, dyt, dxt = m.padded(Vt, fo, dtype), m.padded(Vt, fo, dtype), m.padded(Vt, fi, dtype)
    dyt[:V] = dy.cuda()
    xb = m.padded(Vt, m.pitch(fo, dtype), dtype)
    ranks = []
    for p in range(P):
        vb, ve = bounds[p]
        g = m.Graph(ts, td, num_vertices=V, etype=tt, num_types=R, v_begin=vb, v_end=ve, max_task_edges=64)
        c = m.Conv(g, "rgcn", fi, fo, dtype=dtype, policy=policy, norm="right", self_loop=True, bias=True,
                   fuse_relu=True)
        assert c.bwd_path == 1
        ranks.append((g, c, vb, ve, c.new_saved()))
    for g, c, vb, ve, sv in ranks:
        c.forward_raw(xt, params, y=yt[vb:ve], saved=sv, phase=2)
    torch.cuda.synchronize()
    Wq = {k: f64(v) for k, v in params.items()}
    pre = oracle.rgcn_forward(src, dst, et, V, f64(x), Wq["W"], Wq["W_self"], Wq["bias"], norm="right")
    Wa = {k: np.abs(v) for k, v in Wq.items()}
    mag = oracle.rgcn_forward(src, dst, et, V, np.abs(f64(x)), Wa["W"], Wa["W_self"], Wa["bias"], norm="right")
    band = kink_band(pre, mag, dtype)
    assert_mask_agrees(f64(yt[:V]), pre, band)
    dy_np, _ = relu_dy(f64(dy), pre, band)
    dyt[:V] = torch.from_numpy(dy_np).to(dtype).cuda()
    grads = [{k: torch.zeros_like(v) for k, v in params.items()} for _ in ranks]
    for ph in (1, 2):
        for (g, c, vb, ve, sv), gr in zip(ranks, grads):
            c.backward_raw(dyt[vb:ve], xt, yt[vb:ve], sv, params, dx=dxt[vb:ve], phase=ph, xchg=xb, grads=gr)
    torch.cuda.synchronize()
    yo = np.maximum(pre, 0)
    dyo = f64(dyt[:V]) * (pre > 0)
    dxo, dWo, dW0o, dbo = oracle.rgcn_backward(src, dst, et, V, f64(x), Wq["W"], dyo, Wq["W_self"], norm="right")
    tot = {k: sum(gr[k] for gr in grads) for k in params}
    errs = {"y": rel_err(f64(yt[:V]), yo), "dx": rel_err(f64(dxt[:V]), dxo), "dW": rel_err(f64(tot["W"]), dWo),
            "dW0": rel_err(f64(tot["W_self"]), dW0o), "db": rel_err(f64(tot["bias"]), dbo)}
    assert all(v <= 1e-4 for v in errs.values()), str(errs)


def test_rgcn_gather_cpasync_subprocess():
    """The opt-in cp.async row gather of the fp32 grouped GEMM (WG_GATHER_CPASYNC=1,
    read once per process) on a mixed plan, where the Y GEMM gathers its A rows."""
    import os
    import subprocess
    import sys
    code = ("from tests.test_gpu_conv_rgcn import run, TOL\n"
            "import torch\n"
            "e, _ = run(policy='random', norm='right', self_loop=True)\n"
            "assert max(e.values()) <= TOL[torch.float32], e\n"
            "e, _ = run(policy='random', ints=True, fi=32)\n"
            "assert max(e.values()) == 0.0, e\n"
            "print('ok')\n")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], cwd=root, capture_output=True, text=True, timeout=600,
                       env=dict(os.environ, WG_GATHER_CPASYNC="1"))
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]
