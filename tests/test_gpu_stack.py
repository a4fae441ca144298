"""Multi-layer / multi-partition paths on one GPU.

* the fused softmax cross-entropy against its definition (numpy, fp64);
* the 1-D partition simulated on one GPU: P rank-partitions
  share one exchange table (each PRE phase writes its own rows, so the
  all-gather is implicit), then every POST phase runs; the concatenated rank
  outputs and the summed weight gradients must equal the single-partition
  layer (and hence the oracle, tested elsewhere);
* a short training run of GNNStack decreases the loss.
"""
import numpy as np
import pytest
import torch

import synth
from tests.util import f64, rel_err

pytestmark = pytest.mark.gpu


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


@pytest.mark.parametrize("graph_replay", [False, True])
def test_adam_matches_torch(graph_replay):
    """wg_adam_step (one launch over a flat buffer) == torch.optim.Adam over the
    same tensors for several steps; under CUDA-graph replay the device step
    count advances (bias corrections differ per step)."""
    m = wg()
    gen = torch.Generator().manual_seed(3)
    shapes = [(100, 256), (256,), (7, 33, 5), (3,)]
    params = [{f"t{i}": torch.randn(*sh, generator=gen).cuda() for i, sh in enumerate(shapes[:2])},
              {f"u{i}": torch.randn(*sh, generator=gen).cuda() for i, sh in enumerate(shapes[2:])}]
    ref = [{k: v.clone().requires_grad_(True) for k, v in p.items()} for p in params]
    opt_ref = torch.optim.Adam([v for p in ref for v in p.values()], lr=1e-2)
    opt = m.Adam(params, lr=1e-2)
    grads_seq = [[torch.randn(*t.shape, generator=gen).cuda() for p in params for t in p.values()] for _ in range(4)]
    flat_g = [g for p in opt.grads for g in p.values()]
    if graph_replay:
        src = [torch.empty_like(g) for g in flat_g]
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            cg = torch.cuda.CUDAGraph()
            with torch.cuda.graph(cg):
                for g, t in zip(flat_g, src):
                    g.copy_(t)
                opt.step()
        torch.cuda.current_stream().wait_stream(s)
    for gs in grads_seq:
        if graph_replay:
            for t, g in zip(src, gs):
                t.copy_(g)
            cg.replay()
        else:
            for g, t in zip(flat_g, gs):
                g.copy_(t)
            opt.step()
        for v, g in zip([v for p in ref for v in p.values()], gs):
            v.grad = g.clone()
        opt_ref.step()
    torch.cuda.synchronize()
    assert int(opt.state[0]) == len(grads_seq)
    for p, r in zip(params, ref):
        for k in p:
            torch.testing.assert_close(p[k], r[k].detach(), rtol=2e-5, atol=2e-6)


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("C", [7, 47, 172])
def test_softmax_xent(dtype, C):
    m = wg()
    M = 5000
    x = torch.from_numpy(synth.normal((M, C), seed=C, std=3.0)).to(dtype)
    lab = torch.from_numpy(np.random.default_rng(C).integers(0, C, M)).cuda()
    xd = m.pad_to(x.cuda())
    dl = m.padded(M, C, dtype)
    loss = torch.zeros(1, device="cuda")
    m.softmax_xent(xd, lab, 1.0 / M, dl, loss)
    xo = f64(x)
    p = np.exp(xo - xo.max(1, keepdims=True))
    p /= p.sum(1, keepdims=True)
    onehot = np.zeros_like(p)
    onehot[np.arange(M), lab.cpu().numpy()] = 1
    ref_loss = -np.log(p[np.arange(M), lab.cpu().numpy()]).sum() / M
    tol = 1e-4 if dtype == torch.float32 else 2e-2
    assert abs(loss.item() - ref_loss) / abs(ref_loss) < 1e-4
    assert rel_err(f64(dl), (p - onehot) / M) < tol


@pytest.mark.parametrize("model,policy", [("sage", "edge"), ("sage", "vertex"), ("gcn", "edge"), ("gin", "vertex")])
@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("graph", ["powerlaw", "star"])
def test_1d_partition_phases_match_single(model, policy, P, graph):
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    V, E, fi, fo = 3000, 40000, 48, 40
    dtype = torch.float32
    src, dst, _ = synth.make_graph(V, E, seed=31, alpha=0.6)
    if graph == "star":   # every edge into vertex 5: ranks > 0 own no in-edge (no forward gTask)
        dst = np.full(E, 5, np.int32)
    x = torch.from_numpy(synth.make_features(V, fi, seed=32)).cuda()
    dy = torch.from_numpy(synth.normal((V, fo), seed=33, std=0.2)).cuda()
    params = m.init_params(model, fi, fo, seed=3)
    ts, td = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda()
    # single partition reference (through the same library)
    g1 = m.Graph(ts, td, num_vertices=V)
    c1 = m.Conv(g1, model, fi, fo, dtype=dtype, policy=policy, fuse_relu=True)
    xd = m.pad_to(x)
    y1, s1 = c1.forward_raw(xd, params)
    dx1, gr1 = c1.backward_raw(m.pad_to(dy), xd, y1, s1, params)
    # P rank-partitions sharing one exchange table
    block, bounds = equal_blocks(V, P)
    Vt = block * P
    xt = m.padded(Vt, fi, dtype)
    xt[:V] = x
    ranks = []
    for p in range(P):
        vb, ve = bounds[p]
        g = m.Graph(ts, td, num_vertices=V, v_begin=vb, v_end=ve)
        c = m.Conv(g, model, fi, fo, dtype=dtype, policy=policy, fuse_relu=True)
        ranks.append((g, c, vb, ve))
    wf = m.pitch(fo, dtype)
    xf = m.padded(Vt, wf, dtype) if ranks[0][1].n_vertex_tasks else None
    yt = m.padded(Vt, fo, dtype)
    saved = [c.new_saved() for _, c, _, _ in ranks]
    for ph in (1, 2):
        for (g, c, vb, ve), sv in zip(ranks, saved):
            if xf is None and ph == 1:
                continue
            c.forward_raw(xt, params, y=yt[vb:ve], saved=sv, phase=ph if xf is not None else 0, xchg=xf)
    np.testing.assert_allclose(f64(yt[:V]), f64(y1), rtol=0, atol=1e-5 * max(1.0, f64(y1).max()))
    # backward: dy rows per rank, exchange table of dAgg (dAgg path) or dT (G path)
    bw = ranks[0][1]
    wb = m.pitch(fi if bw.bwd_path == 0 else fo, dtype)
    xb = m.padded(Vt, wb, dtype)
    dyt = m.padded(Vt, fo, dtype)
    dyt[:V] = dy
    dxt = m.padded(Vt, fi, dtype)
    grads = []
    for ph in (1, 2):
        for i, ((g, c, vb, ve), sv) in enumerate(zip(ranks, saved)):
            if ph == 1:
                grads.append({k: torch.zeros_like(v) for k, v in params.items()})
            c.backward_raw(dyt[vb:ve], xt, yt[vb:ve], sv, params, dx=dxt[vb:ve], phase=ph, xchg=xb, grads=grads[i])
    assert rel_err(f64(dxt[:V]), f64(dx1)) < 1e-5
    for k in gr1:
        tot = sum(gr[k] for gr in grads)
        assert rel_err(f64(tot), f64(gr1[k])) < 1e-5, k


def test_stack_relu_fusion_is_exact():
    """dx_mask / dy_masked fusion (adjacent layers) changes no value."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack
    V, E = 3000, 40000
    src, dst, _ = synth.make_graph(V, E, seed=43, alpha=0.6, symmetric=True)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V)
    x = m.padded(V, 24, torch.bfloat16)
    x.copy_(torch.from_numpy(synth.make_features(V, 24, seed=44)))
    dl = m.padded(V, 6, torch.bfloat16)
    dl.copy_(torch.from_numpy(synth.normal((V, 6), seed=45)))
    out = []
    for fuse in (False, True):
        st = GNNStack(g, "sage", [24, 40, 40, 6], dtype=torch.bfloat16, seed=5)
        st.fuse_masks = fuse
        st.forward(x)
        st.backward(dl)
        torch.cuda.synchronize()
        out.append([{k: v.clone() for k, v in gr.items()} for gr in st.grads])
    for a, b in zip(*out):
        for k in a:
            assert torch.equal(a[k], b[k]), k


@pytest.mark.parametrize("model", ["sage", "gcn", "gin", "gat", "rgcn"])
def test_stack_training_decreases_loss(model):
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack
    V, E = 4000, 60000
    R = 6 if model == "rgcn" else 1
    src, dst, et = synth.make_graph(V, E, seed=41, alpha=0.5, symmetric=R == 1, R=R)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V,
                etype=torch.from_numpy(et).cuda() if R > 1 else None, num_types=R)
    dims = [32, 64, 64, 8]
    kw = dict(heads=3) if model == "gat" else dict(R=R, conv_kw={"norm": "right", "self_loop": True}) \
        if model == "rgcn" else {}
    st = GNNStack(g, model, dims, dtype=torch.bfloat16, lr=1e-2, **kw)
    if model == "gat":     # hidden GAT layers read heads * dims[i] columns
        assert [c.f_in for c in st.convs] == [32, 192, 192] and st.h[1].shape[1] >= 192
    x = m.padded(V, 32, torch.bfloat16)
    x.copy_(torch.from_numpy(synth.make_features(V, 32, seed=42)))
    labels = torch.from_numpy(np.random.default_rng(1).integers(0, 8, V)).cuda()
    losses = [float(st.step(x, labels, V).item()) for _ in range(30)]
    # random labels: GCN / GAT (no self term) can only fit them through neighbours, slowly
    assert losses[-1] < losses[0] * (0.99 if model in ("gcn", "gat") else 0.9), losses


@pytest.mark.parametrize("model", ["sage", "gat", "rgcn"])
def test_stack_cuda_graph_replay_equals_eager(model):
    """bench.py times K replays of one CUDA-graph-captured step: the replays
    must do exactly what eager steps do (same kernels, deterministic), so the
    parameters after n replays equal those after n eager steps bit for bit."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack
    V, E = 3000, 40000
    R = 5 if model == "rgcn" else 1
    src, dst, et = synth.make_graph(V, E, seed=51, alpha=0.5, R=R)
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V,
                etype=torch.from_numpy(et).cuda() if R > 1 else None, num_types=R)
    kw = dict(heads=2) if model == "gat" else dict(R=R, conv_kw={"norm": "right", "self_loop": True}) \
        if model == "rgcn" else {}
    dtype = torch.float32 if model == "rgcn" else torch.bfloat16
    x = m.padded(V, 24, dtype)
    x.copy_(torch.from_numpy(synth.make_features(V, 24, seed=52)))
    labels = torch.from_numpy(np.random.default_rng(2).integers(0, 8, V)).cuda()
    runs = []
    for graph in (False, True):
        st = GNNStack(g, model, [24, 32, 8], dtype=dtype, lr=1e-2, seed=9, **kw)
        st.step(x, labels, V)                       # warm-up (buffers, attributes)
        torch.cuda.synchronize()
        if graph:
            side = torch.cuda.Stream()
            side.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(side):
                st.step(x, labels, V)
            torch.cuda.current_stream().wait_stream(side)
            torch.cuda.synchronize()
            cg = torch.cuda.CUDAGraph()
            with torch.cuda.graph(cg):
                loss = st.step(x, labels, V)
            for _ in range(3):
                cg.replay()
        else:                                       # warm-up + 4 = warm-up + side step + 3 replays
            for _ in range(4):
                loss = st.step(x, labels, V)
        torch.cuda.synchronize()
        runs.append(([v.detach().clone() for p in st.params for v in p.values()], float(loss.item())))
    (pa, la), (pb, lb) = runs
    assert la == lb
    for a, b in zip(pa, pb):
        assert torch.equal(a, b)


def test_stack_rank_slice_runs():
    """bench.py --rank-slice: one rank of a P-way 1-D partition on one GPU
    with the emulated communicator (exchanges are copy kernels on the
    communication stream, no data moves between ranks) trains with the rank's
    owned rows only, through the library's distributed entry points."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack, equal_blocks
    V, E, P = 6000, 80000, 4
    block, bounds = equal_blocks(V, P)
    vb, ve = bounds[1]
    src, dst = synth.make_graph_slice(V, E, vb, ve, seed=61, alpha=0.5)
    comm = m.Comm(emulate=(1, P))
    b = [lo for lo, _ in bounds] + [V]
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V, comm=comm, bounds=b)
    assert g.v_begin == vb and g.n_rows == ve - vb
    st = GNNStack(g, "sage", [24, 256, 256, 7], dtype=torch.bfloat16, lr=1e-2)
    assert st.dist and st.rank == 1 and st.rows == ve - vb
    assert any(t is not None for t in st.xchg_f + st.xchg_b)
    assert st.convs[1].xchg_info(1)[2] == 2      # 256 -> 256: a 512-byte exchanged row, 2 chunks
    x = m.padded(V, 24, torch.bfloat16)
    x.copy_(torch.from_numpy(synth.make_features(V, 24, seed=62)))
    labels = torch.from_numpy(np.random.default_rng(3).integers(0, 7, ve - vb)).cuda()
    losses = [float(st.step(x, labels, V).item()) for _ in range(20)]
    assert np.isfinite(losses).all() and losses[-1] < losses[0]
    assert st.h[-1].shape[0] == ve - vb and all(d.shape[0] == ve - vb for d in st.dx[1:])


@pytest.mark.parametrize("model,policy,F", [("sage", "vertex", 256), ("sage", "edge", 256), ("gcn", "vertex", 512),
                                            ("gcn", "edge", 128)])
def test_chunked_exchange_phases_match_single(model, policy, F):
    """Column-chunked exchange tables (wg_plan_xchg): P rank
    partitions on one GPU each write their rows of the chunked table (GEMM
    3-D store maps, chunked second output of the bias-gradient pass) in PRE,
    then every POST gathers chunk by chunk; the rank outputs and summed
    weight gradients equal the single-partition layer."""
    m = wg()
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    V, E, P = 3000, 40000, 3
    dtype = torch.bfloat16
    fi, fo = F, F
    src, dst, _ = synth.make_graph(V, E, seed=71, alpha=0.6)
    x = torch.from_numpy(synth.make_features(V, fi, seed=72)).to(dtype).cuda()
    dy = torch.from_numpy(synth.normal((V, fo), seed=73, std=0.2)).to(dtype).cuda()
    params = m.init_params(model, fi, fo, seed=7)
    ts, td = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda()
    g1 = m.Graph(ts, td, num_vertices=V)
    c1 = m.Conv(g1, model, fi, fo, dtype=dtype, policy=policy, fuse_relu=True)
    xd = m.pad_to(x)
    y1, s1 = c1.forward_raw(xd, params)
    dx1, gr1 = c1.backward_raw(m.pad_to(dy), xd, y1, s1, params)
    block, bounds = equal_blocks(V, P)
    ranks = []
    for p in range(P):
        vb, ve = bounds[p]
        g = m.Graph(ts, td, num_vertices=V, v_begin=vb, v_end=ve)
        c = m.Conv(g, model, fi, fo, dtype=dtype, policy=policy, fuse_relu=True)
        ranks.append((g, c, vb, ve, c.new_saved()))
    c0 = ranks[0][1]
    xf, xb = c0.new_xchg(0), c0.new_xchg(1)
    assert xb is not None and c0.xchg_info(1)[2] == min(4, F * 2 // 256)   # >= 256-byte chunks
    assert (xf is not None) == (policy == "vertex")
    if xf is not None:
        assert c0.xchg_info(0)[2] == min(4, F * 2 // 256)
    y = m.padded(V, fo, dtype)
    for ph in ((1, 2) if xf is not None else (0,)):
        for g, c, vb, ve, sv in ranks:
            c.forward_raw(xd, params, y=y[vb:ve], saved=sv, phase=ph, xchg=xf)
    torch.cuda.synchronize()
    assert rel_err(f64(y), f64(y1)) < 1e-2     # chunked gathers sum in another worker split
    dx = m.padded(V, fi, dtype)
    grads = [{k: torch.zeros_like(v) for k, v in params.items()} for _ in ranks]
    for ph in (1, 2):
        for (g, c, vb, ve, sv), gr in zip(ranks, grads):
            c.backward_raw(m.pad_to(dy)[vb:ve], xd, y[vb:ve], sv, params, dx=dx[vb:ve], phase=ph, xchg=xb, grads=gr)
    torch.cuda.synchronize()
    assert rel_err(f64(dx), f64(dx1)) < 1e-2
    for k in gr1:
        tot = sum(gr[k] for gr in grads)
        assert rel_err(f64(tot), f64(gr1[k])) < 1e-2, k   # G rows round to bf16 after another summation split


@pytest.mark.parametrize("model", ["sage", "gin", "rgcn"])
def test_nccl_world1_dist_calls_match_single(model):
    """The distributed entry points over a real one-rank NCCL communicator
    (ncclGetUniqueId / ncclCommInitRank through the library's dlopen'd NCCL)
    give the single-partition results bit for bit."""
    m = wg()
    V, E, fi, fo, R = 2000, 25000, 64, 48, 4
    src, dst, et = synth.make_graph(V, E, seed=81, alpha=0.6, R=R if model == "rgcn" else 1)
    dtype = torch.bfloat16
    ts, td = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda()
    tt = torch.from_numpy(et).cuda() if model == "rgcn" else None
    kw = dict(etype=tt, num_types=R) if model == "rgcn" else {}
    ckw = dict(norm="right", self_loop=True) if model == "rgcn" else {}
    params = m.init_params(model, fi, fo, R=R, self_loop=model == "rgcn", seed=8)
    x = m.pad_to(torch.from_numpy(synth.make_features(V, fi, seed=82)).to(dtype).cuda())
    dy = m.pad_to(torch.from_numpy(synth.normal((V, fo), seed=83, std=0.2)).to(dtype).cuda())
    g1 = m.Graph(ts, td, num_vertices=V, **kw)
    c1 = m.Conv(g1, model, fi, fo, dtype=dtype, fuse_relu=True, **ckw)
    y1, s1 = c1.forward_raw(x, params)
    dx1, gr1 = c1.backward_raw(dy, x, y1, s1, params)
    comm = m.Comm.single()
    g = m.Graph(ts, td, num_vertices=V, comm=comm, **kw)
    assert list(g.bounds) == [0, V]
    c = m.Conv(g, model, fi, fo, dtype=dtype, fuse_relu=True, **ckw)
    y = m.padded(V, fo, dtype)
    sv = c.new_saved()
    c.forward_dist(x, params, y, sv, x_gathered=True)
    dx = m.padded(V, fi, dtype)
    gr = {k: torch.zeros_like(v) for k, v in params.items()}
    c.backward_dist(dy, x, y, sv, params, dx=dx, grads=gr)
    comm.wait()
    torch.cuda.synchronize()
    assert torch.equal(y, y1) and torch.equal(dx, dx1)
    for k in gr1:
        assert torch.equal(gr[k], gr1[k]), k
    comm.close()
