"""World-size-2 gloo test (CPU) of the 1-D multi-GPU orchestration (§8(e)).

GNNStack's torch.distributed path (the library's edge-balanced T-aligned
partition bounds from wg_partition_1d -- a host computation, no GPU -- PRE /
all-gather-v / POST exchange phases for forward and backward, exchanged table
= activation for EDGE layers or Y = x W for VERTEX layers, dAgg or dT in
backward, one agreed plan per layer, weight-gradient all-reduce) runs on two
CPU processes over gloo.  The layer compute is
a test-only float64 torch implementation of GraphSAGE (and of RGCN with
1/|N_v^r| normalisation and a self-loop: its forward reads the all-gathered
activation, its backward exchanges dT) that honours the library's phase contract (include/wg.h, wg_fwd_args / wg_bwd_args); the CUDA
kernels themselves are covered by tests/test_gpu_*.  Each rank's logits rows
and the all-reduced weight gradients must equal the single-process run."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth


class FakeGraph:
    def __init__(self, src, dst, V, vb=0, ve=None, etype=None):
        self.etype = None if etype is None else torch.from_numpy(etype).long()
        self.src, self.dst, self.V = torch.from_numpy(src).long(), torch.from_numpy(dst).long(), V
        self.v_begin, self.n_rows = vb, (V if ve is None else ve) - vb
        self.device = "cpu"


class FakeSage:
    """GraphSAGE-mean layer in float64 following the PRE/POST phase contract."""

    def __init__(self, graph, model, fi, fo, *, policy="edge", fuse_relu=False, need_dx=True, **kw):
        self.g, self.f_in, self.f_out, self.out_dim = graph, fi, fo, fo
        self.model = model
        self.n_vertex_tasks = 1 if policy == "vertex" else 0
        self.n_edge_tasks = 1 - self.n_vertex_tasks
        self.bwd_path = self.n_vertex_tasks
        self.fuse_relu, self.need_dx = fuse_relu, need_dx
        self.deg = torch.bincount(graph.dst, minlength=graph.V).clamp(min=1).double()
        vb, ve = graph.v_begin, graph.v_begin + graph.n_rows
        self.vb, self.ve = vb, ve
        self.inm = (graph.dst >= vb) & (graph.dst < ve)
        self.outm = (graph.src >= vb) & (graph.src < ve)

    def new_saved(self):
        return {}

    def close(self):
        pass

    def _mean_in(self, table):      # own dst rows: sum_{e in in(v)} table[s] / deg(v)
        s, d = self.g.src[self.inm], self.g.dst[self.inm]
        out = torch.zeros(self.ve - self.vb, table.shape[1], dtype=torch.float64)
        out.index_add_(0, d - self.vb, table[s] / self.deg[d, None])
        return out

    def _mean_out(self, table):     # own src rows: sum_{e in out(u)} table[d] / deg(d)
        s, d = self.g.src[self.outm], self.g.dst[self.outm]
        out = torch.zeros(self.ve - self.vb, table.shape[1], dtype=torch.float64)
        out.index_add_(0, s - self.vb, table[d] / self.deg[d, None])
        return out

    @torch.no_grad()     # the library writes through raw pointers: no autograd on these tables
    def forward_raw(self, x, params, y=None, saved=None, phase=0, xchg=None, stream=None):
        Ws, Wn, b = params["W_self"].double(), params["W"].double(), params["bias"].double()
        xo = x[self.vb:self.ve]
        if self.n_vertex_tasks:
            tab = xchg if xchg is not None else torch.zeros(self.g.V, self.f_out, dtype=torch.float64)
            if phase in (0, 1):
                tab[self.vb:self.ve, :self.f_out] = xo @ Wn
            if phase == 1:
                return y, saved
            out = xo @ Ws + self._mean_in(tab[:, :self.f_out]) + b
        else:
            agg = self._mean_in(x)
            saved["agg"] = agg
            out = xo @ Ws + agg @ Wn + b
        y[:] = torch.relu(out) if self.fuse_relu else out
        return y, saved

    @torch.no_grad()
    def backward_raw(self, dy, x, y, saved, params, dx=None, phase=0, xchg=None, grads=None, stream=None,
                     dx_mask=None, dy_masked=False):
        dx, grads = self._backward(dy, x, y, saved, params, dx, phase, xchg, grads)
        if dx is not None and dx_mask is not None and phase != 1:
            dx *= (dx_mask > 0)
        return dx, grads

    def _backward(self, dy, x, y, saved, params, dx, phase, xchg, grads):
        Ws, Wn = params["W_self"].double(), params["W"].double()
        xo = x[self.vb:self.ve]
        dT = dy * (y > 0) if self.fuse_relu else dy
        fi, fo = self.f_in, self.f_out
        if self.bwd_path == 0:
            tab = xchg if xchg is not None else torch.zeros(self.g.V, fi, dtype=torch.float64)
            if phase in (0, 1):
                grads["W"][:] = saved["agg"].T @ dT
                grads["W_self"][:] = xo.T @ dT
                grads["bias"][:] = dT.sum(0)
                if self.need_dx:
                    tab[self.vb:self.ve, :fi] = dT @ Wn.T
                    saved["dxs"] = dT @ Ws.T
            if phase == 1 or not self.need_dx:
                return dx, grads
            dx[:] = saved["dxs"] + self._mean_out(tab[:, :fi])
        else:
            tab = xchg if xchg is not None else torch.zeros(self.g.V, fo, dtype=torch.float64)
            if phase in (0, 1):
                tab[self.vb:self.ve, :fo] = dT
                grads["W_self"][:] = xo.T @ dT
                grads["bias"][:] = dT.sum(0)
            if phase == 1:
                return dx, grads
            G = self._mean_out(tab[:, :fo])
            grads["W"][:] = xo.T @ G
            if self.need_dx:
                dx[:] = G @ Wn.T + dT @ Ws.T
        return dx, grads


class FakeRgcn:
    """RGCN layer in float64 (c_e = 1/|in_r(dst)|, self-loop W_0, bias) following
    the RGCN phase contract: forward reads all rows of x (no exchange), backward
    PRE writes this rank's dT rows into the exchange table, POST gathers it."""

    def __init__(self, graph, model, fi, fo, *, fuse_relu=False, need_dx=True, **kw):
        self.g, self.f_in, self.f_out, self.out_dim, self.model = graph, fi, fo, fo, model
        self.n_vertex_tasks, self.n_edge_tasks, self.bwd_path = 1, 1, 1   # mixed plans are fine for RGCN
        self.fuse_relu, self.need_dx = fuse_relu, need_dx
        key = graph.dst * R + graph.etype
        cnt = torch.bincount(key, minlength=graph.V * R)
        self.c = 1.0 / cnt[key].double()                  # global |in_r(dst_e)|
        self.vb, self.ve = graph.v_begin, graph.v_begin + graph.n_rows
        self.inm = (graph.dst >= self.vb) & (graph.dst < self.ve)
        self.outm = (graph.src >= self.vb) & (graph.src < self.ve)

    def new_saved(self):
        return {}

    def close(self):
        pass

    @torch.no_grad()
    def forward_raw(self, x, params, y=None, saved=None, phase=0, xchg=None, stream=None):
        if phase == 1:
            return y, saved
        W, W0, b = params["W"].double(), params["W_self"].double(), params["bias"].double()
        m = self.inm
        s, d, t, c = self.g.src[m], self.g.dst[m], self.g.etype[m], self.c[m]
        msg = torch.einsum("ei,eio->eo", x[s], W[t]) * c[:, None]
        out = x[self.vb:self.ve] @ W0 + b
        out.index_add_(0, d - self.vb, msg)
        y[:] = torch.relu(out) if self.fuse_relu else out
        return y, saved

    @torch.no_grad()
    def backward_raw(self, dy, x, y, saved, params, dx=None, phase=0, xchg=None, grads=None, stream=None,
                     dx_mask=None, dy_masked=False):
        W, W0 = params["W"].double(), params["W_self"].double()
        fo = self.f_out
        dT = dy * (y > 0) if (self.fuse_relu and not dy_masked) else dy
        if xchg is None:                          # single process: the table is local
            xchg = torch.zeros(self.g.V, fo, dtype=torch.float64)
        if phase in (0, 1):
            xchg[self.vb:self.ve, :fo] = dT
            grads["W_self"][:] = x[self.vb:self.ve].T @ dT
            grads["bias"][:] = dT.sum(0)
        if phase == 1:
            return dx, grads
        m = self.outm
        s, d, t, c = self.g.src[m], self.g.dst[m], self.g.etype[m], self.c[m]
        gd = xchg[d, :fo] * c[:, None]
        dW = torch.zeros_like(W)
        dW.index_add_(0, t, torch.einsum("ei,eo->eio", x[s], gd))
        grads["W"][:] = dW
        if self.need_dx:
            out = dT @ W0.T
            out.index_add_(0, s - self.vb, torch.einsum("eo,eio->ei", gd, W[t]))
            dx[:] = out * (dx_mask > 0) if dx_mask is not None else out
        return dx, grads


def factory(graph, model, fi, fo, **kw):
    if model == "rgcn":
        return FakeRgcn(graph, model, fi, fo, **kw)
    kw["policy"] = "edge" if fi != 6 else "vertex"    # layer 2 of dims [8, 6, 6, 5] is a VERTEX layer
    return FakeSage(graph, model, fi, fo, **kw)


V, E, DIMS, R = 700, 6000, [8, 6, 6, 5], 3


def run_stack(graph, group, bounds, model="sage"):
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack
    torch.manual_seed(0)
    kw = dict(R=R, conv_kw={"self_loop": True}) if model == "rgcn" else {}
    st = GNNStack(graph, model, DIMS, dtype=torch.float64, group=group, bounds=bounds, conv_factory=factory,
                  device=torch.device("cpu"), seed=3, **kw)
    x = torch.zeros(V, DIMS[0], dtype=torch.float64)
    x[:V] = torch.from_numpy(synth.make_features(V, DIMS[0], seed=4)).double()
    logits = st.forward(x).clone()
    dl = torch.from_numpy(synth.normal((V, DIMS[-1]), seed=5)).double()
    vb = graph.v_begin
    st.backward(dl[vb:vb + graph.n_rows].clone())
    return logits, [{k: v.clone() for k, v in g.items()} for g in st.grads]


def worker(rank, world, port, q, model):
    os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import partition_1d
    src, dst, et = synth.make_graph(V, E, seed=9, alpha=0.5, symmetric=model != "rgcn", R=R if model == "rgcn" else 1)
    et = et if model == "rgcn" else None
    ref_logits, ref_grads = run_stack(FakeGraph(src, dst, V, etype=et), None, None, model)
    bounds = partition_1d(src, dst, num_vertices=V, world=world, tile_rows=128)
    vb, ve = int(bounds[rank]), int(bounds[rank + 1])
    logits, grads = run_stack(FakeGraph(src, dst, V, vb, ve, etype=et), dist.group.WORLD, bounds, model)
    ok = torch.allclose(logits, ref_logits[vb:ve], rtol=1e-10, atol=1e-12)
    for g1, g2 in zip(grads, ref_grads):      # fp32 gradients: all-reduce sums partials in another order
        for k in g1:
            ok &= torch.allclose(g1[k], g2[k], rtol=1e-5, atol=1e-6)
    q.put((rank, bool(ok), (vb, ve)))
    dist.destroy_process_group()


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("model", ["sage", "rgcn"])
@pytest.mark.parametrize("world", [2])
def test_gloo_1d_partition_matches_single(world, model):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, world, port, q, model)) for r in range(world)]
    for p in procs:
        p.start()
    res = []
    for _ in range(world):
        try:
            res.append(q.get(timeout=120))
        except Exception:
            break
    for p in procs:
        p.join(timeout=30)
        if p.is_alive():
            p.kill()
    assert len(res) == world, f"workers failed (exit codes {[p.exitcode for p in procs]})"
    assert all(r[1] for r in res), res
    assert sorted(r[2] for r in res)[0][0] == 0


def test_partition_1d_edge_balanced():
    """wg_partition_1d (host computation, no GPU): T-aligned, covering, every
    rank >= 1 tile, and each rank's in- + out-edges + rows within one tile's
    load of 1/world of the total (greedy nearest-boundary)."""
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import partition_1d
    for Vv, Ee, P, T in [(5000, 60000, 4, 128), (3000, 40000, 3, 128), (1000, 9000, 8, 64), (300, 2000, 2, 128)]:
        src, dst, _ = synth.make_graph(Vv, Ee, seed=Vv, alpha=0.8)
        b = partition_1d(src, dst, num_vertices=Vv, world=P, tile_rows=T)
        assert b[0] == 0 and b[-1] == Vv and all(b[i] < b[i + 1] for i in range(P))
        assert all(x % T == 0 for x in b[:-1])
        w = np.bincount(src, minlength=Vv) + np.bincount(dst, minlength=Vv) + 1
        loads = np.array([w[b[i]:b[i + 1]].sum() for i in range(P)])
        tile_max = max(w[t:t + T].sum() for t in range(0, Vv, T))
        assert np.abs(loads - w.sum() / P).max() <= tile_max + 1, (loads, w.sum() / P, tile_max)
    # CSR input gives the same bounds as COO; too few tiles is an error
    src, dst, _ = synth.make_graph(2000, 20000, seed=1, alpha=0.6)
    order = np.argsort(dst, kind="stable")
    indptr = np.concatenate([[0], np.cumsum(np.bincount(dst, minlength=2000))]).astype(np.int64)
    np.testing.assert_array_equal(partition_1d(src[order], None, num_vertices=2000, world=4, indptr=indptr),
                                  partition_1d(src, dst, num_vertices=2000, world=4))
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import WGError
    with pytest.raises(WGError):
        partition_1d(src, dst, num_vertices=2000, world=40)


def test_equal_blocks():
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    for Vv, P in [(2449029, 8), (1000, 3), (256, 2), (111059956, 8)]:
        block, b = equal_blocks(Vv, P)
        assert block % 128 == 0 and b[0][0] == 0 and b[-1][1] == Vv
        assert all(lo % 128 == 0 and lo < hi for lo, hi in b) and all(b[i][1] == b[i + 1][0] for i in range(P - 1))
    with pytest.raises(ValueError):
        equal_blocks(129, 4)
