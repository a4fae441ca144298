"""Multi-layer full-graph training step over the gTask layer (single GPU and
the 1-D multi-GPU partition of SURVEY §8(e)).

Forward: layer i reads the previous activation table and writes its own rows
straight into the next layer's table.  Distributed (one process per GPU,
torch.distributed / NCCL): rank p owns the T-aligned vertex block
[p*B, (p+1)*B) of every activation and gradient table; before a layer the
table its gathers read is all-gathered in place -- the activation itself for
EDGE (gather-then-transform) layers, or Y = h W for VERTEX layers when the
transformed rows are narrower (transform-before-communicate, P:L2279-2289,
Fig 11c).  Backward mirrors it: the per-layer PRE phase writes this rank's
rows of dAgg (or dT) into the exchange table, the table is all-gathered, and
the POST phase runs the transposed gather over the rank's out-edges.  Weight
gradients are all-reduced (sum).  Rows >= V in the last block are padding.
"""
from __future__ import annotations

import torch

from . import Conv, Graph, init_params, padded, pitch, softmax_xent
from . import _capi as C


class GNNStack:
    """L gTask layers (hidden ReLU fused into the layer epilogue) + CE loss + Adam."""

    def __init__(self, graph: Graph, model: str, dims, *, dtype=torch.bfloat16, heads: int = 1, policy="auto",
                 seed: int = 0, lr: float = 1e-3, group=None, block: int | None = None, R: int = 1,
                 conv_kw: dict | None = None, conv_factory=None, device=None, sim_world: int = 1):
        # conv_kw: extra Conv options for every layer (e.g. RGCN norm / self_loop).
        # conv_factory / device: injection points for the multi-process CPU test
        # of this orchestration (tests/test_dist_gloo.py); the product path uses
        # Conv (libwg.so) on the graph's CUDA device.
        # sim_world > 1 (no group): one rank of a sim_world-way 1-D partition
        # on one GPU -- the rank's own kernels (PRE / POST phases, exchange
        # tables) run, the collectives are skipped (timing of the per-rank
        # compute only; exchanged rows are not filled in).
        Conv_ = conv_factory or Conv
        self.g, self.model, self.dims, self.dtype = graph, model, list(dims), dtype
        self.L = len(dims) - 1
        self.dev = device if device is not None else torch.device("cuda", graph.device)
        self.group = group
        self.sim = group is None and sim_world > 1
        self.dist = (group is not None and torch.distributed.get_world_size(group) > 1) or self.sim
        self.world = torch.distributed.get_world_size(group) if group is not None else sim_world
        self.rank = torch.distributed.get_rank(group) if group is not None else (
            graph.v_begin // block if self.sim else 0)
        self.rows = graph.n_rows
        self.vb = graph.v_begin
        self.block = block if block is not None else self.rows
        self.Vtab = self.block * self.world if self.dist else graph.V
        self.convs, self.params = [], []
        # layer i reads a table of width f_in(i): dims[0], then the previous
        # layer's output width (heads * dims[i] for concatenated GAT heads)
        self.f_in = [dims[0]] + [heads * dims[i] if model == "gat" else dims[i] for i in range(1, self.L)]
        for i in range(self.L):
            last = i == self.L - 1
            kw = dict(dtype=dtype, fuse_relu=not last, need_dx=i > 0, seed=seed + i, **(conv_kw or {}))
            if model == "gat":
                kw.update(heads=heads, concat=not last)
            pol = policy
            fi = self.f_in[i]
            conv = Conv_(graph, model, fi, dims[i + 1], policy=pol, **kw)
            if self.dist and model != "rgcn":   # one uniform plan per layer, the same on every rank
                ne, nv = conv.n_edge_tasks, conv.n_vertex_tasks
                if group is not None:   # ranks plan their own rows: vote by gTask counts
                    dev = self.dev if torch.distributed.get_backend(group) == "nccl" else torch.device("cpu")
                    votes = torch.tensor([ne, nv], dtype=torch.int64, device=dev)
                    torch.distributed.all_reduce(votes, group=group)
                    ne, nv = (int(v) for v in votes.tolist())
                uni = "vertex" if nv > ne else "edge"
                if (conv.n_vertex_tasks if uni == "edge" else conv.n_edge_tasks) or \
                        (uni == "vertex" and not conv.n_vertex_tasks and pol != "vertex"):
                    pol = uni
                    conv.close()
                    conv = Conv_(graph, model, fi, dims[i + 1], policy=pol, **kw)
            self.convs.append(conv)
            self._share_workspace(conv)
            self.params.append(init_params(model, fi, dims[i + 1], heads=heads, concat=not last, R=R,
                                           self_loop=bool((conv_kw or {}).get("self_loop", False)),
                                           bias=bool((conv_kw or {}).get("bias", True)),
                                           device=self.dev, seed=seed + 100 + i))
        # activation tables: h[0] = input, h[i+1] = output of layer i (global
        # rows when distributed: the next layer gathers them; the logits of the
        # last layer are never exchanged, so that table holds the owned rows)
        self.h = [None] + [padded(self.Vtab if i + 1 < self.L else self.rows, c.out_dim, dtype, self.dev)
                           for i, c in enumerate(self.convs)]
        self.saved = [c.new_saved() for c in self.convs]
        # dx of layer i (= dy of layer i-1): owned rows only (the exchange
        # tables carry what other ranks read)
        self.dx = [None] + [padded(self.rows, self.f_in[i], dtype, self.dev) for i in range(1, self.L)]

        self.grads = [{k: torch.zeros_like(v) for k, v in p.items()} for p in self.params]
        self.xchg_f, self.xchg_b = [], []
        for c in self.convs:
            self.xchg_f.append(padded(self.Vtab, pitch(c.f_out, dtype), dtype, self.dev)
                               if self._fwd_xchg(c) else None)
            wb = (c.f_out if c.bwd_path == 1 else c.f_in)
            self.xchg_b.append(padded(self.Vtab, pitch(wb, dtype), dtype, self.dev) if self.dist else None)
        for p in self.params:
            for v in p.values():
                v.requires_grad_(True)
        # capturable: the step count lives on the device, so a whole training
        # step (library launches + Adam) can be captured in one CUDA graph
        self.opt = torch.optim.Adam([v for p in self.params for v in p.values()], lr=lr,
                                    capturable=self.dev.type == "cuda")

    # -------------------------------------------------------------- helpers
    def _share_workspace(self, conv):
        """One workspace for all layers: a layer's scratch lives only inside its
        forward / backward call (the PRE and POST phases of one layer are not
        interleaved with another layer's calls), so every layer uses the
        largest one; shared as each layer is created, so the per-layer buffers
        never coexist."""
        ws = getattr(conv, "workspace", None)
        if not isinstance(ws, torch.Tensor):
            return
        shared = getattr(self, "_ws", None)
        if shared is None or ws.numel() > shared.numel():
            self._ws = ws
            for c in self.convs:
                if isinstance(getattr(c, "workspace", None), torch.Tensor):
                    c.workspace = ws
        else:
            conv.workspace = shared
        if self.dev.type == "cuda":
            torch.cuda.empty_cache()

    def _out(self, i):
        """Rows of layer i's output table this rank writes."""
        return self._own(self.h[i + 1]) if i + 1 < self.L else self.h[self.L]

    def _fwd_xchg(self, c):
        """VERTEX layers exchange Y = h W (transform before communicate); RGCN
        (per-relation transforms) and EDGE layers gather the activation itself."""
        return self.dist and c.n_vertex_tasks > 0 and c.model != "rgcn"

    def _own(self, t):
        return t[self.vb:self.vb + self.rows] if self.dist else t

    def _allgather(self, t):
        if not self.dist or self.sim:
            return
        full = t.as_strided((self.Vtab, t.stride(0)), (t.stride(0), 1))
        mine = full[self.rank * self.block:(self.rank + 1) * self.block]
        torch.distributed.all_gather_into_tensor(full, mine, group=self.group)

    def forward(self, x):
        """x: [V_tab x f0] (replicated input features); returns this rank's logits rows."""
        h = x
        for i, c in enumerate(self.convs):
            y = self._out(i)
            if self._fwd_xchg(c):
                xg = self.xchg_f[i]
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i], phase=C.PHASE_PRE, xchg=xg)
                self._allgather(xg)
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i], phase=C.PHASE_POST, xchg=xg)
            else:
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i])
            if self.dist and i + 1 < self.L and not self._fwd_xchg(self.convs[i + 1]):
                self._allgather(self.h[i + 1])       # next EDGE / RGCN layer gathers raw rows
            h = self.h[i + 1]
        self.x = x
        return self.h[self.L]

    fuse_masks = True

    def backward(self, dlogits):
        g = dlogits
        masked = False
        for i in reversed(range(self.L)):
            c = self.convs[i]
            xin = self.x if i == 0 else self.h[i]
            dx = self.dx[i] if i > 0 else None
            y = self._out(i)
            # fuse layer i-1's ReLU backward into layer i's dx epilogue
            fuse = self.fuse_masks and i > 0 and getattr(self.convs[i - 1], "fuse_relu", False)
            kw = dict(grads=self.grads[i], dy_masked=masked,
                      dx_mask=self._own(self.h[i]) if fuse else None)
            if self.dist:
                xb = self.xchg_b[i]
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, phase=C.PHASE_PRE, xchg=xb, **kw)
                self._allgather(xb)
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, phase=C.PHASE_POST, xchg=xb, **kw)
            else:
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, **kw)
            g = dx
            masked = fuse
        if self.dist and not self.sim:
            flat = torch.cat([v.reshape(-1) for gr in self.grads for v in gr.values()])
            torch.distributed.all_reduce(flat, group=self.group)
            o = 0
            for gr in self.grads:
                for v in gr.values():
                    v.copy_(flat[o:o + v.numel()].view_as(v))
                    o += v.numel()

    def step(self, x, labels, n_global: int):
        """One epoch step: forward, CE loss (mean over all vertices), backward, Adam."""
        logits = self.forward(x)
        if not hasattr(self, "_dl"):
            self._dl = padded(self.rows, logits.shape[1], self.dtype, self.dev, zero=True)
            self._loss = torch.zeros(1, dtype=torch.float32, device=self.dev)
        softmax_xent(logits, labels, 1.0 / n_global, self._dl, self._loss)
        self.backward(self._dl)
        for p, gr in zip(self.params, self.grads):
            for k, v in p.items():
                v.grad = gr[k]
        self.opt.step()
        return self._loss


def partition_1d(V: int, world: int, T: int = 128):
    """Equal T-aligned vertex blocks: returns (block_rows, [(v_begin, v_end)] per rank)."""
    block = -(-(-(-V // world)) // T) * T
    return block, [(min(V, p * block), min(V, (p + 1) * block)) for p in range(world)]
