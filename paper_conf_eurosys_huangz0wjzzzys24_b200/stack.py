"""Multi-layer full-graph training step over the gTask layer (single GPU and
the 1-D multi-GPU partition of SURVEY §8(e)).

Forward: layer i reads the previous activation table and writes its own rows
straight into the next layer's table.  Distributed (one process per GPU):
rank p owns the T-aligned vertex block [b_p, b_{p+1}) of every activation and
gradient table (edge-balanced bounds, wg_partition_1d); tables the next layer
gathers hold all V rows.

* Library path (the product path): the graph carries a ``Comm`` (NCCL over
  the ranks, or the one-GPU emulation of one rank).  Each layer is one
  ``wg_conv_forward_dist`` / ``wg_conv_backward_dist`` call: the library
  exchanges the table its gathers read over NCCL on its communication stream
  -- the activation itself for EDGE layers, Y = h W for VERTEX layers
  (transform before communicate, Fig 11c), dT / dAgg in the
  backward -- column-chunked so the gather of one chunk overlaps the exchange
  of the next, and all-reduces the weight gradients under the next layer's
  backward.  The plan of every layer is one uniform plan on all ranks
  (wg_plan_create_dist).
* torch.distributed path (multi-process CPU tests of this orchestration with
  the test-only layers of tests/test_dist_gloo.py): the same PRE / exchange /
  POST sequence with torch.distributed collectives (all-gather-v as one
  broadcast per rank block) and a per-layer plan vote.
"""
from __future__ import annotations

import torch

from . import Adam, Conv, Graph, init_params, padded, pitch, softmax_xent
from . import _capi as C


class GNNStack:
    """L gTask layers (hidden ReLU fused into the layer epilogue) + CE loss + Adam."""

    def __init__(self, graph: Graph, model: str, dims, *, dtype=torch.bfloat16, heads: int = 1, policy="auto",
                 seed: int = 0, lr: float = 1e-3, group=None, bounds=None, R: int = 1,
                 conv_kw: dict | None = None, conv_factory=None, device=None):
        # conv_kw: extra Conv options for every layer (e.g. RGCN norm / self_loop).
        # group / bounds / conv_factory / device: the torch.distributed path
        # (tests/test_dist_gloo.py); the product path takes the communicator
        # and the partition from the graph (Graph(..., comm=Comm(...))).
        Conv_ = conv_factory or Conv
        self.g, self.model, self.dims, self.dtype = graph, model, list(dims), dtype
        self.L = len(dims) - 1
        self.dev = device if device is not None else torch.device("cuda", graph.device)
        self.comm = getattr(graph, "comm", None)
        self.group = group
        self.tdist = self.comm is None and group is not None and torch.distributed.get_world_size(group) > 1
        if self.comm is not None:
            self.world, self.rank = self.comm.world, self.comm.rank
        elif self.tdist:
            self.world, self.rank = torch.distributed.get_world_size(group), torch.distributed.get_rank(group)
        else:
            self.world, self.rank = 1, 0
        self.dist = self.world > 1
        self.bounds = [int(b) for b in (graph.bounds if self.comm is not None else bounds)] if self.dist else None
        self.rows = graph.n_rows
        self.vb = graph.v_begin
        self.V = graph.V
        self.convs, self.params = [], []
        self.vertex_layer = []
        # layer i reads a table of width f_in(i): dims[0], then the previous
        # layer's output width (heads * dims[i] for concatenated GAT heads)
        self.f_in = [dims[0]] + [heads * dims[i] if model == "gat" else dims[i] for i in range(1, self.L)]
        for i in range(self.L):
            last = i == self.L - 1
            kw = dict(dtype=dtype, fuse_relu=not last, need_dx=i > 0, seed=seed + i, **(conv_kw or {}))
            if conv_factory is None:
                kw["x_replicated"] = i == 0          # the input features are on every rank
            if model == "gat":
                kw.update(heads=heads, concat=not last)
            fi = self.f_in[i]
            conv = Conv_(graph, model, fi, dims[i + 1], policy=policy, **kw)
            if self.tdist and model != "rgcn":
                conv = self._vote(conv, Conv_, graph, model, fi, dims[i + 1], policy, kw)
            # a VERTEX layer exchanges Y; a rank with no gTask follows the agreed policy (G path)
            self.vertex_layer.append(model != "rgcn" and (conv.n_vertex_tasks > 0 or (
                conv.n_edge_tasks == 0 and getattr(conv, "bwd_path", 0) == 1)))
            self.convs.append(conv)
            self._share_workspace(conv)
            self.params.append(init_params(model, fi, dims[i + 1], heads=heads, concat=not last, R=R,
                                           self_loop=bool((conv_kw or {}).get("self_loop", False)),
                                           bias=bool((conv_kw or {}).get("bias", True)),
                                           device=self.dev, seed=seed + 100 + i))
        # activation tables: h[0] = input, h[i+1] = output of layer i (all V
        # rows when distributed: the next layer gathers them; the logits of
        # the last layer are never exchanged, so that table holds owned rows)
        self.h = [None] + [padded(self.V if i + 1 < self.L else self.rows, c.out_dim, dtype, self.dev)
                           for i, c in enumerate(self.convs)]
        self.saved = [c.new_saved() for c in self.convs]
        # dx of layer i (= dy of layer i-1): owned rows only (the exchange
        # tables carry what other ranks read)
        self.dx = [None] + [padded(self.rows, self.f_in[i], dtype, self.dev) for i in range(1, self.L)]
        # optimizer: on the GPU the library's fused Adam (one launch over one
        # flat buffer; params / grads become views of it); the CPU orchestration
        # tests (test-only layers on gloo) use torch's
        if self.dev.type == "cuda":
            self.opt = Adam(self.params, lr=lr)
            self.grads = self.opt.grads
        else:
            self.grads = [{k: torch.zeros_like(v) for k, v in p.items()} for p in self.params]
        self.xchg_f, self.xchg_b = [], []
        for i, c in enumerate(self.convs):
            if self.comm is not None and self.dist:
                self.xchg_f.append(c.new_xchg(0))
                self.xchg_b.append(c.new_xchg(1))
            elif self.tdist:
                self.xchg_f.append(padded(self.V, pitch(c.f_out, dtype), dtype, self.dev)
                                   if self.vertex_layer[i] else None)
                # layer 0 on the dAgg path writes no exchange rows (need_dx = False)
                need_b = model == "rgcn" or getattr(c, "bwd_path", 0) == 1 or i > 0
                wb = c.f_out if (model == "rgcn" or getattr(c, "bwd_path", 0) == 1) else c.f_in
                self.xchg_b.append(padded(self.V, pitch(wb, dtype), dtype, self.dev) if need_b else None)
            else:
                self.xchg_f.append(None)
                self.xchg_b.append(None)
        if self.dev.type != "cuda":
            for p in self.params:
                for v in p.values():
                    v.requires_grad_(True)
            self.opt = torch.optim.Adam([v for p in self.params for v in p.values()], lr=lr)

    # -------------------------------------------------------------- helpers
    def _vote(self, conv, Conv_, graph, model, fi, fo, policy, kw):
        """torch.distributed path: every rank must run the same plan (the
        ranks exchange one table); the ranks' EDGE / VERTEX gTask counts are
        summed and the majority plan is rebuilt where it differs -- including
        on a rank with no gTask, which then follows the agreed policy."""
        ne, nv = conv.n_edge_tasks, conv.n_vertex_tasks
        dev = self.dev if torch.distributed.get_backend(self.group) == "nccl" else torch.device("cpu")
        votes = torch.tensor([ne, nv], dtype=torch.int64, device=dev)
        torch.distributed.all_reduce(votes, group=self.group)
        uni = "vertex" if int(votes[1]) > int(votes[0]) else "edge"
        if (uni == "vertex" and conv.n_edge_tasks) or (uni == "edge" and conv.n_vertex_tasks) or \
                (uni == "vertex" and not conv.n_vertex_tasks and policy != "vertex"):
            conv.close()
            conv = Conv_(graph, model, fi, fo, policy=uni, **kw)
        return conv

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

    # per-layer timing (bench.py): CUDA events on the current stream around each
    # layer's forward / backward when self.layer_events is a list
    layer_events = None

    def _mark(self, key):
        if self.layer_events is None:
            return None
        ev = torch.cuda.Event(enable_timing=True)
        ev.record()
        return (key, ev)

    def _close(self, m):
        if m is not None:
            ev = torch.cuda.Event(enable_timing=True)
            ev.record()
            self.layer_events.append((m[0], m[1], ev))

    def _own(self, t):
        return t[self.vb:self.vb + self.rows] if self.dist else t

    def _allgatherv(self, t):
        """torch.distributed path: every rank's row block of a [V x ld] table,
        in place (one broadcast per rank block: blocks differ in size)."""
        full = t.as_strided((self.V, t.stride(0)), (t.stride(0), 1))
        for q in range(self.world):
            b0, b1 = self.bounds[q], self.bounds[q + 1]
            blk = full[b0:b1]
            src = torch.distributed.get_global_rank(self.group, q) if self.group is not None else q
            torch.distributed.broadcast(blk, src=src, group=self.group)

    # -------------------------------------------------------------- forward / backward
    def forward(self, x):
        """x: [V x f0] (replicated input features); returns this rank's logits rows."""
        h = x
        for i, c in enumerate(self.convs):
            mk = self._mark(("fwd", i))
            y = self._out(i)
            if self.comm is not None and self.dist:
                c.forward_dist(h, self.params[i], y, self.saved[i], xchg=self.xchg_f[i], x_gathered=i == 0)
            elif self.tdist and self.vertex_layer[i]:
                xg = self.xchg_f[i]
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i], phase=C.PHASE_PRE, xchg=xg)
                self._allgatherv(xg)
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i], phase=C.PHASE_POST, xchg=xg)
            else:
                if self.tdist and i > 0:
                    self._allgatherv(h)             # EDGE / RGCN layers gather raw rows
                c.forward_raw(h, self.params[i], y=y, saved=self.saved[i])
            self._close(mk)
            h = self.h[i + 1]
        self.x = x
        return self.h[self.L]

    fuse_masks = True

    def backward(self, dlogits):
        g = dlogits
        masked = False
        for i in reversed(range(self.L)):
            mk = self._mark(("bwd", i))
            c = self.convs[i]
            xin = self.x if i == 0 else self.h[i]
            dx = self.dx[i] if i > 0 else None
            y = self._out(i)
            # fuse layer i-1's ReLU backward into layer i's dx epilogue
            fuse = self.fuse_masks and i > 0 and getattr(self.convs[i - 1], "fuse_relu", False)
            kw = dict(grads=self.grads[i], dy_masked=masked,
                      dx_mask=self._own(self.h[i]) if fuse else None)
            if self.comm is not None and self.dist:
                c.backward_dist(g, xin, y, self.saved[i], self.params[i], dx=dx, xchg=self.xchg_b[i], **kw)
            elif self.tdist and self.xchg_b[i] is not None:
                xb = self.xchg_b[i]
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, phase=C.PHASE_PRE, xchg=xb, **kw)
                self._allgatherv(xb)
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, phase=C.PHASE_POST, xchg=xb, **kw)
            else:
                c.backward_raw(g, xin, y, self.saved[i], self.params[i], dx=dx, **kw)
            self._close(mk)
            g = dx
            masked = fuse
        if self.comm is not None:
            self.comm.wait()                        # the gradient all-reduces left running by backward_dist
        elif self.tdist:
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
        if isinstance(self.opt, Adam):
            self.opt.step()           # the step count is on the device: a captured step replays real steps
        else:
            for p, gr in zip(self.params, self.grads):
                for k, v in p.items():
                    v.grad = gr[k]
            self.opt.step()
        return self._loss


def equal_blocks(V: int, world: int, T: int = 128):
    """Equal T-aligned vertex blocks: (block_rows, [(v_begin, v_end)] per rank).
    Used where only one rank's edges exist (the C5 rank slice, one-GPU phase
    simulations); the product partition is the edge-balanced wg_partition_1d."""
    block = -(-(-(-V // world)) // T) * T
    if (world - 1) * block >= V:
        raise ValueError(f"{world} ranks of {block} rows leave a rank without vertices (V = {V}, T = {T})")
    return block, [(p * block, min(V, (p + 1) * block)) for p in range(world)]
