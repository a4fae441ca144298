"""B200-native gTask graph-convolution layer (WiseGraph, EuroSys '24 hot path).

Python binding over the C ABI of ``include/wg.h`` (``libwg.so``).  PyTorch is
used for device memory, streams and process groups only; every step of the
layer runs in the library's CUDA kernels.  There is no CPU fallback.

    g = Graph(src, dst, num_vertices=V)                  # a1-a3 (GPU partition)
    conv = Conv(g, "sage", f_in, f_out, dtype=torch.bfloat16, fuse_relu=True)
    y = conv(x, params)                                  # autograd-aware
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _capi as C
from ._capi import WGError, TASK_DTYPE

__all__ = ["Graph", "Conv", "Comm", "GPart", "WGError", "TASK_DTYPE", "padded", "pad_to", "ld_of", "launch_count",
           "init_params", "partition_1d", "Adam"]


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, torch.Tensor):
        return ctypes.c_void_p(t.data_ptr())
    if isinstance(t, np.ndarray):
        return t.ctypes.data_as(ctypes.c_void_p)
    return t


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dt(dtype):
    if dtype == torch.float32:
        return C.WG_F32
    if dtype == torch.bfloat16:
        return C.WG_BF16
    raise WGError(f"unsupported dtype {dtype}")


def pitch(F: int, dtype) -> int:
    """Row pitch (elements) of a table the gathers read: rows of <= 32 / <= 64
    bytes padded to 32 / 64 bytes, longer rows to a multiple of 128 bytes, so
    a row touches the fewest 128-byte L2 lines -- random row gathers are
    bound by line accesses (profiles/r02/gran_probe.md)."""
    s = torch.empty((), dtype=dtype).element_size()
    b = F * s
    q = 32 if b <= 32 else 64 if b <= 64 else 128
    return -(-b // q) * q // s


def padded(rows: int, F: int, dtype, device="cuda", zero=True):
    """[rows x F] view of a [rows x pitch(F)] buffer."""
    ld = pitch(F, dtype)
    buf = (torch.zeros if zero else torch.empty)((rows, ld), dtype=dtype, device=device)
    return buf[:, :F]


def ld_of(t: torch.Tensor) -> int:
    if t.dim() != 2 or t.stride(1) != 1:
        raise WGError("vertex tensors must be 2-D row-major views")
    if (t.stride(0) * t.element_size()) % 16:
        raise WGError("row pitch must be a multiple of 16 bytes (use padded())")
    return t.stride(0)


def pad_to(t: torch.Tensor) -> torch.Tensor:
    """Return a view of ``t`` whose row pitch satisfies the ABI (copies if needed)."""
    if t.dim() == 2 and t.stride(1) == 1 and (t.stride(0) * t.element_size()) % 16 == 0 and t.stride(0) >= t.shape[1]:
        return t
    out = padded(t.shape[0], t.shape[1], t.dtype, t.device, zero=True)
    out.copy_(t)
    return out


def launch_count() -> int:
    return int(C.lib().wg_launch_count())


_xent_scratch = {}


def softmax_xent(logits: torch.Tensor, labels: torch.Tensor, scale: float, dlogits: torch.Tensor,
                 loss: torch.Tensor, stream=None):
    """Fused softmax cross-entropy: loss[0] = scale * sum(-log p[label]); dlogits = scale * (p - onehot)."""
    dev = logits.device
    if dev not in _xent_scratch:
        _xent_scratch[dev] = torch.empty(C.XENT_SCRATCH_BYTES, dtype=torch.uint8, device=dev)
    C.check(C.lib().wg_softmax_xent(_dt(logits.dtype), logits.shape[0], logits.shape[1], _ptr(logits), ld_of(logits),
                                    _ptr(labels), scale, _ptr(dlogits), ld_of(dlogits), _ptr(loss),
                                    _ptr(_xent_scratch[dev]), _stream(stream)), "wg_softmax_xent")


class Adam:
    """Adam over every parameter of a model in one flat fp32 buffer: one
    wg_adam_step launch per step (torch.optim.Adam's update, no weight decay).
    The parameter dicts' tensors are replaced by views of the flat buffer and
    ``grads`` holds matching gradient views (what the conv backward writes).
    The step count lives on the device, so a captured step replays real steps."""

    ALIGN = 64          # floats: every tensor starts on a 256-byte boundary

    def __init__(self, params: list, lr: float = 1e-3, betas=(0.9, 0.999), eps: float = 1e-8):
        self.lr, self.betas, self.eps = float(lr), (float(betas[0]), float(betas[1])), float(eps)
        ts = [t for p in params for t in p.values()]
        if not ts:
            raise ValueError("Adam: no parameters")
        dev = ts[0].device
        offs, o = [], 0
        for t in ts:
            if t.dtype != torch.float32:
                raise ValueError("Adam: parameters must be fp32")
            offs.append(o)
            o += -(-t.numel() // self.ALIGN) * self.ALIGN
        self.n = o
        self.param = torch.zeros(o, dtype=torch.float32, device=dev)
        self.grad = torch.zeros_like(self.param)
        self.exp_avg = torch.zeros_like(self.param)
        self.exp_avg_sq = torch.zeros_like(self.param)
        self.state = torch.zeros(2, dtype=torch.int32, device=dev)
        self.grads = []
        i = 0
        for p in params:
            gd = {}
            for k, t in list(p.items()):
                a, n = offs[i], t.numel()
                view = self.param[a:a + n].view(t.shape)
                view.copy_(t.detach())
                p[k] = view
                gd[k] = self.grad[a:a + n].view(t.shape)
                i += 1
            self.grads.append(gd)

    def step(self, stream=None):
        C.check(C.lib().wg_adam_step(self.n, _ptr(self.param), _ptr(self.grad), _ptr(self.exp_avg),
                                     _ptr(self.exp_avg_sq), _ptr(self.state), self.lr, self.betas[0],
                                     self.betas[1], self.eps, _stream(stream)), "wg_adam_step")


def profile(cmd: str):
    """'start' | 'stop' | 'collect' -> {kind: {ms, launches, bytes, flops}} (wg_profile)."""
    L = C.lib()
    if cmd in ("start", "stop"):
        C.check(L.wg_profile(1 if cmd == "start" else 0, None), "wg_profile")
        return None
    out = (ctypes.c_double * (4 * len(C.PROF_KINDS)))()
    C.check(L.wg_profile(2, out), "wg_profile")
    return {k: {"ms": out[4 * i], "launches": int(out[4 * i + 1]), "bytes": out[4 * i + 2], "flops": out[4 * i + 3]}
            for i, k in enumerate(C.PROF_KINDS)}


class Comm:
    """Communicator of the 1-D multi-GPU layer (wg_comm_*): NCCL over the
    ranks of a torch.distributed group (the 128-byte id is broadcast through
    it), or the one-GPU emulation of one rank (emulate=(rank, world); with
    emulate_copy the exchanges are timed as copy kernels, else skipped)."""

    def __init__(self, group=None, *, device: int | None = None, emulate=None, emulate_copy: bool = True):
        L = C.lib()
        self.device = torch.cuda.current_device() if device is None else device
        h = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            if emulate is not None:
                self.rank, self.world = emulate
                C.check(L.wg_comm_init_emulated(self.rank, self.world, self.device, int(emulate_copy),
                                                ctypes.byref(h)),
                        "wg_comm_init_emulated")
            else:
                import torch.distributed as dist
                self.rank, self.world = dist.get_rank(group), dist.get_world_size(group)
                uid = torch.zeros(C.COMM_ID_BYTES, dtype=torch.uint8)
                if self.rank == 0:
                    C.check(L.wg_comm_unique_id(_ptr(uid)), "wg_comm_unique_id")
                dev = torch.device("cuda", self.device) if dist.get_backend(group) == "nccl" else torch.device("cpu")
                u = uid.to(dev)
                dist.broadcast(u, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
                uid = u.cpu().contiguous()
                C.check(L.wg_comm_init(_ptr(uid), self.rank, self.world, self.device, ctypes.byref(h)),
                        "wg_comm_init")
        self._h = h
        self.emulated = emulate is not None

    @classmethod
    def single(cls, device: int | None = None):
        """A one-rank NCCL communicator (no process group needed)."""
        c = cls.__new__(cls)
        L = C.lib()
        c.device = torch.cuda.current_device() if device is None else device
        uid = torch.zeros(C.COMM_ID_BYTES, dtype=torch.uint8)
        h = ctypes.c_void_p()
        with torch.cuda.device(c.device):
            C.check(L.wg_comm_unique_id(_ptr(uid)), "wg_comm_unique_id")
            C.check(L.wg_comm_init(_ptr(uid), 0, 1, c.device, ctypes.byref(h)), "wg_comm_init")
        c._h, c.rank, c.world, c.emulated = h, 0, 1, False
        return c

    @property
    def handle(self):
        return self._h

    def wait(self, stream=None):
        """The current (or given) stream waits for outstanding communication
        (the gradient all-reduce left running by backward_dist)."""
        C.check(C.lib().wg_comm_wait(self._h, _stream(stream)), "wg_comm_wait")

    def close(self):
        if getattr(self, "_h", None):
            C.lib().wg_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _graph_desc(src, dst, num_vertices, indptr, etype, num_types, tile_rows, max_task_edges, v_begin, v_end, keep):
    def arr(a, dt):
        if a is None:
            return None
        if isinstance(a, torch.Tensor):
            a = a.to(dt).contiguous()
        else:
            a = np.ascontiguousarray(a, dtype={torch.int32: np.int32, torch.int64: np.int64}[dt])
        keep.append(a)
        return a

    s = arr(src, torch.int32)
    d = arr(dst, torch.int32)
    ip = arr(indptr, torch.int64)
    et = arr(etype, torch.int32)
    E = (s.shape[0] if s is not None else 0)
    return C.GraphDesc(num_vertices, E, _ptr(ip), _ptr(s), _ptr(d), _ptr(et), num_types, tile_rows,
                       max_task_edges, v_begin, v_end)


def partition_1d(src, dst=None, *, num_vertices: int, world: int, indptr=None, tile_rows: int = 128):
    """Edge-balanced T-aligned 1-D partition bounds [world + 1] (wg_partition_1d,
    a host computation: works without a GPU for host arrays)."""
    keep = []
    desc = _graph_desc(src, dst, num_vertices, indptr, None, 1, tile_rows, 0, 0, 0, keep)
    b = np.zeros(world + 1, np.int64)
    C.check(C.lib().wg_partition_1d(ctypes.byref(desc), world, _ptr(b)), "wg_partition_1d")
    return b


class Graph:
    """Device graph + forward / transposed gTask partitions (wg_graph_create;
    with comm=, this rank's block of the 1-D partition, wg_graph_create_dist)."""

    def __init__(self, src, dst=None, *, num_vertices: int, indptr=None, etype=None, num_types: int = 1,
                 tile_rows: int = 128, max_task_edges: int = 0, v_begin: int = 0, v_end: int = 0,
                 device: int | None = None, stream=None, comm: Comm | None = None, bounds=None):
        L = C.lib()
        self._keep = []
        desc = _graph_desc(src, dst, num_vertices, indptr, etype, num_types, tile_rows, max_task_edges,
                           v_begin, v_end, self._keep)
        self.device = (comm.device if comm is not None else torch.cuda.current_device()) if device is None else device
        h = ctypes.c_void_p()
        self.comm = comm
        with torch.cuda.device(self.device):
            if comm is not None:
                b = None if bounds is None else np.ascontiguousarray(bounds, dtype=np.int64)
                vb, ve = ctypes.c_int64(), ctypes.c_int64()
                C.check(L.wg_graph_create_dist(comm.handle, ctypes.byref(desc), _ptr(b), self.device,
                                               _stream(stream), ctypes.byref(h), ctypes.byref(vb),
                                               ctypes.byref(ve)), "wg_graph_create_dist")
                v_begin = vb.value if comm.world > 1 else 0
            else:
                C.check(L.wg_graph_create(ctypes.byref(desc), self.device, _stream(stream), ctypes.byref(h)),
                        "wg_graph_create")
        self._h = h
        self._keep = []
        info = (ctypes.c_int64 * 10)()
        C.check(L.wg_graph_info(self._h, info), "wg_graph_info")
        (self.V, self.n_rows, self.E_fwd, self.E_T, self.n_tasks, self.n_tasks_T, self.T, self.E_max,
         self.by_type, self.max_in_degree) = list(info)
        self.v_begin = v_begin
        self.num_types = num_types
        self._plans = 0
        self.bounds = None
        if comm is not None:
            b = np.zeros(comm.world + 1, np.int64)
            n = ctypes.c_int32()
            C.check(L.wg_graph_bounds(self._h, _ptr(b), ctypes.byref(n)), "wg_graph_bounds")
            self.bounds = b

    @property
    def handle(self):
        return self._h

    def export(self, transposed: bool = False):
        """(perm int64[E], tasks TASK_DTYPE[n], fwdpos or None) as numpy (host) arrays."""
        E = self.E_T if transposed else self.E_fwd
        n = self.n_tasks_T if transposed else self.n_tasks
        perm = np.empty(max(E, 1), np.int64)
        tasks = np.empty(max(n, 1), TASK_DTYPE)
        fwdpos = np.empty(max(E, 1), np.int64) if (transposed and self.n_rows == self.V) else None
        C.check(C.lib().wg_graph_export(self._h, int(transposed), _ptr(perm), _ptr(tasks), _ptr(fwdpos)),
                "wg_graph_export")
        return perm[:E], tasks[:n], (fwdpos[:E] if fwdpos is not None else None)

    def close(self):
        if getattr(self, "_h", None):
            C.check(C.lib().wg_graph_destroy(self._h), "wg_graph_destroy")
            self._h = None

    def __del__(self):
        try:
            if getattr(self, "_h", None) and self._plans == 0:
                C.lib().wg_graph_destroy(self._h)
                self._h = None
        except Exception:
            pass


class GPart:
    """General restriction engine (wg_gpart_*): gTasks of any uniq() restriction
    set over dst / src / type / dst_degree / edge (Fig 7), and
    the atomic Index / Index-add executor over them.

        gp = GPart(src, dst, num_vertices=V, restrictions=[("src", 32), ("type", 1)], etype=et)
        agg = gp.aggregate(x, norm="both")
    """

    def __init__(self, src, dst=None, *, num_vertices: int, restrictions=(), indptr=None, etype=None,
                 device: int | None = None, stream=None):
        L = C.lib()
        keep = []
        desc = _graph_desc(src, dst, num_vertices, indptr, etype, 1, 128, 0, 0, 0, keep)
        r = (ctypes.c_int32 * (2 * max(1, len(restrictions))))()
        for i, (a, k) in enumerate(restrictions):
            r[2 * i] = C.ATTRS[a]
            r[2 * i + 1] = C.UNIQ_MIN if k == "min" else int(k)
        self.device = torch.cuda.current_device() if device is None else device
        h = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            C.check(L.wg_gpart_create(ctypes.byref(desc), r, len(restrictions), self.device, _stream(stream),
                                      ctypes.byref(h)), "wg_gpart_create")
        self._h = h
        info = (ctypes.c_int64 * 3)()
        C.check(L.wg_gpart_info(h, info), "wg_gpart_info")
        self.V, self.E, self.n_tasks = list(info)

    def export(self):
        perm = np.empty(max(self.E, 1), np.int64)
        tasks = np.empty(max(self.n_tasks, 1), TASK_DTYPE)
        C.check(C.lib().wg_gpart_export(self._h, _ptr(perm), _ptr(tasks)), "wg_gpart_export")
        return perm[:self.E], tasks[:self.n_tasks]

    def aggregate(self, x, norm: str = "none", out=None, stream=None):
        F = x.shape[1]
        if out is None:
            out = padded(self.V, F, x.dtype, x.device, zero=False)
        ws = torch.empty(max(int(C.lib().wg_gpart_workspace(self._h, F)), 256), dtype=torch.uint8, device=x.device)
        C.check(C.lib().wg_gpart_aggregate(self._h, _dt(x.dtype), F, C.NORMS[norm], _ptr(x), ld_of(x), _ptr(out),
                                           ld_of(out), _ptr(ws), _stream(stream)), "wg_gpart_aggregate")
        return out

    def close(self):
        if getattr(self, "_h", None):
            C.lib().wg_gpart_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


PARAM_NAMES = C.PARAM_NAMES


class Conv:
    """One gTask graph-convolution layer bound to a graph (wg_plan_create)."""

    def __init__(self, graph: Graph, model: str, f_in: int, f_out: int, *, dtype=torch.float32, heads: int = 1,
                 concat: bool = True, norm: str = "both", self_loop: bool = False, bias: bool = True,
                 fuse_relu: bool = False, gin_eps: float = 0.0, neg_slope: float = 0.2, policy: str = "auto",
                 seed: int = 0, need_dx: bool = True, x_replicated: bool = False):
        self.graph = graph
        self.model = model
        self.f_in, self.f_out, self.heads, self.concat = f_in, f_out, heads, concat
        self.dtype = dtype
        self.fuse_relu = fuse_relu
        self.bias = bias
        self.need_dx = need_dx
        self.desc = C.ConvDesc(C.MODELS[model], _dt(dtype), f_in, f_out, heads, int(concat), C.NORMS[norm],
                               int(self_loop), int(bias), int(fuse_relu), gin_eps, neg_slope, C.POLICIES[policy],
                               seed, int(need_dx), int(x_replicated))
        h = ctypes.c_void_p()
        self.comm = graph.comm
        if self.comm is not None:   # one uniform plan on every rank (wg_plan_create_dist)
            C.check(C.lib().wg_plan_create_dist(self.comm.handle, graph.handle, ctypes.byref(self.desc),
                                                ctypes.byref(h)), "wg_plan_create_dist")
        else:
            C.check(C.lib().wg_plan_create(graph.handle, ctypes.byref(self.desc), ctypes.byref(h)), "wg_plan_create")
        self._h = h
        graph._plans += 1
        sb, wb = ctypes.c_size_t(), ctypes.c_size_t()
        C.check(C.lib().wg_plan_sizes(self._h, ctypes.byref(sb), ctypes.byref(wb)), "wg_plan_sizes")
        self.saved_bytes, self.ws_bytes = sb.value, wb.value
        dev = torch.device("cuda", graph.device)
        self.workspace = torch.empty(max(self.ws_bytes, 256), dtype=torch.uint8, device=dev)
        stats = (ctypes.c_int64 * 8)()
        C.check(C.lib().wg_plan_export(self._h, None, stats), "wg_plan_export")
        (self.n_edge_tasks, self.n_vertex_tasks, self.bwd_path, self.xchg_fwd, self.xchg_bwd, self.n_items,
         self.n_items_T, self.n_split_rows) = list(stats)
        self.out_dim = heads * f_out if (model == "gat" and concat) else f_out

    def plan_bits(self) -> np.ndarray:
        out = np.empty(max(self.graph.n_tasks, 1), np.uint8)
        C.check(C.lib().wg_plan_export(self._h, _ptr(out), None), "wg_plan_export")
        return out[: self.graph.n_tasks]

    def buffer_view(self, buf: torch.Tensor, name: str, rows: int, F: int, which: int = 0) -> torch.Tensor:
        """[rows x F] view of the named sub-buffer of `saved` (which=0) or the workspace (1)."""
        off = ctypes.c_size_t()
        C.check(C.lib().wg_plan_buffer(self._h, which, name.encode(), ctypes.byref(off)), "wg_plan_buffer")
        es = torch.empty((), dtype=self.dtype).element_size()
        ld = pitch(F, self.dtype)
        raw = buf[off.value: off.value + rows * ld * es]
        return raw.view(self.dtype).view(rows, ld)[:, :F]

    def xchg_info(self, direction: int):
        """(rows, chunk pitch, chunks, bytes) of the forward (0) / backward (1) exchange table."""
        info = (ctypes.c_int64 * 4)()
        C.check(C.lib().wg_plan_xchg(self._h, direction, info), "wg_plan_xchg")
        return tuple(int(v) for v in info)

    def new_xchg(self, direction: int):
        """The caller-owned exchange table ([chunks x rows x pitch] in the conv
        dtype, returned as a [chunks * rows x pitch] tensor; ld_xchg = pitch),
        or None if the layer exchanges no table in that direction."""
        rows, ld, chunks, nbytes = self.xchg_info(direction)
        if nbytes == 0:
            return None
        return torch.zeros((chunks * rows, ld), dtype=self.dtype, device=self.workspace.device)

    def new_saved(self):
        return torch.empty(max(self.saved_bytes, 256), dtype=torch.uint8, device=self.workspace.device)

    # ------------------------------------------------------------------ raw calls
    def forward_raw(self, x, params: dict, y=None, saved=None, phase=C.PHASE_ALL, xchg=None, stream=None):
        rows = self.graph.n_rows
        if y is None:
            y = padded(rows, self.out_dim, self.dtype, x.device, zero=False)
        if saved is None:
            saved = self.new_saved()
        pr = C.Params(*[_ptr(params.get(n)) for n in PARAM_NAMES])
        a = C.FwdArgs(phase, _ptr(x), ld_of(x), _ptr(y), ld_of(y), _ptr(saved), _ptr(self.workspace),
                      _ptr(xchg), ld_of(xchg) if xchg is not None else 0)
        C.check(C.lib().wg_conv_forward(self._h, ctypes.byref(pr), ctypes.byref(a), _stream(stream)),
                "wg_conv_forward")
        return y, saved

    def backward_raw(self, dy, x, y, saved, params: dict, dx=None, phase=C.PHASE_ALL, xchg=None, stream=None,
                     grads: dict | None = None, dx_mask=None, dy_masked: bool = False):
        """dx_mask: write dx already multiplied by [dx_mask > 0] (fusing the previous
        layer's ReLU backward); dy_masked: dy already carries this layer's ReLU mask."""
        dev = dy.device
        if grads is None:
            grads = {n: torch.empty_like(params[n], dtype=torch.float32) for n in PARAM_NAMES
                     if params.get(n) is not None}
        if self.need_dx and dx is None:
            dx = padded(self.graph.n_rows, self.f_in, self.dtype, dev, zero=False)
        pr = C.Params(*[_ptr(params.get(n)) for n in PARAM_NAMES])
        gr = C.Grads(*[_ptr(grads.get(n)) for n in PARAM_NAMES])
        a = C.BwdArgs(phase, _ptr(dy), ld_of(dy), _ptr(x), ld_of(x), _ptr(y), ld_of(y) if y is not None else 0,
                      _ptr(saved), _ptr(dx), ld_of(dx) if dx is not None else 0, _ptr(self.workspace),
                      _ptr(xchg), ld_of(xchg) if xchg is not None else 0,
                      _ptr(dx_mask), ld_of(dx_mask) if dx_mask is not None else 0, int(dy_masked))
        C.check(C.lib().wg_conv_backward(self._h, ctypes.byref(pr), ctypes.byref(a), ctypes.byref(gr),
                                         _stream(stream)), "wg_conv_backward")
        return dx, grads

    # ------------------------------------------------------------------ distributed
    def forward_dist(self, x, params: dict, y, saved, xchg=None, x_gathered: bool = False, stream=None):
        """wg_conv_forward_dist: exchange + forward of this rank's rows (see include/wg.h)."""
        pr = C.Params(*[_ptr(params.get(n)) for n in PARAM_NAMES])
        a = C.FwdArgs(C.PHASE_ALL, _ptr(x), ld_of(x), _ptr(y), ld_of(y), _ptr(saved), _ptr(self.workspace),
                      _ptr(xchg), xchg.stride(0) if xchg is not None else 0)
        C.check(C.lib().wg_conv_forward_dist(self.comm.handle, self._h, ctypes.byref(pr), ctypes.byref(a),
                                             int(x_gathered), _stream(stream)), "wg_conv_forward_dist")
        return y

    def backward_dist(self, dy, x, y, saved, params: dict, dx=None, xchg=None, grads: dict | None = None,
                      dx_mask=None, dy_masked: bool = False, stream=None):
        """wg_conv_backward_dist; the gradients are all-reduced on the
        communicator's stream after return (Comm.wait before reading them)."""
        pr = C.Params(*[_ptr(params.get(n)) for n in PARAM_NAMES])
        gr = C.Grads(*[_ptr((grads or {}).get(n)) for n in PARAM_NAMES])
        a = C.BwdArgs(C.PHASE_ALL, _ptr(dy), ld_of(dy), _ptr(x), ld_of(x), _ptr(y), ld_of(y) if y is not None else 0,
                      _ptr(saved), _ptr(dx), ld_of(dx) if dx is not None else 0, _ptr(self.workspace),
                      _ptr(xchg), xchg.stride(0) if xchg is not None else 0,
                      _ptr(dx_mask), ld_of(dx_mask) if dx_mask is not None else 0, int(dy_masked))
        C.check(C.lib().wg_conv_backward_dist(self.comm.handle, self._h, ctypes.byref(pr), ctypes.byref(a),
                                              ctypes.byref(gr), _stream(stream)), "wg_conv_backward_dist")
        return dx

    # ------------------------------------------------------------------ autograd
    def __call__(self, x, params: dict):
        names = [n for n in PARAM_NAMES if params.get(n) is not None]
        return _ConvFn.apply(self, names, pad_to(x), *[params[n] for n in names])

    def close(self):
        if getattr(self, "_h", None):
            C.check(C.lib().wg_plan_destroy(self._h), "wg_plan_destroy")
            self._h = None
            self.graph._plans -= 1

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class _ConvFn(torch.autograd.Function):
    @staticmethod
    def forward(ctx, conv: Conv, names, x, *tensors):
        params = dict(zip(names, tensors))
        y, saved = conv.forward_raw(x, params)
        ctx.conv, ctx.names = conv, names
        ctx.save_for_backward(x, y, *tensors)
        ctx.saved_buf = saved
        return y

    @staticmethod
    def backward(ctx, dy):
        conv = ctx.conv
        x, y, *tensors = ctx.saved_tensors
        params = dict(zip(ctx.names, tensors))
        dx, grads = conv.backward_raw(pad_to(dy.contiguous() if dy.stride(1) != 1 else dy), x, y, ctx.saved_buf,
                                      params)
        return (None, None, dx if conv.need_dx else None, *[grads.get(n) for n in ctx.names])


def init_params(model: str, f_in: int, f_out: int, *, heads: int = 1, concat: bool = True, R: int = 1,
                self_loop: bool = False, bias: bool = True, device="cuda", seed: int = 0) -> dict:
    """Glorot-initialised fp32 master parameters for one layer (random init, no checkpoint)."""
    g = torch.Generator(device="cpu").manual_seed(seed)

    def glorot(*shape, fan_in, fan_out):
        lim = (6.0 / (fan_in + fan_out)) ** 0.5
        return ((torch.rand(*shape, generator=g) * 2 - 1) * lim).to(device)

    p = {}
    if model == "gat":
        p["W"] = glorot(f_in, heads * f_out, fan_in=f_in, fan_out=heads * f_out)
        p["attn_l"] = glorot(heads, f_out, fan_in=f_out, fan_out=1)
        p["attn_r"] = glorot(heads, f_out, fan_in=f_out, fan_out=1)
        if bias:
            p["bias"] = torch.zeros(heads * f_out if concat else f_out, device=device)
    elif model == "sage_lstm":   # PyTorch nn.LSTM init: U(-1/sqrt(H), 1/sqrt(H)), H = f_in
        k = 1.0 / f_in ** 0.5
        p["W"] = glorot(f_in, f_out, fan_in=f_in, fan_out=f_out)
        p["W_self"] = glorot(f_in, f_out, fan_in=f_in, fan_out=f_out)
        p["Wih"] = ((torch.rand(f_in, 4 * f_in, generator=g) * 2 - 1) * k).to(device)
        p["Whh"] = ((torch.rand(f_in, 4 * f_in, generator=g) * 2 - 1) * k).to(device)
        p["bl"] = ((torch.rand(4 * f_in, generator=g) * 2 - 1) * k).to(device)
        if bias:
            p["bias"] = torch.zeros(f_out, device=device)
    elif model == "rgcn":
        p["W"] = glorot(R, f_in, f_out, fan_in=f_in, fan_out=f_out)
        if self_loop:
            p["W_self"] = glorot(f_in, f_out, fan_in=f_in, fan_out=f_out)
        if bias:
            p["bias"] = torch.zeros(f_out, device=device)
    else:
        p["W"] = glorot(f_in, f_out, fan_in=f_in, fan_out=f_out)
        if model == "sage":
            p["W_self"] = glorot(f_in, f_out, fan_in=f_in, fan_out=f_out)
        if model == "gin":
            p["W2"] = glorot(f_out, f_out, fan_in=f_out, fan_out=f_out)
            p["b2"] = torch.zeros(f_out, device=device)
        if bias or model == "gin":
            p["bias"] = torch.zeros(f_out, device=device)
    return p
