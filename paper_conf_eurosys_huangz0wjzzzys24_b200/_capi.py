"""ctypes declarations of include/wg.h (argument marshalling only).

Loads the in-tree ``libwg.so``.  There is no fallback: if the library is
missing or fails to load, every entry point raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libwg.so")

WG_OK, WG_ERR_INVALID, WG_ERR_RANGE, WG_ERR_NOMEM, WG_ERR_CUDA, WG_ERR_UNSUPPORTED, WG_ERR_STATE = 0, 1, 2, 3, 4, 6, 7
MODELS = {"gcn": 0, "gin": 1, "sage": 2, "gat": 3, "rgcn": 4, "sage_lstm": 5}
NORMS = {"none": 0, "right": 1, "both": 2}
POLICIES = {"auto": 0, "edge": 1, "vertex": 2, "random": 3}
WG_F32, WG_BF16 = 0, 1
PHASE_ALL, PHASE_PRE, PHASE_POST = 0, 1, 2

# every symbol include/wg.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "wg_graph_create", "wg_graph_info", "wg_graph_export", "wg_graph_destroy",
    "wg_plan_create", "wg_plan_sizes", "wg_plan_export", "wg_plan_buffer", "wg_plan_destroy",
    "wg_conv_forward", "wg_conv_backward",
    "wg_status_string", "wg_last_error", "wg_launch_count", "wg_profile", "wg_softmax_xent", "wg_adam_step",
    "wg_comm_unique_id", "wg_comm_init", "wg_comm_init_emulated", "wg_comm_info", "wg_comm_wait",
    "wg_comm_destroy", "wg_partition_1d", "wg_graph_create_dist", "wg_graph_bounds", "wg_plan_create_dist",
    "wg_plan_xchg", "wg_conv_forward_dist", "wg_conv_backward_dist",
    "wg_gpart_create", "wg_gpart_info", "wg_gpart_export", "wg_gpart_workspace", "wg_gpart_aggregate",
    "wg_gpart_destroy",
]
ATTRS = {"dst": 0, "src": 1, "type": 2, "dst_degree": 3, "edge": 4}
UNIQ_MIN = -1
COMM_ID_BYTES = 128
XENT_SCRATCH_BYTES = 8192
PROF_KINDS = ["gather_reduce", "split_combine", "tc_gemm_nt", "tc_gemm_tn", "simt_gemm", "misc", "gat", "rgcn"]

P = ctypes.c_void_p
i32, i64, u64, f32 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_float


class GraphDesc(ctypes.Structure):
    _fields_ = [("num_vertices", i64), ("num_edges", i64), ("indptr", P), ("src", P), ("dst", P),
                ("etype", P), ("num_types", i32), ("tile_rows", i32), ("max_task_edges", i64),
                ("v_begin", i64), ("v_end", i64)]


TASK_DTYPE = np.dtype([
    ("tile", np.int32), ("type", np.int32), ("e_begin", np.int64), ("e_end", np.int64),
    ("d_lo", np.int32), ("d_hi", np.int32), ("flags", np.int32), ("n_uniq_src", np.int32),
])


class ConvDesc(ctypes.Structure):
    _fields_ = [("model", ctypes.c_int), ("dtype", ctypes.c_int), ("f_in", i32), ("f_out", i32), ("heads", i32),
                ("concat_heads", i32), ("norm", ctypes.c_int), ("self_loop", i32), ("bias", i32),
                ("fuse_relu", i32), ("gin_eps", f32), ("neg_slope", f32), ("policy", ctypes.c_int),
                ("policy_seed", u64), ("need_dx", i32), ("x_replicated", i32)]


PARAM_NAMES = ("W", "W_self", "bias", "attn_l", "attn_r", "W2", "b2", "Wih", "Whh", "bl")


class Params(ctypes.Structure):
    _fields_ = [(n, P) for n in PARAM_NAMES]


class Grads(ctypes.Structure):
    _fields_ = [(n, P) for n in PARAM_NAMES]


class FwdArgs(ctypes.Structure):
    _fields_ = [("phase", i32), ("x", P), ("ldx", i64), ("y", P), ("ldy", i64), ("saved", P),
                ("workspace", P), ("xchg", P), ("ld_xchg", i64)]


class BwdArgs(ctypes.Structure):
    _fields_ = [("phase", i32), ("dy", P), ("lddy", i64), ("x", P), ("ldx", i64), ("y", P), ("ldy", i64),
                ("saved", P), ("dx", P), ("lddx", i64), ("workspace", P), ("xchg", P), ("ld_xchg", i64),
                ("dx_mask", P), ("ld_dx_mask", i64), ("dy_masked", i32)]


class WGError(RuntimeError):
    pass


_lib = None


def lib():
    """Load libwg.so (raises if it is absent: there is no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise WGError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    st = ctypes.c_int
    L.wg_graph_create.restype = st
    L.wg_graph_create.argtypes = [ctypes.POINTER(GraphDesc), ctypes.c_int, P, ctypes.POINTER(P)]
    L.wg_graph_info.restype = st
    L.wg_graph_info.argtypes = [P, P]
    L.wg_graph_export.restype = st
    L.wg_graph_export.argtypes = [P, ctypes.c_int, P, P, P]
    L.wg_graph_destroy.restype = st
    L.wg_graph_destroy.argtypes = [P]
    L.wg_plan_create.restype = st
    L.wg_plan_create.argtypes = [P, ctypes.POINTER(ConvDesc), ctypes.POINTER(P)]
    L.wg_plan_sizes.restype = st
    L.wg_plan_sizes.argtypes = [P, ctypes.POINTER(ctypes.c_size_t), ctypes.POINTER(ctypes.c_size_t)]
    L.wg_plan_export.restype = st
    L.wg_plan_export.argtypes = [P, P, P]
    L.wg_plan_buffer.restype = st
    L.wg_plan_buffer.argtypes = [P, ctypes.c_int, ctypes.c_char_p, ctypes.POINTER(ctypes.c_size_t)]
    L.wg_plan_destroy.restype = st
    L.wg_plan_destroy.argtypes = [P]
    L.wg_conv_forward.restype = st
    L.wg_conv_forward.argtypes = [P, ctypes.POINTER(Params), ctypes.POINTER(FwdArgs), P]
    L.wg_conv_backward.restype = st
    L.wg_conv_backward.argtypes = [P, ctypes.POINTER(Params), ctypes.POINTER(BwdArgs), ctypes.POINTER(Grads), P]
    L.wg_status_string.restype = ctypes.c_char_p
    L.wg_status_string.argtypes = [ctypes.c_int]
    L.wg_last_error.restype = ctypes.c_char_p
    L.wg_last_error.argtypes = []
    L.wg_launch_count.restype = i64
    L.wg_launch_count.argtypes = []
    L.wg_profile.restype = st
    L.wg_profile.argtypes = [ctypes.c_int, P]
    L.wg_softmax_xent.restype = st
    L.wg_softmax_xent.argtypes = [ctypes.c_int, i64, i32, P, i64, P, f32, P, i64, P, P, P]
    L.wg_adam_step.restype = st
    L.wg_adam_step.argtypes = [i64, P, P, P, P, P, f32, f32, f32, f32, P]
    # multi-GPU
    L.wg_comm_unique_id.restype = st
    L.wg_comm_unique_id.argtypes = [P]
    L.wg_comm_init.restype = st
    L.wg_comm_init.argtypes = [P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(P)]
    L.wg_comm_init_emulated.restype = st
    L.wg_comm_init_emulated.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(P)]
    L.wg_comm_info.restype = st
    L.wg_comm_info.argtypes = [P, P]
    L.wg_comm_wait.restype = st
    L.wg_comm_wait.argtypes = [P, P]
    L.wg_comm_destroy.restype = st
    L.wg_comm_destroy.argtypes = [P]
    L.wg_partition_1d.restype = st
    L.wg_partition_1d.argtypes = [ctypes.POINTER(GraphDesc), ctypes.c_int, P]
    L.wg_graph_create_dist.restype = st
    L.wg_graph_create_dist.argtypes = [P, ctypes.POINTER(GraphDesc), P, ctypes.c_int, P, ctypes.POINTER(P),
                                       ctypes.POINTER(i64), ctypes.POINTER(i64)]
    L.wg_graph_bounds.restype = st
    L.wg_graph_bounds.argtypes = [P, P, ctypes.POINTER(i32)]
    L.wg_plan_create_dist.restype = st
    L.wg_plan_create_dist.argtypes = [P, P, ctypes.POINTER(ConvDesc), ctypes.POINTER(P)]
    L.wg_plan_xchg.restype = st
    L.wg_plan_xchg.argtypes = [P, ctypes.c_int, P]
    L.wg_conv_forward_dist.restype = st
    L.wg_conv_forward_dist.argtypes = [P, P, ctypes.POINTER(Params), ctypes.POINTER(FwdArgs), ctypes.c_int, P]
    L.wg_conv_backward_dist.restype = st
    L.wg_conv_backward_dist.argtypes = [P, P, ctypes.POINTER(Params), ctypes.POINTER(BwdArgs),
                                        ctypes.POINTER(Grads), P]
    # general restriction engine
    L.wg_gpart_create.restype = st
    L.wg_gpart_create.argtypes = [ctypes.POINTER(GraphDesc), P, i32, ctypes.c_int, P, ctypes.POINTER(P)]
    L.wg_gpart_info.restype = st
    L.wg_gpart_info.argtypes = [P, P]
    L.wg_gpart_export.restype = st
    L.wg_gpart_export.argtypes = [P, P, P]
    L.wg_gpart_workspace.restype = ctypes.c_size_t
    L.wg_gpart_workspace.argtypes = [P, i32]
    L.wg_gpart_aggregate.restype = st
    L.wg_gpart_aggregate.argtypes = [P, ctypes.c_int, i32, ctypes.c_int, P, i64, P, i64, P, P]
    L.wg_gpart_destroy.restype = st
    L.wg_gpart_destroy.argtypes = [P]
    _lib = L
    return L


def check(status: int, what: str = ""):
    if status != WG_OK:
        L = lib()
        raise WGError(f"{what}: {L.wg_status_string(status).decode()} ({status}): {L.wg_last_error().decode()}")
