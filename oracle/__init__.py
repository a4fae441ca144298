"""CPU oracle for the gTask graph-convolution layer -- TEST INFRASTRUCTURE ONLY.

Thin numpy/ctypes wrapper over ``oracle/wg_oracle.c`` (plain C, fp64, one
thread, per-edge loops in the paper's order; see the header of that file for
the citations).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
module.  The product package never imports it, and it never imports the
product package.

Parity status per function (DESIGN.md §"Oracle pins"):

* ``partition``      -- pinned: worked example of Fig 5a/Fig 7 (golden file),
                        limit cases, brute-force invariants.
* ``*_forward``      -- pinned: dense-adjacency brute force (numpy), closed
                        forms on the worked example, integer exactness,
                        special-case reductions.
* ``*_backward``     -- pinned: torch.autograd on the dense fp64 formulation,
                        adjoint identities, finite differences (GAT).
* ``dw_probe``       -- pinned: equals u^T dW v of the pinned backward.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "wg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

TASK_DTYPE = np.dtype([
    ("tile", np.int32), ("type", np.int32), ("e_begin", np.int64), ("e_end", np.int64),
    ("d_lo", np.int32), ("d_hi", np.int32), ("flags", np.int32), ("n_uniq_src", np.int32),
])
SPLIT = 1


def build(force: bool = False) -> str:
    """Compile the oracle with plain ``gcc -O2`` (no SIMD intrinsics, no OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-std=c11", "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i64, i32, f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        _lib.wgo_partition.restype = i64
        _lib.wgo_partition.argtypes = [i64, P, P, P, i32, i32, i64, P, P]
        _lib.wgo_partition_general.restype = i64
        _lib.wgo_partition_general.argtypes = [i64, i64, P, P, P, P, P, i32, P, P]
        _lib.wgo_gcn_forward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P, P, P, P]
        _lib.wgo_gcn_backward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P]
        _lib.wgo_sage_forward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P]
        _lib.wgo_sage_backward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P, P, P]
        _lib.wgo_gin_forward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, f64, P, P, P, P, P, P, P, P, P]
        _lib.wgo_gin_backward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, f64, P, P, P, P, P, P, P, P, P, P, P]
        _lib.wgo_rgcn_forward.argtypes = [i64, i64, P, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P]
        _lib.wgo_rgcn_backward.argtypes = [i64, i64, P, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P, P, P]
        _lib.wgo_gat_forward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, f64, P, P, P, P, P, P, P]
        _lib.wgo_gat_backward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, f64, P, P, P, P, P, P, P, P, P, P]
        _lib.wgo_sage_lstm_forward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P, P, P, P]
        _lib.wgo_sage_lstm_backward.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, P, P, P, P, P,
                                                P, P, P, P, P, P, P]
        _lib.wgo_dw_probe.restype = f64
        _lib.wgo_dw_probe.argtypes = [i64, P, P, P, ctypes.c_int, ctypes.c_int, P, P, P, P]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.int32)


def _f64(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.float64)


def _mask(V, rows):
    if rows is None:
        return None
    m = np.zeros(V, np.uint8)
    m[np.asarray(rows, dtype=np.int64)] = 1
    return m


NORM = {"none": 0, "right": 1, "both": 2}


# ---------------------------------------------------------------------------
# Partition (Q10-Q13)
# ---------------------------------------------------------------------------
def partition(key_vertex, other_vertex, etype=None, *, by_type=False, T=128, E_max):
    """Greedy gTask partition keyed on ``key_vertex``.  Returns (perm int64[E], tasks)."""
    kv, ov, et = _i32(key_vertex), _i32(other_vertex), _i32(etype)
    E = kv.shape[0]
    perm = np.empty(max(E, 1), np.int64)
    tasks = np.empty(max(E, 1), TASK_DTYPE)
    n = _L().wgo_partition(E, _p(kv), _p(ov), _p(et), int(bool(by_type and et is not None)),
                           int(T), int(E_max), _p(perm), _p(tasks))
    return perm[:E].copy(), tasks[:n].copy()


ATTRS = {"dst": 0, "src": 1, "type": 2, "dst_degree": 3, "edge": 4}


def partition_general(src, dst, V, restrictions, etype=None):
    """General restriction engine (f2; Fig 7): restrictions is a
    list of (attribute name, k) with k >= 1 (uniq(a) = k) or "min"
    (uniq(a) = min).  Returns (perm int64[E], tasks)."""
    s, d, et = _i32(src), _i32(dst), _i32(etype)
    E = s.shape[0]
    a = np.array([ATTRS[n] for n, _ in restrictions], np.int32)
    k = np.array([-1 if v == "min" else int(v) for _, v in restrictions], np.int32)
    perm = np.empty(max(E, 1), np.int64)
    tasks = np.empty(max(E, 1), TASK_DTYPE)
    n = _L().wgo_partition_general(V, E, _p(s), _p(d), _p(et), _p(a), _p(k), len(a), _p(perm), _p(tasks))
    if n < 0:
        raise ValueError("bad restriction spec")
    return perm[:E].copy(), tasks[:n].copy()


def transposed(src, dst, etype=None, *, by_type=False, T=128, E_max, perm_fwd):
    """Transposed partition (keyed on src) plus fwdpos_of_T = inv(perm)[perm_T]."""
    perm_t, tasks_t = partition(src, dst, etype, by_type=by_type, T=T, E_max=E_max)
    inv = np.empty_like(perm_fwd)
    inv[perm_fwd] = np.arange(perm_fwd.shape[0], dtype=np.int64)
    return perm_t, tasks_t, inv[perm_t]


def default_emax(V, E, T=128):
    """Q13: E_max = clamp(pow2ceil(4*T*ceil(E/V)), 1024, 65536) (integer rule)."""
    avg = -(-E // max(V, 1))
    x = 4 * T * max(avg, 1)
    p = 1
    while p < x:
        p <<= 1
    return int(min(max(p, 1024), 65536))


# ---------------------------------------------------------------------------
# Convolutions (fp64).  Arrays are numpy; outputs are float64.
# ---------------------------------------------------------------------------
def gcn_forward(src, dst, V, x, W, b=None, norm="both", rows=None):
    x, W, b = _f64(x), _f64(W), _f64(b)
    fi, fo = W.shape
    y = np.zeros((V, fo))
    s, d = _i32(src), _i32(dst)
    m = _mask(V, rows)
    _L().wgo_gcn_forward(V, s.shape[0], _p(s), _p(d), NORM[norm], fi, fo, _p(x), _p(W), _p(b), _p(m), _p(y))
    return y


def gcn_backward(src, dst, V, x, W, dy, norm="both", rows=None):
    x, W, dy = _f64(x), _f64(W), _f64(dy)
    fi, fo = W.shape
    dx, dW, db = np.zeros((V, fi)), np.zeros((fi, fo)), np.zeros(fo)
    s, d = _i32(src), _i32(dst)
    m = _mask(V, rows)
    _L().wgo_gcn_backward(V, s.shape[0], _p(s), _p(d), NORM[norm], fi, fo, _p(x), _p(W), _p(dy), _p(m),
                          _p(dx), _p(dW), _p(db))
    return dx, dW, db


def sage_forward(src, dst, V, x, Ws, Wn, b=None, rows=None):
    x, Ws, Wn, b = _f64(x), _f64(Ws), _f64(Wn), _f64(b)
    fi, fo = Ws.shape
    y = np.zeros((V, fo))
    s, d = _i32(src), _i32(dst)
    m = _mask(V, rows)
    _L().wgo_sage_forward(V, s.shape[0], _p(s), _p(d), fi, fo, _p(x), _p(Ws), _p(Wn), _p(b), _p(m), _p(y))
    return y


def sage_backward(src, dst, V, x, Ws, Wn, dy, rows=None, grads=True):
    """grads=False: only dx (of `rows`) is computed (weight-gradient loops skipped)."""
    x, Ws, Wn, dy = _f64(x), _f64(Ws), _f64(Wn), _f64(dy)
    fi, fo = Ws.shape
    dx, dWs, dWn, db = np.zeros((V, fi)), np.zeros((fi, fo)), np.zeros((fi, fo)), np.zeros(fo)
    s, d = _i32(src), _i32(dst)
    m = _mask(V, rows)
    _L().wgo_sage_backward(V, s.shape[0], _p(s), _p(d), fi, fo, _p(x), _p(Ws), _p(Wn), _p(dy), _p(m),
                           _p(dx), _p(dWs) if grads else None, _p(dWn) if grads else None,
                           _p(db) if grads else None)
    return dx, dWs, dWn, db


def gin_forward(src, dst, V, x, W1, b1, W2, b2, eps=0.0, rows=None, return_za=False):
    """rows: produce only these rows; return_za: also return z [V x fi] and the
    pre-activation a = z W1 + b1 [V x fo] of the produced rows."""
    x, W1, b1, W2, b2 = map(_f64, (x, W1, b1, W2, b2))
    fi, fo = W1.shape
    y = np.zeros((V, fo))
    z = np.zeros((V, fi)) if return_za else None
    a = np.zeros((V, fo)) if return_za else None
    s, d = _i32(src), _i32(dst)
    m = _mask(V, rows)
    _L().wgo_gin_forward(V, s.shape[0], _p(s), _p(d), fi, fo, float(eps), _p(x), _p(W1), _p(b1), _p(W2), _p(b2),
                         _p(m), _p(y), _p(z), _p(a))
    return (y, z, a) if return_za else y


def gin_backward(src, dst, V, x, W1, b1, W2, dy, eps=0.0, dy_rows=None):
    """Exact gradients; the ReLU decision [a > 0] is taken here, in fp64.
    dy_rows: rows of dy outside this set are zero (skipped); dx is still
    produced for every vertex."""
    x, W1, b1, W2, dy = map(_f64, (x, W1, b1, W2, dy))
    fi, fo = W1.shape
    dx, dW1, db1, dW2, db2 = np.zeros((V, fi)), np.zeros((fi, fo)), np.zeros(fo), np.zeros((fo, fo)), np.zeros(fo)
    s, d = _i32(src), _i32(dst)
    m = _mask(V, dy_rows)
    _L().wgo_gin_backward(V, s.shape[0], _p(s), _p(d), fi, fo, float(eps), _p(x), _p(W1), _p(b1), _p(W2), _p(dy),
                          _p(m), _p(dx), _p(dW1), _p(db1), _p(dW2), _p(db2))
    return dx, dW1, db1, dW2, db2


def rgcn_forward(src, dst, etype, V, x, W, W0=None, b=None, norm="none", rows=None):
    x, W, W0, b = _f64(x), _f64(W), _f64(W0), _f64(b)
    R, fi, fo = W.shape
    y = np.zeros((V, fo))
    s, d, t = _i32(src), _i32(dst), _i32(etype)
    m = _mask(V, rows)
    _L().wgo_rgcn_forward(V, s.shape[0], _p(s), _p(d), _p(t), R, NORM[norm], fi, fo, _p(x), _p(W), _p(W0), _p(b),
                          _p(m), _p(y))
    return y


def rgcn_backward(src, dst, etype, V, x, W, dy, W0=None, norm="none", rows=None, grads=True):
    """grads=False: only dx (of `rows`) is computed (weight-gradient loops skipped)."""
    x, W, W0, dy = _f64(x), _f64(W), _f64(W0), _f64(dy)
    R, fi, fo = W.shape
    dx, dW, db = np.zeros((V, fi)), np.zeros((R, fi, fo)), np.zeros(fo)
    dW0 = np.zeros((fi, fo)) if W0 is not None else None
    s, d, t = _i32(src), _i32(dst), _i32(etype)
    m = _mask(V, rows)
    _L().wgo_rgcn_backward(V, s.shape[0], _p(s), _p(d), _p(t), R, NORM[norm], fi, fo, _p(x), _p(W), _p(W0), _p(dy),
                           _p(m), _p(dx), _p(dW) if grads else None, _p(dW0) if grads else None,
                           _p(db) if grads else None)
    return dx, dW, dW0, db


def gat_forward(src, dst, V, x, W, al, ar, b=None, *, heads, concat=True, slope=0.2, return_alpha=False):
    x, W, al, ar, b = map(_f64, (x, W, al, ar, b))
    fi = W.shape[0]
    fo = W.shape[1] // heads
    FO = heads * fo if concat else fo
    y = np.zeros((V, FO))
    s, d = _i32(src), _i32(dst)
    E = s.shape[0]
    alpha = np.zeros((max(E, 1), heads)) if return_alpha else None
    _L().wgo_gat_forward(V, E, _p(s), _p(d), fi, heads, fo, int(concat), float(slope), _p(x), _p(W), _p(al), _p(ar),
                         _p(b), _p(y), _p(alpha))
    return (y, alpha[:E]) if return_alpha else y


def gat_backward(src, dst, V, x, W, al, ar, dy, *, heads, concat=True, slope=0.2):
    x, W, al, ar, dy = map(_f64, (x, W, al, ar, dy))
    fi = W.shape[0]
    fo = W.shape[1] // heads
    FO = heads * fo if concat else fo
    dx, dW = np.zeros((V, fi)), np.zeros_like(W)
    dal, dar, db = np.zeros((heads, fo)), np.zeros((heads, fo)), np.zeros(FO)
    s, d = _i32(src), _i32(dst)
    _L().wgo_gat_backward(V, s.shape[0], _p(s), _p(d), fi, heads, fo, int(concat), float(slope), _p(x), _p(W),
                          _p(al), _p(ar), _p(dy), _p(dx), _p(dW), _p(dal), _p(dar), _p(db))
    return dx, dW, dal, dar, db


def sage_lstm_forward(src, dst, V, x, Ws, Wn, b, Wih, Whh, bl, rows=None, return_h=False):
    """SAGE-LSTM forward (f4; Q26): y = b + x W_s + LSTM(x[in-nbrs in edge-id order]) W_n."""
    x, Ws, Wn, b, Wih, Whh, bl = map(_f64, (x, Ws, Wn, b, Wih, Whh, bl))
    fi, fo = Ws.shape
    y = np.zeros((V, fo))
    hN = np.zeros((V, fi)) if return_h else None
    s, d = _i32(src), _i32(dst)
    _L().wgo_sage_lstm_forward(V, s.shape[0], _p(s), _p(d), fi, fo, _p(x), _p(Ws), _p(Wn), _p(b), _p(Wih), _p(Whh),
                               _p(bl), _p(_mask(V, rows)), _p(y), _p(hN))
    return (y, hN) if return_h else y


def sage_lstm_backward(src, dst, V, x, Ws, Wn, Wih, Whh, bl, dy, dy_rows=None):
    """Exact gradients (BPTT per vertex): dx, dWs, dWn, db, dWih, dWhh, dbl."""
    x, Ws, Wn, Wih, Whh, bl, dy = map(_f64, (x, Ws, Wn, Wih, Whh, bl, dy))
    fi, fo = Ws.shape
    out = [np.zeros((V, fi)), np.zeros((fi, fo)), np.zeros((fi, fo)), np.zeros(fo), np.zeros((fi, 4 * fi)),
           np.zeros((fi, 4 * fi)), np.zeros(4 * fi)]
    s, d = _i32(src), _i32(dst)
    _L().wgo_sage_lstm_backward(V, s.shape[0], _p(s), _p(d), fi, fo, _p(x), _p(Ws), _p(Wn), _p(Wih), _p(Whh), _p(bl),
                                _p(dy), _p(_mask(V, dy_rows)), *[_p(o) for o in out])
    return tuple(out)


def dw_probe(src, dst, x, dy, u, v, coef=None):
    x, dy, u, v, coef = map(_f64, (x, dy, u, v, coef))
    s, d = _i32(src), _i32(dst)
    return _L().wgo_dw_probe(s.shape[0], _p(s), _p(d), _p(coef), x.shape[1], dy.shape[1], _p(x), _p(dy), _p(u), _p(v))
