"""Seeded synthetic inputs shaped like the paper's workloads.

This module is shared input code: it draws graphs, features, weights and
upstream gradients from seeded counter-based generators (numpy Philox).  It
holds none of the method's arithmetic (no partitioning, no aggregation, no
transform), so both the oracle (``oracle/``) and the CUDA path
(``paper_conf_eurosys_huangz0wjzzzys24_b200``) can consume the same inputs
without sharing any code.

Recipe:

* Graph shape: ``V`` vertices, ``E`` directed edges.  Endpoints are drawn from
  a power-law popularity distribution ``w(v) ∝ (rank(v)+1)^(-alpha)`` where
  ``rank`` is a seeded permutation of the vertex ids (hubs are scattered over
  the id space, not clustered at 0).  The inverse CDF of the continuous
  power law gives ``rank = floor(V * u^(1/(1-alpha)))`` for ``u ~ U[0,1)``.
  The paper only says the graphs are power-law; the exponents
  are this build's proposals and the achieved degree statistics are reported.
* ``symmetric=True`` draws ``E/2`` unordered pairs and emits both directions
  (ogbn-products / Cora are undirected graphs stored as directed pairs).
* Relation types (RGCN, Eq. (1)) are Zipf(R, s) distributed.
* Self-loops and multi-edges are kept.
* Features ~ N(0,1) (Cora: Bernoulli bag-of-words), weights Glorot-uniform.
"""
from __future__ import annotations

import dataclasses
import numpy as np

__all__ = [
    "Config", "CONFIGS", "make_graph", "make_graph_slice", "make_features", "glorot", "normal",
    "small_graph", "degree_stats",
]


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    model: str
    V: int
    E: int
    symmetric: bool
    alpha: float
    R: int
    dims: tuple
    dtype: str              # "f32" | "bf16"
    seed: int
    heads: int = 1
    zipf_s: float = 1.0
    xdist: str = "normal"   # "normal" | "bernoulli"
    xp: float = 0.0         # Bernoulli density for xdist == "bernoulli"
    note: str = ""


# BASELINE.json configs[0..4] (C1..C5); SURVEY.md §8(d) d1 table.
CONFIGS = {
    "C1": Config("C1", "gcn", 2708, 10556, True, 0.5, 1, (1433, 16, 7), "f32", 101,
                 xdist="bernoulli", xp=18.0 / 1433.0,
                 note="Cora-shaped, GCN 2-layer, fp32"),
    "C2": Config("C2", "gat", 169343, 1166243, False, 0.7, 1, (128, 64, 64, 40), "f32", 102,
                 heads=4, note="ogbn-arxiv-shaped, GAT 3-layer 4 heads hidden 64 (per head)"),
    "C3": Config("C3", "rgcn", 1939743, 21111007, False, 0.5, 128, (128, 64, 64), "f32", 103,
                 zipf_s=1.0, note="ogbn-mag-shaped heterograph, RGCN 2-layer, R=128"),
    "C4": Config("C4", "sage", 2449029, 61859140, True, 0.5, 1, (100, 256, 256, 47), "bf16", 104,
                 note="ogbn-products-shaped, GraphSAGE/GIN 3-layer hidden 256, bf16"),
    "C5": Config("C5", "sage", 111059956, 1615685872, False, 0.5, 1, (128, 32, 32, 172), "bf16", 105,
                 note="ogbn-papers100M-shaped, SAGE full graph, hidden 32, 8 GPUs"),
}


def _rng(seed: int, stream: int) -> np.random.Generator:
    # Counter-based generator; (seed, stream) selects an independent key.
    return np.random.Generator(np.random.Philox(key=np.uint64(seed) * np.uint64(16) + np.uint64(stream)))


def _powerlaw_vertices(rng, V: int, n: int, alpha: float, rank_to_vertex: np.ndarray,
                       chunk: int = 1 << 24) -> np.ndarray:
    out = np.empty(n, dtype=np.int32)
    expo = 1.0 / (1.0 - alpha)
    for lo in range(0, n, chunk):
        hi = min(n, lo + chunk)
        u = rng.random(hi - lo)
        r = np.minimum((V * np.power(u, expo)).astype(np.int64), V - 1)
        out[lo:hi] = rank_to_vertex[r]
    return out


def make_graph(V: int, E: int, *, seed: int, alpha: float = 0.5, symmetric: bool = False,
               R: int = 1, zipf_s: float = 1.0):
    """Return ``(src, dst, etype)`` int32 arrays of length E (etype None if R == 1).

    Edges are in generation order (a shuffled COO); the partitioner sorts them.
    """
    if symmetric and E % 2:
        raise ValueError("symmetric graphs need an even edge count")
    g = _rng(seed, 0)
    perm_in = g.permutation(V).astype(np.int32)
    perm_out = perm_in if symmetric else g.permutation(V).astype(np.int32)
    if symmetric:
        n = E // 2
        a = _powerlaw_vertices(_rng(seed, 1), V, n, alpha, perm_in)
        b = _powerlaw_vertices(_rng(seed, 2), V, n, alpha, perm_in)
        src = np.empty(E, np.int32)
        dst = np.empty(E, np.int32)
        src[0::2], dst[0::2] = a, b
        src[1::2], dst[1::2] = b, a
    else:
        dst = _powerlaw_vertices(_rng(seed, 1), V, E, alpha, perm_in)
        src = _powerlaw_vertices(_rng(seed, 2), V, E, alpha, perm_out)
    etype = None
    if R > 1:
        w = np.power(np.arange(1, R + 1, dtype=np.float64), -zipf_s)
        cdf = np.cumsum(w / w.sum())
        cdf[-1] = 1.0
        etype = np.empty(E, np.int32)
        tr = _rng(seed, 3)
        chunk = 1 << 24
        for lo in range(0, E, chunk):
            hi = min(E, lo + chunk)
            etype[lo:hi] = np.searchsorted(cdf, tr.random(hi - lo), side="right").astype(np.int32)
        np.minimum(etype, R - 1, out=etype)
    return src, dst, etype


def make_graph_slice(V: int, E: int, lo: int, hi: int, *, seed: int, alpha: float = 0.5,
                     chunk: int = 1 << 24):
    """The edges of ``make_graph(V, E, seed=seed, alpha=alpha)`` (directed,
    untyped) with ``dst`` or ``src`` in ``[lo, hi)``, in generation order,
    without materialising all E edges: the same Philox streams are drawn
    chunk by chunk (``Generator.random`` output does not depend on the chunk
    split) and filtered.  Used for one rank's share of the C5 1-D partition
    (its in-edges for the forward, its out-edges for the backward)."""
    g = _rng(seed, 0)
    perm_in = g.permutation(V).astype(np.int32)
    perm_out = g.permutation(V).astype(np.int32)
    rd, rs = _rng(seed, 1), _rng(seed, 2)
    srcs, dsts = [], []
    for b in range(0, E, chunk):
        n = min(E, b + chunk) - b
        d = _powerlaw_vertices(rd, V, n, alpha, perm_in, chunk=chunk)
        s = _powerlaw_vertices(rs, V, n, alpha, perm_out, chunk=chunk)
        keep = ((d >= lo) & (d < hi)) | ((s >= lo) & (s < hi))
        srcs.append(s[keep])
        dsts.append(d[keep])
    return np.concatenate(srcs), np.concatenate(dsts)


def small_graph(V: int, E: int, *, seed: int, R: int = 1, alpha: float = 0.3,
                symmetric: bool = False):
    """Small power-law graph for parity tests (same recipe, any size)."""
    return make_graph(V, E, seed=seed, alpha=alpha, symmetric=symmetric, R=R)


def make_features(V: int, F: int, *, seed: int, dist: str = "normal", p: float = 0.0,
                  dtype=np.float32) -> np.ndarray:
    g = _rng(seed, 4)
    if dist == "bernoulli":
        return (g.random((V, F)) < p).astype(dtype)
    if dist == "int":   # small integers in {-3..3}: every fp32 partial sum is exact
        return g.integers(-3, 4, size=(V, F)).astype(dtype)
    if dist == "uniform01":
        return g.random((V, F)).astype(dtype)
    return g.standard_normal((V, F), dtype=np.float32).astype(dtype)


def normal(shape, *, seed: int, std: float = 1.0, dtype=np.float32) -> np.ndarray:
    g = _rng(seed, 5)
    return (g.standard_normal(shape, dtype=np.float32) * np.float32(std)).astype(dtype)


def glorot(fan_in: int, fan_out: int, *, seed: int, shape=None, dtype=np.float32) -> np.ndarray:
    g = _rng(seed, 6)
    lim = np.sqrt(6.0 / (fan_in + fan_out))
    shp = shape if shape is not None else (fan_in, fan_out)
    return g.uniform(-lim, lim, size=shp).astype(dtype)


def small_ints(shape, *, seed: int, lo: int = -3, hi: int = 3, dtype=np.float32) -> np.ndarray:
    g = _rng(seed, 7)
    return g.integers(lo, hi + 1, size=shape).astype(dtype)


def degree_stats(idx: np.ndarray, V: int) -> dict:
    d = np.bincount(idx, minlength=V)
    return {"max": int(d.max()), "mean": float(d.mean()), "p99": float(np.percentile(d, 99))}
