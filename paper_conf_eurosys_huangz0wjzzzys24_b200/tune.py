"""Strategy selection by measurement:
candidate partition parameters (T = destination-tile rows, E_max = the
uniq(edge-id) limit that cuts overfill rows) are pruned by a cost model,
the survivors are timed on the device (one forward + backward of every
layer, CUDA events, median of `reps`), and the winner is cached per graph /
layer signature so the search runs once per configuration ("caching ...
to avoid repeated ... testing").

Pruning (the paper's three components): FLOP and memory volume
do not depend on (T, E_max) -- every plan gathers the same rows -- so the
model prunes on parallelism: a candidate whose work items cannot fill the GPU
(< 2 per SM) or whose largest work item holds more than a quarter of all
edges (long tail) is not timed."""
from __future__ import annotations

import hashlib
import json
import os
import time

import numpy as np
import torch

from . import Conv, Graph, init_params, padded

SMS = 148


def signature(src, dst, V, model, dims, dtype, R=1):
    """Cache key: sizes, a log2 in-degree histogram, the layer shapes, dtype."""
    deg = np.bincount(np.asarray(dst), minlength=V)
    hist = np.bincount(np.floor(np.log2(np.maximum(deg, 1))).astype(np.int64), minlength=32)[:32]
    h = hashlib.sha1(hist.tobytes()).hexdigest()[:12]
    return f"V{V}-E{len(src)}-R{R}-{model}-{'x'.join(map(str, dims))}-{str(dtype).split('.')[-1]}-deg{h}"


def default_candidates(V, E, T0=128):
    avg = -(-E // max(V, 1))
    base = 1
    while base < 4 * T0 * max(avg, 1):
        base <<= 1
    base = min(max(base, 1024), 65536)
    return [(T0, base), (T0, base // 4), (T0, base * 4), (64, base), (256, base)]


def _time_layers(g, model, dims, dtype, reps, conv_kw, R):
    torch.manual_seed(0)
    total = []
    for _ in range(reps):
        ms = 0.0
        for i in range(len(dims) - 1):
            fi, fo = dims[i], dims[i + 1]
            conv = Conv(g, model, fi, fo, dtype=dtype, fuse_relu=i < len(dims) - 2, need_dx=i > 0, **conv_kw)
            p = init_params(model, fi, fo, R=R, self_loop=bool(conv_kw.get("self_loop")), device="cuda")
            x = padded(g.V, fi, dtype)
            x.normal_()
            y, saved = conv.forward_raw(x, p)
            dy = padded(g.n_rows, fo, dtype)
            dy.normal_()
            conv.backward_raw(dy, x, y, saved, p)            # warm
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            y, saved = conv.forward_raw(x, p, y=y, saved=saved)
            conv.backward_raw(dy, x, y, saved, p)
            e1.record()
            torch.cuda.synchronize()
            ms += e0.elapsed_time(e1)
            conv.close()
        total.append(ms)
    return float(np.median(total))


def search(src, dst, V, model, dims, dtype=torch.bfloat16, *, etype=None, R=1, candidates=None, reps=3,
           cache_path=None, conv_kw=None):
    """Returns (tile_rows, max_task_edges, report).  report lists every
    candidate with its pruning decision and measured ms."""
    conv_kw = dict(conv_kw or {})
    key = signature(src, dst, V, model, dims, dtype, R)
    cache = {}
    if cache_path and os.path.exists(cache_path):
        cache = json.load(open(cache_path))
        if key in cache:
            c = cache[key]
            return c["T"], c["E_max"], dict(c, cached=True)
    cands = candidates or default_candidates(V, len(src))
    ts, td = torch.as_tensor(src).cuda(), torch.as_tensor(dst).cuda()
    tt = torch.as_tensor(etype).cuda() if etype is not None else None
    rows = []
    t0 = time.perf_counter()
    for T, Em in cands:
        g = Graph(ts, td, num_vertices=V, etype=tt, num_types=R, tile_rows=T, max_task_edges=Em)
        probe = Conv(g, model, dims[0], dims[1], dtype=dtype, **conv_kw)
        items = probe.n_items
        tasks = g.export()[1]
        biggest = int((tasks["e_end"] - tasks["e_begin"]).max()) if len(tasks) else 0
        probe.close()
        r = {"T": T, "E_max": int(g.E_max), "items": int(items), "max_task_edges_seen": biggest}
        if items < 2 * SMS and len(cands) > 1:
            r["pruned"] = "parallelism: fewer than 2 work items per SM"
        elif biggest * 4 > max(len(src), 1):
            r["pruned"] = "parallelism: one gTask holds > 1/4 of the edges"
        else:
            r["ms"] = _time_layers(g, model, dims, dtype, reps, conv_kw, R)
        rows.append(r)
        g.close()
    timed = [r for r in rows if "ms" in r] or rows
    best = min(timed, key=lambda r: r.get("ms", 0.0))
    rep = {"T": best["T"], "E_max": best["E_max"], "candidates": rows, "search_s": time.perf_counter() - t0,
           "key": key, "cached": False}
    if cache_path:
        cache[key] = {k: v for k, v in rep.items() if k != "cached"}
        os.makedirs(os.path.dirname(os.path.abspath(cache_path)), exist_ok=True)
        json.dump(cache, open(cache_path, "w"), indent=1)
    return best["T"], best["E_max"], rep
