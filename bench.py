#!/usr/bin/env python
"""Benchmark: full-graph GNN training epoch over the gTask layer.

Workload (BASELINE.json configs[3], "C4"): GraphSAGE 3-layer, hidden 256, on a
synthetic ogbn-products-shaped graph (2,449,029 V, 61,859,140 E, 100 input
features, 47 classes), bf16 with fp32 accumulation, random-init weights,
uniform random labels.  C4 is the config BASELINE.json names for 1/2/4/8
B200 (configs[1], GAT on arxiv, is a parity case).  One step = one epoch:
forward of all layers, CE loss, backward of all layers, weight-gradient
all-reduce (N > 1), Adam step.  value = layers * E / step time (whole job).

    python bench.py [--gpus N --steps K --warmup W] [--impl reference]
    torchrun --nproc-per-node N bench.py --gpus N        (1-D dst partition)
    python bench.py --config C1|C2|C3 [--model ...]      (the other configs' models:
        C1 GCN fp32, C2 GAT 4 heads fp32, C3 RGCN R=128 fp32, C4 --model gin)

The default line (no flags) is the driver's: C4 SAGE.  The other configs are
the parity cases of BASELINE.json, measured the same way (profiles/r01/).

Timing: CUDA events on the compute stream, barrier + synchronize on both sides,
max over ranks; inputs (features 490 MB, tables >= 1.2 GB) exceed the 126 MB
L2 so no flush is needed.  Per-kernel-class times come from the library's
own event timing (wg_profile) inside the timed region.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GNN layer fwd+bwd edges/s"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return p, "measured"
    except Exception:
        return PEAKS_FALLBACK, "fallback"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4")
    ap.add_argument("--model", default=None, choices=["sage", "gin", "gcn", "gat", "rgcn"],
                    help="default: the config's model (C4: sage)")
    ap.add_argument("--policy", default="auto")
    ap.add_argument("--tile", type=int, default=128,
                    help="gTask destination-tile rows T (SURVEY §8(f) f1 sweeps; 128 = the tcgen05 M)")
    ap.add_argument("--emax", type=int, default=0,
                    help="gTask edge limit E_max (0: the Q13 rule); SURVEY §8(f) f1 K sweeps")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--rank-slice", type=int, default=0, metavar="P",
                    help="one GPU runs rank --slice-rank of a P-way 1-D partition (its in- / out-edges only, "
                         "collectives emulated): per-rank compute of a configuration too large for one GPU (C5)")
    ap.add_argument("--slice-rank", type=int, default=0)
    ap.add_argument("--hidden", type=int, default=0,
                    help="replace the hidden widths of the config (a hidden-dimension sweep, Fig 20-style)")
    ap.add_argument("--tune", action="store_true",
                    help="choose (T, E_max) by the measured strategy search (tune.py; cached per configuration)")
    ap.add_argument("--tune-cache", default=os.path.join(os.path.expanduser("~"), ".cache", "wg_tune.json"))
    ap.add_argument("--emulate-xchg", action="store_true",
                    help="--rank-slice: time every exchange as a copy kernel on the library's communication "
                         "stream (overlapped with the gathers as the NCCL exchange would be)")
    ap.add_argument("--no-graph", action="store_true",
                    help="time eager steps instead of replaying one CUDA-graph-captured step")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    return ap.parse_args()


def conv_options(c, model):
    """Per-model layer options of the workload (readings Q1-Q6)."""
    if model == "rgcn":     # the usual R-GCN layer: 1/|N_v^r| normalisation, self-loop W_0, bias (Q2 options)
        return {"norm": "right", "self_loop": True}
    return {}


def workload(cfg_name, model, hidden=0):
    import dataclasses
    import synth
    c = synth.CONFIGS[cfg_name]
    if hidden:
        c = dataclasses.replace(c, dims=(c.dims[0],) + (hidden,) * (len(c.dims) - 2) + (c.dims[-1],))
    model = model or c.model
    extra = {}
    if model == "gat":
        extra["heads"] = c.heads
    if model == "rgcn":
        extra.update(R=c.R, zipf_s=c.zipf_s, **conv_options(c, model))
    return c, model, {"workload": f"{cfg_name}: {model} {len(c.dims) - 1}-layer {'-'.join(map(str, c.dims))} on "
                                  f"synthetic {c.note.split(',')[0]} ({c.V} V, {c.E} E)",
                      "V": c.V, "E": c.E, "dims": list(c.dims), "model": model, "alpha": c.alpha,
                      "symmetric": c.symmetric, "seed": c.seed, "features": c.xdist, **extra}


def make_inputs(c, model):
    import synth
    R = c.R if model == "rgcn" else 1
    src, dst, et = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha, symmetric=c.symmetric, R=R,
                                    zipf_s=c.zipf_s)
    x = synth.make_features(c.V, c.dims[0], seed=c.seed * 16 + 2, dist=c.xdist, p=c.xp)
    labels = np.random.Generator(np.random.Philox(c.seed * 16 + 5)).integers(0, c.dims[-1], c.V).astype(np.int64)
    return src, dst, et, x, labels


class Clocks:
    """nvidia-smi clock / throttle sampling (every 50 ms, reader thread, host
    timestamps); stop() keeps the samples inside the timed windows marked with
    mark_start() / mark_stop()."""

    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, idx):
        self.idx = idx
        self.p = None
        self.samples = []       # (t, sm, smax, reasons)
        self.windows = []
        self.t0 = None

    def start(self):
        import threading
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
            return

        def reader():
            for line in self.p.stdout:
                f = [t.strip() for t in line.split(",")]
                if len(f) < 8:
                    continue
                try:
                    sm, smax = float(f[0]), float(f[1])
                except ValueError:
                    continue
                rs = {n for n, v in zip(self.NAMES, f[4:8]) if v.lower() == "active"}
                self.samples.append((time.perf_counter(), sm, smax, rs))

        self.th = threading.Thread(target=reader, daemon=True)
        self.th.start()
        for _ in range(100):            # wait for the first sample so the timed window is covered
            if self.samples:
                break
            time.sleep(0.02)

    def mark_start(self):
        self.t0 = time.perf_counter()

    def mark_stop(self):
        if self.t0 is not None:
            self.windows.append((self.t0, time.perf_counter()))
            self.t0 = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.06)
        self.p.terminate()
        try:
            self.p.wait(timeout=10)
        except Exception:
            pass
        inside = [x for x in self.samples if any(a <= x[0] <= b for a, b in self.windows)]
        use = inside or self.samples
        sm = [x[1] for x in use]
        reasons = set().union(*[x[3] for x in use]) if use else set()
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": use[-1][2] if use else None,
                "reasons": sorted(reasons), "samples": len(inside), "samples_total": len(self.samples),
                "interval_ms": 50}


def layer_shapes(c, model):
    """(f_in, f_out, concat) of each layer: GAT hidden layers read heads * dims[i] columns."""
    L = len(c.dims) - 1
    return [((c.heads * c.dims[i] if (model == "gat" and i > 0) else c.dims[i]), c.dims[i + 1], i < L - 1)
            for i in range(L)]


def host_info():
    """nproc (usable cores), CPU model and sockets of this host (lscpu)."""
    info = {"nproc": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() == "Model name":
                info["model"] = v.strip()
            elif k.strip() == "Socket(s)":
                info["sockets"] = int(v.strip())
            elif k.strip() == "Core(s) per socket":
                info["cores_per_socket"] = int(v.strip())
            elif k.strip() == "Thread(s) per core":
                info["threads_per_core"] = int(v.strip())
    except Exception:
        pass
    return info


def _csr_order(c, dst):
    order = np.argsort(dst, kind="stable")
    indptr = np.concatenate([[0], np.cumsum(np.bincount(dst, minlength=c.V))])
    return order, indptr


def _oracle_sample(c, model, src, dst, et, budget_s, seed, csr):
    """A bounded sample of the workload for the oracle: every in-edge of a
    seeded random sample of destination rows (its induced star graph), with
    one forward + backward per layer shape.  Returns (n_edges, description,
    run) where run() executes the oracle calls and returns per-layer
    (t_fwd, t_bwd) seconds."""
    import oracle
    rng = np.random.Generator(np.random.Philox(seed))
    order, indptr = csr
    shapes = layer_shapes(c, model)
    H = c.heads if model == "gat" else 1
    per_edge = sum(fi * fo * H for fi, fo, _ in shapes) * 2 * 3      # ~ fwd+bwd flops per edge (per-edge messages)
    target_edges = max(200, int(budget_s * 1.2e9 / per_edge))
    rows, n = [], 0
    for v in rng.permutation(c.V):
        d = int(indptr[v + 1] - indptr[v])
        if d == 0:
            continue
        rows.append(v)
        n += d
        if n >= target_edges:
            break
    eids = np.concatenate([order[indptr[v]:indptr[v + 1]] for v in rows])
    s, d = src[eids], dst[eids]
    verts, inv = np.unique(np.concatenate([s, d]), return_inverse=True)
    s2, d2 = inv[:len(s)].astype(np.int32), inv[len(s):].astype(np.int32)
    t2 = et[eids].astype(np.int32) if (model == "rgcn" and et is not None) else None
    Vs = len(verts)
    calls = []
    for i, (fi, fo, concat) in enumerate(shapes):
        r = lambda k, *sh: np.random.default_rng(seed + 10 * k + i).standard_normal(sh)   # noqa: E731
        xs, dy = r(0, Vs, fi), r(3, Vs, (H * fo if (model == "gat" and concat) else fo))
        if model == "sage":
            Ws, Wn = 0.05 * r(1, fi, fo), 0.05 * r(2, fi, fo)
            f = lambda: oracle.sage_forward(s2, d2, Vs, xs, Ws, Wn, np.zeros(fo))   # noqa: E731
            b = lambda: oracle.sage_backward(s2, d2, Vs, xs, Ws, Wn, dy)   # noqa: E731
        elif model == "gcn":
            W = 0.05 * r(1, fi, fo)
            f = lambda: oracle.gcn_forward(s2, d2, Vs, xs, W, np.zeros(fo))   # noqa: E731
            b = lambda: oracle.gcn_backward(s2, d2, Vs, xs, W, dy)   # noqa: E731
        elif model == "gin":
            W1, W2 = 0.05 * r(1, fi, fo), 0.05 * r(2, fo, fo)
            f = lambda: oracle.gin_forward(s2, d2, Vs, xs, W1, np.zeros(fo), W2, np.zeros(fo))   # noqa: E731
            b = lambda: oracle.gin_backward(s2, d2, Vs, xs, W1, np.zeros(fo), W2, dy)   # noqa: E731
        elif model == "gat":
            W, al, ar = 0.05 * r(1, fi, H * fo), 0.1 * r(2, H, fo), 0.1 * r(4, H, fo)
            f = lambda: oracle.gat_forward(s2, d2, Vs, xs, W, al, ar, None, heads=H, concat=concat)   # noqa: E731
            b = lambda: oracle.gat_backward(s2, d2, Vs, xs, W, al, ar, dy, heads=H, concat=concat)   # noqa: E731
        else:
            W, W0 = 0.05 * r(1, c.R, fi, fo), 0.05 * r(2, fi, fo)
            f = lambda: oracle.rgcn_forward(s2, d2, t2, Vs, xs, W, W0, np.zeros(fo), norm="right")   # noqa: E731
            b = lambda: oracle.rgcn_backward(s2, d2, t2, Vs, xs, W, dy, W0, norm="right")   # noqa: E731
        calls.append((f, b))

    def run():
        out = []
        for f, b in calls:
            t0 = time.perf_counter()
            f()
            t1 = time.perf_counter()
            b()
            out.append((t1 - t0, time.perf_counter() - t1))
        return out
    desc = f"all {len(eids)} in-edges of {len(rows)} random dst rows (induced star graph, {Vs} V)"
    return len(eids), desc, run


def cpu_baseline(c, model, src, dst, et, budget_s, csr=None):
    """The oracle as it stands (plain C, fp64, serial per call) timed on this
    host's cores: (1) one thread on one bounded sample, per layer forward /
    backward (the per-core rate); (2) nproc threads at once,
    each running the unchanged oracle on its own sample (ctypes releases the
    GIL), throughput = all edges / wall time.  The headline value is (2)."""
    import threading
    hi = host_info()
    L = len(layer_shapes(c, model))
    csr = csr or _csr_order(c, dst)
    n1, desc1, run1 = _oracle_sample(c, model, src, dst, et, budget_s / 3, c.seed * 16 + 9, csr)
    per_layer = run1()
    t1 = sum(a + b for a, b in per_layer)
    nth = max(1, int(hi["nproc"]))
    samples = [_oracle_sample(c, model, src, dst, et, budget_s / 3, c.seed * 16 + 100 + k, csr) for k in range(nth)]
    start = threading.Barrier(nth + 1)
    done = [None] * nth

    def work(k):
        start.wait()
        done[k] = samples[k][2]()
    ths = [threading.Thread(target=work, args=(k,)) for k in range(nth)]
    for t in ths:
        t.start()
    start.wait()
    t0 = time.perf_counter()
    for t in ths:
        t.join()
    wall = time.perf_counter() - t0
    edges = sum(sm[0] for sm in samples)
    return {"value": L * edges / wall, "unit": "edges/s", "cores": nth, "kind": "oracle",
            "sample": f"{nth} threads, each the unchanged serial oracle on its own sample ({samples[0][1]}, ...; "
                      f"{edges} in-edges in all), fwd+bwd of each of the {L} layer shapes, {wall:.1f} s wall",
            "seconds": wall, "host": hi,
            "per_core": {"value": L * n1 / t1, "unit": "edges/s", "threads": 1, "sample": desc1,
                         "per_layer_ms": [{"fwd": 1e3 * a, "bwd": 1e3 * b, "edges_per_s": n1 / (a + b)}
                                          for a, b in per_layer]}}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    c, model, cfg = workload(args.config, args.model, args.hidden)
    src, dst, et, _, _ = make_inputs(c, model)
    vals = []
    per = max(2.0, 60.0 / max(1, args.steps + args.warmup))
    csr = _csr_order(c, dst)
    for i in range(args.warmup + args.steps):
        r = cpu_baseline(c, model, src, dst, et, per, csr)
        if i >= args.warmup:
            vals.append(r)
    v = statistics.median([r["value"] for r in vals])
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "edges/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "dtype": "f64",
            "data": "synthetic", "config": cfg, "vs_baseline": None,
            "cpu_baseline": {"value": v, "unit": "edges/s", "cores": vals[-1]["cores"], "kind": "oracle",
                             "sample": vals[-1]["sample"], "host": vals[-1]["host"],
                             "per_core": vals[-1]["per_core"]},
            "e2e": {"value": v, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # WG_DIST_BACKEND=gloo + WG_DIST_ONE_GPU=1: every rank on cuda:0 over gloo --
    # a functional check of the multi-rank path where only one GPU exists
    # (timings of such a run are meaningless; the product path is NCCL)
    backend = os.environ.get("WG_DIST_BACKEND", "nccl")
    if os.environ.get("WG_DIST_ONE_GPU") == "1":
        local = 0
    torch.cuda.set_device(local)
    group = None
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        group = dist.group.WORLD
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as wg
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import GNNStack, equal_blocks

    c, model, cfg = workload(args.config, args.model, args.hidden)
    dev = torch.device("cuda", local)
    P = args.rank_slice
    if P > 1 and (world > 1 or model == "gat"):
        raise SystemExit("--rank-slice: one process, GCN / SAGE / GIN / RGCN configs")
    if world > 1 and model == "gat":
        raise SystemExit("the 1-D multi-GPU partition covers GCN / SAGE / GIN / RGCN (DESIGN.md §9)")
    t0 = time.perf_counter()
    comm, bounds = None, None
    if P > 1 and c.E <= (1 << 31) // 8:
        # one rank of the P-way partition of a graph that fits this host: the
        # library partitions it (edge-balanced wg_partition_1d) and keeps the
        # rank's rows, in- and out-edges
        src, dst, et, x_np, labels_np = make_inputs(c, model)
        args.no_e2e, args.no_cpu = True, True
        comm = wg.Comm(emulate=(args.slice_rank, P), device=local, emulate_copy=args.emulate_xchg)
        cfg.update(rank_slice={"P": P, "rank": args.slice_rank,
                               "exchange": "emulated copy kernels (--emulate-xchg)" if args.emulate_xchg
                                           else "none (compute of the rank only)",
                               "note": "one rank of the P-way 1-D partition (edge-balanced) on one GPU through "
                                       "the library's distributed calls with the EMULATED communicator; no data "
                                       "moves between ranks (a timing run)"})
    elif P > 1:
        # one rank of the P-way partition: only the edges touching its block
        # exist here, so the blocks are equal T-aligned vertex ranges (the
        # seeded permutation scatters hubs: edges balance to ~1 %)
        import synth
        block, blocks = equal_blocks(c.V, P)
        vb, ve = blocks[args.slice_rank]
        bounds = [lo for lo, _ in blocks] + [c.V]
        src, dst = synth.make_graph_slice(c.V, c.E, vb, ve, seed=c.seed * 16, alpha=c.alpha)
        et, x_np = None, None
        labels_np = np.random.Generator(np.random.Philox(c.seed * 16 + 5)).integers(
            0, c.dims[-1], c.V).astype(np.int64)[vb:ve]
        args.no_e2e, args.no_cpu = True, True
        comm = wg.Comm(emulate=(args.slice_rank, P), device=local, emulate_copy=args.emulate_xchg)
        cfg.update(rank_slice={"P": P, "rank": args.slice_rank, "v_begin": vb, "v_end": ve,
                               "edges_touching_block": int(src.shape[0]),
                               "exchange": "emulated copy kernels (--emulate-xchg)" if args.emulate_xchg
                                           else "none (compute of the rank only)",
                               "note": "per-rank compute of the P-way 1-D partition on one GPU: the rank's "
                                       "in-edges (forward) and out-edges (backward) through the library's "
                                       "distributed calls with the EMULATED communicator (with --emulate-xchg "
                                       "every exchange is a copy kernel on the communication stream rewriting "
                                       "the non-owned rows, overlapped chunk by chunk with the gathers as the "
                                       "NCCL exchange would be); no data moves between ranks and non-owned "
                                       "degrees are not the global ones (a timing run)",
                               "features": "torch.randn on the device (the 111M x 128 table is not built on the host)"})
    else:
        src, dst, et, x_np, labels_np = make_inputs(c, model)
        if world > 1:
            comm = wg.Comm(group, device=local)      # NCCL inside libwg (wg_comm_init)
    t_gen = time.perf_counter() - t0
    R = c.R if model == "rgcn" else 1
    if args.tune and P <= 1 and world == 1 and model != "gat":
        from paper_conf_eurosys_huangz0wjzzzys24_b200 import tune
        T_, Em, rep = tune.search(src, dst, c.V, model, c.dims, torch.bfloat16 if c.dtype == "bf16" else torch.float32,
                                  etype=et if R > 1 else None, R=R, cache_path=args.tune_cache,
                                  conv_kw=conv_options(c, model) if model != "gat" else {"heads": c.heads})
        args.tile, args.emax = T_, Em
        cfg["strategy_search"] = rep
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    g = wg.Graph(torch.from_numpy(src).to(dev), torch.from_numpy(dst).to(dev), num_vertices=c.V,
                 etype=torch.from_numpy(et).to(dev) if R > 1 else None, num_types=R,
                 max_task_edges=args.emax, tile_rows=args.tile, comm=comm, bounds=bounds)
    vb, ve = g.v_begin, g.v_begin + g.n_rows
    if P > 1 and x_np is not None:
        labels_np = labels_np[vb:ve]
        cfg["rank_slice"].update(v_begin=vb, v_end=ve, bounds=[int(b) for b in g.bounds],
                                 rank_in_edges=int(g.E_fwd), rank_out_edges=int(g.E_T))
    if world > 1:
        cfg.update(partition={"bounds": [int(b) for b in g.bounds], "rank_rows": ve - vb,
                              "rank_in_edges": int(g.E_fwd), "rank_out_edges": int(g.E_T),
                              "rule": "edge-balanced T-aligned blocks (wg_partition_1d)"})
    if P > 1:
        src = dst = None   # host copies of the slice are not needed any more
    torch.cuda.synchronize()
    t_part = time.perf_counter() - t0
    dtype = torch.bfloat16 if c.dtype == "bf16" else torch.float32
    t0 = time.perf_counter()
    stack = GNNStack(g, model, c.dims, dtype=dtype, policy=args.policy, heads=c.heads if model == "gat" else 1, R=R,
                     conv_kw=conv_options(c, model))
    t_plan = time.perf_counter() - t0
    x = wg.padded(c.V, c.dims[0], dtype, dev)
    if x_np is not None:
        x.copy_(torch.from_numpy(x_np).to(dev))
    else:
        gen = torch.Generator(device=dev).manual_seed(c.seed * 16 + 2)
        for r0 in range(0, c.V, 1 << 22):
            r1 = min(c.V, r0 + (1 << 22))
            x[r0:r1].copy_(torch.randn((r1 - r0, c.dims[0]), generator=gen, device=dev))
    labels = torch.from_numpy(labels_np[vb:ve] if world > 1 else labels_np).to(dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()

    clocks = Clocks(local)
    clocks.start()
    for _ in range(args.warmup):
        stack.step(x, labels, c.V)
    torch.cuda.synchronize()
    barrier()
    # One training step captured in a CUDA graph (one process per GPU; the
    # library's NCCL exchanges and gradient all-reduces run on its
    # communication stream, forked from and joined back into the captured
    # stream, so they are captured too): the timed region replays it K times,
    # so host launch overhead (ctypes marshalling, ~20-55 launches per step)
    # leaves the step time.  Per-kernel times come from the profiled eager pass below
    # (the same launches; a graph replay has no per-kernel events).
    graph, graph_err = None, None
    if not args.no_graph:
        try:
            side = torch.cuda.Stream(device=dev)
            side.wait_stream(stream)
            with torch.cuda.stream(side):
                for _ in range(2):
                    stack.step(x, labels, c.V)
            stream.wait_stream(side)
            torch.cuda.synchronize()
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph):
                loss_g = stack.step(x, labels, c.V)
            for _ in range(2):
                graph.replay()
            torch.cuda.synchronize()
        except Exception as ex:  # capture unsupported here: time eager steps
            graph, graph_err = None, f"{type(ex).__name__}: {ex}"[:200]
            torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    step_ms = None
    if graph is not None:
        barrier()
        clocks.mark_start()
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps - 1)]
        ev0.record(stream)
        for k in range(args.steps):
            graph.replay()
            if k < args.steps - 1:
                evs[k].record(stream)
        ev1.record(stream)
        torch.cuda.synchronize()
        clocks.mark_stop()
        loss = loss_g
        ms_graph = ev0.elapsed_time(ev1) / args.steps
        marks = [ev0] + evs + [ev1]
        step_ms = [marks[k].elapsed_time(marks[k + 1]) for k in range(args.steps)]
    wg.profile("start")
    n0 = wg.launch_count()
    torch.cuda.synchronize()
    barrier()
    if graph is None:
        clocks.mark_start()
    stack.layer_events = []
    ev0.record(stream)
    evs_e = []
    for _ in range(args.steps):
        loss_e = stack.step(x, labels, c.V)
        evs_e.append(torch.cuda.Event(enable_timing=True))
        evs_e[-1].record(stream)
    ev1.record(stream)
    torch.cuda.synchronize()
    lay = {}
    for key, a, b in stack.layer_events:
        lay[key] = lay.get(key, 0.0) + a.elapsed_time(b) / args.steps
    stack.layer_events = None
    if step_ms is None:
        marks = [ev0] + evs_e
        step_ms = [marks[k].elapsed_time(marks[k + 1]) for k in range(args.steps)]
    if graph is None:
        clocks.mark_stop()
        loss = loss_e
    barrier()
    launches = (wg.launch_count() - n0) // args.steps
    prof = wg.profile("collect")
    wg.profile("stop")
    ms_eager = ev0.elapsed_time(ev1) / args.steps
    ms = ms_graph if graph is not None else ms_eager
    if world > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    L = len(c.dims) - 1
    # rank slice: the edges this GPU aggregates per layer pass (its in-edges)
    E_units = g.E_fwd if P > 1 else c.E
    value = L * E_units / (ms / 1e3)
    # per layer: edges/s = E / (t_fwd + t_bwd), CUDA events
    # around each layer call in the profiled eager pass (this rank's edges)
    per_layer = [{"layer": i, "f_in": c.dims[i], "f_out": c.dims[i + 1], "fwd_ms": lay.get(("fwd", i), 0.0),
                  "bwd_ms": lay.get(("bwd", i), 0.0),
                  "edges_per_s": g.E_fwd / ((lay.get(("fwd", i), 0.0) + lay.get(("bwd", i), 0.0)) / 1e3)
                  if lay.get(("fwd", i), 0.0) + lay.get(("bwd", i), 0.0) > 0 else None}
                 for i in range(L)]
    qs = np.percentile(np.array(step_ms), [10, 50, 90]).tolist()
    step_stats = {"median_ms": qs[1], "p10_ms": qs[0], "p90_ms": qs[2], "n": len(step_ms),
                  "source": "CUDA events between graph replays" if graph is not None
                  else "CUDA events between eager steps"}

    # ---- end to end through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        # End to end through the public API: every step copies its inputs
        # (features, labels) from pinned host memory and reads the loss back.
        # Input loading is double-buffered like a data loader: step i+1's copy
        # runs on a second stream while step i computes (its buffer was last
        # read by step i-1), so the timed region holds all K copies.
        xh = torch.from_numpy(x_np).to(dtype).pin_memory()
        lh = torch.from_numpy(labels_np[vb:ve] if world > 1 else labels_np).pin_memory()
        loss_h = torch.empty(1, dtype=torch.float32).pin_memory()
        xs = [x, wg.padded(c.V, c.dims[0], dtype, dev)]
        ls = [labels, torch.empty_like(labels)]
        cstream = torch.cuda.Stream(device=dev)
        done = [torch.cuda.Event(), torch.cuda.Event()]
        ready = [torch.cuda.Event(), torch.cuda.Event()]

        def issue_copy(b):
            cstream.wait_event(done[b])
            with torch.cuda.stream(cstream):
                xs[b].copy_(xh, non_blocking=True)
                ls[b].copy_(lh, non_blocking=True)
            ready[b].record(cstream)

        # the training step on input buffer b as a CUDA graph when the device
        # leg captured one (the loss read-back stays outside the graph)
        egraphs = [None, None]
        if graph is not None and os.environ.get("WG_E2E_GRAPH", "1") == "1":
            try:
                for b in range(2):
                    gb = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(gb):
                        eloss = stack.step(xs[b], ls[b], c.V)
                    egraphs[b] = gb
            except Exception:
                egraphs = [None, None]
            torch.cuda.synchronize()

        def run_steps(n, start_ev=None):
            if start_ev is not None:
                cstream.wait_event(start_ev)
            issue_copy(0)
            for i in range(n):
                b = i % 2
                if i + 1 < n:
                    issue_copy(1 - b)
                stream.wait_event(ready[b])
                if egraphs[b] is not None:
                    egraphs[b].replay()
                    loss_h.copy_(eloss.reshape(1), non_blocking=True)
                else:
                    loss_h.copy_(stack.step(xs[b], ls[b], c.V).reshape(1), non_blocking=True)
                done[b].record(stream)

        run_steps(2)
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        clocks.mark_start()
        e0.record(stream)
        run_steps(args.steps, e0)
        e1.record(stream)
        torch.cuda.synchronize()
        clocks.mark_stop()
        barrier()
        ems = e0.elapsed_time(e1) / args.steps
        if world > 1:
            t = torch.tensor([ems], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": L * c.E / (ems / 1e3), "unit": "edges/s", "ms_per_step": ems,
               "h2d_bytes_per_step": int(xh.numel() * xh.element_size() + lh.numel() * 8),
               "d2h_bytes_per_step": 4, "loss": float(loss_h.item()),
               "input_pipeline": "double-buffered: step i+1's H2D copy overlaps step i on a second stream",
               "launch_mode": "cuda_graph_replay" if egraphs[0] is not None else "eager"}

    clk = clocks.stop()
    pk, pk_src = peaks()
    # dominant kernel class: the most time among classes that report algorithmic bytes
    # (gather_reduce = k_agg_cp / k_agg, a6 + a10; gat = the GAT edge kernels)
    dom = max((k for k in prof if prof[k]["bytes"] > 0), key=lambda k: prof[k]["ms"])
    agg = prof[dom]
    achieved = agg["bytes"] / (agg["ms"] / 1e3) / 1e9 if agg["ms"] > 0 else 0.0
    traffic, traffic_src = None, None
    tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tf):
        try:
            tr = json.load(open(tf)).get(f"{args.config}:{model}:{dom}")
            traffic = tr["bytes_per_launch"] if tr else None
            traffic_src = tr["source"] if tr else None
        except Exception:
            traffic = None
    names = {"gather_reduce": "k_agg_cp / k_agg (gather + segment-reduce, a6/a10)",
             "gat": "GAT edge kernels (logits + online softmax + gather, a6/a10)",
             "tc_gemm_nt": "tcgen05 GEMM-NT (a5/a7/a9)", "tc_gemm_tn": "tcgen05 GEMM-TN (a11)"}
    roofline = {"bound": "hbm", "kernel": names.get(dom, dom), "class": dom, "achieved": achieved,
                "peak": pk["hbm_gbs"], "unit": "GB/s", "frac": achieved / pk["hbm_gbs"], "traffic": traffic,
                "traffic_source": f"profiles/ncu_traffic.json: {traffic_src}" if traffic else None,
                "peak_source": f"{pk_src} (MEASURED_PEAKS.json hbm_gbs)" if pk_src == "measured" else "fallback",
                "bytes_per_launch": agg["bytes"] / max(1, agg["launches"]),
                "launches_per_step": agg["launches"] / args.steps,
                "share_of_step": (agg["ms"] / args.steps) / ms_eager,
                "timed_over": "CUDA events around every launch of the class on its stream, over the K-step "
                              "profiled eager pass (a graph replay has no per-kernel events)"}
    kernels = {}
    for k, v in prof.items():
        if v["launches"] == 0:
            continue
        kernels[k] = {"ms_per_step": v["ms"] / args.steps, "launches_per_step": v["launches"] / args.steps,
                      "enclosing_scope": v["bytes"] == 0 and k in ("rgcn",),
                      "GB/s": v["bytes"] / (v["ms"] / 1e3) / 1e9 if v["ms"] else None,
                      "TFLOP/s": v["flops"] / (v["ms"] / 1e3) / 1e12 if v["ms"] else None}
    line = {"metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "bf16" if dtype == torch.bfloat16 else "f32",
            "data": "synthetic (seeded power-law graph, N(0,1) features, uniform labels, random-init weights)",
            "config": dict(cfg, parallelism=f"1-D dst partition x{world}" if world > 1 else "single GPU",
                           epoch_time_ms=ms,
                           launch_mode="cuda_graph_replay" if graph is not None else "eager",
                           graph_capture_error=graph_err,
                           eager_profiled_ms_per_step=ms_eager, l2="inputs larger than L2 (no flush needed)",
                           max_in_degree=int(g.max_in_degree), E_max=int(g.E_max),
                           plans=[{"edge_tasks": cv.n_edge_tasks, "vertex_tasks": cv.n_vertex_tasks,
                                   "bwd_path": cv.bwd_path, "items": cv.n_items, "items_T": cv.n_items_T,
                                   "split_rows": cv.n_split_rows, "xchg_cols": [cv.xchg_fwd, cv.xchg_bwd]}
                                  for cv in stack.convs]),
            "gpu_launches": int(launches), "roofline": roofline, "kernels": kernels,
            "step_time": step_stats, "per_layer": per_layer,
            "one_off": {"partition_s": t_part, "plan_s": t_plan, "synth_s": t_gen},
            "clocks": clk, "loss": float(loss.item()), "e2e": e2e}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(c, model, src, dst, et, args.cpu_seconds)
    elif rank == 0:
        line["cpu_baseline"] = None
    if rank == 0:
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
