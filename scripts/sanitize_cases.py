"""Small forward + backward instances of every kernel family, for
compute-sanitizer (memcheck / racecheck / synccheck / initcheck):

  k_agg_cp (every ring shape: 4 / 8 / 16 / 32 lanes per row), k_agg,
  k_combine and the overfill cluster kernel k_agg_heavy (SPLIT rows), k_gemm_nt_p (bf16 and 3xTF32, split / chunked
  outputs), k_tc_gemm (TN split-K), GAT edge kernels, RGCN stage kernels,
  the softmax cross-entropy, the column-sum pass, the general restriction
  engine (k_greedy, k_gagg), the SAGE-LSTM step kernels.

Sizes are tiny (the sanitizers slow kernels down 10-100x) but span several
tiles, a ragged tail and SPLIT chunks.  Usage:
  compute-sanitizer --tool racecheck python scripts/sanitize_cases.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
import paper_conf_eurosys_huangz0wjzzzys24_b200 as m  # noqa: E402


def run(model, dtype, fi, fo, policy="auto", V=700, E=9000, E_max=64, heads=1, R=1, concat=True, alpha=0.8):
    src, dst, et = synth.make_graph(V, E, seed=fi + fo, alpha=alpha if model != "sage_lstm" else 0.3, R=R)
    kw = dict(etype=torch.from_numpy(et).cuda(), num_types=R) if R > 1 else {}
    g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V, max_task_edges=E_max,
                **kw)
    ckw = dict(heads=heads, concat=concat) if model == "gat" else {}
    if model == "sage_lstm":
        policy = "auto"
    if model == "rgcn":
        ckw.update(norm="right", self_loop=True)
    conv = m.Conv(g, model, fi, fo, dtype=dtype, policy=policy, fuse_relu=True, **ckw)
    params = m.init_params(model, fi, fo, heads=heads, concat=concat, R=R, self_loop=model == "rgcn", seed=1)
    x = m.pad_to(torch.from_numpy(synth.make_features(V, fi, seed=2)).to(dtype).cuda())
    y, saved = conv.forward_raw(x, params)
    dy = m.pad_to(torch.randn(y.shape, device="cuda").to(dtype))
    conv.backward_raw(dy, x, y, saved, params)
    torch.cuda.synchronize()


def main():
    for dtype in (torch.bfloat16, torch.float32):
        for F in (16, 32, 47, 64, 128, 256):          # every lanes-per-row ring shape
            run("sage", dtype, F, F, "edge")
        for policy in ("edge", "vertex", "random"):
            run("gcn", dtype, 40, 24, policy)
            run("gin", dtype, 24, 40, policy)
        run("gat", dtype, 32, 16, heads=4)
        run("gat", dtype, 32, 16, heads=2, concat=False)
        for policy in ("edge", "vertex", "random"):
            run("rgcn", dtype, 32, 16, policy, R=5)
    # chunked exchange tables (P = 2 partitions on one GPU)
    from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import equal_blocks
    V, E, F = 1000, 12000, 256
    src, dst, _ = synth.make_graph(V, E, seed=5, alpha=0.7)
    ts, td = torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda()
    _, bl = equal_blocks(V, 2)
    x = m.pad_to(torch.randn(V, F, device="cuda").to(torch.bfloat16))
    params = m.init_params("sage", F, F, seed=3)
    for policy in ("vertex", "edge"):
        parts = []
        for vb, ve in bl:
            g = m.Graph(ts, td, num_vertices=V, v_begin=vb, v_end=ve)
            parts.append((g, m.Conv(g, "sage", F, F, dtype=torch.bfloat16, policy=policy, fuse_relu=True), vb, ve))
        c0 = parts[0][1]
        xf, xb = c0.new_xchg(0), c0.new_xchg(1)
        y = m.padded(V, F, torch.bfloat16)
        sv = [c.new_saved() for _, c, _, _ in parts]
        for ph in ((1, 2) if xf is not None else (0,)):
            for (g, c, vb, ve), s in zip(parts, sv):
                c.forward_raw(x, params, y=y[vb:ve], saved=s, phase=ph, xchg=xf)
        dy = m.pad_to(torch.randn(V, F, device="cuda").to(torch.bfloat16))
        dx = m.padded(V, F, torch.bfloat16)
        for ph in (1, 2):
            for (g, c, vb, ve), s in zip(parts, sv):
                c.backward_raw(dy[vb:ve], x, y[vb:ve], s, params, dx=dx[vb:ve], phase=ph, xchg=xb)
    torch.cuda.synchronize()
    # general restriction engine + atomic executor, SAGE-LSTM
    src, dst, et = synth.make_graph(800, 9000, seed=9, alpha=0.8, R=3)
    for spec in ([("dst", 4)], [("src", 8), ("type", 1)], [("dst", 16), ("dst_degree", "min")], [("edge", 32)]):
        gp = m.GPart(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=800, restrictions=spec,
                     etype=torch.from_numpy(et).cuda())
        gp.aggregate(m.pad_to(torch.randn(800, 32, device="cuda").to(torch.bfloat16)), norm="both")
    run("sage_lstm", torch.float32, 16, 8, "edge", V=300, E=900)   # few LSTM steps (launch count)
    torch.cuda.synchronize()
    # fused softmax cross-entropy
    lg = m.pad_to(torch.randn(3000, 47, device="cuda").to(torch.bfloat16))
    lab = torch.randint(0, 47, (3000,), device="cuda")
    m.softmax_xent(lg, lab, 1.0 / 3000, m.padded(3000, 47, torch.bfloat16), torch.zeros(1, device="cuda"))
    torch.cuda.synchronize()
    print("sanitize cases: done, launches", m.launch_count())


if __name__ == "__main__":
    main()
