"""Fig 19-style breakdown of the differentiated outlier execution (SURVEY
§8(f) f1) on skewed synthetic graphs: one SAGE layer forward +
backward (bf16, C2 / C4 graph shapes) with the overfill cluster kernel and
the underfill merge switched on / off (WG_HEAVY, WG_UNDERFILL are read once
per process, so every variant runs in its own process).

    python scripts/outlier_breakdown.py > profiles/r02/outlier_breakdown.md
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import json, sys, numpy as np, torch
sys.path.insert(0, %(root)r)
import synth, paper_conf_eurosys_huangz0wjzzzys24_b200 as m
cfg, fi, fo, emax = %(cfg)r, %(fi)d, %(fo)d, %(emax)d
c = synth.CONFIGS[cfg]
src, dst, _ = synth.make_graph(c.V, c.E, seed=c.seed * 16, alpha=c.alpha, symmetric=c.symmetric)
g = m.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V, max_task_edges=emax)
conv = m.Conv(g, "sage", fi, fo, dtype=torch.bfloat16, fuse_relu=True, policy="edge")
p = m.init_params("sage", fi, fo, seed=1)
x = m.padded(c.V, fi, torch.bfloat16); x.normal_()
dy = m.padded(c.V, fo, torch.bfloat16); dy.normal_()
y, sv = conv.forward_raw(x, p)
conv.backward_raw(dy, x, y, sv, p)
m.profile("start")
ts = []
for _ in range(10):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); conv.forward_raw(x, p, y=y, saved=sv); conv.backward_raw(dy, x, y, sv, p); e1.record()
    torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
prof = m.profile("collect"); m.profile("stop")
print(json.dumps({"ms": float(np.median(ts)), "split_rows": conv.n_split_rows, "items": conv.n_items,
                  "E_max": int(g.E_max), "max_in_degree": int(g.max_in_degree),
                  "gather_ms": prof["gather_reduce"]["ms"] / 10, "outlier_ms": prof["split_combine"]["ms"] / 10}))
'''


def main():
    rows = []
    for cfg, fi, fo in (("C2", 128, 256), ("C4", 100, 256)):
        for emax in (0, 512):
            for heavy, under in (("0", "0"), ("1", "0"), ("0", "1"), ("1", "1")):
                code = CHILD % dict(root=ROOT, cfg=cfg, fi=fi, fo=fo, emax=emax)
                r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=900,
                                   env=dict(os.environ, WG_HEAVY=heavy, WG_UNDERFILL=under))
                try:
                    d = json.loads(r.stdout.strip().splitlines()[-1])
                except Exception:
                    d = {"error": (r.stderr or r.stdout)[-300:]}
                rows.append((cfg, fi, fo, emax, heavy, under, d))
    print("# Differentiated outlier execution: breakdown (round 2)\n")
    print("One SAGE layer (bf16, EDGE plan, fused ReLU) forward + backward, median of 10 (CUDA events); "
          "`outlier ms` = the overfill cluster kernel (WG_HEAVY=1) or the SPLIT combine (WG_HEAVY=0) per "
          "iteration (wg_profile class split_combine); `gather ms` = k_agg class.\n")
    print("| graph | f_in->f_out | E_max | overfill rows | overfill kernel | underfill merge | work items | ms | gather ms | outlier ms |")
    print("|---|---|---|---|---|---|---|---|---|---|")
    for cfg, fi, fo, emax, heavy, under, d in rows:
        if "error" in d:
            print(f"| {cfg} | {fi}->{fo} | {emax or 'default'} | | {heavy} | {under} | error: {d['error'][:80]} | | | |")
            continue
        print(f"| {cfg} | {fi}->{fo} | {d['E_max']} | {d['split_rows']} | {'cluster' if heavy == '1' else 'partials+combine'} "
              f"| {'on' if under == '1' else 'off'} | {d['items']} | {d['ms']:.3f} | {d['gather_ms']:.3f} | {d['outlier_ms']:.3f} |")


if __name__ == "__main__":
    main()
