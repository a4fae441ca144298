"""Fraction of the non-owned rows a rank's gathers reference (C4 SAGE graph,
edge-balanced T-aligned 1-D partition as wg_partition_1d): what a
boundary-only exchange would save over the all-gather."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import synth  # noqa: E402

V, E, T = 2449029, 61859140, 128
src, dst, _ = synth.make_graph(V, E, seed=104 * 16, alpha=0.5, symmetric=True)
nt = -(-V // T)
w = np.bincount(src // T, minlength=nt) + np.bincount(dst // T, minlength=nt) + np.bincount(np.arange(V) // T, minlength=nt)
S = np.concatenate([[0], np.cumsum(w)])
for P in (2, 4, 8):
    b = [0]
    for q in range(1, P):
        tgt = S[-1] * q / P
        t = int(np.searchsorted(S, tgt))
        if t > 0 and S[t] - tgt > tgt - S[t - 1]:
            t -= 1
        b.append(t * T)
    b.append(V)
    fr = []
    for p in range(P):
        lo, hi = b[p], b[p + 1]
        s = np.unique(src[(dst >= lo) & (dst < hi)])
        fr.append(np.count_nonzero((s < lo) | (s >= hi)) / (V - (hi - lo)))
    print(f"P={P}: referenced fraction of the non-owned rows per rank: min {min(fr):.3f} mean {np.mean(fr):.3f} max {max(fr):.3f}")
