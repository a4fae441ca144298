"""Input generator checks (host only)."""
import numpy as np

import synth


def test_graph_slice_equals_filtered_full_graph():
    """make_graph_slice (one rank's share of the 1-D partition, drawn chunk by
    chunk) returns exactly the full graph's edges touching the block, in order."""
    V, E, lo, hi = 5000, 200000, 1280, 2560
    s, d, _ = synth.make_graph(V, E, seed=7, alpha=0.5)
    ss, dd = synth.make_graph_slice(V, E, lo, hi, seed=7, alpha=0.5, chunk=30000)
    keep = ((d >= lo) & (d < hi)) | ((s >= lo) & (s < hi))
    assert np.array_equal(ss, s[keep]) and np.array_equal(dd, d[keep])
