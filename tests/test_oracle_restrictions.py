"""The general restriction engine of the oracle (P:L1391-1451,
Fig 7) against hand-derived partitions of the paper's worked
example (tests/golden/restrictions.json), limit cases that reduce to the
pinned tile engine or to fixed-size chunks, and brute-force invariants on
random graphs (every restriction holds, the greedy is maximal, the order is
the stated sort key)."""
import json
import os

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "restrictions.json")))


def example():
    E = np.array(GOLD["edges_eid_dst_src_type"])
    return E[:, 2].astype(np.int32), E[:, 1].astype(np.int32), E[:, 3].astype(np.int32), GOLD["V"]


def spec(r):
    return [(a, k) for a, k in r]


@pytest.mark.parametrize("case", GOLD["cases"], ids=[c["fig"] for c in GOLD["cases"]])
def test_worked_example_golden(case):
    s, d, t, V = example()
    perm, tasks = oracle.partition_general(s, d, V, spec(case["restrictions"]), etype=t)
    got = [perm[a:b].tolist() for a, b in zip(tasks["e_begin"], tasks["e_end"])]
    assert got == case["tasks"]


def values(a, s, d, t, deg, e):
    return {"dst": d[e], "src": s[e], "type": t[e] if t is not None else 0, "dst_degree": deg[d[e]], "edge": e}[a]


def check_invariants(s, d, t, V, restr):
    perm, tasks = oracle.partition_general(s, d, V, restr, etype=t)
    E = len(s)
    deg = np.bincount(d, minlength=V)
    assert sorted(perm.tolist()) == list(range(E))
    assert tasks["e_begin"][0] == 0 and tasks["e_end"][-1] == E
    assert (tasks["e_begin"][1:] == tasks["e_end"][:-1]).all() and (tasks["e_end"] > tasks["e_begin"]).all()
    # order: the sort key of Q25
    key = [a for a, k in restr if k == 1] + [a for a, k in restr if k == "min"] + \
          [a for a, k in restr if k not in (1, "min") and a != "edge"]
    key = list(dict.fromkeys(key))
    if "dst" not in key:
        key.append("dst")
    key.append("edge")
    kv = [tuple(values(a, s, d, t, deg, e) for a in key) for e in perm]
    assert kv == sorted(kv)
    lim = [(a, k) for a, k in restr if k != "min"]
    for i, (b, e) in enumerate(zip(tasks["e_begin"], tasks["e_end"])):
        es = perm[b:e]
        for a, k in lim:                              # every restriction holds
            assert len({values(a, s, d, t, deg, x) for x in es}) <= k
        if i + 1 < len(tasks):                        # maximal: the next edge breaks one of them
            nx = perm[e]
            assert any(len({values(a, s, d, t, deg, x) for x in list(es) + [nx]}) > k for a, k in lim)
        assert tasks["d_lo"][i] == d[es].min() and tasks["d_hi"][i] == d[es].max()
        assert tasks["n_uniq_src"][i] == len(set(s[es].tolist()))
    return perm, tasks


@pytest.mark.parametrize("restr", [
    [("dst", 1)], [("dst", 4)], [("src", 3), ("type", 1)], [("dst", 2), ("src", 2)], [("dst_degree", 1)],
    [("dst", 5), ("dst_degree", "min")], [("edge", 7)], [("dst", 8), ("edge", 16)], [("type", 1), ("dst", 3), ("src", 5)],
    [("src", "min"), ("dst", 4)], [("dst_degree", 2), ("type", 1)],
])
def test_random_graph_invariants(restr):
    src, dst, et = synth.make_graph(150, 1200, seed=len(restr) * 7 + len(str(restr)), alpha=0.7, R=4)
    check_invariants(src, dst, et, 150, restr)


def test_reduces_to_tile_engine_and_chunks():
    """uniq(dst) = 1 with no split equals the pinned tile engine at T = 1,
    E_max = inf (the vertex-centric CSR order); uniq(edge) = k alone is the
    edge order cut into k-edge chunks; no restriction at all is one task."""
    src, dst, _ = synth.make_graph(300, 4000, seed=3, alpha=0.6)
    p1, t1 = oracle.partition_general(src, dst, 300, [("dst", 1)])
    p2, t2 = oracle.partition(dst, src, T=1, E_max=1 << 40)
    np.testing.assert_array_equal(p1, p2)
    for k in ("e_begin", "e_end", "d_lo", "d_hi", "n_uniq_src"):
        np.testing.assert_array_equal(t1[k], t2[k])
    p3, t3 = oracle.partition_general(src, dst, 300, [("edge", 64)])
    assert (p3 == np.lexsort((np.arange(4000), dst))).all()      # key (dst, edge)
    assert (t3["e_end"] - t3["e_begin"])[:-1].tolist() == [64] * (len(t3) - 1)
    p4, t4 = oracle.partition_general(src, dst, 300, [])
    assert len(t4) == 1
