"""Pins for the oracle's gTask partition (Fig 7).

The oracle is pinned against: the hand-derived partitions of the paper's
worked example (tests/golden/worked_example.json), the limit cases the paper
names (vertex-centric, edge-centric, K=INF tensor-centric; P:L1583-1592,
P:L3800-3806), and structural invariants that any correct greedy partition
must satisfy (checked by brute force on random graphs).
"""
import numpy as np
import pytest

import oracle
import synth


def _check_against_golden(ex, part):
    src, dst, et = np.array(ex["src"]), np.array(ex["dst"]), np.array(ex["etype"])
    if part["transposed"]:
        kv, ov = src, dst
    else:
        kv, ov = dst, src
    perm, tasks = oracle.partition(kv, ov, et, by_type=part["by_type"], T=part["T"], E_max=part["E_max"])
    assert perm.tolist() == part["perm"], part["name"]
    assert len(tasks) == len(part["tasks"]), part["name"]
    for t, g in zip(tasks, part["tasks"]):
        assert perm[t["e_begin"]:t["e_end"]].tolist() == g["edges"], part["name"]
        for k in ("tile", "type", "d_lo", "d_hi", "flags", "n_uniq_src"):
            assert int(t[k]) == g[k], (part["name"], k)


def test_worked_example_partitions(worked_example):
    for part in worked_example["partitions"]:
        _check_against_golden(worked_example, part)


def test_worked_example_transposed_fwdpos(worked_example):
    ex = worked_example
    src, dst = np.array(ex["src"]), np.array(ex["dst"])
    perm, _ = oracle.partition(dst, src, T=1, E_max=10**6)
    perm_t, tasks_t, fwdpos = oracle.transposed(src, dst, T=1, E_max=10**6, perm_fwd=perm)
    assert (perm[fwdpos] == perm_t).all()


def _invariants(kv, ov, et, by_type, T, E_max, perm, tasks):
    E = kv.shape[0]
    assert sorted(perm.tolist()) == list(range(E))          # perm is a permutation
    ty = et if (by_type and et is not None) else np.zeros(E, np.int64)
    # sorted by (tile, type, kv, eid)
    keys = list(zip(kv[perm] // T, ty[perm], kv[perm], perm))
    assert keys == sorted(keys)
    # tasks contiguous, disjoint, covering [0, E)
    pos = 0
    for t in tasks:
        assert t["e_begin"] == pos and t["e_end"] > t["e_begin"]
        pos = t["e_end"]
    assert pos == E
    seglen = {}
    for v, r in zip(kv, ty):
        seglen[(int(v), int(r))] = seglen.get((int(v), int(r)), 0) + 1
    for i, t in enumerate(tasks):
        ed = perm[t["e_begin"]:t["e_end"]]
        assert len(set((kv[ed] // T).tolist())) == 1 and int(kv[ed][0] // T) == t["tile"]
        assert len(set(ty[ed].tolist())) == 1 and int(ty[ed][0]) == t["type"]
        assert t["d_lo"] == kv[ed].min() and t["d_hi"] == kv[ed].max()
        assert t["n_uniq_src"] == len(set(ov[ed].tolist()))
        n_e = len(ed)
        assert n_e <= E_max
        if t["flags"] & oracle.SPLIT:
            # a SPLIT chunk holds one key vertex whose segment exceeds E_max
            assert t["d_lo"] == t["d_hi"] and seglen[(int(t["d_lo"]), int(t["type"]))] > E_max
        else:
            # every segment in a regular task is whole and not over-long
            for v in set(kv[ed].tolist()):
                assert seglen[(v, int(t["type"]))] <= E_max
                assert int((kv[ed] == v).sum()) == seglen[(v, int(t["type"]))]
    # greedy maximality: a regular task could not have absorbed the next
    # segment of its group (else the greedy scan would have appended it)
    for a, b in zip(tasks[:-1], tasks[1:]):
        if a["flags"] or b["flags"] or a["tile"] != b["tile"] or a["type"] != b["type"]:
            continue
        first_seg = seglen[(int(b["d_lo"]), int(b["type"]))]
        assert (a["e_end"] - a["e_begin"]) + first_seg > E_max


@pytest.mark.parametrize("seed,V,E,R,T,E_max", [
    (1, 50, 400, 1, 8, 16), (2, 64, 900, 3, 16, 40), (3, 200, 3000, 1, 128, 64),
    (4, 37, 500, 5, 4, 7), (5, 300, 5000, 2, 32, 1024),
])
def test_partition_invariants(seed, V, E, R, T, E_max):
    src, dst, et = synth.small_graph(V, E, seed=seed, R=R, alpha=0.6)
    for by_type in ((False, True) if R > 1 else (False,)):
        perm, tasks = oracle.partition(dst, src, et, by_type=by_type, T=T, E_max=E_max)
        _invariants(dst, src, et, by_type, T, E_max, perm, tasks)
        perm_t, tasks_t, fwdpos = oracle.transposed(src, dst, et, by_type=by_type, T=T, E_max=E_max, perm_fwd=perm)
        _invariants(src, dst, et, by_type, T, E_max, perm_t, tasks_t)
        assert (perm[fwdpos] == perm_t).all()


def test_limit_vertex_centric_is_csr():
    # T=1, no type, E_max=inf: one task per non-empty dst row, in CSR order
    src, dst, _ = synth.small_graph(100, 1200, seed=9)
    perm, tasks = oracle.partition(dst, src, T=1, E_max=10**9)
    indptr = np.concatenate([[0], np.cumsum(np.bincount(dst, minlength=100))])
    nz = np.nonzero(np.diff(indptr))[0]
    assert [int(t["d_lo"]) for t in tasks] == nz.tolist()
    assert [int(t["e_begin"]) for t in tasks] == indptr[nz].tolist()
    assert (perm == np.argsort(dst, kind="stable")).all()


def test_limit_edge_centric_singletons():
    src, dst, _ = synth.small_graph(50, 300, seed=10)
    perm, tasks = oracle.partition(dst, src, T=4, E_max=1)
    assert len(tasks) == 300 and all(t["e_end"] - t["e_begin"] == 1 for t in tasks)


def test_limit_tensor_centric_single_task():
    src, dst, _ = synth.small_graph(50, 300, seed=11)
    perm, tasks = oracle.partition(dst, src, T=64, E_max=10**9)
    assert len(tasks) == 1 and tasks[0]["n_uniq_src"] == len(set(src.tolist()))


def test_default_emax_rule():
    # Q13 values quoted in SURVEY.md §8(a) a2 for the BASELINE configs
    assert oracle.default_emax(2708, 10556) == 2048
    assert oracle.default_emax(169343, 1166243) == 4096
    assert oracle.default_emax(1939743, 21111007) == 8192
    assert oracle.default_emax(2449029, 61859140) == 16384
    assert oracle.default_emax(111059956, 1615685872) == 8192
