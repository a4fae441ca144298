"""GPU gTask partition (a2, a3) == oracle, bit for bit (BASELINE north_star:
"The gTask partition and edge permutation must be bit-exact")."""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


def gpu_graph(src, dst, V, et=None, R=1, T=128, E_max=0, vb=0, ve=0):
    return wg().Graph(torch.from_numpy(np.asarray(src, np.int32)).cuda(),
                      torch.from_numpy(np.asarray(dst, np.int32)).cuda(), num_vertices=V,
                      etype=None if et is None else torch.from_numpy(np.asarray(et, np.int32)).cuda(),
                      num_types=R, tile_rows=T, max_task_edges=E_max, v_begin=vb, v_end=ve)


def same_tasks(a, b):
    assert len(a) == len(b)
    for k in ("tile", "type", "e_begin", "e_end", "d_lo", "d_hi", "flags", "n_uniq_src"):
        np.testing.assert_array_equal(a[k], b[k], err_msg=k)


def test_worked_example_partitions(worked_example):
    ex = worked_example
    for part in ex["partitions"]:
        et = ex["etype"] if part["by_type"] else None
        g = gpu_graph(ex["src"], ex["dst"], ex["V"], et, R=2 if et else 1, T=part["T"], E_max=part["E_max"])
        perm, tasks, _ = g.export(transposed=part["transposed"])
        assert perm.tolist() == part["perm"], part["name"]
        assert len(tasks) == len(part["tasks"])
        for t, gt in zip(tasks, part["tasks"]):
            assert perm[t["e_begin"]:t["e_end"]].tolist() == gt["edges"], part["name"]
            for k in ("tile", "type", "d_lo", "d_hi", "flags", "n_uniq_src"):
                assert int(t[k]) == gt[k], (part["name"], k)


@pytest.mark.parametrize("V,E,R,T,E_max,seed,alpha", [
    (1000, 20000, 1, 128, 64, 1, 0.6), (3000, 60000, 7, 64, 200, 2, 0.5), (513, 4000, 1, 32, 1024, 3, 0.8),
    (20000, 400000, 1, 128, 0, 4, 0.5), (5000, 50000, 16, 128, 0, 5, 0.5), (77, 3000, 3, 16, 5, 6, 0.9),
])
def test_random_graphs_bit_exact(V, E, R, T, E_max, seed, alpha):
    src, dst, et = synth.make_graph(V, E, seed=seed, alpha=alpha, R=R)
    g = gpu_graph(src, dst, V, et, R=R, T=T, E_max=E_max)
    emax = g.E_max
    assert emax == (E_max or oracle.default_emax(V, E, T))
    by_type = R > 1
    perm, tasks = oracle.partition(dst, src, et, by_type=by_type, T=T, E_max=emax)
    gp, gt, _ = g.export()
    np.testing.assert_array_equal(gp, perm)
    same_tasks(gt, tasks)
    perm_t, tasks_t, fwdpos = oracle.transposed(src, dst, et, by_type=by_type, T=T, E_max=emax, perm_fwd=perm)
    gpt, gtt, gfp = g.export(transposed=True)
    np.testing.assert_array_equal(gpt, perm_t)
    same_tasks(gtt, tasks_t)
    np.testing.assert_array_equal(gfp, fwdpos)
    assert g.max_in_degree == np.bincount(dst, minlength=V).max()


@pytest.mark.parametrize("P", [2, 4])
def test_1d_partition_tables_are_slices(P):
    """§8(e): with T-aligned rank boundaries, each rank's tables are exact slices
    of the single-GPU oracle tables (edge positions rebased)."""
    V, E, T = 4000, 80000, 128
    src, dst, _ = synth.make_graph(V, E, seed=11, alpha=0.6)
    emax = oracle.default_emax(V, E, T)
    perm, tasks = oracle.partition(dst, src, T=T, E_max=emax)
    perm_t, tasks_t = oracle.partition(src, dst, T=T, E_max=emax)
    tiles = -(-V // T)
    bounds = [min(V, (tiles * p // P) * T) for p in range(P + 1)]
    for p in range(P):
        vb, ve = bounds[p], bounds[p + 1]
        g = gpu_graph(src, dst, V, T=T, E_max=emax, vb=vb, ve=ve)
        for (pm, tk, key, tr) in ((perm, tasks, dst, False), (perm_t, tasks_t, src, True)):
            gp, gt, _ = g.export(transposed=tr)
            sel = (key[pm] >= vb) & (key[pm] < ve)
            lo = int(np.argmax(sel)) if sel.any() else 0
            np.testing.assert_array_equal(gp, pm[sel])
            ts = tk[(tk["d_lo"] >= vb) & (tk["d_lo"] < ve)].copy()
            ts["e_begin"] -= lo
            ts["e_end"] -= lo
            same_tasks(gt, ts)


def test_csr_input_matches_coo():
    V, E = 2000, 30000
    src, dst, _ = synth.make_graph(V, E, seed=12, alpha=0.5)
    order = np.argsort(dst, kind="stable")
    s2, d2 = src[order], dst[order]
    indptr = np.concatenate([[0], np.cumsum(np.bincount(d2, minlength=V))]).astype(np.int64)
    g1 = gpu_graph(s2, d2, V)
    g2 = wg().Graph(torch.from_numpy(s2).cuda(), None, indptr=torch.from_numpy(indptr).cuda(), num_vertices=V)
    for tr in (False, True):
        a, b = g1.export(tr), g2.export(tr)
        np.testing.assert_array_equal(a[0], b[0])
        same_tasks(a[1], b[1])


def test_host_pointers_and_range_errors():
    V, E = 100, 500
    src, dst, _ = synth.make_graph(V, E, seed=13)
    m = wg()
    g = m.Graph(src, dst, num_vertices=V)        # host numpy arrays
    perm, _ = oracle.partition(dst, src, T=128, E_max=g.E_max)
    np.testing.assert_array_equal(g.export()[0], perm)
    bad = dst.copy()
    bad[7] = V
    with pytest.raises(m.WGError, match="out of range"):
        m.Graph(src, bad, num_vertices=V)
    with pytest.raises(m.WGError):
        m.Graph(src, dst, num_vertices=V, v_begin=3, v_end=50)  # not T-aligned


def test_empty_graph():
    g = gpu_graph(np.zeros(0, np.int32), np.zeros(0, np.int32), 10)
    perm, tasks, _ = g.export()
    assert len(perm) == 0 and len(tasks) == 0
