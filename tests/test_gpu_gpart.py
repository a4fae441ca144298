"""General restriction engine on the GPU == the oracle's.

Partition: perm and gTask tables bit-exact against oracle.partition_general
(the greedy of P:L1431-1451 under Fig 7's restrictions, and
Fig 9's source-based ones) on the worked example and on random typed graphs.
Executor: the atomic Index / Index-add aggregation over the gTasks of every
restriction set equals the oracle's aggregation (GCN with W = I, Q3
coefficients) -- one result for every partition plan."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from tests.util import TOL, f64, rel_err

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "restrictions.json")))

SPECS = [
    [("dst", 1)], [("dst", 4)], [("edge", 1)], [("src", 8), ("type", 1)], [("dst", 2), ("src", 2)],
    [("dst_degree", 1)], [("dst", 16), ("dst_degree", "min")], [("dst", 8), ("edge", 64)],
    [("type", 1), ("dst", 3), ("src", 5)], [("src", "min"), ("dst", 32)], [("dst_degree", 2), ("type", 1)], [],
]


def wg():
    import paper_conf_eurosys_huangz0wjzzzys24_b200 as m
    return m


@pytest.mark.parametrize("case", GOLD["cases"], ids=[c["fig"] for c in GOLD["cases"]])
def test_worked_example(case):
    m = wg()
    E = np.array(GOLD["edges_eid_dst_src_type"])
    d, s, t = E[:, 1].astype(np.int32), E[:, 2].astype(np.int32), E[:, 3].astype(np.int32)
    gp = m.GPart(s, d, num_vertices=GOLD["V"], restrictions=[tuple(r) for r in case["restrictions"]], etype=t)
    perm, tasks = gp.export()
    assert [perm[a:b].tolist() for a, b in zip(tasks["e_begin"], tasks["e_end"])] == case["tasks"]


@pytest.mark.parametrize("spec", SPECS, ids=[str(s) for s in SPECS])
def test_partition_bit_exact(spec):
    m = wg()
    V, E, R = 3000, 40000, 6
    src, dst, et = synth.make_graph(V, E, seed=17, alpha=0.8, R=R)
    gp = m.GPart(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V, restrictions=spec,
                 etype=torch.from_numpy(et).cuda())
    perm, tasks = gp.export()
    p_o, t_o = oracle.partition_general(src, dst, V, spec, etype=et)
    np.testing.assert_array_equal(perm, p_o)
    for k in ("tile", "type", "e_begin", "e_end", "d_lo", "d_hi", "flags", "n_uniq_src"):
        np.testing.assert_array_equal(tasks[k], t_o[k], err_msg=k)


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("norm", ["both", "right", "none"])
def test_atomic_executor_plan_invariant(dtype, norm):
    m = wg()
    V, E, F = 2500, 30000, 48
    src, dst, et = synth.make_graph(V, E, seed=23, alpha=0.8, R=4)
    x = torch.from_numpy(synth.make_features(V, F, seed=24)).to(dtype)
    xd = m.pad_to(x.cuda())
    ref = oracle.gcn_forward(src, dst, V, f64(x), np.eye(F), None, norm=norm)
    for spec in SPECS:
        gp = m.GPart(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=V, restrictions=spec,
                     etype=torch.from_numpy(et).cuda())
        out = gp.aggregate(xd, norm=norm)
        torch.cuda.synchronize()
        assert rel_err(f64(out), ref) <= TOL[dtype], (spec, rel_err(f64(out), ref))
