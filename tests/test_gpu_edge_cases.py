"""Degenerate inputs through the C ABI == oracle (fp64), all five models.

The cases the method has at its edges (③ "edge cases"):
  * a graph with no edges: every row is the empty-neighbourhood epilogue
    (bias / self term only), every weight gradient of the neighbour path is 0;
  * a star: all edges into one destination (one row far longer than any
    gTask, so degree-aware splitting cuts it into many SPLIT chunks,
    P:L2630-2636), or all edges out of one source (the same on the
    transposed partition, i.e. in the backward gather);
  * multi-edges (the star repeats every (src, dst) pair) and self-loops;
  * fewer edges than one CTA has workers, one vertex, one ragged row past a
    full tile.
The graphs are hand-built integer arrays (no method arithmetic)."""
import numpy as np
import pytest
import torch

from tests import test_gpu_conv_gat as gat
from tests import test_gpu_conv_lin as lin
from tests import test_gpu_conv_rgcn as rgcn
from tests.util import TOL

pytestmark = pytest.mark.gpu

LIN = ["gcn", "sage", "gin"]
DT = [torch.float32, torch.bfloat16]


def star_in(V, E, hub=0):
    rng = np.random.default_rng(V + E)
    src = rng.integers(0, V, E).astype(np.int32)
    return src, np.full(E, hub, np.int32)


def star_out(V, E, hub=0):
    d, s = star_in(V, E, hub)
    return s, d


def typed(edges, R, seed=0):
    src, dst = edges
    et = np.random.default_rng(seed).integers(0, R, len(src)).astype(np.int32)
    return src, dst, et


def empty():
    return np.zeros(0, np.int32), np.zeros(0, np.int32)


def check_errs(errs, dtype):
    bad = {k: v for k, v in errs.items() if not v <= TOL[dtype]}
    assert not bad, f"errors {errs} (tol {TOL[dtype]})"


# ---------------------------------------------------------------- no edges
@pytest.mark.parametrize("model", LIN)
@pytest.mark.parametrize("dtype", DT)
def test_no_edges_lin(model, dtype):
    res = lin.run(model, dtype, "auto", V=300, E=0, edges=empty(), norm="right" if model == "gcn" else "both")
    lin.check(res, dtype)


@pytest.mark.parametrize("dtype", DT)
def test_no_edges_rgcn(dtype):
    errs, _ = rgcn.run(dtype, V=300, E=0, R=3, self_loop=True, bias=True, edges=typed(empty(), 3))
    check_errs(errs, dtype)


@pytest.mark.parametrize("dtype", DT)
def test_no_edges_gat(dtype):
    errs, _ = gat.run(dtype, 2, True, V=300, E=0, edges=empty())
    check_errs(errs, dtype)


# ---------------------------------------------------------------- stars
@pytest.mark.parametrize("model", LIN)
@pytest.mark.parametrize("shape", [star_in, star_out])
@pytest.mark.parametrize("E_max", [0, 64])
def test_star_lin(model, shape, E_max):
    V, E = 400, 6000
    res = lin.run(model, torch.float32, "auto", V=V, E=E, E_max=E_max, edges=shape(V, E), seed=2)
    lin.check(res, torch.float32)


@pytest.mark.parametrize("shape", [star_in, star_out])
@pytest.mark.parametrize("policy", ["edge", "vertex"])
def test_star_rgcn(shape, policy):
    V, E = 400, 6000
    errs, _ = rgcn.run(torch.float32, policy, V=V, E=E, R=4, E_max=64, edges=typed(shape(V, E), 4), seed=2)
    check_errs(errs, torch.float32)


@pytest.mark.parametrize("shape", [star_in, star_out])
@pytest.mark.parametrize("dtype", DT)
def test_star_gat(shape, dtype):
    V, E = 400, 6000
    # star_out: every in-neighbourhood is copies of the hub, so each softmax is
    # over equal logits and the attention gradients are exactly 0
    errs, _ = gat.run(dtype, 4, True, V=V, E=E, edges=shape(V, E), seed=2, zero_attn=shape is star_out)
    check_errs(errs, dtype)


# ---------------------------------------------------------------- tiny
def test_single_vertex_self_loop():
    e = (np.zeros(3, np.int32), np.zeros(3, np.int32))   # three parallel self-loops on vertex 0
    for model in LIN:
        lin.check(lin.run(model, torch.float32, "auto", V=1, E=3, edges=e), torch.float32)
    check_errs(rgcn.run(torch.float32, V=1, E=3, R=2, self_loop=True, edges=typed(e, 2))[0], torch.float32)
    check_errs(gat.run(torch.float32, 1, True, V=1, E=3, edges=e)[0], torch.float32)


def test_fewer_edges_than_workers_and_ragged_tile():
    # V = T + 1: the last tile holds one row; 5 edges, all into that row or vertex 0
    V = 129
    e = (np.array([3, 7, 128, 0, 5], np.int32), np.array([128, 128, 128, 0, 64], np.int32))
    for model in LIN:
        for dtype in DT:
            lin.check(lin.run(model, dtype, "random", V=V, E=5, edges=e), dtype)
    check_errs(rgcn.run(torch.float32, "random", V=V, E=5, R=3, edges=typed(e, 3))[0], torch.float32)
    check_errs(gat.run(torch.float32, 4, False, V=V, E=5, edges=e)[0], torch.float32)


@pytest.mark.parametrize("policy", ["auto", "edge", "vertex"])
@pytest.mark.parametrize("dtype", DT)
def test_rgcn_many_sparse_relations(policy, dtype):
    # C3 has 100+ relation types with a Zipf mix: on a small graph most
    # relations hold a handful of edges and some none (their dW_r must be 0)
    errs, _ = rgcn.run(dtype, policy, V=800, E=4000, R=120, self_loop=True, bias=True, norm="right", seed=11)
    check_errs(errs, dtype)
