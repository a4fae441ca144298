"""Host logic of the strategy search (tune.py): the cache key
and the candidate set (no GPU)."""
import torch

import synth
from paper_conf_eurosys_huangz0wjzzzys24_b200 import tune


def test_signature_keys_graph_shape_and_layers():
    s, d, _ = synth.make_graph(2000, 20000, seed=1, alpha=0.6)
    s2, d2, _ = synth.make_graph(2000, 20000, seed=1, alpha=0.9)
    k = tune.signature(s, d, 2000, "sage", [16, 32, 8], torch.bfloat16)
    assert k == tune.signature(s, d, 2000, "sage", [16, 32, 8], torch.bfloat16)
    assert k != tune.signature(s2, d2, 2000, "sage", [16, 32, 8], torch.bfloat16)      # degree histogram
    assert k != tune.signature(s, d, 2000, "gcn", [16, 32, 8], torch.bfloat16)
    assert k != tune.signature(s, d, 2000, "sage", [16, 64, 8], torch.bfloat16)
    assert k != tune.signature(s, d, 2000, "sage", [16, 32, 8], torch.float32)


def test_default_candidates_bracket_the_q13_rule():
    import oracle
    for V, E in [(2708, 10556), (2449029, 61859140), (169343, 1166243)]:
        c = tune.default_candidates(V, E)
        base = oracle.default_emax(V, E)
        assert (128, base) in c and (128, base // 4) in c and (128, base * 4) in c
        assert {t for t, _ in c} == {64, 128, 256}
