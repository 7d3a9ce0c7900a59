"""The big-graph oracle helpers (oracle/big.py) against the whole-graph oracle (CPU).

oracle/big.py is what the GDELT/MAG GPU tests compare with, so it is pinned here to
the already-pinned whole-graph functions on graphs the C oracle builds in full: the
per-node segments equal or_build_tcsr's, keyed mini-CSR sampling equals or_sample on
the whole T-CSR, and the recursion equals or_embed_recursive bit for bit.
"""
import numpy as np
import pytest

import oracle
from oracle import big
import synth


def _general(n_edges=30000, n_nodes=700, name="GDELT"):
    cfg = synth.get_config(name).scaled(n_edges, 0, n_nodes, batch=200)
    g = synth.make_graph(cfg)
    return cfg, g


@pytest.mark.parametrize("name", ["GDELT", "MAG", "REDDIT"])
def test_node_segments_equal_tcsr(name):
    if name == "REDDIT":
        cfg = synth.get_config(name).scaled(20000, 300, 80, batch=200)
        g = synth.make_graph(cfg)
    else:
        cfg, g = _general(name=name)
    indptr, nbr, eid, ts = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    rng = np.random.default_rng(1)
    deg = np.diff(indptr)
    nodes = np.concatenate([rng.choice(cfg.n_nodes, 40, replace=False),
                            [int(np.argmax(deg)), int(np.argmin(deg))]])
    segs = big.node_segments(g.src, g.dst, g.t, nodes, cfg.n_nodes)
    for v in nodes:
        a, b = indptr[v], indptr[v + 1]
        got = segs[int(v)]
        assert np.array_equal(got[0], nbr[a:b])
        assert np.array_equal(got[1], eid[a:b])
        assert np.array_equal(got[2], ts[a:b])


@pytest.mark.parametrize("strategy", ["recent", "uniform"])
def test_mini_csr_sampling_equals_whole_graph(strategy):
    cfg, g = _general()
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    rng = np.random.default_rng(2)
    q = rng.integers(0, cfg.n_nodes, 300).astype(np.int32)
    q[:50] = q[0]                                     # repeated nodes, different times
    qt = rng.integers(0, cfg.max_t + 2, 300).astype(np.float32)
    segs = big.node_segments(g.src, g.dst, g.t, q, cfg.n_nodes)
    for layer in (0, 1):
        exp = oracle.sample(tc, q, qt, 10, big.STRATEGY[strategy], 77, layer)
        got = big.sample_nodes(segs, q, qt, 10, strategy, 77, layer)
        for a, b in zip(got, exp):
            assert np.array_equal(a, b)


@pytest.mark.parametrize("name", ["GDELT", "MAG"])
def test_big_recursion_equals_whole_graph_oracle(name):
    cfg, g = _general(n_edges=12000, n_nodes=400, name=name)
    params = synth.gen.model_params(cfg)
    neg = synth.make_negatives(cfg)
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    from oracle import pipeline as opipe
    qn, qt = opipe.roots(*synth.batch_roots_inputs(g, neg, 40))
    pick = np.random.default_rng(3).choice(len(qn), 12, replace=False)
    exp = oracle.embed_recursive(tc, g.nfeat, g.efeat, params, cfg.k,
                                 big.STRATEGY[cfg.strategy], cfg.seeds["sampler"],
                                 qn[pick], qt[pick])
    got = big.embed_recursive(g.src, g.dst, g.t, cfg, params, qn[pick], qt[pick],
                              cfg.seeds["sampler"])
    np.testing.assert_array_equal(got, exp)
