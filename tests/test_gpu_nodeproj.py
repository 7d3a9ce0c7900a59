"""GPU parity of the node-projection path (tgl_node_proj + TGL_NODE_PROJ).

Eqs 4, 5 and 7 are linear in h before the logits, so the tail block (whose h_src and
h_dst are node-feature rows) may take the h terms per node:
  q_i = Wq [h_i ; Phi(0)] + bq,  k_e = Wk[:, :d] h_src + Wk[:, d:] [e ; Phi] + bk, ...
The table Z is checked against those definitions in fp64, and whole pipelines with the
path on against the oracle (north_star tolerances) and against the path off.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle import pipeline as opipe
import synth

from tests.test_gpu_parity import TOL, _gpu_pipeline, _world, cu, cu_pad, np_

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def T():
    from paper_conf_asplos_wangm24_b200 import tgl
    return tgl


@pytest.mark.parametrize("name,n_nodes,precision", [("REDDIT", 1000, "fp32"),
                                                    ("GDELT", 777, "fp32"),
                                                    ("GDELT", 300, "bf16"),
                                                    ("LASTFM", 129, "fp32")])
def test_node_proj_table_vs_definition(T, name, n_nodes, precision):
    cfg = synth.get_config(name)
    p = synth.gen.model_params(cfg)[-1]            # the tail block's layer
    rng = np.random.default_rng(n_nodes)
    X = rng.uniform(-1, 1, (n_nodes, cfg.d_v)).astype(np.float32)
    a = T.AttnParams(p, precision=precision, pack=True)
    xs = T.split_rows(cu_pad(X))
    Z = np_(T.node_proj(a, xs))
    d, dm = cfg.d_v, p["d_model"]
    x = X.astype(np.float64)
    W = {k: np.asarray(p[k], np.float64) for k in ("Wq", "Wk", "Wv", "Wo", "bq", "bk", "phi")}
    zk = x @ W["Wk"][:, :d].T
    zv = x @ W["Wv"][:, :d].T
    phi0 = np.cos(np.asarray(p["phi"], np.float32)).astype(np.float64)   # Phi(0), R10
    zq = x @ W["Wq"][:, :d].T + W["Wq"][:, d:] @ phi0 + W["bq"]
    zo = x @ W["Wo"][:, dm:].T
    dh = dm // 2
    qb = np.stack([zq[:, :dh] @ W["bk"][:dh], zq[:, dh:] @ W["bk"][dh:]], 1)
    tol = 2e-5 if precision == "fp32" else 3e-2
    for got, exp in ((Z[:, 0:100], zk), (Z[:, 100:200], zv), (Z[:, 256:356], zq),
                     (Z[:, 356:358], qb), (Z[:, 384:484], zo)):
        assert np.abs(got - exp).max() <= tol * max(1.0, np.abs(exp).max())


@pytest.mark.parametrize("name,precision,n_edges", [("WIKI", "fp32", None),
                                                    ("REDDIT", "fp32", None),
                                                    ("REDDIT", "bf16", None),
                                                    ("LASTFM", "fp32", None),
                                                    ("GDELT", "fp32", 200000),
                                                    ("GDELT", "bf16", 200000)])
def test_pipeline_node_proj_vs_oracle(T, name, precision, n_edges):
    """Whole batches (first, middle, last) in the captured launch sequence: node
    projections on vs the oracle (1e-3 fp32 / 5e-2 bf16) and vs the path off."""
    cfg, g, neg, params = _world(name, n_edges=n_edges)
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu_pad(g.nfeat), "efeat": cu_pad(g.efeat)}
    on = _gpu_pipeline(T, cfg, g, neg, params, precision, dev=dev, node_proj=True)
    off = _gpu_pipeline(T, cfg, g, neg, params, precision, dev=dev, node_proj=False)
    assert on.node_proj and not off.node_proj
    on.capture()
    off.capture()
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    nb = cfg.n_batches
    n0 = 3 * cfg.batch
    for b in (0, nb // 2, nb - 1):
        e_on = np_(on.run_graph(b * cfg.batch))[:n0].copy()
        e_off = np_(off.run_graph(b * cfg.batch))[:n0].copy()
        torch.cuda.synchronize()
        exp, _ = opipe.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy, cfg.dedup,
                                 cfg.seeds["sampler"], *synth.batch_roots_inputs(g, neg, b))
        assert np.abs(e_on - exp).max() <= TOL[precision], (b, np.abs(e_on - exp).max())
        lim = 2e-4 if precision == "fp32" else 5e-2
        assert np.abs(e_on - e_off).max() <= lim, (b, np.abs(e_on - e_off).max())
