"""Oracle checks for graphs too large for the whole-graph oracle (GDELT, MAG) --
TEST INFRASTRUCTURE ONLY.

The same definitions as oracle.c, applied to the few nodes a check needs:

* `node_segments`: a queried node's T-CSR segment read straight off the COO (one
  vectorised pass over all edges): every incident edge, both directions (R2), in
  (t, eid, forward-before-reverse) order (R3) -- the plain definition of S1 restricted
  to those owners.
* `sample_nodes`: or_sample_keyed on a CSR made of exactly those segments, keyed by the
  original node ids (R6).
* `embed_recursive`: Listing 1 for a handful of roots: samples with the
  oracle, recurses, and runs or_tblock_attn per destination; features are regenerated
  by `synth.feature_rows` (no 100 GB host copy).
"""
from __future__ import annotations

import numpy as np

from . import UNIFORM, RECENT, sample_keyed, tblock_attn

STRATEGY = {"recent": RECENT, "uniform": UNIFORM}


def node_segments(src: np.ndarray, dst: np.ndarray, t: np.ndarray, nodes,
                  num_nodes: int | None = None) -> dict:
    """{v: (nbr int32, eid int32, ts float32)} for each v in `nodes` (undirected T-CSR)."""
    nodes = np.unique(np.asarray(nodes, dtype=np.int64))
    out = {}
    if nodes.size == 0:
        return out
    if num_nodes is None:
        num_nodes = int(max(src.max(initial=0), dst.max(initial=0), nodes.max())) + 1
    mark = np.zeros(num_nodes, dtype=bool)
    mark[nodes] = True
    fwd = np.flatnonzero(mark[src])
    rev = np.flatnonzero(mark[dst])
    owner = np.concatenate([src[fwd], dst[rev]]).astype(np.int64)
    nbr = np.concatenate([dst[fwd], src[rev]]).astype(np.int32)
    eid = np.concatenate([fwd, rev]).astype(np.int64)
    dirn = np.concatenate([np.zeros(fwd.size, np.int8), np.ones(rev.size, np.int8)])
    tt = t[eid]
    order = np.lexsort((dirn, eid, tt, owner))
    owner, nbr, eid, tt = owner[order], nbr[order], eid[order], tt[order]
    bounds = np.searchsorted(owner, nodes, side="left"), np.searchsorted(owner, nodes, "right")
    for v, a, b in zip(nodes, *bounds):
        out[int(v)] = (nbr[a:b].copy(), eid[a:b].astype(np.int32), tt[a:b].copy())
    return out


def mini_tcsr(segs: dict, nodes):
    nodes = [int(v) for v in nodes]
    indptr = np.zeros(len(nodes) + 1, np.int64)
    for i, v in enumerate(nodes):
        indptr[i + 1] = indptr[i] + len(segs[v][0])
    cat = lambda j, dt: (np.concatenate([segs[v][j] for v in nodes]).astype(dt)
                         if nodes else np.zeros(0, dt))
    return indptr, cat(0, np.int32), cat(1, np.int32), cat(2, np.float32)


def sample_nodes(segs: dict, qnode, qtime, k, strategy, seed, layer):
    """Oracle S4 for queries whose nodes are all in `segs`."""
    qnode = np.asarray(qnode, np.int64)
    uniq = sorted(set(int(v) for v in qnode))
    local = {v: i for i, v in enumerate(uniq)}
    tc = mini_tcsr(segs, uniq)
    ql = np.array([local[int(v)] for v in qnode], np.int32)
    return sample_keyed(tc, ql, qnode.astype(np.int32), np.asarray(qtime, np.float32), k,
                        STRATEGY.get(strategy, strategy), seed, layer)


def embed_recursive(src, dst, t, cfg, params, roots_node, roots_t, seed: int,
                    segs: dict | None = None):
    """Root embeddings (fp64) by Listing 1's recursion over the oracle primitives.

    Features are `synth.feature_rows(feat seed, rows, dim)` (node) and
    `feature_rows(feat seed + 7919, eids, d_e)` (edge), the tables `make_graph` and
    `synth.gpu.device_feature_table` materialise."""
    import synth
    L = len(params)
    k = cfg.k
    nseed, eseed = cfg.seeds["feat"], cfg.seeds["feat"] + 7919
    segs = {} if segs is None else segs

    def ensure(nodes):
        need = [int(v) for v in np.unique(nodes) if int(v) not in segs]
        if need:
            segs.update(node_segments(src, dst, t, need, cfg.n_nodes))

    ensure(roots_node)

    def embed(v, tq, depth):
        if depth == L:
            return synth.feature_rows(nseed, np.array([v]), cfg.d_v)[0].astype(np.float64)
        ensure([v])
        sp, nb, ei, ts = sample_nodes(segs, [v], [tq], k, cfg.strategy, seed, depth)
        m = int(sp[-1])
        if depth + 1 < L:
            ensure(nb)
        hi = embed(v, tq, depth + 1).astype(np.float32)
        hs = np.stack([embed(int(nb[j]), float(ts[j]), depth + 1) for j in range(m)]
                      ).astype(np.float32) if m else np.zeros((0, hi.shape[0]), np.float32)
        p = params[depth]
        ef = (synth.feature_rows(eseed, ei.astype(np.int64), cfg.d_e) if cfg.d_e > 0
              else np.zeros((m, 0), np.float32))
        o = tblock_attn(p, np.array([0, m], np.int64), np.array([tq], np.float32),
                        hi[None, :], None, hs if m else np.zeros((1, hi.shape[0]), np.float32),
                        np.arange(m, dtype=np.int32), ef if m else np.zeros((1, max(cfg.d_e, 0)), np.float32),
                        np.arange(m, dtype=np.int32), ts.astype(np.float32))[0]
        return o

    return np.stack([embed(int(v), float(tq), 0) for v, tq in zip(roots_node, roots_t)])
