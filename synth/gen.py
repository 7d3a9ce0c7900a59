"""Seeded synthetic CTDGs, features, weights and batches (recipe: DESIGN.md §3).

Everything here is input generation: random draws with the shapes of the
paper's datasets (Table 3).  No step of the TBlock method
(sampling, dedup, time encoding, attention) is computed here.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .configs import Config

_MASK64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _splitmix64(x: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on uint64 arrays (wrap-around arithmetic)."""
    with np.errstate(over="ignore"):
        x = (x + np.uint64(0x9E3779B97F4A7C15)) & _MASK64
        x = ((x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _MASK64
        x = ((x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _MASK64
        return x ^ (x >> np.uint64(31))


def feature_rows(seed: int, rows: np.ndarray, dim: int) -> np.ndarray:
    """Feature value x(seed, row, col) for the given rows -> float32 [len(rows), dim].

    x = (int(h >> 40) - 2^23) * 2^-23, h = splitmix64(seed * 2^40 + row * dim + col):
    uniform on [-1, 1) and exact in fp32.  A pure function of (seed, row, col),
    so any row can be regenerated without the full table.
    """
    rows = np.asarray(rows, dtype=np.uint64)
    if dim == 0:
        return np.zeros((rows.shape[0], 0), np.float32)
    with np.errstate(over="ignore"):
        base = (np.uint64(seed) << np.uint64(40)) + rows[:, None] * np.uint64(dim)
        h = _splitmix64(base + np.arange(dim, dtype=np.uint64)[None, :])
    v = (h >> np.uint64(40)).astype(np.int64) - (1 << 23)
    return (v.astype(np.float32) * np.float32(2.0 ** -23))


def feature_table(seed: int, n_rows: int, dim: int, chunk: int = 1 << 18) -> np.ndarray:
    out = np.empty((n_rows, dim), np.float32)
    for r0 in range(0, n_rows, chunk):
        r1 = min(n_rows, r0 + chunk)
        out[r0:r1] = feature_rows(seed, np.arange(r0, r1), dim)
    return out


def _zipf(rng: np.random.Generator, n: int, a: float, size: int) -> np.ndarray:
    """Rank r in [0, n) with P(r) ~ (r+1)^-a (continuous inverse-CDF draw); a=0: uniform."""
    u = rng.random(size)
    if a == 0.0:
        r = np.floor(u * n)
    elif abs(a - 1.0) < 1e-12:
        r = np.floor(np.exp(u * np.log(n + 1.0))) - 1.0
    else:
        b = 1.0 - a
        r = np.floor(np.power(u * (np.power(n + 1.0, b) - 1.0) + 1.0, 1.0 / b)) - 1.0
    return np.clip(r, 0, n - 1).astype(np.int64)


@dataclass
class Graph:
    cfg: Config
    src: np.ndarray      # int32 [E]
    dst: np.ndarray      # int32 [E]
    t: np.ndarray        # float32 [E], non-decreasing (COO sorted by time)
    nfeat: np.ndarray    # float32 [N, d_v]
    efeat: np.ndarray    # float32 [E, d_e]

    @property
    def num_nodes(self) -> int:
        return self.cfg.n_nodes

    @property
    def num_edges(self) -> int:
        return int(self.src.shape[0])


def make_graph(cfg: Config, with_features: bool = True) -> Graph:
    """Seeded CTDG shaped like `cfg` (DESIGN.md §3 recipe)."""
    rng = np.random.default_rng(cfg.seeds["graph"])
    E = cfg.n_edges
    t_int = np.sort(rng.integers(0, cfg.max_t + 1, size=E, dtype=np.int64))
    t = t_int.astype(np.float32)  # RNE once; monotone so still sorted
    if cfg.bipartite:
        perm_u = rng.permutation(cfg.n_users)
        perm_i = rng.permutation(cfg.n_items)
        users = perm_u[_zipf(rng, cfg.n_users, cfg.zipf_src, E)]
        fresh = perm_i[_zipf(rng, cfg.n_items, cfg.zipf_dst, E)]
        repeat = rng.random(E) < cfg.repeat_p
        order = np.argsort(users, kind="stable")
        us = users[order]
        rep = repeat[order].copy()
        first = np.ones(E, bool)
        first[1:] = us[1:] != us[:-1]
        rep[first] = False
        idx = np.where(~rep, np.arange(E), 0)
        idx = np.maximum.accumulate(idx)
        items = np.empty(E, np.int64)
        items[order] = fresh[order][idx]
        src = users.astype(np.int32)
        dst = (items + cfg.n_users).astype(np.int32)
    else:
        n = cfg.n_items
        perm = rng.permutation(n)
        if cfg.src_uniform:
            src = rng.integers(0, n, size=E).astype(np.int32)
        else:
            src = perm[_zipf(rng, n, cfg.zipf_src, E)].astype(np.int32)
        dst = perm[_zipf(rng, n, cfg.zipf_dst, E)].astype(np.int32)
    if with_features:
        nfeat = feature_table(cfg.seeds["feat"], cfg.n_nodes, cfg.d_v)
        efeat = feature_table(cfg.seeds["feat"] + 7919, E, cfg.d_e)
    else:
        nfeat = np.zeros((0, cfg.d_v), np.float32)
        efeat = np.zeros((0, cfg.d_e), np.float32)
    return Graph(cfg, src, dst, t, nfeat, efeat)


def make_negatives(cfg: Config) -> np.ndarray:
    """One uniform negative destination per edge (items for bipartite graphs)."""
    rng = np.random.default_rng(cfg.seeds["neg"])
    if cfg.bipartite:
        return (rng.integers(0, cfg.n_items, size=cfg.n_edges) + cfg.n_users).astype(np.int32)
    return rng.integers(0, cfg.n_nodes, size=cfg.n_edges).astype(np.int32)


def batch_roots_inputs(g: Graph, neg: np.ndarray, b: int):
    """Slices (src, dst, t, neg) of batch b = edges [b*B, (b+1)*B)."""
    B = g.cfg.batch
    s = slice(b * B, min((b + 1) * B, g.num_edges))
    return g.src[s], g.dst[s], g.t[s], neg[s]


def make_time_params(cfg: Config, random_phi: bool = False, seed: int = 0):
    """omega_j = 1/10^(9 j/(d_t-1)) (TGL TimeEncode init, [ext]); phi = 0 or U(-pi, pi)."""
    omega = (np.float32(1.0) / np.power(np.float32(10.0),
             np.linspace(0, 9, cfg.d_t, dtype=np.float32))).astype(np.float32)
    if random_phi:
        phi = np.random.default_rng(seed).uniform(-np.pi, np.pi, cfg.d_t).astype(np.float32)
    else:
        phi = np.zeros(cfg.d_t, np.float32)
    return omega, phi


def make_layer_params(cfg: Config, layer: int, d_hdst: int, d_hsrc: int,
                      random_ln: bool = False, random_phi: bool = False) -> dict:
    """PyTorch-Linear-style U(+-1/sqrt(fan_in)) weights for one TBlock attention layer."""
    rng = np.random.default_rng(cfg.seeds["weights"] + 17 * layer)
    dm, dt, de = cfg.d_model, cfg.d_t, cfg.d_e

    def lin(out_f, in_f):
        bound = 1.0 / np.sqrt(in_f)
        W = rng.uniform(-bound, bound, (out_f, in_f)).astype(np.float32)
        b = rng.uniform(-bound, bound, out_f).astype(np.float32)
        return W, b

    Wq, bq = lin(dm, d_hdst + dt)
    Wk, bk = lin(dm, d_hsrc + de + dt)
    Wv, bv = lin(dm, d_hsrc + de + dt)
    Wo, bo = lin(dm, dm + d_hdst)
    if random_ln:
        gamma = rng.uniform(0.5, 1.5, dm).astype(np.float32)
        beta = rng.uniform(-0.5, 0.5, dm).astype(np.float32)
    else:
        gamma = np.ones(dm, np.float32)
        beta = np.zeros(dm, np.float32)
    omega, phi = make_time_params(cfg, random_phi, seed=cfg.seeds["weights"] + layer)
    return dict(d_hdst=d_hdst, d_hsrc=d_hsrc, d_e=de, d_t=dt, d_model=dm,
                n_heads=cfg.n_heads, d_out=dm, Wq=Wq, bq=bq, Wk=Wk, bk=bk, Wv=Wv, bv=bv,
                Wo=Wo, bo=bo, ln_gamma=gamma, ln_beta=beta, ln_eps=1e-5,
                omega=omega, phi=phi, leaky_slope=0.2, logit_scale=1.0)


def model_params(cfg: Config, **kw) -> list:
    """Per-block parameters, index = block (0 = head, L-1 = tail on raw features)."""
    out = []
    for l in range(cfg.n_layers):
        d_h = cfg.d_v if l == cfg.n_layers - 1 else cfg.d_model
        out.append(make_layer_params(cfg, l, d_h, d_h, **kw))
    return out


def make_gru_params(cfg: Config, d_mem: int = 100, random_phi: bool = True) -> dict:
    """TGN memory updater (N3): PyTorch-GRUCell-style U(+-1/sqrt(d_mem)) weights for input
    [mail (2 d_mem + d_e) ; Phi (d_t)], plus the time encoder (Listing 4's GRUMemoryUpdater)."""
    rng = np.random.default_rng(cfg.seeds["weights"] + 1000)
    d_x = 2 * d_mem + cfg.d_e + cfg.d_t
    bound = 1.0 / np.sqrt(d_mem)
    u = lambda *s: rng.uniform(-bound, bound, s).astype(np.float32)
    omega, phi = make_time_params(cfg, random_phi, seed=cfg.seeds["weights"] + 1001)
    return dict(d_mem=d_mem, W_ih=u(3 * d_mem, d_x), W_hh=u(3 * d_mem, d_mem), b_ih=u(3 * d_mem),
                b_hh=u(3 * d_mem), omega=omega, phi=phi)
