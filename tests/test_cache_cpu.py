"""cache() memoisation: oracle pins and host-side ABI
checks, no GPU.

Pins (independent of the memo's own code): brute-force hit masks from a list scan
with value equality; -0 == +0 and NaN never hits (R8, R22); semantics preservation
-- memoised root embeddings over overlapping batches equal the recursive Listing-1
embeddings of every root, bitwise ("without changing model semantics").
"""
import ctypes as C

import numpy as np
import pytest

import oracle
from oracle import pipeline
from oracle.cache import Memo, cached_embed
import synth
from paper_conf_asplos_wangm24_b200 import tgl


def brute_hits(seen, node, t):
    return np.array([any(v == sv and float(ti) == float(st) for sv, st in seen)
                     for v, ti in zip(node, t)], dtype=bool)


def test_memo_hits_equal_list_scan():
    rng = np.random.default_rng(5)
    memo, seen = Memo(), []
    for _ in range(5):
        node = rng.integers(0, 15, 40).astype(np.int32)
        t = rng.integers(0, 6, 40).astype(np.float32)
        t[::9] = -0.0
        hit, miss = memo.lookup(node, t)
        assert np.array_equal(hit, brute_hits(seen, node, t))
        assert np.array_equal(miss, np.flatnonzero(~hit))
        rows = np.stack([np.full(3, v * 100.0 + ti, np.float32) for v, ti in zip(node, t)])
        memo.store(node[miss], t[miss], rows[miss])
        seen += [(int(v), float(ti)) for v, ti in zip(node[miss], t[miss])]
        out = memo.combine(node, t, hit, rows[miss])
        assert np.array_equal(out, rows)   # every row is the one its pair was stored with


def test_memo_signed_zero_and_nan():
    memo = Memo()
    memo.store(np.array([3, 4], np.int32), np.array([0.0, np.nan], np.float32),
               np.ones((2, 2), np.float32))
    hit, _ = memo.lookup(np.array([3, 4, 3], np.int32), np.array([-0.0, np.nan, 1.0], np.float32))
    assert hit.tolist() == [True, False, False]


def test_memoised_roots_equal_recursive_embeddings():
    """cache() preserves semantics -- bitwise in the oracle."""
    from dataclasses import replace
    cfg = replace(synth.get_config("REDDIT").scaled(2000, 120, 30, batch=30),
                  strategy="uniform", n_layers=2, k=4, d_v=16, d_e=8)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    tcsr = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    params = synth.gen.model_params(cfg, random_ln=True, random_phi=True)

    def embed(qn, qt):
        if len(qn) == 0:
            return np.zeros((0, 100))
        return oracle.embed_recursive(tcsr, g.nfeat, g.efeat, params, cfg.k,
                                      pipeline.STRATEGY["uniform"], 11, qn, qt)

    memo, hits = Memo(), 0
    for start in (600, 600, 610, 1500):             # repeated and overlapping batches
        sb, db, tb, nb = (a[start:start + 30] for a in (g.src, g.dst, g.t, neg))
        qn, qt = pipeline.roots(sb, db, tb, nb)
        h, _ = memo.lookup(qn, qt)
        hits += int(h.sum())
        got = cached_embed(memo, qn, qt, embed)
        assert np.array_equal(got, embed(qn, qt))
    assert hits >= 90                                # the repeated batch hit everywhere


def test_cache_abi_validation():
    lib = tgl.lib()
    nb = C.c_size_t(0)
    assert lib.tgl_cache_lookup(None, 5000, None, None, None, None, None, None, None, None,
                                C.byref(nb), None) == 0 and nb.value >= 8 * 10
    bad = tgl.CacheC(3, 100, 256, 256)                # not a power of two
    assert lib.tgl_cache_store(C.byref(bad), 10, None, None, None, None, 100, None) == -1
    assert b"power of two" in lib.tgl_last_error()
    ok = tgl.CacheC(1024, 100, 256, 256)
    assert lib.tgl_cache_combine(C.byref(ok), 10, None, None, None, 50, None, 100, None) == -1
    assert lib.tgl_cache_store(None, 10, None, None, None, None, 100, None) == -1
    assert lib.tgl_cache_merge(C.byref(bad), 10, None, None, None, None, None, None, 100, None,
                               100, None) == -1
    assert lib.tgl_cache_merge(C.byref(ok), 10, None, None, None, None, None, None, 100, None,
                               100, None) == -1          # null arrays
