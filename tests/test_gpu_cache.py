"""GPU parity of the cache() operator (include/tgl.h
tgl_cache_*) against the dictionary oracle (oracle/cache.py): hit masks, compacted
miss lists and combined rows bit-exact; a small table that overflows stays correct
(every served row is the one its pair was stored with, R22)."""
import numpy as np
import pytest
import torch

from oracle.cache import Memo

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def T():
    from paper_conf_asplos_wangm24_b200 import tgl
    return tgl


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def rows_of(node, t, d):
    c = np.arange(d, dtype=np.float32)
    return (node[:, None].astype(np.float32) * np.float32(1e-3) + t[:, None] * np.float32(1e-6)
            + c[None, :]).astype(np.float32)


def bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


@pytest.mark.parametrize("d", [100, 37])
def test_cache_rounds_bit_exact(T, d):
    rng = np.random.default_rng(d)
    cache = T.EmbeddingCache(1 << 16, d)
    memo = Memo()
    for n in (1, 1000, 5001, 777, 20000):
        node = rng.integers(0, 400, n).astype(np.int32)
        t = rng.integers(0, 30, n).astype(np.float32)
        if n > 20:
            t[::13] = -0.0
            t[::29] = np.nan
        slot, mn, mt, nm = T.cache_lookup(cache, cu(node), cu(t))
        hit, miss = memo.lookup(node, t)
        s = slot.cpu().numpy()[:n]
        m = int(nm.item())
        assert np.array_equal(s >= 0, hit)
        assert m == len(miss)
        assert np.array_equal(s[miss], -1 - np.arange(m))
        assert np.array_equal(mn.cpu().numpy()[:m], node[miss])
        assert np.array_equal(bits(mt.cpu().numpy()[:m]), bits(t[miss]))
        comp = rows_of(node[miss], t[miss], d)
        comp_dev = cu(comp) if m else torch.zeros(1, d, device="cuda")
        T.cache_store(cache, mn, mt, comp_dev, n_dev=nm, n_max=n)
        memo.store(node[miss], t[miss], comp)
        out = T.cache_combine(cache, slot, comp_dev, n_max=n).cpu().numpy()[:n]
        exp = memo.combine(node, t, hit, comp)
        assert np.array_equal(bits(out), bits(exp))


def test_cache_overflow_serves_only_true_rows(T):
    rng = np.random.default_rng(1)
    d = 100
    cache = T.EmbeddingCache(64, d)
    node = rng.permutation(100000)[:3000].astype(np.int32)
    t = rng.integers(0, 10**6, 3000).astype(np.float32)
    truth = rows_of(node, t, d)
    total_hits = 0
    for _ in range(3):
        slot, mn, mt, nm = T.cache_lookup(cache, cu(node), cu(t))
        s = slot.cpu().numpy()
        m = int(nm.item())
        miss = np.flatnonzero(s < 0)
        assert m == len(miss) and np.array_equal(mn.cpu().numpy()[:m], node[miss])
        total_hits += int((s >= 0).sum())
        comp = cu(truth[miss])
        T.cache_store(cache, mn, mt, comp, n_dev=nm, n_max=len(node))
        out = T.cache_combine(cache, slot, comp).cpu().numpy()
        assert np.array_equal(out, truth)
    assert 0 < total_hits <= 2 * 64


def test_cache_device_count(T):
    rng = np.random.default_rng(2)
    cache = T.EmbeddingCache(1 << 12, 100)
    node = rng.integers(0, 50, 3000).astype(np.int32)
    t = rng.integers(0, 5, 3000).astype(np.float32)
    memo = Memo()
    for n in (0, 1234, 3000):
        ndev = torch.tensor([n], dtype=torch.int64, device="cuda")
        slot, mn, mt, nm = T.cache_lookup(cache, cu(node), cu(t), n_dev=ndev)
        hit, miss = memo.lookup(node[:n], t[:n])
        assert int(nm.item()) == len(miss)
        assert np.array_equal(slot.cpu().numpy()[:n] >= 0, hit)
        comp = rows_of(node[:n][miss], t[:n][miss], 100)
        comp_dev = cu(comp) if len(miss) else torch.zeros(1, 100, device="cuda")
        T.cache_store(cache, mn, mt, comp_dev, n_dev=nm, n_max=3000)
        memo.store(node[:n][miss], t[:n][miss], comp)


def test_pipeline_root_cache_vs_oracle(T):
    """TGATPipeline(cache_capacity>0), one table per layer: memoised embeddings over
    repeated and consecutive batches match the oracle (no cache) within the fp32
    tolerance; a repeated batch computes nothing at the head block; inner-layer pairs
    hit across consecutive batches; graph replay == eager."""
    from oracle import pipeline as opipe
    import oracle
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler
    from tests.test_gpu_parity import _world
    cfg, g, neg, params = _world("REDDIT", n_edges=60000)
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    tc = T.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = TGATPipeline(dev, tc, params, cfg.batch,
                        TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), True,
                        cfg.precompute, cfg.window, "fp32", cache_capacity=1 << 16)
    otc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    n0 = 3 * cfg.batch
    seen, inner_hits = {}, 0
    for b in (70, 70, 71, 70, 72):
        pipe.start_dev.fill_(b * cfg.batch)
        emb = pipe.forward().cpu().numpy()[:n0].copy()
        misses = int(pipe.blocks[0].u_dev.item())
        b1 = pipe.blocks[1]
        inner_hits += int(b1.ws["cache"]["u"].item()) - int(b1.u_dev.item())
        if b in seen:
            assert misses == 0
            assert np.array_equal(emb, seen[b])
        exp, _ = opipe.run_batch(otc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy, True,
                                 cfg.seeds["sampler"], *synth_roots(g, neg, b))
        assert np.abs(emb - exp).max() <= 1e-3
        seen[b] = emb
    assert inner_hits > 0                # layer-1 pairs recur across consecutive batches
    pipe.capture()                       # replays hit the now-warm cache
    e_g = pipe.run_graph(72 * cfg.batch).cpu().numpy()[:n0]
    assert np.array_equal(e_g, seen[72])


def synth_roots(g, neg, b):
    import synth
    return synth.batch_roots_inputs(g, neg, b)


@pytest.mark.parametrize("d", [100, 37])   # float4 copies / scalar copies
def test_cache_merge_equals_store_then_combine(T, d):
    """tgl_cache_merge (the launch the chain uses) == tgl_cache_store + tgl_cache_combine,
    read through an index (the S14 inverse) with repeated entries."""
    rng = np.random.default_rng(7)
    cache = T.EmbeddingCache(1 << 14, d)
    memo = Memo()
    for n in (3000, 2500, 4000):
        node = np.unique(rng.integers(0, 600, n)).astype(np.int32)   # dedup space: unique pairs
        t = np.full(len(node), 5.0, np.float32)
        slot, mn, mt, nm = T.cache_lookup(cache, cu(node), cu(t))
        hit, miss = memo.lookup(node, t)
        assert np.array_equal(slot.cpu().numpy()[:len(node)] >= 0, hit)
        comp = rows_of(node[miss], t[miss], d)
        comp_dev = cu(comp) if len(miss) else torch.zeros(1, d, device="cuda")
        # surjective like the dedup inverse: every pair is read (and so stored) at least once
        idx = np.concatenate([rng.permutation(len(node)),
                              rng.integers(0, len(node), len(node))]).astype(np.int32)
        out = T.cache_merge(cache, cu(node), cu(t), slot, comp_dev, idx=cu(idx)).cpu().numpy()
        memo.store(node[miss], t[miss], comp)
        exp = memo.combine(node, t, hit, comp)[idx]
        assert np.array_equal(bits(out[:len(idx)]), bits(exp))
    # every pair merged so far is now a hit
    slot, _, _, nm = T.cache_lookup(cache, cu(node), cu(t))
    assert int(nm.item()) == 0


def test_pipeline_cache_full_reddit_vs_oracle(T):
    """Full-size REDDIT in the bench's launch configuration (graph replay, consecutive
    batches from 70 % of the stream, a warm per-layer cache) against the uncached
    oracle: max abs <= 1e-3 on every root."""
    from oracle import pipeline as opipe
    import oracle
    import synth
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler
    from tests.test_gpu_parity import _world
    cfg, g, neg, params = _world("REDDIT")
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    tc = T.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = TGATPipeline(dev, tc, params, cfg.batch,
                        TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), True,
                        cfg.precompute, cfg.window, "fp32", cache_capacity=1 << 20)
    pipe.capture()
    otc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    b0 = int(0.7 * cfg.n_batches)
    n0 = 3 * cfg.batch
    for b in range(b0, b0 + 6):
        emb = pipe.run_graph(b * cfg.batch).cpu().numpy()[:n0]
        if b < b0 + 4:
            continue                       # warm the cache like the bench's warm-up
        exp, _ = opipe.run_batch(otc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy, True,
                                 cfg.seeds["sampler"], *synth.batch_roots_inputs(g, neg, b))
        assert np.abs(emb - exp).max() <= 1e-3
