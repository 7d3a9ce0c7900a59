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
