"""Oracle of the cache() operator (memoisation) -- TEST INFRASTRUCTURE ONLY.

P:149: "memoization exploits the observation that previously computed embeddings
could be reused and cached, thus avoids running computations altogether".
P:297: "cache() will filter destination node-time pairs to ones that have not been
cached and register a hook to combine computed outputs with cached results".
TGOpt's cache_lookup / cache_store (Listing 1 lines 10-23) key the
store by layer, so one `Memo` per layer.

The plain definition: an unbounded dictionary from the pair (node, t) -- compared
as values, so -0.0 == +0.0 (reading R8) and a NaN time equals nothing (R22) -- to
the embedding row stored for it.  Pure Python, no blocking, no hashing of our own.
"""
from __future__ import annotations

import math

import numpy as np


class Memo:
    def __init__(self):
        self.rows = {}

    @staticmethod
    def _key(v, t):
        # float(-0.0) == 0.0 and hash(-0.0) == hash(0.0): the dict already equates them
        return (int(v), float(t))

    def lookup(self, node, t):
        """P:297 filter: returns (hit[n] bool, miss_index[m] in input order)."""
        hit = np.zeros(len(node), dtype=bool)
        for i, (v, ti) in enumerate(zip(node, t)):
            hit[i] = (not math.isnan(float(ti))) and self._key(v, ti) in self.rows
        return hit, np.flatnonzero(~hit)

    def store(self, node, t, emb):
        """Listing 1 cache_store: remember emb[i] for (node[i], t[i])."""
        for v, ti, row in zip(node, t, emb):
            if not math.isnan(float(ti)):
                self.rows[self._key(v, ti)] = np.array(row)

    def combine(self, node, t, hit, computed):
        """P:297 hook: out[i] = cached row if hit[i] else the next computed row."""
        out = np.zeros((len(node), computed.shape[1]), computed.dtype)
        j = 0
        for i, (v, ti) in enumerate(zip(node, t)):
            if hit[i]:
                out[i] = self.rows[self._key(v, ti)]
            else:
                out[i] = computed[j]
                j += 1
        return out


def cached_embed(memo: Memo, node, t, compute):
    """Memoised evaluation of compute(node_subset, t_subset) -> rows (P:297 flow:
    filter, compute the misses, store them, combine)."""
    hit, miss = memo.lookup(node, t)
    computed = compute(node[miss], t[miss])
    memo.store(node[miss], t[miss], computed)
    return memo.combine(node, t, hit, computed)
