"""Workload table (BASELINE.json `configs`).

Shapes follow PAPER.md Table 3: |V|, |E|, d_v, d_e, max(t).
Batch sizes: 600, GDELT 4000, LastFM 2000 and MAG 60000
(BASELINE.json configs[2], configs[4]).  Model dims are the TGL defaults the
paper inherits: d_t = d_model = 100, 2 heads.
"""
from dataclasses import dataclass, field, replace


@dataclass(frozen=True)
class Config:
    name: str
    n_users: int          # bipartite: first n_users ids are users; general: 0
    n_items: int          # bipartite: next n_items ids are items; general: all nodes
    n_edges: int
    max_t: int            # timestamps are integers U[0, max_t]
    d_v: int              # node feature dim
    d_e: int              # edge feature dim
    batch: int            # edges per batch; roots = 3 * batch (src, dst, neg)
    n_layers: int         # TBlocks per batch (TGAT 2 layers)
    k: int                # neighbours per query
    strategy: str         # 'recent' | 'uniform'
    dedup: bool
    precompute: bool
    zipf_src: float
    zipf_dst: float
    repeat_p: float       # prob. a user repeats its previous item (bipartite)
    bipartite: bool
    src_uniform: bool = False
    d_t: int = 100
    d_model: int = 100
    n_heads: int = 2
    window: int = 65536   # time-precompute table size (integer dt in [0, W))
    seeds: dict = field(default_factory=dict)

    @property
    def n_nodes(self) -> int:
        return self.n_users + self.n_items

    @property
    def n_roots(self) -> int:
        return 3 * self.batch

    @property
    def n_batches(self) -> int:
        return self.n_edges // self.batch

    def scaled(self, n_edges: int, n_users: int | None = None,
               n_items: int | None = None, batch: int | None = None) -> "Config":
        """Same recipe at a smaller size (oracle-sized parity cases)."""
        return replace(self, n_edges=n_edges,
                       n_users=self.n_users if n_users is None else n_users,
                       n_items=self.n_items if n_items is None else n_items,
                       batch=self.batch if batch is None else batch)


def _seeds(i: int) -> dict:
    return {"graph": 1000 + i, "neg": 2000 + i, "feat": 3000 + i,
            "weights": 4000, "sampler": 0x74676C00}


CONFIGS = {
    # configs[0]: WIKI-shaped, 1-layer, recent 10, fp32
    "WIKI": Config("WIKI", 8227, 1000, 157_474, 2_700_000, 172, 172, 600, 1, 10,
                   "recent", False, False, 0.8, 1.0, 0.5, True, seeds=_seeds(0)),
    # configs[1]: REDDIT-shaped, 2-layer, uniform 10, dedup + time-precompute on
    # precompute window 2^22 covers every integer dt <= max(t) = 2.7e6 (reading R11)
    "REDDIT": Config("REDDIT", 10_000, 984, 672_447, 2_700_000, 172, 172, 600, 2, 10,
                     "uniform", True, True, 0.8, 1.0, 0.5, True, window=1 << 22,
                     seeds=_seeds(1)),
    # configs[2]: LastFM-shaped, heavy skew, 2-layer, recent 20, batch 2000
    "LASTFM": Config("LASTFM", 980, 1000, 1_293_103, 140_000_000, 128, 128, 2000, 2, 20,
                     "recent", False, False, 1.0, 1.3, 0.5, True, seeds=_seeds(2)),
    # configs[3]: GDELT-shaped, general graph, 2-layer uniform 10, batch 4000
    "GDELT": Config("GDELT", 0, 16_682, 191_290_882, 180_000, 413, 186, 4000, 2, 10,
                    "uniform", False, False, 1.1, 1.1, 0.0, False, seeds=_seeds(3)),
    # configs[4]: MAG-shaped, 1-layer recent 10, batch 60000 (d_v 128, d_e 0: SURVEY §8(d))
    "MAG": Config("MAG", 0, 121_751_665, 1_297_748_926, 120, 128, 0, 60_000, 1, 10,
                  "recent", False, False, 0.0, 1.0, 0.0, False, src_uniform=True,
                  seeds=_seeds(4)),
}


def get_config(name: str) -> Config:
    return CONFIGS[name.upper()]
