"""On-device synthetic inputs for the large configs (GDELT, MAG): same recipe as gen.py.

* Features: the counter hash of `feature_rows` evaluated with torch int64 ops (two's
  complement wrap-around == uint64 arithmetic), so any row equals
  `gen.feature_rows(seed, rows, dim)` bit for bit -- the oracle side regenerates rows
  on the host instead of copying 142 GB back.
* Graphs: drawn with a seeded torch CUDA generator (timestamps, Zipf ranks, node
  permutation); the host copy for the oracle checks is a plain `.cpu()` of these inputs.
No method arithmetic here (input generation only).
"""
from __future__ import annotations

import torch

from .configs import Config

_C1 = 0x9E3779B97F4A7C15 - (1 << 64)   # as signed int64
_C2 = 0xBF58476D1CE4E5B9 - (1 << 64)
_C3 = 0x94D049BB133111EB - (1 << 64)


def _lsr(x: torch.Tensor, k: int) -> torch.Tensor:
    return (x >> k) & ((1 << (64 - k)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    x = x + _C1
    x = (x ^ _lsr(x, 30)) * _C2
    x = (x ^ _lsr(x, 27)) * _C3
    return x ^ _lsr(x, 31)


def feature_rows_torch(seed: int, rows: torch.Tensor, dim: int) -> torch.Tensor:
    """== gen.feature_rows(seed, rows, dim) (float32 [len(rows), dim])."""
    rows = rows.to(torch.int64)
    cols = torch.arange(dim, dtype=torch.int64, device=rows.device)
    h = splitmix64((seed << 40) + rows[:, None] * dim + cols[None, :])
    v = _lsr(h, 40) - (1 << 23)
    return v.to(torch.float32) * (2.0 ** -23)


def device_feature_table(seed: int, n_rows: int, dim: int, device, chunk_elems: int = 1 << 27,
                         pitch_mult: int = 1):
    """[n_rows, dim] feature table on `device`; with pitch_mult > 1 the rows are stored with
    a pitch rounded up to a multiple of pitch_mult floats (e.g. 4: 16-byte row pitch, the
    layout the cp.async gathers of the K|V kernel take) and a [:, :dim] view is returned.
    The padding columns are zero and never read."""
    pitch = max(pitch_mult, (dim + pitch_mult - 1) // pitch_mult * pitch_mult) if dim else 0
    out = torch.empty((n_rows, pitch), dtype=torch.float32, device=device)
    if pitch > dim:
        out[:, dim:] = 0
    if dim == 0 or n_rows == 0:
        return out[:, :dim]
    rows_per = max(1, chunk_elems // dim)
    for r0 in range(0, n_rows, rows_per):
        r1 = min(n_rows, r0 + rows_per)
        out[r0:r1, :dim] = feature_rows_torch(seed, torch.arange(r0, r1, device=device), dim)
    return out[:, :dim]


def _zipf_rank(u: torch.Tensor, n: int, a: float) -> torch.Tensor:
    if a == 0.0:
        r = torch.floor(u * n)
    elif abs(a - 1.0) < 1e-12:
        r = torch.floor(torch.exp(u * torch.log(torch.tensor(n + 1.0, dtype=u.dtype)))) - 1.0
    else:
        b = 1.0 - a
        r = torch.floor(torch.pow(u * ((n + 1.0) ** b - 1.0) + 1.0, 1.0 / b)) - 1.0
    return torch.clamp(r, 0, n - 1).to(torch.int64)


def device_graph(cfg: Config, device):
    """(src int32, dst int32, t float32 sorted) for a general (non-bipartite) config."""
    assert not cfg.bipartite, "device_graph is for the large general configs"
    g = torch.Generator(device=device)
    g.manual_seed(cfg.seeds["graph"])
    E, n = cfg.n_edges, cfg.n_items
    t = torch.randint(0, cfg.max_t + 1, (E,), generator=g, device=device, dtype=torch.int64)
    t = torch.sort(t).values.to(torch.float32)
    perm = torch.randperm(n, generator=g, device=device)
    if cfg.src_uniform:
        src = torch.randint(0, n, (E,), generator=g, device=device, dtype=torch.int64)
    else:
        src = perm[_zipf_rank(torch.rand(E, generator=g, device=device, dtype=torch.float64),
                              n, cfg.zipf_src)]
    src = src.to(torch.int32)
    dst = perm[_zipf_rank(torch.rand(E, generator=g, device=device, dtype=torch.float64),
                          n, cfg.zipf_dst)].to(torch.int32)
    return src, dst, t


def device_negatives(cfg: Config, device):
    g = torch.Generator(device=device)
    g.manual_seed(cfg.seeds["neg"])
    return torch.randint(0, cfg.n_nodes, (cfg.n_edges,), generator=g, device=device,
                         dtype=torch.int64).to(torch.int32)
