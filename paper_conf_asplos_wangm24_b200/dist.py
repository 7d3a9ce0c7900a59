"""Multi-GPU plumbing (S16) -- one process per GPU, torch.distributed over NCCL.

The TBlock path shards by batch: every rank holds the full T-CSR, features and
weights in its HBM (replicated), processes its own batch of the
edge stream, and the root embeddings of all ranks are all-gathered so every rank
sees the whole step's embeddings (the only collective; NVLink via NCCL).  The
per-rank work is fixed as ranks are added (weak scaling).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def rank_batch(step: int, rank: int, world: int, first: int, n_avail: int) -> int:
    """Batch index processed by `rank` at `step`: consecutive batches of the stream are
    dealt round-robin to the ranks, wrapping inside the `n_avail` batches from `first`."""
    return first + ((step * world + rank) % n_avail)


def allgather_embeddings(local: torch.Tensor, out: torch.Tensor | None = None, group=None):
    """[n, d] per rank -> [world * n, d] in rank order (NCCL all_gather_into_tensor)."""
    world = dist.get_world_size(group)
    if out is None:
        out = torch.empty(world * local.shape[0], *local.shape[1:], dtype=local.dtype,
                          device=local.device)
    dist.all_gather_into_tensor(out, local.contiguous(), group=group)
    return out
