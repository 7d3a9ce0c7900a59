"""Multi-GPU root sharding (S16) -- one process per GPU.

Every rank holds the whole T-CSR, feature tables and weights in its own HBM
(replicated; GDELT ~147 GB fits the 180 GB of a B200).  Per batch every rank forms
the roots (and dedups them, when the config does) redundantly, computes S4-S15 for
its contiguous slice of the unique roots (`TGATPipeline(shard=(rank, world))`), and
the slices are all-gathered -- the one collective of the path -- so that every rank
ends the step with the batch's root embeddings (`tgl_shard_gather` applies the
roots' dedup inverse).  Total work per batch is fixed as ranks are added (strong
scaling).

The paper trains and serves on one GPU; TGL's multi-GPU support is
the contrast it names.  The embedding of a root depends only on <node, t> (content-
keyed sampling, R6; fixed-order reductions), so the sharded result equals the
single-GPU one.

`ShardedRunner` overlaps batch b's all-gather (and the inverse gather) on a comm
stream with batch b+1's compute: the pipeline captures one CUDA graph per slot, each
with its own roots / send buffers, and slot s is replayed again only after its
previous all-gather has finished.  NCCL gathers device tensors in place; the gloo
backend (CPU tests) goes through host copies.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_bounds(U: int, rank: int, world: int) -> tuple[int, int]:
    """[lo, hi) of rank's slice of U unique roots (the tgl_shard_slice rule)."""
    c = -(-U // world) if U else 0
    lo = min(rank * c, U)
    return lo, min(lo + c, U)


def allgather_rows(local: torch.Tensor, out: torch.Tensor, group=None):
    """[c, d] per rank -> out [world * c, d] in rank order."""
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(out, local.contiguous(), group=group)
        return out
    world = dist.get_world_size(group)        # gloo: host round trip
    host = torch.empty((world * local.shape[0],) + tuple(local.shape[1:]), dtype=local.dtype)
    dist.all_gather_into_tensor(host, local.detach().cpu().contiguous(), group=group)
    out.copy_(host)
    return out


class ShardedRunner:
    """Drives a sharded TGATPipeline: step(start) replays the slot's graph on the
    compute stream, then all-gathers the slice and rebuilds the batch's root
    embeddings on a comm stream.  Returns the embeddings tensor of that batch (valid
    once `wait(slot)` or `drain()` returned on the compute stream)."""

    def __init__(self, pipe, group=None):
        assert pipe.shard is not None and pipe.graphs, "capture() a sharded pipeline first"
        self.p = pipe
        self.group = group
        self.world = pipe.world
        d = pipe.send[0].shape[1]
        dev = pipe.dev
        self.gathered = [torch.empty(self.world * pipe.c_max, d, device=dev) for _ in range(2)]
        self.emb = [torch.empty(3 * pipe.batch, d, device=dev) for _ in range(2)]
        self.comm = torch.cuda.Stream(device=dev)
        self.done = [None, None]
        self.i = 0

    def step(self, start: int):
        p, slot = self.p, self.i % 2
        self.i += 1
        cs = torch.cuda.current_stream()
        if self.done[slot] is not None:          # slot's previous all-gather finished
            cs.wait_event(self.done[slot])
        p.start_dev.fill_(start)
        p.graphs[slot].replay()
        ready = torch.cuda.Event()
        ready.record(cs)
        with torch.cuda.stream(self.comm):
            self.comm.wait_event(ready)
            allgather_rows(p.send[slot], self.gathered[slot], self.group)
            p.combine(slot, self.gathered[slot], out=self.emb[slot], stream=self.comm)
            ev = torch.cuda.Event()
            ev.record(self.comm)
        self.done[slot] = ev
        return self.emb[slot]

    def drain(self):
        """Make the current stream wait for every outstanding all-gather."""
        cs = torch.cuda.current_stream()
        for ev in self.done:
            if ev is not None:
                cs.wait_event(ev)
