"""Root sharding (S16) -- host logic on CPU, world_size 2 over gloo.

Each rank forms the batch's roots, dedups them (when the config does), takes its
contiguous slice `dist.shard_bounds`, runs the ORACLE chain (Listing 2's blocks) on
that slice only, and the slices are all-gathered with `dist.allgather_rows`; rank 0
rebuilds the batch through the roots' inverse.  That must equal the unsharded oracle
batch BITWISE (an embedding depends only on <node, t>: content-keyed sampling, R6).
The libtgl version of the same test (two processes on one GPU) is
tests/test_gpu_shard.py.
"""
import importlib.util
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _pdist():
    """paper_conf_asplos_wangm24_b200/dist.py by path (the package itself needs libtgl.so
    only for its CUDA entry points; the host logic here does not)."""
    spec = importlib.util.spec_from_file_location(
        "pdist", os.path.join(ROOT, "paper_conf_asplos_wangm24_b200", "dist.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _world(name, n_edges=4000):
    import synth
    base = synth.get_config(name)
    cfg = base.scaled(n_edges, 300 if base.bipartite else 0, 60 if base.bipartite else 400,
                      batch=30)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    return cfg, g, neg, params


def _sharded_slice(cfg, g, neg, params, b, rank, world, pdist):
    """This rank's slice of the batch's unique roots, computed by the oracle chain."""
    import oracle
    import synth
    from oracle import pipeline
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    qn, qt = pipeline.roots(*synth.batch_roots_inputs(g, neg, b))
    if cfg.dedup:
        un, ut, inv = oracle.dedup(qn, qt)
    else:
        un, ut, inv = qn, qt, None
    lo, hi = pdist.shard_bounds(len(un), rank, world)
    c = -(-len(un) // world)
    blocks = pipeline.build_blocks(tc, un[lo:hi], ut[lo:hi], len(params), cfg.k, cfg.strategy,
                                   cfg.dedup, cfg.seeds["sampler"])
    head = pipeline.aggregate(blocks, params, g.nfeat, g.efeat)
    if blocks[0].inv is not None:          # slice pairs are unique: identity inverse
        head = head[blocks[0].inv]
    out = np.zeros((c, head.shape[1]), np.float64)
    out[:hi - lo] = head
    return out, inv, len(un), c


def _worker(rank, world, port, name, out_path):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    pdist = _pdist()
    cfg, g, neg, params = _world(name)
    b = int(0.7 * cfg.n_batches)
    local, inv, U, c = _sharded_slice(cfg, g, neg, params, b, rank, world, pdist)
    gathered = torch.empty(world * c, local.shape[1], dtype=torch.float64)
    pdist.allgather_rows(torch.from_numpy(local), gathered)
    full = np.concatenate([gathered.numpy()[r * c: r * c + (pdist.shard_bounds(U, r, world)[1] -
                                                            pdist.shard_bounds(U, r, world)[0])]
                           for r in range(world)])
    emb = full[inv] if inv is not None else full
    if rank == 0:
        np.save(out_path, emb)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name", ["REDDIT", "GDELT"])
def test_two_rank_root_sharding_equals_unsharded(tmp_path, name):
    """REDDIT: roots deduped before the slice; GDELT: dedup off (slice of raw roots)."""
    import oracle
    import synth
    from oracle import pipeline
    out = str(tmp_path / "emb.npy")
    mp.spawn(_worker, args=(2, _free_port(), name, out), nprocs=2, join=True)
    got = np.load(out)
    cfg, g, neg, params = _world(name)
    b = int(0.7 * cfg.n_batches)
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    exp, _ = pipeline.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy, cfg.dedup,
                                cfg.seeds["sampler"], *synth.batch_roots_inputs(g, neg, b))
    assert got.shape == exp.shape
    np.testing.assert_array_equal(got, exp)


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_shard_bounds_partition(world):
    """The slices are contiguous, disjoint, cover [0, U) and differ in size by <= c."""
    pdist = _pdist()
    for U in (0, 1, 7, 8, 1799, 1800, 12000):
        spans = [pdist.shard_bounds(U, r, world) for r in range(world)]
        assert spans[0][0] == 0 and spans[-1][1] == U
        for (a0, a1), (b0, b1) in zip(spans[:-1], spans[1:]):
            assert a1 == b0 and a0 <= a1
        c = -(-U // world) if U else 0
        assert all(hi - lo <= c for lo, hi in spans)
