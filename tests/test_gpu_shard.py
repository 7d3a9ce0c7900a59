"""Root sharding (S16) through libtgl on the GPU.

1. One GPU, G in {2, 4, 8}: the G shard pipelines (TGATPipeline(shard=(r, G))) run one
   after another on the same batch; their slices are concatenated in rank order (what
   the all-gather produces) and rebuilt with tgl_shard_gather.  The result must match
   the unsharded pipeline within 1e-3 (an embedding depends only on <node, t>; the
   summation order inside a softmax segment may differ), and every sampled segment of
   every shard must equal, bit for bit, the unsharded run's segment of the same (node, t) (content-keyed
   Philox, reading R6).
2. Two processes on one GPU over gloo, each running libtgl through dist.ShardedRunner
   (the driver the bench uses with NCCL): rank 0's batch embeddings match the
   unsharded pipeline within 1e-3.
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _world(name, n_edges):
    base = synth.get_config(name)
    cfg = base.scaled(n_edges, batch=base.batch if name != "GDELT" else 400)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    return cfg, g, neg, params, dev


def _pipe(cfg, params, dev, tc, shard=None):
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler
    return TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy,
                                                             cfg.seeds["sampler"]),
                        cfg.dedup, cfg.precompute, cfg.window, "fp32", shard=shard)


def _segments(pipe):
    """{(layer, node, t bits): (nbr, eid, ts)} over every block's sampled segments."""
    out = {}
    for l, b in enumerate(pipe.blocks):
        U = int(b.u_dev.item())
        un = b.uniq_node[:U].cpu().numpy()
        ut = b.uniq_t[:U].cpu().numpy().view(np.uint32)
        sp = b.seg_ptr[:U + 1].cpu().numpy()
        m = int(sp[-1])
        nb, ei = b.nbr[:m].cpu().numpy(), b.eid[:m].cpu().numpy()
        ts = b.ts[:m].cpu().numpy().view(np.uint32)
        for i in range(U):
            out[(l, int(un[i]), int(ut[i]))] = (nb[sp[i]:sp[i + 1]].tobytes(),
                                                ei[sp[i]:sp[i + 1]].tobytes(),
                                                ts[sp[i]:sp[i + 1]].tobytes())
    return out


@pytest.mark.parametrize("name,n_edges", [("REDDIT", 120000), ("GDELT", 200000)])
def test_shard_slices_compose_to_unsharded(name, n_edges):
    from paper_conf_asplos_wangm24_b200 import tgl
    cfg, g, neg, params, dev = _world(name, n_edges)
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    ref = _pipe(cfg, params, dev, tc)
    n0 = 3 * cfg.batch
    for b in (0, cfg.n_batches // 2, cfg.n_batches - 1):   # first, middle, last batch
        ref.start_dev.fill_(b * cfg.batch)
        exp = ref.forward()[:n0].cpu().numpy().copy()
        exp_segs = _segments(ref)
        for G in (2, 4, 8):
            pipes = [_pipe(cfg, params, dev, tc, shard=(r, G)) for r in range(G)]
            gathered = torch.zeros(G * pipes[0].c_max, cfg.d_model, device="cuda")
            for r, p in enumerate(pipes):
                p.start_dev.fill_(b * cfg.batch)
                sl = p.forward(slot=0)
                gathered[r * p.c_max:(r + 1) * p.c_max] = sl
                for key, val in _segments(p).items():   # bit-exact samples per (node, t)
                    assert exp_segs[key] == val, (G, r, key)
            got = pipes[0].combine(0, gathered).cpu().numpy()[:n0]
            err = np.abs(got - exp).max()
            # same math per <node, t>; only the lane alignment of a segment inside the
            # K|V kernel's 32-row bins (its shuffle-scan order) differs between the runs
            assert err <= 1e-3, (b, G, err)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_path):
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_asplos_wangm24_b200 import tgl
    from paper_conf_asplos_wangm24_b200.dist import ShardedRunner
    cfg, g, neg, params, dev = _world("REDDIT", 120000)
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = _pipe(cfg, params, dev, tc, shard=(rank, world))
    pipe.capture()
    run = ShardedRunner(pipe)
    outs = []
    for b in (10, 11, 12):       # consecutive batches: slot 0, 1, 0 (overlapped gathers)
        e = run.step(b * cfg.batch)
        run.drain()
        torch.cuda.synchronize()
        outs.append(e.cpu().numpy().copy())
    if rank == 0:
        np.save(out_path, np.stack(outs))
    dist.barrier()
    dist.destroy_process_group()


def test_two_process_sharded_runner_libtgl(tmp_path):
    import torch.multiprocessing as mp
    from paper_conf_asplos_wangm24_b200 import tgl
    out = str(tmp_path / "emb.npy")
    mp.spawn(_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    got = np.load(out)
    cfg, g, neg, params, dev = _world("REDDIT", 120000)
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    ref = _pipe(cfg, params, dev, tc)
    n0 = 3 * cfg.batch
    for i, b in enumerate((10, 11, 12)):
        ref.start_dev.fill_(b * cfg.batch)
        exp = ref.forward()[:n0].cpu().numpy()
        assert np.abs(got[i] - exp).max() <= 1e-3
