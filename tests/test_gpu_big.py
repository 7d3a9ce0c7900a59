"""GDELT- and MAG-shaped configs at full size (configs[3], configs[4]) on the GPU.

The whole-graph oracle cannot hold these graphs, so parity is checked the way ③ allows
at full size: T-CSR `indptr` bit-exact against a host bincount of the COO, whole-array
invariants on the device output, and sampled nodes / queries / roots one by one
against oracle/big.py (pinned to the whole-graph oracle in test_oracle_big.py).  The
pipeline runs in the launch configuration bench.py times (captured CUDA graph).
"""
import os

import numpy as np
import pytest
import torch

import synth
from oracle import big
from oracle import pipeline as opipe

pytestmark = pytest.mark.gpu


def _mem_available_gb() -> float:
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) / 2**20
    except OSError:
        pass
    return 0.0


def _need(host_gb: float, dev_gb: float):
    if _mem_available_gb() < host_gb:
        pytest.skip(f"needs {host_gb} GB host RAM (have {_mem_available_gb():.0f})")
    if torch.cuda.get_device_properties(0).total_memory / 2**30 < dev_gb:
        pytest.skip(f"needs {dev_gb} GiB of device memory")


def _check_tcsr(cfg, src, dst, t, tc, src_h, dst_h, t_h, rng):
    N = cfg.n_nodes
    # indptr: bit-exact against the plain definition (degree counts, both directions)
    deg = np.bincount(src_h, minlength=N).astype(np.int64) + np.bincount(dst_h, minlength=N)
    exp = np.zeros(N + 1, np.int64)
    np.cumsum(deg, out=exp[1:])
    indptr = tc.indptr.cpu().numpy()
    assert np.array_equal(indptr, exp)
    # whole-array invariants: each eid twice, endpoints consistent, times sorted per owner
    M = 2 * cfg.n_edges
    cnt = torch.zeros(cfg.n_edges, dtype=torch.int32, device=src.device)
    for c0 in range(0, M, 1 << 28):
        e = tc.eid[c0:c0 + (1 << 28)].long()
        cnt.index_add_(0, e, torch.ones_like(e, dtype=torch.int32))
    assert bool((cnt == 2).all())
    del cnt
    for c0 in range(0, M, 1 << 28):
        c1 = min(M, c0 + (1 << 28))
        p = torch.arange(c0, c1, device=src.device)
        owner = torch.searchsorted(tc.indptr, p, right=True) - 1
        e = tc.eid[c0:c1].long()
        nb = tc.nbr[c0:c1]
        s_, d_ = src[e], dst[e]
        ok = ((s_ == owner) & (d_ == nb)) | ((d_ == owner) & (s_ == nb))
        assert bool(ok.all())
        assert torch.equal(tc.ts[c0:c1], t[e])
        if c1 - c0 > 1:
            same = owner[1:] == owner[:-1]
            ts = tc.ts[c0:c1]
            assert bool(((ts[1:] >= ts[:-1]) | ~same).all())
        del p, owner, e, nb, s_, d_, ok
    # segments of sampled owners (incl. the largest) against the oracle's definition
    nodes = np.concatenate([rng.choice(N, 20, replace=False), [int(np.argmax(deg))]])
    segs = big.node_segments(src_h, dst_h, t_h, nodes, N)
    for v in nodes:
        a, b = int(indptr[v]), int(indptr[v + 1])
        assert np.array_equal(tc.nbr[a:b].cpu().numpy(), segs[int(v)][0])
        assert np.array_equal(tc.eid[a:b].cpu().numpy(), segs[int(v)][1])
        assert np.array_equal(tc.ts[a:b].cpu().numpy(), segs[int(v)][2])
    return segs


def _run(name, host_gb, dev_gb):
    _need(host_gb, dev_gb)
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
    from synth import gpu as sg
    cfg = synth.get_config(name)
    dev = torch.device("cuda")
    rng = np.random.default_rng(5)
    src, dst, t = sg.device_graph(cfg, dev)
    neg = sg.device_negatives(cfg, dev)
    src_h, dst_h, t_h, neg_h = (x.cpu().numpy() for x in (src, dst, t, neg))
    torch.cuda.empty_cache()
    tc = tgl.build_tcsr(cfg.n_nodes, src, dst, t, True, True, packed=name != "MAG")
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    segs = _check_tcsr(cfg, src, dst, t, tc, src_h, dst_h, t_h, rng)
    torch.cuda.empty_cache()

    # the bench's layout (bench.load_world_device): split16 operand tables for every gather
    # (edge features, and MAG's node table, built chunk by chunk: those fp32 tables never
    # exist), fp32 node rows beside them where they fit (GDELT), so the kernels the bench
    # times run here
    rows_fn = lambda seed, dim: (lambda r0, r1: sg.feature_rows_torch(
        seed, torch.arange(r0, r1, device=dev), dim))
    if name == "MAG":
        nfeat = None
        nsplit = tgl.split_table(cfg.n_nodes, cfg.d_v, rows_fn(cfg.seeds["feat"], cfg.d_v))
    else:
        nfeat = sg.device_feature_table(cfg.seeds["feat"], cfg.n_nodes, cfg.d_v, dev,
                                        pitch_mult=4)
        nsplit = tgl.split_rows(nfeat)
    efeat = None
    efeat_split = (tgl.split_table(cfg.n_edges, cfg.d_e, rows_fn(cfg.seeds["feat"] + 7919, cfg.d_e))
                   if cfg.d_e else None)
    rows = rng.integers(0, cfg.n_nodes, 5)
    want_rows = torch.from_numpy(synth.feature_rows(cfg.seeds["feat"], rows, cfg.d_v)).to(dev)
    got_rows = nsplit[torch.from_numpy(rows).to(dev)].contiguous().view(torch.int32)
    assert torch.equal(got_rows, tgl.split_rows(want_rows).contiguous().view(torch.int32))
    params = synth.gen.model_params(cfg)
    graph = {"src": src, "dst": dst, "t": t, "neg": neg, "nfeat": nfeat, "efeat": efeat,
             "nfeat_split": nsplit, "efeat_split": efeat_split}
    layout = "split"
    pipe = TGATPipeline(graph, tc, params, cfg.batch,
                        TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), cfg.dedup,
                        cfg.precompute, cfg.window, "fp32", layout=layout)
    pipe.capture()
    pipe16 = TGATPipeline(graph, tc, params, cfg.batch,
                          TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), cfg.dedup,
                          cfg.precompute, cfg.window, "bf16", layout=layout)
    pipe16.capture()
    # the K|V kernel the bench times on this layout
    probe = tgl.KvProbe()
    tail = pipe.L - 1
    pipe.attn[tail].attach_probe(probe)
    pipe.start_dev.fill_(int(0.7 * cfg.n_batches) * cfg.batch)
    pipe.forward()
    torch.cuda.synchronize()
    pipe.attn[tail].attach_probe(None)
    want = "pre"
    assert probe.kernel == tgl.KV_KERNEL[want], (probe.kernel, want)

    class _G:   # host view for batch slicing
        pass
    gh = _G()
    gh.cfg, gh.src, gh.dst, gh.t, gh.num_edges = cfg, src_h, dst_h, t_h, cfg.n_edges
    for b in (0, int(0.7 * cfg.n_batches), cfg.n_batches - 1):   # first, bench region, last
        emb = pipe.run_graph(b * cfg.batch)
        torch.cuda.synchronize()
        emb = emb.cpu().numpy().copy()
        qn, qt = opipe.roots(*synth.batch_roots_inputs(gh, neg_h, b))
        assert emb.shape[0] == qn.shape[0] and np.isfinite(emb).all()
        # S4 per block on sampled queries (bit-exact)
        for l, blk in enumerate(pipe.blocks):
            n = int(blk.n_dev.item())
            dn, dt_ = blk.dst_node[:n].cpu().numpy(), blk.dst_t[:n].cpu().numpy()
            if l == 0:
                assert np.array_equal(dn, qn) and np.array_equal(dt_, qt)
            sp = blk.seg_ptr[:n + 1].cpu().numpy()
            pick = np.sort(rng.choice(n, min(n, 48), replace=False))
            segs.update(big.node_segments(src_h, dst_h, t_h,
                                          [v for v in dn[pick] if int(v) not in segs], cfg.n_nodes))
            esp, enb, eei, ets = big.sample_nodes(segs, dn[pick], dt_[pick], cfg.k, cfg.strategy,
                                                  cfg.seeds["sampler"], l)
            for j, i in enumerate(pick):
                a, c = int(sp[i]), int(sp[i + 1])
                ea, ec = int(esp[j]), int(esp[j + 1])
                assert np.array_equal(blk.nbr[a:c].cpu().numpy(), enb[ea:ec])
                assert np.array_equal(blk.eid[a:c].cpu().numpy(), eei[ea:ec])
                assert np.array_equal(blk.ts[a:c].cpu().numpy(), ets[ea:ec])
        # embeddings of sampled roots against Listing 1's recursion
        pick = rng.choice(qn.shape[0], 6, replace=False)
        exp = big.embed_recursive(src_h, dst_h, t_h, cfg, params, qn[pick], qt[pick],
                                  cfg.seeds["sampler"], segs=segs)
        err = np.abs(emb[pick] - exp).max()
        assert err <= 1e-3, err
        # bf16 projections (north_star: 5e-2) on the same batch
        e16 = pipe16.run_graph(b * cfg.batch)
        torch.cuda.synchronize()
        err16 = np.abs(e16.cpu().numpy()[pick] - exp).max()
        assert err16 <= 5e-2, err16
    del pipe, pipe16, graph, nfeat, nsplit, efeat, efeat_split, tc, src, dst, t, neg
    torch.cuda.empty_cache()


def test_gdelt_full_size():
    _run("GDELT", host_gb=24, dev_gb=170)


def test_mag_full_size():
    _run("MAG", host_gb=56, dev_gb=170)
