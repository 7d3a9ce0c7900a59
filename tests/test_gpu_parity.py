"""GPU parity: every C-ABI call against the CPU oracle on the same seeded inputs.

Bit-exact for T-CSR, sampling and dedup; <= 2 ulp for the time encoder;
max abs 1e-3 (fp32) / 5e-2 (bf16) for attention outputs and embeddings
(north_star tolerances).  Sizes span several tiles and a ragged tail.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle import pipeline as opipe
import synth

pytestmark = pytest.mark.gpu

TOL = {"fp32": 1e-3, "bf16": 5e-2, "fp32_simt": 1e-3}


@pytest.fixture(scope="module")
def T():
    from paper_conf_asplos_wangm24_b200 import tgl
    return tgl


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def np_(t):
    return t.detach().cpu().numpy()


def rand_graph(rng, N, E, max_t, sort=True):
    src = rng.integers(0, N, E).astype(np.int32)
    dst = rng.integers(0, N, E).astype(np.int32)
    dst[::13] = src[::13]
    t = rng.integers(0, max_t, E).astype(np.float32)
    if sort:
        o = np.argsort(t, kind="stable")
        src, dst, t = src[o], dst[o], t[o]
    return src, dst, t


# ------------------------------------------------------------------ S1
@pytest.mark.parametrize("undirected", [True, False])
@pytest.mark.parametrize("sort", [True, False])
@pytest.mark.parametrize("N,E,max_t", [(1, 5, 3), (50, 3000, 40), (3000, 20000, 10**6),
                                       (70000, 5000, 100), (300, 0, 1)])
def test_tcsr_bit_exact(T, N, E, max_t, undirected, sort):
    rng = np.random.default_rng(N * 7 + E)
    src, dst, t = rand_graph(rng, N, E, max_t, sort)
    g = T.build_tcsr(N, cu(src), cu(dst), cu(t), undirected=undirected, time_sorted=sort)
    exp = oracle.build_tcsr(N, src, dst, t, undirected)
    got = (np_(g.indptr), np_(g.nbr), np_(g.eid), np_(g.ts))
    for a, b in zip(got, exp):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("N,E,max_t,sort", [(20000, 300000, 50, True), (45000, 250000, 10**7, False),
                                            (256, 70000, 3, True), (257, 70000, 3, True)])
def test_tcsr_ex_indexes_and_tiles(T, N, E, max_t, sort):
    """tgl_build_tcsr_ex (one sweep of 16-byte records, indexes written by the last pass)
    over many 4,096-entry tiles with heavy time ties: T-CSR bit-exact against the oracle,
    ts_coarse / entries bit-exact against tgl_tcsr_index run on the result, and the
    one-pass (N <= 256) / two-pass, degree / owner-key indptr variants."""
    import torch
    rng = np.random.default_rng(N + E)
    src, dst, t = rand_graph(rng, N, E, max_t, sort)
    g = T.build_tcsr(N, cu(src), cu(dst), cu(t), True, sort)
    exp = oracle.build_tcsr(N, src, dst, t, True)
    for a, b in zip((g.indptr, g.nbr, g.eid, g.ts), exp):
        assert np.array_equal(np_(a), b)
    ref = T.TemporalCSR(g.indptr, g.nbr, g.eid, g.ts, coarse=True, packed=True)
    torch.cuda.synchronize()
    assert np.array_equal(np_(g.ts_coarse).view(np.uint32), np_(ref.ts_coarse).view(np.uint32))
    assert np.array_equal(np_(g.entries), np_(ref.entries))


@pytest.mark.parametrize("name", ["WIKI", "REDDIT", "LASTFM"])
def test_tcsr_full_configs(T, name):
    cfg = synth.get_config(name)
    gr = synth.make_graph(cfg, with_features=False)
    g = T.build_tcsr(cfg.n_nodes, cu(gr.src), cu(gr.dst), cu(gr.t), True, True)
    exp = oracle.build_tcsr(cfg.n_nodes, gr.src, gr.dst, gr.t, True)
    for a, b in zip((g.indptr, g.nbr, g.eid, g.ts), exp):
        assert np.array_equal(np_(a), b)


# ------------------------------------------------------------------ S4
@pytest.mark.parametrize("index", ["coarse+packed", "none", "coarse"])
@pytest.mark.parametrize("strategy", ["recent", "uniform"])
@pytest.mark.parametrize("k", [1, 10, 20, 45])
def test_sample_bit_exact(T, strategy, k, index):
    """Bit-exact against the oracle with and without the sampler indexes of
    tgl_tcsr_index (fence index ts_coarse, packed 16-byte entries)."""
    rng = np.random.default_rng(k)
    N, E = 400, 60000
    src, dst, t = rand_graph(rng, N, E, 5000)
    src[:20000] = 7  # one huge segment (multi-round search)
    o = np.argsort(t, kind="stable")
    src, dst, t = src[o], dst[o], t[o]
    g = T.build_tcsr(N, cu(src), cu(dst), cu(t), True, True, coarse="coarse" in index,
                     packed="packed" in index)
    tc = oracle.build_tcsr(N, src, dst, t, True)
    nq = 3001
    qn = rng.integers(0, N, nq).astype(np.int32)
    qn[::5] = 7
    qt = rng.uniform(-10, 5100, nq).astype(np.float32)
    qt[::17] = np.nan
    qt[::19] = 0.0
    qt[1::19] = -0.0
    qt[::23] = t[rng.integers(0, E, len(qt[::23]))]   # exact ties
    sid = 0x74676C00 + k
    seg, nb, ei, ts = T.sample(g, cu(qn), cu(qt), k, strategy, seed=sid, layer=1)
    es, en, ee, et = oracle.sample(tc, qn, qt, k, opipe.STRATEGY[strategy], sid, 1)
    m = int(es[-1])
    assert np.array_equal(np_(seg), es)
    assert np.array_equal(np_(nb)[:m], en)
    assert np.array_equal(np_(ei)[:m], ee)
    assert np.array_equal(np_(ts)[:m], et)


def test_sample_device_count_and_empty(T):
    rng = np.random.default_rng(3)
    src, dst, t = rand_graph(rng, 100, 5000, 1000)
    g = T.build_tcsr(100, cu(src), cu(dst), cu(t), True, True)
    tc = oracle.build_tcsr(100, src, dst, t, True)
    qn = rng.integers(0, 100, 500).astype(np.int32)
    qt = rng.uniform(0, 1000, 500).astype(np.float32)
    for nq in (0, 1, 31, 32, 33, 499):
        ndev = torch.tensor([nq], dtype=torch.int64, device="cuda")
        seg, nb, ei, ts = T.sample(g, cu(qn), cu(qt), 10, "uniform", seed=1, nq_dev=ndev)
        es, en, ee, et = oracle.sample(tc, qn[:nq], qt[:nq], 10, 1, 1, 0)
        assert np.array_equal(np_(seg)[:nq + 1], es)
        assert np.array_equal(np_(nb)[:int(es[-1])], en)


# ------------------------------------------------------------------ S3
@pytest.mark.parametrize("n", [0, 1, 1800, 2047, 2048, 2049, 4096, 4097, 8193, 20000, 32768, 32769, 200001])
def test_dedup_bit_exact(T, n):
    rng = np.random.default_rng(n + 1)
    node = rng.integers(0, max(2, n // 8), n).astype(np.int32)
    t = rng.integers(0, 50, n).astype(np.float32)
    if n > 10:
        t[::7] = -0.0
        t[::11] = 0.0
    un, ut, nu, inv = T.dedup(cu(node), cu(t)) if n else T.dedup(
        torch.zeros(1, dtype=torch.int32, device="cuda"),
        torch.zeros(1, dtype=torch.float32, device="cuda"), n_max=0)
    eu, eut, einv = oracle.dedup(node, t)
    U = int(np_(nu)[0])
    assert U == len(eu)
    assert np.array_equal(np_(un)[:U], eu)
    assert np.array_equal(np_(ut)[:U].view(np.uint32), eut.view(np.uint32))
    assert np.array_equal(np_(inv)[:n], einv)


@pytest.mark.parametrize("n_max,n", [(10000, 6001), (4000, 1234)])   # multi-kernel / 1-CTA
def test_dedup_device_count(T, n_max, n):
    rng = np.random.default_rng(9)
    node = rng.integers(0, 300, n_max).astype(np.int32)
    t = rng.integers(0, 30, n_max).astype(np.float32)
    ndev = torch.tensor([n], dtype=torch.int64, device="cuda")
    un, ut, nu, inv = T.dedup(cu(node), cu(t), n_dev=ndev)
    eu, eut, einv = oracle.dedup(node[:n], t[:n])
    U = int(np_(nu)[0])
    assert U == len(eu) and np.array_equal(np_(un)[:U], eu)
    assert np.array_equal(np_(inv)[:n], einv)


# ------------------------------------------------------------------ S6
def ulp_diff(a, b):
    a = a.astype(np.float32)
    b = b.astype(np.float32)
    sp = np.spacing(np.maximum(np.abs(a), np.abs(b)))
    return np.abs(a.astype(np.float64) - b) / sp


def test_time_encode_ulp_and_table(T):
    cfg = synth.get_config("LASTFM")
    for random_phi in (False, True):
        omega, phi = synth.make_time_params(cfg, random_phi, seed=4)
        rng = np.random.default_rng(5)
        dt = np.concatenate([np.arange(0, 70000, 7, dtype=np.float32),
                             rng.uniform(0, 1.4e8, 20000).astype(np.float32),
                             np.array([0.5, -0.0, 65535, 65536, 3.3e-3], np.float32)])
        o, p = cu(omega), cu(phi)
        direct = np_(T.time_encode(cu(dt), o, p))
        exp = oracle.time_encode(dt, omega, phi)
        assert ulp_diff(direct, exp).max() <= 2.0
        tab = T.time_precompute(65536, o, p)
        assert np.array_equal(np_(tab).view(np.uint32),
                              np_(T.time_encode(cu(np.arange(65536, dtype=np.float32)), o, p)).view(np.uint32))
        with_tab = np_(T.time_encode(cu(dt), o, p, table=tab))
        assert np.array_equal(with_tab.view(np.uint32), direct.view(np.uint32))


# ------------------------------------------------------------------ S7-S13
def attn_case(rng, n_dst, kmax, d_h, d_e, empty=True, long_every=0):
    from dataclasses import replace
    cfg = replace(synth.get_config("REDDIT"), d_e=d_e)
    p = synth.make_layer_params(cfg, 0, d_h, d_h, random_ln=True, random_phi=True)
    lens = rng.integers(0 if empty else 1, kmax + 1, n_dst)
    if long_every:
        lens[::long_every] = 300          # segments longer than one 128-row chunk
    seg = np.zeros(n_dst + 1, np.int64)
    seg[1:] = np.cumsum(lens)
    E = int(seg[-1])
    N = 500
    nfeat = rng.uniform(-1, 1, (N, d_h)).astype(np.float32)
    efeat = rng.uniform(-1, 1, (2000, max(d_e, 1))).astype(np.float32)[:, :d_e]
    dst_node = rng.integers(0, N, n_dst).astype(np.int32)
    dst_t = rng.integers(10**5, 2 * 10**6, n_dst).astype(np.float32)
    src_node = rng.integers(0, N, E).astype(np.int32)
    eid = rng.integers(0, 2000, E).astype(np.int32)
    gap = rng.integers(1, 200000, E)
    gap[::3] = rng.integers(1, 60000, len(gap[::3]))
    edge_t = (np.repeat(dst_t, lens) - gap).astype(np.float32)
    return p, seg, dst_t, nfeat, dst_node, src_node, efeat, eid, edge_t


def cu_pad(a, mult=4):
    """Device copy whose rows are padded to a multiple of `mult` columns (16-B pitch
    for fp32), returned as a view of the true width -- the layout TMA gathers need."""
    n, d = a.shape
    dp = max(mult, (d + mult - 1) // mult * mult)
    t = torch.zeros(n, dp, dtype=torch.float32, device="cuda")
    t[:, :d] = cu(a)
    return t[:, :d]


@pytest.mark.parametrize("precision,kv", [("fp32", "pre"), ("bf16", "pre"), ("fp32", "pre2"),
                                          ("bf16", "pre2"),
                                          ("fp32", "split"), ("bf16", "split"),
                                          ("fp32", "split_pad"), ("bf16", "split_pad"),
                                          ("fp32", "async"), ("bf16", "async"), ("fp32", "bin"),
                                          ("bf16", "bin"), ("fp32_simt", None)])
@pytest.mark.parametrize("n_dst,kmax,d_h,d_e,long_every", [(1, 10, 172, 172, 0),
                                                          (777, 10, 172, 172, 0),
                                                          (300, 20, 128, 128, 0),
                                                          (200, 10, 100, 0, 0),
                                                          (333, 10, 413, 186, 0),
                                                          (517, 10, 128, 0, 0),
                                                          (150, 10, 24, 12, 7),
                                                          (148 * 12 + 37, 10, 413, 186, 0)])
def test_attention_vs_oracle(T, monkeypatch, precision, kv, n_dst, kmax, d_h, d_e, long_every):
    """tgl_attn_params.kv_kernel selects the K|V kernel: "split" (default: loader /
    converter warps, K chunks cut contiguously over [h | e | Phi] when the widths are
    multiples of 4, else per-segment padded), "split_pad" (the same kernel with every
    segment padded to 32 columns), "async" (single-role cp.async producers) -- all three
    need 16-B row pitches: the odd GDELT widths 413/186 go in row-padded views -- or "bin"
    (register gathers).  The 413/186 case with 1,813 destinations is 14k edges, ~120
    tiles: several tiles per CTA, so the persistent loop runs the padded plan through
    the alternating-K weight reuse (the path the GDELT bench times)."""
    rng = np.random.default_rng(n_dst + kmax)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, n_dst, kmax, d_h, d_e,
                                                          long_every=long_every)
    if kv in ("pre", "pre2") and np.diff(seg).max() > 32:
        pytest.skip("the pre-split kernel takes segments <= 32 rows (binned epilogue)")
    sel = kv if (kv and np.diff(seg).max() <= 32) else "auto"   # longer: general kernel
    exp = oracle.tblock_attn(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    P = T.AttnParams(p, precision=precision, pack=(n_dst % 2 == 1), kv_kernel=sel)
    probe = T.KvProbe()
    P.attach_probe(probe)
    tab = T.time_precompute(65536, P.t["omega"], P.t["phi"])
    put = cu_pad if kv in ("async", "split", "split_pad") else cu
    nf = put(nfeat)
    hs, efd = nf, (put(ef) if d_e else None)
    tables = [(None, 0, nf), (tab, 0, nf)]
    if kv in ("pre", "pre2"):  # split16 operand tables (tgl_split_rows), fp32 h_dst
        hs = T.split_rows(nf)
        efd = T.split_rows(efd) if d_e else None
        base = T.SPLIT_HSRC | (T.SPLIT_E if d_e else 0)
        ts = T.split_rows(tab)
        tables = [(None, base, nf), (tab, base, nf), (ts, base | T.SPLIT_TABLE, nf),
                  # split16 h_dst too: converter-free Q / FFN (dense_pre)
                  (ts, base | T.SPLIT_TABLE | T.SPLIT_HDST, hs),
                  (None, base | T.SPLIT_HDST, hs)]
    for table, layout, hd in tables:
        P.struct.input_layout = layout
        got = T.tblock_attn(P, cu(seg), cu(dst_t), hd, cu(dn), hs, cu(sn),
                            efd, cu(eid) if d_e else None, cu(et),
                            table=table, max_seg=int(np.diff(seg).max()))
        err = np.abs(np_(got)[:n_dst] - exp).max()
        assert err <= TOL[precision], err
        if kv in ("pre", "pre2") and sel == "auto":   # long segments: no split path
            continue
        if sel != "auto" and precision != "fp32_simt":   # the requested kernel really ran
            want = T.KV_KERNEL[sel]
            if sel == "split" and (d_h % 4 or d_e % 4):
                want = T.KV_KERNEL["split_pad"]
            assert probe.kernel == want, (probe.kernel, want)


@pytest.mark.parametrize("d", [1, 8, 100, 186, 413])
def test_split_rows_is_the_bf16_operand_split(T, d):
    """tgl_split_rows: per row bf16 RNE(x) of the 8-padded columns, then bf16 RNE(x - hi)
    (torch's float -> bfloat16 conversion is RNE), zeros past d; bit-exact."""
    rng = np.random.default_rng(d)
    x = rng.uniform(-3, 3, (517, d)).astype(np.float32)
    x[0, :] = 0.0
    x[1, :min(d, 4)] = [1e-30, -2.5e-8, 3.0e30, -0.0][:min(d, 4)]
    got = T.split_rows(cu_pad(x))[:517].cpu().numpy().view(np.uint16)   # [n, 2 dp] bf16
    dp = T.split_width(d)
    xt = torch.zeros(517, dp)
    xt[:, :d] = torch.from_numpy(x)
    hi = xt.to(torch.bfloat16)
    lo = (xt - hi.float()).to(torch.bfloat16)
    exp = torch.cat([hi, lo], 1).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(got, exp)


def test_attention_async_rejects_unaligned_pitch(T, monkeypatch):
    """kv_kernel=async on a 413-float row pitch (1652 B, not a multiple of 16):
    EUNSUPPORTED, while the default dispatch falls back to the register-gather kernel."""
    rng = np.random.default_rng(5)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, 64, 10, 413, 186)
    exp = oracle.tblock_attn(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    P = T.AttnParams(p, kv_kernel="async")
    args = (cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn), cu(ef), cu(eid), cu(et))
    with pytest.raises(T.TGLError):
        T.tblock_attn(P, *args, max_seg=10)
    P.set_kv_kernel("auto")
    probe = T.KvProbe()
    P.attach_probe(probe)
    got = T.tblock_attn(P, *args, max_seg=10)
    assert probe.kernel == T.KV_KERNEL["bin"]
    assert np.abs(np_(got)[:64] - exp).max() <= 1e-3


def test_attention_general_path_any_segment_length(T):
    """max_seg <= 0 (unknown) routes to the general kernel: segments of any length."""
    rng = np.random.default_rng(21)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, 120, 40, 172, 172,
                                                          long_every=9)
    exp = oracle.tblock_attn(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    P = T.AttnParams(p)
    got = T.tblock_attn(P, cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn), cu(ef),
                        cu(eid), cu(et), max_seg=0)
    assert np.abs(np_(got)[:120] - exp).max() <= 1e-3


def test_attention_offsets_and_identity(T):
    """hdst_idx = NULL (identity), hsrc rows at a device offset (the S14 layout)."""
    rng = np.random.default_rng(11)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, 90, 10, 100, 172)
    E = int(seg[-1])
    table = rng.uniform(-1, 1, (90 + E + 5, 100)).astype(np.float32)
    off = 90
    exp = oracle.tblock_attn(p, seg, dst_t, table, None, table, np.arange(off, off + E), ef, eid, et)
    P = T.AttnParams(p)
    offd = torch.tensor([off], dtype=torch.int64, device="cuda")
    nd = torch.tensor([90], dtype=torch.int64, device="cuda")
    got = T.tblock_attn(P, cu(seg), cu(dst_t), cu(table), None, cu(table), None, cu(ef),
                        cu(eid), cu(et), max_seg=10, n_dst_max=90, n_dst_dev=nd,
                        hsrc_off_dev=offd)
    assert np.abs(np_(got)[:90] - exp).max() <= 1e-3


# ------------------------------------------------------------------ pipeline (all rows)
def _world(name, n_edges=None, dedup=None, strategy=None):
    from dataclasses import replace
    cfg = synth.get_config(name)
    if n_edges:
        cfg = cfg.scaled(n_edges)
    if dedup is not None:
        cfg = replace(cfg, dedup=dedup)
    if strategy is not None:
        cfg = replace(cfg, strategy=strategy)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    return cfg, g, neg, params


def _gpu_pipeline(T, cfg, g, neg, params, precision="fp32", dev=None, layout=None,
                  node_proj=None):
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler
    if dev is None:
        dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
               "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    tc = T.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = TGATPipeline(dev, tc, params, cfg.batch,
                        TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), cfg.dedup,
                        cfg.precompute, cfg.window, precision, layout=layout,
                        node_proj=node_proj)
    return pipe


@pytest.mark.parametrize("name,precision", [("WIKI", "fp32"), ("REDDIT", "fp32"),
                                            ("LASTFM", "fp32"), ("REDDIT", "bf16")])
def test_pipeline_full_config_vs_oracle(T, name, precision):
    """Full-size configs[0..2], whole batches -- the first (roots at the earliest times:
    empty segments), one in the middle, the bench region (70 %) and the last -- in the launch configuration bench.py times (captured CUDA graph):
    every block's structure bit-exact, every root embedding within the north_star
    tolerance (1e-3 fp32, 5e-2 bf16)."""
    cfg, g, neg, params = _world(name)
    pipe = _gpu_pipeline(T, cfg, g, neg, params, precision)
    pipe.capture()
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    nb = cfg.n_batches
    for b in (0, nb // 2, int(0.7 * nb), nb - 1):
        emb = pipe.run_graph(b * cfg.batch)
        torch.cuda.synchronize()
        exp, blocks = opipe.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy,
                                      cfg.dedup, cfg.seeds["sampler"],
                                      *synth.batch_roots_inputs(g, neg, b))
        # bit-exact block structure
        for gb, ob in zip(pipe.blocks, blocks):
            U = len(ob.uniq_node)
            assert int(np_(gb.u_dev)[0]) == U
            assert np.array_equal(np_(gb.uniq_node)[:U], ob.uniq_node)
            assert np.array_equal(np_(gb.seg_ptr)[:U + 1], ob.seg_ptr)
            m = int(ob.seg_ptr[-1])
            assert np.array_equal(np_(gb.nbr)[:m], ob.nbr)
            assert np.array_equal(np_(gb.eid)[:m], ob.eid)
            if ob.inv is not None:
                assert np.array_equal(np_(gb.inv)[:len(ob.inv)], ob.inv)
        n0 = 3 * cfg.batch
        err = np.abs(np_(emb)[:n0] - exp).max()
        assert err <= TOL[precision], (b, err)


@pytest.mark.parametrize("name", ["REDDIT", "GDELT"])
def test_pipeline_layouts_agree(T, name):
    """The product layout (split16 operand tables, kv_pre) and fp32 tables converted in
    the SM (kv_split) compute the same operands (bf16 hi / lo of the same fp32 values):
    both within 1e-3 of the oracle, within 1e-4 of each other (the K chunking and so
    the fp32 accumulation order differ; LayerNorm scales the difference up)."""
    cfg, g, neg, params = _world(name, n_edges=120000)
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu_pad(g.nfeat), "efeat": cu_pad(g.efeat)}
    ps = _gpu_pipeline(T, cfg, g, neg, params, dev=dev, layout="split")
    pf = _gpu_pipeline(T, cfg, g, neg, params, dev=dev, layout="fp32")
    b = int(0.7 * cfg.n_batches)
    n0 = 3 * cfg.batch
    for p in (ps, pf):
        p.start_dev.fill_(b * cfg.batch)
    es, ef = np_(ps.forward())[:n0].copy(), np_(pf.forward())[:n0].copy()
    exp, _ = opipe.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy, cfg.dedup,
                             cfg.seeds["sampler"], *synth.batch_roots_inputs(g, neg, b))
    assert np.abs(es - exp).max() <= 1e-3
    assert np.abs(ef - exp).max() <= 1e-3
    assert np.abs(es - ef).max() <= 1e-4


def test_pipeline_dedup_on_off_and_graph_replay(T):
    """Semantics preservation on the GPU and CUDA-graph replay == eager."""
    cfg, g, neg, params = _world("REDDIT", n_edges=60000)
    from dataclasses import replace
    p_on = _gpu_pipeline(T, cfg, g, neg, params)
    p_off = _gpu_pipeline(T, replace(cfg, dedup=False), g, neg, params)
    b = 80
    p_on.start_dev.fill_(b * cfg.batch)
    p_off.start_dev.fill_(b * cfg.batch)
    e_on = np_(p_on.forward()).copy()
    e_off = np_(p_off.forward())[:3 * cfg.batch]
    assert np.abs(e_on - e_off).max() <= 1e-4
    p_on.capture()
    e_g = np_(p_on.run_graph(b * cfg.batch))
    assert np.array_equal(e_g, e_on)


def test_pipeline_lastfm_sampled_roots(T):
    """LastFM-shaped (k=20, heavy skew): roots checked one by one with the recursive oracle."""
    cfg, g, neg, params = _world("LASTFM")
    pipe = _gpu_pipeline(T, cfg, g, neg, params)
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    b = int(0.7 * cfg.n_batches)
    pipe.start_dev.fill_(b * cfg.batch)
    emb = np_(pipe.forward())
    qn, qt = opipe.roots(*synth.batch_roots_inputs(g, neg, b))
    pick = np.random.default_rng(0).choice(len(qn), 24, replace=False)
    exp = oracle.embed_recursive(tc, g.nfeat, g.efeat, params, cfg.k, opipe.STRATEGY[cfg.strategy],
                                 cfg.seeds["sampler"], qn[pick], qt[pick])
    assert np.abs(emb[pick] - exp).max() <= 1e-3


def test_host_stream_matches_graph(T):
    """The pipelined public host API (HostStream: H2D, replay, D2D ring, D2H on a copy
    stream) returns, batch by batch, exactly the captured graph's embeddings."""
    from paper_conf_asplos_wangm24_b200 import HostStream, TGATPipeline, TSampler
    cfg, g, neg, params = _world("REDDIT", n_edges=60000)
    ref = _gpu_pipeline(T, cfg, g, neg, params)
    ref.capture()
    dev = ref.g
    ph = TGATPipeline(dev, ref.tcsr, params, cfg.batch,
                      TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), cfg.dedup,
                      cfg.precompute, cfg.window, "fp32", staging=True)
    ph.capture()
    n0 = 3 * cfg.batch
    hs = HostStream(ph, n0, cfg.d_model)
    outs = [torch.empty(n0, cfg.d_model).pin_memory() for _ in range(2)]
    batches = [60, 61, 62, 63, 64]
    evs, got = [], []
    for i, b in enumerate(batches):
        hb = [torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
              for x in synth.batch_roots_inputs(g, neg, b)]
        evs.append(hs.submit(*hb, outs[i % 2]))
        if i >= 1:
            evs[i - 1].synchronize()
            got.append(outs[(i - 1) % 2].numpy().copy())
    evs[-1].synchronize()
    got.append(outs[(len(batches) - 1) % 2].numpy().copy())
    for b, e in zip(batches, got):
        exp = np_(ref.run_graph(b * cfg.batch))[:n0]
        assert np.array_equal(e, exp), b


@pytest.mark.parametrize("d_h,d_e", [(172, 172), (413, 186)])
def test_fused_phi_matches_exact_table(T, d_h, d_e):
    """The K|V kernels evaluate Phi in the SM (reduced argument + SFU cosine, abs error
    < 2e-6, DESIGN R10 / tenc.cuh); the precompute table holds the exact R10 values
    (bit-identical to tgl_time_encode).  With every dt an integer inside the window, the
    same call with and without the table differs only by the fused Phi's error: pinned
    here at 3e-5 on the outputs -- 30x tighter than the 1e-3 parity bound, so a Phi bug
    that stays under that bound still fails here."""
    rng = np.random.default_rng(d_h + d_e)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, 1500, 10, d_h, d_e)
    P = T.AttnParams(p, precision="fp32", pack=True, kv_kernel="pre")
    dt = np.repeat(dst_t, np.diff(seg)) - et
    assert (dt == np.round(dt)).all() and dt.min() >= 0 and dt.max() < (1 << 18)
    tab = T.split_rows(T.time_precompute(1 << 18, P.t["omega"], P.t["phi"]))
    nf = cu(nfeat)
    hs, efd = T.split_rows(nf), T.split_rows(cu(ef))
    base = T.SPLIT_HSRC | T.SPLIT_E
    outs = []
    for table, layout in ((None, base), (tab, base | T.SPLIT_TABLE)):
        P.struct.input_layout = layout
        got = T.tblock_attn(P, cu(seg), cu(dst_t), nf, cu(dn), hs, cu(sn), efd, cu(eid),
                            cu(et), table=table, max_seg=10)
        outs.append(np_(got)[:1500].copy())
    exp = oracle.tblock_attn(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    assert np.abs(outs[1] - exp).max() <= 1e-3
    assert np.abs(outs[0] - outs[1]).max() <= 3e-5, np.abs(outs[0] - outs[1]).max()
