"""N2: tgl_tblock_attn_backward against the fp64 backward oracle.

oracle/backward.py is pinned on the CPU (tests/test_backward_cpu.py) by the C forward,
central finite differences of every parameter and input row, and closed forms.  Here
the CUDA backward (recomputed fp32 forward, strided fp32 GEMMs, segment kernels) must
match it on random layers at the configs' widths: every gradient tensor within
max|got - exp| <= 2e-4 * (1 + max|exp|) (fp32 products and sums over up to a few
thousand terms), including empty segments, duplicate source rows (scatter-adds), the
Listing-2-literal identity logit and an index offset for h_src.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import backward as ob

pytestmark = pytest.mark.gpu


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _case(rng, n_dst, kmax, d_h, d_e, slope=0.2):
    from dataclasses import replace
    cfg = replace(synth.get_config("REDDIT"), d_e=d_e)
    p = synth.make_layer_params(cfg, 0, d_h, d_h, random_ln=True, random_phi=True)
    p["leaky_slope"] = slope
    lens = rng.integers(0, kmax + 1, n_dst)
    seg = np.zeros(n_dst + 1, np.int64)
    seg[1:] = np.cumsum(lens)
    E = int(seg[-1])
    N = 300
    nfeat = rng.uniform(-1, 1, (N, d_h)).astype(np.float32)
    efeat = rng.uniform(-1, 1, (900, max(d_e, 1))).astype(np.float32)[:, :d_e]
    dst_node = rng.integers(0, N, n_dst).astype(np.int32)
    dst_t = rng.integers(10**5, 2 * 10**6, n_dst).astype(np.float32)
    src_node = rng.integers(0, N, E).astype(np.int32)
    eid = rng.integers(0, 900, E).astype(np.int32)
    edge_t = (np.repeat(dst_t, lens) - rng.integers(1, 200000, E)).astype(np.float32)
    return p, seg, dst_t, nfeat, dst_node, src_node, efeat, eid, edge_t


def _close(got, exp, what):
    got = np.asarray(got, np.float64)
    tol = 2e-4 * (1.0 + np.abs(exp).max())
    err = np.abs(got - exp).max() if exp.size else 0.0
    assert err <= tol, (what, err, tol)


@pytest.mark.parametrize("n_dst,kmax,d_h,d_e,slope", [(1, 10, 172, 172, 0.2),
                                                       (257, 10, 172, 172, 0.2),
                                                       (200, 20, 128, 128, 0.2),
                                                       (150, 10, 100, 0, 0.2),
                                                       (96, 10, 413, 186, 0.2),
                                                       (120, 10, 64, 16, -1.0)])
def test_backward_vs_oracle(n_dst, kmax, d_h, d_e, slope):
    from paper_conf_asplos_wangm24_b200 import tgl
    rng = np.random.default_rng(n_dst + d_h)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = _case(rng, n_dst, kmax, d_h, d_e, slope)
    G = rng.standard_normal((n_dst, p["d_out"])).astype(np.float32)
    _, tape = ob.tblock_forward(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    exp = ob.tblock_backward(p, tape, G.astype(np.float64), nfeat.shape[0], nfeat.shape[0])
    P = tgl.AttnParams(p, precision="fp32")
    grads = tgl.zero_grads(P)
    ghd = torch.zeros(nfeat.shape, device="cuda")
    ghs = torch.zeros(nfeat.shape, device="cuda")
    E = int(seg[-1])
    tgl.tblock_attn_backward(P, cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn),
                             cu(ef) if d_e else None, cu(eid) if d_e else None, cu(et), cu(G),
                             grads, ghd, ghs, n_edges_max=max(E, 1))
    torch.cuda.synchronize()
    for n in tgl.GRAD_NAMES:
        _close(grads[n].cpu().numpy(), exp[n], n)
    _close(ghd.cpu().numpy(), exp["hdst"], "hdst")
    _close(ghs.cpu().numpy(), exp["hsrc"], "hsrc")


def test_backward_device_counts_and_offset():
    """n_dst on the device (capacity larger), h_src rows at a device offset (the S14
    layout of the forward), and repeated calls accumulate."""
    from paper_conf_asplos_wangm24_b200 import tgl
    rng = np.random.default_rng(9)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = _case(rng, 70, 10, 100, 172)
    E = int(seg[-1])
    off = 70
    table = rng.uniform(-1, 1, (off + E + 3, 100)).astype(np.float32)
    G = rng.standard_normal((70, 100)).astype(np.float32)
    _, tape = ob.tblock_forward(p, seg, dst_t, table, None, table, np.arange(off, off + E), ef,
                                eid, et)
    exp = ob.tblock_backward(p, tape, G.astype(np.float64), table.shape[0], table.shape[0])
    P = tgl.AttnParams(p, precision="fp32")
    grads = tgl.zero_grads(P)
    gh = torch.zeros(table.shape, device="cuda")
    seg_cap = np.concatenate([seg, np.full(30, seg[-1])])        # capacity 100 destinations
    nd = torch.tensor([70], dtype=torch.int64, device="cuda")
    offd = torch.tensor([off], dtype=torch.int64, device="cuda")
    dst_cap = np.concatenate([dst_t, np.zeros(30, np.float32)])
    G_cap = np.concatenate([G, np.zeros((30, 100), np.float32)])
    for _ in range(2):
        tgl.tblock_attn_backward(P, cu(seg_cap), cu(dst_cap), cu(table), None, cu(table), None,
                                 cu(ef), cu(eid), cu(et), cu(G_cap), grads, gh, gh,
                                 n_dst_max=100, n_dst_dev=nd, n_edges_max=E + 40,
                                 hsrc_off_dev=offd)
    torch.cuda.synchronize()
    for n in tgl.GRAD_NAMES:
        _close(grads[n].cpu().numpy() / 2, exp[n], n)
    _close(gh.cpu().numpy() / 2, exp["hdst"] + exp["hsrc"], "h rows (dst + src, one table)")


def _oracle_chain_grads(cfg, g, neg, params, b, G):
    """Listing 2's block chain forward (oracle.pipeline's routing) with backward tapes,
    then the chain rule from the roots down: dL/d(emb) -> head rows (S14 adjoint) -> each
    block's input rows -> the block below."""
    import oracle
    from oracle import pipeline as opipe
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    qn, qt = opipe.roots(*synth.batch_roots_inputs(g, neg, b))
    blocks = opipe.build_blocks(tc, qn, qt, len(params), cfg.k, cfg.strategy, cfg.dedup,
                                cfg.seeds["sampler"])
    L = len(blocks)
    tapes, tables = [None] * L, [None] * L
    for l in range(L - 1, -1, -1):
        bl = blocks[l]
        if l == L - 1:
            hd, hd_idx, hs, hs_idx = g.nfeat, bl.uniq_node, g.nfeat, bl.nbr
        else:
            nxt = blocks[l + 1]
            tab = tables[l + 1].astype(np.float32)            # fp32 between layers (R17)
            U = bl.uniq_node.shape[0]
            if nxt.inv is not None:
                hd_idx, hs_idx = nxt.inv[:U], nxt.inv[U:]
            else:
                hd_idx = np.arange(U)
                hs_idx = np.arange(U, nxt.dst_node.shape[0])
            hd = hs = tab
        out, tape = ob.tblock_forward(params[l], bl.seg_ptr, bl.uniq_t, hd, hd_idx, hs, hs_idx,
                                      g.efeat, bl.eid, bl.ts)
        tapes[l], tables[l] = tape, out
    b0 = blocks[0]
    U0 = b0.uniq_node.shape[0]
    g_out = np.zeros((U0, params[0]["d_out"]))
    if b0.inv is not None:
        np.add.at(g_out, b0.inv, G)
    else:
        g_out += G
    res = []
    for l in range(L):
        rows = tables[l + 1].shape[0] if l + 1 < L else g.nfeat.shape[0]
        gr = ob.tblock_backward(params[l], tapes[l], g_out, rows, rows)
        res.append(gr)
        g_out = gr["hdst"] + gr["hsrc"]
    return res


@pytest.mark.parametrize("name,dedup", [("REDDIT", True), ("REDDIT", False), ("WIKI", False)])
def test_pipeline_backward_vs_oracle_chain(name, dedup):
    """TGATPipeline.backward: every layer's parameter gradients of a whole batch (the
    training step of the chain) against the oracle's chain rule over the same blocks."""
    from dataclasses import replace
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
    cfg = replace(synth.get_config(name).scaled(30000, batch=200), dedup=dedup)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy,
                                                             cfg.seeds["sampler"]),
                        cfg.dedup, cfg.precompute, cfg.window, "fp32")
    b = int(0.7 * cfg.n_batches)
    pipe.start_dev.fill_(b * cfg.batch)
    pipe.forward()
    G = np.random.default_rng(4).standard_normal((3 * cfg.batch, cfg.d_model)).astype(np.float32)
    grads = pipe.backward(cu(G))
    torch.cuda.synchronize()
    exp = _oracle_chain_grads(cfg, g, neg, params, b, G.astype(np.float64))
    for l in range(len(params)):
        for n in tgl.GRAD_NAMES:
            _close(grads[l][n].cpu().numpy(), exp[l][n], f"layer {l} {n}")
