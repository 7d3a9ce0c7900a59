"""N3: the TGN memory path through libtgl against oracle/memory.py.

tgl_mailbox_store: unique nodes, picks (coalesce by='latest', R26) and the stored mailbox
rows / times are compared bit for bit (index work and row copies); tgl_memory_update:
memory rows within 1e-5 * (1 + |s|) (fp32 GEMMs of <= 600 exact products, fp32 sums,
accurate expf / tanhf), mem_ts bit for bit, rows of other nodes untouched; a TGN loop
(update the batch's nodes, then store its messages, Listing 4) over consecutive batches
of a seeded graph keeps the state within 1e-4 of the fp64 oracle.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import memory as om

pytestmark = pytest.mark.gpu


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _mem(N, dm, de, p):
    from paper_conf_asplos_wangm24_b200 import tgl
    return tgl.TGNMemory(N, dm, de, p)


def _params(de, dm=100, name="REDDIT"):
    from dataclasses import replace
    return synth.make_gru_params(replace(synth.get_config(name), d_e=de), d_mem=dm)


@pytest.mark.parametrize("B,N,de,tmax", [(600, 1000, 172, 10**6), (600, 40, 172, 5),
                                         (1, 10, 0, 10), (2000, 300000, 186, 100),
                                         (777, 64, 16, 1)])
def test_mailbox_store_exact(B, N, de, tmax):
    rng = np.random.default_rng(B + N)
    dm = 100
    M = _mem(N, dm, de, _params(de, dm))
    mem = rng.uniform(-1, 1, (N, dm)).astype(np.float32)
    M.mem.copy_(cu(mem))
    src = rng.integers(0, N, B).astype(np.int32)
    dst = rng.integers(0, N, B).astype(np.int32)
    t = np.sort(rng.integers(0, tmax, B)).astype(np.float32)     # ties when tmax is small
    E = 5000
    ef = rng.uniform(-1, 1, (E, max(de, 1))).astype(np.float32)[:, :de]
    eid = rng.integers(0, E, B).astype(np.int32)
    uniq, pick, nu = M.store(cu(src), cu(dst), cu(t), cu(ef) if de else None, cu(eid))
    torch.cuda.synchronize()
    mail = np.zeros((N, 2 * dm + de), np.float64)
    mail_ts = np.zeros(N, np.float32)
    eu, ep = om.mailbox_store(mail, mail_ts, mem, src, dst, t, eid, ef if de else None)
    n = int(nu.item())
    assert n == len(eu)
    assert uniq[:n].cpu().numpy().tolist() == eu.tolist()
    assert pick[:n].cpu().numpy().tolist() == ep.tolist()
    assert np.array_equal(M.mail.cpu().numpy(), mail.astype(np.float32))
    assert np.array_equal(M.mail_ts.cpu().numpy().view(np.uint32), mail_ts.view(np.uint32))


def test_mailbox_store_device_count_and_eid0():
    """B on the device (capacity larger), edge ids eid0 + j (consecutive edge rows), and
    an empty batch (B = 0) that stores nothing."""
    rng = np.random.default_rng(7)
    N, dm, de, B, Bcap = 500, 32, 8, 300, 512
    M = _mem(N, dm, de, _params(de, dm))
    mem = rng.uniform(-1, 1, (N, dm)).astype(np.float32)
    M.mem.copy_(cu(mem))
    src = rng.integers(0, N, Bcap).astype(np.int32)
    dst = rng.integers(0, N, Bcap).astype(np.int32)
    t = np.sort(rng.integers(0, 50, Bcap)).astype(np.float32)
    ef = rng.uniform(-1, 1, (2000, de)).astype(np.float32)
    for Bn in (0, B):
        M.mail.zero_()
        M.mail_ts.zero_()
        bd = torch.tensor([Bn], dtype=torch.int64, device="cuda")
        uniq, pick, nu = M.store(cu(src), cu(dst), cu(t), cu(ef), None, eid0=1000, B_dev=bd)
        torch.cuda.synchronize()
        mail = np.zeros((N, 2 * dm + de))
        mail_ts = np.zeros(N, np.float32)
        eu, ep = om.mailbox_store(mail, mail_ts, mem, src[:Bn], dst[:Bn], t[:Bn],
                                  1000 + np.arange(Bn), ef)
        n = int(nu.item())
        assert n == len(eu)
        assert uniq[:n].cpu().numpy().tolist() == eu.tolist()
        assert pick[:n].cpu().numpy().tolist() == ep.tolist()
        assert np.array_equal(M.mail.cpu().numpy(), mail.astype(np.float32))


@pytest.mark.parametrize("n,N,dm,de", [(1, 10, 100, 172), (1300, 5000, 100, 172),
                                       (257, 1000, 100, 0), (500, 600, 64, 186)])
def test_memory_update_vs_oracle(n, N, dm, de):
    rng = np.random.default_rng(n + N)
    p = _params(de, dm)
    M = _mem(N, dm, de, p)
    mem = rng.uniform(-1, 1, (N, dm)).astype(np.float32)
    mem_ts = rng.integers(0, 10**6, N).astype(np.float32)
    mail = rng.uniform(-1, 1, (N, 2 * dm + de)).astype(np.float32)
    mail_ts = (mem_ts + rng.integers(0, 10**6, N)).astype(np.float32)
    for a, b in ((M.mem, mem), (M.mem_ts, mem_ts), (M.mail, mail), (M.mail_ts, mail_ts)):
        a.copy_(cu(b))
    nodes = rng.choice(N, n, replace=False).astype(np.int32)
    M.update(cu(nodes))
    torch.cuda.synchronize()
    exp_mem, exp_ts = mem.astype(np.float64), mem_ts.copy()
    om.memory_update(exp_mem, exp_ts, mail, mail_ts, nodes, p)
    got = M.mem.cpu().numpy()
    err = np.abs(got - exp_mem).max()
    assert err <= 1e-5 * (1 + np.abs(exp_mem).max()), err
    assert np.array_equal(M.mem_ts.cpu().numpy(), exp_ts)
    keep = np.setdiff1d(np.arange(N), nodes)
    assert np.array_equal(got[keep], mem[keep])


def test_memory_update_device_count():
    rng = np.random.default_rng(11)
    N, dm, de = 800, 100, 172
    p = _params(de, dm)
    M = _mem(N, dm, de, p)
    mail = rng.uniform(-1, 1, (N, 2 * dm + de)).astype(np.float32)
    mail_ts = rng.integers(1, 1000, N).astype(np.float32)
    M.mail.copy_(cu(mail))
    M.mail_ts.copy_(cu(mail_ts))
    nodes = rng.choice(N, 400, replace=False).astype(np.int32)
    M.update(cu(nodes), n_dev=torch.tensor([123], dtype=torch.int64, device="cuda"))
    torch.cuda.synchronize()
    exp_mem, exp_ts = np.zeros((N, dm)), np.zeros(N, np.float32)
    om.memory_update(exp_mem, exp_ts, mail, mail_ts, nodes[:123], p)
    assert np.abs(M.mem.cpu().numpy() - exp_mem).max() <= 1e-5
    assert np.array_equal(M.mem_ts.cpu().numpy(), exp_ts)


@pytest.mark.parametrize("name", ["WIKI", "REDDIT"])
def test_tgn_loop_vs_oracle(name):
    """Listing 4's per-batch order: update the batch's (distinct) nodes from their
    mailboxes, then store the batch's coalesced messages -- 6 consecutive batches."""
    cfg = synth.get_config(name).scaled(20000, batch=600)
    g = synth.make_graph(cfg)
    dm, de = 100, cfg.d_e
    p = synth.make_gru_params(cfg, d_mem=dm)
    M = _mem(cfg.n_nodes, dm, de, p)
    ef = cu(g.efeat)
    mem, mem_ts = np.zeros((cfg.n_nodes, dm)), np.zeros(cfg.n_nodes, np.float32)
    mail, mail_ts = np.zeros((cfg.n_nodes, 2 * dm + de)), np.zeros(cfg.n_nodes, np.float32)
    for b in range(6):
        s = slice(b * cfg.batch, (b + 1) * cfg.batch)
        src, dst, t = g.src[s], g.dst[s], g.t[s]
        nodes = np.unique(np.concatenate([src, dst])).astype(np.int32)
        M.update(cu(nodes))
        M.store(cu(src), cu(dst), cu(t), ef, None, eid0=s.start)
        om.memory_update(mem, mem_ts, mail, mail_ts, nodes, p)
        om.mailbox_store(mail, mail_ts, mem.astype(np.float32), src, dst, t,
                         np.arange(s.start, s.stop), g.efeat)
    torch.cuda.synchronize()
    assert np.abs(M.mem.cpu().numpy() - mem).max() <= 1e-4
    assert np.abs(M.mail.cpu().numpy() - mail).max() <= 1e-4
    assert np.array_equal(M.mem_ts.cpu().numpy(), mem_ts)
    assert np.array_equal(M.mail_ts.cpu().numpy(), mail_ts)
