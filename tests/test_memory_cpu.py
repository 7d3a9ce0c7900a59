"""N3 oracle pins (oracle/memory.py): the TGN memory path of PAPER.md eqs 9-11 / Listings 3-4.

Each pin is independent of the oracle's own code path:
  * coalesce(by='latest') against a lexsort over (node, t, position) and a hand fixture
    with ties (R26);
  * the messages of a two-edge batch written out by hand (eq 9, Listing 3 L16-17);
  * the GRU cell against torch.nn.GRUCell in fp64 (the library routine eq 11 names);
  * closed forms of eq 11: zero weights give s' = s / 2; a saturated update gate keeps
    s; the time-encoder input equals the C oracle's tgl_time_encode (pinned in
    test_oracle_pins.py) of dt = mail_ts - mem_ts;
  * the store/update sequence keeps mem_ts = mail_ts of the updated nodes and the
    mailbox time = the node's latest batch time.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import memory as om


def test_coalesce_fixture_ties():
    # node 3 at t=5 twice (positions 0, 2) -> the later one; node 1: t=5 then t=6 -> 4
    uniq, pick = om.coalesce_latest([3, 1, 3, 2, 1], np.float32([5, 5, 5, 4, 6]))
    assert uniq.tolist() == [3, 1, 2] and pick.tolist() == [2, 4, 3]
    # an earlier time later in the order does not replace a later time
    uniq, pick = om.coalesce_latest([7, 7, 7], np.float32([9, 3, 9]))
    assert uniq.tolist() == [7] and pick.tolist() == [2]
    uniq, pick = om.coalesce_latest([], np.float32([]))
    assert uniq.size == 0 and pick.size == 0


@pytest.mark.parametrize("seed,n_nodes", [(0, 5), (1, 40), (2, 1000)])
def test_coalesce_vs_lexsort(seed, n_nodes):
    rng = np.random.default_rng(seed)
    n = 700
    nodes = rng.integers(0, n_nodes, n)
    times = rng.integers(0, 30, n).astype(np.float32)           # many equal times
    uniq, pick = om.coalesce_latest(nodes, times)
    pos = np.arange(n)
    order = np.lexsort((pos, times, nodes))                   # by node, then t, then position
    last = order[np.r_[nodes[order][1:] != nodes[order][:-1], True]]
    exp_pick = dict(zip(nodes[last].tolist(), last.tolist()))
    _, first = np.unique(nodes, return_index=True)
    exp_uniq = nodes[np.sort(first)]
    assert uniq.tolist() == exp_uniq.tolist()
    assert pick.tolist() == [exp_pick[v] for v in exp_uniq.tolist()]


def test_messages_by_hand():
    mem = np.array([[1., 2.], [3., 4.], [5., 6.]])
    ef = np.array([[10.], [20.], [30.]])
    msgs = om.messages(mem, np.array([0, 2]), np.array([1, 0]), np.array([2, 1]), ef)
    assert msgs.tolist() == [[1, 2, 3, 4, 30], [5, 6, 1, 2, 20],      # sources
                             [3, 4, 1, 2, 30], [1, 2, 5, 6, 20]]      # destinations


def test_gru_matches_torch_grucell():
    rng = np.random.default_rng(3)
    d, dx = 7, 11
    cell = torch.nn.GRUCell(dx, d).double()
    x, h = rng.standard_normal(dx), rng.standard_normal(d)
    exp = cell(torch.from_numpy(x)[None], torch.from_numpy(h)[None])[0].detach().numpy()
    got = om.gru_cell(x, h, cell.weight_ih.detach().numpy(), cell.weight_hh.detach().numpy(),
                      cell.bias_ih.detach().numpy(), cell.bias_hh.detach().numpy())
    assert np.abs(got - exp).max() < 1e-14


def _state(rng, N, dm, de):
    mem = rng.uniform(-1, 1, (N, dm))
    mem_ts = rng.integers(0, 1000, N).astype(np.float32)
    mail = rng.uniform(-1, 1, (N, 2 * dm + de))
    mail_ts = (mem_ts + rng.integers(0, 1000, N)).astype(np.float32)
    return mem, mem_ts, mail, mail_ts


def test_update_closed_forms():
    rng = np.random.default_rng(5)
    N, dm, de, dt_ = 20, 4, 3, 5
    mem, mem_ts, mail, mail_ts = _state(rng, N, dm, de)
    dx = 2 * dm + de + dt_
    z = lambda *s: np.zeros(s)
    p = dict(W_ih=z(3 * dm, dx), W_hh=z(3 * dm, dm), b_ih=z(3 * dm), b_hh=z(3 * dm),
             omega=np.ones(dt_, np.float32), phi=np.zeros(dt_, np.float32))
    m0 = mem.copy()
    nodes = np.array([3, 7, 11])
    om.memory_update(mem, mem_ts, mail, mail_ts, nodes, p)       # r = z = 1/2, n = 0
    assert np.allclose(mem[nodes], 0.5 * m0[nodes], atol=1e-15)
    assert (mem_ts[nodes] == mail_ts[nodes]).all()
    keep = np.setdiff1d(np.arange(N), nodes)
    assert (mem[keep] == m0[keep]).all()
    p["b_ih"][dm:2 * dm] = 60.0                                  # update gate saturated: s' = s
    m1 = mem.copy()
    om.memory_update(mem, mem_ts, mail, mail_ts, np.array([0, 1]), p)
    assert np.allclose(mem[[0, 1]], m1[[0, 1]], atol=1e-12)


def test_update_time_input_is_time_encode():
    """x's Phi part equals the C oracle's time encoder of dt (pinned elsewhere): checked
    through a GRU whose only non-zero weight reads one Phi column into the n gate."""
    import oracle
    rng = np.random.default_rng(6)
    N, dm, de, dt_ = 6, 3, 2, 4
    mem, mem_ts, mail, mail_ts = _state(rng, N, dm, de)
    mem[:] = 0.0
    dx = 2 * dm + de + dt_
    omega = np.float32([1.0, 0.1, 0.01, 0.001])
    phi = np.float32([0.3, -1.0, 2.0, 0.0])
    for j in range(dt_):
        W_ih = np.zeros((3 * dm, dx))
        W_ih[2 * dm, 2 * dm + de + j] = 1.0                      # n_0 = tanh(Phi_j)
        p = dict(W_ih=W_ih, W_hh=np.zeros((3 * dm, dm)), b_ih=np.zeros(3 * dm),
                 b_hh=np.zeros(3 * dm), omega=omega, phi=phi)
        mm, mt = mem.copy(), mem_ts.copy()
        out = om.memory_update(mm, mt, mail, mail_ts, np.arange(N), p)
        dt = (mail_ts - mem_ts).astype(np.float32)
        enc = oracle.time_encode(dt, omega, phi)[:, j]
        assert np.allclose(out[:, 0], 0.5 * np.tanh(enc), atol=1e-12)   # (1 - 1/2) n


def test_store_then_update_sequence():
    cfg = synth.get_config("WIKI").scaled(3000, batch=200)
    g = synth.make_graph(cfg)
    p = synth.make_gru_params(cfg, d_mem=16)
    N, dm, de = cfg.n_nodes, 16, cfg.d_e
    mem, mem_ts = np.zeros((N, dm)), np.zeros(N, np.float32)
    mail, mail_ts = np.zeros((N, 2 * dm + de)), np.zeros(N, np.float32)
    for b in range(3):
        s = slice(b * cfg.batch, (b + 1) * cfg.batch)
        src, dst, t = g.src[s], g.dst[s], g.t[s]
        nodes = np.unique(np.concatenate([src, dst]))
        om.memory_update(mem, mem_ts, mail, mail_ts, nodes, p)
        assert (mem_ts[nodes] == mail_ts[nodes]).all()
        uniq, _ = om.mailbox_store(mail, mail_ts, mem, src, dst, t, np.arange(s.start, s.stop),
                                   g.efeat)
        assert sorted(uniq.tolist()) == nodes.tolist()
        for v in nodes[:50]:
            assert mail_ts[v] == t[(src == v) | (dst == v)].max()
    assert np.abs(mem).max() > 0 and np.isfinite(mem).all()
