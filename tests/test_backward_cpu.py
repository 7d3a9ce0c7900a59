"""Pins of the TBlock backward oracle (oracle/backward.py), CPU only.

* its forward equals the C oracle's tblock_attn (oracle.c, eqs 4-7) on the same inputs;
* every gradient -- all 12 parameter tensors and both input row tables -- equals central
  finite differences of the (exact-Phi) forward, L = sum(out * G) for a random G;
* closed forms: dL/dbeta = sum_i G_i, dL/dgamma = sum_i G_i * xhat_i; with no edges at
  all the K / V / omega gradients vanish and h_src gets nothing.
"""
import numpy as np
import pytest

import oracle
from oracle import backward as ob


def _case(seed=0, lens=(0, 1, 3, 2, 4, 1), d_hd=6, d_hs=5, d_e=3, d_t=4, dm=4, slope=0.2):
    rng = np.random.default_rng(seed)
    u = lambda *s: rng.uniform(-1, 1, s)
    p = dict(d_hdst=d_hd, d_hsrc=d_hs, d_e=d_e, d_t=d_t, d_model=dm, n_heads=2, d_out=dm,
             Wq=u(dm, d_hd + d_t) * 0.7, bq=u(dm) * 0.3, Wk=u(dm, d_hs + d_e + d_t) * 0.7,
             bk=u(dm) * 0.3, Wv=u(dm, d_hs + d_e + d_t) * 0.7, bv=u(dm) * 0.3,
             Wo=u(dm, dm + d_hd) * 0.7, bo=u(dm) * 0.3, ln_gamma=1 + 0.5 * u(dm),
             ln_beta=0.5 * u(dm), ln_eps=1e-5, omega=np.abs(u(d_t)) + 0.1, phi=u(d_t) * 3,
             leaky_slope=slope, logit_scale=1.0)
    lens = np.asarray(lens)
    seg = np.zeros(len(lens) + 1, np.int64)
    seg[1:] = np.cumsum(lens)
    E = int(seg[-1])
    hdst = u(9, d_hd)
    hsrc = u(11, d_hs)
    efeat = u(7, d_e)
    hdst_idx = rng.integers(0, 9, len(lens)).astype(np.int32)
    hsrc_idx = rng.integers(0, 11, E).astype(np.int32)
    eid = rng.integers(0, 7, E).astype(np.int32)
    dst_t = rng.integers(50, 100, len(lens)).astype(np.float32)
    edge_t = (np.repeat(dst_t, lens) - rng.integers(1, 40, E)).astype(np.float32)
    return p, seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid, edge_t


def _loss(p, args, G):
    seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid, edge_t = args
    out, _ = ob.tblock_forward(p, seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid,
                               edge_t, exact_phi=True)
    return float((out * G).sum())


def test_forward_equals_c_oracle():
    p, *args = _case(1)
    p32 = {k: (np.asarray(v, np.float32) if isinstance(v, np.ndarray) else v) for k, v in p.items()}
    seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid, edge_t = args
    f = lambda a: np.asarray(a, np.float32)
    got, _ = ob.tblock_forward(p32, seg, dst_t, f(hdst), hdst_idx, f(hsrc), hsrc_idx, f(efeat),
                               eid, edge_t)
    exp = oracle.tblock_attn(p32, seg, dst_t, f(hdst), hdst_idx, f(hsrc), hsrc_idx, f(efeat),
                             eid, edge_t)
    np.testing.assert_allclose(got, exp, rtol=0, atol=1e-8)   # fp64 summation order only


@pytest.mark.parametrize("slope", [0.2, -1.0])
def test_gradients_equal_finite_differences(slope):
    p, *args = _case(2, slope=slope)
    seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid, edge_t = args
    rng = np.random.default_rng(7)
    G = rng.standard_normal((len(seg) - 1, p["d_out"]))
    _, tape = ob.tblock_forward(p, *args, exact_phi=True)
    an = ob.tblock_backward(p, tape, G, hdst.shape[0], hsrc.shape[0])
    h = 1e-5
    for name in ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo", "ln_gamma", "ln_beta",
                 "omega", "phi"):
        base = np.array(p[name], np.float64)
        for flat in rng.choice(base.size, min(base.size, 8), replace=False):
            idx = np.unravel_index(flat, base.shape)
            pp, pm = dict(p), dict(p)
            bp, bm = base.copy(), base.copy()
            bp[idx] += h
            bm[idx] -= h
            pp[name], pm[name] = bp, bm
            fd = (_loss(pp, args, G) - _loss(pm, args, G)) / (2 * h)
            assert abs(fd - an[name][idx]) <= 1e-6 * max(1.0, abs(fd)), (name, idx, fd,
                                                                         an[name][idx])
    for tab, key, pos in ((hdst, "hdst", 2), (hsrc, "hsrc", 4)):
        for r in range(tab.shape[0]):
            for c in range(tab.shape[1]):
                tp, tm = tab.copy(), tab.copy()
                tp[r, c] += h
                tm[r, c] -= h
                ap, am = list(args), list(args)
                ap[pos], am[pos] = tp, tm
                fd = (_loss(p, ap, G) - _loss(p, am, G)) / (2 * h)
                assert abs(fd - an[key][r, c]) <= 1e-6 * max(1.0, abs(fd)), (key, r, c)


def test_closed_forms_and_empty_segments():
    p, *args = _case(3, lens=(0, 0, 0))
    seg, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid, edge_t = args
    G = np.random.default_rng(1).standard_normal((3, p["d_out"]))
    out, tape = ob.tblock_forward(p, *args)
    an = ob.tblock_backward(p, tape, G, hdst.shape[0], hsrc.shape[0])
    np.testing.assert_allclose(an["ln_beta"], G.sum(0), atol=1e-12)
    xh = np.stack([T["xh"] for T in tape])
    np.testing.assert_allclose(an["ln_gamma"], (G * xh).sum(0), atol=1e-12)
    for k in ("Wk", "bk", "Wv", "bv", "omega"):
        assert not an[k].any(), k                    # no edges: K / V / Phi(dt) unused
    assert not an["hsrc"].any()
    # r = 0 for empty segments: the first d_model columns of dWo see zeros
    assert not an["Wo"][:, :p["d_model"]].any()
