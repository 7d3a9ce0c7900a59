"""Backward pass of one TBlock attention layer -- TEST INFRASTRUCTURE ONLY.

The forward is the layer of eqs 4-7 (Listing 2 TemporalAttnLayer.forward,
P:245-256) exactly as oracle.c computes it (readings R10-R13, R19); training
(the paper's headline; Fig 7 times the backward) needs its gradients.
Everything here is fp64 numpy, one destination at a time, in the forward's order:

  zq = [h_i ; Phi(0)]            q = Wq zq + bq                         (eq 4)
  z_e = [h_src(e) ; e_e ; Phi(dt_e)]   k_e, v_e = W{k,v} z_e + b{k,v}  (eq 5)
  u_e^h = scale <q^h, k_e^h>,  s = LeakyReLU(u)  alpha = softmax_e(s)    (L2.33-34, R12)
  r = sum_e alpha_e v_e  (r = 0 for an empty segment, R19)              (L2.36)
  y = Wo [r ; h_i] + bo,  a = ReLU(y),  out = (a - mean) / sqrt(var + eps) * g + b (eq 7, R13)

and the backward applies the chain rule step by step in reverse order (LayerNorm,
ReLU, output projection, weighted sum, segmented softmax, LeakyReLU, the K/V and Q
projections, the time encoder Phi_j(dt) = cos(omega_j dt + phi_j) with
dPhi/domega = -sin(.) dt, dPhi/dphi = -sin(.)).  The time encoder's argument is the
R10 fp32 value b = fl(fl(omega*dt) + phi) in the forward (as oracle.c); its derivative
treats those roundings as exact (the derivative of the real function), which is what
`exact_phi=True` evaluates -- the finite-difference pins use that variant.

Pins (tests/test_backward_cpu.py): the forward equals oracle.tblock_attn (the C
oracle) on the same inputs; every gradient equals central finite differences of the
exact forward; closed forms (dL/dbeta = sum g, an empty segment leaves Wk / Wv / omega
gradients at zero, ...).
"""
from __future__ import annotations

import numpy as np


def _phi(dt, omega, phi, exact: bool):
    """Phi(dt) and its argument b: R10 (fp32 product, fp32 sum, cosine rounded to fp32, as
    oracle.c) or exact fp64 (exact=True, for finite differences)."""
    if exact:
        b = np.asarray(omega, np.float64) * float(dt) + np.asarray(phi, np.float64)
    else:
        a = (np.float32(dt) * np.asarray(omega, np.float32)).astype(np.float32)
        b = (a + np.asarray(phi, np.float32)).astype(np.float32).astype(np.float64)
        return np.cos(b).astype(np.float32).astype(np.float64), b   # Phi rounded to fp32
    return np.cos(b), b


def tblock_forward(p: dict, seg_ptr, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid,
                   edge_t, exact_phi: bool = False):
    """Returns (out fp64 [n_dst, d_out], tape) -- tape = per-destination intermediates."""
    f64 = lambda a: np.asarray(a, dtype=np.float64)
    Wq, bq, Wk, bk = f64(p["Wq"]), f64(p["bq"]), f64(p["Wk"]), f64(p["bk"])
    Wv, bv, Wo, bo = f64(p["Wv"]), f64(p["bv"]), f64(p["Wo"]), f64(p["bo"])
    gam, bet = f64(p["ln_gamma"]), f64(p["ln_beta"])
    om, ph = np.asarray(p["omega"]), np.asarray(p["phi"])      # (cast per mode in _phi)
    dm, H = p["d_model"], p["n_heads"]
    eps = float(np.float32(p["ln_eps"]))      # an fp32 field of tgl_attn_params, as oracle.c
    dh = dm // H
    slope, scale = float(p["leaky_slope"]), float(p["logit_scale"])
    seg_ptr = np.asarray(seg_ptr, np.int64)
    n = seg_ptr.shape[0] - 1
    out = np.zeros((n, p["d_out"]))
    tape = []
    for i in range(n):
        row = int(hdst_idx[i]) if hdst_idx is not None else i
        h = f64(hdst[row])
        ph0, b0 = _phi(0.0, om, ph, exact_phi)
        zq = np.concatenate([h, ph0])
        q = Wq @ zq + bq
        e0, e1 = int(seg_ptr[i]), int(seg_ptr[i + 1])
        Z, B, DT, rows = [], [], [], []
        for e in range(e0, e1):
            hs = f64(hsrc[int(hsrc_idx[e])])
            ef = f64(efeat[int(eid[e])]) if p["d_e"] > 0 else np.zeros(0)
            dt = np.float32(np.float32(dst_t[i]) - np.float32(edge_t[e]))   # R18
            phe, b = _phi(dt, om, ph, exact_phi)
            Z.append(np.concatenate([hs, ef, phe]))
            B.append(b)
            DT.append(float(dt))
            rows.append(int(hsrc_idx[e]))
        m = e1 - e0
        r = np.zeros(dm)
        if m:
            Z = np.stack(Z)
            K = Z @ Wk.T + bk
            V = Z @ Wv.T + bv
            U = np.stack([scale * (K[:, hh * dh:(hh + 1) * dh] @ q[hh * dh:(hh + 1) * dh])
                          for hh in range(H)], 1)                       # [m, H]
            S = np.where(U < 0, U * slope, U) if slope >= 0 else U.copy()
            A = np.exp(S - S.max(0))
            A /= A.sum(0)
            for hh in range(H):
                r[hh * dh:(hh + 1) * dh] = A[:, hh] @ V[:, hh * dh:(hh + 1) * dh]
        else:
            K = V = U = A = None
        zo = np.concatenate([r, h])
        y = Wo @ zo + bo
        a = np.maximum(y, 0.0)
        mu = a.mean()
        var = ((a - mu) ** 2).mean()
        sig = np.sqrt(var + eps)
        xh = (a - mu) / sig
        out[i] = xh * gam + bet
        tape.append(dict(row=row, zq=zq, q=q, b0=b0, m=m, Z=Z, B=B, DT=DT, rows=rows, K=K, V=V,
                         U=U, A=A, zo=zo, y=y, xh=xh, sig=sig))
    return out, tape


def tblock_backward(p: dict, tape: list, g_out, n_hdst_rows: int, n_hsrc_rows: int) -> dict:
    """Gradients of L = sum(out * g_out) for the layer's parameters and input rows
    (grad_hdst [n_hdst_rows, d_hdst], grad_hsrc [n_hsrc_rows, d_hsrc]); fp64."""
    f64 = lambda a: np.asarray(a, dtype=np.float64)
    Wq, Wk, Wv, Wo = f64(p["Wq"]), f64(p["Wk"]), f64(p["Wv"]), f64(p["Wo"])
    gam = f64(p["ln_gamma"])
    dm, H = p["d_model"], p["n_heads"]
    dh = dm // H
    slope, scale = float(p["leaky_slope"]), float(p["logit_scale"])
    dhd, dhs, de, dt_ = p["d_hdst"], p["d_hsrc"], p["d_e"], p["d_t"]
    G = {k: np.zeros(np.shape(p[k])) for k in ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo",
                                               "ln_gamma", "ln_beta", "omega", "phi")}
    g_hdst = np.zeros((n_hdst_rows, dhd))
    g_hsrc = np.zeros((n_hsrc_rows, dhs))
    g_out = f64(g_out)
    for i, T in enumerate(tape):
        g = g_out[i]
        # LayerNorm (biased variance, eps inside the root) and ReLU
        G["ln_gamma"] += g * T["xh"]
        G["ln_beta"] += g
        gx = g * gam
        xh, sig = T["xh"], T["sig"]
        ga = (gx - gx.mean() - xh * (gx * xh).mean()) / sig
        gy = ga * (T["y"] > 0)
        # output projection y = Wo [r ; h] + bo
        G["Wo"] += np.outer(gy, T["zo"])
        G["bo"] += gy
        gzo = Wo.T @ gy
        gr, gh = gzo[:dm], gzo[dm:].copy()
        gq = np.zeros(dm)
        if T["m"]:
            A, V, K, U, Z = T["A"], T["V"], T["K"], T["U"], T["Z"]
            gV = np.zeros_like(V)
            gK = np.zeros_like(K)
            for hh in range(H):
                cs = slice(hh * dh, (hh + 1) * dh)
                gV[:, cs] = np.outer(A[:, hh], gr[cs])            # r = sum_e alpha v
                galpha = V[:, cs] @ gr[cs]
                gs = A[:, hh] * (galpha - (A[:, hh] * galpha).sum())   # softmax
                gu = gs * np.where(U[:, hh] < 0, slope, 1.0) if slope >= 0 else gs
                gq[cs] += scale * (gu @ K[:, cs])
                gK[:, cs] = scale * np.outer(gu, T["q"][cs])
            G["Wk"] += gK.T @ Z
            G["bk"] += gK.sum(0)
            G["Wv"] += gV.T @ Z
            G["bv"] += gV.sum(0)
            gZ = gK @ Wk + gV @ Wv                                  # [m, d_hs + d_e + d_t]
            for j, rw in enumerate(T["rows"]):
                g_hsrc[rw] += gZ[j, :dhs]
                gphi = gZ[j, dhs + de:]
                sn = -np.sin(T["B"][j])
                G["omega"] += gphi * sn * T["DT"][j]
                G["phi"] += gphi * sn
        # query projection q = Wq [h ; Phi(0)] + bq
        G["Wq"] += np.outer(gq, T["zq"])
        G["bq"] += gq
        gzq = Wq.T @ gq
        gh += gzq[:dhd]
        G["phi"] += gzq[dhd:] * -np.sin(T["b0"])                  # Phi(0) = cos(phi)
        g_hdst[T["row"]] += gh
    G["hdst"] = g_hdst
    G["hsrc"] = g_hsrc
    return G
