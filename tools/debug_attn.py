"""Debug helper: compare the q / r scratch rows of tgl_tblock_attn with numpy."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import oracle
import synth
from paper_conf_asplos_wangm24_b200 import tgl
from tests.test_gpu_parity import attn_case, cu


def main(prec="fp32", n_dst=40, pack=False):
    rng = np.random.default_rng(1)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, n_dst, 10, 172, 172)
    P = tgl.AttnParams(p, precision=prec, pack=pack)
    ws = tgl.Workspace()
    out = tgl.tblock_attn(P, cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn), cu(ef),
                          cu(eid), cu(et), max_seg=10, ws=ws)
    torch.cuda.synchronize()
    buf = ws.buf.view(torch.float32).cpu().numpy()
    n = n_dst
    q = buf[:n * 128].reshape(n, 128)[:, :100]
    nrows = max(n, 1)
    roff = ((128 * 4 * nrows + 255) // 256) * 256 // 4
    r = buf[roff:roff + n * 128].reshape(n, 128)[:, :100]
    phi0 = np.cos(p["phi"].astype(np.float64))
    zq = np.concatenate([nfeat[dn].astype(np.float64), np.tile(phi0, (n, 1))], 1)
    q_exp = zq @ p["Wq"].astype(np.float64).T + p["bq"]
    print("q err", np.abs(q - q_exp).max(), "q sample", q[0, :4], q_exp[0, :4])
    exp = oracle.tblock_attn(p, seg, dst_t, nfeat, dn, nfeat, sn, ef, eid, et)
    print("out err", np.abs(out.cpu().numpy()[:n] - exp).max())
    # r via the oracle pieces: run with Wo = [I | 0], bo = 0, LN off is not possible; print r stats
    print("r sample", r[0, :6], "r finite", np.isfinite(r).all())




def ffn_check(prec="fp32"):
    rng = np.random.default_rng(1)
    n = 40
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, n, 10, 172, 172)
    P = tgl.AttnParams(p, precision=prec)
    ws = tgl.Workspace()
    out = tgl.tblock_attn(P, cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn), cu(ef),
                          cu(eid), cu(et), max_seg=10, ws=ws).cpu().numpy()[:n]
    buf = ws.buf.view(torch.float32).cpu().numpy()
    roff = ((128 * 4 * n + 255) // 256) * 256 // 4
    r = buf[roff:roff + n * 128].reshape(n, 128)[:, :100].astype(np.float64)
    z = np.concatenate([r, nfeat[dn].astype(np.float64)], 1)
    o = np.maximum(z @ p["Wo"].astype(np.float64).T + p["bo"], 0)
    pre = o.copy()
    o = (o - o.mean(1, keepdims=True)) / np.sqrt(o.var(1, keepdims=True) + 1e-5)
    o = o * p["ln_gamma"] + p["ln_beta"]
    print("ffn err given gpu r:", np.abs(out - o).max())
    print("row0 gpu", out[0, :5], "exp", o[0, :5])
    print("row1 gpu", out[1, :5], "exp", o[1, :5])
    print("pre-LN row0", pre[0, :5])


def r_compare(n=40):
    rng = np.random.default_rng(1)
    p, seg, dst_t, nfeat, dn, sn, ef, eid, et = attn_case(rng, n, 10, 172, 172)
    rs = {}
    for prec in ("fp32", "fp32_simt"):
        P = tgl.AttnParams(p, precision=prec)
        ws = tgl.Workspace()
        tgl.tblock_attn(P, cu(seg), cu(dst_t), cu(nfeat), cu(dn), cu(nfeat), cu(sn), cu(ef),
                        cu(eid), cu(et), max_seg=10, ws=ws)
        buf = ws.buf.view(torch.float32).cpu().numpy()
        roff = ((128 * 4 * n + 255) // 256) * 256 // 4
        rs[prec] = buf[roff:roff + n * 128].reshape(n, 128)[:, :100]
    d = np.abs(rs["fp32"] - rs["fp32_simt"]).max(1)
    print("per-dst r err:", np.round(d, 4).tolist())
    print("seg lens:", np.diff(seg).tolist())


if __name__ == "__main__":
    main(*(sys.argv[1:2] or ["fp32"]))
    ffn_check(*(sys.argv[1:2] or ["fp32"]))
    r_compare()
