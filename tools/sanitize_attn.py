"""Tiny TBlock attention calls for compute-sanitizer (racecheck / synccheck / memcheck):
the product K|V kernels (kv_pre on split16 tables, kv_split on fp32 rows) plus the Q / FFN
dense kernels, one small launch each, fp32 and bf16.

    compute-sanitizer --tool racecheck python tools/sanitize_attn.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from dataclasses import replace
from paper_conf_asplos_wangm24_b200 import tgl

rng = np.random.default_rng(3)
cfg = replace(synth.get_config("REDDIT"), d_e=172)
p = synth.make_layer_params(cfg, 0, 172, 172, random_ln=True, random_phi=True)
n_dst = 300
lens = rng.integers(0, 11, n_dst)
seg = np.zeros(n_dst + 1, np.int64)
seg[1:] = np.cumsum(lens)
E = int(seg[-1])
cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
nfeat = cu(rng.uniform(-1, 1, (500, 172)).astype(np.float32))
efeat = cu(rng.uniform(-1, 1, (2000, 172)).astype(np.float32))
dn = cu(rng.integers(0, 500, n_dst).astype(np.int32))
sn = cu(rng.integers(0, 500, E).astype(np.int32))
eid = cu(rng.integers(0, 2000, E).astype(np.int32))
dst_t = rng.integers(10**5, 2 * 10**6, n_dst).astype(np.float32)
et = cu((np.repeat(dst_t, lens) - rng.integers(1, 200000, E)).astype(np.float32))
outs = {}
for prec in ("fp32", "bf16"):
    for kv in ("pre", "split"):
        P = tgl.AttnParams(p, precision=prec, pack=True, kv_kernel=kv)
        hs, ef = nfeat, efeat
        if kv == "pre":
            hs, ef = tgl.split_rows(nfeat), tgl.split_rows(efeat)
            P.struct.input_layout = tgl.SPLIT_HSRC | tgl.SPLIT_E
        o = tgl.tblock_attn(P, cu(seg), cu(dst_t), nfeat, dn, hs, sn, ef, eid, et, max_seg=10)
        torch.cuda.synchronize()
        outs[(prec, kv)] = o[:n_dst].cpu().numpy()
    # node projections (tgl_node_proj + TGL_NODE_PROJ): Z rows initialise the accumulator
    P = tgl.AttnParams(p, precision=prec, pack=True)
    Z = tgl.node_proj(P, tgl.split_rows(nfeat))
    P.struct.input_layout = tgl.SPLIT_HSRC | tgl.SPLIT_E | tgl.NODE_PROJ
    P.struct.node_proj = tgl._p(Z)
    o = tgl.tblock_attn(P, cu(seg), cu(dst_t), nfeat, dn, nfeat, sn, tgl.split_rows(efeat), eid,
                        et, max_seg=10)
    torch.cuda.synchronize()
    outs[(prec, "np")] = o[:n_dst].cpu().numpy()
for prec in ("fp32", "bf16"):
    d = np.abs(outs[(prec, "pre")] - outs[(prec, "split")]).max()
    dn_ = np.abs(outs[(prec, "pre")] - outs[(prec, "np")]).max()
    print(f"{prec}: |pre - split| = {d:.2e}  |pre - node_proj| = {dn_:.2e}")
print("sanitize_attn done")
