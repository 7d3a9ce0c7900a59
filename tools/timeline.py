"""Per-tile role timeline of the tail kv_bin kernel (TGL_DEBUG_MASK=32)."""
import ctypes as C
import os
import sys

os.environ["TGL_DEBUG_MASK"] = str(32 | int(os.environ.get("EXTRA_MASK", "0")))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl

cfg = synth.get_config("REDDIT")
g = synth.make_graph(cfg)
neg = synth.make_negatives(cfg)
params = synth.gen.model_params(cfg)
cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg), "nfeat": cu(g.nfeat),
       "efeat": cu(g.efeat)}
tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
pipe = TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]),
                    cfg.dedup, cfg.precompute, cfg.window, sys.argv[1] if len(sys.argv) > 1 else "fp32")
b0 = int(0.7 * cfg.n_batches)
for i in range(3):
    pipe.start_dev.fill_((b0 + i) * cfg.batch)
    rec = {}
    pipe.forward(record=rec)
torch.cuda.synchronize()
# last call of the kernel family was the HEAD block; rerun only the tail attention
b = pipe.blocks[1]
a = pipe.attn[1]
lib = tgl.lib()
lib.tgl_debug_timeline.argtypes = [C.c_void_p, C.c_size_t]
N = 148 * 32 * 8
host = (C.c_ulonglong * N)()
# rerun ONLY the tail-block attention so the timeline holds that launch
from paper_conf_asplos_wangm24_b200.block import _call_ws
ef = dev["efeat"]
_call_ws(lib.tgl_tblock_attn,
         [tgl.C.byref(a.struct), b.n_max, tgl._p(b.u_dev), tgl._p(b.seg_ptr), tgl._p(b.uniq_t),
          tgl._p(dev["nfeat"]), tgl._p(b.uniq_node), dev["nfeat"].shape[1], tgl._p(dev["nfeat"]),
          tgl._p(b.nbr), None, dev["nfeat"].shape[1], tgl._p(ef), tgl._p(b.eid), ef.shape[1],
          tgl._p(b.ts), tgl._p(pipe.tables[1]), pipe.tables[1].shape[0], cfg.k, tgl._p(b.out)],
         b.ws["attn"], None, "tail attn")
torch.cuda.synchronize()
lib.tgl_debug_timeline(host, N)
t = np.frombuffer(host, dtype=np.uint64).reshape(148, 32, 8).astype(np.float64)
names = ["desc_start", "desc_done", "prod_start", "prod_done", "mma_start", "epi_ready",
         "epi_have_acc", "epi_done"]
# the head-block kernel ran last and overwrote tiles 0..k of each CTA; use CTAs' tiles where
# epi_done is the maximum (consistent)
base = np.where(t[:, :, 0] > 0, t[:, :, 0], np.inf).min(axis=1, keepdims=True)
rel = (t - base[:, :, None]) / 1000.0
for tile in range(0, 12):
    row = []
    for e in range(8):
        v = rel[:, tile, e]
        v = v[(t[:, tile, e] > 0)]
        row.append(f"{np.median(v):7.1f}" if len(v) else "    -  ")
    print(f"tile {tile:2d} " + " ".join(row))
print("events:", names)
