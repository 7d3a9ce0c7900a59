"""Time tgl_sample on each block of a config's pipeline, alone (CUDA events), L2 flushed or warm.

    CFG=GDELT python tools/sample_probe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import bench
import synth
from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
from paper_conf_asplos_wangm24_b200.block import _call_ws

name = os.environ.get("CFG", "GDELT")
if name in bench.BIG:
    cfg, g, neg, params, dev = bench.load_world_device(name)
else:
    cfg, g, neg, params = bench.load_world(name)
    cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg), "nfeat": cu(g.nfeat),
           "efeat": cu(g.efeat)}
tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
pipe = TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]),
                    cfg.dedup, cfg.precompute, cfg.window, "fp32",
                    layout=bench.LAYOUT.get(cfg.name, "split"))
b0 = int(0.7 * cfg.n_batches)
pipe.start_dev.fill_(b0 * cfg.batch)
pipe.forward()
torch.cuda.synchronize()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
lib = tgl.lib()
for l, b in enumerate(pipe.blocks):
    nq = int(b.u_dev.item())

    def call():
        _call_ws(lib.tgl_sample,
                 [tgl.C.byref(tc.struct), b.n_max, tgl._p(b.u_dev), tgl._p(b.uniq_node),
                  tgl._p(b.uniq_t), cfg.k, tgl.STRATEGY[cfg.strategy], cfg.seeds["sampler"], l,
                  tgl._p(b.seg_ptr), tgl._p(b.nbr), tgl._p(b.eid), tgl._p(b.ts)],
                 b.ws["sample"], None, "tgl_sample")
    for fl in (True, False):
        ts = []
        for it in range(10):
            if fl:
                flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            call()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        E = int(b.seg_ptr[nq].item())
        print(f"block {l}: {nq} queries, {E} sampled edges, L2 {'flushed' if fl else 'warm'}: "
              f"{np.median(ts[2:]) * 1e3:.1f} us")
