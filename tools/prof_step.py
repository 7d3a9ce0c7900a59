"""Run a few eager TBlock steps (for ncu): python tools/prof_step.py [CONFIG] [precision] [steps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import synth
from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "REDDIT"
    prec = sys.argv[2] if len(sys.argv) > 2 else "fp32"
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    cfg = synth.get_config(name)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    pipe = TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy,
                                                               cfg.seeds["sampler"]),
                        cfg.dedup, cfg.precompute, cfg.window, prec)
    b0 = int(0.7 * cfg.n_batches)
    for i in range(steps):
        pipe.start_dev.fill_((b0 + i) * cfg.batch)
        pipe.forward()
    torch.cuda.synchronize()
    print("done", name, prec, steps)


if __name__ == "__main__":
    main()
