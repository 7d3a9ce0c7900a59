"""Time the GDELT-sized T-CSR build (S1) alone: two builds, CUDA events around each
(the second is reported), optionally under ncu for the per-kernel launch list."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from synth.gpu import device_graph  # noqa: E402
from paper_conf_asplos_wangm24_b200 import tgl  # noqa: E402

cfg = synth.get_config(os.environ.get("CFG", "GDELT"))
dev = torch.device("cuda")
src, dst, t = device_graph(cfg, dev)
ws = tgl.Workspace(dev)
for i in range(int(os.environ.get("REPS", "3"))):
    torch.cuda.synchronize()
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record()
    tc = tgl.build_tcsr(cfg.n_nodes, src, dst, t, True, True, ws=ws, coarse=False, packed=False)
    e1.record()
    tgl.TemporalCSR(tc.indptr, tc.nbr, tc.eid, tc.ts, coarse=True, packed=True)
    e2.record()
    torch.cuda.synchronize()
    M = tc.nbr.numel()
    alg = cfg.n_edges * 12 + M * 12 + (cfg.n_nodes + 1) * 8
    ms = e0.elapsed_time(e2)
    print(f"build {i}: csr {e0.elapsed_time(e1):.2f} ms, index {e1.elapsed_time(e2):.2f} ms, "
          f"total {ms:.2f} ms, alg {alg / 1e9:.2f} GB -> {alg / ms / 1e6:.0f} GB/s", flush=True)
    del tc
