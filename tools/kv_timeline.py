"""Per-tile role timeline of the REDDIT tail K|V kernel (TGL_DEBUG_MASK=32).

    TGL_KV=async|bin python tools/kv_timeline.py [precision]

Events (globaltimer, us from the CTA's first descriptor): 0 desc start, 1 desc done,
2 producer start, 3 conversion/producer done, 4 MMA start,
5 epilogue ready (q fetched), 6 accumulator ready, 7 epilogue done.
"""
import ctypes as C
import os
import sys

os.environ["TGL_DEBUG_MASK"] = str(32 | int(os.environ.get("EXTRA_MASK", "0")))
sys.argv = [sys.argv[0]] + sys.argv[1:]
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

here = os.path.dirname(os.path.abspath(__file__))
src = open(os.path.join(here, "kv_probe.py")).read()
src = src[:src.index("flush = torch.empty")]          # setup only (graph, pipeline, call())
exec(compile(src, "kv_probe_setup", "exec"))
lib = tgl.lib()
lib.tgl_debug_timeline.argtypes = [C.c_void_p, C.c_size_t]
N = 148 * 32 * 8
host = (C.c_ulonglong * N)()
C.memset(host, 0, C.sizeof(host))
for _ in range(2):
    call()
torch.cuda.synchronize()
lib.tgl_debug_timeline(host, N)
t = np.frombuffer(host, dtype=np.uint64).reshape(148, 32, 8).astype(np.float64)
base = np.where(t[:, :, 0] > 0, t[:, :, 0], np.inf).min(axis=1, keepdims=True)
rel = (t - base[:, :, None]) / 1000.0
names = ["desc0", "desc1", "load0", "load1", "mma0", "epiQ", "epiAcc", "epi1"]
print("tile " + " ".join(f"{n:>7s}" for n in names))
for tile in range(0, 16):
    row = []
    for e in range(8):
        v = rel[:, tile, e][t[:, tile, e] > 0]
        row.append(f"{np.median(v):7.1f}" if len(v) else "      -")
    print(f"{tile:4d} " + " ".join(row))
end = np.nanmax(np.where(t[:, :, 7] > 0, rel[:, :, 7], np.nan), axis=1)
print("per-CTA last epilogue done (us): median %.1f  max %.1f" % (np.nanmedian(end), np.nanmax(end)))
