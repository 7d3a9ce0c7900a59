"""Time the tail-block tgl_tblock_attn call per K|V kernel and debug mask (CFG=REDDIT|GDELT|...).

Needs a probe build: TGL_NVCC_EXTRA="-DTGL_PROBE [-DTGL_KV_PROF]" (the debug mask and the
instrumentation readers exist only there).

    python tools/kv_probe.py [precision]

TGL_DEBUG_MASK bits (profiling only): 1 skip epilogue math, 2 skip A gathers,
4 skip MMAs, 8 skip weight copies, 16 skip descriptor index loads, 64 skip the
converters (kv_async), 32 per-tile timeline.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
from paper_conf_asplos_wangm24_b200.block import _call_ws

prec = sys.argv[1] if len(sys.argv) > 1 else "fp32"
cfg = synth.get_config(os.environ.get("CFG", "REDDIT"))
if cfg.name in ("GDELT", "MAG"):     # device-generated, 16-byte row pitch (as bench.py)
    import bench
    cfg, g, neg, params, dev = bench.load_world_device(cfg.name)
else:
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
pipe = TGATPipeline(dev, tc, params, cfg.batch, TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]),
                    cfg.dedup, cfg.precompute, cfg.window, prec)
b0 = int(0.7 * cfg.n_batches)
pipe.start_dev.fill_(b0 * cfg.batch)
pipe.forward()
torch.cuda.synchronize()
L = len(pipe.blocks) - 1
b = pipe.blocks[L]
a = pipe.attn[L]
lib = tgl.lib()
nf, ef = dev["nfeat"], dev["efeat"]
tab = pipe.tables[L] if pipe.tables[L] is not None else None
if os.environ.get("PROBE_WINDOW"):          # 0 = direct evaluation, else a smaller table
    w = int(os.environ["PROBE_WINDOW"])
    tab = tgl.time_precompute(w, a.t["omega"], a.t["phi"]) if w > 0 else None


hs = pipe.nfeat_split if pipe.split else nf          # operand tables of the pipeline layout
hd = hs if pipe.split else nf                         # (split layouts: h_dst split16 too)
if pipe.split:
    ef = pipe.efeat_split


def call():
    _call_ws(lib.tgl_tblock_attn,
             [tgl.C.byref(a.struct), b.n_max, tgl._p(b.u_dev), tgl._p(b.seg_ptr), tgl._p(b.uniq_t),
              tgl._prow(hd), tgl._p(b.uniq_node), hd.stride(0), tgl._prow(hs), tgl._p(b.nbr), None,
              hs.stride(0), tgl._prow(ef), tgl._p(b.eid), ef.stride(0), tgl._p(b.ts),
              tgl._p(tab), 0 if tab is None else tab.shape[0], cfg.k, tgl._p(b.out)],
             b.ws["attn"], None, "tail attn")


flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
nd = int(b.u_dev.item())
ne = int(b.seg_ptr[nd].item())
print(f"tail block: {nd} dst, {ne} edges, precision {prec}")
ref = None
KVS = os.environ.get("PROBE_KV", "bin,async").split(",")
MASKS = [int(m) for m in os.environ.get("PROBE_MASKS", "0,1,2,4,8,64,6,95").split(",")]
for kv in KVS:
    for mask in MASKS:
        if kv == "bin" and mask & 64:
            continue
        a.set_kv_kernel(kv)
        os.environ["TGL_DEBUG_MASK"] = str(mask)
        ts = []
        for it in range(8):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            call()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        out = b.out[:nd].clone()
        if mask == 0:
            if ref is None:
                ref = out
            err = (out - ref).abs().max().item()
        else:
            err = float("nan")
        print(f"{kv:4s} mask {mask:3d}: {np.median(ts[2:]) * 1e3:8.1f} us  (vs bin: {err:.2e})")
os.environ["TGL_DEBUG_MASK"] = "0"

if os.environ.get("PROBE_PROF"):
    import ctypes as C
    lib.tgl_debug_prof.argtypes = [C.c_void_p, C.c_int]
    host = (C.c_ulonglong * (148 * 16))()
    for kv in (os.environ.get("PROBE_PROF_KV", "split"),):
        a.set_kv_kernel(kv)
        os.environ["TGL_DEBUG_MASK"] = str(512 | int(os.environ.get("PROBE_PROF_MASK", "0")))
        call(); torch.cuda.synchronize()
        lib.tgl_debug_prof(None, 1)
        call(); torch.cuda.synchronize()
        lib.tgl_debug_prof(host, 0)
        v = np.frombuffer(host, dtype=np.uint64).reshape(148, 16).astype(np.float64)
        names = (["L:aempty-wait", "T:aempty-wait", "T:work", "W:wempty-wait", "R:afull-wait",
                  "R:wfull-wait", "M:tempty-wait", "M:afull-wait", "M:pfull-wait", "M:wfull-wait",
                  "D:slot-wait", "E:acc-wait", "E:work", "total"] if kv == "pre2" else
                 ["T:aempty-wait", "T:phi+split+st", "T:compute+sts", "T:fence", "T:nontime-pass",
                  "L:aempty-wait", "6",
                  "M:tempty-wait", "M:afull-wait(gathered)", "M:afull-wait(time)",
                  "M:wfull-wait", "E:acc-wait", "E:work"] if kv == "pre" else
                 ["C:ffull-wait", "C:lds+phi", "C:bempty-wait", "C:cvt+sts", "C:fence",
                  "L:fempty-wait", "L:issue", "M:bfull-wait", "M:wfull-wait", "9", "10",
                  "E:acc-wait", "E:work"] if kv == "split" else
                 ["P:stage-free", "P:issue", "P:data-wait", "P:convert", "P:fence+arrive",
                 "MMA:A-wait", "MMA:W-wait", "MMA:acc-wait", "MMA:tile", "D:slot-wait",
                 "D:build", "E:acc-wait", "E:work"])
        if kv == "pre2":
            for who, rows in (("leader", v[0::2, :14]), ("peer", v[1::2, :14])):
                med = np.median(rows, axis=0)
                print(kv, who, "cycles per CTA (median):",
                      "  ".join(f"{n} {m:.0f}" for n, m in zip(names, med) if m > 0))
        else:
            med = np.median(v[:, :13], axis=0)
            print(kv, "cycles per CTA (median):", "  ".join(f"{n} {m:.0f}" for n, m in zip(names, med)))
    os.environ["TGL_DEBUG_MASK"] = "0"

if os.environ.get("PROBE_TRACE"):
    import ctypes as C
    lib.tgl_debug_trace.argtypes = [C.c_void_p, C.c_int]
    host = (C.c_ulonglong * 8192)()
    a.set_kv_kernel(os.environ.get("PROBE_TRACE_KV", "split"))
    os.environ["TGL_DEBUG_MASK"] = str(4096 | int(os.environ.get("PROBE_TRACE_MASK", "0")))
    call(); torch.cuda.synchronize()
    lib.tgl_debug_trace(None, 1)
    call(); torch.cuda.synchronize()
    lib.tgl_debug_trace(host, 0)
    v = np.frombuffer(host, dtype=np.uint64).reshape(32, 256)
    v = np.concatenate([r[:int(r[255] & 0xff)] for r in v])
    t = (v >> 16).astype(np.int64)
    ev = ((v >> 8) & 0xff).astype(int)
    k = (v & 0xff).astype(int)
    o = np.argsort(t, kind="stable")
    t0 = t[o[0]]
    names = {30: "Dn.desc-built", 31: "Dn.prod-done", 33: "Dn.mma-done", 34: "Dn.epi-start",
             35: "Dn.epi-end", 36: "Dn.warp-start", 37: "Dn.init-done", 20: "D.build-start", 21: "D.built", 1: "P.load-issued", 3: "P.data-ready", 4: "P.converted", 5: "M.A-ready", 6: "M.issued",
             7: "M.tile-start", 9: "E.acc-ready", 10: "E.done", 11: "W.issue", 12: "M.B-full"}
    for x in o[:int(os.environ.get('PROBE_TRACE_N', '400'))]:
        print(f"{(t[x] - t0) / 1965:8.2f} us  {names.get(ev[x], ev[x]):14s} {k[x]}")
    os.environ["TGL_DEBUG_MASK"] = "0"
