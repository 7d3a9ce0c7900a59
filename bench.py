#!/usr/bin/env python
"""Benchmark of the TBlock hot path (BASELINE.json metric) -- one JSON line on rank 0.

    python bench.py [--gpus N --steps K --warmup W --config REDDIT --precision fp32]
    python bench.py --impl reference ...      # the CPU oracle on the host cores

A step = one batch through every §8(a) row: roots (S2) -> [dedup (S3)] ->
sample (S4) -> next block (S5) -> ... -> TBlock attention tail..head (S6-S13,
S15) -> dedup inverse at the roots (S14), replayed as one CUDA graph with the
graph, features and batch edges resident in HBM.  Between timed steps L2 is
flushed by writing a 256 MiB buffer (outside the timed events).  With N GPUs
(torchrun) every rank runs its own batch of the stream (weak scaling) and the
root embeddings of all ranks are all-gathered over NCCL inside the step (S16).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "sampled edges/s and TBlock embeddings/s at 1/2/4/8 B200; % HBM roofline"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="REDDIT")
    ap.add_argument("--precision", default="fp32", choices=["fp32", "bf16", "fp32_simt"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--dedup", default="config", choices=["config", "on", "off"],
                    help="override the config's dedup setting (ablation only)")
    ap.add_argument("--cache", type=int, default=0,
                    help="cache() table slots per layer (0 = off, the BASELINE configs)")
    return ap.parse_args()


# ---------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "samples": len(sm), "reasons": sorted(reasons)}


# ---------------------------------------------------------------------- shared inputs
def load_world(cfg_name: str):
    import synth
    cfg = synth.get_config(cfg_name)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    return cfg, g, neg, params


def oracle_rate(cfg, g, neg, params, batches, seconds: float):
    """CPU oracle (as it stands) on whole batches until `seconds` of CPU work."""
    import oracle
    from oracle import pipeline as opipe
    t0 = time.perf_counter()
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    t_build = time.perf_counter() - t0
    done, edges, t_run, nb = 0, 0, 0.0, 0
    for b in batches:
        nb += 1
        t0 = time.perf_counter()
        emb, blocks = opipe.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy,
                                      cfg.dedup, cfg.seeds["sampler"],
                                      *synth_batch(g, neg, b))
        t_run += time.perf_counter() - t0
        done += emb.shape[0]
        edges += sum(int(bl.seg_ptr[-1]) for bl in blocks)
        if t_run >= seconds:
            break
    return {"emb_per_s": done / t_run, "edges_per_s": edges / t_run, "batches": nb,
            "roots": done, "seconds": t_run,
        "cores": oracle.num_threads(), "tcsr_build_s": t_build}


BIG = ("GDELT", "MAG")   # generated on the device (synth.gpu); host RAM holds only the COO


class HostGraph:
    """Host view of a device-generated graph: what batch slicing and the oracle need."""

    def __init__(self, cfg, src, dst, t):
        self.cfg, self.src, self.dst, self.t, self.num_edges = cfg, src, dst, t, cfg.n_edges


def load_world_device(cfg_name: str):
    """GDELT/MAG: COO, negatives and feature tables generated on cuda (synth.gpu, the
    same counter-based values as synth.make_graph), host copies of the COO only."""
    import synth
    import torch
    from synth import gpu as sg
    cfg = synth.get_config(cfg_name)
    d = torch.device("cuda")
    src, dst, t = sg.device_graph(cfg, d)
    neg = sg.device_negatives(cfg, d)
    # 16-byte row pitch (GDELT's 413 / 186 floats padded to 416 / 188): the K|V kernel's
    # cp.async gathers need it; the values are the same counter-based features
    nfeat = sg.device_feature_table(cfg.seeds["feat"], cfg.n_nodes, cfg.d_v, d, pitch_mult=4)
    efeat = (sg.device_feature_table(cfg.seeds["feat"] + 7919, cfg.n_edges, cfg.d_e, d,
                                     pitch_mult=4)
             if cfg.d_e else torch.zeros((0, 0), dtype=torch.float32, device=d))
    g = HostGraph(cfg, src.cpu().numpy(), dst.cpu().numpy(), t.cpu().numpy())
    neg_h = neg.cpu().numpy()
    dev = {"src": src, "dst": dst, "t": t, "neg": neg, "nfeat": nfeat, "efeat": efeat}
    return cfg, g, neg_h, synth.gen.model_params(cfg), dev


def oracle_rate_big(cfg, g, neg, params, batches, seconds: float, frac: int = 0):
    """Listing 1's recursion (oracle/big.py) root by root on whole-graph-free segments:
    the whole-graph oracle cannot hold GDELT/MAG.  Bounded by `seconds` of CPU work."""
    import oracle
    from oracle import big
    from oracle import pipeline as opipe
    segs, done, t_run, nb = {}, 0, 0.0, 0
    for b in batches:
        nb += 1
        qn, qt = opipe.roots(*synth_batch(g, neg, b))
        for v, tq in zip(qn, qt):
            t0 = time.perf_counter()
            big.embed_recursive(g.src, g.dst, g.t, cfg, params, [v], [tq],
                                cfg.seeds["sampler"], segs=segs)
            t_run += time.perf_counter() - t0
            done += 1
            if t_run >= seconds:
                break
        if t_run >= seconds:
            break
    return {"emb_per_s": done / t_run, "batches": nb, "roots": done, "seconds": t_run,
            "cores": oracle.num_threads(), "edges_per_s": float("nan")}


def synth_batch(g, neg, b):
    import synth
    return synth.batch_roots_inputs(g, neg, b)


# ---------------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    if args.config.upper() in BIG:
        return run_reference_big(args)
    cfg, g, neg, params = load_world(args.config)
    import oracle
    from oracle import pipeline as opipe
    tc = oracle.build_tcsr(cfg.n_nodes, g.src, g.dst, g.t, True)
    b0 = int(0.7 * cfg.n_batches)
    # bounded sample: a slice of each batch's roots (first `frac` of its edges)
    frac_edges = max(1, cfg.batch // 8)
    times, roots, edges = [], 0, 0
    for i in range(args.warmup + args.steps):
        b = b0 + i
        src_b, dst_b, t_b, neg_b = synth_batch(g, neg, b)
        sl = slice(0, frac_edges)
        t0 = time.perf_counter()
        emb, blocks = opipe.run_batch(tc, g.nfeat, g.efeat, params, cfg.k, cfg.strategy,
                                      cfg.dedup, cfg.seeds["sampler"], src_b[sl], dst_b[sl],
                                      t_b[sl], neg_b[sl])
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
            roots += emb.shape[0]
            edges += sum(int(bl.seg_ptr[-1]) for bl in blocks)
    T = sum(times)
    val = roots / T
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "embeddings/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * T / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "batch_edges_per_step": frac_edges,
                       "roots_per_step": 3 * frac_edges, "layers": cfg.n_layers, "k": cfg.k,
                       "strategy": cfg.strategy, "dedup": cfg.dedup,
                       "precompute": cfg.precompute},
            "sampled_edges_per_s": edges / T,
            "cpu_baseline": {"value": val, "unit": "embeddings/s",
                             "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"first {frac_edges} of each {cfg.batch}-edge batch "
                                       f"({3 * frac_edges} roots) from 70% of the stream"},
            "e2e": {"value": val, "unit": "embeddings/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_reference_big(args):
    """--impl reference on GDELT/MAG: the oracle's recursion (oracle/big.py) on a few roots
    per step; the COO comes from the same seeded generator as our arm (synth.gpu on a
    GPU box -- input generation only -- else synth.make_graph)."""
    import oracle
    import synth
    from oracle import big
    from oracle import pipeline as opipe
    import torch
    cfg = synth.get_config(args.config.upper())
    if torch.cuda.is_available():                   # the same COO our arm generates
        from synth import gpu as sg
        d = torch.device("cuda")
        src, dst, t = sg.device_graph(cfg, d)
        gg = HostGraph(cfg, src.cpu().numpy(), dst.cpu().numpy(), t.cpu().numpy())
        neg = sg.device_negatives(cfg, d).cpu().numpy()
        del src, dst, t
    else:
        gg = synth.make_graph(cfg, with_features=False)
        neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)
    b0 = int(0.7 * cfg.n_batches)
    per_step = 2                                    # roots per step (bounded sample)
    times, roots, segs = [], 0, {}
    for i in range(args.warmup + args.steps):
        qn, qt = opipe.roots(*synth_batch(gg, neg, b0 + i))
        t0 = time.perf_counter()
        big.embed_recursive(gg.src, gg.dst, gg.t, cfg, params, qn[:per_step], qt[:per_step],
                            cfg.seeds["sampler"], segs=segs)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
            roots += per_step
    T = sum(times)
    val = roots / T
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "embeddings/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * T / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "roots_per_step": per_step, "layers": cfg.n_layers,
                       "k": cfg.k, "strategy": cfg.strategy, "dedup": cfg.dedup,
                       "precompute": cfg.precompute},
            "cpu_baseline": {"value": val, "unit": "embeddings/s",
                             "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"first {per_step} roots of each batch from 70% of the "
                                       f"stream, Listing 1's recursion (oracle/big.py)"},
            "e2e": {"value": val, "unit": "embeddings/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------- our arm
def algorithmic_attn(cfg, n_dst: int, n_edges: int, d_hdst: int, d_hsrc: int):
    """Per tgl_tblock_attn call: FLOPs and bytes the method must do."""
    dm, dt, de = cfg.d_model, cfg.d_t, cfg.d_e
    kkv = d_hsrc + de + dt
    flops = (n_edges * 2 * (2 * dm) * kkv          # K and V projections (S9)
             + n_dst * 2 * dm * (d_hdst + dt)       # Q (S8)
             + n_dst * 2 * dm * (dm + d_hdst)       # FFN (S13)
             + n_edges * 4 * dm)                    # logits + weighted sum (S10-S12)
    bytes_ = (n_edges * (4 * (d_hsrc + de) + 4 + 4 + 4 + 8)   # gathers + nbr/eid/ts + idx
              + n_dst * (4 * d_hdst * 2 + 8 + 8 + 4 * cfg.d_model))  # h_dst (Q and FFN), t, seg, out
    return flops, bytes_


def algorithmic_kv(cfg, n_dst: float, n_edges: float, d_hsrc: int):
    """Per launch of the K|V attention kernel (S6, S7, S9-S12):
    FLOPs = E * (2 * 2*d_model * K) for [K;V] = W [h ; e ; Phi] (K = d_hs + d_e + d_t)
            + E * 4 * d_model for the logits and the alpha-weighted sum;
    bytes = E * (4 (d_hs + d_e) + 12)  (gathered rows + nbr/eid/ts; Phi computed or
            table-read, counted 0 as in SURVEY §8(d))
            + n_dst * (8 + 4 + 4 (d_model + 2) + 4 d_model)  (seg_ptr, t, q row, r row)."""
    dm = cfg.d_model
    k = d_hsrc + cfg.d_e + cfg.d_t
    flops = n_edges * (2 * 2 * dm * k + 4 * dm)
    bytes_ = n_edges * (4 * (d_hsrc + cfg.d_e) + 12) + n_dst * (12 + 4 * (dm + 2) + 4 * dm)
    return flops, bytes_


def ncu_traffic(config: str, precision: str):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of the K|V kernel from the
    committed `ncu --set full` capture of this config and precision (profiles/), or None."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "r01_kv_split_traffic.json")))
        return d[config][precision]
    except Exception:
        return None


KV_KERNELS = {0: "kv_split_kernel (contiguous K plan)", 1: "kv_split_kernel (padded K plan)",
              2: "kv_async_kernel", 3: "kv_bin_kernel", 4: "kv_kernel (general)"}


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import synth
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
    from paper_conf_asplos_wangm24_b200 import dist as pdist

    cu = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    if args.config.upper() in BIG:
        cfg, g, neg, params, dev = load_world_device(args.config.upper())
    else:
        cfg, g, neg, params = load_world(args.config)
        dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
               "nfeat": cu(g.nfeat), "efeat": cu(g.efeat)}
    if args.dedup != "config" or (args.cache and not cfg.dedup):
        from dataclasses import replace              # cache() sits behind each block's dedup
        cfg = replace(cfg, dedup=args.dedup == "on" or bool(args.cache))   # (P:578 pairs them)
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    ev1.record()
    torch.cuda.synchronize()
    tcsr_ms = ev0.elapsed_time(ev1)
    sampler = TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"])
    pipe = TGATPipeline(dev, tc, params, cfg.batch, sampler, cfg.dedup, cfg.precompute,
                        cfg.window, args.precision, cache_capacity=args.cache)
    pipe.capture()
    n0 = 3 * cfg.batch
    gathered = torch.empty(world * n0, cfg.d_model, device="cuda") if world > 1 else None
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    b0 = int(0.7 * cfg.n_batches)
    nb_avail = cfg.n_batches - b0

    def batch_of(i):
        return pdist.rank_batch(i, rank, world, b0, nb_avail)

    # per-step device counters read after timing (outside the events)
    cnt_e = torch.zeros(args.warmup + args.steps, dtype=torch.int64, device="cuda")
    stream = torch.cuda.current_stream()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]

    def counts_into(i):
        tot = torch.zeros((), dtype=torch.int64, device="cuda")
        for b in pipe.blocks:
            tot = tot + b.seg_ptr.index_select(0, b.u_dev.clamp(max=b.n_max)).squeeze()
        cnt_e[i] = tot

    for i in range(args.warmup):
        pipe.start_dev.fill_(batch_of(i) * cfg.batch)
        out = pipe.run_graph()
        if world > 1:
            pdist.allgather_embeddings(out[:n0], gathered)
        counts_into(i)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = ClockSampler(local)
    clk.start()
    time.sleep(0.3)
    torch.cuda.synchronize()
    for i in range(args.steps):
        j = args.warmup + i
        flush.zero_()                                  # L2 flush, outside the events
        pipe.start_dev.fill_(batch_of(j) * cfg.batch)
        starts[i].record(stream)
        out = pipe.run_graph()
        if world > 1:
            pdist.allgather_embeddings(out[:n0], gathered)   # S16
        ends[i].record(stream)
        counts_into(j)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = clk.stop()
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    total_ms = sum(step_ms)
    t_max = torch.tensor([total_ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
    total_ms = float(t_max.item())
    edges_local = int(cnt_e[args.warmup:].sum().item())
    e_tot = torch.tensor([edges_local], dtype=torch.int64, device="cuda")
    if world > 1:
        dist.all_reduce(e_tot)
    roots_all = world * n0 * args.steps
    emb_per_s = roots_all / (total_ms / 1e3)
    edges_per_s = int(e_tot.item()) / (total_ms / 1e3)

    # ---- dominant call: tgl_tblock_attn on the tail block, timed eagerly with events
    rec_ms, rec_shape, brk, kv_ms = [], None, {}, []
    lib = tgl.lib()
    for i in range(max(3, min(args.steps, 20))):
        flush.zero_()
        pipe.start_dev.fill_(batch_of(args.warmup + i) * cfg.batch)
        rec = {}
        lib.tgl_kv_timing(1)          # CUDA events around each K|V kernel, on its stream
        pipe.forward(record=rec)
        torch.cuda.synchronize()
        kv_ms.append(lib.tgl_kv_timing_ms(0))   # the tail block runs first
        tail = pipe.L - 1
        rec_ms.append(rec[tail][0].elapsed_time(rec[tail][1]))
        mk = rec["_marks"]
        for (n0_, e0_), (n1_, e1_) in zip(mk[:-1], mk[1:]):
            brk.setdefault(n1_, []).append(e0_.elapsed_time(e1_))
        bt = pipe.blocks[tail]
        U = int(bt.u_dev.item())
        E = int(bt.seg_ptr[U].item())
        rec_shape = (rec_shape or []) + [(U, E)]
    U_avg = sum(u for u, _ in rec_shape) / len(rec_shape)
    E_avg = sum(e for _, e in rec_shape) / len(rec_shape)
    fl, by = algorithmic_attn(cfg, U_avg, E_avg, cfg.d_v, cfg.d_v)
    attn_ms = sum(rec_ms) / len(rec_ms)
    lib.tgl_kv_timing(0)
    kv_fl, kv_by = algorithmic_kv(cfg, U_avg, E_avg, cfg.d_v)
    kv_ok = [m for m in kv_ms if m > 0]
    kv_avg = sum(kv_ok) / len(kv_ok) if kv_ok else float("nan")
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    sm_max = clocks.get("sm_max_mhz") or peaks.get("sm_max_mhz", 1965.0)
    hbm_peak = peaks.get("hbm_gbs", 6545.9)
    bf16_peak = peaks.get("bf16_tflops", 1613.6)
    kv_tf = kv_fl / (kv_avg / 1e3) / 1e12
    kv_gbs = kv_by / (kv_avg / 1e3) / 1e9
    if args.precision == "fp32_simt":
        peak = 148 * 128 * 2 * sm_max * 1e6 / 1e12     # TFLOP/s, FFMA on all SMs
        bound, unit, ach = "alu", "TFLOP/s", kv_tf
        note = "FP32 FFMA peak = 148 SM x 128 lanes x 2 x clocks.max.sm (derived)"
    elif args.precision == "fp32":
        # fp32 = 3 bf16 MMA passes per algorithmic FLOP: the tensor roofline for fp32
        # operands is the measured bf16 burst peak / 3; it binds before HBM
        peak, bound, unit, ach = bf16_peak / 3, "tensor", "TFLOP/s", kv_tf
        note = "measured cuBLAS bf16 burst peak (MEASURED_PEAKS.json) / 3 passes"
    else:
        peak, bound, unit, ach = hbm_peak, "hbm", "GB/s", kv_gbs
        note = "measured HBM copy bandwidth (MEASURED_PEAKS.json); bf16 MMA time < HBM time"
    tr = ncu_traffic(cfg.name, args.precision)
    kname = KV_KERNELS.get(int(lib.tgl_kv_timing_kernel(0)), "?")
    roofline = {"kernel": f"{kname}: K|V attention of the tail block (S6,S7,S9-S12)",
                "bound": bound, "achieved": ach, "peak": peak, "unit": unit,
                "frac": ach / peak,
                "traffic": tr["dram_bytes_per_launch"] if tr else None,
                "traffic_note": (f"ncu --set full, {tr['source']}" if tr else None),
                "per_launch_ms": kv_avg, "launches_timed": len(kv_ok),
                "algorithmic_flops": kv_fl, "algorithmic_bytes": kv_by,
                "tensor_tflops": kv_tf, "tensor_frac_bf16_peak": kv_tf / bf16_peak,
                "hbm_gbs": kv_gbs, "hbm_frac": kv_gbs / hbm_peak,
                "n_dst_avg": U_avg, "n_edges_avg": E_avg, "peak_note": note,
                "attn_call_ms": attn_ms, "attn_call_tflops": fl / (attn_ms / 1e3) / 1e12}

    # ---- e2e through the public API: pinned host batch -> device -> host embeddings
    e2e = None
    if world >= 1:
        pipe_h = TGATPipeline(dev, tc, params, cfg.batch, sampler, cfg.dedup, cfg.precompute,
                              cfg.window, args.precision, staging=True,
                              cache_capacity=args.cache)
        pipe_h.capture()
        from paper_conf_asplos_wangm24_b200 import HostStream
        outs = [torch.empty(n0, cfg.d_model, dtype=torch.float32).pin_memory() for _ in range(2)]
        host_batches = []
        for i in range(args.steps):
            sb, db, tb, nb_ = synth.batch_roots_inputs(g, neg, batch_of(args.warmup + i))
            host_batches.append(tuple(torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
                                      for x in (sb, db, tb, nb_)))
        hs = HostStream(pipe_h, n0, cfg.d_model)
        for i in range(min(3, args.steps)):
            hs.submit(*host_batches[i], outs[i % 2]).synchronize()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        # serving loop: batch i's embeddings are on the host (event synchronised) before
        # batch i+1's are requested; the D2H of batch i overlaps batch i+1's compute
        t0 = time.perf_counter()
        prev = None
        for i in range(args.steps):
            done = hs.submit(*host_batches[i], outs[i % 2])
            if world > 1:
                pdist.allgather_embeddings(pipe_h.graph_out[:n0], gathered)
            if prev is not None:
                prev.synchronize()
            prev = done
        prev.synchronize()
        torch.cuda.synchronize()
        el = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(el, op=dist.ReduceOp.MAX)
        h2d = cfg.batch * (4 + 4 + 4 + 4)
        e2e = {"value": world * n0 * args.steps / float(el.item()), "unit": "embeddings/s",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": n0 * cfg.d_model * 4,
               "timing": "host wall clock over the serving loop (HostStream): per batch H2D "
                         "of its edges, graph replay, D2H of its embeddings on a copy stream, "
                         "host waits for batch i before batch i+2 is submitted"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate = oracle_rate_big if cfg.name in BIG else oracle_rate
        r = rate(cfg, g, neg, params, [batch_of(i) for i in range(200)], args.cpu_seconds)
        smp = (f"{r['roots']} roots of {r['batches']} batch(es) from 70% of the stream, one "
               f"at a time by Listing 1's recursion (oracle/big.py), {r['seconds']:.1f} s"
               if cfg.name in BIG else
               f"{r['batches']} whole batch(es) ({r['roots']} roots) from 70% of the stream, "
               f"{r['seconds']:.1f} s")
        cpu = {"value": r["emb_per_s"], "unit": "embeddings/s", "cores": r["cores"],
               "kind": "oracle", "sample": smp, "sampled_edges_per_s": r["edges_per_s"]}

    if rank == 0:
        line = {"metric": METRIC, "value": emb_per_s, "unit": "embeddings/s",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": {"fp32": "f32 (3-pass bf16 tensor-core split)",
                                             "bf16": "bf16", "fp32_simt": "f32"}[args.precision], "data": "synthetic",
                "config": {"workload": cfg.name, "batch_edges": cfg.batch, "roots_per_step": n0,
                           "roots_per_step_all_ranks": world * n0, "layers": cfg.n_layers,
                           "k": cfg.k, "strategy": cfg.strategy, "dedup": cfg.dedup,
                           "precompute": cfg.precompute, "precision": args.precision,
                           "cache_slots_per_layer": args.cache,
                           "parallelism": f"root-sharded dp{world}" if world > 1 else "single",
                           "l2": "flushed (256 MiB write) between timed steps",
                           "timing": "CUDA events per step on the launch stream; max over ranks"},
                "sampled_edges_per_s": edges_per_s,
                "tcsr_build_ms": tcsr_ms,
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "gpu_launches": pipe.launches_per_forward * args.steps,
                "gpu_launches_per_step": pipe.launches_per_forward,
                "step_ms_p50": statistics.median(step_ms),
                "breakdown_ms_eager": {k_: statistics.median(v_) for k_, v_ in brk.items()}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
