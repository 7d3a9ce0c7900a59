"""TBlock chain for one batch on one GPU (S2-S15) -- host bookkeeping only.

Names follow the paper: a `TBlock` holds destination <node, time> pairs and,
once sampled, its source nodes / edges (Table 2); `TSampler`
(L2.5) fills a block; `dedup` filters a block's destinations and keeps the
inverse hook; `aggregate` runs the attention layers from the tail block
back to the head (L2.18-19).  Every step is a libtgl kernel launch on one
stream; sizes stay on the device (capacity-bounded buffers + device counts), so
`TGATPipeline.forward` is a fixed launch sequence that `capture()` records into
a CUDA graph.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import torch

from . import tgl


@dataclass
class TBlock:
    """One TBlock (Fig 3): dst pairs (+ dedup hook) and sampled sources."""
    layer: int
    n_max: int                     # capacity of the dst arrays before dedup
    dst_node: torch.Tensor
    dst_t: torch.Tensor
    n_dev: torch.Tensor            # device count of dst pairs
    uniq_node: torch.Tensor = None  # after dedup (aliases dst_* when dedup is off)
    uniq_t: torch.Tensor = None
    u_dev: torch.Tensor = None
    inv: torch.Tensor = None       # dedup inverse hook (None when dedup is off)
    seg_ptr: torch.Tensor = None   # sampled sources
    nbr: torch.Tensor = None
    eid: torch.Tensor = None
    ts: torch.Tensor = None
    out: torch.Tensor = None       # layer output [n_max, d_out]
    out_split: torch.Tensor = None  # the same rows as a split16 table (layout="split")
    ws: dict = field(default_factory=dict)


class TSampler:
    """`tg.TSampler(n_nbr, 'recent' | 'uniform')` (L2.5)."""

    def __init__(self, k: int, strategy: str = "recent", seed: int = 0x74676C00):
        self.k, self.strategy, self.seed = k, strategy, seed


class TGATPipeline:
    """L-layer TGAT over TBlocks (Listing 2) with all buffers preallocated.

    graph: dict of device tensors src, dst, t, neg (per edge), nfeat, efeat.
    params: list of per-block weight dicts (block 0 = head, block L-1 = raw features).
    """

    def __init__(self, graph: dict, tcsr: tgl.TemporalCSR, params: list, batch: int,
                 sampler: TSampler, use_dedup: bool, precompute: bool, window: int = 65536,
                 precision: str = "fp32", staging: bool = False, device=None,
                 cache_capacity: int = 0, shard: tuple | None = None,
                 layout: str | None = None, host_features: bool = False,
                 node_proj: bool | None = None):
        """shard = (rank, world): root sharding (S16).  The batch's roots
        (deduped when use_dedup) are formed on every rank; this pipeline computes the
        contiguous slice `rank` of them (tgl_shard_slice) and forward(slot) returns the
        slice's embeddings [c_max, d_out] in `send[slot]`; `combine(slot, gathered)`
        rebuilds the whole batch from the all-gathered slices (tgl_shard_gather).  Two
        slots (two captured graphs) let batch b's all-gather overlap batch b+1.

        layout: "split" (default for the tensor-core precisions) gathers the K|V operands
        from split16 tables (tgl_split_rows: bf16 hi / lo halves, the kv_pre kernel) --
        graph["nfeat_split"] / graph["efeat_split"] when given, else split here once --
        and every inner layer output is split once for the layer above; "fp32" gathers
        fp32 rows and converts in the SM (kv_split).

        host_features: the operand tables live in pinned host memory (preload(), P:299-301;
        graphs whose features exceed HBM): every block first copies the rows it gathers --
        edge rows by eid, and for the tail block node rows by nbr / dst -- into device staging
        tables with tgl_preload_rows (the GPU reads host memory directly), then runs on them
        with identity indices.  Device tables passed in are moved to pinned host memory.

        node_proj: the tail block's projections of h (eqs 4, 5, 7 are linear in h) are
        computed once per node per forward (tgl_node_proj into Z [n_nodes, 512]) and
        gathered, so the tail's per-edge MMAs cover [e | Phi] only and it has no Q launch.
        None (default) = on when the node table is split16 and device-resident, has at
        most 1/16 of the rows the tail block gathers per batch, d_h >= 2 d_model (the h
        columns dominate the projections) and Z fits 2 GB."""
        self.dev = device or torch.device("cuda")
        self.g = graph
        self.tcsr = tcsr
        self.L = len(params)
        self.batch = batch
        self.sampler = sampler
        self.use_dedup = use_dedup
        self.E = graph["src"].numel()
        self.attn = [tgl.AttnParams(p, self.dev, precision, pack=True) for p in params]
        self.tables = [tgl.time_precompute(window, a.t["omega"], a.t["phi"]) if precompute else None
                       for a in self.attn]
        if layout is None:
            layout = "fp32" if precision == "fp32_simt" else "split"
        self.split = layout == "split"
        if self.split:
            assert precision != "fp32_simt", "split16 tables feed the tensor-core path"
            nf = graph.get("nfeat_split")
            if nf is None:
                nf = tgl.split_rows(graph["nfeat"])
            ef = graph.get("efeat_split")
            if ef is None and graph.get("efeat") is not None and graph["efeat"].numel():
                ef = tgl.split_rows(graph["efeat"])
            self.nfeat_split, self.efeat_split = nf, ef
            for l, a in enumerate(self.attn):
                a.struct.input_layout = (tgl.SPLIT_HSRC | (tgl.SPLIT_E if a.host["d_e"] else 0) |
                                         tgl.SPLIT_TABLE | tgl.SPLIT_HDST)
            # the precompute tables as split16 rows too: gathered like features
            self.tables = [None if t is None else tgl.split_rows(t) for t in self.tables]
        k = sampler.k
        i32, f32, i64 = torch.int32, torch.float32, torch.int64
        z = lambda n, dt: torch.zeros(max(int(n), 1), dtype=dt, device=self.dev)
        self.host = host_features
        if host_features:        # N4: operand tables in pinned host memory
            pin = lambda t: None if t is None else (t if (not t.is_cuda and t.is_pinned())
                                                    else t.cpu().pin_memory())
            if self.split:
                self.nfeat_host, self.efeat_host = pin(self.nfeat_split), pin(self.efeat_split)
                self.nfeat_split = self.efeat_split = None
            else:
                self.nfeat_host = pin(graph["nfeat"])
                ef = graph.get("efeat")
                self.efeat_host = pin(ef) if ef is not None and ef.numel() else None
        self.start_dev = torch.zeros(1, dtype=i64, device=self.dev)
        self.blocks = []
        n_max = 3 * batch
        self.shard = shard
        if shard is not None:
            rank, world = shard
            assert 0 <= rank < world and cache_capacity == 0
            self.world = world
            self.c_max = -(-n_max // world)          # rows per rank slice (padded)
            # per slot: the batch's roots (S2) and, with dedup, their unique pairs + inverse
            self.roots = []
            for _ in range(2):
                r = {"node": z(n_max, i32), "t": z(n_max, f32), "n": z(1, i64)}
                if use_dedup:
                    r.update(unode=z(n_max, i32), ut=z(n_max, f32), u=z(1, i64), inv=z(n_max, i32))
                self.roots.append(r)
            n_max = self.c_max
        for l in range(self.L):
            b = TBlock(l, n_max, z(n_max, i32), z(n_max, f32), z(1, i64))
            if use_dedup and not (shard is not None and l == 0):   # sharded head: roots
                b.uniq_node, b.uniq_t, b.u_dev, b.inv = z(n_max, i32), z(n_max, f32), z(1, i64), z(n_max, i32)
            else:
                b.uniq_node, b.uniq_t, b.u_dev = b.dst_node, b.dst_t, b.n_dev
            b.seg_ptr = z(n_max + 1, i64)
            b.nbr, b.eid, b.ts = z(n_max * k, i32), z(n_max * k, i32), z(n_max * k, f32)
            b.out = z(n_max * self.attn[l].d_out, f32).view(-1, self.attn[l].d_out)
            if self.split and l > 0:       # the layer above gathers its rows split
                dpo = tgl.split_width(self.attn[l].d_out)
                b.out_split = z(n_max * dpo, f32).view(-1, dpo)
            self.blocks.append(b)
            n_max = n_max + n_max * k
        self.emb = z(3 * batch * self.attn[0].d_out, f32).view(-1, self.attn[0].d_out)
        # node projections for the tail block (its h_src / h_dst are node-feature rows)
        nft = graph.get("nfeat") if graph.get("nfeat") is not None else graph.get("nfeat_split")
        n_nodes = nft.shape[0] if nft is not None else 0
        tail = self.blocks[-1]
        np_ok = (self.split and precision in ("fp32", "bf16") and not host_features and
                 n_nodes > 0 and self.attn[-1].host["n_heads"] == 2)
        if node_proj is None:
            # a clear win only when the h columns dominate the projections and the node
            # table is small next to the rows the tail block gathers (measured: GDELT
            # 7.8e6 -> 1.03e7 emb/s; REDDIT / LASTFM / WIKI, d_v <= 172, lose 3-12 %)
            d_h = self.attn[-1].host["d_hdst"]
            node_proj = (np_ok and n_nodes * 16 <= tail.n_max * k and
                         d_h >= 2 * self.attn[-1].host["d_model"] and
                         n_nodes * 2048 <= (2 << 30))
        assert not node_proj or np_ok, "node_proj needs the split16 device-resident tables"
        self.node_proj = bool(node_proj)
        self.zproj = None
        if self.node_proj:
            self.zproj = torch.empty(n_nodes, tgl.NODE_PROJ_LD, dtype=f32, device=self.dev)
            at = self.attn[-1]
            at.struct.input_layout |= tgl.NODE_PROJ
            at.struct.node_proj = tgl._p(self.zproj)
            # Z depends on the weights and the node table only: it is computed on a side
            # stream that forks at the start of a forward and joins before the tail block,
            # so it overlaps the latency-bound roots / dedup / sampling launches
            self.np_stream = torch.cuda.Stream(device=self.dev)
            self.np_fork = torch.cuda.Event()
            self.np_join = torch.cuda.Event()
        if self.host:            # device staging tables for the preloaded rows, per block
            cap = max(b.n_max * k for b in self.blocks)
            self.iota = torch.arange(max(cap, 1), dtype=i32, device=self.dev)
            for b in self.blocks:
                if self.efeat_host is not None:
                    pe = self.efeat_host.shape[1]
                    b.ws["epre"] = torch.zeros(max(b.n_max * k, 1), pe, dtype=f32, device=self.dev)
            tail = self.blocks[-1]
            pv = self.nfeat_host.shape[1]
            tail.ws["nsrc"] = torch.zeros(max(tail.n_max * k, 1), pv, dtype=f32, device=self.dev)
            tail.ws["ndst"] = torch.zeros(max(tail.n_max, 1), pv, dtype=f32, device=self.dev)
        if shard is not None:   # the head block writes the slice into send[slot]
            d0 = self.attn[0].d_out
            self.send = [z(self.c_max * d0, f32).view(-1, d0) for _ in range(2)]
        # staging mode: the batch's edges arrive from host memory each step (public API)
        self.staging = staging
        if staging:
            self.stage = {"src": z(batch, i32), "dst": z(batch, i32), "t": z(batch, f32),
                          "neg": z(batch, i32)}
            self.stage_n = batch
        # kernels launched per forward (libtgl only; memsets excluded)
        # dedup: one single-CTA kernel up to 4096 pairs (dedup.cu kSmallN), else three
        dedup_launches = [(1 if b.n_max <= 4096 else 3) if use_dedup else 0 for b in self.blocks]
        if shard is not None:   # roots' dedup (before the slice) replaces block 0's + slice
            dedup_launches[0] = ((1 if 3 * batch <= 4096 else 3) if use_dedup else 0) + 1
        # per block: next_block, dedup, sample (count + pick), Q + K|V + FFN, split
        per_block = [(1 if l > 0 else 0) + dedup_launches[l] + 2 + 3 + (1 if self.split and l > 0
                                                                         else 0)
                     for l in range(self.L)]
        self.launches_per_forward = 1 + sum(per_block) + (1 if use_dedup and shard is None
                                                          else 0)
        if host_features:        # preload launches: edge rows per block, node rows (tail)
            self.launches_per_forward += (self.L if self.efeat_host is not None else 0) + 2
        # cache() (TGOpt per-layer store, Listing 1 L23; inference): every
        # block's dst pairs after dedup are looked up in that layer's table; only the
        # misses are sampled and computed, then stored, and the combine hook rebuilds the
        # block's rows in dedup order (b.comb) for the block above / the roots.
        self.cache_on = bool(cache_capacity)
        if self.cache_on:
            assert use_dedup, "cache() sits behind each block's dedup"
            for b in self.blocks:
                d = self.attn[b.layer].d_out
                c = {"table": tgl.EmbeddingCache(cache_capacity, d, self.dev),
                     "node": z(b.n_max, i32), "t": z(b.n_max, f32), "u": z(1, i64),
                     "slot": z(b.n_max, i32), "comb": z(b.n_max * d, f32).view(-1, d)}
                nb = tgl.ws_bytes("tgl_cache_lookup", None, b.n_max, None, None, None, None,
                                  None, None, None)
                c["ws"] = torch.empty(max(nb, 256), dtype=torch.uint8, device=self.dev)
                b.ws["cache"] = c
            self.launches_per_forward += 2 * self.L - 1   # lookups + merges - gather
        self._alloc_workspaces()
        self.graph_exec = None

    # ------------------------------------------------------------------ workspaces
    def _alloc_workspaces(self):
        k = self.sampler.k
        if self.shard is not None and self.use_dedup:
            nb = tgl.ws_bytes("tgl_dedup", 3 * self.batch, None, None, None, None, None, None,
                              None)
            self.roots_ws = torch.empty(max(nb, 256), dtype=torch.uint8, device=self.dev)
        for b in self.blocks:
            if self.use_dedup and b.inv is not None:
                nb = tgl.ws_bytes("tgl_dedup", b.n_max, None, None, None, None, None, None, None)
                b.ws["dedup"] = torch.empty(max(nb, 256), dtype=torch.uint8, device=self.dev)
            nb = tgl.ws_bytes("tgl_sample", C_TCSR(self.tcsr), b.n_max, None, None, None, k, 0,
                              0, 0, None, None, None, None)
            b.ws["sample"] = torch.empty(max(nb, 256), dtype=torch.uint8, device=self.dev)
            a = self.attn[b.layer]
            nb = tgl.ws_bytes("tgl_tblock_attn", C_ATTN(a), b.n_max, None, None, None, None, None,
                              0, None, None, None, 0, None, None, 0, None, None, 0, k, None)
            b.ws["attn"] = torch.empty(max(nb, 256), dtype=torch.uint8, device=self.dev)

    # ------------------------------------------------------------------ the batch
    def forward(self, stream=None, record: dict | None = None, slot: int = 0):
        """Enqueue one batch (edges [start, start+batch) with start = self.start_dev).

        record: optional dict; eager mode only -- CUDA events around each
        tgl_tblock_attn call are stored as record[layer] = (start, end).
        slot: sharded mode only -- which roots / send buffers this batch uses."""
        g, k, s = self.g, self.sampler.k, stream
        b0 = self.blocks[0]
        if self.shard is not None:
            return self._forward_sharded(slot, s, record)
        marks = None if record is None else record.setdefault("_marks", [])

        def mark(name):
            if marks is not None:
                ev = torch.cuda.Event(enable_timing=True)
                ev.record(s if s is not None else torch.cuda.current_stream())
                marks.append((name, ev))

        mark("start")
        if self.staging:
            st = self.stage
            tgl.batch_roots(self.batch, self.stage_n, None, st["src"], st["dst"], st["t"],
                            st["neg"], b0.dst_node, b0.dst_t, b0.n_dev, stream=s)
        else:
            tgl.batch_roots(self.batch, self.E, self.start_dev, g["src"], g["dst"], g["t"],
                            g["neg"], b0.dst_node, b0.dst_t, b0.n_dev, stream=s)
        mark("roots")
        return self._chain(s, record, mark)

    def _node_proj_fork(self, s):
        """Enqueue tgl_node_proj on the side stream, ordered after the work already on s."""
        cur = s if s is not None else torch.cuda.current_stream()
        self.np_fork.record(cur)
        self.np_stream.wait_event(self.np_fork)
        tgl.node_proj(self.attn[-1], self.nfeat_split, n_nodes=self.zproj.shape[0],
                      out=self.zproj, stream=self.np_stream)
        self.np_join.record(self.np_stream)

    def _chain(self, s, record, mark):
        """S3-S15 from block 0's dst pairs to the head output (b0.out / the roots)."""
        g, k = self.g, self.sampler.k
        if self.node_proj and record is None:
            self._node_proj_fork(s)
        b0 = self.blocks[0]
        for l, b in enumerate(self.blocks):
            if l > 0:  # S5 next_block (R14): [dst after dedup ; sampled src]
                p = self.blocks[l - 1]
                tgl.next_block(p.n_max, p.u_dev, p.uniq_node, p.uniq_t, p.n_max * k, p.seg_ptr,
                               p.nbr, p.ts, b.dst_node, b.dst_t, b.n_dev, stream=s)
                mark(f"next_block{l}")
            c = b.ws.get("cache")
            if self.use_dedup and b.inv is not None:  # S3
                un, ut, ud = ((c["node"], c["t"], c["u"]) if c is not None
                              else (b.uniq_node, b.uniq_t, b.u_dev))
                _call_ws(tgl.lib().tgl_dedup,
                         [b.n_max, tgl._p(b.n_dev), tgl._p(b.dst_node), tgl._p(b.dst_t),
                          tgl._p(un), tgl._p(ut), tgl._p(ud),
                          tgl._p(b.inv)], b.ws["dedup"], s, "tgl_dedup")
                mark(f"dedup{l}")
            if c is not None:  # cache() filter: the misses become the block's dsts
                _call_ws(tgl.lib().tgl_cache_lookup,
                         [tgl.C.byref(c["table"].struct), b.n_max, tgl._p(c["u"]),
                          tgl._p(c["node"]), tgl._p(c["t"]), tgl._p(c["slot"]),
                          tgl._p(b.uniq_node), tgl._p(b.uniq_t), tgl._p(b.u_dev)],
                         c["ws"], s, "tgl_cache_lookup")
                mark(f"cache_lookup{l}")
            # S4 sample
            _call_ws(tgl.lib().tgl_sample,
                     [tgl.C.byref(self.tcsr.struct), b.n_max, tgl._p(b.u_dev),
                      tgl._p(b.uniq_node), tgl._p(b.uniq_t), k,
                      tgl.STRATEGY[self.sampler.strategy], self.sampler.seed, l,
                      tgl._p(b.seg_ptr), tgl._p(b.nbr), tgl._p(b.eid), tgl._p(b.ts)],
                     b.ws["sample"], s, "tgl_sample")
            mark(f"sample{l}")
        # S15 aggregate: tail -> head
        for l in range(self.L - 1, -1, -1):
            b = self.blocks[l]
            a = self.attn[l]
            if l == self.L - 1:
                hdst, hdst_idx, hsrc, hsrc_idx, off = g["nfeat"], b.uniq_node, g["nfeat"], b.nbr, None
                if self.split:
                    hdst = hsrc = self.nfeat_split
                if self.node_proj:   # Z rows for every node, then the tail indexes them
                    if record is None:           # join the side stream (forked above)
                        (s if s is not None else torch.cuda.current_stream()).wait_event(
                            self.np_join)
                    else:                        # eager timing: in line, its own mark
                        tgl.node_proj(a, self.nfeat_split, n_nodes=self.zproj.shape[0],
                                      out=self.zproj, stream=s)
                        mark("node_proj")
            else:
                nx = self.blocks[l + 1]
                hdst = hsrc = nx.ws["cache"]["comb"] if self.cache_on else nx.out
                if self.split:
                    hdst = hsrc = nx.out_split
                off = b.u_dev        # S14: rows [U_l + e] of the next block hold the sources
                if self.use_dedup:
                    hdst_idx = hsrc_idx = nx.inv
                else:
                    hdst_idx = hsrc_idx = None
            ef = self.efeat_split if self.split else g["efeat"]
            eid = b.eid
            if self.host:        # N4 preload(): the block's rows from pinned host memory
                ef = None
                if self.efeat_host is not None:
                    ef, eid = b.ws["epre"], self.iota
                    tgl.preload_rows(b.eid, self.efeat_host, ef, n_max=b.n_max * k,
                                     n_dev=b.seg_ptr, n_at=b.u_dev, stream=s)
                if l == self.L - 1:
                    hsrc, hdst = b.ws["nsrc"], b.ws["ndst"]
                    tgl.preload_rows(b.nbr, self.nfeat_host, hsrc, n_max=b.n_max * k,
                                     n_dev=b.seg_ptr, n_at=b.u_dev, stream=s)
                    tgl.preload_rows(b.uniq_node, self.nfeat_host, hdst, n_max=b.n_max,
                                     n_dev=b.u_dev, stream=s)
                    hdst_idx = hsrc_idx = None
                mark(f"preload{l}")
            ld_e = ef.stride(0) if (ef is not None and ef.dim() == 2 and ef.shape[1] > 0) else 0
            if record is not None:
                ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                ev[0].record(s if s is not None else torch.cuda.current_stream())
            _call_ws(tgl.lib().tgl_tblock_attn,
                     [tgl.C.byref(a.struct), b.n_max, tgl._p(b.u_dev), tgl._p(b.seg_ptr),
                      tgl._p(b.uniq_t), tgl._prow(hdst), tgl._p(hdst_idx), hdst.stride(0),
                      tgl._prow(hsrc), tgl._p(hsrc_idx), tgl._p(off), hsrc.stride(0),
                      tgl._prow(ef) if ld_e else None, tgl._p(eid) if ld_e else None, ld_e,
                      tgl._p(b.ts), tgl._p(self.tables[l]),
                      0 if self.tables[l] is None else self.tables[l].shape[0], k,
                      tgl._p(b.out)], b.ws["attn"], s, "tgl_tblock_attn")
            if record is not None:
                ev[1].record(s if s is not None else torch.cuda.current_stream())
                record[l] = ev
            mark(f"attn{l}")
            if self.cache_on and l > 0:  # store the misses + combine hook, one launch
                c = b.ws["cache"]
                tgl.cache_merge(c["table"], c["node"], c["t"], c["slot"], b.out,
                                n_dev=c["u"], n_max=b.n_max, out=c["comb"], stream=s)
                mark(f"cache_merge{l}")
            if self.split and l > 0:     # the operands the layer above gathers (split16)
                tgl.split_rows(b.ws["cache"]["comb"] if self.cache_on else b.out,
                               out=b.out_split, n_rows=b.n_max, stream=s)
                mark(f"split{l}")
        if self.shard is not None:
            return b0.out
        if self.cache_on:  # head: store + combine + S14 inverse in one launch
            c = b0.ws["cache"]
            tgl.cache_merge(c["table"], c["node"], c["t"], c["slot"], b0.out, idx=b0.inv,
                            n_dev=b0.n_dev, n_max=b0.n_max, out=self.emb, stream=s)
            mark("cache_merge0")
            return self.emb
        head = b0.out
        if self.use_dedup:  # S14 at the roots
            tgl.gather_rows(b0.inv, head, n_dev=b0.n_dev, n_max=b0.n_max, out=self.emb, stream=s)
            mark("gather")
            return self.emb
        return b0.out[:3 * self.batch]

    def _forward_sharded(self, slot, s, record):
        b0 = self.blocks[0]
        marks = None if record is None else record.setdefault("_marks", [])

        def mark(name):
            if marks is not None:
                ev = torch.cuda.Event(enable_timing=True)
                ev.record(s if s is not None else torch.cuda.current_stream())
                marks.append((name, ev))

        mark("start")
        r = self.roots[slot]
        g = self.stage if self.staging else self.g
        tgl.batch_roots(self.batch, self.stage_n if self.staging else self.E,
                        None if self.staging else self.start_dev, g["src"], g["dst"], g["t"],
                        g["neg"], r["node"], r["t"], r["n"], stream=s)
        mark("roots")
        un, ut, un_dev = r["node"], r["t"], r["n"]
        if self.use_dedup:   # the roots' dedup, redundant on every rank (S3)
            _call_ws(tgl.lib().tgl_dedup,
                     [3 * self.batch, tgl._p(r["n"]), tgl._p(r["node"]), tgl._p(r["t"]),
                      tgl._p(r["unode"]), tgl._p(r["ut"]), tgl._p(r["u"]), tgl._p(r["inv"])],
                     self.roots_ws, s, "tgl_dedup")
            un, ut, un_dev = r["unode"], r["ut"], r["u"]
            mark("dedup_roots")
        rank, world = self.shard
        tgl.shard_slice(un, ut, rank, world, n_dev=un_dev, n_max=3 * self.batch,
                        out=(b0.dst_node, b0.dst_t, b0.n_dev), stream=s)
        mark("shard_slice")
        b0.out = self.send[slot]
        return self._chain(s, record, mark)

    def combine(self, slot: int, gathered: torch.Tensor, out: torch.Tensor | None = None,
                stream=None):
        """Root embeddings of the batch in `slot` from the all-gathered slices
        ([world * c_max, d], rank-major): S14 through the roots' inverse."""
        r = self.roots[slot]
        out = self.emb if out is None else out
        n0 = 3 * self.batch
        if self.use_dedup:
            return tgl.shard_gather(gathered, self.c_max, self.world, n0, u_dev=r["u"],
                                    idx=r["inv"], n_max=n0, n_dev=r["n"], out=out, stream=stream)
        return tgl.shard_gather(gathered, self.c_max, self.world, n0, u_dev=r["n"], idx=None,
                                n_max=n0, n_dev=r["n"], out=out, stream=stream)

    # ------------------------------------------------------------------ N2 backward
    def backward(self, grad_emb: torch.Tensor, grads: list | None = None, stream=None):
        """Training step of the TBlock chain: given dL/d(root embeddings)
        [3B, d_out] of the batch the last forward() ran, accumulate every layer's parameter
        gradients (grads[l]: tgl.zero_grads(attn[l]), created when None) -- the head block
        first, its input-row gradients routed to the block below through the same dedup
        hooks the forward used (S14 / S15 adjoints), down to the tail (raw features get
        none).  Needs fp32 feature tables (layout="fp32" or both tables present)."""
        assert self.shard is None and not self.cache_on, "backward: unsharded, no cache()"
        g = self.g
        assert g.get("efeat") is not None or self.attn[-1].host["d_e"] == 0, \
            "backward gathers fp32 edge rows"
        s = stream
        if grads is None:
            grads = [tgl.zero_grads(a) for a in self.attn]
        b0 = self.blocks[0]
        d0 = self.attn[0].d_out
        # S14 adjoint at the roots: dL/d(head rows) = scatter-add of dL/d(emb) through inv_0
        g_out = torch.zeros(b0.n_max, d0, device=self.dev)
        if self.use_dedup:
            tgl.scatter_add_rows(b0.inv, grad_emb, g_out, n_dev=b0.n_dev, n_max=b0.n_max,
                                 stream=s)
        else:
            tgl.scatter_add_rows(None, grad_emb, g_out, n_dev=b0.n_dev, n_max=b0.n_max,
                                 stream=s)
        k = self.sampler.k
        for l, b in enumerate(self.blocks):
            a = self.attn[l]
            tail = l == self.L - 1
            ef = g["efeat"] if a.host["d_e"] else None
            if tail:
                hdst = hsrc = g["nfeat"]
                hdst_idx, hsrc_idx, off, g_next = b.uniq_node, b.nbr, None, None
            else:
                nx = self.blocks[l + 1]
                hdst = hsrc = nx.out
                hdst_idx = hsrc_idx = nx.inv if self.use_dedup else None
                off = b.u_dev
                g_next = torch.zeros_like(nx.out)     # dL/d(rows of the block below)
            tgl.tblock_attn_backward(a, b.seg_ptr, b.uniq_t, hdst, hdst_idx, hsrc, hsrc_idx, ef,
                                     b.eid if ef is not None else None, b.ts, g_out, grads[l],
                                     g_next, g_next, n_dst_max=b.n_max, n_dst_dev=b.u_dev,
                                     n_edges_max=b.n_max * k, hsrc_off_dev=off, stream=s)
            g_out = g_next
        return grads

    # ------------------------------------------------------------------ CUDA graph
    def capture(self):
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            for _ in range(2):
                self.forward()
        torch.cuda.current_stream().wait_stream(s)
        torch.cuda.synchronize()
        if self.shard is not None:        # one graph per slot (its own roots / send)
            self.graphs = []
            for slot in range(2):
                gs = torch.cuda.CUDAGraph()
                with torch.cuda.graph(gs):
                    self.forward(slot=slot)
                self.graphs.append(gs)
            self.graph_exec, self.graph_out = self.graphs[0], self.send[0]
            return self.graphs
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            out = self.forward()
        self.graph_exec = g
        self.graph_out = out
        return g

    def run_graph(self, start: int | None = None, slot: int = 0):
        if start is not None:
            self.start_dev.fill_(start)
        if self.shard is not None:
            self.graphs[slot].replay()
            return self.send[slot]
        self.graph_exec.replay()
        return self.graph_out

    def embed_host(self, src_h, dst_h, t_h, neg_h, out_h):
        """Public end-to-end call: one batch from (pinned) host arrays to host embeddings.

        H2D of the batch's edges, the captured TBlock chain, D2H of the root
        embeddings; returns after the stream has finished."""
        assert self.staging and self.graph_exec is not None
        n = src_h.shape[0]
        assert n == self.batch, "staging pipeline is captured for a full batch"
        for k_, h in (("src", src_h), ("dst", dst_h), ("t", t_h), ("neg", neg_h)):
            self.stage[k_][:n].copy_(h, non_blocking=True)
        self.graph_exec.replay()
        out_h.copy_(self.graph_out[:3 * n], non_blocking=True)
        torch.cuda.current_stream().synchronize()
        return out_h


class HostStream:
    """Serving loop over a staging TGATPipeline: batch i's H2D, graph replay and D2H are
    enqueued without waiting for batch i-1's result to reach the host.  The root
    embeddings go through a 2-deep device ring (a D2D copy at the end of the step) and are
    read back on a side copy stream, so the D2H of batch i overlaps the compute of batch
    i+1.  Every batch still pays its own H2D (its edges) and D2H (its embeddings)."""

    def __init__(self, pipe: "TGATPipeline", n_out: int, d_out: int):
        assert pipe.staging and pipe.graph_exec is not None
        self.p = pipe
        self.n_out = n_out
        self.ring = [torch.empty(n_out, d_out, dtype=torch.float32, device=pipe.dev)
                     for _ in range(2)]
        self.copy_stream = torch.cuda.Stream()
        self.d2h_done = [None, None]
        self.i = 0

    def submit(self, src_h, dst_h, t_h, neg_h, out_h) -> torch.cuda.Event:
        """Enqueue one batch; returns the event after which out_h holds its embeddings."""
        p, slot = self.p, self.i % 2
        self.i += 1
        cs = torch.cuda.current_stream()
        n = src_h.shape[0]
        assert n == p.batch, "staging pipeline is captured for a full batch"
        for k_, h in (("src", src_h), ("dst", dst_h), ("t", t_h), ("neg", neg_h)):
            p.stage[k_][:n].copy_(h, non_blocking=True)
        p.graph_exec.replay()
        if self.d2h_done[slot] is not None:     # ring slot still being read back
            cs.wait_event(self.d2h_done[slot])
        self.ring[slot].copy_(p.graph_out[:self.n_out], non_blocking=True)
        ready = torch.cuda.Event()
        ready.record(cs)
        with torch.cuda.stream(self.copy_stream):
            self.copy_stream.wait_event(ready)
            out_h.copy_(self.ring[slot], non_blocking=True)
            done = torch.cuda.Event()
            done.record(self.copy_stream)
        self.d2h_done[slot] = done
        return done


def C_TCSR(t: tgl.TemporalCSR):
    return tgl.C.byref(t.struct)


def C_ATTN(a: tgl.AttnParams):
    return tgl.C.byref(a.struct)


def _call_ws(fn, args, ws_buf: torch.Tensor, stream, what):
    nb = tgl.C.c_size_t(ws_buf.numel())
    tgl._check(fn(*args, ws_buf.data_ptr(), tgl.C.byref(nb), tgl._s(stream)), what)
