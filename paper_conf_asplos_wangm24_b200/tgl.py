"""Thin ctypes binding of libtgl.so (include/tgl.h) -- argument marshalling only.

Every function takes CUDA torch tensors, passes their device pointers and the
current torch stream to the C ABI, and raises `TGLError` on a non-zero status.
No step of the method runs here: if libtgl.so is missing this module fails to
import (there is no CPU fallback).
"""
from __future__ import annotations

import ctypes as C
import os

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libtgl.so")

TGL_UNDIRECTED = 1
TGL_INPUT_TIME_SORTED = 2
RECENT, UNIFORM = 0, 1
FP32, BF16, FP32_SIMT = 0, 1, 2
# tgl_attn_params.kv_kernel (include/tgl.h TGL_KV_*)
KV_KERNEL = {"auto": 0, "split": 1, "split_pad": 2, "async": 3, "bin": 4, "general": 5,
             "pre": 7, "pre2": 8}
SPLIT_HSRC, SPLIT_E, SPLIT_TABLE, SPLIT_HDST, NODE_PROJ = 1, 2, 4, 8, 16
NODE_PROJ_LD = 512       # tgl.h TGL_NODE_PROJ_LD: Z row pitch (floats)
KV_KERNEL_NAME = {1: "kv_split_kernel (contiguous K plan)", 2: "kv_split_kernel (padded K plan)",
                  3: "kv_async_kernel", 4: "kv_bin_kernel", 5: "kv_kernel (general)",
                  6: "kv_attn_kernel (SIMT)", 7: "kv_pre_kernel (pre-split operands)",
                  8: "kv_pre2_kernel (pre-split operands, 2-SM MMA)"}
STRATEGY = {"recent": RECENT, "uniform": UNIFORM}
PRECISION = {"fp32": FP32, "bf16": BF16, "fp32_simt": FP32_SIMT}

SYMBOLS = ["tgl_version", "tgl_status_string", "tgl_last_error", "tgl_build_tcsr",
           "tgl_batch_roots", "tgl_dedup", "tgl_sample", "tgl_next_block",
           "tgl_time_precompute", "tgl_time_encode", "tgl_tblock_attn", "tgl_gather_rows",
           "tgl_attn_packed_bytes", "tgl_attn_pack", "tgl_cache_lookup", "tgl_cache_store", "tgl_cache_combine",
           "tgl_cache_merge", "tgl_shard_slice", "tgl_shard_gather", "tgl_split_rows",
           "tgl_tcsr_index", "tgl_tblock_attn_backward", "tgl_scatter_add_rows",
           "tgl_preload_rows", "tgl_mailbox_store", "tgl_memory_update", "tgl_build_tcsr_ex",
           "tgl_node_proj"]


class TGLError(RuntimeError):
    pass


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -m "
                          f"paper_conf_asplos_wangm24_b200.build` (no CPU fallback exists)")
    lib = C.CDLL(LIB_PATH)
    vp, i64, i32, u32, u64 = C.c_void_p, C.c_int64, C.c_int32, C.c_uint32, C.c_uint64
    sz = C.POINTER(C.c_size_t)
    lib.tgl_version.restype = C.c_char_p
    lib.tgl_status_string.restype = C.c_char_p
    lib.tgl_status_string.argtypes = [i32]
    lib.tgl_last_error.restype = C.c_char_p
    sig = {
        "tgl_build_tcsr": [i64, i64, vp, vp, vp, u32, vp, vp, vp, vp, vp, sz, vp],
        "tgl_build_tcsr_ex": [i64, i64, vp, vp, vp, u32, vp, vp, vp, vp, vp, vp, vp, sz, vp],
        "tgl_batch_roots": [i64, i64, vp, vp, vp, vp, vp, vp, vp, vp, vp],
        "tgl_dedup": [i64, vp, vp, vp, vp, vp, vp, vp, vp, sz, vp],
        "tgl_sample": [vp, i64, vp, vp, vp, i32, i32, u64, u32, vp, vp, vp, vp, vp, sz, vp],
        "tgl_next_block": [i64, vp, vp, vp, i64, vp, vp, vp, vp, vp, vp, vp],
        "tgl_time_precompute": [i64, i32, vp, vp, vp, vp],
        "tgl_time_encode": [i64, vp, i32, vp, vp, vp, i64, vp, vp],
        "tgl_tblock_attn": [vp, i64, vp, vp, vp, vp, vp, i64, vp, vp, vp, i64, vp, vp, i64, vp,
                            vp, i64, i32, vp, vp, sz, vp],
        "tgl_gather_rows": [i64, vp, vp, vp, i64, i32, vp, i64, vp],
        "tgl_attn_pack": [vp, vp, C.c_size_t, vp],
        "tgl_node_proj": [vp, i64, vp, i64, vp, vp],
        "tgl_cache_lookup": [vp, i64, vp, vp, vp, vp, vp, vp, vp, vp, sz, vp],
        "tgl_cache_store": [vp, i64, vp, vp, vp, vp, i64, vp],
        "tgl_cache_combine": [vp, i64, vp, vp, vp, i64, vp, i64, vp],
        "tgl_cache_merge": [vp, i64, vp, vp, vp, vp, vp, vp, i64, vp, i64, vp],
        "tgl_shard_slice": [i64, vp, vp, vp, i32, i32, vp, vp, vp, vp],
        "tgl_shard_gather": [i64, vp, vp, i64, vp, i32, vp, i64, i32, vp, i64, vp],
        "tgl_split_rows": [i64, i32, vp, i64, vp, i64, vp],
        "tgl_tcsr_index": [vp, vp, vp, vp],
        "tgl_scatter_add_rows": [i64, vp, vp, vp, i64, i32, vp, i64, vp],
        "tgl_preload_rows": [i64, vp, vp, vp, vp, i64, i64, vp, i64, vp],
        "tgl_mailbox_store": [vp, i64, vp, vp, vp, vp, vp, i64, vp, i64, vp, vp, vp, vp, sz, vp],
        "tgl_memory_update": [vp, vp, i64, vp, vp, vp, sz, vp],
        "tgl_tblock_attn_backward": [vp, i64, vp, i64, vp, vp, vp, vp, i64, vp, vp, vp, i64, vp,
                                     vp, i64, vp, vp, i64, vp, vp, i64, vp, i64, vp, sz, vp],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = i32
    lib.tgl_attn_packed_bytes.argtypes = [vp]
    lib.tgl_attn_packed_bytes.restype = C.c_size_t
    return lib


_lib = _load()


def lib():
    return _lib


def version() -> str:
    return _lib.tgl_version().decode()


def _check(status: int, what: str):
    if status != 0:
        raise TGLError(f"{what}: {_lib.tgl_status_string(status).decode()}: "
                       f"{_lib.tgl_last_error().decode()}")


def _p(t):
    if t is None:
        return None
    if isinstance(t, int):
        return t
    assert t.is_cuda and t.is_contiguous(), "expected a contiguous CUDA tensor"
    return t.data_ptr()


def _prow(t):
    """Pointer of a row table: contiguous, or a row-padded 2-D view (unit column
    stride, pitch = stride(0)) such as the 16-byte pitches the TMA gathers need."""
    if t is None:
        return None
    assert t.is_cuda and (t.is_contiguous() or (t.dim() == 2 and t.stride(1) == 1)), \
        "expected a CUDA row table with unit column stride"
    return t.data_ptr()


def _s(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


class Workspace:
    """Grow-only device scratch (uint8) owned by the caller, per the ABI."""

    def __init__(self, device=None):
        self.device = device or torch.device("cuda")
        self.buf = None

    def get(self, nbytes: int) -> torch.Tensor:
        nbytes = max(int(nbytes), 256)
        if self.buf is None or self.buf.numel() < nbytes:
            self.buf = torch.empty(nbytes, dtype=torch.uint8, device=self.device)
        return self.buf


def _ws_call(fn, args_before_ws, ws: Workspace | None, stream, what):
    """CUB-style protocol: query (ws=NULL) then call."""
    nb = C.c_size_t(0)
    _check(fn(*args_before_ws, None, C.byref(nb), stream), what + " (size query)")
    ws = ws or Workspace()
    buf = ws.get(nb.value)
    nb2 = C.c_size_t(buf.numel())
    _check(fn(*args_before_ws, buf.data_ptr(), C.byref(nb2), stream), what)


def ws_bytes(fn_name: str, *args_before_ws) -> int:
    nb = C.c_size_t(0)
    _check(getattr(_lib, fn_name)(*args_before_ws, None, C.byref(nb), None), fn_name)
    return nb.value


# --------------------------------------------------------------------------- S1
class TCSR(C.Structure):
    _fields_ = [("num_nodes", C.c_int64), ("num_entries", C.c_int64), ("indptr", C.c_void_p),
                ("nbr", C.c_void_p), ("eid", C.c_void_p), ("ts", C.c_void_p),
                ("ts_coarse", C.c_void_p), ("entries", C.c_void_p)]


class TemporalCSR:
    """Device-resident T-CSR + the host struct the ABI takes."""

    def __init__(self, indptr, nbr, eid, ts, coarse: bool = True, packed: bool = True,
                 stream=None, ts_coarse=None, entries=None):
        """coarse / packed: build the sampler's fence index (M/32 floats) and the packed
        16-byte entry records (16 B per entry) with tgl_tcsr_index, unless they are passed
        in already built (ts_coarse / entries, as tgl_build_tcsr_ex writes them)."""
        self.indptr, self.nbr, self.eid, self.ts = indptr, nbr, eid, ts
        M = nbr.numel()
        self.ts_coarse, self.entries = ts_coarse, entries
        self.struct = TCSR(indptr.numel() - 1, M, _p(indptr), _p(nbr), _p(eid), _p(ts),
                           _p(ts_coarse), _p(entries))
        if ts_coarse is not None or entries is not None:
            return
        if M > 0 and (coarse or packed):
            if coarse:
                self.ts_coarse = torch.empty((M + 31) // 32, dtype=torch.float32,
                                             device=ts.device)
            if packed:
                self.entries = torch.empty(M, 4, dtype=torch.int32, device=ts.device)
            _check(_lib.tgl_tcsr_index(C.byref(self.struct), _p(self.ts_coarse),
                                       _p(self.entries), _s(stream)), "tgl_tcsr_index")
            self.struct.ts_coarse = _p(self.ts_coarse)
            self.struct.entries = _p(self.entries)

    @property
    def num_nodes(self):
        return self.indptr.numel() - 1


def build_tcsr(num_nodes: int, src, dst, t, undirected=True, time_sorted=False,
               ws: Workspace | None = None, stream=None, coarse: bool = True,
               packed: bool = True) -> TemporalCSR:
    dev = src.device
    E = src.numel()
    M = 2 * E if undirected else E
    indptr = torch.empty(num_nodes + 1, dtype=torch.int64, device=dev)
    nbr = torch.empty(max(M, 1), dtype=torch.int32, device=dev)[:M]
    eid = torch.empty(max(M, 1), dtype=torch.int32, device=dev)[:M]
    ts = torch.empty(max(M, 1), dtype=torch.float32, device=dev)[:M]
    flags = (TGL_UNDIRECTED if undirected else 0) | (TGL_INPUT_TIME_SORTED if time_sorted else 0)
    # the sampler indexes are written by the same sweep (tgl_build_tcsr_ex)
    tsc = torch.empty((M + 31) // 32, dtype=torch.float32, device=dev) if coarse and M else None
    ent = torch.empty(M, 4, dtype=torch.int32, device=dev) if packed and M else None
    _ws_call(_lib.tgl_build_tcsr_ex, [num_nodes, E, _p(src), _p(dst), _p(t), flags, _p(indptr),
                                      _p(nbr), _p(eid), _p(ts), _p(tsc), _p(ent)], ws,
             _s(stream), "tgl_build_tcsr_ex")
    return TemporalCSR(indptr, nbr, eid, ts, coarse=False, packed=False, stream=stream,
                       ts_coarse=tsc, entries=ent)


# --------------------------------------------------------------------------- S2
def batch_roots(batch: int, num_edges: int, start_dev, src, dst, t, neg, qnode, qtime,
                n_roots_dev, stream=None):
    _check(_lib.tgl_batch_roots(batch, num_edges, _p(start_dev), _p(src), _p(dst), _p(t),
                                _p(neg), _p(qnode), _p(qtime), _p(n_roots_dev), _s(stream)),
           "tgl_batch_roots")


# --------------------------------------------------------------------------- S3
def dedup(node, t, n_dev=None, n_max=None, out=None, ws: Workspace | None = None, stream=None):
    """Returns (uniq_node, uniq_t, num_uniq_dev, inv) with capacity n_max."""
    n_max = node.numel() if n_max is None else n_max
    dev = node.device
    if out is None:
        out = (torch.empty(max(n_max, 1), dtype=torch.int32, device=dev),
               torch.empty(max(n_max, 1), dtype=torch.float32, device=dev),
               torch.zeros(1, dtype=torch.int64, device=dev),
               torch.empty(max(n_max, 1), dtype=torch.int32, device=dev))
    un, ut, nu, inv = out
    _ws_call(_lib.tgl_dedup, [n_max, _p(n_dev), _p(node), _p(t), _p(un), _p(ut), _p(nu), _p(inv)],
             ws, _s(stream), "tgl_dedup")
    return un, ut, nu, inv


# --------------------------------------------------------------------------- S4
def sample(g: TemporalCSR, qnode, qtime, k: int, strategy, seed: int = 0, layer: int = 0,
           nq_dev=None, nq_max=None, out=None, ws: Workspace | None = None, stream=None):
    """Returns (seg_ptr[nq_max+1], nbr, eid, ts) with capacity nq_max*k."""
    strategy = STRATEGY.get(strategy, strategy)
    nq_max = qnode.numel() if nq_max is None else nq_max
    dev = qnode.device
    cap = max(nq_max * k, 1)
    if out is None:
        out = (torch.empty(nq_max + 1, dtype=torch.int64, device=dev),
               torch.empty(cap, dtype=torch.int32, device=dev),
               torch.empty(cap, dtype=torch.int32, device=dev),
               torch.empty(cap, dtype=torch.float32, device=dev))
    seg, nb, ei, ts = out
    _ws_call(_lib.tgl_sample, [C.byref(g.struct), nq_max, _p(nq_dev), _p(qnode), _p(qtime), k,
                               strategy, seed & 0xFFFFFFFFFFFFFFFF, layer, _p(seg), _p(nb),
                               _p(ei), _p(ts)], ws, _s(stream), "tgl_sample")
    return seg, nb, ei, ts


# --------------------------------------------------------------------------- S5
def next_block(n_dst_max, n_dst_dev, dst_node, dst_t, n_src_max, seg_ptr, src_node, src_t,
               out_node, out_t, n_out_dev, stream=None):
    _check(_lib.tgl_next_block(n_dst_max, _p(n_dst_dev), _p(dst_node), _p(dst_t), n_src_max,
                               _p(seg_ptr), _p(src_node), _p(src_t), _p(out_node), _p(out_t),
                               _p(n_out_dev), _s(stream)), "tgl_next_block")


# --------------------------------------------------------------------------- S6
def time_precompute(window: int, omega, phi, stream=None):
    table = torch.empty(max(window, 1), omega.numel(), dtype=torch.float32, device=omega.device)
    _check(_lib.tgl_time_precompute(window, omega.numel(), _p(omega), _p(phi), _p(table),
                                    _s(stream)), "tgl_time_precompute")
    return table


def time_encode(dt, omega, phi, table=None, stream=None):
    n = dt.numel()
    out = torch.empty(max(n, 1), omega.numel(), dtype=torch.float32, device=dt.device)[:n]
    window = 0 if table is None else table.shape[0]
    _check(_lib.tgl_time_encode(n, _p(dt), omega.numel(), _p(omega), _p(phi), _p(table), window,
                                _p(out), _s(stream)), "tgl_time_encode")
    return out


# --------------------------------------------------------------------------- S7-S13
class AttnParamsC(C.Structure):
    _fields_ = [("d_hdst", C.c_int32), ("d_hsrc", C.c_int32), ("d_e", C.c_int32),
                ("d_t", C.c_int32), ("d_model", C.c_int32), ("n_heads", C.c_int32),
                ("d_out", C.c_int32),
                ("Wq", C.c_void_p), ("bq", C.c_void_p), ("Wk", C.c_void_p),
                ("bk", C.c_void_p), ("Wv", C.c_void_p), ("bv", C.c_void_p),
                ("Wo", C.c_void_p), ("bo", C.c_void_p), ("ln_gamma", C.c_void_p),
                ("ln_beta", C.c_void_p), ("ln_eps", C.c_float),
                ("omega", C.c_void_p), ("phi", C.c_void_p),
                ("leaky_slope", C.c_float), ("logit_scale", C.c_float),
                ("precision", C.c_int32), ("packed", C.c_void_p),
                ("kv_kernel", C.c_int32), ("probe", C.c_void_p),
                ("input_layout", C.c_int32), ("node_proj", C.c_void_p)]


class KvProbeC(C.Structure):
    _fields_ = [("ev_start", C.c_void_p), ("ev_stop", C.c_void_p), ("kernel", C.c_int32)]


class KvProbe:
    """Caller-owned measurement record (tgl.h tgl_kv_probe): two CUDA events the call
    records around its K|V attention kernel, and which kernel ran.  Attach with
    `AttnParams.attach_probe(p)` for eager calls only (never inside graph capture)."""

    def __init__(self):
        self.start = torch.cuda.Event(enable_timing=True)
        self.stop = torch.cuda.Event(enable_timing=True)
        self.start.record()                 # torch creates the CUDA events lazily
        self.stop.record()
        assert self.start.cuda_event and self.stop.cuda_event
        self.struct = KvProbeC(self.start.cuda_event, self.stop.cuda_event, -1)

    def ms(self) -> float:
        self.stop.synchronize()
        return self.start.elapsed_time(self.stop)

    @property
    def kernel(self) -> int:
        return int(self.struct.kernel)


_WEIGHTS = ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo", "ln_gamma", "ln_beta", "omega", "phi")


class AttnParams:
    """Device copies of one layer's weights + the host struct of the ABI.

    pack=True runs tgl_attn_pack once (tensor-core weight layout) so that every
    tgl_tblock_attn call streams the packed weights instead of re-packing them."""

    def __init__(self, p: dict, device=None, precision="fp32", pack: bool = False,
                 kv_kernel: str | int = "auto"):
        device = device or torch.device("cuda")
        self.host = p
        self.t = {k: torch.as_tensor(p[k], dtype=torch.float32).contiguous().to(device)
                  for k in _WEIGHTS}
        self.precision = PRECISION.get(precision, precision)
        self.d_model = p["d_model"]
        self.d_out = p["d_out"]
        self.d_t = p["d_t"]
        self.struct = AttnParamsC(p["d_hdst"], p["d_hsrc"], p["d_e"], p["d_t"], p["d_model"],
                                  p["n_heads"], p["d_out"],
                                  *[_p(self.t[k]) for k in _WEIGHTS[:10]], float(p["ln_eps"]),
                                  _p(self.t["omega"]), _p(self.t["phi"]),
                                  float(p["leaky_slope"]), float(p["logit_scale"]),
                                  self.precision, None,
                                  KV_KERNEL.get(kv_kernel, kv_kernel), None, 0, None)
        self.packed = None
        if pack and self.precision != FP32_SIMT:
            nb = _lib.tgl_attn_packed_bytes(C.byref(self.struct))
            self.packed = torch.empty(max(nb, 256), dtype=torch.uint8, device=device)
            _check(_lib.tgl_attn_pack(C.byref(self.struct), _p(self.packed), nb, _s()),
                   "tgl_attn_pack")
            self.struct.packed = _p(self.packed)

    def attach_probe(self, probe: "KvProbe | None"):
        """Record the next calls' K|V kernel into `probe` (None detaches)."""
        self._probe = probe
        self.struct.probe = None if probe is None else C.cast(C.pointer(probe.struct),
                                                              C.c_void_p).value

    def set_kv_kernel(self, kv_kernel: str | int):
        self.struct.kv_kernel = KV_KERNEL.get(kv_kernel, kv_kernel)


def node_proj(P: AttnParams, hnode, n_nodes: int | None = None, out=None, stream=None):
    """tgl_node_proj: Z [n_nodes, NODE_PROJ_LD] fp32 per-node projections of the split16
    node table `hnode` (needs P packed).  Attach with P.struct.node_proj + NODE_PROJ."""
    n = hnode.shape[0] if n_nodes is None else n_nodes
    if out is None:
        out = torch.empty(max(n, 1), NODE_PROJ_LD, dtype=torch.float32, device=hnode.device)
    _check(_lib.tgl_node_proj(C.byref(P.struct), n, _prow(hnode), hnode.stride(0), _p(out),
                              _s(stream)), "tgl_node_proj")
    return out


def tblock_attn(P: AttnParams, seg_ptr, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid,
                edge_t, table=None, max_seg=10, n_dst_max=None, n_dst_dev=None,
                hsrc_off_dev=None, out=None, ws: Workspace | None = None, stream=None):
    n_dst_max = seg_ptr.numel() - 1 if n_dst_max is None else n_dst_max
    if out is None:
        out = torch.empty(max(n_dst_max, 1), P.d_out, dtype=torch.float32,
                          device=seg_ptr.device)
    window = 0 if table is None else table.shape[0]
    # row pitches from the strides: row-padded views (16-byte pitches) are passed as is
    for t in (hdst, hsrc, efeat):
        if t is not None and t.dim() == 2 and t.shape[1] > 0 and t.stride(1) != 1:
            raise ValueError("feature tables need unit column stride")
    ld_e = efeat.stride(0) if (efeat is not None and efeat.dim() == 2 and efeat.shape[1]) else 0
    _ws_call(_lib.tgl_tblock_attn,
             [C.byref(P.struct), n_dst_max, _p(n_dst_dev), _p(seg_ptr), _p(dst_t), _prow(hdst),
              _p(hdst_idx), hdst.stride(0), _prow(hsrc), _p(hsrc_idx), _p(hsrc_off_dev),
              hsrc.stride(0), _prow(efeat) if ld_e else None, _p(eid) if ld_e else None, ld_e,
              _p(edge_t), _p(table), window, max_seg, _p(out)], ws, _s(stream),
             "tgl_tblock_attn")
    return out


# --------------------------------------------------------------------------- S14
def gather_rows(idx, table, n_dev=None, n_max=None, out=None, stream=None):
    n_max = idx.numel() if n_max is None else n_max
    d = table.shape[1]
    if out is None:
        out = torch.empty(max(n_max, 1), d, dtype=table.dtype, device=table.device)
    _check(_lib.tgl_gather_rows(n_max, _p(n_dev), _p(idx), _p(table), table.stride(0), d,
                                _p(out), out.stride(0), _s(stream)), "tgl_gather_rows")
    return out


# --------------------------------------------------------------------------- N1 cache()
class CacheC(C.Structure):
    _fields_ = [("capacity", C.c_int64), ("d", C.c_int32), ("keys", C.c_void_p),
                ("vals", C.c_void_p)]


class EmbeddingCache:
    """One layer's memo table (P:297 cache(); include/tgl.h tgl_cache): device keys
    [capacity] u64 (zeroed here, 0 = empty) and rows [capacity, d] fp32."""

    def __init__(self, capacity: int, d: int, device=None):
        dev = device or torch.device("cuda")
        self.keys = torch.zeros(capacity, dtype=torch.int64, device=dev)
        self.vals = torch.zeros(capacity, d, dtype=torch.float32, device=dev)
        self.struct = CacheC(capacity, d, self.keys.data_ptr(), self.vals.data_ptr())
        self.capacity, self.d = capacity, d

    def clear(self):
        self.keys.zero_()


def cache_lookup(cache: EmbeddingCache, node, t, n_dev=None, n_max=None, out=None,
                 ws: Workspace | None = None, stream=None):
    """Returns (slot[n_max], miss_node, miss_t, num_miss_dev)."""
    n_max = node.numel() if n_max is None else n_max
    dev = node.device
    if out is None:
        out = (torch.empty(max(n_max, 1), dtype=torch.int32, device=dev),
               torch.empty(max(n_max, 1), dtype=torch.int32, device=dev),
               torch.empty(max(n_max, 1), dtype=torch.float32, device=dev),
               torch.zeros(1, dtype=torch.int64, device=dev))
    slot, mn, mt, nm = out
    _ws_call(_lib.tgl_cache_lookup, [C.byref(cache.struct), n_max, _p(n_dev), _p(node), _p(t),
                                     _p(slot), _p(mn), _p(mt), _p(nm)], ws, _s(stream),
             "tgl_cache_lookup")
    return slot, mn, mt, nm


def cache_store(cache: EmbeddingCache, node, t, emb, n_dev=None, n_max=None, stream=None):
    n_max = node.numel() if n_max is None else n_max
    _check(_lib.tgl_cache_store(C.byref(cache.struct), n_max, _p(n_dev), _p(node), _p(t),
                                _p(emb), emb.stride(0), _s(stream)), "tgl_cache_store")


def cache_combine(cache: EmbeddingCache, slot, computed, n_dev=None, n_max=None, out=None,
                  stream=None):
    n_max = slot.numel() if n_max is None else n_max
    if out is None:
        out = torch.empty(max(n_max, 1), cache.d, dtype=torch.float32, device=slot.device)
    _check(_lib.tgl_cache_combine(C.byref(cache.struct), n_max, _p(n_dev), _p(slot),
                                  _p(computed), computed.stride(0), _p(out), out.stride(0),
                                  _s(stream)), "tgl_cache_combine")
    return out


def cache_merge(cache: EmbeddingCache, node, t, slot, computed, idx=None, n_dev=None,
                n_max=None, out=None, stream=None):
    """Store + combine in one launch; out[j] = merged row idx[j] (identity if None)."""
    n_max = (slot.numel() if idx is None else idx.numel()) if n_max is None else n_max
    if out is None:
        out = torch.empty(max(n_max, 1), cache.d, dtype=torch.float32, device=slot.device)
    _check(_lib.tgl_cache_merge(C.byref(cache.struct), n_max, _p(n_dev), _p(idx), _p(node),
                                _p(t), _p(slot), _p(computed), computed.stride(0), _p(out),
                                out.stride(0), _s(stream)), "tgl_cache_merge")
    return out


# --------------------------------------------------------------------------- S16 sharding
def shard_slice(node, t, rank: int, world: int, n_dev=None, n_max=None, out=None, stream=None):
    """Slice `rank` of the U = *n_dev unique roots: returns (node, t, n_dev) with capacity
    ceil(n_max / world)."""
    n_max = node.numel() if n_max is None else n_max
    cap = max(1, -(-n_max // world))
    dev = node.device
    if out is None:
        out = (torch.empty(cap, dtype=torch.int32, device=dev),
               torch.empty(cap, dtype=torch.float32, device=dev),
               torch.zeros(1, dtype=torch.int64, device=dev))
    on, ot, od = out
    _check(_lib.tgl_shard_slice(n_max, _p(n_dev), _p(node), _p(t), rank, world, _p(on), _p(ot),
                                _p(od), _s(stream)), "tgl_shard_slice")
    return on, ot, od


def shard_gather(gathered, c_max: int, world: int, u_max: int, u_dev=None, idx=None,
                 n_max=None, n_dev=None, out=None, stream=None):
    """Rebuild the batch's root rows from the all-gathered slices (rank-major, c_max rows
    each), through the roots' dedup inverse `idx` (None = identity)."""
    d = gathered.shape[1]
    n_max = (idx.numel() if idx is not None else u_max) if n_max is None else n_max
    if out is None:
        out = torch.empty(max(n_max, 1), d, dtype=torch.float32, device=gathered.device)
    _check(_lib.tgl_shard_gather(n_max, _p(n_dev), _p(idx), u_max, _p(u_dev), world,
                                 _p(gathered), c_max, d, _p(out), out.stride(0), _s(stream)),
           "tgl_shard_gather")
    return out


# --------------------------------------------------------------------------- split16 tables
def split_width(d: int) -> int:
    """Row pitch (4-byte words) of a split16 table of d columns."""
    return (d + 7) // 8 * 8


def split_rows(src, out=None, n_rows=None, stream=None):
    """fp32 [n, d] (unit column stride) -> split16 table viewed as float32 [n, dp]
    (bf16 hi of dp columns, then bf16 lo; tgl_split_rows)."""
    n = src.shape[0] if n_rows is None else n_rows
    d = src.shape[1]
    dp = split_width(d)
    if out is None:
        out = torch.empty(max(n, 1), dp, dtype=torch.float32, device=src.device)
    assert out.stride(1) == 1 and out.shape[1] >= dp
    _check(_lib.tgl_split_rows(n, d, _prow(src), src.stride(0), out.data_ptr(), out.stride(0),
                               _s(stream)), "tgl_split_rows")
    return out


def split_table(n_rows: int, d: int, make_rows, chunk_rows: int = 1 << 20, device=None,
                stream=None):
    """A split16 table of n_rows x d built chunk by chunk: make_rows(r0, r1) returns the fp32
    rows [r0, r1) on the device; each chunk is split into place, so the fp32 table never
    exists whole (GDELT's 142 GB of edge features)."""
    device = device or torch.device("cuda")
    dp = split_width(d)
    out = torch.empty(max(n_rows, 1), dp, dtype=torch.float32, device=device)
    for r0 in range(0, n_rows, chunk_rows):
        r1 = min(n_rows, r0 + chunk_rows)
        rows = make_rows(r0, r1)
        split_rows(rows, out=out[r0:r1], stream=stream)
        del rows
    return out


# --------------------------------------------------------------------------- N2 backward
GRAD_NAMES = ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo", "ln_gamma", "ln_beta", "omega",
              "phi")


class AttnGradsC(C.Structure):
    _fields_ = [(f"d{n}", C.c_void_p) for n in ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo",
                                                 "gamma", "beta", "omega", "phi")]


def zero_grads(P: AttnParams) -> dict:
    """Gradient accumulators (zeros) shaped like the layer's weights."""
    return {n: torch.zeros_like(P.t[n]) for n in GRAD_NAMES}


def tblock_attn_backward(P: AttnParams, seg_ptr, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat,
                         eid, edge_t, grad_out, grads: dict, grad_hdst=None, grad_hsrc=None,
                         n_dst_max=None, n_dst_dev=None, n_edges_max=None, hsrc_off_dev=None,
                         ws: Workspace | None = None, stream=None):
    """Backward of tgl_tblock_attn (N2): accumulates into `grads` (zero_grads) and, when
    given, into grad_hdst / grad_hsrc (row tables shaped like hdst / hsrc)."""
    n_dst_max = seg_ptr.numel() - 1 if n_dst_max is None else n_dst_max
    n_edges_max = (int(edge_t.numel()) if n_edges_max is None else n_edges_max)
    G = AttnGradsC(*[_p(grads[n]) for n in GRAD_NAMES])
    ld_e = efeat.stride(0) if (efeat is not None and efeat.dim() == 2 and efeat.shape[1]) else 0
    _ws_call(_lib.tgl_tblock_attn_backward,
             [C.byref(P.struct), n_dst_max, _p(n_dst_dev), n_edges_max, _p(seg_ptr), _p(dst_t),
              _prow(hdst), _p(hdst_idx), hdst.stride(0), _prow(hsrc), _p(hsrc_idx),
              _p(hsrc_off_dev), hsrc.stride(0), _prow(efeat) if ld_e else None,
              _p(eid) if ld_e else None, ld_e, _p(edge_t), _prow(grad_out), grad_out.stride(0),
              C.byref(G), _prow(grad_hdst), grad_hdst.stride(0) if grad_hdst is not None else 0,
              _prow(grad_hsrc), grad_hsrc.stride(0) if grad_hsrc is not None else 0], ws,
             _s(stream), "tgl_tblock_attn_backward")
    return grads


def scatter_add_rows(idx, src, out, n_dev=None, n_max=None, stream=None):
    """out[idx[j]] += src[j] for j < n (identity when idx is None)."""
    n_max = (src.shape[0] if idx is None else idx.numel()) if n_max is None else n_max
    _check(_lib.tgl_scatter_add_rows(n_max, _p(n_dev), _p(idx), _prow(src), src.stride(0),
                                     src.shape[1], _prow(out), out.stride(0), _s(stream)),
           "tgl_scatter_add_rows")
    return out


# --------------------------------------------------------------------------- N4 preload()
def preload_rows(idx, src, out, n_max=None, n_dev=None, n_at=None, stream=None):
    """out[j] = src[idx[j]] for j < n (n = n_dev[*n_at] or *n_dev, on the device); `src` may
    be a pinned host tensor (read by the GPU over the host link).  Row tables are 2-D with
    unit column stride; a row is src.shape[1] elements."""
    assert src.stride(1) == 1 and out.stride(1) == 1
    assert src.is_cuda or src.is_pinned(), "host tables must be pinned (page-locked)"
    n_max = (idx.numel() if idx is not None else src.shape[0]) if n_max is None else n_max
    es = src.element_size()
    _check(_lib.tgl_preload_rows(n_max, _p(n_dev), _p(n_at), _p(idx), src.data_ptr(),
                                 src.stride(0) * es, src.shape[1] * es, out.data_ptr(),
                                 out.stride(0) * out.element_size(), _s(stream)),
           "tgl_preload_rows")
    return out


# --------------------------------------------------------------------------- N3 TGN memory
class MemoryC(C.Structure):
    _fields_ = [("n_nodes", C.c_int64), ("d_mem", C.c_int32), ("d_e", C.c_int32),
                ("mem", C.c_void_p), ("mem_ts", C.c_void_p), ("mail", C.c_void_p),
                ("mail_ts", C.c_void_p)]


class GruParamsC(C.Structure):
    _fields_ = [("d_t", C.c_int32)] + [(n, C.c_void_p) for n in ("W_ih", "W_hh", "b_ih", "b_hh",
                                                                  "omega", "phi")]


class TGNMemory:
    """Node memory + one-slot mailbox of TGN (eqs 9-11, Listings 3-4), device fp32
    state owned here: mem [N, d_mem], mem_ts [N], mail [N, 2 d_mem + d_e], mail_ts [N]
    (all zero at start, as TGN's reset).  `params` = GRU + time-encoder weights
    (W_ih, W_hh, b_ih, b_hh, omega, phi as arrays / tensors)."""

    def __init__(self, n_nodes: int, d_mem: int, d_e: int, params: dict, device=None):
        dev = device or torch.device("cuda")
        f = lambda a: torch.as_tensor(a, dtype=torch.float32).to(dev).contiguous()
        self.n_nodes, self.d_mem, self.d_e = n_nodes, d_mem, d_e
        self.mem = torch.zeros(n_nodes, d_mem, device=dev)
        self.mem_ts = torch.zeros(n_nodes, device=dev)
        self.mail = torch.zeros(n_nodes, 2 * d_mem + d_e, device=dev)
        self.mail_ts = torch.zeros(n_nodes, device=dev)
        self.p = {k: f(params[k]) for k in ("W_ih", "W_hh", "b_ih", "b_hh", "omega", "phi")}
        assert self.p["W_ih"].shape[1] == 2 * d_mem + d_e + self.p["omega"].numel()
        self.struct = MemoryC(n_nodes, d_mem, d_e, self.mem.data_ptr(), self.mem_ts.data_ptr(),
                              self.mail.data_ptr(), self.mail_ts.data_ptr())
        self.gru = GruParamsC(self.p["omega"].numel(), *[self.p[k].data_ptr() for k in
                                                         ("W_ih", "W_hh", "b_ih", "b_hh",
                                                          "omega", "phi")])
        self.ws = Workspace(dev)

    def store(self, src, dst, t, efeat=None, eid=None, eid0: int = 0, B_dev=None, B_max=None,
              out=None, stream=None):
        """save_raw_msgs (Listing 4 L20-25): coalesce the batch's messages by latest and
        store them.  Returns (uniq [2B], pick [2B], n_uniq_dev [1])."""
        B_max = src.numel() if B_max is None else B_max
        dev = self.mem.device
        if out is None:
            out = (torch.empty(max(2 * B_max, 1), dtype=torch.int32, device=dev),
                   torch.empty(max(2 * B_max, 1), dtype=torch.int64, device=dev),
                   torch.empty(1, dtype=torch.int64, device=dev))
        uniq, pick, n_u = out
        ld_e = efeat.stride(0) if (efeat is not None and self.d_e) else 0
        _ws_call(_lib.tgl_mailbox_store,
                 [C.byref(self.struct), B_max, _p(B_dev), _p(src), _p(dst), _p(t), _p(eid), eid0,
                  _prow(efeat) if ld_e else None, ld_e, _p(uniq), _p(pick), _p(n_u)], self.ws,
                 _s(stream), "tgl_mailbox_store")
        return uniq, pick, n_u

    def update(self, nodes, n_dev=None, n_max=None, stream=None):
        """update_memory (Listing 4 L11-17, eq 11) for distinct nodes."""
        n_max = nodes.numel() if n_max is None else n_max
        _ws_call(_lib.tgl_memory_update,
                 [C.byref(self.struct), C.byref(self.gru), n_max, _p(n_dev), _p(nodes)], self.ws,
                 _s(stream), "tgl_memory_update")
