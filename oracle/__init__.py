"""CPU oracle for the TBlock hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
`--impl reference`) may import this package.  It shares no code with the CUDA
path (paper_conf_asplos_wangm24_b200/); neither imports the other.  The only
module both sides use is `synth` (seeded input generation, no method
arithmetic).

The arithmetic lives in oracle.c (plain C, fp64 except where the paper's code
fixes fp32); this file is ctypes marshalling plus the block bookkeeping of
Listing 2 in `oracle.pipeline`.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-shared", "-fPIC",
          "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> oracle/liboracle.so (gcc)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
        i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
        f32p = np.ctypeslib.ndpointer(np.float32, flags="C_CONTIGUOUS")
        f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")
        u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")
        L.or_num_threads.restype = C.c_int
        L.or_set_num_threads.argtypes = [C.c_int]
        L.or_tcsr_num_entries.restype = C.c_int64
        L.or_tcsr_num_entries.argtypes = [C.c_int64, C.c_int]
        L.or_build_tcsr.restype = C.c_int
        L.or_build_tcsr.argtypes = [C.c_int64, C.c_int64, i32p, i32p, f32p, C.c_int,
                                    i64p, i32p, i32p, f32p]
        L.or_philox4x32_10.argtypes = [u32p, u32p, u32p]
        L.or_sample.restype = C.c_int
        L.or_sample.argtypes = [C.c_int64, i64p, i32p, i32p, f32p, C.c_int64, i32p, f32p,
                                C.c_int32, C.c_int32, C.c_uint64, C.c_uint32, i64p, i32p,
                                i32p, f32p]
        L.or_sample_keyed.restype = C.c_int
        L.or_sample_keyed.argtypes = [C.c_int64, i64p, i32p, i32p, f32p, C.c_int64, i32p, i32p,
                                      f32p, C.c_int32, C.c_int32, C.c_uint64, C.c_uint32, i64p,
                                      i32p, i32p, f32p]
        L.or_dedup.restype = C.c_int64
        L.or_dedup.argtypes = [C.c_int64, i32p, f32p, i32p, f32p, i32p]
        L.or_time_encode.argtypes = [C.c_int64, f32p, C.c_int32, f32p, f32p, f32p]
        L.or_time_precompute.argtypes = [C.c_int64, C.c_int32, f32p, f32p, f32p]
        L.or_tblock_attn.restype = C.c_int
        L.or_tblock_attn.argtypes = [C.c_void_p, C.c_int64, i64p, f32p, f32p, C.c_void_p,
                                     C.c_int64, f32p, i32p, C.c_int64, C.c_void_p,
                                     C.c_void_p, C.c_int64, f32p, f64p]
        L.or_embed_recursive.argtypes = [C.c_void_p, C.c_int64, i32p, f32p, f64p]
        _lib = L
    return _lib


def num_threads() -> int:
    return lib().or_num_threads()


def set_num_threads(n: int) -> None:
    lib().or_set_num_threads(int(n))


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


# --------------------------------------------------------------------------
# S1  T-CSR
# --------------------------------------------------------------------------
def build_tcsr(num_nodes: int, src, dst, t, undirected: bool = True):
    src, dst, t = _c(src, np.int32), _c(dst, np.int32), _c(t, np.float32)
    E = src.shape[0]
    M = lib().or_tcsr_num_entries(E, int(undirected))
    indptr = np.zeros(num_nodes + 1, np.int64)
    nbr = np.zeros(M, np.int32)
    eid = np.zeros(M, np.int32)
    ts = np.zeros(M, np.float32)
    rc = lib().or_build_tcsr(num_nodes, E, src, dst, t, int(undirected), indptr, nbr, eid, ts)
    if rc != 0:
        raise ValueError("node id out of range")
    return indptr, nbr, eid, ts


# --------------------------------------------------------------------------
# Philox4x32-10 and S4 sampling
# --------------------------------------------------------------------------
def philox4x32_10(ctr, key) -> np.ndarray:
    out = np.zeros(4, np.uint32)
    lib().or_philox4x32_10(_c(ctr, np.uint32), _c(key, np.uint32), out)
    return out


RECENT, UNIFORM = 0, 1


def sample(tcsr, qnode, qtime, k: int, strategy: int, seed: int = 0, layer: int = 0):
    indptr, nbr, eid, ts = tcsr
    qnode, qtime = _c(qnode, np.int32), _c(qtime, np.float32)
    nq = qnode.shape[0]
    seg_ptr = np.zeros(nq + 1, np.int64)
    cap = max(nq * k, 1)
    o_nbr = np.zeros(cap, np.int32)
    o_eid = np.zeros(cap, np.int32)
    o_ts = np.zeros(cap, np.float32)
    rc = lib().or_sample(indptr.shape[0] - 1, indptr, nbr, eid, ts, nq, qnode, qtime, k,
                         strategy, C.c_uint64(seed & 0xFFFFFFFFFFFFFFFF), layer, seg_ptr,
                         o_nbr, o_eid, o_ts)
    if rc != 0:
        raise ValueError("bad sample arguments")
    m = int(seg_ptr[-1])
    return seg_ptr, o_nbr[:m].copy(), o_eid[:m].copy(), o_ts[:m].copy()


def sample_keyed(tcsr, qnode, qkey, qtime, k: int, strategy: int, seed: int = 0,
                 layer: int = 0):
    """`sample` on a CSR whose owners are renumbered: qkey = original node ids (R6 key)."""
    indptr, nbr, eid, ts = tcsr
    qnode, qkey, qtime = _c(qnode, np.int32), _c(qkey, np.int32), _c(qtime, np.float32)
    nq = qnode.shape[0]
    seg_ptr = np.zeros(nq + 1, np.int64)
    cap = max(nq * k, 1)
    o_nbr = np.zeros(cap, np.int32)
    o_eid = np.zeros(cap, np.int32)
    o_ts = np.zeros(cap, np.float32)
    rc = lib().or_sample_keyed(indptr.shape[0] - 1, indptr, nbr, eid, ts, nq, qnode, qkey,
                               qtime, k, strategy, seed & 0xFFFFFFFFFFFFFFFF, layer, seg_ptr,
                               o_nbr, o_eid, o_ts)
    if rc != 0:
        raise ValueError("bad sample arguments")
    m = int(seg_ptr[-1])
    return seg_ptr, o_nbr[:m].copy(), o_eid[:m].copy(), o_ts[:m].copy()


# --------------------------------------------------------------------------
# S3 dedup
# --------------------------------------------------------------------------
def dedup(node, t):
    node, t = _c(node, np.int32), _c(t, np.float32)
    n = node.shape[0]
    un = np.zeros(max(n, 1), np.int32)
    ut = np.zeros(max(n, 1), np.float32)
    inv = np.zeros(max(n, 1), np.int32)
    U = lib().or_dedup(n, node, t, un, ut, inv)
    return un[:U].copy(), ut[:U].copy(), inv[:n].copy()


# --------------------------------------------------------------------------
# S6 time encoding (eq 8)
# --------------------------------------------------------------------------
def time_encode(dt, omega, phi) -> np.ndarray:
    dt = _c(dt, np.float32)
    omega, phi = _c(omega, np.float32), _c(phi, np.float32)
    out = np.zeros((dt.shape[0], omega.shape[0]), np.float32)
    lib().or_time_encode(dt.shape[0], dt, omega.shape[0], omega, phi, out)
    return out


def time_precompute(window: int, omega, phi) -> np.ndarray:
    omega, phi = _c(omega, np.float32), _c(phi, np.float32)
    out = np.zeros((window, omega.shape[0]), np.float32)
    lib().or_time_precompute(window, omega.shape[0], omega, phi, out)
    return out


# --------------------------------------------------------------------------
# S7-S13 TBlock attention (eqs 4-7)
# --------------------------------------------------------------------------
class _AttnParams(C.Structure):
    _fields_ = [("d_hdst", C.c_int32), ("d_hsrc", C.c_int32), ("d_e", C.c_int32),
                ("d_t", C.c_int32), ("d_model", C.c_int32), ("n_heads", C.c_int32),
                ("d_out", C.c_int32),
                ("Wq", C.c_void_p), ("bq", C.c_void_p), ("Wk", C.c_void_p),
                ("bk", C.c_void_p), ("Wv", C.c_void_p), ("bv", C.c_void_p),
                ("Wo", C.c_void_p), ("bo", C.c_void_p), ("ln_gamma", C.c_void_p),
                ("ln_beta", C.c_void_p), ("ln_eps", C.c_float),
                ("omega", C.c_void_p), ("phi", C.c_void_p),
                ("leaky_slope", C.c_float), ("logit_scale", C.c_float)]


def _params_struct(p: dict):
    keep = {}
    for name in ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo", "ln_gamma", "ln_beta",
                 "omega", "phi"):
        keep[name] = _c(p[name], np.float32)
    s = _AttnParams(p["d_hdst"], p["d_hsrc"], p["d_e"], p["d_t"], p["d_model"], p["n_heads"],
                    p["d_out"], *[keep[n].ctypes.data for n in
                                  ("Wq", "bq", "Wk", "bk", "Wv", "bv", "Wo", "bo",
                                   "ln_gamma", "ln_beta")],
                    float(p["ln_eps"]), keep["omega"].ctypes.data, keep["phi"].ctypes.data,
                    float(p["leaky_slope"]), float(p["logit_scale"]))
    return s, keep


def tblock_attn(p: dict, seg_ptr, dst_t, hdst, hdst_idx, hsrc, hsrc_idx, efeat, eid,
                edge_t) -> np.ndarray:
    """Returns fp64 [n_dst, d_out].  hdst_idx None = identity."""
    s, keep = _params_struct(p)
    seg_ptr = _c(seg_ptr, np.int64)
    n_dst = seg_ptr.shape[0] - 1
    dst_t = _c(dst_t, np.float32)
    hdst = _c(hdst, np.float32)
    hsrc = _c(hsrc, np.float32)
    hsrc_idx = _c(hsrc_idx, np.int32)
    edge_t = _c(edge_t, np.float32)
    hidx = None if hdst_idx is None else _c(hdst_idx, np.int32)
    ef = _c(efeat, np.float32) if p["d_e"] > 0 else None
    ei = _c(eid, np.int32) if p["d_e"] > 0 else None
    out = np.zeros((n_dst, p["d_out"]), np.float64)
    rc = lib().or_tblock_attn(C.byref(s), n_dst, seg_ptr, dst_t, hdst,
                              None if hidx is None else hidx.ctypes.data,
                              hdst.shape[1] if hdst.ndim == 2 else 0, hsrc, hsrc_idx,
                              hsrc.shape[1] if hsrc.ndim == 2 else 0,
                              None if ef is None else ef.ctypes.data,
                              None if ei is None else ei.ctypes.data,
                              ef.shape[1] if ef is not None else 0, edge_t, out)
    if rc != 0:
        raise ValueError("bad attention parameters")
    del keep
    return out


class _Model(C.Structure):
    _fields_ = [("num_nodes", C.c_int64), ("indptr", C.c_void_p), ("nbr", C.c_void_p),
                ("eid", C.c_void_p), ("ts", C.c_void_p), ("nfeat", C.c_void_p),
                ("d_v", C.c_int64), ("efeat", C.c_void_p), ("d_e", C.c_int64),
                ("k", C.c_int32), ("strategy", C.c_int32), ("n_layers", C.c_int32),
                ("seed", C.c_uint64), ("params", C.c_void_p)]


def embed_recursive(tcsr, nfeat, efeat, params: list, k: int, strategy: int, seed: int,
                    node, t) -> np.ndarray:
    """Listing 1 recursive embedding of roots -> fp64 [n, d_out]."""
    indptr, nbr, eid, ts = [np.ascontiguousarray(a) for a in tcsr]
    nfeat = _c(nfeat, np.float32)
    efeat = _c(efeat, np.float32)
    structs, keeps = [], []
    for p in params:
        s, kp = _params_struct(p)
        structs.append(s)
        keeps.append(kp)
    arr = (_AttnParams * len(params))(*structs)
    M = _Model(indptr.shape[0] - 1, indptr.ctypes.data, nbr.ctypes.data, eid.ctypes.data,
               ts.ctypes.data, nfeat.ctypes.data, nfeat.shape[1], efeat.ctypes.data,
               efeat.shape[1] if efeat.ndim == 2 else 0, k, strategy, len(params),
               seed & 0xFFFFFFFFFFFFFFFF, C.cast(arr, C.c_void_p))
    node, t = _c(node, np.int32), _c(t, np.float32)
    out = np.zeros((node.shape[0], params[0]["d_out"]), np.float64)
    lib().or_embed_recursive(C.byref(M), node.shape[0], node, t, out)
    del keeps
    return out
