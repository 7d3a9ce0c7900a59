"""Host-side checks of the C ABI that need no GPU (run on the CPU box).

- libtgl.so loads and exports every symbol include/tgl.h declares;
- the workspace-size protocol (ws == NULL) and host-side argument validation,
  which return before any launch.
"""
import ctypes as C
import os
import re

import pytest

from paper_conf_asplos_wangm24_b200 import tgl

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "tgl.h")).read()
    return sorted(set(re.findall(r"\b(tgl_[a-z_0-9]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    decl = declared_symbols()
    assert set(decl) == set(tgl.SYMBOLS)
    lib = C.CDLL(tgl.LIB_PATH)
    for name in decl:
        assert hasattr(lib, name), name


def test_version_and_status_strings():
    assert "sm_100a" in tgl.version()
    assert tgl.lib().tgl_status_string(0) == b"TGL_OK"
    assert tgl.lib().tgl_status_string(-2) == b"TGL_EWORKSPACE"


def test_workspace_queries_do_not_launch():
    # sizes grow with the problem and are 256-aligned chunks
    a = tgl.ws_bytes("tgl_dedup", 1000, None, None, None, None, None, None, None)
    b = tgl.ws_bytes("tgl_dedup", 100000, None, None, None, None, None, None, None)
    assert 0 < a < b
    g = tgl.TCSR(10, 0, None, None, None, None)
    s = tgl.ws_bytes("tgl_sample", C.byref(g), 5000, None, None, None, 10, 0, 0, 0, None, None,
                     None, None)
    assert s >= 8 * (5000 // 32)
    t = tgl.ws_bytes("tgl_build_tcsr", 100, 1000, None, None, None, 1, None, None, None, None)
    assert t >= 4 * 4 * 2000


def test_host_validation_errors():
    lib = tgl.lib()
    nb = C.c_size_t(0)
    g = tgl.TCSR(10, 0, None, None, None, None)
    # k <= 0
    st = lib.tgl_sample(C.byref(g), 10, None, None, None, 0, 0, 0, 0, None, None, None, None,
                        None, C.byref(nb), None)
    assert st == -1 and b"k must be" in lib.tgl_last_error()
    # bad strategy
    st = lib.tgl_sample(C.byref(g), 10, None, None, None, 3, 7, 0, 0, None, None, None, None,
                        None, C.byref(nb), None)
    assert st == -1
    # bad flags
    st = lib.tgl_build_tcsr(10, 10, None, None, None, 8, None, None, None, None, None,
                            C.byref(nb), None)
    assert st == -1
    # too many entries
    st = lib.tgl_build_tcsr(10, 1 << 31, None, None, None, 1, None, None, None, None, None,
                            C.byref(nb), None)
    assert st == -4
    # workspace too small (non-NULL ws, size 0) -> EWORKSPACE before any launch
    small = C.c_size_t(0)
    st = lib.tgl_dedup(100, None, None, None, None, None, None, None, C.c_void_p(256),
                       C.byref(small), None)
    assert st == -2
    # attention shape limits
    p = tgl.AttnParamsC(10, 10, 0, 100, 200, 2, 200)
    st = lib.tgl_tblock_attn(C.byref(p), 10, None, None, None, None, None, 10, None, None, None,
                             10, None, None, 0, None, None, 0, 10, None, None, C.byref(nb), None)
    assert st == -5
    p = tgl.AttnParamsC(10, 10, 0, 100, 100, 3, 100)
    st = lib.tgl_tblock_attn(C.byref(p), 10, None, None, None, None, None, 10, None, None, None,
                             10, None, None, 0, None, None, 0, 10, None, None, C.byref(nb), None)
    assert st == -1


def test_no_cpu_fallback_in_product():
    """The product package must not import the oracle or run compute on the host."""
    pkg = os.path.join(ROOT, "paper_conf_asplos_wangm24_b200")
    for fn in os.listdir(pkg):
        if fn.endswith(".py"):
            src = open(os.path.join(pkg, fn)).read()
            assert "import oracle" not in src and "from oracle" not in src, fn


def test_product_library_has_no_debug_surface():
    """Product builds export exactly the tgl.h entry points (the probe-only tgl_debug_*
    readers and any timing hooks exist only in -DTGL_PROBE builds) and read no
    environment variables (kernel choice is tgl_attn_params.kv_kernel)."""
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", tgl.LIB_PATH], capture_output=True,
                         text=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if ln.split()[-1].startswith("tgl_")}
    assert exported == set(declared_symbols()), exported ^ set(declared_symbols())
    blob = open(tgl.LIB_PATH, "rb").read()      # (cudart itself calls getenv: check ours)
    for var in (b"TGL_DEBUG_MASK", b"TGL_KV\x00"):
        assert var not in blob, var


def test_shard_validation_errors():
    lib = tgl.lib()
    # rank outside [0, world)
    st = lib.tgl_shard_slice(10, None, None, None, 2, 2, None, None, None, None)
    assert st == -1 and b"rank" in lib.tgl_last_error()
    # c_max smaller than ceil(u_max / world)
    st = lib.tgl_shard_gather(10, None, None, 10, None, 4, None, 2, 100, None, 100, None)
    assert st == -1 and b"c_max" in lib.tgl_last_error()


def test_node_proj_validation_errors():
    """tgl_node_proj rejects shapes / arguments before any launch (no GPU needed)."""
    lib = tgl.lib()
    # d_model != 100 -> EUNSUPPORTED
    p = tgl.AttnParamsC(172, 172, 172, 100, 64, 2, 64)
    st = lib.tgl_node_proj(C.byref(p), 10, None, 176, C.c_void_p(256), None)
    assert st == -5
    # d_hsrc != d_hdst (the tail block indexes one node table) -> EUNSUPPORTED
    p = tgl.AttnParamsC(172, 128, 172, 100, 100, 2, 100)
    st = lib.tgl_node_proj(C.byref(p), 10, None, 176, C.c_void_p(256), None)
    assert st == -5
    # no packed weights -> EINVAL
    p = tgl.AttnParamsC(172, 172, 172, 100, 100, 2, 100)
    st = lib.tgl_node_proj(C.byref(p), 10, None, 176, C.c_void_p(256), None)
    assert st == -1 and b"packed" in lib.tgl_last_error()
    # null Z -> EINVAL
    st = lib.tgl_node_proj(C.byref(p), 10, None, 176, None, None)
    assert st == -1


def test_bench_node_proj_accounting():
    """bench.algorithmic_kv: the node-projection plan counts what its kernel reads per edge
    (a Z row of 2 d_model floats + the e row + 12 B) and the MMAs over [e ; Phi] only."""
    import bench
    import synth
    cfg = synth.get_config("GDELT")
    f0, b0 = bench.algorithmic_kv(cfg, 132000, 1.32e6, cfg.d_v)
    f1, b1 = bench.algorithmic_kv(cfg, 132000, 1.32e6, cfg.d_v, node_proj=True)
    dm = cfg.d_model
    per_dst = 12 + 4 * (dm + 2) + 4 * dm
    assert b0 == 1.32e6 * (4 * (cfg.d_v + cfg.d_e) + 12) + 132000 * per_dst
    assert b1 == 1.32e6 * (4 * (2 * dm + cfg.d_e) + 12) + 132000 * per_dst
    assert f1 == 1.32e6 * (4 * dm * (cfg.d_e + cfg.d_t) + 6 * dm)
    assert f1 < f0 and b1 < b0
