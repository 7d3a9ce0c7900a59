// common.cuh -- shared device/host helpers for libtgl (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include <atomic>

#include "../../include/tgl.h"

namespace tgl {

// ------------------------------------------------------------------ errors
void set_error(const char* fmt, ...);
tgl_status cuda_check(cudaError_t e, const char* what);
tgl_status launch_check(const char* what);

#define TGL_REQUIRE(cond, ...)            \
  do {                                    \
    if (!(cond)) {                        \
      ::tgl::set_error(__VA_ARGS__);      \
      return TGL_EINVAL;                  \
    }                                     \
  } while (0)

#define TGL_TRY(expr)                     \
  do {                                    \
    tgl_status _s = (expr);               \
    if (_s != TGL_OK) return _s;          \
  } while (0)

inline cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

// ------------------------------------------------------------------ workspace carving
struct WsLayout {
  size_t off = 0;
  size_t take(size_t bytes) {  // returns offset of a 256-aligned chunk
    size_t o = off;
    off += (bytes + 255) & ~size_t(255);
    return o;
  }
};

// ws == NULL -> report; else check size.  Returns TGL_OK and sets *done when only
// a size query was made.
inline tgl_status ws_protocol(void* ws, size_t* ws_bytes, size_t need, bool* query_only) {
  *query_only = false;
  if (ws_bytes == nullptr) {
    set_error("ws_bytes is NULL");
    return TGL_EINVAL;
  }
  if (ws == nullptr) {
    *ws_bytes = need;
    *query_only = true;
    return TGL_OK;
  }
  if (*ws_bytes < need) {
    set_error("workspace too small: %zu < %zu bytes", *ws_bytes, need);
    return TGL_EWORKSPACE;
  }
  if ((reinterpret_cast<uintptr_t>(ws) & 255) != 0) {
    set_error("workspace must be 256-byte aligned");
    return TGL_EINVAL;
  }
  return TGL_OK;
}

constexpr int kNumSMs = 148;

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------------------------ programmatic dependent launch
// Every kernel of a batch's launch chain is launched with programmatic stream
// serialisation: its CTAs may start (launch latency, constant staging, barrier init,
// TMEM allocation) while the previous kernel drains.  pdl_wait() (griddepcontrol.wait)
// blocks until the previous grid has completed and its writes are visible; EVERY thread
// of every PDL-launched kernel calls it before touching global data a predecessor wrote
// (and before exiting), so completion stays transitive along the chain.  pdl_trigger()
// lets the next kernel's CTAs be scheduled early.  Both are no-ops without the attribute.
__device__ __forceinline__ void pdl_wait() {
#ifndef TGL_NO_PDL
  asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}
__device__ __forceinline__ void pdl_trigger() {
#ifndef TGL_NO_PDL
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                              cudaStream_t s, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
#ifndef TGL_NO_PDL
  cfg.numAttrs = 1;
#else
  cfg.numAttrs = 0;
#endif
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// ------------------------------------------------------------------ device helpers
__device__ __forceinline__ int64_t dev_count(const int64_t* n_dev, int64_t n_max) {
  if (n_dev == nullptr) return n_max;
  int64_t n = *n_dev;
  return n < n_max ? n : n_max;
}

__device__ __forceinline__ uint32_t time_key_bits(float t) {
  // -0.0 and +0.0 are the same time (R8)
  return t == 0.0f ? 0u : __float_as_uint(t);
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T u = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += u;
  }
  return v;
}

// ------------------------------------------------------------------ single-pass scan state
// Decoupled look-back (Merrill & Garland) tile status: one 64-bit word per tile,
// flag in bits 62-63 (0 = not published, 1 = aggregate, 2 = inclusive prefix),
// value in bits 0-61.  Tiles take ids from an atomic ticket so a tile only ever
// waits on tiles that have already started.  Status words are read and written with
// relaxed gpu-scope accesses: a tile consumes only the status words themselves (no data
// published alongside them), and acquire loads would invalidate L1 on every poll
// (CCTL.IVALL in SASS -- the top stall of the T-CSR scatter before this).
constexpr unsigned long long kFlagAgg = 1ull << 62;
constexpr unsigned long long kFlagPrefix = 2ull << 62;
constexpr unsigned long long kValMask = (1ull << 62) - 1;

__device__ __forceinline__ void st_status(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_status(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Called by all 32 lanes of ONE warp.  Returns the exclusive prefix of `tile`.
__device__ __forceinline__ int64_t lookback(unsigned long long* status, int64_t tile,
                                            int64_t aggregate, int lane) {
  if (lane == 0)
    st_status(status + tile, (tile == 0 ? kFlagPrefix : kFlagAgg) | (unsigned long long)aggregate);
  if (tile == 0) return 0;
  int64_t excl = 0;
  int64_t base = tile - 1;
  while (true) {
    int64_t idx = base - lane;
    unsigned long long s = idx >= 0 ? ld_status(status + idx) : kFlagPrefix;
    unsigned flag = (unsigned)(s >> 62);
    unsigned pmask = __ballot_sync(0xffffffffu, flag == 2u);
    unsigned zmask = __ballot_sync(0xffffffffu, flag == 0u);
    int stop = pmask ? (__ffs(pmask) - 1) : 31;
    unsigned need = stop == 31 ? 0xffffffffu : ((1u << (stop + 1)) - 1u);
    if (zmask & need) continue;  // a predecessor has not published yet
    int64_t v = lane <= stop ? (int64_t)(s & kValMask) : 0;
    excl += warp_sum(v);
    if (pmask) break;
    base -= 32;
  }
  if (lane == 0) st_status(status + tile, kFlagPrefix | (unsigned long long)(excl + aggregate));
  return excl;
}

// ------------------------------------------------------------------ Philox4x32-10 (R6)
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
    k.x += 0x9E3779B9u;
    k.y += 0xBB67AE85u;
  }
  return c;
}


// cudaFuncSetAttribute applies per device: remember which device ordinals were set up
// (one bit each; atomic, so two threads racing on a new device merely repeat the
// idempotent call).  This is the library's only process state (tgl.h conventions).
struct PerDeviceOnce {
  std::atomic<unsigned long long> done{0};
  template <class F>
  cudaError_t run(F&& f) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const unsigned long long bit = dev < 64 ? (1ull << dev) : 0ull;
    if (bit && (done.load(std::memory_order_acquire) & bit)) return cudaSuccess;
    e = f();
    if (e == cudaSuccess && bit) done.fetch_or(bit, std::memory_order_acq_rel);
    return e;
  }
};

}  // namespace tgl
