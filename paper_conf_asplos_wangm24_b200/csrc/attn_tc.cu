// attn_tc.cu -- S7-S13 on the 5th-generation tensor cores (tcgen05 + TMEM).
//
// Same math as attn.cu (eqs 4-7; Listing 2), with the three
// projections as tcgen05.mma GEMMs whose A operand is GATHERED on the fly:
//   prep   : W{q,kv,o} fp32 -> bf16 hi/lo pairs, K laid out as [seg0|seg1|seg2]
//            (each padded to 8) and pre-swizzled into the exact SW128 shared-memory
//            image of a 64-wide K chunk, so the mainloop moves them with ONE
//            cp.async.bulk per chunk (TMA engine, mbarrier complete_tx).
//   q      : q_i = Wq [h_i ; Phi(0)] + bq                       (S8)
//   kv     : per destination group, 128 edge rows per M-tile: producers gather
//            [h_src ; e ; Phi(dt)] rows (S6+S7 fused: vector loads + cosf / table),
//            split fp32 -> bf16 hi + lo and store them swizzled; one thread issues
//            tcgen05.mma into a TMEM accumulator [128 x 2*d_model] (K|V, S9);
//            the epilogue reads TMEM (tcgen05.ld), forms logits + LeakyReLU (S10),
//            runs the online segmented softmax (S11) and the alpha-weighted
//            scatter-sum (S12) in shared memory -- deterministic order, no atomics.
//   ffn    : out_i = LayerNorm(ReLU(Wo [r_i ; h_i] + bo))          (S13)
// Precision: TGL_FP32 = 3 bf16 passes (hi*hi + lo*hi + hi*lo, fp32 accumulate;
// operand error ~2^-16, inside the 1e-3 contract); TGL_BF16 = 1 pass.
// Pipeline: 2 smem stages; the gather of chunk c+1 overlaps the MMAs of chunk c.
#include <cuda_bf16.h>
#include <stdlib.h>
#include <string.h>

#include "common.cuh"
#include "tc.cuh"
#include "tenc.cuh"

namespace tgl {
namespace tca {

using namespace tc;

constexpr int kThreads = 256;
constexpr int kBM = 128;
constexpr int kChunk = 64;                 // bf16 K elements per chunk (one 128 B swizzle row)
constexpr int kAPart = kBM * 128;          // bytes of A_hi (or A_lo) per stage
constexpr int kMaxDpb = 16;
constexpr int kQLd = 128;                  // q / r scratch leading dim (floats)
constexpr int kDPN = 104;                  // d_model padded to 8: N of dense_pre, r split16 width
constexpr int kMaxModel = 128;

__host__ __device__ __forceinline__ int pad8(int x) { return (x + 7) & ~7; }

struct Seg3 {
  int d0, d1, d2;  // true widths of [seg0 | seg1 | time]
  int p0, p1, p2;  // padded to multiples of 8
  int kpad, nchunks;
};

static Seg3 make_seg3(int d0, int d1, int d2) {
  Seg3 s;
  s.d0 = d0; s.d1 = d1; s.d2 = d2;
  s.p0 = pad8(d0); s.p1 = pad8(d1); s.p2 = pad8(d2);
  s.kpad = s.p0 + s.p1 + s.p2;
  s.nchunks = (s.kpad + kChunk - 1) / kChunk;
  return s;
}

// ------------------------------------------------------------------ weight packing
struct PackJob {
  const float* W0;  // rows [0, n0)
  const float* W1;  // rows [n0, n)   (may be null when n0 == n)
  int n0, n, np, ksrc;
  Seg3 sg;
  uint8_t* out;     // nchunks * 2 * np * 128 bytes
};

__global__ void pack_weights_kernel(PackJob j0, PackJob j1, PackJob j2) {
  const PackJob& J = blockIdx.y == 0 ? j0 : (blockIdx.y == 1 ? j1 : j2);
  const int kw = J.sg.nchunks * kChunk;
  const int64_t total = (int64_t)J.np * kw;
  const int chunk_bytes = 2 * J.np * 128;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(x / kw), kp = (int)(x % kw);
    float v = 0.f;
    if (n < J.n) {
      const float* row = n < J.n0 ? J.W0 + (int64_t)n * J.ksrc : J.W1 + (int64_t)(n - J.n0) * J.ksrc;
      int src = -1;
      if (kp < J.sg.p0) {
        if (kp < J.sg.d0) src = kp;
      } else if (kp < J.sg.p0 + J.sg.p1) {
        const int lc = kp - J.sg.p0;
        if (lc < J.sg.d1) src = J.sg.d0 + lc;
      } else if (kp < J.sg.kpad) {
        const int lc = kp - J.sg.p0 - J.sg.p1;
        if (lc < J.sg.d2) src = J.sg.d0 + J.sg.d1 + lc;
      }
      if (src >= 0) v = row[src];
    }
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    const int c = kp / kChunk, cc = kp % kChunk, jj = cc >> 3, e = cc & 7;
    const int64_t off = (int64_t)c * chunk_bytes + (n >> 3) * 1024 + (n & 7) * 128 +
                        ((jj ^ (n & 7)) << 4) + e * 2;
    *reinterpret_cast<__nv_bfloat16*>(J.out + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(J.out + off + J.np * 128) = lo;
  }
}

// ------------------------------------------------------------------ shared state
struct Args {
  tgl_attn_params P;
  int64_t n_dst_max;
  const int64_t* n_dst_dev;
  const int64_t* seg_ptr;
  const float* dst_t;
  const float* hdst;
  const int32_t* hdst_idx;
  int64_t ld_hdst;
  const float* hsrc;
  const int32_t* hsrc_idx;
  const int64_t* hsrc_off_dev;
  int64_t ld_hsrc;
  const float* efeat;
  const int32_t* eid;
  int64_t ld_e;
  const float* edge_t;
  const float* table;
  int64_t window;
  float* out;
  float* qbuf;
  float* rbuf;
  uint8_t* rsplit;     // split16 r rows [n_dst_max][104 words] for dense_pre FFN (or null)
  const uint8_t* wq;   // packed
  const uint8_t* wkv;
  const uint8_t* wo;
  Seg3 sq, skv, so;
  int np_q, np_kv, np_o;
  int dpb;
  int split;           // 1 = 3-pass fp32 mode
  // node projections (TGL_NODE_PROJ, tgl_node_proj): per-node rows of Z [n_nodes][z_ld]
  // = [h Wk_h^T | h Wv_h^T | pad | q (+ q.b_k) | h Wo_h^T]; the K|V accumulator starts
  // from zkv[row], the FFN adds zo[row]; the epilogue reads q row q_idx[d] (stride q_ld)
  const float* zkv;
  const float* zo;
  int64_t z_ld;
  const int32_t* q_idx;
  int64_t q_ld;
  int dbg;             // TGL_DEBUG_MASK (profiling only): 1 skip epilogue math, 2 skip gathers, 4 skip MMAs
};

// an empty (0) or overflowed (NaN) segment's r row, called by one warp: fp32 scratch row, or
// the split16 row dense_pre gathers (hi = value, lo = 0, padding columns 100..103 zero)
__device__ __forceinline__ void fill_r_row(const Args& a, int64_t row, float fill, int lane,
                                           int dm) {
  if (a.rsplit == nullptr) {
    for (int c = lane; c < dm; c += 32) a.rbuf[row * kQLd + c] = fill;
    return;
  }
  uint16_t* rp = reinterpret_cast<uint16_t*>(a.rsplit + row * (4 * kDPN));
  const __nv_bfloat16 h = __float2bfloat16_rn(fill);
  const uint16_t hb = *reinterpret_cast<const uint16_t*>(&h);
  for (int c = lane; c < kDPN; c += 32) {
    rp[c] = c < dm ? hb : (uint16_t)0;
    rp[kDPN + c] = c < dm && fill != fill ? hb : (uint16_t)0;
  }
}

// offset (not integer round-trip) so the compiler keeps the shared address space
__device__ __forceinline__ uint8_t* align1024(uint8_t* p) {
  return p + ((1024u - (static_cast<uint32_t>(__cvta_generic_to_shared(p)) & 1023u)) & 1023u);
}

// ------------------------------------------------------------------ warp-specialized CTA
// 15 warps: 0-3 epilogue (TMEM lane quarter = warp), 4 MMA issuer, 5 row-descriptor
// builder, 6 weight loader (bulk copies), 7-14 producers (gather -> bf16 hi/lo ->
// swizzled smem).  Rings: A (gathered rows) 2 stages, W (weights) 2 stages,
// row descriptors 3 slots, TMEM accumulators 2.  mbarriers only in the steady state.
constexpr int kEpiWarps = 4;
constexpr int kMmaWarp = 4;
constexpr int kDescWarp = 5;
constexpr int kWWarp = 6;
constexpr int kProdWarp0 = 7;
constexpr int kProdWarps = 16;
constexpr int kGPT = 1024 / (kProdWarps * 32);   // 16-byte groups per producer thread per chunk
constexpr int kGPR = 8 / kGPT;                    // producer threads per row
constexpr int kProdThreads = kProdWarps * 32;
constexpr int kWsThreads = (kProdWarp0 + kProdWarps) * 32;   // 736
constexpr int kAStages = 2;
constexpr int kWStages = 2;
constexpr int kDSlots = 3;
constexpr int kBarEpi = 2;    // named barrier id for the 4 epilogue warps

struct RowDesc {
  const float* p0[kBM];
  const float* p1[kBM];
  float dt[kBM];
  int trow[kBM];
  int rdst[kBM];
};

struct Bars {
  uint64_t afull[kAStages], aempty[kAStages];
  uint64_t wfull[kWStages], wempty[kWStages];
  uint64_t dfull[kDSlots], dempty[kDSlots];
  uint64_t tfull[2], tempty[2];
};

template <int NP>
struct Pipe {
  static constexpr int kAStage = 2 * kAPart;        // A_hi | A_lo
  static constexpr int kWStage = 2 * NP * 128;      // W_hi | W_lo
  static constexpr int kBytes = kAStages * kAStage + kWStages * kWStage;
  static __device__ __forceinline__ uint8_t* a(uint8_t* pipe, uint32_t s) {
    return pipe + s * kAStage;
  }
  static __device__ __forceinline__ uint8_t* w(uint8_t* pipe, uint32_t s) {
    return pipe + kAStages * kAStage + s * kWStage;
  }
};

// code-size knob (experiment): -DTGL_SMALL_CODE keeps the epilogue's transpose passes and
// the time warps' group loop rolled (the K|V kernel's body exceeds the instruction cache)
#ifdef TGL_SMALL_CODE
#define TGL_SMALL_UNROLL _Pragma("unroll 1")
#else
#define TGL_SMALL_UNROLL _Pragma("unroll")
#endif

// ---- profiling instrumentation: compiled only into probe builds (-DTGL_PROBE, tools/);
// product builds have no debug state, read no environment and take no debug branches
#ifdef TGL_PROBE
#define TGL_DBG(a) ((a).dbg)
// ---- profiling timeline (TGL_DEBUG_MASK & 32): [cta][tile][event] globaltimer stamps
constexpr int kTlTiles = 32, kTlEvents = 8;
__device__ unsigned long long g_timeline[kNumSMs * kTlTiles * kTlEvents];
__device__ unsigned long long g_trace[8192];         // (TGL_DEBUG_MASK & 4096) CTA-0 event trace
__device__ unsigned int g_trace_n;
// per-warp slices of 512 events; the per-warp count lives in shared memory
__shared__ unsigned s_trace_n[32];
__device__ __forceinline__ void trace(const Args& a, int ev, uint32_t k) {
  if ((a.dbg & 4096) && blockIdx.x == 0 && (threadIdx.x & 31) == 0) {
    // SM cycle counter (cheap, consistent within the CTA); the probe converts at 1965 MHz
    const unsigned long long t = (unsigned long long)clock64();
    const int w = (threadIdx.x >> 5) & 31;           // 32 slices of 256 events
    const unsigned n = s_trace_n[w];
    if (n < 255) {
      g_trace[w * 256 + n] = (t << 16) | ((unsigned long long)(ev & 0xff) << 8) | (k & 0xff);
      g_trace[w * 256 + 255] = n + 1;
      s_trace_n[w] = n + 1;
    }
  }
}
__device__ unsigned long long g_prof[kNumSMs * 16];   // (TGL_DEBUG_MASK & 512) cycle counters
__device__ __forceinline__ void prof_add(const Args& a, int slot, long long dt) {
  if ((a.dbg & 512) && (threadIdx.x & 31) == 0 && blockIdx.x < (unsigned)kNumSMs)
    atomicAdd(&g_prof[blockIdx.x * 16 + slot], (unsigned long long)dt);
}
__device__ __forceinline__ void tl_mark(const Args& a, uint32_t tt, int ev) {
  if ((a.dbg & 32) && tt < (uint32_t)kTlTiles && blockIdx.x < (unsigned)kNumSMs) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_timeline[(blockIdx.x * kTlTiles + tt) * kTlEvents + ev] = t;
  }
}

#define TGL_TRACE_RESET() \
  if (threadIdx.x < 32) s_trace_n[threadIdx.x] = 0
#else
#define TGL_DBG(a) 0
#define TGL_TRACE_RESET() (void)0
__device__ __forceinline__ void trace(const Args&, int, uint32_t) {}
__device__ __forceinline__ void prof_add(const Args&, int, long long) {}
__device__ __forceinline__ void tl_mark(const Args&, uint32_t, int) {}
#endif

__device__ __forceinline__ void named_bar(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// wait for the (u-1)-th completion of a ring slot (no wait on first use)
__device__ __forceinline__ void wait_free(uint64_t* bar, uint32_t u) {
  if (u >= 1) mbar_wait(bar, (u - 1) & 1u);
}
__device__ __forceinline__ void wait_free_sleep(uint64_t* bar, uint32_t u, uint32_t ns) {
  if (u >= 1) mbar_wait_sleep(bar, (u - 1) & 1u, ns);
}

__device__ __forceinline__ void load8(const float* p, int lc, int d, float* x) {
  if (p != nullptr && lc + 8 <= d && ((reinterpret_cast<uintptr_t>(p + lc) & 15) == 0)) {
    const float4 a = __ldg(reinterpret_cast<const float4*>(p + lc));
    const float4 b = __ldg(reinterpret_cast<const float4*>(p + lc + 4));
    x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w;
    x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
  } else {
#pragma unroll
    for (int e = 0; e < 8; ++e) x[e] = (p != nullptr && lc + e < d) ? __ldg(p + lc + e) : 0.f;
  }
}

// producer thread pt (0..255): row pt/2, 16-byte groups jb..jb+3 of a 64-wide chunk
template <int GPT, class RD>
__device__ __forceinline__ void load_chunk(int c, const Seg3& sg, const RD& rd, int r, int jb,
                                           const float* s_omega, const float* s_phi,
                                           const float* table, float* x) {
#pragma unroll
  for (int jj = 0; jj < GPT; ++jj) {
    float* y = x + jj * 8;
    const int kp = c * kChunk + (jb + jj) * 8;
#pragma unroll
    for (int e = 0; e < 8; ++e) y[e] = 0.f;
    if (rd.rdst[r] < 0 || kp >= sg.kpad) continue;
    if (kp < sg.p0) {
      load8(rd.p0[r], kp, sg.d0, y);
    } else if (kp < sg.p0 + sg.p1) {
      load8(rd.p1[r], kp - sg.p0, sg.d1, y);
    } else {
      const int j0 = kp - sg.p0 - sg.p1;
      const int trow = rd.trow[r];
      if (trow >= 0) {
        load8(table + (int64_t)trow * sg.d2, j0, sg.d2, y);
      } else {
        const float dt = rd.dt[r];
#pragma unroll
        for (int e = 0; e < 8; ++e)
          if (j0 + e < sg.d2) y[e] = tenc_fast(dt, s_omega[j0 + e], s_phi[j0 + e]);
      }
    }
  }
}

template <int GPT>
__device__ __forceinline__ void store_chunk(const float* x, uint8_t* a_hi, uint8_t* a_lo, int r,
                                            int jb, bool split) {
  const uint32_t hb = smem_u32(a_hi), lb = smem_u32(a_lo);
#pragma unroll
  for (int jj = 0; jj < GPT; ++jj) {
    uint32_t h[4], l[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) split2(x[jj * 8 + 2 * e], x[jj * 8 + 2 * e + 1], h[e], l[e]);
    const uint32_t off = sw128_off(r, jb + jj);
    st_shared_v4(hb + off, h[0], h[1], h[2], h[3]);
    if (split) st_shared_v4(lb + off, l[0], l[1], l[2], l[3]);
  }
}

// ---- tile schedules (every role walks the same sequence) --------------------------
struct DenseSched {   // q / ffn: tile = 128 consecutive destinations
  int64_t n, tile, stride;
  __device__ DenseSched(int64_t n_) : n(n_), tile(blockIdx.x), stride(gridDim.x) {}
  __device__ bool next(int64_t& i0, int& rows) {
    const int64_t ntiles = (n + kBM - 1) / kBM;
    if (tile >= ntiles) return false;
    i0 = tile * kBM;
    rows = (int)((n - i0) < kBM ? (n - i0) : kBM);
    tile += stride;
    return true;
  }
};

struct GroupSched {   // kv: groups of `dpb` destinations, each cut into 128-row tiles
  const int64_t* seg_ptr;
  int64_t n, groups, g, stride;
  int dpb;
  int64_t d0, e1, c0;
  int nd;
  __device__ GroupSched(const int64_t* sp, int64_t n_, int dpb_)
      : seg_ptr(sp), n(n_), groups((n_ + dpb_ - 1) / dpb_), g(blockIdx.x), stride(gridDim.x),
        dpb(dpb_), d0(0), e1(0), c0(0), nd(0) {}
  __device__ bool next_group() {
    if (g >= groups) return false;
    d0 = g * dpb;
    nd = (int)((n - d0) < dpb ? (n - d0) : dpb);
    c0 = seg_ptr[d0];
    e1 = seg_ptr[d0 + nd];
    g += stride;
    return true;
  }
  __device__ bool next_tile(int64_t& t0, int& rows) {
    if (c0 >= e1) return false;
    t0 = c0;
    rows = (int)((e1 - c0) < kBM ? (e1 - c0) : kBM);
    c0 += kBM;
    return true;
  }
  // flat walk over tiles (for roles that do not care about group boundaries)
  __device__ bool next(int64_t& t0, int& rows) {
    while (!next_tile(t0, rows))
      if (!next_group()) return false;
    return true;
  }
};

// ---- roles ------------------------------------------------------------------------
// K-chunk order alternates per tile (forward, backward, ...) so the last two weight
// chunks of a tile are the first two of the next one and stay resident in the W
// ring: (n-2)/n of the weight bytes per tile after the first (25% less at n = 8).
__device__ __forceinline__ int chunk_of(uint32_t tt, int i, int n) {
  return (tt & 1u) ? n - 1 - i : i;
}
__device__ __forceinline__ int w_reused(uint32_t tt, int n) { return (tt > 0 && n >= 4) ? 2 : 0; }

template <int NP, int N>
__device__ __forceinline__ void mma_tile(const Seg3& sg, bool split, uint8_t* pipe, Bars& B,
                                         uint32_t tmem_acc, uint32_t& ait, uint32_t& wl,
                                         uint32_t tt, bool nomma = false, bool nowait_w = false) {
  using PP = Pipe<NP>;
  constexpr uint32_t idesc = idesc_bf16(kBM, N);
  wait_free(&B.tempty[tt & 1u], tt >> 1);    // epilogue drained this accumulator
  tc_fence_after();
  const int n = sg.nchunks, r0 = w_reused(tt, n);
  for (int i = 0; i < n; ++i, ++ait) {
    const int c = chunk_of(tt, i, n);
    const uint32_t sa = ait % kAStages;
    mbar_wait(&B.afull[sa], (ait / kAStages) & 1u);
    uint32_t k;
    if (i < r0) {
      k = wl - 1 - i;                          // resident from the previous tile
    } else {
      k = wl + (i - r0);
      if (!nowait_w) mbar_wait(&B.wfull[k % kWStages], (k / kWStages) & 1u);
    }
    const uint32_t sw = k % kWStages;
    tc_fence_after();
    const uint32_t ahb = smem_u32(PP::a(pipe, sa)), alb = ahb + kAPart;
    const uint32_t whb = smem_u32(PP::w(pipe, sw)), wlb = whb + NP * 128;
    const int rem = sg.kpad - c * kChunk;
    const int nk = nomma ? 0 : (rem >= kChunk ? 4 : (rem + 15) / 16);
    for (int ks = 0; ks < nk; ++ks) {
      const uint64_t ah = desc_sw128(ahb + ks * 32), bh = desc_sw128(whb + ks * 32);
      mma_bf16(tmem_acc, ah, bh, idesc, (i | ks) != 0);
      if (split) {
        mma_bf16(tmem_acc, desc_sw128(alb + ks * 32), bh, idesc, 1u);
        mma_bf16(tmem_acc, ah, desc_sw128(wlb + ks * 32), idesc, 1u);
      }
    }
    if (nomma && nowait_w) mbar_arrive(&B.aempty[sa]);   // profiling: plain arrive
    else mma_commit(&B.aempty[sa]);
    const bool keep = (n >= 4) && (i >= n - 2);   // reused by the next tile
    if (!keep) mma_commit(&B.wempty[sw]);
  }
  wl += n - r0;
  mma_commit(&B.tfull[tt & 1u]);
}

template <int NP>
__device__ __forceinline__ void wload_tile(const Seg3& sg, uint8_t* pipe, Bars& B,
                                           const uint8_t* wpack, uint32_t& wl, uint32_t tt) {
  using PP = Pipe<NP>;
  const int n = sg.nchunks, r0 = w_reused(tt, n);
  for (int i = r0; i < n; ++i) {
    const uint32_t k = wl + (i - r0);
    const uint32_t sw = k % kWStages;
    wait_free(&B.wempty[sw], k / kWStages);
    mbar_arrive_expect_tx(&B.wfull[sw], PP::kWStage);
    bulk_g2s(PP::w(pipe, sw), wpack + (size_t)chunk_of(tt, i, n) * PP::kWStage, PP::kWStage,
             &B.wfull[sw]);
  }
  wl += n - r0;
}

template <int NP, int PW0, int GPT, class RD>
__device__ __forceinline__ void produce_tile(const Seg3& sg, bool split, uint8_t* pipe, Bars& B,
                                             uint32_t& ait, uint32_t tt, const RD& rd,
                                             const float* s_omega, const float* s_phi,
                                             const float* table, bool noload = false,
                                             int dbg = 0) {
  using PP = Pipe<NP>;
  constexpr int GPR = 8 / GPT;                 // producer threads per row
  const int pt = threadIdx.x - PW0 * 32;
  const int r = pt / GPR, jb = (pt % GPR) * GPT;
  const int lane = threadIdx.x & 31;
  const int n = sg.nchunks;
  constexpr int kX = 8 * GPT;
  constexpr bool kDeep = GPT <= 2;             // two chunks ahead when registers allow
  float x0[kX], x1[kX], x2[kDeep ? kX : 1];
#pragma unroll
  for (int q = 0; q < kX; ++q) x0[q] = x1[q] = 0.f;
  if (!noload) {
    load_chunk<GPT>(chunk_of(tt, 0, n), sg, rd, r, jb, s_omega, s_phi, table, x0);
    if (kDeep && n > 1) load_chunk<GPT>(chunk_of(tt, 1, n), sg, rd, r, jb, s_omega, s_phi, table, x1);
  }
  for (int i = 0; i < n; ++i, ++ait) {
    const uint32_t sa = ait % kAStages;
    const int ahead = kDeep ? 2 : 1;
    if (i + ahead < n && !noload)
      load_chunk<GPT>(chunk_of(tt, i + ahead, n), sg, rd, r, jb, s_omega, s_phi, table,
                      kDeep ? x2 : x1);
    wait_free(&B.aempty[sa], ait / kAStages);
    uint8_t* st = PP::a(pipe, sa);
    store_chunk<GPT>(x0, st, st + kAPart, r, jb, split);
    if (!(dbg & 2048)) fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) mbar_arrive(&B.afull[sa]);
#pragma unroll
    for (int q = 0; q < kX; ++q) {
      x0[q] = x1[q];
      if (kDeep) x1[q] = x2[q < (kDeep ? kX : 1) ? q : 0];
    }
  }
}

__device__ __forceinline__ void ws_init(Bars& B, uint32_t* s_tmem, uint32_t ncols,
                                        uint32_t dempty_count = kProdWarps + kEpiWarps,
                                        uint32_t afull_count = kProdWarps,
                                        uint32_t tempty_count = kEpiWarps,
                                        int mma_warp = kMmaWarp) {
  if (threadIdx.x == 0) {
    for (int s = 0; s < kAStages; ++s) {
      mbar_init(&B.afull[s], afull_count);
      mbar_init(&B.aempty[s], 1);
    }
    for (int s = 0; s < kWStages; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], dempty_count);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&B.tfull[a], 1);
      mbar_init(&B.tempty[a], tempty_count);
    }
    fence_mbar_init();
  }
  if ((threadIdx.x >> 5) == mma_warp) tmem_alloc(s_tmem, ncols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
}

__device__ __forceinline__ void ws_teardown(uint32_t tmem, uint32_t ncols,
                                            int mma_warp = kMmaWarp) {
  tc_fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == mma_warp) tmem_dealloc(tmem, ncols);
}

// per-warp arrive (all lanes done with a resource)
__device__ __forceinline__ void warp_arrive(uint64_t* bar) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive(bar);
}

// ------------------------------------------------------------------ S8 / S13 (dense rows)
constexpr int kNPq = 104;   // d_model padded to a multiple of 8 (rows of Wq / Wo)

template <bool kFfn>
__global__ void __launch_bounds__(kWsThreads, 1) dense_kernel(Args a) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ Bars B;
  __shared__ uint32_t s_tmem;
  __shared__ RowDesc rd[kDSlots];
  __shared__ float s_omega[256], s_phi[256];
  constexpr uint32_t kCols = 128;
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const Seg3& sg = kFfn ? a.so : a.sq;
  const uint8_t* wpack = kFfn ? a.wo : a.wq;
  const bool split = a.split != 0;
  // epilogue vectors staged once in shared memory: read inside the TMEM loops, a global
  // load there is a dependent L2/HBM round trip per 32-column piece
  __shared__ float s_v0[kMaxModel], s_v1[kMaxModel], s_v2[kMaxModel];
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < P.d_model; j += blockDim.x) {
    if (kFfn) {
      s_v0[j] = P.bo[j];
      s_v1[j] = P.ln_gamma[j];
      s_v2[j] = P.ln_beta[j];
    } else {
      s_v0[j] = P.bq[j];
      s_v1[j] = P.bk[j];
    }
  }
  TGL_TRACE_RESET();
  if ((threadIdx.x & 31) == 0) trace(a, 36, 0);     // per-warp start stamp
  ws_init(B, &s_tmem, 2 * kCols);
  const uint32_t tmem = s_tmem;
  if (threadIdx.x == 0) trace(a, 37, 0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  DenseSched sched(n);
  int64_t i0;
  int rows;
  uint32_t tt = 0;
  if (warp == kDescWarp) {                           // ---------------- row descriptors
    for (; sched.next(i0, rows); ++tt) {
      const uint32_t ds = tt % kDSlots;
      wait_free(&B.dempty[ds], tt / kDSlots);
      RowDesc& R = rd[ds];
      int64_t hrows[kBM / 32];                       // all index loads of the warp in flight
#pragma unroll
      for (int u = 0; u < kBM / 32; ++u) {
        const int r = lane + 32 * u;
        hrows[u] = (r < rows) ? (a.hdst_idx ? (int64_t)a.hdst_idx[i0 + r] : i0 + r) : 0;
      }
#pragma unroll
      for (int u = 0; u < kBM / 32; ++u) {
        const int r = lane + 32 * u;
        const float *p0 = nullptr, *p1 = nullptr;
        if (r < rows) {
          const int64_t i = i0 + r;
          const int64_t hrow = hrows[u];
          if (kFfn) {
            p0 = a.rbuf + i * kQLd;                    // [r_i ; h_i]  (eq 7)
            p1 = a.hdst + hrow * a.ld_hdst;
          } else {
            p0 = a.hdst + hrow * a.ld_hdst;            // [h_i ; Phi(0)] (eq 4)
          }
        }
        R.p0[r] = p0;
        R.p1[r] = p1;
        R.dt[r] = 0.f;
        // precomputed_zeros = table row 0 (fp32 tables only; a split16 table is read by
        // kv_pre alone, so Phi(0) = cos(phi) is evaluated -- bit-identical, R11)
        R.trow[r] = (!kFfn && a.table != nullptr && !(P.input_layout & TGL_SPLIT_TABLE)) ? 0 : -1;
        R.rdst[r] = r < rows ? r : -1;
      }
      warp_arrive(&B.dfull[ds]);
      trace(a, 30, tt);
    }
  } else if (warp == kWWarp) {                       // ---------------- weight loader
    uint32_t wit = 0;
    if (lane == 0)
      for (; sched.next(i0, rows); ++tt) wload_tile<kNPq>(sg, pipe, B, wpack, wit, tt);
    __syncwarp();
  } else if (warp >= kProdWarp0) {                   // ---------------- producers
    uint32_t ait = 0;
    for (; sched.next(i0, rows); ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      produce_tile<kNPq, kProdWarp0, kGPT>(sg, split, pipe, B, ait, tt, rd[ds], s_omega, s_phi, a.table);
      if (warp == kProdWarp0) trace(a, 31, tt);
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp == kMmaWarp) {                     // ---------------- MMA issuer
    uint32_t ait = 0, wit = 0;
    if (lane == 0)
      for (; sched.next(i0, rows); ++tt)
        mma_tile<kNPq, kNPq>(sg, split, pipe, B, tmem + (tt & 1u) * kCols, ait, wit, tt);
    __syncwarp();
    trace(a, 33, 0);
  } else {                                           // ---------------- epilogue
    const int row = warp * 32 + lane;
    const int D = P.d_model;
    for (; sched.next(i0, rows); ++tt) {
      const uint32_t ab = tt & 1u, ds = tt % kDSlots;
      mbar_wait(&B.tfull[ab], (tt >> 1) & 1u);
      if (warp == 0) trace(a, 34, tt);
      tc_fence_after();
      warp_arrive(&B.dempty[ds]);                     // descriptors not needed here
      (void)ds;
      const uint32_t ta = tmem + ab * kCols + ((uint32_t)(warp * 32) << 16);
      float v[32];
      if (!kFfn) {
        float* q = a.qbuf + (i0 + row) * kQLd;
        // also q . bk per head (cols 100, 101 of the scratch row): the K bias folded
        // into one scalar per destination for the K|V epilogue
        const int dhq = D / P.n_heads;
        float qb0 = 0.f, qb1 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (row < rows) {
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              const int col = cq * 32 + j;
              if (col < D) {
                float4 o = make_float4(v[j] + s_v0[col], v[j + 1] + s_v0[col + 1],
                                       v[j + 2] + s_v0[col + 2], v[j + 3] + s_v0[col + 3]);
                *reinterpret_cast<float4*>(q + col) = o;   // D % 4 == 0 (D == 100)
                const float oq[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {       // per column: a float4 may straddle heads
                  const float pb = oq[e] * s_v1[col + e];
                  if (col + e < dhq) qb0 += pb; else qb1 += pb;
                }
              }
            }
          }
        }
        if (row < rows && D + 2 <= kQLd) {
          q[D] = qb0;
          q[D + 1] = qb1;
        }
      } else {
        // out = LayerNorm(ReLU(acc + bo)): two passes over TMEM -- sum and sum of squares
        // (fp32; the ReLU outputs are O(1), so E[x^2] - mean^2 loses < 1e-6), then write
        float s = 0.f, s2 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int col = cq * 32 + j;
            if (col < D) {
              const float y = fmaxf(v[j] + s_v0[col], 0.f);
              s += y;
              s2 = fmaf(y, y, s2);
            }
          }
        }
        const float mean = s / (float)D;
        const float var = fmaxf(s2 / (float)D - mean * mean, 0.f);
        const float inv = rsqrtf(var + P.ln_eps);
        float* o = a.out + (i0 + row) * D;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (row < rows) {
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              const int col = cq * 32 + j;
              if (col < D) {
                float r4[4];
#pragma unroll
                for (int e = 0; e < 4; ++e)
                  r4[e] = (fmaxf(v[j + e] + s_v0[col + e], 0.f) - mean) * inv * s_v1[col + e] +
                          s_v2[col + e];
                *reinterpret_cast<float4*>(o + col) = make_float4(r4[0], r4[1], r4[2], r4[3]);
              }
            }
          }
        }
      }
      tc_fence_before();
      warp_arrive(&B.tempty[ab]);
      if (warp == 0) trace(a, 35, tt);
    }
  }
  ws_teardown(tmem, 2 * kCols);
}

// ------------------------------------------------------------------ S6,S7,S9-S12 (edge rows)
constexpr int kNPkv = 200;   // [Wk ; Wv] rows (2 * d_model)
constexpr int kKvEpiBytes = (2 * kMaxDpb * kMaxModel + kBM * 33) * 4;   // s_q, s_r, s_pv

__global__ void __launch_bounds__(kWsThreads, 1) kv_kernel(Args a) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ Bars B;
  __shared__ uint32_t s_tmem;
  __shared__ RowDesc rd[kDSlots];
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  // epilogue state (one destination group at a time); big arrays live after the pipe
  float (*s_q)[kMaxModel] = reinterpret_cast<float (*)[kMaxModel]>(pipe + Pipe<200>::kBytes);
  float (*s_r)[kMaxModel] = s_q + kMaxDpb;
  float (*s_pv)[33] = reinterpret_cast<float (*)[33]>(s_r + kMaxDpb);
  __shared__ float s_logit[kBM][2];
  __shared__ float s_p[kBM][2];
  __shared__ float s_m[kMaxDpb][2], s_l[kMaxDpb][2], s_sc[kMaxDpb][2];
  __shared__ int64_t s_seg[kMaxDpb + 1];
  constexpr uint32_t kCols = 256;
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const bool split = a.split != 0;
  const int dm = P.d_model, H = P.n_heads, dh = dm / H;
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  ws_init(B, &s_tmem, 2 * kCols);
  const uint32_t tmem = s_tmem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  GroupSched sched(a.seg_ptr, n, a.dpb);
  int64_t t0;
  int rows;
  uint32_t tt = 0;
  if (warp == kDescWarp) {                           // ---------------- row descriptors
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    while (sched.next_group()) {
      // this group's segment offsets, kept in registers (lane d holds seg_ptr[d0+d])
      const int64_t segl = lane <= sched.nd ? a.seg_ptr[sched.d0 + lane] : INT64_MAX;
      const float tdl = lane < sched.nd ? a.dst_t[sched.d0 + lane] : 0.f;
      for (; sched.next_tile(t0, rows); ++tt) {
        const uint32_t ds = tt % kDSlots;
        wait_free(&B.dempty[ds], tt / kDSlots);
        RowDesc& R = rd[ds];
#pragma unroll 1
        for (int r = lane; r < kBM; r += 32) {
          const int64_t e = t0 + r;
          // local destination = #{1 <= d < nd : seg[d] <= e}  (offsets broadcast by shuffle)
          int ld = 0;
          for (int dd = 1; dd < sched.nd; ++dd)
            ld += (__shfl_sync(0xffffffffu, segl, dd) <= e) ? 1 : 0;
          const float td = __shfl_sync(0xffffffffu, tdl, ld & 31);
          const float *p0 = nullptr, *p1 = nullptr;
          float dt = 0.f;
          int trow = -1, rr = -1;
          if (r < rows) {
            rr = ld;
            const int64_t hr = a.hsrc_idx ? (int64_t)a.hsrc_idx[hoff + e] : hoff + e;
            p0 = a.hsrc + hr * a.ld_hsrc;
            if (P.d_e > 0) p1 = a.efeat + (int64_t)a.eid[e] * a.ld_e;
            dt = td - a.edge_t[e];                       // fp32 delta (R18)
            trow = (int)tenc_table_row(dt, a.table, a.window);
          }
          R.p0[r] = p0;
          R.p1[r] = p1;
          R.dt[r] = dt;
          R.trow[r] = trow;
          R.rdst[r] = rr;
        }
        warp_arrive(&B.dfull[ds]);
      }
    }
  } else if (warp == kWWarp) {                       // ---------------- weight loader
    uint32_t wit = 0;
    if (lane == 0)
      for (; sched.next(t0, rows); ++tt) wload_tile<kNPkv>(a.skv, pipe, B, a.wkv, wit, tt);
    __syncwarp();
  } else if (warp >= kProdWarp0) {                   // ---------------- producers
    uint32_t ait = 0;
    for (; sched.next(t0, rows); ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      produce_tile<kNPkv, kProdWarp0, kGPT>(a.skv, split, pipe, B, ait, tt, rd[ds], s_omega,
                                            s_phi, a.table, (TGL_DBG(a) & 2) != 0);
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp == kMmaWarp) {                     // ---------------- MMA issuer
    uint32_t ait = 0, wit = 0;
    if (lane == 0)
      for (; sched.next(t0, rows); ++tt)
        mma_tile<kNPkv, kNPkv>(a.skv, split, pipe, B, tmem + (tt & 1u) * kCols, ait, wit, tt,
                               (TGL_DBG(a) & 4) != 0);
    __syncwarp();
  } else {                                           // ---------------- epilogue (128 threads)
    const int tid = threadIdx.x;                      // 0..127
    const int row = tid;
    // q rows of a group: nd * dm floats as float4 (dm % 4 == 0), prefetched one group ahead
    constexpr int kQv = (kMaxDpb * kMaxModel / 4 + kBM - 1) / kBM;   // float4 per thread
    const int dm4 = dm / 4;
    float4 qpre[kQv];
    auto prefetch_q = [&](int64_t gd0, int gnd) {
#pragma unroll
      for (int u = 0; u < kQv; ++u) {
        const int x = tid + u * kBM;
        const int dd = x / dm4, c4 = x % dm4;
        qpre[u] = dd < gnd ? *reinterpret_cast<const float4*>(a.qbuf + (gd0 + dd) * kQLd + 4 * c4)
                           : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    };
    {
      GroupSched peek = sched;
      if (peek.next_group()) prefetch_q(peek.d0, peek.nd);
    }
    __shared__ int s_lo[kMaxDpb], s_hi[kMaxDpb];
    while (sched.next_group()) {
      const int64_t d0 = sched.d0;
      const int nd = sched.nd;
#pragma unroll
      for (int u = 0; u < kQv; ++u) {
        const int x = tid + u * kBM;
        const int dd = x / dm4, c4 = x % dm4;
        if (dd < kMaxDpb) *reinterpret_cast<float4*>(&s_q[dd][4 * c4]) = qpre[u];
      }
      for (int x = tid; x < nd * dm; x += kBM) s_r[x / dm][x % dm] = 0.f;
      if (tid < kMaxDpb * 2) {
        s_m[tid >> 1][tid & 1] = -INFINITY;
        s_l[tid >> 1][tid & 1] = 0.f;
      }
      if (tid <= nd) s_seg[tid] = a.seg_ptr[d0 + tid];
      {
        GroupSched peek = sched;                      // next group's q, in flight meanwhile
        if (peek.next_group()) prefetch_q(peek.d0, peek.nd);
      }
      named_bar(kBarEpi, kBM);
      for (; sched.next_tile(t0, rows); ++tt) {
        const int64_t c0 = t0;
        const uint32_t ab = tt & 1u, ds = tt % kDSlots;
        mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
        mbar_wait(&B.tfull[ab], (tt >> 1) & 1u);
        tc_fence_after();
        const int d = rd[ds].rdst[row];
        warp_arrive(&B.dempty[ds]);
        if (TGL_DBG(a) & 1) {
          tc_fence_before();
          warp_arrive(&B.tempty[ab]);
          continue;
        }
        if (tid < nd) {   // this tile's row range of each destination
          const int64_t lo = s_seg[tid] > c0 ? s_seg[tid] : c0;
          const int64_t hi = s_seg[tid + 1] < c0 + rows ? s_seg[tid + 1] : c0 + rows;
          s_lo[tid] = (int)(lo - c0);
          s_hi[tid] = (int)(hi > lo ? hi - c0 : lo - c0);
        }
        const uint32_t ta = tmem + ab * kCols + ((uint32_t)(warp * 32) << 16);
        float v[32];
        // S10: logits per head from the K columns [0, dm)
        float p0 = 0.f, p1 = 0.f;
        const float* qrow = &s_q[d >= 0 ? d : 0][0];
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int col = cq * 32 + j;
            if (col < dm) {
              const float pr = qrow[col] * (v[j] + s_bias[col]);
              if (col < dh) p0 += pr; else p1 += pr;
            }
          }
        }
        if (d >= 0) {
          float s0 = p0 * P.logit_scale, s1 = p1 * P.logit_scale;
          if (P.leaky_slope >= 0.f) {
            s0 = s0 < 0.f ? s0 * P.leaky_slope : s0;
            s1 = s1 < 0.f ? s1 * P.leaky_slope : s1;
          }
          s_logit[row][0] = s0;
          s_logit[row][1] = s1;
        }
        named_bar(kBarEpi, kBM);
        // S11: online segmented softmax statistics, one thread per (dst, head)
        if (tid < nd * H) {
          const int dd = tid / H, h = tid % H;
          const int lo = s_lo[dd], hi = s_hi[dd];
          float sc = 1.f;
          if (lo < hi) {
            float mc = -INFINITY;
            for (int e = lo; e < hi; ++e) mc = fmaxf(mc, s_logit[e][h]);
            const float mo = s_m[dd][h];
            const float mn = fmaxf(mo, mc);
            sc = (mo == -INFINITY) ? 0.f : expf(mo - mn);
            float l = s_l[dd][h] * sc;
            for (int e = lo; e < hi; ++e) {
              const float pe = expf(s_logit[e][h] - mn);
              s_p[e][h] = pe;
              l += pe;
            }
            s_m[dd][h] = mn;
            s_l[dd][h] = l;
          }
          s_sc[dd][h] = sc;
        }
        named_bar(kBarEpi, kBM);
        // S12: r = r * sc + sum_rows p * v, 32 V columns at a time (fixed order)
        const float w0 = d >= 0 ? s_p[row][0] : 0.f;
        const float w1 = d >= 0 ? s_p[row][H > 1 ? 1 : 0] : 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + dm + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int col = cq * 32 + j;
            s_pv[row][j] = col < dm ? (col < dh ? w0 : w1) * (v[j] + s_bias[dm + col]) : 0.f;
          }
          named_bar(kBarEpi, kBM);
          for (int x = tid; x < nd * 32; x += kBM) {
            const int dd = x >> 5, j = x & 31, col = cq * 32 + j;
            const int lo = s_lo[dd], hi = s_hi[dd];
            if (col >= dm || lo >= hi) continue;
            float acc = s_r[dd][col] * s_sc[dd][col < dh ? 0 : 1];
            for (int e = lo; e < hi; ++e) acc += s_pv[e][j];
            s_r[dd][col] = acc;
          }
          named_bar(kBarEpi, kBM);
        }
        tc_fence_before();
        warp_arrive(&B.tempty[ab]);
      }
      // normalise; empty segment -> 0 (R19)
      for (int x = tid; x < nd * dm; x += kBM) {
        const int dd = x / dm, col = x % dm;
        const float l = s_l[dd][col < dh ? 0 : 1];
        a.rbuf[(d0 + dd) * kQLd + col] = l > 0.f ? s_r[dd][col] / l : 0.f;
      }
      named_bar(kBarEpi, kBM);
    }
  }
  ws_teardown(tmem, 2 * kCols);
}

// ------------------------------------------------------------------ binned K|V attention
// Tile = 4 bins of 32 rows.  The descriptor warp packs whole destination segments
// (<= 32 rows) into bins without straddling, so a destination's rows sit in one TMEM
// lane quarter.  Epilogue warp w owns lane quarter w%4 and head w/4 (two heads): its
// logits, softmax (shuffle scans over the segment) and alpha-weighted V sums (a 32x33
// smem transpose per warp) need nothing from any other warp -- no block barriers, no
// state across tiles; r is written straight to global.  Empty segments get r = 0 from
// the descriptor warp (R19); a segment longer than 32 rows (max_seg hint violated)
// gets a NaN row.
#ifndef TGL_SLEEP_EPI
#define TGL_SLEEP_EPI 128
#endif
constexpr int kBEpi = 8;                    // warps 0-7
constexpr int kBarBinEpi = 1;               // named barrier of the 8 epilogue warps
constexpr int kBMma = 8;
constexpr int kBDesc = 9;
constexpr int kBW = 10;
constexpr int kBProd0 = 11;
constexpr int kBProdWarps = 8;              // warps 11-18, 4 groups of 8 columns each
constexpr int kBGPT = 1024 / (kBProdWarps * 32);
constexpr int kBThreads = (kBProd0 + kBProdWarps) * 32;   // 608

struct BinDesc {
  const float* p0[kBM];
  const float* p1[kBM];
  float dt[kBM];
  int trow[kBM];
  int rdst[kBM];          // global destination of the row, -1 for padding rows
  int64_t e[kBM];         // edge index of the row
  float td[kBM];          // destination time of the row
  int live;               // 0 = end-of-work marker
};

// Epilogue of the binned K|V kernels (warps 0-7): S10-S12 for one tile per trip.
// Warp w owns TMEM lane quarter w%4 and head w/4; see kv_bin_kernel.
// kPW: row pitch of the per-warp transpose buffer (33: 32 columns per pass; 17: 16
// columns per pass, half the shared memory -- the split kernel spends it on stages)
template <int NS, class D, int kPW = 33, bool kLowReg = false>
__device__ __forceinline__ void bin_epilogue(const Args& a, uint64_t* dfull, uint64_t* dempty,
                                             uint64_t* tfull, uint64_t* tempty, const D* bd,
                                             uint32_t tmem, float* s_pvf,
                                             const float* s_bias, uint32_t tempty_cl = 0) {
  // tempty_cl != 0: the accumulator barriers live in the leader CTA of a pair (2-SM MMA);
  // release them there with cluster-scope remote arrives
  auto release = [&](uint32_t ab) {
    if (tempty_cl) {
      __syncwarp();
      if ((threadIdx.x & 31) == 0)
        asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(
                         tempty_cl + ab * 8)
                     : "memory");
    } else {
      warp_arrive(&tempty[ab]);
    }
  };
  constexpr uint32_t kCols = 256;
  constexpr int dm = 100, dh = 50;
  const tgl_attn_params& P = a.P;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint32_t tt = 0;
  const int q4 = warp & 3, head = warp >> 2;
  const int cb = head * dh;                        // this warp's columns [cb, cb + dh)
  constexpr int kCW = kPW - 1;                     // columns per transpose pass
  float* pvw = s_pvf + warp * 32 * kPW;
  for (;; ++tt) {
    const uint32_t ab = tt & 1u, ds = tt % NS;
    // one warp polls, the other seven block in bar.sync (no issue slots spent waiting)
    if (warp == 0) mbar_wait_sleep(&dfull[ds], (tt / NS) & 1u, TGL_SLEEP_EPI);
    named_bar(kBarBinEpi, kBEpi * 32);
    if (!bd[ds].live) {
      warp_arrive(&dempty[ds]);
      break;
    }
    const int d = bd[ds].rdst[q4 * 32 + lane];
    warp_arrive(&dempty[ds]);
    // segment structure of this bin from the row destinations
    const int dprev = __shfl_up_sync(0xffffffffu, d, 1);
    const int dnext = __shfl_down_sync(0xffffffffu, d, 1);
    const bool valid = d >= 0;
    const unsigned smask = __ballot_sync(0xffffffffu, valid && (lane == 0 || dprev != d));
    const unsigned emask = __ballot_sync(0xffffffffu, valid && (lane == 31 || dnext != d));
    const int lo = 31 - __clz(smask & (0xffffffffu >> (31 - lane)));   // last start <= lane
    const int hi = __ffs(emask & (0xffffffffu << lane));              // last end >= lane, +1
    // this row's q (head columns) and q . bk, fetched before waiting for the accumulator
    // (kLowReg: read piecewise after the wait instead -- 64-register budget)
    const int64_t qr = valid ? (a.q_idx ? (int64_t)a.q_idx[d] : (int64_t)d) : 0;
    const float* qrow = a.qbuf + qr * a.q_ld;
    float qv[kLowReg ? 1 : dh];
    if (!kLowReg) {
#pragma unroll
      for (int j = 0; j < dh; j += 2) {
        const float2 q2 = __ldg(reinterpret_cast<const float2*>(qrow + cb + j));
        qv[j] = q2.x;
        qv[j + 1] = q2.y;
      }
    }
    const float qb = __ldg(qrow + dm + head);
    if (threadIdx.x == 0) tl_mark(a, tt, 5);
    const long long e0c = clock64();
    if (warp == 0) mbar_wait_sleep(&tfull[ab], (tt >> 1) & 1u, TGL_SLEEP_EPI);
    named_bar(kBarBinEpi, kBEpi * 32);
    const long long e1c = clock64();
    if (warp == 0) trace(a, 9, tt);
    if (warp == 0) prof_add(a, 11, e1c - e0c);      // epilogue: wait for the accumulator
    tc_fence_after();
    if (threadIdx.x == 0) tl_mark(a, tt, 6);
    if (TGL_DBG(a) & 1) {
      tc_fence_before();
      release(ab);
      continue;
    }
    const uint32_t ta = tmem + ab * kCols + ((uint32_t)(q4 * 32) << 16);
    float v[32];
    // S10: this head's logit <q_dst, k_row + bk> = <q_dst, k_row> + (q_dst . bk_head)
    float p = qb;
    if (kLowReg) {
#pragma unroll 1
      for (int cq = 0; cq < 4; ++cq) {               // 16-column pieces
        tmem_ld16(ta + cb + cq * 16, v);
        float qq[16];
#pragma unroll
        for (int j = 0; j < 16; j += 2) {
          const float2 q2 = cq * 16 + j < dh ? __ldg(reinterpret_cast<const float2*>(
                                                   qrow + cb + cq * 16 + j))
                                             : make_float2(0.f, 0.f);
          qq[j] = q2.x;
          qq[j + 1] = q2.y;
        }
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if (cq * 16 + j < dh) p = fmaf(qq[j], v[j], p);
      }
    } else {
#pragma unroll
      for (int cq = 0; cq < 2; ++cq) {
        tmem_ld32(ta + cb + cq * 32, v);
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 32; ++j)
          if (cq * 32 + j < dh) p = fmaf(qv[cq * 32 + j], v[j], p);
      }
    }
    float s = p * P.logit_scale;
    if (P.leaky_slope >= 0.f) s = s < 0.f ? s * P.leaky_slope : s;
    // S11: softmax over the segment [lo, hi): suffix max / sum, broadcast from lo
    if (!valid) s = -INFINITY;
    float m = s;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const float y = __shfl_down_sync(0xffffffffu, m, off);
      if (lane + off < hi) m = fmaxf(m, y);
    }
    const float mseg = __shfl_sync(0xffffffffu, m, valid ? lo : lane);
    const float ex = valid ? expf(s - mseg) : 0.f;
    float t = ex;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const float y = __shfl_down_sync(0xffffffffu, t, off);
      if (lane + off < hi) t += y;
    }
    const float l = __shfl_sync(0xffffffffu, t, valid ? lo : lane);
    const float w = valid ? ex / l : 0.f;
    // S12: r_dst = sum_seg w * (v + bv) = sum_seg w * v + bv  (sum_seg w = 1); lane j owns
    // column j of the 32-column piece and walks each segment's rows in order
#pragma unroll 1
    for (int cq = 0; cq < 2; ++cq) {
      tmem_ld32(ta + dm + cb + cq * 32, v);
      tmem_wait_ld();
TGL_SMALL_UNROLL
      for (int hh = 0; hh < 32 / kCW; ++hh) {
#pragma unroll
        for (int j = 0; j < kCW; ++j) pvw[lane * kPW + j] = w * v[hh * kCW + j];
        __syncwarp();
        const int c = cq * 32 + hh * kCW + lane;     // this lane's column in the head
        const bool act = lane < kCW && c < dh;
        const float bvc = act ? s_bias[dm + cb + c] : 0.f;
        unsigned sm = smask, em = emask;
        while (sm) {
          const int slo = __ffs(sm) - 1, shi = __ffs(em);   // [slo, shi)
          sm &= sm - 1;
          em &= em - 1;
          const int dr = __shfl_sync(0xffffffffu, d, slo);
          float acc = 0.f;
          for (int r = slo; r < shi; ++r) acc += pvw[r * kPW + (lane & (kCW - 1))];
          if (act) {
            const float rv = acc + bvc;
            if (a.rsplit != nullptr) {                 // split16 operand row for dense_pre
              uint8_t* rp = a.rsplit + (int64_t)dr * (4 * kDPN);
              const __nv_bfloat16 rh = __float2bfloat16_rn(rv);
              const __nv_bfloat16 rl = __float2bfloat16_rn(rv - __bfloat162float(rh));
              *reinterpret_cast<__nv_bfloat16*>(rp + 2 * (cb + c)) = rh;
              *reinterpret_cast<__nv_bfloat16*>(rp + 2 * kDPN + 2 * (cb + c)) = rl;
              if (cb + c < kDPN - dm) {                // zero the padding columns 100..103
                *reinterpret_cast<uint16_t*>(rp + 2 * (dm + cb + c)) = 0;
                *reinterpret_cast<uint16_t*>(rp + 2 * kDPN + 2 * (dm + cb + c)) = 0;
              }
            } else {
              a.rbuf[(int64_t)dr * kQLd + cb + c] = rv;
            }
          }
        }
        __syncwarp();
      }
    }
    tc_fence_before();
    if (warp == 0) trace(a, 10, tt);
    if (warp == 0) prof_add(a, 12, clock64() - e1c);   // epilogue: tile work
    release(ab);
    if (threadIdx.x == 0) tl_mark(a, tt, 7);
  }
}

__global__ void __launch_bounds__(kBThreads, 1) kv_bin_kernel(Args a) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ Bars B;
  __shared__ uint32_t s_tmem;
  __shared__ BinDesc bd[kDSlots];
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  float (*s_pv)[32][33] = reinterpret_cast<float (*)[32][33]>(pipe + Pipe<kNPkv>::kBytes);
  constexpr uint32_t kCols = 256;
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const bool split = a.split != 0;
  constexpr int dm = 100, dh = 50;                 // d_model 100, two heads (host-checked)
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  ws_init(B, &s_tmem, 2 * kCols, kBEpi + kBProdWarps + 2, kBProdWarps, kBEpi, kBMma);
  const uint32_t tmem = s_tmem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t D0 = n * blockIdx.x / gridDim.x, D1 = n * (blockIdx.x + 1) / gridDim.x;
  uint32_t tt = 0;

  if (warp == kBDesc) {                              // ---------------- tile builder
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    int64_t d = D0;
    int64_t wbase = D0;   // windows: lane l holds seg_ptr[wbase + l] and dst_t[wbase + l]
    int64_t segw = a.seg_ptr[(wbase + lane) < n ? (wbase + lane) : n];
    float tdw = (wbase + lane) < n ? a.dst_t[wbase + lane] : 0.f;
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      wait_free(&B.dempty[ds], tt / kDSlots);
      if (lane == 0) tl_mark(a, tt, 0);
      BinDesc& R = bd[ds];
      int bin = 0, used = 0, cnt = 0;
      int u0 = 0, u1 = 0, u2 = 0, u3 = 0;              // rows used per bin
      while (d < D1) {
        if (d + 1 - wbase > 31) {
          wbase = d;
          segw = a.seg_ptr[(wbase + lane) < n ? (wbase + lane) : n];
          tdw = (wbase + lane) < n ? a.dst_t[wbase + lane] : 0.f;
        }
        const int64_t s0 = __shfl_sync(0xffffffffu, segw, (int)(d - wbase));
        const int64_t s1 = __shfl_sync(0xffffffffu, segw, (int)(d - wbase + 1));
        const float td = __shfl_sync(0xffffffffu, tdw, (int)(d - wbase));
        const int L = (int)(s1 - s0);
        if (L == 0 || L > 32) {                        // empty -> r = 0; overflow -> NaN
          const float fill = L == 0 ? 0.f : __int_as_float(0x7fc00000);
          for (int c = lane; c < dm; c += 32) a.rbuf[d * kQLd + c] = fill;
          ++d;
          continue;
        }
        if (used + L > 32) {
          if (bin == 3) break;                         // tile full
          ++bin;
          used = 0;
        }
        const int row0 = bin * 32 + used;
        if (lane < L) {
          R.rdst[row0 + lane] = (int)d;
          R.e[row0 + lane] = s0 + lane;
          R.td[row0 + lane] = td;
        }
        used += L;
        if (bin == 0) u0 = used; else if (bin == 1) u1 = used; else if (bin == 2) u2 = used; else u3 = used;
        ++cnt;
        ++d;
      }
      // padding rows
      if (lane >= u0) R.rdst[lane] = -1;
      if (lane >= u1) R.rdst[32 + lane] = -1;
      if (lane >= u2) R.rdst[64 + lane] = -1;
      if (lane >= u3) R.rdst[96 + lane] = -1;
      R.live = cnt > 0 ? 1 : 0;
      __syncwarp();
      if (cnt > 0) {
        int dst[4];
        int64_t e[4];
        float tdr[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int r = 32 * u + lane;
          dst[u] = R.rdst[r];
          e[u] = dst[u] >= 0 ? R.e[r] : 0;
          tdr[u] = dst[u] >= 0 ? R.td[r] : 0.f;
        }
        int32_t hi[4], ei[4];
        float et[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {              // all loads of the lane's 4 rows in flight
          const bool ok = dst[u] >= 0 && !(TGL_DBG(a) & 16);
          hi[u] = ok ? (a.hsrc_idx ? a.hsrc_idx[hoff + e[u]] : (int32_t)(hoff + e[u])) : 0;
          ei[u] = (ok && P.d_e > 0) ? a.eid[e[u]] : 0;
          if (TGL_DBG(a) & 128) ei[u] &= 0x3FF;            // profiling: edge rows in 700 KB
          if (TGL_DBG(a) & 256) hi[u] &= 0x3FF;
          et[u] = ok ? a.edge_t[e[u]] : 0.f;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int r = 32 * u + lane;
          const bool ok = dst[u] >= 0;
          const float dt = tdr[u] - et[u];          // fp32 delta (R18)
          R.p0[r] = ok ? a.hsrc + (int64_t)hi[u] * a.ld_hsrc : nullptr;
          R.p1[r] = (ok && P.d_e > 0) ? a.efeat + (int64_t)ei[u] * a.ld_e : nullptr;
          R.dt[r] = ok ? dt : 0.f;
          R.trow[r] = ok ? (int)tenc_table_row(dt, a.table, a.window) : -1;
        }
      }
      warp_arrive(&B.dfull[ds]);
      if (lane == 0) tl_mark(a, tt, 1);
      if (cnt == 0) break;                             // end marker published
    }
  } else if (warp == kBW) {                          // ---------------- weight loader
    uint32_t wl = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0 && !(TGL_DBG(a) & 8)) wload_tile<kNPkv>(a.skv, pipe, B, a.wkv, wl, tt);
      __syncwarp();
    }
  } else if (warp >= kBProd0) {                      // ---------------- producers
    uint32_t ait = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      if (!bd[ds].live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      if (threadIdx.x == kBProd0 * 32) tl_mark(a, tt, 2);
      produce_tile<kNPkv, kBProd0, kBGPT>(a.skv, split, pipe, B, ait, tt, bd[ds], s_omega,
                                          s_phi, a.table, (TGL_DBG(a) & 2) != 0, TGL_DBG(a));
      if (threadIdx.x == kBProd0 * 32) tl_mark(a, tt, 3);
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp == kBMma) {                        // ---------------- MMA issuer
    uint32_t ait = 0, wl = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) tl_mark(a, tt, 4);
      if (lane == 0)
        mma_tile<kNPkv, kNPkv>(a.skv, split, pipe, B, tmem + (tt & 1u) * kCols, ait, wl, tt,
                               (TGL_DBG(a) & 4) != 0, (TGL_DBG(a) & 8) != 0);
      __syncwarp();
    }
  } else {                                           // ---------------- epilogue warps 0-7
    bin_epilogue<kDSlots>(a, B.dfull, B.dempty, B.tfull, B.tempty, bd, tmem, &s_pv[0][0][0],
                          s_bias);
  }
  ws_teardown(tmem, 2 * kCols, kBMma);
}

// ------------------------------------------------------------------ async-gathered K|V attention
// kv_async_kernel: the binned K|V attention with the A operand gathered by LDGSTS
// (cp.async, 16 B per lane, no register staging) so that ~80 KB of row gathers are in
// flight per SM.  K is cut into 32-column fp32 chunks per concat segment ([h_src | e |
// Phi], each padded to 32; the padding K step is skipped when a chunk holds <= 16 real
// columns).  Per chunk and tile:
//   producers  : 8 warps; warp w owns the 8-row groups w and w + 8 of the 128-row tile.
//                It issues the cp.async of a 2-chunk unit kAheadU units before
//                converting it;
//                the 16 KB fp32 image (row r at r*128 B) is rewritten IN PLACE, group by
//                group, as bf16 hi | lo (512 B each) in the SW64 K-major UMMA layout;
//                Phi(Delta t) = cos(w Delta t + phi) is evaluated for rows the
//                precompute table does not cover (their time chunks are not loaded);
//   MMA warp   : tcgen05.mma M=128 N=200 K=16 from the converted image and a SW64
//                weight chunk (hi|lo, one bulk copy), 3 passes in fp32 mode;
//   epilogue   : logits, segment softmax and alpha-weighted V sums from TMEM (bin_epilogue).
// (A TMA tile::gather4 variant of the producers was measured at ~5 B/clk/SM on B200 --
// 128-byte row boxes -- and dropped.)
constexpr int kTC = 32;                       // fp32 columns per K chunk
constexpr int kTAStage = kBM * kTC * 4;       // 16 KB
#ifndef TGL_KV_ASTAGES
#define TGL_KV_ASTAGES 6
#endif
#ifndef TGL_KV_AHEAD
#define TGL_KV_AHEAD (TGL_KV_ASTAGES / 2 - 1)
#endif
#ifndef TGL_KV_WSTAGES
#define TGL_KV_WSTAGES 3
#endif
#ifndef TGL_KV_DSLOTS
#define TGL_KV_DSLOTS 4
#endif
constexpr int kTAStages = TGL_KV_ASTAGES;
constexpr int kAheadU = TGL_KV_AHEAD;         // 2-chunk units of gathers in flight per producer
constexpr int kTWStages = TGL_KV_WSTAGES;
constexpr int kTWHalf = kNPkv * 64;           // one of W_hi / W_lo of a chunk (12.8 KB)
constexpr int kTWStage = 2 * kTWHalf;
constexpr int kTMma = 8, kTW = 9, kTDesc0 = 10, kTDescWarps = 2, kTProd0 = 12, kTProdWarps = 8;
constexpr int kTThreads = (kTProd0 + kTProdWarps) * 32;   // 640 (96 registers per thread)
constexpr int kTDSlots = TGL_KV_DSLOTS;
constexpr int kTPipeBytes = kTAStages * kTAStage + kTWStages * kTWStage;
constexpr int kTSmem = 1024 + kTPipeBytes + kBEpi * 32 * 33 * 4;

struct KvPlan {       // 32-column chunks of the three K segments
  int d[3];           // widths (h_src, e, time)
  int c[3];           // chunks per segment
  int n;              // total chunks
  int contig;         // 1: chunks cut the concatenation [h | e | Phi] without per-segment
                      //    padding (segment widths multiples of 4: a 16-byte piece never
                      //    straddles two segments); 0: each segment padded to 32
};
static KvPlan make_plan(int d0, int d1, int d2) {
  KvPlan p;
  p.d[0] = d0; p.d[1] = d1; p.d[2] = d2;
  for (int s = 0; s < 3; ++s) p.c[s] = (p.d[s] + kTC - 1) / kTC;
  p.n = p.c[0] + p.c[1] + p.c[2];
  p.contig = 0;
  return p;
}
static bool contig_ok(int d0, int d1) { return d0 % 4 == 0 && d1 % 4 == 0; }
static KvPlan make_plan_contig(int d0, int d1, int d2) {
  KvPlan p = make_plan(d0, d1, d2);
  p.n = (d0 + d1 + d2 + kTC - 1) / kTC;
  p.contig = 1;
  return p;
}
__host__ __device__ __forceinline__ void plan_chunk(const KvPlan& p, int c, int& seg, int& col) {
  seg = c < p.c[0] ? 0 : (c < p.c[0] + p.c[1] ? 1 : 2);
  col = (c - (seg > 0 ? p.c[0] : 0) - (seg > 1 ? p.c[1] : 0)) * kTC;
}
__device__ __forceinline__ int col_of_time(const KvPlan& p, int c) {
  return (c - p.c[0] - p.c[1]) * kTC;
}
__device__ __forceinline__ int plan_ksteps(const KvPlan& p, int c) {
  int seg, col;
  plan_chunk(p, c, seg, col);
  return p.d[seg] - col > 16 ? 2 : 1;
}

struct TBars {
  uint64_t aready[kTAStages], aempty[kTAStages];
  uint64_t wfull[kTWStages], wempty[kTWStages];
  uint64_t dfull[kTDSlots], dempty[kTDSlots];
  uint64_t tfull[2], tempty[2];
};

struct TDesc {
  int hrow[kBM];      // row of h_src
  int erow[kBM];      // row of the edge features
  int trow[kBM];      // precompute-table row, -1 = evaluate eq 8 directly
  float dt[kBM];
  int rdst[kBM];      // destination of the row, -1 = padding
  int live;
};

// 16-byte LDGSTS with zero fill past src_bytes (0..16)
__device__ __forceinline__ void cp_async16_zfill(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
               "r"(src_bytes)
               : "memory");
}
// L2 cache policies (createpolicy): streamed-once rows evict first, reused operands last
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void cp_async16_zfill_hint(uint32_t dst, const void* src,
                                                      uint32_t src_bytes, uint64_t pol) {
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(dst),
               "l"(src), "r"(src_bytes), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s_hint(void* dst_smem, const void* src_gmem, uint32_t bytes,
                                              uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], "
      "[%1], %2, [%3], %4;" ::"r"(smem_u32(dst_smem)),
      "l"(src_gmem), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void cp_async_wait_dyn(int pending) {   // <= pending groups left
  switch (pending) {
    case 0: cp_async_wait<0>(); break;
    case 1: cp_async_wait<1>(); break;
    case 2: cp_async_wait<2>(); break;
    case 3: cp_async_wait<3>(); break;
    case 4: cp_async_wait<4>(); break;
    default: cp_async_wait<5>(); break;
  }
}

// K-major SW64 descriptor: rows of 64 B (32 bf16), 8-row groups `sbo` bytes apart.
__device__ __forceinline__ uint64_t desc_sw64(uint32_t saddr, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)1u << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1u << 46;
  d |= (uint64_t)4u << 61;
  return d;
}
// byte offset of bf16 column c (0..31) of row r in an SW64 K-major 8-row atom
__device__ __forceinline__ uint32_t sw64_off(int r, int c) {
  return (uint32_t)((r & 7) * 64 + ((((c >> 3) ^ ((r >> 1) & 3)) & 3) << 4) + (c & 7) * 2);
}

__global__ void pack_kv64_kernel(const float* Wk, const float* Wv, int dm, int ksrc, KvPlan p,
                                 uint8_t* out) {
  const int kw = p.n * kTC;
  const int64_t total = (int64_t)kNPkv * kw;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(x / kw), kp = (int)(x % kw);
    const int c = kp / kTC, cc = kp % kTC;
    float v = 0.f;
    if (p.contig) {                                // K column kp of [h | e | Phi]
      if (n < 2 * dm && kp < ksrc)
        v = n < dm ? Wk[(int64_t)n * ksrc + kp] : Wv[(int64_t)(n - dm) * ksrc + kp];
    } else {
      int seg, col;
      plan_chunk(p, c, seg, col);
      if (n < 2 * dm && col + cc < p.d[seg]) {
        const int src = (seg > 0 ? p.d[0] : 0) + (seg > 1 ? p.d[1] : 0) + col + cc;
        v = n < dm ? Wk[(int64_t)n * ksrc + src] : Wv[(int64_t)(n - dm) * ksrc + src];
      }
    }
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    const int64_t off = (int64_t)c * kTWStage + (n >> 3) * 512 + sw64_off(n, cc);
    *reinterpret_cast<__nv_bfloat16*>(out + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(out + off + kTWHalf) = lo;
  }
}

// 16 bytes of row `row` (columns cb..cb+3, zero past `width`; row < 0 -> zeros)
__device__ __forceinline__ float4 ld_row4(const float* base, int row, int64_t ld, int cb,
                                          int width) {
  if (row < 0 || cb >= width) return make_float4(0.f, 0.f, 0.f, 0.f);
  const float* p = base + (int64_t)row * ld + cb;
  if (cb + 4 <= width) return __ldg(reinterpret_cast<const float4*>(p));
  float4 v = make_float4(__ldg(p), 0.f, 0.f, 0.f);
  if (cb + 1 < width) v.y = __ldg(p + 1);
  if (cb + 2 < width) v.z = __ldg(p + 2);
  return v;
}

__global__ void __launch_bounds__(kTThreads, 1)
    kv_async_kernel(const Args a, const KvPlan plan, const uint8_t* __restrict__ wkv,
                    const int bdst) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ TBars B;
  __shared__ uint32_t s_tmem;
  __shared__ TDesc bd[kTDSlots];
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  __shared__ int64_t s_seg[kTDescWarps][4 * 32 + 1];   // descriptor warps' tile scratch
  __shared__ float s_td[kTDescWarps][4 * 32];
  float (*s_pv)[32][33] = reinterpret_cast<float (*)[32][33]>(pipe + kTPipeBytes);
  constexpr uint32_t kCols = 256;
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const bool split = a.split != 0;
  constexpr int dm = 100;
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  if (threadIdx.x == 0) {
    for (int s = 0; s < kTAStages; ++s) {
      mbar_init(&B.aready[s], kTProdWarps);
      mbar_init(&B.aempty[s], 1);
    }
    for (int s = 0; s < kTWStages; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kTDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kBEpi + kTProdWarps + 2);   // epilogue, producers, mma, w
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&B.tfull[s], 1);
      mbar_init(&B.tempty[s], kBEpi);
    }
    fence_mbar_init();
  }
  TGL_TRACE_RESET();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == kTMma) tmem_alloc(&s_tmem, 2 * kCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = s_tmem;
  const int nch = plan.n;
  uint32_t tt = 0;

  if (warp >= kTDesc0 && warp < kTDesc0 + kTDescWarps) {   // ------- tile builders
    // Fixed packing: tile T holds destinations [T*dpt, (T+1)*dpt), dpt = 4*bdst, bin u
    // the bdst destinations [u*bdst, (u+1)*bdst) of the tile, their segments
    // concatenated (<= 32 rows when every segment has <= max_seg = 32/bdst rows), so a
    // destination's rows sit in one TMEM lane quarter.  Tiles go round-robin over the
    // CTAs; descriptor warp w builds the CTA's tiles tt = w, w+2, ... into slot tt % 4.
    const int dw = warp - kTDesc0;
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    const int dpt = 4 * bdst;
    const int64_t ntiles = (n + dpt - 1) / dpt;
    int64_t* sg = s_seg[dw];
    float* stdv = s_td[dw];
    for (tt = dw;; tt += kTDescWarps) {
      const uint32_t ds = tt % kTDSlots;
      const long long d0c = clock64();
      wait_free_sleep(&B.dempty[ds], tt / kTDSlots, 1000);
      const long long d1c = clock64();
      if (dw == 0) prof_add(a, 9, d1c - d0c);        // desc: wait for a slot
      trace(a, 20, tt);
      if (lane == 0) tl_mark(a, tt, 0);
      TDesc& R = bd[ds];
      const int64_t T = blockIdx.x + (int64_t)tt * gridDim.x;
      if (T >= ntiles) {                             // end marker
        if (lane == 0) R.live = 0;
        warp_arrive(&B.dfull[ds]);
        break;
      }
      const int64_t d0 = T * dpt;
      const int nd = (int)((n - d0) < dpt ? (n - d0) : dpt);
      for (int j = lane; j <= nd; j += 32) sg[j] = a.seg_ptr[d0 + j];
      for (int j = lane; j < nd; j += 32) stdv[j] = a.dst_t[d0 + j];
      __syncwarp();
      int64_t er[4] = {0, 0, 0, 0};
      float tr[4] = {0.f, 0.f, 0.f, 0.f};
      int dr[4] = {-1, -1, -1, -1};
      unsigned ovf_bins = 0;                         // bins whose rows overflow 32
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j0 = u * bdst;
        if (j0 >= nd) continue;
        const int j1 = (j0 + bdst) < nd ? j0 + bdst : nd;
        const int64_t e0 = sg[j0], e1 = sg[j1];
        if (e1 - e0 > 32) {                          // max_seg violated: NaN rows
          ovf_bins |= 1u << u;
          continue;
        }
        const int64_t e = e0 + lane;
        if (e < e1) {
          int j = j0;
          while (sg[j + 1] <= e) ++j;
          dr[u] = (int)(d0 + j);
          er[u] = e;
          tr[u] = stdv[j];
        }
      }
      // empty segments -> r = 0 (R19); destinations of an overflowing bin -> NaN
      for (int j = 0; j < nd; ++j) {
        const bool ovf = (ovf_bins >> (j / bdst)) & 1u;
        if (sg[j + 1] == sg[j] || ovf) {
          const float fill = ovf ? __int_as_float(0x7fc00000) : 0.f;
          fill_r_row(a, d0 + j, fill, lane, dm);
        }
      }
      R.live = 1;
      int32_t hi[4], ei[4];
      float et[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {                   // all loads of the lane's 4 rows in flight
        const bool ok = dr[u] >= 0 && !(TGL_DBG(a) & 16);
        hi[u] = ok ? (a.hsrc_idx ? a.hsrc_idx[hoff + er[u]] : (int32_t)(hoff + er[u])) : 0;
        ei[u] = (ok && P.d_e > 0) ? a.eid[er[u]] : 0;
        et[u] = ok ? a.edge_t[er[u]] : 0.f;
        if (TGL_DBG(a) & 128) ei[u] &= 0x3FF;              // profiling: edge rows in 700 KB
        if (TGL_DBG(a) & 256) hi[u] &= 0x3FF;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int r = 32 * u + lane;
        const bool ok = dr[u] >= 0;
        const float dt = tr[u] - et[u];               // fp32 delta (R18)
        R.hrow[r] = ok ? hi[u] : -1;
        R.erow[r] = ok ? ei[u] : -1;
        R.dt[r] = ok ? dt : 0.f;
        R.trow[r] = ok ? (int)tenc_table_row(dt, a.table, a.window) : -1;
        R.rdst[r] = dr[u];
      }
      warp_arrive(&B.dfull[ds]);
      if (dw == 0) prof_add(a, 10, clock64() - d1c); // desc: build
      trace(a, 21, tt);
      if (lane == 0) tl_mark(a, tt, 1);
    }
  } else if (warp == kTW) {                          // ---------------- weight loader
    uint32_t wl = 0;
    const uint32_t wbytes = split ? kTWStage : kTWHalf;
    for (;; ++tt) {
      const uint32_t ds = tt % kTDSlots;
      mbar_wait_sleep(&B.dfull[ds], (tt / kTDSlots) & 1u, 1000);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) {
        const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
        for (int i = r0; i < nch; ++i) {
          const uint32_t k = wl + (i - r0);
          const uint32_t sw = k % kTWStages;
          wait_free_sleep(&B.wempty[sw], k / kTWStages, 500);
          if (TGL_DBG(a) & 8) {
            mbar_arrive(&B.wfull[sw]);
            continue;
          }
          mbar_arrive_expect_tx(&B.wfull[sw], wbytes);
          bulk_g2s(pipe + kTAStages * kTAStage + sw * kTWStage,
                   wkv + (size_t)chunk_of(tt, i, nch) * kTWStage, wbytes, &B.wfull[sw]);
        }
        wl += nch - r0;
      }
      __syncwarp();
    }
  } else if (warp >= kTProd0) {                      // ---------------- producers
    // Work unit = two consecutive chunks of a tile (one cp.async group, one fence):
    // loads run kAheadU units ahead of the conversion.  Lane: rows rr and rr + 4 of
    // groups pw and pw + 8 (rows u = 0..3 -> rw0..rw3), 16-byte column piece j.
    const int pw = warp - kTProd0;
    const int rr = lane >> 3, j = lane & 7;
    const int rw0 = pw * 8 + rr, rw1 = rw0 + 4, rw2 = rw0 + 64, rw3 = rw0 + 68;
    const int npair = (nch + 1) >> 1;
    const uint32_t pipe_s = smem_u32(pipe);
    uint32_t lt = 0, ct = 0, al = 0, ac = 0, ul = 0, uc = 0;
    int lp = 0, cp = 0;
    bool lend = false;
    int hr0, hr1, hr2, hr3, er0, er1, er2, er3, tr0, tr1, tr2, tr3;
    float cdt0 = 0.f, cdt1 = 0.f, cdt2 = 0.f, cdt3 = 0.f;
    int ctr0 = -1, ctr1 = -1, ctr2 = -1, ctr3 = -1;
#define TGL_ENTER_LOAD_TILE()                                                          \
  do {                                                                                 \
    const uint32_t ds_ = lt % kTDSlots;                                                \
    mbar_wait_sleep(&B.dfull[ds_], (lt / kTDSlots) & 1u, 500);                         \
    const TDesc& R_ = bd[ds_];                                                         \
    if (!R_.live) {                                                                    \
      lend = true;                                                                     \
      break;                                                                           \
    }                                                                                  \
    hr0 = R_.hrow[rw0]; hr1 = R_.hrow[rw1]; hr2 = R_.hrow[rw2]; hr3 = R_.hrow[rw3];    \
    er0 = R_.erow[rw0]; er1 = R_.erow[rw1]; er2 = R_.erow[rw2]; er3 = R_.erow[rw3];    \
    tr0 = R_.trow[rw0]; tr1 = R_.trow[rw1]; tr2 = R_.trow[rw2]; tr3 = R_.trow[rw3];    \
  } while (0)
    TGL_ENTER_LOAD_TILE();
    for (;;) {
      // ---- keep kAheadU units of gathers in flight
      while (!lend && ul < uc + kAheadU && lt < ct + kTDSlots - 1) {
        const int i0 = 2 * lp, cnt = (nch - i0) < 2 ? (nch - i0) : 2;
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          if (q >= cnt) break;
          const int c = chunk_of(lt, i0 + q, nch);
          const int seg = c < plan.c[0] ? 0 : (c < plan.c[0] + plan.c[1] ? 1 : 2);
          const int col = (c - (seg > 0 ? plan.c[0] : 0) - (seg > 1 ? plan.c[1] : 0)) * kTC;
          const int width = seg == 0 ? plan.d[0] : (seg == 1 ? plan.d[1] : plan.d[2]);
          const uint32_t s = (al + q) % kTAStages;
          wait_free(&B.aempty[s], (al + q) / kTAStages);
          const uint32_t sb = pipe_s + s * kTAStage + rw0 * 128 + j * 16;
          const int cb = col + 4 * j;                // first fp32 column of this lane
          const uint32_t nb = cb >= width ? 0u : (uint32_t)min(16, (width - cb) * 4);
          if (!(TGL_DBG(a) & 2)) {
            const float* base = seg == 0 ? a.hsrc : (seg == 1 ? a.efeat : a.table);
            const int64_t ld = seg == 0 ? a.ld_hsrc : (seg == 1 ? a.ld_e : (int64_t)P.d_t);
            const int x0 = seg == 0 ? hr0 : (seg == 1 ? er0 : tr0);
            const int x1 = seg == 0 ? hr1 : (seg == 1 ? er1 : tr1);
            const int x2 = seg == 0 ? hr2 : (seg == 1 ? er2 : tr2);
            const int x3 = seg == 0 ? hr3 : (seg == 1 ? er3 : tr3);
            // padding rows and rows the table misses (time chunks) load nothing
            const float* b = base + cb;
            if (x0 >= 0) cp_async16_zfill(sb, b + (int64_t)x0 * ld, nb);
            if (x1 >= 0) cp_async16_zfill(sb + 512, b + (int64_t)x1 * ld, nb);
            if (x2 >= 0) cp_async16_zfill(sb + 8192, b + (int64_t)x2 * ld, nb);
            if (x3 >= 0) cp_async16_zfill(sb + 8192 + 512, b + (int64_t)x3 * ld, nb);
          }
        }
        cp_async_commit();
        if (pw == 0) trace(a, 1, ul);
        al += cnt;
        ++ul;
        if (++lp == npair) {
          lp = 0;
          ++lt;
          TGL_ENTER_LOAD_TILE();
        }
      }
      if (uc == ul) break;                           // everything loaded has been converted
      // ---- convert unit uc (loaded kAheadU units ago)
      if (cp == 0) {                                 // entering tile ct: per-row time inputs
        const uint32_t ds = ct % kTDSlots;
        const TDesc& R = bd[ds];
        cdt0 = R.dt[rw0]; cdt1 = R.dt[rw1]; cdt2 = R.dt[rw2]; cdt3 = R.dt[rw3];
        ctr0 = R.trow[rw0]; ctr1 = R.trow[rw1]; ctr2 = R.trow[rw2]; ctr3 = R.trow[rw3];
        warp_arrive(&B.dempty[ds]);                  // last read of this slot by the warp
        if (threadIdx.x == kTProd0 * 32) tl_mark(a, ct, 2);
      }
      const int i0 = 2 * cp, cnt = (nch - i0) < 2 ? (nch - i0) : 2;
      cp_async_wait_dyn((int)(ul - uc - 1));
      __syncwarp();
      if (pw == 0) trace(a, 3, uc);
      float4 x[2][4];
      uint32_t gb[2];
#pragma unroll
      for (int q = 0; q < 2; ++q) {                  // all shared loads of the unit first
        gb[q] = pipe_s + ((ac + q) % kTAStages) * kTAStage + pw * 1024;
        if (q < cnt) {
          x[q][0] = ld_shared_f4(gb[q] + rr * 128 + j * 16);
          x[q][1] = ld_shared_f4(gb[q] + (rr + 4) * 128 + j * 16);
          x[q][2] = ld_shared_f4(gb[q] + 8192 + rr * 128 + j * 16);
          x[q][3] = ld_shared_f4(gb[q] + 8192 + (rr + 4) * 128 + j * 16);
        }
      }
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        if (q >= cnt) break;
        const int c = chunk_of(ct, i0 + q, nch);
        if (c >= plan.c[0] + plan.c[1] && !(TGL_DBG(a) & 1024)) {   // time chunk: Phi where the table misses
          const int cc = col_of_time(plan, c) + 4 * j;
          float w[4], f[4];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const bool ok = cc + e < P.d_t;
            w[e] = ok ? s_omega[cc + e] : 0.f;
            f[e] = ok ? s_phi[cc + e] : 0.f;
          }
#define TGL_PHI4(X, DT, TR)                                                              \
  if (TR < 0) {                                                                          \
    X.x = (cc < P.d_t) ? tenc_fast(DT, w[0], f[0]) : 0.f;                                \
    X.y = (cc + 1 < P.d_t) ? tenc_fast(DT, w[1], f[1]) : 0.f;                            \
    X.z = (cc + 2 < P.d_t) ? tenc_fast(DT, w[2], f[2]) : 0.f;                            \
    X.w = (cc + 3 < P.d_t) ? tenc_fast(DT, w[3], f[3]) : 0.f;                            \
  }
          TGL_PHI4(x[q][0], cdt0, ctr0)
          TGL_PHI4(x[q][1], cdt1, ctr1)
          TGL_PHI4(x[q][2], cdt2, ctr2)
          TGL_PHI4(x[q][3], cdt3, ctr3)
#undef TGL_PHI4
        }
      }
      __syncwarp();
      if (!(TGL_DBG(a) & 64)) {
        const uint32_t o0 = sw64_off(rr, 4 * j), o1 = sw64_off(rr + 4, 4 * j);
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          if (q >= cnt) break;
          uint32_t h0, h1, l0, l1;
#define TGL_SPLIT_STORE(X, ADDR)                                                         \
  split2(X.x, X.y, h0, l0);                                                              \
  split2(X.z, X.w, h1, l1);                                                              \
  asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(ADDR), "r"(h0), "r"(h1) : "memory"); \
  if (split)                                                                             \
    asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"((ADDR) + 512), "r"(l0), "r"(l1)   \
                 : "memory");
          TGL_SPLIT_STORE(x[q][0], gb[q] + o0)
          TGL_SPLIT_STORE(x[q][1], gb[q] + o1)
          TGL_SPLIT_STORE(x[q][2], gb[q] + 8192 + o0)
          TGL_SPLIT_STORE(x[q][3], gb[q] + 8192 + o1)
#undef TGL_SPLIT_STORE
        }
      }
      if (!(TGL_DBG(a) & 2048)) fence_proxy_async_smem();   // 2048: profiling only (unsafe)
      __syncwarp();
      if (pw == 0) trace(a, 4, uc);
      if (lane == 0) {
        mbar_arrive(&B.aready[ac % kTAStages]);
        if (cnt == 2) mbar_arrive(&B.aready[(ac + 1) % kTAStages]);
      }
      ac += cnt;
      ++uc;
      if (++cp == npair) {
        cp = 0;
        if (threadIdx.x == kTProd0 * 32) tl_mark(a, ct, 3);
        ++ct;
      }
    }
#undef TGL_ENTER_LOAD_TILE
  } else if (warp == kTMma) {                        // ---------------- MMA issuer
    // The whole warp walks the loop (uniform control flow; one elected lane issues),
    // two K chunks per trip to halve the per-chunk handshake cost.
    uint32_t ait = 0, wl = 0;
    constexpr uint32_t idesc = idesc_bf16(kBM, kNPkv);
    const uint32_t pipe_s = smem_u32(pipe);
    const uint32_t w_s = pipe_s + kTAStages * kTAStage;
    for (;; ++tt) {
      const uint32_t ds = tt % kTDSlots;
      mbar_wait(&B.dfull[ds], (tt / kTDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const uint32_t acc = tmem + (tt & 1u) * kCols;
      const long long m2 = clock64();
      wait_free_sleep(&B.tempty[tt & 1u], tt >> 1, 200);
      prof_add(a, 7, clock64() - m2);                  // MMA: wait for the accumulator
      tc_fence_after();
      trace(a, 7, tt);
      if (lane == 0) tl_mark(a, tt, 4);
      const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
      for (int i = 0; i < nch; i += 2, ait += 2) {
        const int cnt = (nch - i) < 2 ? (nch - i) : 2;
        uint32_t st[2], kw[2];
        int cc[2];
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          if (q >= cnt) break;
          const uint32_t a_ = ait + q;
          st[q] = a_ % kTAStages;
          cc[q] = chunk_of(tt, i + q, nch);
          mbar_wait(&B.aready[st[q]], (a_ / kTAStages) & 1u);
          if (i + q < r0) {
            kw[q] = wl - 1 - (i + q);                  // resident from the previous tile
          } else {
            kw[q] = wl + (i + q - r0);
            mbar_wait(&B.wfull[kw[q] % kTWStages], (kw[q] / kTWStages) & 1u);
          }
        }
        tc_fence_after();
        trace(a, 5, ait);
        if (elect_one()) {
#pragma unroll
          for (int q = 0; q < 2; ++q) {
            if (q >= cnt) break;
            const uint32_t ab = pipe_s + st[q] * kTAStage;
            const uint32_t wb = w_s + (kw[q] % kTWStages) * kTWStage;
            const int nk = (TGL_DBG(a) & 4) ? 0 : plan_ksteps(plan, cc[q]);
            for (int ks = 0; ks < nk; ++ks) {
              const uint64_t ah = desc_sw64(ab + ks * 32, 1024), bh = desc_sw64(wb + ks * 32, 512);
              mma_bf16(acc, ah, bh, idesc, ((i + q) | ks) != 0);
              if (split) {
                mma_bf16(acc, desc_sw64(ab + 512 + ks * 32, 1024), bh, idesc, 1u);
                mma_bf16(acc, ah, desc_sw64(wb + kTWHalf + ks * 32, 512), idesc, 1u);
              }
            }
          }
#pragma unroll
          for (int q = 0; q < 2; ++q) {
            if (q >= cnt) break;
            mma_commit(&B.aempty[st[q]]);
            const bool keep = (nch >= 4) && (i + q >= nch - 2);   // reused by the next tile
            if (!keep) mma_commit(&B.wempty[kw[q] % kTWStages]);
          }
        }
        __syncwarp();
      }
      ait -= (uint32_t)((nch & 1) ? 1 : 0);            // the last trip may hold one chunk
      wl += nch - r0;
      if (elect_one()) mma_commit(&B.tfull[tt & 1u]);
      __syncwarp();
      prof_add(a, 8, clock64() - m2);                  // MMA: whole tile
    }
  } else {                                           // ---------------- epilogue warps 0-7
    bin_epilogue<kTDSlots>(a, B.dfull, B.dempty, B.tfull, B.tempty, bd, tmem, &s_pv[0][0][0],
                           s_bias);
  }
  ws_teardown(tmem, 2 * kCols, kTMma);
}

// ------------------------------------------------------------------ split-role K|V attention
// kv_split_kernel: the binned K|V attention of kv_async_kernel with the gather and the
// bf16 conversion in DIFFERENT warps, so that neither waits on the other's latency:
//   loaders    (4 warps): per 32-column chunk, 8 LDGSTS of 16 B per lane into an fp32
//                         row image (row r at r*128 B); completion is tracked by the
//                         stage's mbarrier (cp.async.mbarrier.arrive.noinc), so a loader
//                         never waits for its own copies -- only for a free stage, and it
//                         runs up to kSF chunks (64 KB) ahead;
//   converters (4 warps): fp32 image -> bf16 hi | lo in the SW64 K-major UMMA layout of a
//                         separate bf16 ring (Phi(dt) evaluated for rows the precompute
//                         table does not cover), then release the fp32 stage;
//   MMA warp, weight warp, descriptor warps and the 8 epilogue warps as in kv_async.
// Per-chunk bookkeeping (segment, column, width, K steps) comes from a shared table, so
// the steady-state loops are straight-line code.
#ifndef TGL_KV_FSTAGES
#define TGL_KV_FSTAGES 3
#endif
#ifndef TGL_KV_BSTAGES
#define TGL_KV_BSTAGES 4
#endif
// poll back-off (ns) of the roles that usually wait long: polling warps take issue
// slots and sync-unit bandwidth from the converters (measured: ~1/3 of all executed
// instructions were try_wait re-polls before back-off)
#ifndef TGL_SLEEP_DESC
#define TGL_SLEEP_DESC 256
#endif
#ifndef TGL_SLEEP_W
#define TGL_SLEEP_W 64
#endif
#ifndef TGL_SLEEP_LOAD
#define TGL_SLEEP_LOAD 64
#endif
#ifndef TGL_KV_LAG
#define TGL_KV_LAG 0
#endif
// per-role cycle counters of kv_split_kernel (profiling builds: -DTGL_KV_PROF)
#ifdef TGL_KV_PROF
#define TGL_PROF_CLK(v) const long long v = clock64()
#else
#define TGL_PROF_CLK(v) (void)0
#endif
#ifndef TGL_KV_SPLIT_WSTAGES
#define TGL_KV_SPLIT_WSTAGES 2
#endif
constexpr int kSW = TGL_KV_SPLIT_WSTAGES;           // weight stages (25.6 KB each)
constexpr int kSF = TGL_KV_FSTAGES;            // fp32 image stages (16 KB each)
constexpr int kSB = TGL_KV_BSTAGES;            // bf16 hi|lo stages (16 KB each)
constexpr int kSStage = kBM * kTC * 4;         // 16 KB
constexpr int kSLoad0 = kTProd0, kSLoadWarps = 4;
#ifndef TGL_KV_CONV_WARPS
#define TGL_KV_CONV_WARPS 8
#endif
constexpr int kSConv0 = kTProd0 + kSLoadWarps, kSConvWarps = TGL_KV_CONV_WARPS;
constexpr int kSRowsPerConv = kBM / kSConvWarps;     // 16 (8 warps) or 32 (4 warps)
constexpr int kSKc = kSRowsPerConv / 4;              // rows per converter lane
constexpr int kSThreads = (kSConv0 + kSConvWarps) * 32;   // 768 with 8 converter warps
constexpr int kSPipeBytes = (kSF + kSB) * kSStage + kSW * kTWStage;
#ifndef TGL_KV_SPLIT_DSLOTS
#define TGL_KV_SPLIT_DSLOTS 3
#endif
constexpr int kSDSlots = TGL_KV_SPLIT_DSLOTS;       // tile descriptor ring
constexpr int kSPW = 17;                             // 16-column epilogue transposes
constexpr int kSSmem = 1024 + kSPipeBytes + kBEpi * 32 * kSPW * 4;
constexpr int kSMaxChunks = 48;

struct SBars {
  uint64_t ffull[kSF], fempty[kSF];
  uint64_t bfull[kSB], bempty[kSB];
  uint64_t wfull[kSW], wempty[kSW];
  uint64_t dfull[kSDSlots], dempty[kSDSlots];
  uint64_t tfull[2], tempty[2];
};

// arrive on `bar` once every cp.async this thread issued so far has landed
__device__ __forceinline__ void cp_async_mbar_arrive_noinc(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}

__global__ void __launch_bounds__(kSThreads, 1)
    kv_split_kernel(const Args a, const KvPlan plan, const uint8_t* __restrict__ wkv,
                    const int bdst) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ SBars B;
  __shared__ uint32_t s_tmem;
  __shared__ TDesc bd[kSDSlots];
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  __shared__ int64_t s_seg[kTDescWarps][4 * 32 + 1];
  __shared__ float s_td[kTDescWarps][4 * 32];
  __shared__ int4 s_chunk[kSMaxChunks];          // {segment, first column, width, K steps}
  float* s_pvf = reinterpret_cast<float*>(pipe + kSPipeBytes);
  constexpr uint32_t kCols = 256;
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const bool split = a.split != 0;
  constexpr int dm = 100;
  const int nch = plan.n;
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  const int ktot = plan.d[0] + plan.d[1] + plan.d[2];
  const int e0 = plan.d[0], e1 = plan.d[0] + plan.d[1];   // segment starts in [h | e | Phi]
  for (int c = threadIdx.x; c < nch; c += blockDim.x) {
    if (plan.contig) {                               // seg -1: resolved per 16-byte piece
      s_chunk[c] = make_int4(-1, c * kTC, ktot, ktot - c * kTC > 16 ? 2 : 1);
    } else {
      int seg, col;
      plan_chunk(plan, c, seg, col);
      const int width = seg == 0 ? plan.d[0] : (seg == 1 ? plan.d[1] : plan.d[2]);
      s_chunk[c] = make_int4(seg, col, width, width - col > 16 ? 2 : 1);
    }
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < kSF; ++s) {
      mbar_init(&B.ffull[s], TGL_KV_LAG > 0 ? kSLoadWarps : kSLoadWarps * 32);
      mbar_init(&B.fempty[s], kSConvWarps);
    }
    for (int s = 0; s < kSB; ++s) {
      mbar_init(&B.bfull[s], kSConvWarps);
      mbar_init(&B.bempty[s], 1);
    }
    for (int s = 0; s < kSW; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kSDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kBEpi + kSLoadWarps + kSConvWarps + 2);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&B.tfull[s], 1);
      mbar_init(&B.tempty[s], kBEpi);
    }
    fence_mbar_init();
  }
  TGL_TRACE_RESET();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == kTMma) tmem_alloc(&s_tmem, 2 * kCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = s_tmem;
  const uint32_t pipe_s = smem_u32(pipe);
  const uint32_t f_s = pipe_s;                                  // fp32 ring
  const uint32_t b_s = pipe_s + kSF * kSStage;                  // bf16 ring
  const uint32_t w_s = pipe_s + (kSF + kSB) * kSStage;          // weight ring
  uint32_t tt = 0;

  if (warp >= kTDesc0 && warp < kTDesc0 + kTDescWarps) {   // ------- tile builders
    // identical to kv_async_kernel (fixed packing of bdst destinations per 32-row bin)
    const int dw = warp - kTDesc0;
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    const int dpt = 4 * bdst;
    const int64_t ntiles = (n + dpt - 1) / dpt;
    int64_t* sg = s_seg[dw];
    float* stdv = s_td[dw];
    for (tt = dw;; tt += kTDescWarps) {
      const uint32_t ds = tt % kSDSlots;
      wait_free_sleep(&B.dempty[ds], tt / kSDSlots, TGL_SLEEP_DESC);
      trace(a, 20, tt);
      TDesc& R = bd[ds];
      const int64_t T = blockIdx.x + (int64_t)tt * gridDim.x;
      if (T >= ntiles) {
        if (lane == 0) R.live = 0;
        warp_arrive(&B.dfull[ds]);
        break;
      }
      const int64_t d0 = T * dpt;
      const int nd = (int)((n - d0) < dpt ? (n - d0) : dpt);
      for (int j = lane; j <= nd; j += 32) sg[j] = a.seg_ptr[d0 + j];
      for (int j = lane; j < nd; j += 32) stdv[j] = a.dst_t[d0 + j];
      __syncwarp();
      int64_t er[4] = {0, 0, 0, 0};
      float tr[4] = {0.f, 0.f, 0.f, 0.f};
      int dr[4] = {-1, -1, -1, -1};
      unsigned ovf_bins = 0;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j0 = u * bdst;
        if (j0 >= nd) continue;
        const int j1 = (j0 + bdst) < nd ? j0 + bdst : nd;
        const int64_t e0 = sg[j0], e1 = sg[j1];
        if (e1 - e0 > 32) {
          ovf_bins |= 1u << u;
          continue;
        }
        const int64_t e = e0 + lane;
        if (e < e1) {
          int j = j0;
          while (sg[j + 1] <= e) ++j;
          dr[u] = (int)(d0 + j);
          er[u] = e;
          tr[u] = stdv[j];
        }
      }
      for (int j = 0; j < nd; ++j) {
        const bool ovf = (ovf_bins >> (j / bdst)) & 1u;
        if (sg[j + 1] == sg[j] || ovf) {
          const float fill = ovf ? __int_as_float(0x7fc00000) : 0.f;
          fill_r_row(a, d0 + j, fill, lane, dm);
        }
      }
      R.live = 1;
      int32_t hi[4], ei[4];
      float et[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const bool ok = dr[u] >= 0;
        hi[u] = ok ? (a.hsrc_idx ? a.hsrc_idx[hoff + er[u]] : (int32_t)(hoff + er[u])) : 0;
        ei[u] = (ok && P.d_e > 0) ? a.eid[er[u]] : 0;
        et[u] = ok ? a.edge_t[er[u]] : 0.f;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int r = 32 * u + lane;
        const bool ok = dr[u] >= 0;
        const float dt = tr[u] - et[u];               // fp32 delta (R18)
        R.hrow[r] = ok ? hi[u] : -1;
        R.erow[r] = ok ? ei[u] : -1;
        R.dt[r] = ok ? dt : 0.f;
        R.trow[r] = ok ? (int)tenc_table_row(dt, a.table, a.window) : -1;
        R.rdst[r] = dr[u];
      }
      warp_arrive(&B.dfull[ds]);
      trace(a, 21, tt);
    }
  } else if (warp == kTW) {                          // ---------------- weight loader
    uint32_t wl = 0;
    const uint32_t wbytes = split ? kTWStage : kTWHalf;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait_sleep(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_W);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) {
        const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
        for (int i = r0; i < nch; ++i) {
          const uint32_t k = wl + (i - r0);
          const uint32_t sw = k % kSW;
          wait_free_sleep(&B.wempty[sw], k / kSW, TGL_SLEEP_W);
          trace(a, 11, k);
          if (TGL_DBG(a) & 8) {                           // profiling: no weight bytes
            mbar_arrive(&B.wfull[sw]);
            continue;
          }
          mbar_arrive_expect_tx(&B.wfull[sw], wbytes);
          bulk_g2s(pipe + (kSF + kSB) * kSStage + sw * kTWStage,
                   wkv + (size_t)chunk_of(tt, i, nch) * kTWStage, wbytes, &B.wfull[sw]);
        }
        wl += nch - r0;
      }
      __syncwarp();
    }
  } else if (warp >= kSLoad0 && warp < kSLoad0 + kSLoadWarps) {   // ---------- loaders
    // lane: rows lw*32 + (lane>>3) + 4k (k = 0..7), 16-byte piece (lane & 7) of the chunk
    const int lw = warp - kSLoad0;
    const int r0 = lw * 32 + (lane >> 3), pc = lane & 7;
    const uint32_t lofs = (uint32_t)r0 * 128 + pc * 16;
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait_sleep(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_LOAD);
      const TDesc& R = bd[ds];
      if (!R.live) {
#if TGL_KV_LAG > 0
        cp_async_wait<0>();                          // the last LAG chunks
        __syncwarp();
        if (lane == 0)
          for (uint32_t j = g >= TGL_KV_LAG ? g - TGL_KV_LAG : 0; j < g; ++j)
            mbar_arrive(&B.ffull[j % kSF]);
#endif
        warp_arrive(&B.dempty[ds]);
        break;
      }
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = chunk_of(tt, i, nch);
        const int4 ch = s_chunk[c];
        int seg = ch.x, cb = ch.y + 4 * pc;
        uint32_t nb;
        if (seg < 0) {                               // contiguous plan: this lane's segment
          const int g = cb;
          seg = g < e0 ? 0 : (g < e1 ? 1 : 2);
          cb = g - (seg == 0 ? 0 : (seg == 1 ? e0 : e1));
          nb = g < ktot ? 16u : 0u;                  // widths are multiples of 4
        } else {
          nb = cb >= ch.z ? 0u : (uint32_t)min(16, (ch.z - cb) * 4);
        }
        const float* base = seg == 0 ? a.hsrc : (seg == 1 ? a.efeat : a.table);
        const int64_t ld = seg == 0 ? a.ld_hsrc : (seg == 1 ? a.ld_e : (int64_t)P.d_t);
        const int* ridx = seg == 0 ? R.hrow : (seg == 1 ? R.erow : R.trow);
        const float* b = base + (nb ? cb : 0);
        int x[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) x[k] = ridx[r0 + 4 * k];
        const uint32_t sf = g % kSF;
        TGL_PROF_CLK(l0);
        wait_free_sleep(&B.fempty[sf], g / kSF, TGL_SLEEP_LOAD);
        TGL_PROF_CLK(l1);
        const uint32_t dst = f_s + sf * kSStage + lofs;
#pragma unroll
        if (!(TGL_DBG(a) & 2))                            // profiling: no gathers
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (x[k] >= 0) cp_async16_zfill(dst + k * 512, b + (int64_t)x[k] * ld, nb);
#if TGL_KV_LAG > 0
        // one arrive per warp: chunk g - LAG is complete once at most LAG newer groups
        // are pending (far fewer mbarrier operations than one noinc arrive per thread)
        cp_async_commit();
        if (g >= TGL_KV_LAG) {
          cp_async_wait<TGL_KV_LAG>();
          __syncwarp();
          if (lane == 0) mbar_arrive(&B.ffull[(g - TGL_KV_LAG) % kSF]);
        }
#else
        cp_async_mbar_arrive_noinc(&B.ffull[sf]);
#endif
#ifdef TGL_KV_PROF
        if (lw == 0) {
          prof_add(a, 5, l1 - l0);
          prof_add(a, 6, clock64() - l1);
        }
#endif
        if (lw == 0) trace(a, 1, g);
      }
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp >= kSConv0 && warp < kSConv0 + kSConvWarps) {   // -------- converters
    // lane: rows cw*32 + (lane>>3) + 4k; row r lands in 8-row group r>>3 of the bf16
    // stage ([hi 512 B | lo 512 B] per group, SW64 K-major)
    const int cw = warp - kSConv0;
    const int r0 = cw * kSRowsPerConv + (lane >> 3), pc = lane & 7;
    const uint32_t lofs = (uint32_t)r0 * 128 + pc * 16;
    const uint32_t o_even = sw64_off(lane >> 3, 4 * pc), o_odd = sw64_off((lane >> 3) + 4, 4 * pc);
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait(&B.dfull[ds], (tt / kSDSlots) & 1u);
      const TDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      float dtk[kSKc];
      int trk[kSKc];
#pragma unroll
      for (int k = 0; k < kSKc; ++k) {
        dtk[k] = R.dt[r0 + 4 * k];
        trk[k] = R.rdst[r0 + 4 * k] >= 0 ? R.trow[r0 + 4 * k] : 0;   // padding: no Phi
      }
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = chunk_of(tt, i, nch);
        const int4 ch = s_chunk[c];
        const uint32_t sf = g % kSF, sb = g % kSB;
        TGL_PROF_CLK(c0);
        mbar_wait(&B.ffull[sf], (g / kSF) & 1u);
        TGL_PROF_CLK(c1);
        if (cw == 0) trace(a, 3, g);
        float4 x[kSKc];
        const uint32_t src = f_s + sf * kSStage + lofs;
        if (TGL_DBG(a) & 64) {                            // profiling: no conversion work
          wait_free(&B.bempty[sb], g / kSB);
          __syncwarp();
          if (lane == 0) {
            mbar_arrive(&B.fempty[sf]);
            mbar_arrive(&B.bfull[sb]);
          }
          continue;
        }
#pragma unroll
        for (int k = 0; k < kSKc; ++k) x[k] = ld_shared_f4(src + k * 512);
        if (ch.x < 0 && ch.y + 4 * pc >= ktot) {     // K padding of the contiguous plan
#pragma unroll
          for (int k = 0; k < kSKc; ++k) x[k] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        // time columns of this lane's piece: Phi where the table misses
        const bool tpiece = ch.x == 2 || (ch.x < 0 && ch.y + 4 * pc >= e1 && ch.y + 4 * pc < ktot);
        // branch-free fast path for the 4 x kSKc elements of a time piece (w = 0 past d_t
        // gives cos(0) there, zeroed below); the rare |b| >= 1e9 takes the accurate cosf
        // after ONE warp vote, taken outside the per-lane condition (a chunk of the
        // contiguous plan mixes time and edge-feature pieces)
        const int cc = ch.x < 0 ? ch.y + 4 * pc - e1 : ch.y + 4 * pc;
        float w[4], f[4], cv[kSKc][4];
        bool bad = false;
        bool need = false;                           // a row of this lane misses the table
#pragma unroll
        for (int k = 0; k < kSKc; ++k) need |= trk[k] < 0;
        if (tpiece && need) {
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const bool ok = cc + e < P.d_t;
            w[e] = ok ? s_omega[cc + e] : 0.f;
            f[e] = ok ? s_phi[cc + e] : 0.f;
          }
#pragma unroll
          for (int k = 0; k < kSKc; ++k)
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const float bb = __fadd_rn(__fmul_rn(w[e], dtk[k]), f[e]);   // R10 argument
              bad |= !(fabsf(bb) < 1e9f) && trk[k] < 0;
              cv[k][e] = tenc_cos_reduced(bb);
            }
        }
        if (__any_sync(0xffffffffu, bad) && tpiece && need) {
#pragma unroll
          for (int k = 0; k < kSKc; ++k)
#pragma unroll
            for (int e = 0; e < 4; ++e) cv[k][e] = tenc_fast(dtk[k], w[e], f[e]);
        }
        if (tpiece && need) {
#pragma unroll
          for (int k = 0; k < kSKc; ++k) {
            if (trk[k] < 0) {
              x[k].x = (cc < P.d_t) ? cv[k][0] : 0.f;
              x[k].y = (cc + 1 < P.d_t) ? cv[k][1] : 0.f;
              x[k].z = (cc + 2 < P.d_t) ? cv[k][2] : 0.f;
              x[k].w = (cc + 3 < P.d_t) ? cv[k][3] : 0.f;
            }
          }
        }
        TGL_PROF_CLK(c2a);
        wait_free(&B.bempty[sb], g / kSB);
        TGL_PROF_CLK(c2);
        const uint32_t dst = b_s + sb * kSStage + (uint32_t)cw * (kSRowsPerConv / 8) * 1024;
#pragma unroll
        for (int k = 0; k < kSKc; ++k) {
          // row r0 + 4k: group cw*(rows/8) + k/2, row-in-group (lane>>3) + 4*(k&1)
          const uint32_t ad = dst + (k >> 1) * 1024 + ((k & 1) ? o_odd : o_even);
          uint32_t h0, h1, l0, l1;
          split2(x[k].x, x[k].y, h0, l0);
          split2(x[k].z, x[k].w, h1, l1);
          asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(ad), "r"(h0), "r"(h1) : "memory");
          if (split)
            asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(ad + 512), "r"(l0), "r"(l1)
                         : "memory");
        }
        TGL_PROF_CLK(c3);
        fence_proxy_async_smem();
        __syncwarp();
#ifdef TGL_KV_PROF
        const long long c4 = clock64();
        if (cw == 0) {
          prof_add(a, 0, c1 - c0);
          prof_add(a, 1, c2a - c1);
          prof_add(a, 2, c2 - c2a);
          prof_add(a, 3, c3 - c2);
          prof_add(a, 4, c4 - c3);
        }
#endif
        if (cw == 0) trace(a, 4, g);
        if (lane == 0) {
          mbar_arrive(&B.fempty[sf]);
          mbar_arrive(&B.bfull[sb]);
        }
      }
    }
  } else if (warp == kTMma) {                        // ---------------- MMA issuer
    uint32_t g = 0, wl = 0;
    constexpr uint32_t idesc = idesc_bf16(kBM, kNPkv);
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait(&B.dfull[ds], (tt / kSDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const uint32_t acc = tmem + (tt & 1u) * kCols;
      wait_free(&B.tempty[tt & 1u], tt >> 1);
      tc_fence_after();
      trace(a, 7, tt);
      const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = chunk_of(tt, i, nch);
        const int nk = s_chunk[c].w;
        const uint32_t sb = g % kSB;
        TGL_PROF_CLK(m0);
        mbar_wait(&B.bfull[sb], (g / kSB) & 1u);
        TGL_PROF_CLK(m1);
#ifdef TGL_KV_PROF
        prof_add(a, 7, m1 - m0);
#endif
        trace(a, 12, g);
        uint32_t kw;
        if (i < r0) {
          kw = wl - 1 - i;                           // resident from the previous tile
        } else {
          kw = wl + (i - r0);
          mbar_wait(&B.wfull[kw % kSW], (kw / kSW) & 1u);
        }
        tc_fence_after();
#ifdef TGL_KV_PROF
        prof_add(a, 8, clock64() - m1);
#endif
        trace(a, 5, g);
        if (elect_one()) {
          // descriptors built once per chunk; a K step (32 B) / the lo half advance the
          // 14-bit start-address field (addr >> 4) by plain adds (no carry: smem < 256 KB)
          const uint64_t a0 = desc_sw64(b_s + sb * kSStage, 1024);
          const uint64_t w0 = desc_sw64(w_s + (kw % kSW) * kTWStage, 512);
          if (!(TGL_DBG(a) & 4)) {                        // profiling: no MMAs
#pragma unroll
            for (int ks = 0; ks < 2; ++ks) {
              if (ks < nk) {
                const uint64_t ah = a0 + 2 * ks, bh = w0 + 2 * ks;
                mma_bf16(acc, ah, bh, idesc, (i | ks) != 0);
                if (split) {
                  mma_bf16(acc, ah + (512 >> 4), bh, idesc, 1u);
                  mma_bf16(acc, ah, bh + (kTWHalf >> 4), idesc, 1u);
                }
              }
            }
          }
          const bool keep = (nch >= 4) && (i >= nch - 2);   // reused by the next tile
          if (TGL_DBG(a) & 8192) {                        // profiling: plain arrives, no commit
            mbar_arrive(&B.bempty[sb]);
            if (!keep) mbar_arrive(&B.wempty[kw % kSW]);
          } else {
            mma_commit(&B.bempty[sb]);
            if (!keep) mma_commit(&B.wempty[kw % kSW]);
          }
        }
        __syncwarp();
      }
      wl += nch - r0;
      if (elect_one()) mma_commit(&B.tfull[tt & 1u]);
      __syncwarp();
    }
  } else if (warp < kBEpi) {                         // ---------------- epilogue warps 0-7
    bin_epilogue<kSDSlots, TDesc, kSPW, (kSThreads > 768)>(a, B.dfull, B.dempty, B.tfull,
                                                           B.tempty, bd, tmem, s_pvf, s_bias);
  }
  ws_teardown(tmem, 2 * kCols, kTMma);
}


// ------------------------------------------------------------------ pre-split K|V kernel
// kv_pre_kernel: the split-role design without the converter stage.  The gathered
// feature tables (h_src, e) are stored PRE-SPLIT (tgl_split_rows: per row the bf16 hi
// halves of its columns, then the bf16 lo halves, every segment padded to 8 columns),
// i.e. the exact operands the converters of kv_split_kernel produced on every gather
// -- so loaders move 16-byte hi / lo pieces with LDGSTS straight into the swizzled
// SW64 A stages the MMA reads, and completion is an mbarrier arrival
// (cp.async.mbarrier.arrive.noinc; CUTLASS's sm100 cp.async + UMMA mainloop relies on
// the same ordering).  Only the time columns are produced in the SM: 4 time warps
// evaluate Phi(dt) (table row or direct), split and store them.  K is the contiguous
// concatenation K' = [h (dp0) | e (dp1) | Phi (dpt)] of 8-column groups, cut into
// 32-column chunks; [Wk ; Wv] is packed in the same K' order (zero rows for padding).
// In bf16 mode only the hi halves are loaded (half the gather bytes).
// Roles: epilogue warps 0-7 (bin_epilogue), MMA 8, weights 9, tile descriptors 10-11,
// loaders 12-15, time warps 16-19: 640 threads.
// 4 A stages, 5 weight stages, 4 weight chunks kept across a tile boundary (measured on
// GDELT with node projections: K|V 0.823 -> 0.789 ms against 7 / 3 / 2 -- fewer weight
// refills beat a deeper A ring; the shared-memory budget allows no more)
#ifndef TGL_KV_PRE_ASTAGES
#define TGL_KV_PRE_ASTAGES 4
#endif
#ifndef TGL_KV_PRE_WSTAGES
#define TGL_KV_PRE_WSTAGES 5
#endif
constexpr int kPAStages = TGL_KV_PRE_ASTAGES;         // A stages (hi | lo, 16 KB each)
constexpr int kPAStage = kBM * kTC * 4;                // 16 KB
// weight stages (25.6 KB each): 3, so that a chunk can stream in while the two chunks
// kept across the tile boundary (alternating K order) are still being read -- with 2
// stages the MMA waited ~18 % of the kernel for weights (probe counters, GDELT)
constexpr int kPW = TGL_KV_PRE_WSTAGES;
// weight chunks kept across a tile boundary (the K order alternates per tile).  Kept
// chunks pin weight stages at the boundary, so the next loads queue behind them.
#ifndef TGL_KV_PRE_REUSE
#define TGL_KV_PRE_REUSE 4
#endif
constexpr int kPreReuse = TGL_KV_PRE_REUSE;
static_assert(kPreReuse < kPW, "kept weight chunks must leave a weight stage to stream into");
constexpr int kPLoad0 = 12, kPLoadWarps = 4;
constexpr int kPTime0 = 16, kPTimeWarps = 4;
constexpr int kPThreads = (kPTime0 + kPTimeWarps) * 32;   // 640
constexpr int kPPipeBytes = kPAStages * kPAStage + kPW * kTWStage;
constexpr int kPSmem = 1024 + kPPipeBytes + kBEpi * 32 * kSPW * 4;
constexpr int kPMaxChunks = 64;

struct PrePlan {      // K' = [h: dp0 | e: dp1 | Phi: dpt], 8-column groups, 32-column chunks
  int d0, d1, dt;     // true widths
  int dp0, dp1, dpt;  // padded to multiples of 8
  int k;              // dp0 + dp1 + dpt
  int n;              // chunks
  // issue order of the chunks inside a tile: the chunks holding time columns (produced by
  // the time warps, the slowest producer) spread evenly among the gathered ones, so they
  // never queue back to back at a tile boundary; odd tiles walk the order backwards
  unsigned char order[64];
};
static int pad8h(int x) { return (x + 7) & ~7; }
static PrePlan make_pre_plan(int d0, int d1, int dt) {
  PrePlan p;
  p.d0 = d0; p.d1 = d1; p.dt = dt;
  p.dp0 = pad8h(d0); p.dp1 = pad8h(d1); p.dpt = pad8h(dt);
  p.k = p.dp0 + p.dp1 + p.dpt;
  p.n = (p.k + kTC - 1) / kTC;
  const int ct = (p.dp0 + p.dp1) / kTC;            // first chunk holding time columns
  const int nt = p.n - ct, nf = ct;
  int pos = 0, f = 0, t = 0;
  for (int i = 0; i < p.n && i < 64; ++i) {
    // time chunk j goes to position floor((j + 0.5) n / nt)
    const bool take_t = t < nt && (f >= nf || i >= (int)((t + 0.5) * p.n / (nt > 0 ? nt : 1)));
    p.order[pos++] = (unsigned char)(take_t ? ct + t++ : f++);
  }
  return p;
}

// col_off: the W column of K' column 0 (d_hsrc for the node-projection plan, whose K'
// starts at the e columns)
__global__ void pack_kv_pre_kernel(const float* Wk, const float* Wv, int dm, int ksrc, PrePlan p,
                                   uint8_t* out, int col_off) {
  const int kw = p.n * kTC;
  const int64_t total = (int64_t)kNPkv * kw;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(x / kw), kp = (int)(x % kw);
    const int c = kp / kTC, cc = kp % kTC;
    int src = -1;                                   // column of [h | e | Phi] in W
    if (kp < p.dp0) {
      if (kp < p.d0) src = kp;
    } else if (kp < p.dp0 + p.dp1) {
      if (kp - p.dp0 < p.d1) src = p.d0 + (kp - p.dp0);
    } else if (kp < p.k) {
      if (kp - p.dp0 - p.dp1 < p.dt) src = p.d0 + p.d1 + (kp - p.dp0 - p.dp1);
    }
    float v = 0.f;
    if (src >= 0) src += col_off;
    if (n < 2 * dm && src >= 0)
      v = n < dm ? Wk[(int64_t)n * ksrc + src] : Wv[(int64_t)(n - dm) * ksrc + src];
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    const int64_t off = (int64_t)c * kTWStage + (n >> 3) * 512 + sw64_off(n, cc);
    *reinterpret_cast<__nv_bfloat16*>(out + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(out + off + kTWHalf) = lo;
  }
}

// kv_pre waits: test_wait + nanosleep back-off (default) or the suspend-hint try_wait
// (-DTGL_PRE_SUSPEND: the waiting warp sleeps in hardware, no polling instructions)
#ifdef TGL_PRE_SUSPEND
#define PRE_WAIT_SLEEP(bar, par, ns) mbar_wait(bar, par)
#define PRE_FREE_SLEEP(bar, u, ns) wait_free(bar, u)
#else
#define PRE_WAIT_SLEEP(bar, par, ns) mbar_wait_sleep(bar, par, ns)
#define PRE_FREE_SLEEP(bar, u, ns) wait_free_sleep(bar, u, ns)
#endif

// ring depths as template parameters: <4, 5, 4> (the default) keeps 4 weight chunks across
// a tile boundary; <7, 3, 2> (a deeper A ring) serves k > 16 (LASTFM: one destination per
// 32-row bin, so a tile holds few rows and its gathers need more stages in flight)
template <int AS, int WS>
constexpr int pre_smem_bytes() {
  return 1024 + AS * kPAStage + WS * kTWStage + kBEpi * 32 * kSPW * 4;
}
template <int AS, int WS>
struct PBars {
  uint64_t afull[AS], aempty[AS];
  uint64_t wfull[WS], wempty[WS];
  uint64_t dfull[kSDSlots], dempty[kSDSlots];
  uint64_t tfull[2], tempty[2];
  uint64_t zfull[2];    // node projections: the accumulator holds zkv[row] (loaders)
};

template <int AS, int WS, int RU>
__global__ void __launch_bounds__(kPThreads, 1)
    kv_pre_kernel(const Args a, const PrePlan plan, const uint8_t* __restrict__ wkv,
                  const int bdst) {
  constexpr int kPAStages = AS, kPW = WS, kPreReuse = RU;
  constexpr int kPPipeBytes = AS * kPAStage + WS * kTWStage;
  static_assert(RU < WS, "kept weight chunks must leave a weight stage to stream into");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ PBars<AS, WS> B;
  __shared__ uint32_t s_tmem;
  __shared__ TDesc bd[kSDSlots];
  __shared__ __align__(16) float s_omega[256];
  __shared__ __align__(16) float s_phi[256];
  __shared__ unsigned char s_order[64];      // plan.order (indexed: smem, not a local copy)
  __shared__ float s_bias[2 * kMaxModel];
  __shared__ int64_t s_seg[kTDescWarps][4 * 32 + 1];
  __shared__ float s_td[kTDescWarps][4 * 32];
  float* s_pvf = reinterpret_cast<float*>(pipe + kPPipeBytes);
  constexpr uint32_t kCols = 256;
  constexpr int dm = 100;
  const tgl_attn_params& P = a.P;
  const bool split = a.split != 0;
  const bool np = a.zkv != nullptr;   // TGL_NODE_PROJ: h_src columns come from zkv rows
  const int nch = plan.n;
  // weight chunks kept across a tile boundary: the alternating K order maps tile t+1's
  // chunk i to tile t's stage only while no kept chunk was itself kept (nch >= 2 reuse)
  const int reuse = nch < 4 ? 0 : (nch / 2 < kPreReuse ? nch / 2 : kPreReuse);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // prologue independent of the predecessor grid (PDL): barriers, TMEM, constants
  if (threadIdx.x == 0) {
    for (int s = 0; s < kPAStages; ++s) {
      mbar_init(&B.afull[s], kPLoadWarps * 32 + kPTimeWarps);
      mbar_init(&B.aempty[s], 1);
    }
    for (int s = 0; s < kPW; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kSDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kBEpi + kPLoadWarps + kPTimeWarps + 2);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&B.tfull[s], 1);
      mbar_init(&B.tempty[s], kBEpi);
      mbar_init(&B.zfull[s], kPLoadWarps);
    }
    fence_mbar_init();
  }
  TGL_TRACE_RESET();
  if (warp == kTMma) tmem_alloc(&s_tmem, 2 * kCols);
  for (int j = threadIdx.x; j < 64; j += blockDim.x) s_order[j] = plan.order[j];
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const uint32_t tmem = s_tmem;
  const uint32_t pipe_s = smem_u32(pipe);
  const uint32_t a_s = pipe_s;                                  // A ring
  const uint32_t w_s = pipe_s + kPAStages * kPAStage;           // weight ring
  uint32_t tt = 0;
  const int kt0 = plan.dp0 + plan.dp1;                          // first time column of K'

  if (warp >= kTDesc0 && warp < kTDesc0 + kTDescWarps) {   // ------- tile builders
    const int dw = warp - kTDesc0;
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    const int dpt = 4 * bdst;
    const int64_t ntiles = (n + dpt - 1) / dpt;
    int64_t* sg = s_seg[dw];
    float* stdv = s_td[dw];
    for (tt = dw;; tt += kTDescWarps) {
      const uint32_t ds = tt % kSDSlots;
      PRE_FREE_SLEEP(&B.dempty[ds], tt / kSDSlots, TGL_SLEEP_DESC);
      TDesc& R = bd[ds];
      const int64_t T = blockIdx.x + (int64_t)tt * gridDim.x;
      if (T >= ntiles) {
        if (lane == 0) R.live = 0;
        warp_arrive(&B.dfull[ds]);
        break;
      }
      const int64_t d0 = T * dpt;
      const int nd = (int)((n - d0) < dpt ? (n - d0) : dpt);
      for (int j = lane; j <= nd; j += 32) sg[j] = a.seg_ptr[d0 + j];
      for (int j = lane; j < nd; j += 32) stdv[j] = a.dst_t[d0 + j];
      __syncwarp();
      int64_t er[4] = {0, 0, 0, 0};
      float tr[4] = {0.f, 0.f, 0.f, 0.f};
      int dr[4] = {-1, -1, -1, -1};
      unsigned ovf_bins = 0;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j0 = u * bdst;
        if (j0 >= nd) continue;
        const int j1 = (j0 + bdst) < nd ? j0 + bdst : nd;
        const int64_t e0 = sg[j0], e1 = sg[j1];
        if (e1 - e0 > 32) {
          ovf_bins |= 1u << u;
          continue;
        }
        const int64_t e = e0 + lane;
        if (e < e1) {
          int j = j0;
          while (sg[j + 1] <= e) ++j;
          dr[u] = (int)(d0 + j);
          er[u] = e;
          tr[u] = stdv[j];
        }
      }
      for (int j = 0; j < nd; ++j) {
        const bool ovf = (ovf_bins >> (j / bdst)) & 1u;
        if (sg[j + 1] == sg[j] || ovf) {
          const float fill = ovf ? __int_as_float(0x7fc00000) : 0.f;
          fill_r_row(a, d0 + j, fill, lane, dm);
        }
      }
      R.live = 1;
      int32_t hi[4], ei[4];
      float et[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const bool ok = dr[u] >= 0;
        hi[u] = ok ? (a.hsrc_idx ? a.hsrc_idx[hoff + er[u]] : (int32_t)(hoff + er[u])) : 0;
        ei[u] = (ok && P.d_e > 0) ? a.eid[er[u]] : 0;
        et[u] = ok ? a.edge_t[er[u]] : 0.f;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int r = 32 * u + lane;
        const bool ok = dr[u] >= 0;
        const float dt = tr[u] - et[u];               // fp32 delta (R18)
        R.hrow[r] = ok ? hi[u] : -1;
        R.erow[r] = ok ? ei[u] : -1;
        R.dt[r] = ok ? dt : 0.f;
        R.trow[r] = ok ? (int)tenc_table_row(dt, a.table, a.window) : -1;
        R.rdst[r] = dr[u];
      }
      warp_arrive(&B.dfull[ds]);
    }
  } else if (warp == kTW) {                          // ---------------- weight loader
    uint32_t wl = 0;
    const uint64_t wpol = l2_policy_evict_last();    // weights: re-read by every tile
    const uint32_t wbytes = split ? kTWStage : kTWHalf;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_W);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) {
        const int r0 = tt > 0 ? reuse : 0;
        for (int i = r0; i < nch; ++i) {
          const uint32_t k = wl + (i - r0);
          const uint32_t sw = k % kPW;
          PRE_FREE_SLEEP(&B.wempty[sw], k / kPW, TGL_SLEEP_W);
          mbar_arrive_expect_tx(&B.wfull[sw], wbytes);
          bulk_g2s_hint(pipe + kPAStages * kPAStage + sw * kTWStage,
                        wkv + (size_t)s_order[chunk_of(tt, i, nch)] * kTWStage, wbytes,
                        &B.wfull[sw], wpol);
        }
        wl += nch - r0;
      }
      __syncwarp();
    }
  } else if (warp >= kPLoad0 && warp < kPLoad0 + kPLoadWarps) {   // ---------- loaders
    // lane: rows lw*32 + (lane>>3) + 4k (k = 0..7); piece pc = lane & 7 of the row's
    // 32-column chunk: hi group pc (pc < 4) or lo group pc - 4, 16 bytes each
    const int lw = warp - kPLoad0;
    const int r0 = lw * 32 + (lane >> 3), pc = lane & 7;
    const bool lo_piece = pc >= 4;
    const int j = pc & 3;
    const uint32_t ofs0 = (uint32_t)(r0 >> 3) * 1024 + (lo_piece ? 512 : 0);
    const bool active = split || !lo_piece;         // bf16 mode: hi halves only
    // split16 precompute table: its rows are gathered like features (time warps only
    // evaluate Phi for the rows the table misses)
    const bool tsplit = (P.input_layout & TGL_SPLIT_TABLE) && a.table != nullptr;
    const uint8_t* hbase = reinterpret_cast<const uint8_t*>(a.hsrc);
    const uint8_t* ebase = reinterpret_cast<const uint8_t*>(a.efeat);
    const uint8_t* tbase = reinterpret_cast<const uint8_t*>(a.table);
    const int64_t hld = 4 * a.ld_hsrc, eld = 4 * a.ld_e, tld = 4 * plan.dpt;
    const uint64_t epol = l2_policy_evict_first();
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_LOAD);
      const TDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      int hrow[8], erow[8], trw[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        hrow[k] = R.hrow[r0 + 4 * k];
        erow[k] = R.erow[r0 + 4 * k];
        trw[k] = (tsplit && R.rdst[r0 + 4 * k] >= 0) ? R.trow[r0 + 4 * k] : -1;
      }
      const int zn = np ? R.hrow[lw * 32 + lane] : -1;   // this lane's TMEM row
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      if (np) {
        // the row's h_src part of K|V (eq 5) = zkv[node] (tgl_node_proj): it initialises
        // the accumulator, the MMAs add [e | Phi] W^T on top (padding rows: zeros)
        // 16-column rounds, the next round's loads in flight while this one is stored; the
        // first round is loaded before waiting for the accumulator to be released
        const uint32_t tz = tmem + (tt & 1u) * 256u + ((uint32_t)(lw * 32) << 16);
        const float* zr = a.zkv + (int64_t)(zn >= 0 ? zn : 0) * a.z_ld;
        float4 zb[2][4];
#pragma unroll
        for (int q = 0; q < 4; ++q)
          zb[0][q] = zn >= 0 ? __ldg(reinterpret_cast<const float4*>(zr + 4 * q))
                             : make_float4(0.f, 0.f, 0.f, 0.f);
        wait_free(&B.tempty[tt & 1u], tt >> 1);
        tc_fence_after();
#pragma unroll
        for (int c0 = 0; c0 < 2 * 100; c0 += 16) {
          const int cur = (c0 >> 4) & 1;
          if (c0 + 16 < 2 * 100) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int cc = c0 + 16 + 4 * q;
              zb[cur ^ 1][q] = (zn >= 0 && cc < 200)
                                   ? __ldg(reinterpret_cast<const float4*>(zr + cc))
                                   : make_float4(0.f, 0.f, 0.f, 0.f);
            }
          }
          const float* zv = reinterpret_cast<const float*>(&zb[cur][0]);
          tmem_st8(tz + c0, zv);
          if (c0 + 8 < 2 * 100) tmem_st8(tz + c0 + 8, zv + 8);
        }
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&B.zfull[tt & 1u]);
      }
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = s_order[chunk_of(tt, i, nch)];
        const int col = c * kTC + 8 * j;             // K' column of this piece
        const int ks = (plan.k - c * kTC) > 16 ? 2 : 1;   // K steps the MMA issues
        const uint32_t sa = g % kPAStages;
        TGL_PROF_CLK(l0);
        PRE_FREE_SLEEP(&B.aempty[sa], g / kPAStages, TGL_SLEEP_LOAD);
#ifdef TGL_KV_PROF
        if (lw == 0) prof_add(a, 5, clock64() - l0);  // loader: wait for a free stage
#endif
        const bool in_k = active && col < c * kTC + 16 * ks && !(TGL_DBG(a) & 2);
        const uint32_t dst = a_s + sa * kPAStage + ofs0;
        if (in_k && col < kt0) {                     // a gathered feature piece
          const bool seg_h = col < plan.dp0;
          const uint8_t* base = seg_h ? hbase : ebase;
          const int64_t ldb = seg_h ? hld : eld;
          const uint32_t pofs = seg_h ? (uint32_t)(lo_piece ? 2 * plan.dp0 : 0) + 2 * col
                                      : (uint32_t)(lo_piece ? 2 * plan.dp1 : 0) +
                                            2 * (col - plan.dp0);
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const int row = seg_h ? hrow[k] : erow[k];
            const int rr = (r0 + 4 * k) & 7;
            const uint32_t d = dst + (uint32_t)(k >> 1) * 1024 + rr * 64 +
                               (((j ^ (rr >> 1)) & 3) << 4);
            const void* src = base + (row >= 0 ? (int64_t)row * ldb + pofs : 0);
            if (seg_h)
              cp_async16_zfill(d, src, row >= 0 ? 16u : 0u);
            else                                       // edge rows: streamed once
              cp_async16_zfill_hint(d, src, row >= 0 ? 16u : 0u, epol);
          }
        } else if (in_k && tsplit && col < plan.k) {  // a time piece of a table row
          const uint32_t pofs = (uint32_t)(lo_piece ? 2 * plan.dpt : 0) + 2 * (col - kt0);
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            if (trw[k] < 0) continue;                  // Phi evaluated by the time warps
            const int rr = (r0 + 4 * k) & 7;
            const uint32_t d = dst + (uint32_t)(k >> 1) * 1024 + rr * 64 +
                               (((j ^ (rr >> 1)) & 3) << 4);
            cp_async16_zfill(d, tbase + (int64_t)trw[k] * tld + pofs, 16u);
          }
        }                                            // (other time + K padding: time warps)
        cp_async_mbar_arrive_noinc(&B.afull[sa]);
      }
    }
  } else if (warp >= kPTime0 && warp < kPTime0 + kPTimeWarps) {   // -------- time warps
    // thread: row w*32 + lane, the 8-column groups of every chunk that holds time
    // columns: Phi (eq 8, R10 argument; reduced + SFU cosine, the accurate cosf only
    // where a row's |argument| >= 1e9) -> bf16 hi / lo -> the A stage
    const int tw = warp - kPTime0;
    const int r = tw * 32 + lane;
    const int rr = r & 7;
    const bool tsplit = (P.input_layout & TGL_SPLIT_TABLE) && a.table != nullptr;
    const uint32_t rofs = (uint32_t)(r >> 3) * 1024 + rr * 64;
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_LOAD);
      const TDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      const float dtr = R.dt[r];
      // 0: evaluate Phi; 1: table row (split16: gathered by the loaders, fp32: read here);
      // 2: padding row (zeros)
      const int trow = R.trow[r];
      const int mode = R.rdst[r] < 0 ? 2 : (trow >= 0 ? 1 : 0);
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = s_order[chunk_of(tt, i, nch)];
        const int ks = (plan.k - c * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kPAStages;
        const bool has_time = (c + 1) * kTC > kt0 && !(TGL_DBG(a) & 64);
        if (has_time) {
          TGL_PROF_CLK(t0);
          wait_free(&B.aempty[sa], g / kPAStages);
          TGL_PROF_CLK(t1);
          const uint32_t dst = a_s + sa * kPAStage + rofs;
TGL_SMALL_UNROLL
          for (int jj = 0; jj < 4; ++jj) {
            const int col = c * kTC + 8 * jj;
            if (col < kt0 || col >= c * kTC + 16 * ks) continue;     // warp-uniform
            const int tc = col - kt0;                 // time column of the group
            if (tsplit && mode == 1 && col < plan.k) continue;   // gathered from the table
            float x[8];
            if (mode == 0) {
              // omega / phi of the group as four 16-byte loads (tc is a multiple of 8): the
              // shared-memory pipe is busy with the tensor core's operand reads, so each
              // scalar load waited its turn (the group's 16 of them, not the cosine, were
              // the time warps' cost)
              float om[8], ph[8];
              *reinterpret_cast<float4*>(om) = *reinterpret_cast<const float4*>(s_omega + tc);
              *reinterpret_cast<float4*>(om + 4) =
                  *reinterpret_cast<const float4*>(s_omega + tc + 4);
              *reinterpret_cast<float4*>(ph) = *reinterpret_cast<const float4*>(s_phi + tc);
              *reinterpret_cast<float4*>(ph + 4) = *reinterpret_cast<const float4*>(s_phi + tc + 4);
              bool bad = false;
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                const float bb = __fadd_rn(__fmul_rn(om[e], dtr), ph[e]);
                bad |= !(fabsf(bb) < 1e9f);
                x[e] = tenc_cos_reduced(bb);
              }
              if (bad) {                              // rare: |b| >= 1e9 or non-finite
#pragma unroll
                for (int e = 0; e < 8; ++e) x[e] = tenc_fast(dtr, s_omega[tc + e], s_phi[tc + e]);
              }
            } else if (mode == 1 && !tsplit) {
#pragma unroll
              for (int e = 0; e < 8; ++e)
                x[e] = tc + e < P.d_t ? __ldg(a.table + (int64_t)trow * P.d_t + tc + e) : 0.f;
            } else {
#pragma unroll
              for (int e = 0; e < 8; ++e) x[e] = 0.f;
            }
            if (tc + 8 > P.d_t) {                     // padding columns of the time segment
#pragma unroll
              for (int e = 0; e < 8; ++e)
                if (tc + e >= P.d_t) x[e] = 0.f;
            }
            uint32_t h[4], l[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) split2(x[2 * e], x[2 * e + 1], h[e], l[e]);
            const uint32_t po = (uint32_t)(((jj ^ (rr >> 1)) & 3) << 4);
            st_shared_v4_nc(dst + po, h[0], h[1], h[2], h[3]);
            if (split) st_shared_v4_nc(dst + 512 + po, l[0], l[1], l[2], l[3]);
          }
          TGL_PROF_CLK(t2);
          fence_proxy_async_smem();
          TGL_PROF_CLK(t3);
          __syncwarp();
#ifdef TGL_KV_PROF
          if (tw == 0) {
            prof_add(a, 0, t1 - t0);                   // time warp: wait for a free stage
            prof_add(a, 1, clock64() - t1);            // time warp: Phi + split + store
            prof_add(a, 2, t2 - t1);                   //   of which Phi + split + st.shared
            prof_add(a, 3, t3 - t2);                   //   of which fence.proxy.async
          }
#endif
          if (lane == 0) mbar_arrive(&B.afull[sa]);
        } else {
          // no time columns: arrive once the stage's previous use is released, so the
          // arrival counts toward this chunk's phase
          TGL_PROF_CLK(n0);
          if (lane == 0) {
            wait_free(&B.aempty[sa], g / kPAStages);
            mbar_arrive(&B.afull[sa]);
          }
          __syncwarp();
#ifdef TGL_KV_PROF
          if (tw == 0) prof_add(a, 4, clock64() - n0);  // time warp: non-time chunk pass
#endif
        }
      }
    }
  } else if (warp == kTMma) {                        // ---------------- MMA issuer
    uint32_t g = 0, wl = 0;
    constexpr uint32_t idesc = idesc_bf16(kBM, kNPkv);
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait(&B.dfull[ds], (tt / kSDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const uint32_t acc = tmem + (tt & 1u) * kCols;
      TGL_PROF_CLK(mt0);
      wait_free(&B.tempty[tt & 1u], tt >> 1);
      if (np) mbar_wait(&B.zfull[tt & 1u], (tt >> 1) & 1u);   // zkv rows stored
      TGL_PROF_CLK(mt1);
#ifdef TGL_KV_PROF
      prof_add(a, 7, mt1 - mt0);                     // MMA: wait for an accumulator
#endif
      tc_fence_after();
      const int r0 = tt > 0 ? reuse : 0;
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = s_order[chunk_of(tt, i, nch)];
        const int nk = (plan.k - c * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kPAStages;
        TGL_PROF_CLK(ma0);
        mbar_wait(&B.afull[sa], (g / kPAStages) & 1u);
        TGL_PROF_CLK(ma1);
        uint32_t kw;
        if (i < r0) {
          kw = wl - 1 - i;                           // resident from the previous tile
        } else {
          kw = wl + (i - r0);
          mbar_wait(&B.wfull[kw % kPW], (kw / kPW) & 1u);
        }
#ifdef TGL_KV_PROF
        prof_add(a, (c + 1) * kTC > kt0 ? 9 : 8, ma1 - ma0);   // MMA: A wait (time / gathered)
        prof_add(a, 10, clock64() - ma1);            // MMA: W wait
#endif
        tc_fence_after();
        if (elect_one()) {
          const uint64_t a0 = desc_sw64(a_s + sa * kPAStage, 1024);
          const uint64_t w0 = desc_sw64(w_s + (kw % kPW) * kTWStage, 512);
#pragma unroll
          for (int ks = 0; ks < 2; ++ks) {
            if (ks < nk && !(TGL_DBG(a) & 4)) {
              const uint64_t ah = a0 + 2 * ks, bh = w0 + 2 * ks;
              mma_bf16(acc, ah, bh, idesc, np || (i | ks) != 0);
              if (split) {
                mma_bf16(acc, ah + (512 >> 4), bh, idesc, 1u);
                mma_bf16(acc, ah, bh + (kTWHalf >> 4), idesc, 1u);
              }
            }
          }
          const bool keep = reuse > 0 && i >= nch - reuse;   // reused by the next tile
          mma_commit(&B.aempty[sa]);
          if (!keep) mma_commit(&B.wempty[kw % kPW]);
        }
        __syncwarp();
      }
      wl += nch - r0;
      if (elect_one()) mma_commit(&B.tfull[tt & 1u]);
      __syncwarp();
    }
  } else if (warp < kBEpi) {                         // ---------------- epilogue warps 0-7
    bin_epilogue<kSDSlots, TDesc, kSPW, false>(a, B.dfull, B.dempty, B.tfull, B.tempty, bd,
                                               tmem, s_pvf, s_bias);
  }
  ws_teardown(tmem, 2 * kCols, kTMma);
}


// ------------------------------------------------------------------ S8 / S13 on split16 rows
// dense_pre_kernel<kFfn>: the dense projections with converter-free operands, the same
// scheme as kv_pre.  A = [seg0 | seg1] of split16 rows (8-column groups, 32-column
// chunks), gathered by LDGSTS straight into the SW64 stages; the MMA is M=128 N=104.
//   Q   (kFfn = 0): seg0 = h_dst (hdst split16, row hdst_idx[i]); Phi(0) = cos(phi) is the
//       same for every destination, so Wq[:, d_hdst:] Phi(0) is folded into the bias
//       (computed once by the pack kernel, fp64 accumulate) -- K = d_hdst only.
//   FFN (kFfn = 1): seg0 = r_i (the K|V epilogue writes it split16), seg1 = h_dst.
// Roles: epilogue warps 0-3 (one row per thread, TMEM lane quarter = warp), MMA 4,
// descriptors 5, weights 6, loaders 7-10: 352 threads.
constexpr int kDPAStages = 6;
constexpr int kDPWStage = 2 * kDPN * 64;               // hi | lo of a 32-column chunk
// 8 weight stages: tgl_node_proj applies 4 weight chunks to every A chunk, so a 4-deep
// ring could not fetch ahead across A chunks (latency-bound: 36 us for GDELT's nodes)
constexpr int kDPW = 8;
constexpr int kDPLoad0 = 7, kDPLoadWarps = 4;
constexpr int kDPThreads = (kDPLoad0 + kDPLoadWarps) * 32;   // 352
constexpr int kDPPipeBytes = kDPAStages * kPAStage + kDPW * kDPWStage;
constexpr int kDPSmem = 1024 + kDPPipeBytes;

struct DPPlan {        // K' = [seg0: dp0 | seg1: dp1], 32-column chunks
  int d0, d1, dp0, dp1, k, n;
};
static DPPlan make_dp_plan(int d0, int d1) {
  DPPlan p;
  p.d0 = d0; p.d1 = d1;
  p.dp0 = pad8h(d0); p.dp1 = pad8h(d1);
  p.k = p.dp0 + p.dp1;
  p.n = (p.k + kTC - 1) / kTC;
  return p;
}

// W [n_out][ksrc] (columns [c0, c0 + d0) then [c1, c1 + d1)) in the K' order, packed as
// kv_pre packs [Wk ; Wv] but with N = 104 rows; qfold != nullptr (Q only): bias'[n] =
// b[n] + sum_j W[n][d_hdst + j] cos(phi_j) (Phi(0), R10: fl(omega * 0 + phi) = phi)
__global__ void pack_dense_pre_kernel(const float* W, int n_out, int ksrc, int c0, int c1,
                                      DPPlan p, uint8_t* out, const float* b, const float* phi,
                                      int d_t, int col_t, float* bias_out) {
  const int kw = p.n * kTC;
  const int64_t total = (int64_t)kDPN * kw;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(x / kw), kp = (int)(x % kw);
    const int c = kp / kTC, cc = kp % kTC;
    int src = -1;
    if (kp < p.dp0) {
      if (kp < p.d0) src = c0 + kp;
    } else if (kp < p.k) {
      if (kp - p.dp0 < p.d1) src = c1 + (kp - p.dp0);
    }
    const float v = (n < n_out && src >= 0) ? W[(int64_t)n * ksrc + src] : 0.f;
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    const int64_t off = (int64_t)c * kDPWStage + (n >> 3) * 512 + sw64_off(n, cc);
    *reinterpret_cast<__nv_bfloat16*>(out + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(out + off + kDPN * 64) = lo;
  }
  if (bias_out != nullptr && blockIdx.x == 0) {
    for (int n = threadIdx.x; n < n_out; n += blockDim.x) {
      double acc = b != nullptr ? b[n] : 0.0;
      if (phi != nullptr)
        for (int j = 0; j < d_t; ++j)
          acc += (double)W[(int64_t)n * ksrc + col_t + j] * (double)cosf(phi[j]);
      bias_out[n] = (float)acc;
    }
  }
}

struct DPBars {
  uint64_t afull[kDPAStages], aempty[kDPAStages];
  uint64_t wfull[kDPW], wempty[kDPW];
  uint64_t dfull[kDSlots], dempty[kDSlots];
  uint64_t tfull[2], tempty[2];
  uint64_t zfull[2];    // FFN on node projections: the accumulator holds zo[row] (loaders)
};
// what one grid row (blockIdx.y) of dense_pre computes: Q form (kFfn = 0) writes
// out[i] = A_i W^T + bias (+ q.b_k per head after column D when qbk != null) with row
// pitch ld; the FFN form writes LayerNorm(ReLU(A_i W^T + b_o [+ zo[node_i]])) rows
struct DPJob {
  const uint8_t* wpk;
  const float* bias;
  const float* qbk;
  float* out;
  int64_t ld;
};
struct DPJobs {
  DPJob j[4];
  int n;         // > 1: n jobs share each A chunk (Q form, gridDim.y == 1)
};

struct DPDesc {
  int row0[kBM];
  int row1[kBM];
  int live;
  int rows;
  int64_t i0;
};

template <bool kFfn>
__global__ void __launch_bounds__(kDPThreads, 1)
    dense_pre_kernel(const Args a, const DPPlan plan, const DPJobs jobs) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ DPBars B;
  __shared__ uint32_t s_tmem;
  __shared__ DPDesc bd[kDSlots];
  // Q form with nj > 1 (tgl_node_proj): nj jobs share every A chunk (one accumulator
  // of 128 columns each, single-buffered); else one job per grid row, double-buffered
  __shared__ float s_v0[4 * kMaxModel], s_v1[4 * kMaxModel], s_v2[kMaxModel];
  constexpr uint32_t kCols = 128;
  const tgl_attn_params& P = a.P;
  const int nj = (!kFfn && jobs.n > 1) ? jobs.n : 1;
  const bool zo = kFfn && a.zo != nullptr;   // FFN on node projections (TGL_NODE_PROJ)
  const DPJob& J = jobs.j[nj > 1 ? 0 : blockIdx.y];
  const uint32_t tcols = nj > 1 ? 512u : 2u * kCols;
  const bool split = a.split != 0;
  const int nch = plan.n;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kDPAStages; ++s) {
      mbar_init(&B.afull[s], kDPLoadWarps * 32);
      mbar_init(&B.aempty[s], 1);
    }
    for (int s = 0; s < kDPW; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kEpiWarps + kDPLoadWarps + 2);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&B.tfull[s], 1);
      mbar_init(&B.tempty[s], kEpiWarps);
      mbar_init(&B.zfull[s], kDPLoadWarps);
    }
    fence_mbar_init();
  }
  if (warp == kMmaWarp) tmem_alloc(&s_tmem, tcols);
  for (int j = threadIdx.x; j < P.d_model; j += blockDim.x) {
    if (kFfn) {
      s_v0[j] = P.bo[j];
      s_v1[j] = P.ln_gamma[j];
      s_v2[j] = P.ln_beta[j];
    } else {
      for (int jj = 0; jj < nj; ++jj) {
        const DPJob& Jj = jobs.j[nj > 1 ? jj : blockIdx.y];
        s_v0[jj * kMaxModel + j] = Jj.bias ? Jj.bias[j] : 0.f;   // bq + Wq[:, d_hdst:] Phi(0)
        s_v1[jj * kMaxModel + j] = Jj.qbk ? Jj.qbk[j] : 0.f;
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const uint32_t tmem = s_tmem;
  const uint32_t a_s = smem_u32(pipe);
  const uint32_t w_s = a_s + kDPAStages * kPAStage;
  const int64_t ntiles = (n + kBM - 1) / kBM;
  uint32_t tt = 0;
  // split16 row tables: seg0 / seg1 base and pitch (bytes)
  const uint8_t* b0 = reinterpret_cast<const uint8_t*>(kFfn ? (const void*)a.rsplit
                                                            : (const void*)a.hdst);
  const int64_t ld0 = kFfn ? 4 * (int64_t)kDPN : 4 * a.ld_hdst;
  const uint8_t* b1 = reinterpret_cast<const uint8_t*>(a.hdst);
  const int64_t ld1 = 4 * a.ld_hdst;

  if (warp == kDescWarp) {                           // ---------------- row descriptors
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      wait_free(&B.dempty[ds], tt / kDSlots);
      DPDesc& R = bd[ds];
      const int64_t T = blockIdx.x + (int64_t)tt * gridDim.x;
      if (T >= ntiles) {
        if (lane == 0) R.live = 0;
        warp_arrive(&B.dfull[ds]);
        break;
      }
      const int64_t i0 = T * kBM;
      const int rows = (int)((n - i0) < kBM ? (n - i0) : kBM);
#pragma unroll
      for (int u = 0; u < kBM / 32; ++u) {
        const int r = lane + 32 * u;
        int hrow = -1;
        if (r < rows) hrow = a.hdst_idx ? a.hdst_idx[i0 + r] : (int)(i0 + r);
        R.row0[r] = kFfn ? (r < rows ? (int)(i0 + r) : -1) : hrow;
        R.row1[r] = kFfn ? hrow : -1;
      }
      if (lane == 0) {
        R.live = 1;
        R.rows = rows;
        R.i0 = i0;
      }
      warp_arrive(&B.dfull[ds]);
    }
  } else if (warp == kWWarp) {                       // ---------------- weight loader
    uint32_t k = 0;
    const uint32_t wbytes = split ? kDPWStage : kDPN * 64;
    const uint64_t wpol = l2_policy_evict_last();
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) {
        for (int i = 0; i < nch; ++i) {
          for (int jj = 0; jj < nj; ++jj, ++k) {
            const uint32_t sw = k % kDPW;
            wait_free(&B.wempty[sw], k / kDPW);
            mbar_arrive_expect_tx(&B.wfull[sw], wbytes);
            bulk_g2s_hint(pipe + kDPAStages * kPAStage + sw * kDPWStage,
                          jobs.j[nj > 1 ? jj : blockIdx.y].wpk + (size_t)i * kDPWStage, wbytes,
                          &B.wfull[sw], wpol);
          }
        }
      }
      __syncwarp();
    }
  } else if (warp >= kDPLoad0 && warp < kDPLoad0 + kDPLoadWarps) {   // ---------- loaders
    const int lw = warp - kDPLoad0;
    const int r0 = lw * 32 + (lane >> 3), pc = lane & 7;
    const bool lo_piece = pc >= 4;
    const int j = pc & 3;
    const uint32_t ofs0 = (uint32_t)(r0 >> 3) * 1024 + (lo_piece ? 512 : 0);
    const bool active = split || !lo_piece;
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const DPDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      int x0[8], x1[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        x0[k] = R.row0[r0 + 4 * k];
        x1[k] = R.row1[r0 + 4 * k];
      }
      const int tq = warp & 3;                       // this warp's TMEM lane quarter
      const int zn = zo ? R.row1[tq * 32 + lane] : -1;
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      if (zo) {
        // h_i Wo_h^T = zo[node_i] (tgl_node_proj) initialises the accumulator; the MMAs
        // add r_i Wo_r^T.  16-column rounds, the next round's loads in flight.
        const uint32_t tz = tmem + (tt & 1u) * kCols + ((uint32_t)(tq * 32) << 16);
        const float* zr = a.zo + (int64_t)(zn >= 0 ? zn : 0) * a.z_ld;
        float4 zb[2][4];
#pragma unroll
        for (int q = 0; q < 4; ++q)
          zb[0][q] = zn >= 0 ? __ldg(reinterpret_cast<const float4*>(zr + 4 * q))
                             : make_float4(0.f, 0.f, 0.f, 0.f);
        wait_free(&B.tempty[tt & 1u], tt >> 1);
        tc_fence_after();
#pragma unroll
        for (int c0 = 0; c0 < kDPN; c0 += 16) {
          const int cur = (c0 >> 4) & 1;
          if (c0 + 16 < kDPN) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int cc = c0 + 16 + 4 * q;
              zb[cur ^ 1][q] = (zn >= 0 && cc < P.d_model)
                                   ? __ldg(reinterpret_cast<const float4*>(zr + cc))
                                   : make_float4(0.f, 0.f, 0.f, 0.f);
            }
          }
          const float* zv = reinterpret_cast<const float*>(&zb[cur][0]);
          tmem_st8(tz + c0, zv);
          if (c0 + 8 < kDPN) tmem_st8(tz + c0 + 8, zv + 8);
        }
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&B.zfull[tt & 1u]);
      }
      for (int i = 0; i < nch; ++i, ++g) {
        const int col = i * kTC + 8 * j;
        const int ks = (plan.k - i * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kDPAStages;
        wait_free(&B.aempty[sa], g / kDPAStages);
        if (active && col < i * kTC + 16 * ks) {
          const bool s0 = col < plan.dp0;
          const bool pad = col >= plan.k;
          const uint8_t* base = s0 ? b0 : b1;
          const int64_t ldb = s0 ? ld0 : ld1;
          const int dpw = s0 ? plan.dp0 : plan.dp1;
          const int lc = s0 ? col : col - plan.dp0;
          const uint32_t pofs = (uint32_t)(lo_piece ? 2 * dpw : 0) + 2 * lc;
          const uint32_t dst = a_s + sa * kPAStage + ofs0;
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const int row = s0 ? x0[k] : x1[k];
            const int rr = (r0 + 4 * k) & 7;
            const uint32_t d = dst + (uint32_t)(k >> 1) * 1024 + rr * 64 +
                               (((j ^ (rr >> 1)) & 3) << 4);
            const bool ok = row >= 0 && !pad;
            cp_async16_zfill(d, ok ? base + (int64_t)row * ldb + pofs : b0, ok ? 16u : 0u);
          }
        }
        cp_async_mbar_arrive_noinc(&B.afull[sa]);
      }
    }
  } else if (warp == kMmaWarp) {                     // ---------------- MMA issuer
    uint32_t g = 0, k = 0;
    constexpr uint32_t idesc = idesc_bf16(kBM, kDPN);
    for (;; ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const uint32_t ab = nj > 1 ? 0u : (tt & 1u);
      const uint32_t acc0 = tmem + ab * kCols;
      if (nj > 1) wait_free(&B.tempty[0], tt);
      else wait_free(&B.tempty[ab], tt >> 1);
      if (zo) mbar_wait(&B.zfull[ab], (tt >> 1) & 1u);   // zo rows stored
      tc_fence_after();
      for (int i = 0; i < nch; ++i, ++g) {
        const int nk = (plan.k - i * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kDPAStages;
        mbar_wait(&B.afull[sa], (g / kDPAStages) & 1u);
        for (int jj = 0; jj < nj; ++jj, ++k) {
          const uint32_t sw = k % kDPW;
          const uint32_t acc = acc0 + (uint32_t)jj * kCols;
          mbar_wait(&B.wfull[sw], (k / kDPW) & 1u);
          tc_fence_after();
          if (elect_one()) {
            const uint64_t a0 = desc_sw64(a_s + sa * kPAStage, 1024);
            const uint64_t w0 = desc_sw64(w_s + sw * kDPWStage, 512);
#pragma unroll
            for (int ks = 0; ks < 2; ++ks) {
              if (ks < nk) {
                const uint64_t ah = a0 + 2 * ks, bh = w0 + 2 * ks;
                mma_bf16(acc, ah, bh, idesc, zo || (i | ks) != 0);
                if (split) {
                  mma_bf16(acc, ah + (512 >> 4), bh, idesc, 1u);
                  mma_bf16(acc, ah, bh + ((kDPN * 64) >> 4), idesc, 1u);
                }
              }
            }
            mma_commit(&B.wempty[sw]);
            if (jj == nj - 1) mma_commit(&B.aempty[sa]);
          }
          __syncwarp();
        }
      }
      if (elect_one()) mma_commit(&B.tfull[ab]);
      __syncwarp();
    }
  } else if (warp < kEpiWarps) {                     // ---------------- epilogue
    const int row = warp * 32 + lane;
    const int D = P.d_model;
    for (;; ++tt) {
      const uint32_t ab = nj > 1 ? 0u : (tt & 1u), ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      const int live = bd[ds].live;
      const int rows = bd[ds].rows;
      const int64_t i0 = bd[ds].i0;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      mbar_wait(&B.tfull[ab], (nj > 1 ? tt : (tt >> 1)) & 1u);
      tc_fence_after();
      float v[32];
      if (!kFfn) {
#pragma unroll 1
       for (int jb = 0; jb < nj; ++jb) {
        const DPJob& Jj = jobs.j[nj > 1 ? jb : blockIdx.y];
        const float* sb = s_v0 + jb * kMaxModel;
        const float* sk = s_v1 + jb * kMaxModel;
        const uint32_t ta = tmem + (ab + (uint32_t)jb) * kCols + ((uint32_t)(warp * 32) << 16);
        float* q = Jj.out + (i0 + row) * Jj.ld;
        const int dhq = D / P.n_heads;
        float qb0 = 0.f, qb1 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (row < rows) {
#pragma unroll
            for (int jj = 0; jj < 32; jj += 4) {
              const int col = cq * 32 + jj;
              if (col < D) {
                float4 o = make_float4(v[jj] + sb[col], v[jj + 1] + sb[col + 1],
                                       v[jj + 2] + sb[col + 2], v[jj + 3] + sb[col + 3]);
                *reinterpret_cast<float4*>(q + col) = o;
                const float oq[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                  const float pb = oq[e] * sk[col + e];
                  if (col + e < dhq) qb0 += pb; else qb1 += pb;
                }
              }
            }
          }
        }
        if (row < rows && Jj.qbk != nullptr && D + 2 <= Jj.ld) {
          q[D] = qb0;
          q[D + 1] = qb1;
        }
       }
      } else {
        // (node projections: the accumulator already holds + h_i Wo_h^T, see the loaders)
        const uint32_t ta = tmem + ab * kCols + ((uint32_t)(warp * 32) << 16);
        float s = 0.f, s2 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) {
            const int col = cq * 32 + jj;
            if (col < D) {
              const float y = fmaxf(v[jj] + s_v0[col], 0.f);
              s += y;
              s2 = fmaf(y, y, s2);
            }
          }
        }
        const float mean = s / (float)D;
        const float var = fmaxf(s2 / (float)D - mean * mean, 0.f);
        const float inv = rsqrtf(var + P.ln_eps);
        float* o = J.out + (i0 + row) * J.ld;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (row < rows) {
#pragma unroll
            for (int jj = 0; jj < 32; jj += 4) {
              const int col = cq * 32 + jj;
              if (col < D) {
                float r4[4];
#pragma unroll
                for (int e = 0; e < 4; ++e)
                  r4[e] = (fmaxf(v[jj + e] + s_v0[col + e], 0.f) - mean) * inv * s_v1[col + e] +
                          s_v2[col + e];
                *reinterpret_cast<float4*>(o + col) = make_float4(r4[0], r4[1], r4[2], r4[3]);
              }
            }
          }
        }
      }
      tc_fence_before();
      warp_arrive(&B.tempty[ab]);
    }
  }
  ws_teardown(tmem, tcols, kMmaWarp);
}

// ------------------------------------------------------------------ 2-SM pre-split K|V kernel
// kv_pre2_kernel: kv_pre on a CTA pair (cluster of 2 on one TPC), one
// tcgen05.mma.cta_group::2 of M = 256 per K step: rows 0-127 are the leader's tile, rows
// 128-255 the peer's (two independent 128-row tiles), and the weight chunk's N = 208
// rows ([Wk ; Wv] padded with 8 zero rows) are split between the two shared memories
// (104 rows each), so every SM reads and fills HALF of the weight stream -- per 32-column
// chunk ~72 KB of shared-memory traffic per SM instead of ~104 KB, below the MMA time.
// The leader issues the MMAs; the peer's MMA warp relays its A / W readiness to the
// leader (local barrier wait, then a cluster-scope remote arrive); MMA completion is
// committed to both CTAs' barriers (multicast); the peer's epilogue releases the
// leader's accumulator barrier remotely.  Each CTA's epilogue reads its own TMEM rows.
#ifndef TGL_KV_PRE2_ASTAGES
#define TGL_KV_PRE2_ASTAGES 8
#endif
#ifndef TGL_KV_PRE2_WSTAGES
#define TGL_KV_PRE2_WSTAGES 4
#endif
constexpr int kP2AStages = TGL_KV_PRE2_ASTAGES;
#ifndef TGL_KV_PRE_AUTO_PAIR
#define TGL_KV_PRE_AUTO_PAIR 0
#endif
constexpr bool kPreAutoPair = TGL_KV_PRE_AUTO_PAIR != 0;   // AUTO picks the pair kernel
constexpr int kP2N = 208;                              // N of the pair MMA (multiple of 16)
constexpr int kP2Half = (kP2N / 2) * 64;               // 6656 B: one of hi / lo per CTA
constexpr int kP2WStage = 2 * kP2Half;                 // 13312 B per CTA per chunk
constexpr int kP2W = TGL_KV_PRE2_WSTAGES;
constexpr int kP2PipeBytes = kP2AStages * kPAStage + kP2W * kP2WStage;
constexpr int kP2Smem = 1024 + kP2PipeBytes + kBEpi * 32 * kSPW * 4;

__global__ void pack_kv_pre2_kernel(const float* Wk, const float* Wv, int dm, int ksrc,
                                    PrePlan p, uint8_t* out) {
  const int kw = p.n * kTC;
  const int64_t total = (int64_t)kP2N * kw;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(x / kw), kp = (int)(x % kw);
    const int c = kp / kTC, cc = kp % kTC;
    int src = -1;
    if (kp < p.dp0) {
      if (kp < p.d0) src = kp;
    } else if (kp < p.dp0 + p.dp1) {
      if (kp - p.dp0 < p.d1) src = p.d0 + (kp - p.dp0);
    } else if (kp < p.k) {
      if (kp - p.dp0 - p.dp1 < p.dt) src = p.d0 + p.d1 + (kp - p.dp0 - p.dp1);
    }
    float v = 0.f;
    if (n < 2 * dm && src >= 0)
      v = n < dm ? Wk[(int64_t)n * ksrc + src] : Wv[(int64_t)(n - dm) * ksrc + src];
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    const int r = n / (kP2N / 2), nn = n % (kP2N / 2);
    const int64_t off = (int64_t)c * 2 * kP2WStage + r * kP2WStage + (nn >> 3) * 512 +
                        sw64_off(nn, cc);
    *reinterpret_cast<__nv_bfloat16*>(out + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(out + off + kP2Half) = lo;
  }
}

__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa_shared(uint32_t saddr, uint32_t rank) {
  uint32_t d;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(d) : "r"(saddr), "r"(rank));
  return d;
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cl_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cl_addr)
               : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.b32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;"
               ::: "memory");
}
__device__ __forceinline__ void mma_bf16_pair(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                              uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma_commit_pair(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64"
      " [%0], %1;" ::"r"(smem_u32(bar)), "h"((uint16_t)3)
      : "memory");
}

struct P2Bars {
  uint64_t afull[kP2AStages], aempty[kP2AStages], pfull[kP2AStages];
  uint64_t wfull[kP2W], wempty[kP2W];
  uint64_t dfull[kSDSlots], dempty[kSDSlots];
  uint64_t tfull[2], tempty[2];
};

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kPThreads, 1)
    kv_pre2_kernel(const Args a, const PrePlan plan, const uint8_t* __restrict__ wkv,
                   const int bdst) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ P2Bars B;
  __shared__ uint32_t s_tmem;
  __shared__ TDesc bd[kSDSlots];
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  __shared__ int64_t s_seg[kTDescWarps][4 * 32 + 1];
  __shared__ float s_td[kTDescWarps][4 * 32];
  float* s_pvf = reinterpret_cast<float*>(pipe + kP2PipeBytes);
  constexpr uint32_t kCols = 256;
  constexpr int dm = 100;
  const tgl_attn_params& P = a.P;
  const bool split = a.split != 0;
  const int nch = plan.n;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;
#ifdef TGL_KV_PROF
  const long long k0c = clock64();
#endif
  const int64_t pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kP2AStages; ++s) {
      mbar_init(&B.afull[s], kPLoadWarps * 32 + kPTimeWarps);
      mbar_init(&B.aempty[s], 1);
      mbar_init(&B.pfull[s], 1);
    }
    for (int s = 0; s < kP2W; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kSDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kBEpi + kPLoadWarps + kPTimeWarps + 2);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&B.tfull[s], 1);
      mbar_init(&B.tempty[s], 2 * kBEpi);             // both CTAs' epilogues
    }
    fence_mbar_init();
  }
  TGL_TRACE_RESET();
  if (warp == kTMma) {                               // paired TMEM allocation
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&s_tmem)),
                 "r"(2 * kCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = threadIdx.x; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  tc_fence_before();
  cluster_sync_all();                                // peer barriers initialised
  tc_fence_after();
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const uint32_t tmem = s_tmem;
  const uint32_t pipe_s = smem_u32(pipe);
  const uint32_t a_s = pipe_s;
  const uint32_t w_s = pipe_s + kP2AStages * kPAStage;
  const int dpt = 4 * bdst;
  const int64_t ntiles = (n + dpt - 1) / dpt;
  const int64_t npt = (ntiles + 1) / 2;               // pair tiles
  uint32_t tt = 0;
  const int kt0 = plan.dp0 + plan.dp1;

  if (warp >= kTDesc0 && warp < kTDesc0 + kTDescWarps) {   // ------- tile builders
    const int dw = warp - kTDesc0;
    const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
    int64_t* sg = s_seg[dw];
    float* stdv = s_td[dw];
    for (tt = dw;; tt += kTDescWarps) {
      const uint32_t ds = tt % kSDSlots;
      TGL_PROF_CLK(d0c);
      PRE_FREE_SLEEP(&B.dempty[ds], tt / kSDSlots, TGL_SLEEP_DESC);
#ifdef TGL_KV_PROF
      if (dw == 0) prof_add(a, 10, clock64() - d0c);  // desc: wait for a slot
#endif
      TDesc& R = bd[ds];
      const int64_t PT = pair + (int64_t)tt * npairs;
      if (PT >= npt) {
        if (lane == 0) R.live = 0;
        warp_arrive(&B.dfull[ds]);
        break;
      }
      const int64_t T = 2 * PT + rank;                 // this CTA's 128-row tile
      const int64_t d0 = T * dpt;
      int nd = (int)((n - d0) < dpt ? (n - d0) : dpt);
      nd = nd < 0 ? 0 : nd;
      for (int j = lane; j <= nd; j += 32) sg[j] = a.seg_ptr[d0 + j];
      for (int j = lane; j < nd; j += 32) stdv[j] = a.dst_t[d0 + j];
      __syncwarp();
      int64_t er[4] = {0, 0, 0, 0};
      float tr[4] = {0.f, 0.f, 0.f, 0.f};
      int dr[4] = {-1, -1, -1, -1};
      unsigned ovf_bins = 0;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j0 = u * bdst;
        if (j0 >= nd) continue;
        const int j1 = (j0 + bdst) < nd ? j0 + bdst : nd;
        const int64_t e0 = sg[j0], e1 = sg[j1];
        if (e1 - e0 > 32) {
          ovf_bins |= 1u << u;
          continue;
        }
        const int64_t e = e0 + lane;
        if (e < e1) {
          int j = j0;
          while (sg[j + 1] <= e) ++j;
          dr[u] = (int)(d0 + j);
          er[u] = e;
          tr[u] = stdv[j];
        }
      }
      for (int j = 0; j < nd; ++j) {
        const bool ovf = (ovf_bins >> (j / bdst)) & 1u;
        if (sg[j + 1] == sg[j] || ovf) {
          const float fill = ovf ? __int_as_float(0x7fc00000) : 0.f;
          fill_r_row(a, d0 + j, fill, lane, dm);
        }
      }
      R.live = 1;
      int32_t hi[4], ei[4];
      float et[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const bool ok = dr[u] >= 0;
        hi[u] = ok ? (a.hsrc_idx ? a.hsrc_idx[hoff + er[u]] : (int32_t)(hoff + er[u])) : 0;
        ei[u] = (ok && P.d_e > 0) ? a.eid[er[u]] : 0;
        et[u] = ok ? a.edge_t[er[u]] : 0.f;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int r = 32 * u + lane;
        const bool ok = dr[u] >= 0;
        const float dt = tr[u] - et[u];
        R.hrow[r] = ok ? hi[u] : -1;
        R.erow[r] = ok ? ei[u] : -1;
        R.dt[r] = ok ? dt : 0.f;
        R.trow[r] = ok ? (int)tenc_table_row(dt, a.table, a.window) : -1;
        R.rdst[r] = dr[u];
      }
      warp_arrive(&B.dfull[ds]);
    }
  } else if (warp == kTW) {                          // ---------------- weight loader (half)
    uint32_t wl = 0;
    const uint32_t wbytes = split ? kP2WStage : kP2Half;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_W);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      if (lane == 0) {
        const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
        for (int i = r0; i < nch; ++i) {
          const uint32_t k = wl + (i - r0);
          const uint32_t sw = k % kP2W;
          TGL_PROF_CLK(w0c);
          PRE_FREE_SLEEP(&B.wempty[sw], k / kP2W, TGL_SLEEP_W);
#ifdef TGL_KV_PROF
          prof_add(a, 3, clock64() - w0c);             // weights: wait for a free stage
#endif
          mbar_arrive_expect_tx(&B.wfull[sw], wbytes);
          bulk_g2s(pipe + kP2AStages * kPAStage + sw * kP2WStage,
                   wkv + (size_t)plan.order[chunk_of(tt, i, nch)] * 2 * kP2WStage +
                       rank * kP2WStage,
                   wbytes, &B.wfull[sw]);
        }
        wl += nch - r0;
      }
      __syncwarp();
    }
  } else if (warp >= kPLoad0 && warp < kPLoad0 + kPLoadWarps) {   // ---------- loaders
    const int lw = warp - kPLoad0;
    const int r0 = lw * 32 + (lane >> 3), pc = lane & 7;
    const bool lo_piece = pc >= 4;
    const int j = pc & 3;
    const uint32_t ofs0 = (uint32_t)(r0 >> 3) * 1024 + (lo_piece ? 512 : 0);
    const bool active = split || !lo_piece;
    const bool tsplit = (P.input_layout & TGL_SPLIT_TABLE) && a.table != nullptr;
    const uint8_t* hbase = reinterpret_cast<const uint8_t*>(a.hsrc);
    const uint8_t* ebase = reinterpret_cast<const uint8_t*>(a.efeat);
    const uint8_t* tbase = reinterpret_cast<const uint8_t*>(a.table);
    const int64_t hld = 4 * a.ld_hsrc, eld = 4 * a.ld_e, tld = 4 * plan.dpt;
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_LOAD);
      const TDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      int hrow[8], erow[8], trw[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        hrow[k] = R.hrow[r0 + 4 * k];
        erow[k] = R.erow[r0 + 4 * k];
        trw[k] = (tsplit && R.rdst[r0 + 4 * k] >= 0) ? R.trow[r0 + 4 * k] : -1;
      }
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = plan.order[chunk_of(tt, i, nch)];
        const int col = c * kTC + 8 * j;
        const int ks = (plan.k - c * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kP2AStages;
        TGL_PROF_CLK(l0);
        PRE_FREE_SLEEP(&B.aempty[sa], g / kP2AStages, TGL_SLEEP_LOAD);
#ifdef TGL_KV_PROF
        if (lw == 0) prof_add(a, 0, clock64() - l0);  // loader: wait for a free stage
#endif
        const bool in_k = active && col < c * kTC + 16 * ks && !(TGL_DBG(a) & 2);
        const uint32_t dst = a_s + sa * kPAStage + ofs0;
        if (in_k && col < kt0) {
          const bool seg_h = col < plan.dp0;
          const uint8_t* base = seg_h ? hbase : ebase;
          const int64_t ldb = seg_h ? hld : eld;
          const uint32_t pofs = seg_h ? (uint32_t)(lo_piece ? 2 * plan.dp0 : 0) + 2 * col
                                      : (uint32_t)(lo_piece ? 2 * plan.dp1 : 0) +
                                            2 * (col - plan.dp0);
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const int row = seg_h ? hrow[k] : erow[k];
            const int rr = (r0 + 4 * k) & 7;
            const uint32_t d = dst + (uint32_t)(k >> 1) * 1024 + rr * 64 +
                               (((j ^ (rr >> 1)) & 3) << 4);
            cp_async16_zfill(d, base + (row >= 0 ? (int64_t)row * ldb + pofs : 0),
                             row >= 0 ? 16u : 0u);
          }
        } else if (in_k && tsplit && col < plan.k) {
          const uint32_t pofs = (uint32_t)(lo_piece ? 2 * plan.dpt : 0) + 2 * (col - kt0);
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            if (trw[k] < 0) continue;
            const int rr = (r0 + 4 * k) & 7;
            const uint32_t d = dst + (uint32_t)(k >> 1) * 1024 + rr * 64 +
                               (((j ^ (rr >> 1)) & 3) << 4);
            cp_async16_zfill(d, tbase + (int64_t)trw[k] * tld + pofs, 16u);
          }
        }
        cp_async_mbar_arrive_noinc(&B.afull[sa]);
      }
    }
  } else if (warp >= kPTime0 && warp < kPTime0 + kPTimeWarps) {   // -------- time warps
    const int tw = warp - kPTime0;
    const int r = tw * 32 + lane;
    const int rr = r & 7;
    const bool tsplit = (P.input_layout & TGL_SPLIT_TABLE) && a.table != nullptr;
    const uint32_t rofs = (uint32_t)(r >> 3) * 1024 + rr * 64;
    uint32_t g = 0;
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      PRE_WAIT_SLEEP(&B.dfull[ds], (tt / kSDSlots) & 1u, TGL_SLEEP_LOAD);
      const TDesc& R = bd[ds];
      if (!R.live) {
        warp_arrive(&B.dempty[ds]);
        break;
      }
      const float dtr = R.dt[r];
      const int trow = R.trow[r];
      const int mode = R.rdst[r] < 0 ? 2 : (trow >= 0 ? 1 : 0);
      __syncwarp();
      warp_arrive(&B.dempty[ds]);
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = plan.order[chunk_of(tt, i, nch)];
        const int ks = (plan.k - c * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kP2AStages;
        const bool has_time = (c + 1) * kTC > kt0 && !(TGL_DBG(a) & 64);
        if (has_time) {
          TGL_PROF_CLK(t0);
          wait_free(&B.aempty[sa], g / kP2AStages);
          TGL_PROF_CLK(t1);
#ifdef TGL_KV_PROF
          if (tw == 0) prof_add(a, 1, t1 - t0);        // time warp: wait for a free stage
#endif
          const uint32_t dst = a_s + sa * kPAStage + rofs;
#pragma unroll
          for (int jj = 0; jj < 4; ++jj) {
            const int col = c * kTC + 8 * jj;
            if (col < kt0 || col >= c * kTC + 16 * ks) continue;
            const int tc = col - kt0;
            if (tsplit && mode == 1 && col < plan.k) continue;
            float x[8];
            if (mode == 0) {
              bool bad = false;
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                const float bb = __fadd_rn(__fmul_rn(s_omega[tc + e], dtr), s_phi[tc + e]);
                bad |= !(fabsf(bb) < 1e9f);
                x[e] = tenc_cos_reduced(bb);
              }
              if (bad) {
#pragma unroll
                for (int e = 0; e < 8; ++e) x[e] = tenc_fast(dtr, s_omega[tc + e], s_phi[tc + e]);
              }
            } else if (mode == 1 && !tsplit) {
#pragma unroll
              for (int e = 0; e < 8; ++e)
                x[e] = tc + e < P.d_t ? __ldg(a.table + (int64_t)trow * P.d_t + tc + e) : 0.f;
            } else {
#pragma unroll
              for (int e = 0; e < 8; ++e) x[e] = 0.f;
            }
            if (tc + 8 > P.d_t) {
#pragma unroll
              for (int e = 0; e < 8; ++e)
                if (tc + e >= P.d_t) x[e] = 0.f;
            }
            uint32_t h[4], l[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) split2(x[2 * e], x[2 * e + 1], h[e], l[e]);
            const uint32_t po = (uint32_t)(((jj ^ (rr >> 1)) & 3) << 4);
            st_shared_v4(dst + po, h[0], h[1], h[2], h[3]);
            if (split) st_shared_v4(dst + 512 + po, l[0], l[1], l[2], l[3]);
          }
          fence_proxy_async_smem();
          __syncwarp();
#ifdef TGL_KV_PROF
          if (tw == 0) prof_add(a, 2, clock64() - t1);  // time warp: Phi + split + store
#endif
          if (lane == 0) mbar_arrive(&B.afull[sa]);
        } else {
          if (lane == 0) {
            wait_free(&B.aempty[sa], g / kP2AStages);
            mbar_arrive(&B.afull[sa]);
          }
          __syncwarp();
        }
      }
    }
  } else if (warp == kTMma && !leader) {             // ---------------- peer relay
    // the leader's MMA reads this CTA's A stage and weight half: tell it when both landed
    uint32_t g = 0, wl = 0;
    const uint32_t pfull0 = mapa_shared(smem_u32(&B.pfull[0]), 0);
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait(&B.dfull[ds], (tt / kSDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
      for (int i = 0; i < nch; ++i, ++g) {
        const uint32_t sa = g % kP2AStages;
        TGL_PROF_CLK(r0c);
        mbar_wait(&B.afull[sa], (g / kP2AStages) & 1u);
        TGL_PROF_CLK(r1c);
        if (i >= r0) {
          const uint32_t kw = wl + (i - r0);
          mbar_wait(&B.wfull[kw % kP2W], (kw / kP2W) & 1u);
        }
#ifdef TGL_KV_PROF
        prof_add(a, 4, r1c - r0c);                     // relay: A wait
        prof_add(a, 5, clock64() - r1c);               // relay: W wait
#endif
        if (lane == 0) mbar_arrive_remote(pfull0 + sa * 8);
        __syncwarp();
      }
      wl += nch - r0;
    }
  } else if (warp == kTMma) {                        // ---------------- MMA issuer (leader)
    uint32_t g = 0, wl = 0;
    constexpr uint32_t idesc = idesc_bf16(2 * kBM, kP2N);
    for (;; ++tt) {
      const uint32_t ds = tt % kSDSlots;
      mbar_wait(&B.dfull[ds], (tt / kSDSlots) & 1u);
      const int live = bd[ds].live;
      warp_arrive(&B.dempty[ds]);
      if (!live) break;
      const uint32_t acc = tmem + (tt & 1u) * kCols;
      TGL_PROF_CLK(mt0);
      if (tt >= 2) mbar_wait_cluster(&B.tempty[tt & 1u], ((tt >> 1) - 1) & 1u);
#ifdef TGL_KV_PROF
      prof_add(a, 6, clock64() - mt0);               // MMA: wait for an accumulator
#endif
      tc_fence_after();
      const int r0 = (tt > 0 && nch >= 4) ? 2 : 0;
      for (int i = 0; i < nch; ++i, ++g) {
        const int c = plan.order[chunk_of(tt, i, nch)];
        const int nk = (plan.k - c * kTC) > 16 ? 2 : 1;
        const uint32_t sa = g % kP2AStages;
        TGL_PROF_CLK(ma0);
        mbar_wait(&B.afull[sa], (g / kP2AStages) & 1u);
        TGL_PROF_CLK(ma1);
        mbar_wait_cluster(&B.pfull[sa], (g / kP2AStages) & 1u);
        TGL_PROF_CLK(ma2);
        uint32_t kw;
        if (i < r0) {
          kw = wl - 1 - i;
        } else {
          kw = wl + (i - r0);
          mbar_wait(&B.wfull[kw % kP2W], (kw / kP2W) & 1u);
        }
#ifdef TGL_KV_PROF
        prof_add(a, 7, ma1 - ma0);                     // MMA: local A wait
        prof_add(a, 8, ma2 - ma1);                     // MMA: peer relay wait
        prof_add(a, 9, clock64() - ma2);               // MMA: W wait
#endif
        tc_fence_after();
        if (elect_one()) {
          const uint64_t a0 = desc_sw64(a_s + sa * kPAStage, 1024);
          const uint64_t w0 = desc_sw64(w_s + (kw % kP2W) * kP2WStage, 512);
#pragma unroll
          for (int ks = 0; ks < 2; ++ks) {
            if (ks < nk && !(TGL_DBG(a) & 4)) {
              const uint64_t ah = a0 + 2 * ks, bh = w0 + 2 * ks;
              mma_bf16_pair(acc, ah, bh, idesc, (i | ks) != 0);
              if (split) {
                mma_bf16_pair(acc, ah + (512 >> 4), bh, idesc, 1u);
                mma_bf16_pair(acc, ah, bh + (kP2Half >> 4), idesc, 1u);
              }
            }
          }
          const bool keep = (nch >= 4) && (i >= nch - 2);
          mma_commit_pair(&B.aempty[sa]);
          if (!keep) mma_commit_pair(&B.wempty[kw % kP2W]);
        }
        __syncwarp();
      }
      wl += nch - r0;
      if (elect_one()) mma_commit_pair(&B.tfull[tt & 1u]);
      __syncwarp();
    }
  } else if (warp < kBEpi) {                         // ---------------- epilogue warps 0-7
    bin_epilogue<kSDSlots, TDesc, kSPW, false>(a, B.dfull, B.dempty, B.tfull, B.tempty, bd, tmem,
                                               s_pvf, s_bias,
                                               mapa_shared(smem_u32(&B.tempty[0]), 0));
  }
  tc_fence_before();
  __syncthreads();
#ifdef TGL_KV_PROF
  if (threadIdx.x == 0) prof_add(a, 13, clock64() - k0c);   // whole kernel
#endif
  cluster_sync_all();                                // the peer's smem / barriers stay valid
  if (warp == kTMma)
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"(2 * kCols)
                 : "memory");
}

}  // namespace tca

// ------------------------------------------------------------------ host side
namespace tca {

struct PackedLayout {
  size_t oq, okv, oo, okv64, okvc, okvp, okvp2, oqp, oop, obq;
  size_t okvn, onk, onv, ono, oor;   // node projections (TGL_NODE_PROJ)
  size_t total;
};

static PackedLayout packed_layout(const tgl_attn_params* P) {
  PackedLayout L;
  WsLayout W;
  const Seg3 sq = make_seg3(P->d_hdst, 0, P->d_t);
  const Seg3 skv = make_seg3(P->d_hsrc, P->d_e, P->d_t);
  const Seg3 so = make_seg3(P->d_model, P->d_hdst, 0);
  L.oq = W.take((size_t)sq.nchunks * 2 * kNPq * 128);
  L.okv = W.take((size_t)skv.nchunks * 2 * kNPkv * 128);
  L.oo = W.take((size_t)so.nchunks * 2 * kNPq * 128);
  L.okv64 = W.take((size_t)make_plan(P->d_hsrc, P->d_e, P->d_t).n * kTWStage);
  L.okvc = W.take((size_t)make_plan_contig(P->d_hsrc, P->d_e, P->d_t).n * kTWStage);
  L.okvp = W.take((size_t)make_pre_plan(P->d_hsrc, P->d_e, P->d_t).n * kTWStage);
  L.okvp2 = W.take((size_t)make_pre_plan(P->d_hsrc, P->d_e, P->d_t).n * 2 * kP2WStage);
  L.oqp = W.take((size_t)make_dp_plan(P->d_hdst, 0).n * kDPWStage);
  L.oop = W.take((size_t)make_dp_plan(P->d_model, P->d_hdst).n * kDPWStage);
  L.obq = W.take(sizeof(float) * kDPN);
  // node projections: the per-edge K|V plan over [e | Phi] only, the per-node Wk_h / Wv_h /
  // Wo_h projections (tgl_node_proj) and the FFN over r only
  L.okvn = W.take((size_t)make_pre_plan(0, P->d_e, P->d_t).n * kTWStage);
  L.onk = W.take((size_t)make_dp_plan(P->d_hsrc, 0).n * kDPWStage);
  L.onv = W.take((size_t)make_dp_plan(P->d_hsrc, 0).n * kDPWStage);
  L.ono = W.take((size_t)make_dp_plan(P->d_hdst, 0).n * kDPWStage);
  L.oor = W.take((size_t)make_dp_plan(P->d_model, 0).n * kDPWStage);
  L.total = W.off;
  return L;
}

static tgl_status launch_pack(const tgl_attn_params* P, uint8_t* base, cudaStream_t s) {
  const PackedLayout L = packed_layout(P);
  const Seg3 sq = make_seg3(P->d_hdst, 0, P->d_t);
  const Seg3 skv = make_seg3(P->d_hsrc, P->d_e, P->d_t);
  const Seg3 so = make_seg3(P->d_model, P->d_hdst, 0);
  PackJob jq{P->Wq, nullptr, P->d_model, P->d_model, kNPq, P->d_hdst + P->d_t, sq, base + L.oq};
  PackJob jkv{P->Wk, P->Wv, P->d_model, 2 * P->d_model, kNPkv, P->d_hsrc + P->d_e + P->d_t, skv,
              base + L.okv};
  PackJob jo{P->Wo, nullptr, P->d_out, P->d_out, kNPq, P->d_model + P->d_hdst, so, base + L.oo};
  pack_weights_kernel<<<dim3(64, 3), 256, 0, s>>>(jq, jkv, jo);
  TGL_TRY(launch_check("pack_weights"));
  pack_kv64_kernel<<<64, 256, 0, s>>>(P->Wk, P->Wv, P->d_model, P->d_hsrc + P->d_e + P->d_t,
                                      make_plan(P->d_hsrc, P->d_e, P->d_t), base + L.okv64);
  TGL_TRY(launch_check("pack_kv64"));
  pack_kv64_kernel<<<64, 256, 0, s>>>(P->Wk, P->Wv, P->d_model, P->d_hsrc + P->d_e + P->d_t,
                                      make_plan_contig(P->d_hsrc, P->d_e, P->d_t),
                                      base + L.okvc);
  TGL_TRY(launch_check("pack_kv64 contiguous"));
  pack_kv_pre_kernel<<<64, 256, 0, s>>>(P->Wk, P->Wv, P->d_model, P->d_hsrc + P->d_e + P->d_t,
                                        make_pre_plan(P->d_hsrc, P->d_e, P->d_t),
                                        base + L.okvp, 0);
  TGL_TRY(launch_check("pack_kv_pre"));
  pack_kv_pre_kernel<<<64, 256, 0, s>>>(P->Wk, P->Wv, P->d_model, P->d_hsrc + P->d_e + P->d_t,
                                        make_pre_plan(0, P->d_e, P->d_t), base + L.okvn,
                                        P->d_hsrc);
  TGL_TRY(launch_check("pack_kv_pre node-proj"));
  const int kin = P->d_hsrc + P->d_e + P->d_t;
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wk, P->d_model, kin, 0, 0,
                                           make_dp_plan(P->d_hsrc, 0), base + L.onk, nullptr,
                                           nullptr, 0, 0, nullptr);
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wv, P->d_model, kin, 0, 0,
                                           make_dp_plan(P->d_hsrc, 0), base + L.onv, nullptr,
                                           nullptr, 0, 0, nullptr);
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wo, P->d_out, P->d_model + P->d_hdst, P->d_model,
                                           0, make_dp_plan(P->d_hdst, 0), base + L.ono, nullptr,
                                           nullptr, 0, 0, nullptr);
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wo, P->d_out, P->d_model + P->d_hdst, 0, 0,
                                           make_dp_plan(P->d_model, 0), base + L.oor, nullptr,
                                           nullptr, 0, 0, nullptr);
  TGL_TRY(launch_check("pack node-proj"));
  pack_kv_pre2_kernel<<<64, 256, 0, s>>>(P->Wk, P->Wv, P->d_model, P->d_hsrc + P->d_e + P->d_t,
                                         make_pre_plan(P->d_hsrc, P->d_e, P->d_t),
                                         base + L.okvp2);
  TGL_TRY(launch_check("pack_kv_pre2"));
  // dense_pre: Q over h_dst only (Phi(0) folded into the bias), FFN over [r | h_dst]
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wq, P->d_model, P->d_hdst + P->d_t, 0, 0,
                                           make_dp_plan(P->d_hdst, 0), base + L.oqp, P->bq,
                                           P->phi, P->d_t, P->d_hdst,
                                           reinterpret_cast<float*>(base + L.obq));
  TGL_TRY(launch_check("pack_dense_pre q"));
  pack_dense_pre_kernel<<<64, 256, 0, s>>>(P->Wo, P->d_out, P->d_model + P->d_hdst, 0,
                                           P->d_model, make_dp_plan(P->d_model, P->d_hdst),
                                           base + L.oop, nullptr, nullptr, 0, 0, nullptr);
  return launch_check("pack_dense_pre ffn");
}

}  // namespace tca

namespace tca {

// The async gathers move 16-byte pieces of feature rows: a row table qualifies when
// its base is 16-byte aligned and its row pitch a multiple of 16 bytes.
static bool rows_16b(const float* base, int width, int64_t ld) {
  if (width <= 0) return true;                       // segment absent
  return base != nullptr && !(reinterpret_cast<uintptr_t>(base) & 15) && !((ld * 4) & 15);
}

}  // namespace tca

// dynamic shared memory opt-in of every tensor-core kernel (per device, once)
static tgl_status set_smem_attrs(int smem_q, int smem_kv, int smem_kvb) {
  using namespace tca;
  static PerDeviceOnce once;
  return cuda_check(once.run([=] {
    cudaError_t e = cudaFuncSetAttribute(dense_kernel<false>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem_q);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(dense_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               smem_q);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_kv);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_bin_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               smem_kvb);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_async_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kTSmem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_split_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kSSmem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_pre_kernel<kPAStages, kPW, kPreReuse>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize,
                               pre_smem_bytes<kPAStages, kPW>());
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_pre_kernel<7, 3, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               pre_smem_bytes<7, 3>());
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kv_pre2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kP2Smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(dense_pre_kernel<false>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, kDPSmem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(dense_pre_kernel<true>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, kDPSmem);
    return e;
  }), "smem attributes");
}

// host entry used by tgl_tblock_attn (attn.cu) for TGL_FP32 / TGL_BF16
size_t tc_attn_ws_bytes(const tgl_attn_params* P, int64_t n_dst_max, size_t* o_q, size_t* o_r,
                        size_t* o_pack) {
  using namespace tca;
  WsLayout L;
  const int64_t nrows = n_dst_max > 0 ? n_dst_max : 1;
  *o_q = L.take(sizeof(float) * kQLd * nrows);
  *o_r = L.take(sizeof(float) * kQLd * nrows);
  *o_pack = L.take(P->packed ? 0 : packed_layout(P).total);
  return L.off;
}

bool tc_attn_supported(const tgl_attn_params* P) {
  return P->d_model == 100 && P->d_out == 100 && P->n_heads >= 1 && P->n_heads <= 2 &&
         P->d_t <= 256 && P->d_hdst >= 0 && P->d_hsrc >= 0 && P->d_e >= 0;
}

tgl_status tc_attn_launch(const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev,
                          const int64_t* seg_ptr, const float* dst_t, const float* hdst,
                          const int32_t* hdst_idx, int64_t ld_hdst, const float* hsrc,
                          const int32_t* hsrc_idx, const int64_t* hsrc_off_dev, int64_t ld_hsrc,
                          const float* efeat, const int32_t* eid, int64_t ld_e,
                          const float* edge_t, const float* table, int64_t window,
                          int32_t max_seg, float* out, void* ws, cudaStream_t s) {
  using namespace tca;
  size_t o_q, o_r, o_pack;
  tc_attn_ws_bytes(P, n_dst_max, &o_q, &o_r, &o_pack);
  char* w = static_cast<char*>(ws);
  uint8_t* pk = P->packed ? const_cast<uint8_t*>(static_cast<const uint8_t*>(P->packed))
                          : reinterpret_cast<uint8_t*>(w + o_pack);
  if (!P->packed) TGL_TRY(launch_pack(P, pk, s));   // otherwise packed once by tgl_attn_pack
  const PackedLayout PL = packed_layout(P);
  Args a;
  a.P = *P;
  a.n_dst_max = n_dst_max;
  a.n_dst_dev = n_dst_dev;
  a.seg_ptr = seg_ptr;
  a.dst_t = dst_t;
  a.hdst = hdst;
  a.hdst_idx = hdst_idx;
  a.ld_hdst = ld_hdst;
  a.hsrc = hsrc;
  a.hsrc_idx = hsrc_idx;
  a.hsrc_off_dev = hsrc_off_dev;
  a.ld_hsrc = ld_hsrc;
  a.efeat = efeat;
  a.eid = eid;
  a.ld_e = ld_e;
  a.edge_t = edge_t;
  a.table = window > 0 ? table : nullptr;
  a.window = window;
  a.out = out;
  a.qbuf = reinterpret_cast<float*>(w + o_q);
  a.rbuf = reinterpret_cast<float*>(w + o_r);
  a.rsplit = nullptr;
  a.zkv = nullptr;
  a.zo = nullptr;
  a.z_ld = 0;
  a.q_idx = nullptr;
  a.q_ld = kQLd;
  a.wq = pk + PL.oq;
  a.wkv = pk + PL.okv;
  a.wo = pk + PL.oo;
  a.sq = make_seg3(P->d_hdst, 0, P->d_t);
  a.skv = make_seg3(P->d_hsrc, P->d_e, P->d_t);
  a.so = make_seg3(P->d_model, P->d_hdst, 0);
  a.np_q = kNPq;
  a.np_kv = kNPkv;
  a.np_o = kNPq;
  const int ms = max_seg > 0 ? max_seg : 1;
  int dpb = kBM / ms;
  a.dpb = dpb < 1 ? 1 : (dpb > kMaxDpb ? kMaxDpb : dpb);
  a.split = P->precision == TGL_FP32 ? 1 : 0;
#ifdef TGL_PROBE
  a.dbg = getenv("TGL_DEBUG_MASK") ? atoi(getenv("TGL_DEBUG_MASK")) : 0;   // probe builds only
#else
  a.dbg = 0;
#endif

  const int smem_q = Pipe<kNPq>::kBytes + 1024;
  const int smem_kv = Pipe<kNPkv>::kBytes + 1024 + kKvEpiBytes;
  const int smem_kvb = Pipe<kNPkv>::kBytes + 1024 + kBEpi * 32 * 33 * 4;
  TGL_TRY(set_smem_attrs(smem_q, smem_kv, smem_kvb));
  const int64_t tiles = ceil_div(n_dst_max, kBM);
  const unsigned gq = (unsigned)(tiles < kNumSMs ? tiles : kNumSMs);
  if (P->input_layout & TGL_NODE_PROJ) {
    // node projections (tgl_node_proj, P->node_proj = Z): q_i, the h_src part of k_e / v_e
    // and the h_i part of the FFN input are rows of Z (eqs 4, 5, 7 are linear in h); the
    // per-edge MMAs cover [e | Phi] only, the FFN's cover r only.  No Q launch.
    const PrePlan plan = make_pre_plan(0, P->d_e, P->d_t);
    const DPPlan rplan = make_dp_plan(P->d_model, 0);
    const bool e_ok = P->d_e == 0 || ((P->input_layout & TGL_SPLIT_E) && ld_e >= plan.dp1 &&
                                      rows_16b(efeat, 1, ld_e));
    const bool t_ok = !(P->input_layout & TGL_SPLIT_TABLE) || table == nullptr ||
                      rows_16b(table, 1, plan.dpt);
    const int sel = P->kv_kernel;
    if (P->node_proj == nullptr || (reinterpret_cast<uintptr_t>(P->node_proj) & 15) || !e_ok ||
        !t_ok || !(sel == TGL_KV_AUTO || sel == TGL_KV_PRE) ||
        !(max_seg > 0 && max_seg <= 32 && P->n_heads == 2) || P->d_hsrc != P->d_hdst ||
        plan.n > kPMaxChunks || rplan.n > kPMaxChunks) {
      set_error("TGL_NODE_PROJ: needs P->node_proj (tgl_node_proj output, 16-byte aligned), "
                "d_hsrc == d_hdst, split16 e / table (input_layout), kv_kernel AUTO/PRE, "
                "max_seg <= 32, 2 heads");
      return TGL_EUNSUPPORTED;
    }
    a.zkv = P->node_proj;
    a.zo = P->node_proj + TGL_NODE_PROJ_O;
    a.z_ld = TGL_NODE_PROJ_LD;
    a.qbuf = const_cast<float*>(P->node_proj) + TGL_NODE_PROJ_Q;
    a.q_ld = TGL_NODE_PROJ_LD;
    a.q_idx = hdst_idx;
    a.rsplit = reinterpret_cast<uint8_t*>(a.rbuf);   // r rows split16 for the FFN
    tgl_kv_probe* probe = P->probe;
    if (probe) {
      probe->kernel = TGL_KV_PRE;
      if (probe->ev_start)
        TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_start), s),
                           "probe event"));
    }
    const int bdst = 32 / max_seg;
    const int64_t ttiles = ceil_div(n_dst_max, 4 * bdst);
    const unsigned gt = (unsigned)(ttiles < kNumSMs ? (ttiles > 0 ? ttiles : 1) : kNumSMs);
    if (max_seg > 16)     // few destinations per tile: the deeper A ring
      launch_pdl(kv_pre_kernel<7, 3, 2>, dim3(gt), dim3(kPThreads), pre_smem_bytes<7, 3>(), s, a,
                 plan, pk + PL.okvn, bdst);
    else
      launch_pdl(kv_pre_kernel<kPAStages, kPW, kPreReuse>, dim3(gt), dim3(kPThreads),
                 pre_smem_bytes<kPAStages, kPW>(), s, a, plan, pk + PL.okvn, bdst);
    TGL_TRY(launch_check("tc kv pre kernel (node proj)"));
    if (probe && probe->ev_stop)
      TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_stop), s),
                         "probe event"));
    DPJobs jo{};
    jo.j[0] = DPJob{pk + PL.oor, nullptr, nullptr, a.out, P->d_model};
    launch_pdl(dense_pre_kernel<true>, dim3(gq), dim3(kDPThreads), kDPSmem, s, a, rplan, jo);
    return launch_check("tc ffn kernel (node proj)");
  }
  // split16 h_dst (and so split16 r, written by the K|V epilogue): converter-free Q / FFN
  const bool dpre = (P->input_layout & TGL_SPLIT_HDST) != 0;
  const DPPlan qplan = make_dp_plan(P->d_hdst, 0), oplan = make_dp_plan(P->d_model, P->d_hdst);
  if (dpre) {
    if (!(P->input_layout & (TGL_SPLIT_HSRC | TGL_SPLIT_E)) ||
        !rows_16b(hdst, 1, ld_hdst) || ld_hdst < qplan.dp0 || P->d_model != 100 ||
        qplan.n > kPMaxChunks || oplan.n > kPMaxChunks) {
      set_error("TGL_SPLIT_HDST needs the pre-split K|V path (TGL_SPLIT_HSRC / _E), a 16-byte "
                "aligned split16 h_dst table with ld >= round8(d_hdst)");
      return TGL_EUNSUPPORTED;
    }
    a.rsplit = reinterpret_cast<uint8_t*>(a.rbuf);   // r scratch rows hold the split16 rows
    DPJobs jq{};
    jq.j[0] = DPJob{pk + PL.oqp, reinterpret_cast<const float*>(pk + PL.obq), P->bk, a.qbuf,
                    kQLd};
    launch_pdl(dense_pre_kernel<false>, dim3(gq), dim3(kDPThreads), kDPSmem, s, a, qplan, jq);
  } else {
    launch_pdl(dense_kernel<false>, dim3(gq), dim3(kWsThreads), smem_q, s, a);
  }
  TGL_TRY(launch_check("tc q kernel"));
  const int sel = P->kv_kernel;
  if (sel < TGL_KV_AUTO || sel > TGL_KV_PRE2 || sel == TGL_KV_SIMT) {
    set_error("kv_kernel %d: not a TGL_KV_* id", sel);
    return TGL_EINVAL;
  }
  const bool pre_in = (P->input_layout & (TGL_SPLIT_HSRC | TGL_SPLIT_E | TGL_SPLIT_TABLE)) != 0;
  if (pre_in || sel == TGL_KV_PRE || sel == TGL_KV_PRE2) {
    // pre-split h_src / e tables (tgl_split_rows): every gathered table present must be
    // split, rows 16-byte aligned; max_seg <= 32 and 2 heads (the binned epilogue)
    const PrePlan plan = make_pre_plan(P->d_hsrc, P->d_e, P->d_t);
    const bool hs_ok = P->d_hsrc == 0 || ((P->input_layout & TGL_SPLIT_HSRC) &&
                                          ld_hsrc >= plan.dp0 && rows_16b(hsrc, 1, ld_hsrc));
    const bool e_ok = P->d_e == 0 || ((P->input_layout & TGL_SPLIT_E) && ld_e >= plan.dp1 &&
                                      rows_16b(efeat, 1, ld_e));
    const bool t_ok = !(P->input_layout & TGL_SPLIT_TABLE) || table == nullptr ||
                      rows_16b(table, 1, plan.dpt);
    if (!(sel == TGL_KV_AUTO || sel == TGL_KV_PRE || sel == TGL_KV_PRE2) || !hs_ok || !e_ok ||
        !t_ok ||
        !(max_seg > 0 && max_seg <= 32 && P->n_heads == 2) || plan.n > kPMaxChunks) {
      set_error("pre-split inputs: kv_kernel must be AUTO/PRE, every gathered table split "
                "(input_layout), 16-byte rows, ld >= padded width, max_seg <= 32, 2 heads");
      return TGL_EUNSUPPORTED;
    }
    const bool pair = sel == TGL_KV_PRE2 || (sel == TGL_KV_AUTO && kPreAutoPair);
    tgl_kv_probe* probe = P->probe;
    if (probe) {
      probe->kernel = pair ? TGL_KV_PRE2 : TGL_KV_PRE;
      if (probe->ev_start)
        TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_start), s),
                           "probe event"));
    }
    const int bdst = 32 / max_seg;
    const int64_t ttiles = ceil_div(n_dst_max, 4 * bdst);
    const unsigned gt = (unsigned)(ttiles < kNumSMs ? (ttiles > 0 ? ttiles : 1) : kNumSMs);
    if (pair) {                                    // CTA pairs: even grid of <= 148 CTAs
      const int64_t npt = ceil_div(ttiles > 0 ? ttiles : 1, 2);
      const unsigned gp = 2u * (unsigned)(npt < kNumSMs / 2 ? npt : kNumSMs / 2);
      launch_pdl(kv_pre2_kernel, dim3(gp), dim3(kPThreads), kP2Smem, s, a, plan, pk + PL.okvp2,
                 bdst);
    } else {
      if (max_seg > 16)   // few destinations per tile: the deeper A ring
        launch_pdl(kv_pre_kernel<7, 3, 2>, dim3(gt), dim3(kPThreads), pre_smem_bytes<7, 3>(), s,
                   a, plan, pk + PL.okvp, bdst);
      else
        launch_pdl(kv_pre_kernel<kPAStages, kPW, kPreReuse>, dim3(gt), dim3(kPThreads),
                   pre_smem_bytes<kPAStages, kPW>(), s, a, plan, pk + PL.okvp, bdst);
    }
    TGL_TRY(launch_check("tc kv pre kernel"));
    if (probe && probe->ev_stop)
      TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_stop), s),
                         "probe event"));
    if (dpre) {
      DPJobs jo{};
      jo.j[0] = DPJob{pk + PL.oop, nullptr, nullptr, a.out, P->d_model};
      launch_pdl(dense_pre_kernel<true>, dim3(gq), dim3(kDPThreads), kDPSmem, s, a, oplan, jo);
    }
    else
      launch_pdl(dense_kernel<true>, dim3(gq), dim3(kWsThreads), smem_q, s, a);
    return launch_check("tc ffn kernel");
  }
  const bool binned = max_seg > 0 && max_seg <= 32 && P->n_heads == 2;
  const bool async = binned && rows_16b(hsrc, P->d_hsrc, ld_hsrc) && rows_16b(efeat, P->d_e, ld_e) &&
                     rows_16b(table, table ? P->d_t : 0, P->d_t);
  const bool contig = contig_ok(P->d_hsrc, P->d_e);
  int kind;
  if (sel == TGL_KV_AUTO) {
    kind = async ? TGL_KV_SPLIT : (binned ? TGL_KV_BIN : TGL_KV_GENERAL);
  } else {
    kind = sel;
    const bool ok = (sel == TGL_KV_GENERAL) || (sel == TGL_KV_BIN && binned) ||
                    ((sel == TGL_KV_SPLIT || sel == TGL_KV_SPLIT_PAD || sel == TGL_KV_ASYNC) &&
                     async);
    if (!ok) {
      set_error("kv_kernel %d cannot take this call (16-byte row pitches, max_seg <= 32, "
                "2 heads)", sel);
      return TGL_EUNSUPPORTED;
    }
  }
  if (kind == TGL_KV_SPLIT && !contig) kind = TGL_KV_SPLIT_PAD;   // plan follows the widths
  tgl_kv_probe* probe = P->probe;
  if (probe) {
    probe->kernel = kind;
    if (probe->ev_start)
      TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_start), s),
                         "probe event"));
  }
  if (kind == TGL_KV_SPLIT || kind == TGL_KV_SPLIT_PAD) {
    const int bdst = 32 / max_seg;                 // destinations per 32-row bin
    const int64_t ttiles = ceil_div(n_dst_max, 4 * bdst);
    const unsigned gt = (unsigned)(ttiles < kNumSMs ? (ttiles > 0 ? ttiles : 1) : kNumSMs);
    const bool cplan = kind == TGL_KV_SPLIT;
    const KvPlan plan = cplan ? make_plan_contig(P->d_hsrc, P->d_e, P->d_t)
                              : make_plan(P->d_hsrc, P->d_e, P->d_t);
    if (plan.n > kSMaxChunks) {
      set_error("K|V attention: %d K chunks > %d", plan.n, kSMaxChunks);
      return TGL_EUNSUPPORTED;
    }
    launch_pdl(kv_split_kernel, dim3(gt), dim3(kSThreads), kSSmem, s, a, plan,
               pk + (cplan ? PL.okvc : PL.okv64), bdst);
  } else if (kind == TGL_KV_ASYNC) {
    const int bdst = 32 / max_seg;                 // destinations per 32-row bin
    const int64_t ttiles = ceil_div(n_dst_max, 4 * bdst);
    const unsigned gt = (unsigned)(ttiles < kNumSMs ? (ttiles > 0 ? ttiles : 1) : kNumSMs);
    launch_pdl(kv_async_kernel, dim3(gt), dim3(kTThreads), kTSmem, s, a,
               make_plan(P->d_hsrc, P->d_e, P->d_t), pk + PL.okv64, bdst);
  } else if (kind == TGL_KV_BIN) {
    // binned path: whole segments per epilogue warp (no block barriers)
    const unsigned gkv = (unsigned)(n_dst_max < kNumSMs ? (n_dst_max > 0 ? n_dst_max : 1) : kNumSMs);
    launch_pdl(kv_bin_kernel, dim3(gkv), dim3(kBThreads), smem_kvb, s, a);
  } else {
    const int64_t groups = ceil_div(n_dst_max, a.dpb);
    const unsigned gkv = (unsigned)(groups < kNumSMs ? groups : kNumSMs);
    launch_pdl(kv_kernel, dim3(gkv), dim3(kWsThreads), smem_kv, s, a);
  }
  TGL_TRY(launch_check("tc kv kernel"));
  if (probe && probe->ev_stop)
    TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_stop), s),
                       "probe event"));
  launch_pdl(dense_kernel<true>, dim3(gq), dim3(kWsThreads), smem_q, s, a);
  return launch_check("tc ffn kernel");
}

}  // namespace tgl

using namespace tgl;

extern "C" size_t tgl_attn_packed_bytes(const tgl_attn_params* P) {
  if (P == nullptr || !tc_attn_supported(P)) return 0;
  return tca::packed_layout(P).total;
}

extern "C" tgl_status tgl_attn_pack(const tgl_attn_params* P, void* packed, size_t bytes,
                                    void* stream) {
  TGL_REQUIRE(P != nullptr && packed != nullptr, "null pointer");
  if (!tc_attn_supported(P)) {
    set_error("tensor-core path needs d_model == d_out == 100, n_heads <= 2, d_t <= 256");
    return TGL_EUNSUPPORTED;
  }
  TGL_REQUIRE(P->Wq && P->Wk && P->Wv && P->Wo, "null weight");
  if (bytes < tca::packed_layout(P).total) {
    set_error("packed buffer too small: %zu < %zu", bytes, tca::packed_layout(P).total);
    return TGL_EWORKSPACE;
  }
  TGL_REQUIRE((reinterpret_cast<uintptr_t>(packed) & 255) == 0, "packed must be 256-aligned");
  return tca::launch_pack(P, static_cast<uint8_t*>(packed), as_stream(stream));
}

extern "C" tgl_status tgl_node_proj(const tgl_attn_params* P, int64_t n_nodes, const void* hnode,
                                    int64_t ld, float* Z, void* stream) {
  using namespace tca;
  TGL_REQUIRE(P != nullptr && Z != nullptr, "null pointer");
  TGL_REQUIRE(n_nodes >= 0, "n_nodes < 0");
  if (!tc_attn_supported(P) || P->n_heads != 2 || P->d_hsrc != P->d_hdst ||
      !(P->precision == TGL_FP32 || P->precision == TGL_BF16)) {
    set_error("tgl_node_proj: tensor-core precisions, d_model == 100, 2 heads, d_hsrc == d_hdst");
    return TGL_EUNSUPPORTED;
  }
  TGL_REQUIRE(P->packed != nullptr, "tgl_node_proj needs P->packed (tgl_attn_pack)");
  const DPPlan plan = make_dp_plan(P->d_hsrc, 0);
  TGL_REQUIRE(plan.n <= kPMaxChunks, "d_hsrc too large");
  TGL_REQUIRE(!(reinterpret_cast<uintptr_t>(Z) & 15), "Z must be 16-byte aligned");
  if (n_nodes == 0) return TGL_OK;
  TGL_REQUIRE(hnode != nullptr && !(reinterpret_cast<uintptr_t>(hnode) & 15) && ld % 4 == 0 &&
                  ld >= plan.dp0,
              "hnode: split16 rows, 16-byte aligned, ld >= round8(d_hsrc)");
  cudaStream_t s = as_stream(stream);
  TGL_TRY(set_smem_attrs(Pipe<kNPq>::kBytes + 1024, Pipe<kNPkv>::kBytes + 1024 + kKvEpiBytes,
                         Pipe<kNPkv>::kBytes + 1024 + kBEpi * 32 * 33 * 4));
  const uint8_t* pk = static_cast<const uint8_t*>(P->packed);
  const PackedLayout PL = packed_layout(P);
  Args a{};
  a.P = *P;
  a.n_dst_max = n_nodes;
  a.n_dst_dev = nullptr;
  a.hdst = static_cast<const float*>(hnode);
  a.hdst_idx = nullptr;
  a.ld_hdst = ld;
  a.q_ld = kQLd;
  a.split = P->precision == TGL_FP32 ? 1 : 0;
  DPJobs j{};
  j.j[0] = DPJob{pk + PL.onk, nullptr, nullptr, Z + TGL_NODE_PROJ_K, TGL_NODE_PROJ_LD};
  j.j[1] = DPJob{pk + PL.onv, nullptr, nullptr, Z + TGL_NODE_PROJ_V, TGL_NODE_PROJ_LD};
  j.j[2] = DPJob{pk + PL.oqp, reinterpret_cast<const float*>(pk + PL.obq), P->bk,
                 Z + TGL_NODE_PROJ_Q, TGL_NODE_PROJ_LD};
  j.j[3] = DPJob{pk + PL.ono, nullptr, nullptr, Z + TGL_NODE_PROJ_O, TGL_NODE_PROJ_LD};
  j.n = 4;                                    // the four share every gathered A chunk
  const int64_t tiles = ceil_div(n_nodes, kBM);
  const unsigned gx = (unsigned)(tiles < kNumSMs ? tiles : kNumSMs);
  launch_pdl(dense_pre_kernel<false>, dim3(gx, 1), dim3(kDPThreads), kDPSmem, s, a, plan, j);
  return launch_check("tgl_node_proj");
}

#ifdef TGL_PROBE
// probe builds only (tools/): read back the instrumentation buffers
extern "C" int tgl_debug_timeline(unsigned long long* host, size_t n) {
  const size_t cap = sizeof(tca::g_timeline) / sizeof(unsigned long long);
  return (int)cudaMemcpyFromSymbol(host, tca::g_timeline,
                                   (n < cap ? n : cap) * sizeof(unsigned long long));
}

extern "C" int tgl_debug_prof(unsigned long long* host, int reset) {
  if (reset) {
    static unsigned long long z[tgl::kNumSMs * 16];
    return (int)cudaMemcpyToSymbol(tgl::tca::g_prof, z, sizeof(z));
  }
  return (int)cudaMemcpyFromSymbol(host, tgl::tca::g_prof, sizeof(unsigned long long) * tgl::kNumSMs * 16);
}

extern "C" int tgl_debug_trace(unsigned long long* host, int reset) {
  if (reset) {
    static unsigned long long z[8192];
    return (int)cudaMemcpyToSymbol(tgl::tca::g_trace, z, sizeof(z));
  }
  return (int)cudaMemcpyFromSymbol(host, tgl::tca::g_trace, sizeof(unsigned long long) * 8192);
}
#endif  // TGL_PROBE
