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
  const uint8_t* wq;   // packed
  const uint8_t* wkv;
  const uint8_t* wo;
  Seg3 sq, skv, so;
  int np_q, np_kv, np_o;
  int dpb;
  int split;           // 1 = 3-pass fp32 mode
};

__device__ __forceinline__ uint8_t* align1024(uint8_t* p) {
  return reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(p) + 1023) & ~uintptr_t(1023));
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
constexpr int kProdWarps = 8;
constexpr int kProdThreads = kProdWarps * 32;
constexpr int kWsThreads = (kProdWarp0 + kProdWarps) * 32;   // 480
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
__device__ __forceinline__ void load_chunk(int c, const Seg3& sg, const RowDesc& rd, int r, int jb,
                                           const float* s_omega, const float* s_phi,
                                           const float* table, float* x) {
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
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
          if (j0 + e < sg.d2) y[e] = tenc_direct(dt, s_omega[j0 + e], s_phi[j0 + e]);
      }
    }
  }
}

__device__ __forceinline__ void store_chunk(const float* x, uint8_t* a_hi, uint8_t* a_lo, int r,
                                            int jb, bool split) {
  const uint32_t hb = smem_u32(a_hi), lb = smem_u32(a_lo);
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
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
template <int NP, int N>
__device__ __forceinline__ void mma_tile(const Seg3& sg, bool split, uint8_t* pipe, Bars& B,
                                         uint32_t tmem_acc, uint32_t& ait, uint32_t& wit,
                                         uint32_t tt) {
  using PP = Pipe<NP>;
  constexpr uint32_t idesc = idesc_bf16(kBM, N);
  wait_free(&B.tempty[tt & 1u], tt >> 1);    // epilogue drained this accumulator
  tc_fence_after();
  for (int c = 0; c < sg.nchunks; ++c, ++ait, ++wit) {
    const uint32_t sa = ait % kAStages, sw = wit % kWStages;
    mbar_wait(&B.afull[sa], (ait / kAStages) & 1u);
    mbar_wait(&B.wfull[sw], (wit / kWStages) & 1u);
    tc_fence_after();
    const uint32_t ahb = smem_u32(PP::a(pipe, sa)), alb = ahb + kAPart;
    const uint32_t whb = smem_u32(PP::w(pipe, sw)), wlb = whb + NP * 128;
    const int rem = sg.kpad - c * kChunk;
    const int nk = rem >= kChunk ? 4 : (rem + 15) / 16;
    for (int ks = 0; ks < nk; ++ks) {
      const uint64_t ah = desc_sw128(ahb + ks * 32), bh = desc_sw128(whb + ks * 32);
      mma_bf16(tmem_acc, ah, bh, idesc, (c | ks) != 0);
      if (split) {
        mma_bf16(tmem_acc, desc_sw128(alb + ks * 32), bh, idesc, 1u);
        mma_bf16(tmem_acc, ah, desc_sw128(wlb + ks * 32), idesc, 1u);
      }
    }
    mma_commit(&B.aempty[sa]);
    mma_commit(&B.wempty[sw]);
  }
  mma_commit(&B.tfull[tt & 1u]);
}

template <int NP>
__device__ __forceinline__ void wload_tile(const Seg3& sg, uint8_t* pipe, Bars& B,
                                           const uint8_t* wpack, uint32_t& wit) {
  using PP = Pipe<NP>;
  for (int c = 0; c < sg.nchunks; ++c, ++wit) {
    const uint32_t sw = wit % kWStages;
    wait_free(&B.wempty[sw], wit / kWStages);
    mbar_arrive_expect_tx(&B.wfull[sw], PP::kWStage);
    bulk_g2s(PP::w(pipe, sw), wpack + (size_t)c * PP::kWStage, PP::kWStage, &B.wfull[sw]);
  }
}

template <int NP>
__device__ __forceinline__ void produce_tile(const Seg3& sg, bool split, uint8_t* pipe, Bars& B,
                                             uint32_t& ait, const RowDesc& rd,
                                             const float* s_omega, const float* s_phi,
                                             const float* table) {
  using PP = Pipe<NP>;
  const int pt = threadIdx.x - kProdWarp0 * 32;
  const int r = pt >> 1, jb = (pt & 1) * 4;
  const int lane = threadIdx.x & 31;
  float cur[32], nxt[32];
  load_chunk(0, sg, rd, r, jb, s_omega, s_phi, table, cur);
  for (int c = 0; c < sg.nchunks; ++c, ++ait) {
    const uint32_t sa = ait % kAStages;
    if (c + 1 < sg.nchunks) load_chunk(c + 1, sg, rd, r, jb, s_omega, s_phi, table, nxt);
    wait_free(&B.aempty[sa], ait / kAStages);
    uint8_t* st = PP::a(pipe, sa);
    store_chunk(cur, st, st + kAPart, r, jb, split);
    fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) mbar_arrive(&B.afull[sa]);
#pragma unroll
    for (int i = 0; i < 32; ++i) cur[i] = nxt[i];
  }
}

__device__ __forceinline__ void ws_init(Bars& B, uint32_t* s_tmem, uint32_t ncols) {
  if (threadIdx.x == 0) {
    for (int s = 0; s < kAStages; ++s) {
      mbar_init(&B.afull[s], kProdWarps);
      mbar_init(&B.aempty[s], 1);
    }
    for (int s = 0; s < kWStages; ++s) {
      mbar_init(&B.wfull[s], 1);
      mbar_init(&B.wempty[s], 1);
    }
    for (int s = 0; s < kDSlots; ++s) {
      mbar_init(&B.dfull[s], 1);
      mbar_init(&B.dempty[s], kProdWarps + kEpiWarps);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&B.tfull[a], 1);
      mbar_init(&B.tempty[a], kEpiWarps);
    }
    fence_mbar_init();
  }
  if ((threadIdx.x >> 5) == kMmaWarp) tmem_alloc(s_tmem, ncols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
}

__device__ __forceinline__ void ws_teardown(uint32_t tmem, uint32_t ncols) {
  tc_fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == kMmaWarp) tmem_dealloc(tmem, ncols);
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
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  ws_init(B, &s_tmem, 2 * kCols);
  const uint32_t tmem = s_tmem;
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
      for (int r = lane; r < kBM; r += 32) {
        const float *p0 = nullptr, *p1 = nullptr;
        if (r < rows) {
          const int64_t i = i0 + r;
          const int64_t hrow = a.hdst_idx ? (int64_t)a.hdst_idx[i] : i;
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
        R.trow[r] = (!kFfn && a.table != nullptr) ? 0 : -1;   // precomputed_zeros = row 0
        R.rdst[r] = r < rows ? r : -1;
      }
      warp_arrive(&B.dfull[ds]);
    }
  } else if (warp == kWWarp) {                       // ---------------- weight loader
    uint32_t wit = 0;
    if (lane == 0)
      while (sched.next(i0, rows)) wload_tile<kNPq>(sg, pipe, B, wpack, wit);
    __syncwarp();
  } else if (warp >= kProdWarp0) {                   // ---------------- producers
    uint32_t ait = 0;
    for (; sched.next(i0, rows); ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      produce_tile<kNPq>(sg, split, pipe, B, ait, rd[ds], s_omega, s_phi, a.table);
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp == kMmaWarp) {                     // ---------------- MMA issuer
    uint32_t ait = 0, wit = 0;
    if (lane == 0)
      for (; sched.next(i0, rows); ++tt)
        mma_tile<kNPq, kNPq>(sg, split, pipe, B, tmem + (tt & 1u) * kCols, ait, wit, tt);
    __syncwarp();
  } else {                                           // ---------------- epilogue
    const int row = warp * 32 + lane;
    const int D = P.d_model;
    for (; sched.next(i0, rows); ++tt) {
      const uint32_t ab = tt & 1u, ds = tt % kDSlots;
      mbar_wait(&B.tfull[ab], (tt >> 1) & 1u);
      tc_fence_after();
      warp_arrive(&B.dempty[ds]);                     // descriptors not needed here
      (void)ds;
      const uint32_t ta = tmem + ab * kCols + ((uint32_t)(warp * 32) << 16);
      float v[32];
      if (!kFfn) {
        float* q = a.qbuf + (i0 + row) * kQLd;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (row < rows) {
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              const int col = cq * 32 + j;
              if (col < D) {
                float4 o = make_float4(v[j] + P.bq[col], v[j + 1] + P.bq[col + 1],
                                       v[j + 2] + P.bq[col + 2], v[j + 3] + P.bq[col + 3]);
                *reinterpret_cast<float4*>(q + col) = o;   // D % 4 == 0 (D == 100)
              }
            }
          }
        }
      } else {
        // out = LayerNorm(ReLU(acc + bo)): three passes over TMEM (sum, squares, write)
        float s = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int col = cq * 32 + j;
            if (col < D) s += fmaxf(v[j] + P.bo[col], 0.f);
          }
        }
        const float mean = s / (float)D;
        float q2 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int col = cq * 32 + j;
            if (col < D) {
              const float d = fmaxf(v[j] + P.bo[col], 0.f) - mean;
              q2 += d * d;
            }
          }
        }
        const float inv = rsqrtf(q2 / (float)D + P.ln_eps);
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
                  r4[e] = (fmaxf(v[j + e] + P.bo[col + e], 0.f) - mean) * inv * P.ln_gamma[col + e] +
                          P.ln_beta[col + e];
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
  ws_teardown(tmem, 2 * kCols);
}

// ------------------------------------------------------------------ S6,S7,S9-S12 (edge rows)
constexpr int kNPkv = 200;   // [Wk ; Wv] rows (2 * d_model)
constexpr int kKvEpiBytes = (2 * kMaxDpb * kMaxModel + kBM * 33) * 4;   // s_q, s_r, s_pv

__global__ void __launch_bounds__(kWsThreads, 1) kv_kernel(Args a) {
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
      while (sched.next(t0, rows)) wload_tile<kNPkv>(a.skv, pipe, B, a.wkv, wit);
    __syncwarp();
  } else if (warp >= kProdWarp0) {                   // ---------------- producers
    uint32_t ait = 0;
    for (; sched.next(t0, rows); ++tt) {
      const uint32_t ds = tt % kDSlots;
      mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
      produce_tile<kNPkv>(a.skv, split, pipe, B, ait, rd[ds], s_omega, s_phi, a.table);
      warp_arrive(&B.dempty[ds]);
    }
  } else if (warp == kMmaWarp) {                     // ---------------- MMA issuer
    uint32_t ait = 0, wit = 0;
    if (lane == 0)
      for (; sched.next(t0, rows); ++tt)
        mma_tile<kNPkv, kNPkv>(a.skv, split, pipe, B, tmem + (tt & 1u) * kCols, ait, wit, tt);
    __syncwarp();
  } else {                                           // ---------------- epilogue (128 threads)
    const int tid = threadIdx.x;                      // 0..127
    const int row = tid;
    while (sched.next_group()) {
      const int64_t d0 = sched.d0;
      const int nd = sched.nd;
      for (int x = tid; x < kMaxDpb * kMaxModel; x += kBM) {
        const int d = x / kMaxModel, c = x % kMaxModel;
        s_q[d][c] = (d < nd && c < dm) ? a.qbuf[(d0 + d) * kQLd + c] : 0.f;
        s_r[d][c] = 0.f;
      }
      if (tid < kMaxDpb * 2) {
        s_m[tid >> 1][tid & 1] = -INFINITY;
        s_l[tid >> 1][tid & 1] = 0.f;
      }
      if (tid <= nd) s_seg[tid] = a.seg_ptr[d0 + tid];
      named_bar(kBarEpi, kBM);
      for (; sched.next_tile(t0, rows); ++tt) {
        const int64_t c0 = t0;
        const uint32_t ab = tt & 1u, ds = tt % kDSlots;
        mbar_wait(&B.dfull[ds], (tt / kDSlots) & 1u);
        mbar_wait(&B.tfull[ab], (tt >> 1) & 1u);
        tc_fence_after();
        const int d = rd[ds].rdst[row];
        warp_arrive(&B.dempty[ds]);
        const uint32_t ta = tmem + ab * kCols + ((uint32_t)(warp * 32) << 16);
        float v[32];
        // S10: logits per head from the K columns [0, dm)
        float p0 = 0.f, p1 = 0.f;
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + cq * 32, v);
          tmem_wait_ld();
          if (d >= 0) {
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              const int col = cq * 32 + j;
              if (col < dm) {
                const float pr = s_q[d][col] * (v[j] + s_bias[col]);
                if (col < dh) p0 += pr; else p1 += pr;
              }
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
          const int64_t a0 = s_seg[dd] > c0 ? s_seg[dd] : c0;
          const int64_t a1 = s_seg[dd + 1] < c0 + rows ? s_seg[dd + 1] : c0 + rows;
          float sc = 1.f;
          if (a0 < a1) {
            float mc = -INFINITY;
            for (int64_t e = a0; e < a1; ++e) mc = fmaxf(mc, s_logit[e - c0][h]);
            const float mo = s_m[dd][h];
            const float mn = fmaxf(mo, mc);
            sc = (mo == -INFINITY) ? 0.f : expf(mo - mn);
            float l = s_l[dd][h] * sc;
            for (int64_t e = a0; e < a1; ++e) {
              const float pe = expf(s_logit[e - c0][h] - mn);
              s_p[e - c0][h] = pe;
              l += pe;
            }
            s_m[dd][h] = mn;
            s_l[dd][h] = l;
          }
          s_sc[dd][h] = sc;
        }
        named_bar(kBarEpi, kBM);
        // S12: r = r * sc + sum_rows p * v, 32 V columns at a time (fixed order)
#pragma unroll 1
        for (int cq = 0; cq < 4; ++cq) {
          tmem_ld32(ta + dm + cq * 32, v);
          tmem_wait_ld();
          if (d >= 0) {
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              const int col = cq * 32 + j;
              s_pv[row][j] = col < dm ? s_p[row][col < dh ? 0 : 1] * (v[j] + s_bias[dm + col]) : 0.f;
            }
          }
          named_bar(kBarEpi, kBM);
          for (int x = tid; x < nd * 32; x += kBM) {
            const int dd = x >> 5, j = x & 31, col = cq * 32 + j;
            if (col >= dm) continue;
            const int64_t a0 = s_seg[dd] > c0 ? s_seg[dd] : c0;
            const int64_t a1 = s_seg[dd + 1] < c0 + rows ? s_seg[dd + 1] : c0 + rows;
            if (a0 >= a1) continue;
            float acc = s_r[dd][col] * s_sc[dd][col < dh ? 0 : 1];
            for (int64_t e = a0; e < a1; ++e) acc += s_pv[e - c0][j];
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

}  // namespace tca

// ------------------------------------------------------------------ host side
namespace tca {

struct PackedLayout {
  size_t oq, okv, oo, total;
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
  return launch_check("pack_weights");
}

}  // namespace tca

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

  const int smem_q = Pipe<kNPq>::kBytes + 1024;
  const int smem_kv = Pipe<kNPkv>::kBytes + 1024 + kKvEpiBytes;
  static bool attr_done = false;   // cached cudaFuncSetAttribute (idempotent)
  if (!attr_done) {
    TGL_TRY(cuda_check(cudaFuncSetAttribute(dense_kernel<false>,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize, smem_q),
                       "attr q"));
    TGL_TRY(cuda_check(cudaFuncSetAttribute(dense_kernel<true>,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize, smem_q),
                       "attr ffn"));
    TGL_TRY(cuda_check(cudaFuncSetAttribute(kv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            smem_kv), "attr kv"));
    attr_done = true;
  }
  const int64_t tiles = ceil_div(n_dst_max, kBM);
  const unsigned gq = (unsigned)(tiles < kNumSMs ? tiles : kNumSMs);
  dense_kernel<false><<<gq, kWsThreads, smem_q, s>>>(a);
  TGL_TRY(launch_check("tc q kernel"));
  const int64_t groups = ceil_div(n_dst_max, a.dpb);
  const unsigned gkv = (unsigned)(groups < kNumSMs ? groups : kNumSMs);
  kv_kernel<<<gkv, kWsThreads, smem_kv, s>>>(a);
  TGL_TRY(launch_check("tc kv kernel"));
  dense_kernel<true><<<gq, kWsThreads, smem_q, s>>>(a);
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
