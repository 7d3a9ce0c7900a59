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

// Per-CTA shared-memory image (dynamic, 1024-aligned base).
struct RowDesc {
  const float* p0[kBM];
  const float* p1[kBM];
  float dt[kBM];
  int trow[kBM];
  int rdst[kBM];
};

template <int NP>
struct Smem {
  static constexpr int kWChunk = 2 * NP * 128;
  static constexpr int kStage = 2 * kAPart + kWChunk;   // A_hi, A_lo, W (hi|lo)
  static constexpr int kStages = 2;
  static constexpr int kPipe = kStages * kStage;
};

__device__ __forceinline__ void load8(const float* p, int lc, int d, float (&x)[8]) {
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

// Producer: rows' 64-wide K chunk c -> swizzled bf16 hi (and lo) tiles.
__device__ __forceinline__ void gather_chunk(int c, const Seg3& sg, bool split, uint8_t* a_hi,
                                             uint8_t* a_lo, const RowDesc& rd, int rows,
                                             const float* s_omega, const float* s_phi,
                                             const float* table) {
  const int t = threadIdx.x;
  const int r = t >> 1, jb = (t & 1) * 4;
  const uint32_t hi_base = smem_u32(a_hi), lo_base = smem_u32(a_lo);
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
    const int j = jb + jj;
    const int kp = c * kChunk + j * 8;
    float x[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) x[e] = 0.f;
    if (r < rows && kp < sg.kpad) {
      if (kp < sg.p0) {
        load8(rd.p0[r], kp, sg.d0, x);
      } else if (kp < sg.p0 + sg.p1) {
        load8(rd.p1[r], kp - sg.p0, sg.d1, x);
      } else {
        const int j0 = kp - sg.p0 - sg.p1;
        const int trow = rd.trow[r];
        if (trow >= 0) {
          load8(table + (int64_t)trow * sg.d2, j0, sg.d2, x);
        } else {
          const float dt = rd.dt[r];
#pragma unroll
          for (int e = 0; e < 8; ++e)
            if (j0 + e < sg.d2) x[e] = tenc_direct(dt, s_omega[j0 + e], s_phi[j0 + e]);
        }
      }
    }
    uint32_t h[4], l[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) split2(x[2 * e], x[2 * e + 1], h[e], l[e]);
    const uint32_t off = sw128_off(r, j);
    st_shared_v4(hi_base + off, h[0], h[1], h[2], h[3]);
    if (split) st_shared_v4(lo_base + off, l[0], l[1], l[2], l[3]);
  }
}

// One M-tile of 128 rows: all K chunks through the 2-stage pipeline.  All threads
// gather; thread 0 moves W chunks (bulk copy) and issues the MMAs.  On return the
// accumulator in TMEM is complete and visible (after tc_fence_after).
template <int NP, int N>
__device__ __forceinline__ void mainloop(const Seg3& sg, bool split, uint8_t* pipe,
                                         const uint8_t* wpack, uint64_t* w_bar,
                                         uint64_t* mma_bar, uint32_t tmem_d, uint32_t& it,
                                         const RowDesc& rd, int rows, const float* s_omega,
                                         const float* s_phi, const float* table) {
  using S = Smem<NP>;
  constexpr uint32_t idesc = idesc_bf16(kBM, N);
  uint32_t last_stage = 0, last_parity = 0;
  for (int c = 0; c < sg.nchunks; ++c) {
    const uint32_t s = it & 1u;
    uint8_t* st = pipe + s * S::kStage;
    uint8_t* a_hi = st;
    uint8_t* a_lo = st + kAPart;
    uint8_t* w = st + 2 * kAPart;
    if (it >= 2) mbar_wait(&mma_bar[s], ((it - 2) >> 1) & 1u);
    if (threadIdx.x == 0) {
      mbar_arrive_expect_tx(&w_bar[s], S::kWChunk);
      bulk_g2s(w, wpack + (size_t)c * S::kWChunk, S::kWChunk, &w_bar[s]);
    }
    gather_chunk(c, sg, split, a_hi, a_lo, rd, rows, s_omega, s_phi, table);
    fence_proxy_async_smem();
    __syncthreads();
    if (threadIdx.x == 0) {
      mbar_wait(&w_bar[s], (it >> 1) & 1u);
      tc_fence_after();
      const int rem = sg.kpad - c * kChunk;
      const int nk = rem >= kChunk ? 4 : (rem + 15) / 16;
      const uint32_t ahb = smem_u32(a_hi), alb = smem_u32(a_lo), whb = smem_u32(w);
      const uint32_t wlb = whb + NP * 128;
      for (int ks = 0; ks < nk; ++ks) {
        const uint64_t ah = desc_sw128(ahb + ks * 32), bh = desc_sw128(whb + ks * 32);
        mma_bf16(tmem_d, ah, bh, idesc, (c | ks) != 0);
        if (split) {
          const uint64_t al = desc_sw128(alb + ks * 32), bl = desc_sw128(wlb + ks * 32);
          mma_bf16(tmem_d, al, bh, idesc, 1u);
          mma_bf16(tmem_d, ah, bl, idesc, 1u);
        }
      }
      mma_commit(&mma_bar[s]);
    }
    last_stage = s;
    last_parity = (it >> 1) & 1u;
    ++it;
  }
  mbar_wait(&mma_bar[last_stage], last_parity);
  tc_fence_after();
}

__device__ __forceinline__ uint8_t* align1024(uint8_t* p) {
  return reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(p) + 1023) & ~uintptr_t(1023));
}

// common prologue: barriers + TMEM allocation
template <int NCOLS>
__device__ __forceinline__ uint32_t prologue(uint64_t* w_bar, uint64_t* mma_bar, uint32_t* s_tmem) {
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&w_bar[i], 1);
      mbar_init(&mma_bar[i], 1);
    }
    fence_mbar_init();
  }
  if ((threadIdx.x >> 5) == 0) tmem_alloc(s_tmem, NCOLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  return *s_tmem;
}

template <int NCOLS>
__device__ __forceinline__ void epilogue_teardown(uint32_t tmem) {
  tc_fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tmem_dealloc(tmem, NCOLS);
}

// ------------------------------------------------------------------ S8: q projection
constexpr int kNPq = 104;   // d_model padded to a multiple of 8 (rows of Wq / Wo)

__global__ void __launch_bounds__(kThreads, 1) q_kernel(Args a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  using S = Smem<kNPq>;
  __shared__ uint64_t w_bar[2], mma_bar[2];
  __shared__ uint32_t s_tmem;
  __shared__ RowDesc rd;
  __shared__ float s_omega[256], s_phi[256];
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t tiles = (n + kBM - 1) / kBM;
  const uint32_t tmem = prologue<128>(w_bar, mma_bar, &s_tmem);
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  uint32_t it = 0;
  const int dm = P.d_model;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q4 = warp & 3, half = warp >> 2;
  const int HC = (dm + 1) / 2;
  for (int64_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const int64_t i0 = tile * kBM;
    const int rows = (int)((n - i0) < kBM ? (n - i0) : kBM);
    if (threadIdx.x < kBM) {
      const int r = threadIdx.x;
      const float* p0 = nullptr;
      if (r < rows) {
        const int64_t i = i0 + r;
        const int64_t row = a.hdst_idx ? (int64_t)a.hdst_idx[i] : i;
        p0 = a.hdst + row * a.ld_hdst;
      }
      rd.p0[r] = p0;
      rd.p1[r] = nullptr;
      rd.dt[r] = 0.0f;                          // Phi(0): eq 4 / L2.27
      rd.trow[r] = a.table != nullptr ? 0 : -1;  // precomputed_zeros == table row 0
    }
    __syncthreads();
    mainloop<kNPq, kNPq>(a.sq, a.split, pipe, a.wq, w_bar, mma_bar, tmem, it, rd, rows, s_omega,
                         s_phi, a.table);
    // epilogue: thread (quarter q4, lane) = row, half selects columns [cb, cb+HC)
    const int row = q4 * 32 + lane;
    const int cb = half * HC;
    float v[64];
    const uint32_t ta = tmem + ((uint32_t)(q4 * 32) << 16) + cb;
    tmem_ld32(ta, &v[0]);
    tmem_ld32(ta + 32, &v[32]);
    tmem_wait_ld();
    if (row < rows) {
      float* q = a.qbuf + (i0 + row) * kQLd;
#pragma unroll
      for (int j = 0; j < 64; ++j)
        if (j < HC && cb + j < dm) q[cb + j] = v[j] + P.bq[cb + j];
    }
    tc_fence_before();
    __syncthreads();
  }
  epilogue_teardown<128>(tmem);
}

// ------------------------------------------------------------------ S13: FFN
__global__ void __launch_bounds__(kThreads, 1) ffn_kernel(Args a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ uint64_t w_bar[2], mma_bar[2];
  __shared__ uint32_t s_tmem;
  __shared__ RowDesc rd;
  __shared__ float s_part[2][kBM];
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t tiles = (n + kBM - 1) / kBM;
  const uint32_t tmem = prologue<128>(w_bar, mma_bar, &s_tmem);
  uint32_t it = 0;
  const int D = P.d_out;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q4 = warp & 3, half = warp >> 2;
  const int HC = (D + 1) / 2;
  for (int64_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    const int64_t i0 = tile * kBM;
    const int rows = (int)((n - i0) < kBM ? (n - i0) : kBM);
    if (threadIdx.x < kBM) {
      const int r = threadIdx.x;
      const float *p0 = nullptr, *p1 = nullptr;
      if (r < rows) {
        const int64_t i = i0 + r;
        const int64_t row = a.hdst_idx ? (int64_t)a.hdst_idx[i] : i;
        p0 = a.rbuf + i * kQLd;                 // [r_i ; h_i], eq 7
        p1 = a.hdst + row * a.ld_hdst;
      }
      rd.p0[r] = p0;
      rd.p1[r] = p1;
      rd.dt[r] = 0.f;
      rd.trow[r] = -1;
    }
    __syncthreads();
    mainloop<kNPq, kNPq>(a.so, a.split, pipe, a.wo, w_bar, mma_bar, tmem, it, rd, rows, nullptr,
                         nullptr, nullptr);
    const int row = q4 * 32 + lane;
    const int cb = half * HC;
    const int ce = cb + HC < D ? cb + HC : D;
    float v[64];
    const uint32_t ta = tmem + ((uint32_t)(q4 * 32) << 16) + cb;
    tmem_ld32(ta, &v[0]);
    tmem_ld32(ta + 32, &v[32]);
    tmem_wait_ld();
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < 64; ++j) {
      const int col = cb + j;
      const float o = col < ce ? fmaxf(v[j] + P.bo[col], 0.f) : 0.f;   // ReLU
      v[j] = o;
      s += o;
    }
    s_part[half][row] = s;
    __syncthreads();
    const float mean = (s_part[0][row] + s_part[1][row]) / (float)D;
    float q = 0.f;
#pragma unroll
    for (int j = 0; j < 64; ++j) {
      const float d = cb + j < ce ? v[j] - mean : 0.f;
      q += d * d;
    }
    __syncthreads();
    s_part[half][row] = q;
    __syncthreads();
    const float var = (s_part[0][row] + s_part[1][row]) / (float)D;
    const float inv = rsqrtf(var + P.ln_eps);
    if (row < rows) {
      float* o = a.out + (i0 + row) * D;
#pragma unroll
      for (int j = 0; j < 64; ++j) {
        const int col = cb + j;
        if (col < ce) o[col] = (v[j] - mean) * inv * P.ln_gamma[col] + P.ln_beta[col];
      }
    }
    tc_fence_before();
    __syncthreads();
  }
  epilogue_teardown<128>(tmem);
}

// ------------------------------------------------------------------ S6,S7,S9-S12
constexpr int kNPkv = 200;   // 2 * d_model rows of [Wk ; Wv] (d_model = 100)

__global__ void __launch_bounds__(kThreads, 1) kv_kernel(Args a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* pipe = align1024(smem_raw);
  __shared__ uint64_t w_bar[2], mma_bar[2];
  __shared__ uint32_t s_tmem;
  __shared__ RowDesc rd;
  __shared__ float s_omega[256], s_phi[256];
  __shared__ float s_bias[2 * kMaxModel];
  __shared__ float s_q[kMaxDpb][kMaxModel];
  __shared__ float s_r[kMaxDpb][kMaxModel];
  __shared__ float s_lpart[2][kBM][2];
  __shared__ float s_logit[kBM][2];
  __shared__ float s_p[kBM][2];
  __shared__ float s_m[kMaxDpb][2], s_l[kMaxDpb][2], s_sc[kMaxDpb][2];
  __shared__ int64_t s_seg[kMaxDpb + 1];
  __shared__ float s_tdst[kMaxDpb];
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t groups = (n + a.dpb - 1) / a.dpb;
  const uint32_t tmem = prologue<256>(w_bar, mma_bar, &s_tmem);
  const int dm = P.d_model, H = P.n_heads, dh = dm / H;
  const int tid = threadIdx.x;
  for (int j = tid; j < P.d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
  for (int j = tid; j < 2 * dm; j += blockDim.x) s_bias[j] = j < dm ? P.bk[j] : P.bv[j - dm];
  const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
  const int warp = tid >> 5, lane = tid & 31;
  const int q4 = warp & 3, half = warp >> 2;
  const int HC = (dm + 1) / 2;
  const int cb = half * HC, ce = cb + HC < dm ? cb + HC : dm;
  float* s_pv = reinterpret_cast<float*>(pipe);   // [kBM][dm+1] scratch, reuses stage memory
  const int pv_ld = dm + 1;
  uint32_t it = 0;

  for (int64_t g = blockIdx.x; g < groups; g += gridDim.x) {
    const int64_t d0 = g * a.dpb;
    const int nd = (int)((n - d0) < a.dpb ? (n - d0) : a.dpb);
    for (int x = tid; x < kMaxDpb * kMaxModel; x += blockDim.x) {
      const int d = x / kMaxModel, c = x % kMaxModel;
      s_q[d][c] = (d < nd && c < dm) ? a.qbuf[(d0 + d) * kQLd + c] : 0.f;
      s_r[d][c] = 0.f;
    }
    if (tid < kMaxDpb * 2) {
      s_m[tid >> 1][tid & 1] = -INFINITY;
      s_l[tid >> 1][tid & 1] = 0.f;
    }
    if (tid <= nd) s_seg[tid] = a.seg_ptr[d0 + tid];
    if (tid < nd) s_tdst[tid] = a.dst_t[d0 + tid];
    __syncthreads();
    const int64_t e_begin = s_seg[0], e_end = s_seg[nd];
    for (int64_t c0 = e_begin; c0 < e_end; c0 += kBM) {
      const int rows = (int)((e_end - c0) < kBM ? (e_end - c0) : kBM);
      if (tid < kBM) {
        const int r = tid;
        int ld = -1;
        const float *p0 = nullptr, *p1 = nullptr;
        float dt = 0.f;
        int trow = -1;
        if (r < rows) {
          const int64_t e = c0 + r;
          int lo = 0, hi = nd;
          while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (s_seg[mid] <= e) lo = mid; else hi = mid;
          }
          ld = lo;
          const int64_t hr = a.hsrc_idx ? (int64_t)a.hsrc_idx[hoff + e] : hoff + e;
          p0 = a.hsrc + hr * a.ld_hsrc;
          if (P.d_e > 0) p1 = a.efeat + (int64_t)a.eid[e] * a.ld_e;
          dt = s_tdst[ld] - a.edge_t[e];          // fp32 delta (R18)
          trow = (int)tenc_table_row(dt, a.table, a.window);
        }
        rd.p0[r] = p0;
        rd.p1[r] = p1;
        rd.dt[r] = dt;
        rd.trow[r] = trow;
        rd.rdst[r] = ld;
      }
      __syncthreads();
      mainloop<kNPkv, kNPkv>(a.skv, a.split, pipe, a.wkv, w_bar, mma_bar, tmem, it, rd, rows,
                             s_omega, s_phi, a.table);
      // ---- epilogue: TMEM lane = row; warp half selects columns [cb, ce)
      const int row = q4 * 32 + lane;
      const int d = row < rows ? rd.rdst[row] : -1;
      const uint32_t ta = tmem + ((uint32_t)(q4 * 32) << 16);
      float v[64];
      tmem_ld32(ta + cb, &v[0]);        // K columns
      tmem_ld32(ta + cb + 32, &v[32]);
      tmem_wait_ld();
      float p0 = 0.f, p1 = 0.f;
      if (d >= 0) {
#pragma unroll
        for (int j = 0; j < 64; ++j) {
          const int col = cb + j;
          if (col < ce) {
            const float pr = s_q[d][col] * (v[j] + s_bias[col]);
            if (col / dh == 0) p0 += pr; else p1 += pr;
          }
        }
      }
      s_lpart[half][row][0] = p0;
      s_lpart[half][row][1] = p1;
      __syncthreads();
      if (tid < kBM && tid < rows) {   // S10: logits + LeakyReLU
        float s0 = (s_lpart[0][tid][0] + s_lpart[1][tid][0]) * P.logit_scale;
        float s1 = (s_lpart[0][tid][1] + s_lpart[1][tid][1]) * P.logit_scale;
        if (P.leaky_slope >= 0.f) {
          s0 = s0 < 0.f ? s0 * P.leaky_slope : s0;
          s1 = s1 < 0.f ? s1 * P.leaky_slope : s1;
        }
        s_logit[tid][0] = s0;
        s_logit[tid][1] = s1;
      }
      __syncthreads();
      if (tid < nd * H) {               // S11: online segmented softmax statistics
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
      __syncthreads();
      tmem_ld32(ta + dm + cb, &v[0]);    // V columns
      tmem_ld32(ta + dm + cb + 32, &v[32]);
      tmem_wait_ld();
      if (row < rows) {
#pragma unroll
        for (int j = 0; j < 64; ++j) {
          const int col = cb + j;
          if (col < ce) s_pv[row * pv_ld + col] = s_p[row][col / dh] * (v[j] + s_bias[dm + col]);
        }
      }
      __syncthreads();
      // S12: r = r * sc + sum over this chunk's rows (fixed order -> deterministic)
      for (int x = tid; x < nd * dm; x += blockDim.x) {
        const int dd = x / dm, col = x % dm;
        const int64_t a0 = s_seg[dd] > c0 ? s_seg[dd] : c0;
        const int64_t a1 = s_seg[dd + 1] < c0 + rows ? s_seg[dd + 1] : c0 + rows;
        if (a0 >= a1) continue;
        float acc = s_r[dd][col] * s_sc[dd][col / dh];
        for (int64_t e = a0; e < a1; ++e) acc += s_pv[(e - c0) * pv_ld + col];
        s_r[dd][col] = acc;
      }
      fence_proxy_async_smem();   // generic s_pv accesses before the next async-proxy writes
      tc_fence_before();
      __syncthreads();
    }
    // normalise (empty segment -> 0, R19)
    for (int x = tid; x < nd * dm; x += blockDim.x) {
      const int dd = x / dm, col = x % dm;
      const float l = s_l[dd][col / dh];
      a.rbuf[(d0 + dd) * kQLd + col] = l > 0.f ? s_r[dd][col] / l : 0.f;
    }
    __syncthreads();
  }
  epilogue_teardown<256>(tmem);
}

}  // namespace tca

// host entry used by tgl_tblock_attn (attn.cu) for TGL_FP32 / TGL_BF16
size_t tc_attn_ws_bytes(const tgl_attn_params* P, int64_t n_dst_max, size_t* o_q, size_t* o_r,
                        size_t* o_wq, size_t* o_wkv, size_t* o_wo) {
  using namespace tca;
  WsLayout L;
  const int64_t nrows = n_dst_max > 0 ? n_dst_max : 1;
  *o_q = L.take(sizeof(float) * kQLd * nrows);
  *o_r = L.take(sizeof(float) * kQLd * nrows);
  const Seg3 sq = make_seg3(P->d_hdst, 0, P->d_t);
  const Seg3 skv = make_seg3(P->d_hsrc, P->d_e, P->d_t);
  const Seg3 so = make_seg3(P->d_model, P->d_hdst, 0);
  *o_wq = L.take((size_t)sq.nchunks * 2 * kNPq * 128);
  *o_wkv = L.take((size_t)skv.nchunks * 2 * kNPkv * 128);
  *o_wo = L.take((size_t)so.nchunks * 2 * kNPq * 128);
  return L.off;
}

bool tc_attn_supported(const tgl_attn_params* P) {
  return P->d_model == 100 && P->d_out == 100 && P->n_heads >= 1 && P->n_heads <= 2 &&
         P->d_t <= 256;
}

tgl_status tc_attn_launch(const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev,
                          const int64_t* seg_ptr, const float* dst_t, const float* hdst,
                          const int32_t* hdst_idx, int64_t ld_hdst, const float* hsrc,
                          const int32_t* hsrc_idx, const int64_t* hsrc_off_dev, int64_t ld_hsrc,
                          const float* efeat, const int32_t* eid, int64_t ld_e,
                          const float* edge_t, const float* table, int64_t window,
                          int32_t max_seg, float* out, void* ws, cudaStream_t s) {
  using namespace tca;
  size_t o_q, o_r, o_wq, o_wkv, o_wo;
  tc_attn_ws_bytes(P, n_dst_max, &o_q, &o_r, &o_wq, &o_wkv, &o_wo);
  char* w = static_cast<char*>(ws);
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
  a.wq = reinterpret_cast<const uint8_t*>(w + o_wq);
  a.wkv = reinterpret_cast<const uint8_t*>(w + o_wkv);
  a.wo = reinterpret_cast<const uint8_t*>(w + o_wo);
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

  // 1. pack weights (bf16 hi/lo, padded K, pre-swizzled)
  PackJob jq{P->Wq, nullptr, P->d_model, P->d_model, kNPq, P->d_hdst + P->d_t, a.sq,
             reinterpret_cast<uint8_t*>(w + o_wq)};
  PackJob jkv{P->Wk, P->Wv, P->d_model, 2 * P->d_model, kNPkv, P->d_hsrc + P->d_e + P->d_t,
              a.skv, reinterpret_cast<uint8_t*>(w + o_wkv)};
  PackJob jo{P->Wo, nullptr, P->d_out, P->d_out, kNPq, P->d_model + P->d_hdst, a.so,
             reinterpret_cast<uint8_t*>(w + o_wo)};
  pack_weights_kernel<<<dim3(64, 3), 256, 0, s>>>(jq, jkv, jo);
  TGL_TRY(launch_check("pack_weights"));

  const int smem_q = Smem<kNPq>::kPipe + 1024;
  const int smem_kv = Smem<kNPkv>::kPipe + 1024;
  static bool attr_done = false;   // cached cudaFuncSetAttribute (idempotent)
  if (!attr_done) {
    TGL_TRY(cuda_check(cudaFuncSetAttribute(q_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            smem_q), "attr q"));
    TGL_TRY(cuda_check(cudaFuncSetAttribute(ffn_kernel,
                                            cudaFuncAttributeMaxDynamicSharedMemorySize, smem_q),
                       "attr ffn"));
    TGL_TRY(cuda_check(cudaFuncSetAttribute(kv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            smem_kv), "attr kv"));
    attr_done = true;
  }
  const int64_t tiles = ceil_div(n_dst_max, kBM);
  const unsigned gq = (unsigned)(tiles < kNumSMs ? tiles : kNumSMs);
  q_kernel<<<gq, kThreads, smem_q, s>>>(a);
  TGL_TRY(launch_check("tc q_kernel"));
  const int64_t groups = ceil_div(n_dst_max, a.dpb);
  const unsigned gkv = (unsigned)(groups < kNumSMs ? groups : kNumSMs);
  kv_kernel<<<gkv, kThreads, smem_kv, s>>>(a);
  TGL_TRY(launch_check("tc kv_kernel"));
  ffn_kernel<<<gq, kThreads, smem_q, s>>>(a);
  return launch_check("tc ffn_kernel");
}

}  // namespace tgl
