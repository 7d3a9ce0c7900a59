// attn.cu -- S7-S13: one TBlock of TGAT temporal attention (eqs 4-7, P:104-119;
// Listing 2 TemporalAttnLayer.forward; readings R10-R13, R19).
//
// Three kernels, all on the caller's stream, no host sync:
//   1. q_proj     : q_i = Wq [h_i ; Phi(0)] + bq                  (S8)
//   2. kv_attn    : per CTA a run of destinations; their edges are processed in
//                   128-row chunks: gather [h_src ; e ; Phi(dt)] rows straight
//                   into shared memory (S6+S7 fused, nothing materialised in HBM),
//                   K|V = Z W^T + b (S9), logits + LeakyReLU (S10), online
//                   segmented softmax (S11) and the alpha-weighted scatter-sum
//                   (S12) finish in shared memory; only r_i leaves the SM.
//   3. out_ffn    : out_i = LayerNorm(ReLU(Wo [r_i ; h_i] + bo))      (S13)
// This file is the SIMT (FFMA) implementation, selected by TGL_FP32_SIMT (exact fp32
// products on the CUDA cores, fp32 accumulation; the slow reference mode).  TGL_FP32
// and TGL_BF16 run on the tensor cores (attn_tc.cu); tgl_tblock_attn below dispatches.
#include <cuda_bf16.h>

#include "common.cuh"
#include "tenc.cuh"

namespace tgl {

constexpr int kAttnThreads = 256;
constexpr int kMaxModel = 128;  // d_model limit (heads split it)
constexpr int kQLd = 128;       // leading dim of the q / r scratch rows

struct AttnArgs {
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
  float* qbuf;  // [n_dst_max][kQLd]
  float* rbuf;  // [n_dst_max][kQLd]
  int dpb;      // destinations per CTA in kv_attn
};

__device__ __forceinline__ float maybe_bf16(float x, bool bf16) {
  return bf16 ? __bfloat162float(__float2bfloat16_rn(x)) : x;
}

// ----------------------------------------------------------------------------
// Generic 64 x 128 SIMT tile:  C[64][128] = A[64][K] * W[128][K]^T, A rows
// produced by a loader functor, W rows beyond N are zero.  256 threads, thread
// tile 4 rows x 8 cols (cols cg + 16 c).
// ----------------------------------------------------------------------------
constexpr int kTBM = 64, kTBN = 128, kTBK = 32;

template <class LoadA>
__device__ __forceinline__ void tile_gemm_64x128(const LoadA& loadA, const float* __restrict__ W,
                                                 int N, int K, bool bf16, float (&acc)[4][8],
                                                 float (*As)[kTBM], float (*Ws)[kTBN]) {
  const int tid = threadIdx.x;
  const int rg = tid >> 4, cg = tid & 15;
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int c = 0; c < 8; ++c) acc[i][c] = 0.f;
  for (int k0 = 0; k0 < K; k0 += kTBK) {
    {  // A tile: thread -> row tid/4, cols (tid%4)*8 .. +7
      const int r = tid >> 2, kb = (tid & 3) * 8;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int kk = kb + u;
        const int col = k0 + kk;
        As[kk][r] = col < K ? maybe_bf16(loadA(r, col), bf16) : 0.f;
      }
    }
    {  // W tile: thread -> n = tid/2, kk = (tid%2)*16 .. +15
      const int n = tid >> 1, kb = (tid & 1) * 16;
#pragma unroll
      for (int u = 0; u < 16; ++u) {
        const int kk = kb + u, col = k0 + kk;
        Ws[kk][n] = (n < N && col < K) ? maybe_bf16(__ldg(W + (int64_t)n * K + col), bf16) : 0.f;
      }
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < kTBK; ++kk) {
      const float4 a = *reinterpret_cast<const float4*>(&As[kk][rg * 4]);
      float b[8];
#pragma unroll
      for (int c = 0; c < 8; ++c) b[c] = Ws[kk][cg + 16 * c];
      const float av[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int c = 0; c < 8; ++c) acc[i][c] = fmaf(av[i], b[c], acc[i][c]);
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------- S8
__global__ void __launch_bounds__(kAttnThreads) q_proj_kernel(AttnArgs a) {
  __shared__ __align__(16) float As[kTBK][kTBM];
  __shared__ __align__(16) float Ws[kTBK][kTBN];
  __shared__ float s_phi0[256];
  __shared__ int64_t s_row[kTBM];
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t i0 = (int64_t)blockIdx.x * kTBM;
  if (i0 >= n) return;
  const bool bf16 = P.precision == TGL_BF16;
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x)
    s_phi0[j] = tenc_direct(0.0f, P.omega[j], P.phi[j]);  // Phi(0), eq 4 / L2.27
  if (threadIdx.x < kTBM) {
    int64_t i = i0 + threadIdx.x;
    int64_t row = -1;
    if (i < n) row = a.hdst_idx ? (int64_t)a.hdst_idx[i] : i;
    s_row[threadIdx.x] = row;
  }
  __syncthreads();
  const int dh = P.d_hdst;
  auto loadA = [&](int r, int col) -> float {
    const int64_t row = s_row[r];
    if (row < 0) return 0.f;
    return col < dh ? __ldg(a.hdst + row * a.ld_hdst + col) : s_phi0[col - dh];
  };
  float acc[4][8];
  tile_gemm_64x128(loadA, P.Wq, P.d_model, dh + P.d_t, bf16, acc, As, Ws);
  const int rg = threadIdx.x >> 4, cg = threadIdx.x & 15;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int64_t r = i0 + rg * 4 + i;
    if (r >= n) continue;
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int col = cg + 16 * c;
      if (col < P.d_model) a.qbuf[r * kQLd + col] = acc[i][c] + P.bq[col];
    }
  }
}

// ---------------------------------------------------------------------- S13
__global__ void __launch_bounds__(kAttnThreads) out_ffn_kernel(AttnArgs a) {
  // the GEMM operand tiles and the epilogue tile share one buffer
  __shared__ __align__(16) float sbuf[kTBM * (kTBN + 1)];
  auto As = reinterpret_cast<float(*)[kTBM]>(sbuf);
  auto Ws = reinterpret_cast<float(*)[kTBN]>(sbuf + kTBK * kTBM);
  auto Cs = reinterpret_cast<float(*)[kTBN + 1]>(sbuf);
  __shared__ int64_t s_row[kTBM];
  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t i0 = (int64_t)blockIdx.x * kTBM;
  if (i0 >= n) return;
  const bool bf16 = P.precision == TGL_BF16;
  if (threadIdx.x < kTBM) {
    int64_t i = i0 + threadIdx.x;
    int64_t row = -1;
    if (i < n) row = a.hdst_idx ? (int64_t)a.hdst_idx[i] : i;
    s_row[threadIdx.x] = row;
  }
  __syncthreads();
  const int dm = P.d_model;
  auto loadA = [&](int r, int col) -> float {
    const int64_t row = s_row[r];
    if (row < 0) return 0.f;
    return col < dm ? a.rbuf[(i0 + r) * kQLd + col]
                    : __ldg(a.hdst + row * a.ld_hdst + (col - dm));  // [r ; h], eq 7
  };
  float acc[4][8];
  tile_gemm_64x128(loadA, P.Wo, P.d_out, dm + P.d_hdst, bf16, acc, As, Ws);
  const int rg = threadIdx.x >> 4, cg = threadIdx.x & 15;
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int col = cg + 16 * c;
      float v = 0.f;
      if (col < P.d_out) v = fmaxf(acc[i][c] + P.bo[col], 0.f);  // ReLU
      Cs[rg * 4 + i][col] = v;
    }
  __syncthreads();
  // LayerNorm per row (biased variance, eps inside the sqrt): one warp per 8 rows
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int D = P.d_out;
  for (int rr = warp; rr < kTBM; rr += kAttnThreads / 32) {
    const int64_t r = i0 + rr;
    if (r >= n) break;
    float s = 0.f;
    for (int c = lane; c < D; c += 32) s += Cs[rr][c];
    const float mean = warp_sum(s) / (float)D;
    float q = 0.f;
    for (int c = lane; c < D; c += 32) {
      const float d = Cs[rr][c] - mean;
      q += d * d;
    }
    const float var = warp_sum(q) / (float)D;
    const float inv = rsqrtf(var + P.ln_eps);
    for (int c = lane; c < D; c += 32)
      a.out[r * D + c] = (Cs[rr][c] - mean) * inv * P.ln_gamma[c] + P.ln_beta[c];
  }
}

// ---------------------------------------------------------------------- S6,S7,S9-S12
constexpr int kKvBM = 128;                 // edge rows per chunk
constexpr int kKvBN = 208;                 // k (0..99) | v (100..199) | pad
constexpr int kKvBK = 16;
constexpr int kKvTN = kKvBN / 16;          // 13 columns per thread
constexpr int kMaxDpb = 16;

__global__ void __launch_bounds__(kAttnThreads, 1) kv_attn_kernel(AttnArgs a) {
  __shared__ __align__(16) float As[kKvBK][kKvBM];
  __shared__ float Ws[kKvBK][kKvBN];
  __shared__ int64_t s_hrow[kKvBM];
  __shared__ int64_t s_erow[kKvBM];
  __shared__ float s_dt[kKvBM];
  __shared__ int s_rdst[kKvBM];          // local destination of each chunk row (-1 = none)
  __shared__ float s_logit[kKvBM][2];
  __shared__ float s_p[kKvBM][2];
  __shared__ float s_q[kMaxDpb][kMaxModel];
  __shared__ float s_r[kMaxDpb][kMaxModel];
  __shared__ float s_m[kMaxDpb][2], s_l[kMaxDpb][2], s_sc[kMaxDpb][2];
  __shared__ int64_t s_seg[kMaxDpb + 1];
  __shared__ float s_tdst[kMaxDpb];
  __shared__ float s_omega[256], s_phi[256];

  const tgl_attn_params& P = a.P;
  const int64_t n = dev_count(a.n_dst_dev, a.n_dst_max);
  const int64_t d0 = (int64_t)blockIdx.x * a.dpb;
  if (d0 >= n) return;
  const int nd = (int)((n - d0) < a.dpb ? (n - d0) : a.dpb);
  const bool bf16 = P.precision == TGL_BF16;
  const int tid = threadIdx.x;
  const int dm = P.d_model, H = P.n_heads, dh = dm / H;
  const int d_hs = P.d_hsrc, d_e = P.d_e, d_t = P.d_t;
  const int K = d_hs + d_e + d_t;
  const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;

  for (int j = tid; j < d_t; j += blockDim.x) {
    s_omega[j] = P.omega[j];
    s_phi[j] = P.phi[j];
  }
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
  const int rg = tid >> 4, cg = tid & 15;

  for (int64_t c0 = e_begin; c0 < e_end; c0 += kKvBM) {
    const int rows = (int)((e_end - c0) < kKvBM ? (e_end - c0) : kKvBM);
    // per-row gather descriptors
    if (tid < kKvBM) {
      const int r = tid;
      int ld = -1;
      if (r < rows) {
        const int64_t e = c0 + r;
        // local destination: the d with s_seg[d] <= e < s_seg[d+1]
        int lo = 0, hi = nd;  // invariant s_seg[lo] <= e < s_seg[hi]
        while (hi - lo > 1) {
          const int mid = (lo + hi) >> 1;
          if (s_seg[mid] <= e) lo = mid; else hi = mid;
        }
        ld = lo;
        const int64_t hr = a.hsrc_idx ? (int64_t)a.hsrc_idx[hoff + e] : hoff + e;
        s_hrow[r] = hr * a.ld_hsrc;
        s_erow[r] = d_e > 0 ? (int64_t)a.eid[e] * a.ld_e : 0;
        s_dt[r] = s_tdst[ld] - a.edge_t[e];  // fp32 delta (R18)
      }
      s_rdst[r] = ld;
    }
    __syncthreads();

    float acc[8][kKvTN];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int c = 0; c < kKvTN; ++c) acc[i][c] = 0.f;

    for (int k0 = 0; k0 < K; k0 += kKvBK) {
      {  // Z tile: thread -> row tid/2, cols (tid%2)*8 .. +7
        const int r = tid >> 1, kb = (tid & 1) * 8;
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int col = k0 + kb + u;
          float v = 0.f;
          if (r < rows && col < K) {
            if (col < d_hs) {
              v = __ldg(a.hsrc + s_hrow[r] + col);
            } else if (col < d_hs + d_e) {
              v = __ldg(a.efeat + s_erow[r] + (col - d_hs));
            } else {
              const int j = col - d_hs - d_e;
              const float dt = s_dt[r];
              const int64_t trow = tenc_table_row(dt, a.table, a.window);
              v = trow >= 0 ? __ldg(a.table + trow * d_t + j) : tenc_direct(dt, s_omega[j], s_phi[j]);
            }
          }
          As[kb + u][r] = maybe_bf16(v, bf16);
        }
      }
      if (tid < kKvBN) {  // W tile: Ws[kk][n] = W{k|v}[n][k0+kk]
        const int nn = tid;
        const float* wrow = nn < dm ? P.Wk + (int64_t)nn * K
                                    : (nn < 2 * dm ? P.Wv + (int64_t)(nn - dm) * K : nullptr);
#pragma unroll
        for (int kk = 0; kk < kKvBK; ++kk) {
          const int col = k0 + kk;
          Ws[kk][nn] = (wrow && col < K) ? maybe_bf16(__ldg(wrow + col), bf16) : 0.f;
        }
      }
      __syncthreads();
#pragma unroll 4
      for (int kk = 0; kk < kKvBK; ++kk) {
        const float4 x0 = *reinterpret_cast<const float4*>(&As[kk][rg * 8]);
        const float4 x1 = *reinterpret_cast<const float4*>(&As[kk][rg * 8 + 4]);
        const float av[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
        float b[kKvTN];
#pragma unroll
        for (int c = 0; c < kKvTN; ++c) b[c] = Ws[kk][cg + 16 * c];
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int c = 0; c < kKvTN; ++c) acc[i][c] = fmaf(av[i], b[c], acc[i][c]);
      }
      __syncthreads();
    }
    // bias
#pragma unroll
    for (int c = 0; c < kKvTN; ++c) {
      const int col = cg + 16 * c;
      const float bb = col < dm ? P.bk[col] : (col < 2 * dm ? P.bv[col - dm] : 0.f);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i][c] += bb;
    }
    // S10 logits: per row and head, <q_dst, k_row> over the head's channels
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = rg * 8 + i;
      const int ld = r < rows ? s_rdst[r] : -1;
      float p0 = 0.f, p1 = 0.f;
      if (ld >= 0) {
#pragma unroll
        for (int c = 0; c < kKvTN; ++c) {
          const int col = cg + 16 * c;
          if (col < dm) {
            const float pr = s_q[ld][col] * acc[i][c];
            if (col / dh == 0) p0 += pr; else p1 += pr;
          }
        }
      }
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) {
        p0 += __shfl_xor_sync(0xffffffffu, p0, o);
        p1 += __shfl_xor_sync(0xffffffffu, p1, o);
      }
      if (cg == 0 && ld >= 0) {
        float s0 = p0 * P.logit_scale, s1 = p1 * P.logit_scale;
        if (P.leaky_slope >= 0.f) {
          s0 = s0 < 0.f ? s0 * P.leaky_slope : s0;
          s1 = s1 < 0.f ? s1 * P.leaky_slope : s1;
        }
        s_logit[r][0] = s0;
        s_logit[r][1] = s1;
      }
    }
    __syncthreads();
    // S11 online segmented softmax statistics, one thread per (dst, head)
    if (tid < nd * H) {
      const int d = tid / H, h = tid % H;
      const int64_t a0 = s_seg[d] > c0 ? s_seg[d] : c0;
      const int64_t a1 = s_seg[d + 1] < c0 + rows ? s_seg[d + 1] : c0 + rows;
      float sc = 1.f;
      if (a0 < a1) {
        float mc = -INFINITY;
        for (int64_t e = a0; e < a1; ++e) mc = fmaxf(mc, s_logit[e - c0][h]);
        const float mo = s_m[d][h];
        const float mn = fmaxf(mo, mc);
        sc = (mo == -INFINITY) ? 0.f : expf(mo - mn);
        float l = s_l[d][h] * sc;
        for (int64_t e = a0; e < a1; ++e) {
          const float p = expf(s_logit[e - c0][h] - mn);
          s_p[e - c0][h] = p;
          l += p;
        }
        s_m[d][h] = mn;
        s_l[d][h] = l;
      }
      s_sc[d][h] = sc;
    }
    __syncthreads();
    for (int x = tid; x < nd * dm; x += blockDim.x) {
      const int d = x / dm, c = x % dm;
      s_r[d][c] *= s_sc[d][c / dh];
    }
    __syncthreads();
    // S12 scatter-sum of p * v into the destination accumulators
#pragma unroll
    for (int c = 0; c < kKvTN; ++c) {
      const int col = cg + 16 * c;
      if (col < dm || col >= 2 * dm) continue;
      const int cv = col - dm, h = cv / dh;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = rg * 8 + i;
        if (r < rows) atomicAdd(&s_r[s_rdst[r]][cv], s_p[r][h] * acc[i][c]);
      }
    }
    __syncthreads();
  }
  // normalise; empty segment -> 0 (R19)
  for (int x = tid; x < nd * dm; x += blockDim.x) {
    const int d = x / dm, c = x % dm;
    const float l = s_l[d][c / dh];
    a.rbuf[(d0 + d) * kQLd + c] = l > 0.f ? s_r[d][c] / l : 0.f;
  }
}

// tensor-core implementation (attn_tc.cu)
size_t tc_attn_ws_bytes(const tgl_attn_params* P, int64_t n_dst_max, size_t* o_q, size_t* o_r,
                        size_t* o_pack);
bool tc_attn_supported(const tgl_attn_params* P);
tgl_status tc_attn_launch(const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev,
                          const int64_t* seg_ptr, const float* dst_t, const float* hdst,
                          const int32_t* hdst_idx, int64_t ld_hdst, const float* hsrc,
                          const int32_t* hsrc_idx, const int64_t* hsrc_off_dev, int64_t ld_hsrc,
                          const float* efeat, const int32_t* eid, int64_t ld_e,
                          const float* edge_t, const float* table, int64_t window,
                          int32_t max_seg, float* out, void* ws, cudaStream_t s);

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_tblock_attn(const tgl_attn_params* P, int64_t n_dst_max,
                                      const int64_t* n_dst_dev, const int64_t* seg_ptr,
                                      const float* dst_t, const float* hdst,
                                      const int32_t* hdst_idx, int64_t ld_hdst, const float* hsrc,
                                      const int32_t* hsrc_idx, const int64_t* hsrc_off_dev,
                                      int64_t ld_hsrc, const float* efeat, const int32_t* eid,
                                      int64_t ld_e, const float* edge_t, const float* tenc_table,
                                      int64_t window, int32_t max_seg, float* out, void* ws,
                                      size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(P != nullptr, "null params");
  TGL_REQUIRE(n_dst_max >= 0, "negative n_dst_max");
  TGL_REQUIRE(P->n_heads > 0 && P->d_model > 0 && P->d_model % P->n_heads == 0,
              "d_model %% n_heads != 0");
  if (P->d_model > kMaxModel || P->d_out != P->d_model || P->n_heads > 2 || P->d_t > 256 ||
      P->d_t <= 0 || P->d_hdst < 0 || P->d_hsrc < 0 || P->d_e < 0) {
    set_error("unsupported shape: need d_out == d_model <= %d, n_heads <= 2, 0 < d_t <= 256",
              kMaxModel);
    return TGL_EUNSUPPORTED;
  }
  TGL_REQUIRE(P->precision == TGL_FP32 || P->precision == TGL_BF16 ||
                  P->precision == TGL_FP32_SIMT,
              "unknown precision");
  const bool use_tc = P->precision != TGL_FP32_SIMT;
  if (!use_tc && P->input_layout != 0) {
    set_error("split16 inputs (input_layout) feed the tensor-core path only");
    return TGL_EUNSUPPORTED;
  }
  if (use_tc && !tc_attn_supported(P)) {
    set_error("tensor-core path needs d_model == d_out == 100 (use TGL_FP32_SIMT otherwise)");
    return TGL_EUNSUPPORTED;
  }
  WsLayout L;
  const int64_t nrows = n_dst_max > 0 ? n_dst_max : 1;
  const size_t o_q = L.take(sizeof(float) * kQLd * nrows);
  const size_t o_r = L.take(sizeof(float) * kQLd * nrows);
  size_t need = L.off;
  if (use_tc) {
    size_t a0, a1, a2;
    need = tc_attn_ws_bytes(P, n_dst_max, &a0, &a1, &a2);
  }
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, need, &query));
  if (query) return TGL_OK;
  if (n_dst_max == 0) return TGL_OK;
  TGL_REQUIRE(seg_ptr && dst_t && hdst && hsrc && edge_t && out, "null pointer");
  TGL_REQUIRE(P->Wq && P->bq && P->Wk && P->bk && P->Wv && P->bv && P->Wo && P->bo &&
                  P->ln_gamma && P->ln_beta && P->omega && P->phi,
              "null weight");
  TGL_REQUIRE(P->d_e == 0 || (efeat && eid), "null efeat/eid with d_e > 0");
  TGL_REQUIRE(ld_hdst >= P->d_hdst && ld_hsrc >= P->d_hsrc && ld_e >= P->d_e, "bad leading dim");
  AttnArgs a;
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
  a.table = window > 0 ? tenc_table : nullptr;
  a.window = window;
  a.out = out;
  char* w = static_cast<char*>(ws);
  a.qbuf = reinterpret_cast<float*>(w + o_q);
  a.rbuf = reinterpret_cast<float*>(w + o_r);
  int ms = max_seg > 0 ? max_seg : 1;
  int dpb = kKvBM / ms;
  a.dpb = dpb < 1 ? 1 : (dpb > kMaxDpb ? kMaxDpb : dpb);
  cudaStream_t s = as_stream(stream);
  if (use_tc)
    return tc_attn_launch(P, n_dst_max, n_dst_dev, seg_ptr, dst_t, hdst, hdst_idx, ld_hdst, hsrc,
                          hsrc_idx, hsrc_off_dev, ld_hsrc, efeat, eid, ld_e, edge_t,
                          a.table, window, max_seg, out, ws, s);
  const unsigned g64 = (unsigned)ceil_div(n_dst_max, kTBM);
  q_proj_kernel<<<g64, kAttnThreads, 0, s>>>(a);
  TGL_TRY(launch_check("q_proj"));
  tgl_kv_probe* probe = P->probe;
  if (probe) probe->kernel = TGL_KV_SIMT;
  if (probe && probe->ev_start)
    TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_start), s), "probe"));
  kv_attn_kernel<<<(unsigned)ceil_div(n_dst_max, a.dpb), kAttnThreads, 0, s>>>(a);
  TGL_TRY(launch_check("kv_attn"));
  if (probe && probe->ev_stop)
    TGL_TRY(cuda_check(cudaEventRecord(static_cast<cudaEvent_t>(probe->ev_stop), s), "probe"));
  out_ffn_kernel<<<g64, kAttnThreads, 0, s>>>(a);
  return launch_check("out_ffn");
}
