// attn_bwd.cu -- §8(f) N2: backward of one TBlock attention layer (training; the paper's
// headline workload, whose Fig 7 times the backward).
//
// Forward (eqs 4-7; Listing 2) recomputed in fp32, then the chain
// rule in reverse order (oracle: oracle/backward.py):
//   materialise  Zq = [h_i ; Phi(0)], Ze = [h_src(e) ; e_e ; Phi(dt_e)]      (gathers, R10)
//   GEMM         Q = Zq Wq^T + bq,  KV = Ze [Wk ; Wv]^T                     (S8, S9)
//   per dst      logits, segment softmax, r = sum alpha v  -> Zo = [r ; h]   (S10-S12)
//   GEMM         Y = Zo Wo^T
//   per dst      ReLU + LayerNorm forward and backward -> dY, dgamma, dbeta  (S13)
//   GEMM         dWo += dY^T Zo,  dZo = dY Wo
//   per dst      weighted-sum / softmax / LeakyReLU / logit backward -> dK|dV, dQ
//   GEMM         d[Wk;Wv] += d[K|V]^T Ze,  dZe = dK Wk + dV Wv,  dWq += dQ^T Zq,  dZq = dQ Wq
//   per edge     dh_src rows (scatter-add), domega, dphi (time encoder: -sin(b) dt, -sin(b))
//   per dst      dh_dst rows (scatter-add), dphi of Phi(0)
// The GEMMs are a strided fp32 SIMT kernel (64x64 tiles, exact fp32 products, fp32
// accumulation); reductions over rows use per-thread partial sums and one atomicAdd per
// thread, so gradients are reproducible to fp32 summation order.  Data-dependent sizes
// stay on the device: the GEMMs run over the host bounds (n_dst_max, n_edges_max) on
// zero-padded rows, which contribute nothing.
#include "common.cuh"
#include "sgemm.cuh"
#include "tenc.cuh"

namespace tgl {
namespace bwd {

constexpr int kDm = 128;      // d_model limit (2 heads)

// column sums out[c] += sum_r X[r][c] (rows < n_rows)
__global__ void colsum_kernel(int64_t rows, int cols, const float* __restrict__ X, int64_t ld,
                              float* __restrict__ out) {
  for (int c = threadIdx.x; c < cols; c += blockDim.x) {
    float acc = 0.f;
    for (int64_t r = blockIdx.x; r < rows; r += gridDim.x) acc += X[r * ld + c];
    atomicAdd(out + c, acc);
  }
}

struct BArgs {
  tgl_attn_params P;
  int64_t n_max, e_max;
  const int64_t* n_dev;
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
  const float* gout;
  int64_t ld_gout;
  tgl_attn_grads G;
  float* ghdst;
  int64_t ld_ghdst;
  float* ghsrc;
  int64_t ld_ghsrc;
  // workspace (row-major fp32)
  float *Zq, *Q, *Ze, *KV, *DT, *U, *A, *Zo, *Y, *GY, *GZo, *GA, *GKV, *GQ, *GZe, *GZq;
  int kq, ke, ko;
};

__device__ __forceinline__ int64_t n_of(const BArgs& a) { return dev_count(a.n_dev, a.n_max); }

// ---- 1. gathers: Zq, Zo[:, dm:], Ze, DT (warp per destination)
__global__ void bw_gather_kernel(BArgs a) {
  const tgl_attn_params& P = a.P;
  const int lane = threadIdx.x & 31;
  const int64_t n = n_of(a);
  const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
  const int dm = P.d_model;
  for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < n;
       i += (int64_t)gridDim.x * (blockDim.x >> 5)) {
    const int64_t row = a.hdst_idx ? a.hdst_idx[i] : i;
    const float* h = a.hdst + row * a.ld_hdst;
    for (int c = lane; c < P.d_hdst; c += 32) {
      a.Zq[i * a.kq + c] = h[c];
      a.Zo[i * a.ko + dm + c] = h[c];
    }
    for (int j = lane; j < P.d_t; j += 32)
      a.Zq[i * a.kq + P.d_hdst + j] = tenc_direct(0.f, P.omega[j], P.phi[j]);
    const int64_t e0 = a.seg_ptr[i], e1 = a.seg_ptr[i + 1];
    const float td = a.dst_t[i];
    for (int64_t e = e0; e < e1; ++e) {
      const int64_t hr = a.hsrc_idx ? a.hsrc_idx[hoff + e] : hoff + e;
      const float* hs = a.hsrc + hr * a.ld_hsrc;
      float* z = a.Ze + e * a.ke;
      for (int c = lane; c < P.d_hsrc; c += 32) z[c] = hs[c];
      if (P.d_e > 0) {
        const float* ef = a.efeat + (int64_t)a.eid[e] * a.ld_e;
        for (int c = lane; c < P.d_e; c += 32) z[P.d_hsrc + c] = ef[c];
      }
      const float dt = td - a.edge_t[e];                   // fp32 delta (R18)
      for (int j = lane; j < P.d_t; j += 32)
        z[P.d_hsrc + P.d_e + j] = tenc_direct(dt, P.omega[j], P.phi[j]);
      if (lane == 0) a.DT[e] = dt;
    }
  }
}

// ---- 2. attention forward per destination: logits U, alpha A, r -> Zo[:, :dm]
__global__ void bw_attn_fwd_kernel(BArgs a) {
  const tgl_attn_params& P = a.P;
  const int lane = threadIdx.x & 31;
  const int64_t n = n_of(a);
  const int dm = P.d_model, H = P.n_heads, dh = dm / H;
  for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < n;
       i += (int64_t)gridDim.x * (blockDim.x >> 5)) {
    float* qw = a.Q + i * dm;
    for (int c = lane; c < dm; c += 32) qw[c] += P.bq[c];   // q = Zq Wq^T + bq (eq 4)
    __syncwarp();
    const float* q = qw;
    const int64_t e0 = a.seg_ptr[i], e1 = a.seg_ptr[i + 1];
    for (int64_t e = e0; e < e1; ++e) {                    // logits (lanes over columns)
      const float* kv = a.KV + e * 2 * dm;
      float p[2] = {0.f, 0.f};
      for (int c = lane; c < dm; c += 32) p[c / dh] = fmaf(q[c], kv[c] + P.bk[c], p[c / dh]);
      for (int h = 0; h < H; ++h) {
        float u = warp_sum(p[h]) * P.logit_scale;
        if (lane == 0) a.U[e * 2 + h] = u;
      }
    }
    __syncwarp();
    for (int h = 0; h < H; ++h) {                          // segment softmax
      float mx = -INFINITY;
      for (int64_t e = e0 + lane; e < e1; e += 32) {
        float u = a.U[e * 2 + h];
        const float s = (P.leaky_slope >= 0.f && u < 0.f) ? u * P.leaky_slope : u;
        mx = fmaxf(mx, s);
      }
      for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
      float den = 0.f;
      for (int64_t e = e0 + lane; e < e1; e += 32) {
        float u = a.U[e * 2 + h];
        const float s = (P.leaky_slope >= 0.f && u < 0.f) ? u * P.leaky_slope : u;
        den += expf(s - mx);
      }
      den = warp_sum(den);
      for (int64_t e = e0 + lane; e < e1; e += 32) {
        float u = a.U[e * 2 + h];
        const float s = (P.leaky_slope >= 0.f && u < 0.f) ? u * P.leaky_slope : u;
        a.A[e * 2 + h] = expf(s - mx) / den;
      }
    }
    __syncwarp();
    for (int c = lane; c < dm; c += 32) {                  // r = sum alpha (v + bv)
      float r = 0.f;
      for (int64_t e = e0; e < e1; ++e)
        r = fmaf(a.A[e * 2 + c / dh], a.KV[e * 2 * dm + dm + c] + P.bv[c], r);
      a.Zo[i * a.ko + c] = r;                              // 0 for an empty segment (R19)
    }
  }
}

// ---- 3. ReLU + LayerNorm forward and backward per destination -> GY, dgamma, dbeta
__global__ void bw_ln_kernel(BArgs a) {
  const tgl_attn_params& P = a.P;
  const int lane = threadIdx.x & 31;
  const int64_t n = n_of(a);
  const int D = P.d_out;
  float pg[kDm / 32] = {}, pb[kDm / 32] = {};             // per-lane dgamma / dbeta partials
  for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < n;
       i += (int64_t)gridDim.x * (blockDim.x >> 5)) {
    float y[kDm / 32], av[kDm / 32], g[kDm / 32];
    float s1 = 0.f;
#pragma unroll
    for (int u = 0; u < kDm / 32; ++u) {
      const int c = lane + 32 * u;
      y[u] = c < D ? a.Y[i * D + c] + P.bo[c] : 0.f;
      av[u] = c < D ? fmaxf(y[u], 0.f) : 0.f;
      g[u] = c < D ? a.gout[i * a.ld_gout + c] : 0.f;
      s1 += av[u];
    }
    const float mean = warp_sum(s1) / D;
    float s2 = 0.f;
#pragma unroll
    for (int u = 0; u < kDm / 32; ++u) {
      const int c = lane + 32 * u;
      if (c < D) s2 += (av[u] - mean) * (av[u] - mean);
    }
    const float var = warp_sum(s2) / D;
    const float sig = sqrtf(var + P.ln_eps);
    float m1 = 0.f, m2 = 0.f, xh[kDm / 32], gx[kDm / 32];
#pragma unroll
    for (int u = 0; u < kDm / 32; ++u) {
      const int c = lane + 32 * u;
      xh[u] = c < D ? (av[u] - mean) / sig : 0.f;
      gx[u] = c < D ? g[u] * P.ln_gamma[c] : 0.f;
      pg[u] += g[u] * xh[u];
      pb[u] += g[u];
      m1 += gx[u];
      m2 += gx[u] * xh[u];
    }
    m1 = warp_sum(m1) / D;
    m2 = warp_sum(m2) / D;
#pragma unroll
    for (int u = 0; u < kDm / 32; ++u) {
      const int c = lane + 32 * u;
      if (c < D) {
        const float ga = (gx[u] - m1 - xh[u] * m2) / sig;
        a.GY[i * D + c] = y[u] > 0.f ? ga : 0.f;
      }
    }
  }
#pragma unroll
  for (int u = 0; u < kDm / 32; ++u) {
    const int c = lane + 32 * u;
    if (c < D) {
      atomicAdd(a.G.dgamma + c, pg[u]);
      atomicAdd(a.G.dbeta + c, pb[u]);
    }
  }
}

// ---- 4. attention backward per destination: d[K|V] rows, dQ rows
__global__ void bw_attn_bwd_kernel(BArgs a) {
  const tgl_attn_params& P = a.P;
  const int lane = threadIdx.x & 31;
  const int64_t n = n_of(a);
  const int dm = P.d_model, H = P.n_heads, dh = dm / H;
  for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < n;
       i += (int64_t)gridDim.x * (blockDim.x >> 5)) {
    const float* gr = a.GZo + i * a.ko;                    // dr = dZo[:, :dm]
    const float* q = a.Q + i * dm;
    const int64_t e0 = a.seg_ptr[i], e1 = a.seg_ptr[i + 1];
    float sa[2] = {0.f, 0.f};                              // sum_e alpha dalpha per head
    for (int64_t e = e0; e < e1; ++e) {
      const float* kv = a.KV + e * 2 * dm;
      float p[2] = {0.f, 0.f};
      for (int c = lane; c < dm; c += 32) p[c / dh] = fmaf(gr[c], kv[dm + c] + P.bv[c], p[c / dh]);
      for (int h = 0; h < H; ++h) {
        const float ga = warp_sum(p[h]);
        if (lane == 0) a.GA[e * 2 + h] = ga;
        sa[h] += a.A[e * 2 + h] * ga;
      }
    }
    __syncwarp();
    float gq[kDm / 32] = {};
    for (int64_t e = e0; e < e1; ++e) {
      float gu[2];
      for (int h = 0; h < H; ++h) {
        const float al = a.A[e * 2 + h];
        const float gs = al * (a.GA[e * 2 + h] - sa[h]);  // softmax backward
        const float u = a.U[e * 2 + h];
        gu[h] = (P.leaky_slope >= 0.f && u < 0.f) ? gs * P.leaky_slope : gs;
      }
      const float* kv = a.KV + e * 2 * dm;
      float* gkv = a.GKV + e * 2 * dm;
#pragma unroll
      for (int u = 0; u < kDm / 32; ++u) {
        const int c = lane + 32 * u;
        if (c < dm) {
          const int h = c / dh;
          const float g = gu[h] * P.logit_scale;
          gkv[c] = g * q[c];                               // dK
          gkv[dm + c] = a.A[e * 2 + h] * gr[c];            // dV
          gq[u] = fmaf(g, kv[c] + P.bk[c], gq[u]);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < kDm / 32; ++u) {
      const int c = lane + 32 * u;
      if (c < dm) a.GQ[i * dm + c] = gq[u];
    }
  }
}

// ---- 5. per-edge input / time-encoder gradients: dh_src rows, domega, dphi
__global__ void bw_edge_kernel(BArgs a, int64_t e_total_max) {
  const tgl_attn_params& P = a.P;
  const int64_t n = n_of(a);
  const int64_t E = a.seg_ptr[n];
  const int64_t hoff = a.hsrc_off_dev ? *a.hsrc_off_dev : 0;
  const int kt = P.d_hsrc + P.d_e;
  (void)e_total_max;
  // time encoder: thread j of the block owns column j; partial sums over the block's edges
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    float pw = 0.f, pp = 0.f;
    for (int64_t e = blockIdx.x; e < E; e += gridDim.x) {
      const float dt = a.DT[e];
      const float b = __fadd_rn(__fmul_rn(P.omega[j], dt), P.phi[j]);   // R10 argument
      const float gphi = a.GZe[e * a.ke + kt + j] * -sinf(b);
      pw = fmaf(gphi, dt, pw);
      pp += gphi;
    }
    atomicAdd(a.G.domega + j, pw);
    atomicAdd(a.G.dphi + j, pp);
  }
  if (a.ghsrc != nullptr) {
    for (int64_t e = blockIdx.x; e < E; e += gridDim.x) {
      const int64_t hr = a.hsrc_idx ? a.hsrc_idx[hoff + e] : hoff + e;
      for (int c = threadIdx.x; c < P.d_hsrc; c += blockDim.x)
        atomicAdd(a.ghsrc + hr * a.ld_ghsrc + c, a.GZe[e * a.ke + c]);
    }
  }
}

// ---- 6. per-destination: dh_dst rows (FFN + Q paths), dphi of Phi(0)
__global__ void bw_dst_kernel(BArgs a) {
  const tgl_attn_params& P = a.P;
  const int64_t n = n_of(a);
  const int dm = P.d_model;
  for (int j = threadIdx.x; j < P.d_t; j += blockDim.x) {
    float pp = 0.f;
    const float s0 = -sinf(P.phi[j]);                      // b = fl(omega * 0 + phi) = phi
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) pp += a.GZq[i * a.kq + P.d_hdst + j];
    atomicAdd(a.G.dphi + j, pp * s0);
  }
  if (a.ghdst != nullptr) {
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) {
      const int64_t row = a.hdst_idx ? a.hdst_idx[i] : i;
      for (int c = threadIdx.x; c < P.d_hdst; c += blockDim.x)
        atomicAdd(a.ghdst + row * a.ld_ghdst + c, a.GZo[i * a.ko + dm + c] + a.GZq[i * a.kq + c]);
    }
  }
}

}  // namespace bwd
}  // namespace tgl

using namespace tgl;
using namespace tgl::bwd;

extern "C" tgl_status tgl_tblock_attn_backward(
    const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev, int64_t n_edges_max,
    const int64_t* seg_ptr, const float* dst_t, const float* hdst, const int32_t* hdst_idx,
    int64_t ld_hdst, const float* hsrc, const int32_t* hsrc_idx, const int64_t* hsrc_off_dev,
    int64_t ld_hsrc, const float* efeat, const int32_t* eid, int64_t ld_e, const float* edge_t,
    const float* grad_out, int64_t ld_gout, const tgl_attn_grads* G, float* grad_hdst,
    int64_t ld_ghdst, float* grad_hsrc, int64_t ld_ghsrc, void* ws, size_t* ws_bytes,
    void* stream) {
  TGL_REQUIRE(P != nullptr && G != nullptr, "null params / grads");
  TGL_REQUIRE(n_dst_max >= 0 && n_edges_max >= 0, "negative size");
  TGL_REQUIRE(P->n_heads >= 1 && P->n_heads <= 2 && P->d_model % P->n_heads == 0 &&
                  P->d_model <= kDm && P->d_out == P->d_model,
              "backward needs d_out == d_model <= %d, 1-2 heads", kDm);
  const int64_t n1 = n_dst_max > 0 ? n_dst_max : 1, e1 = n_edges_max > 0 ? n_edges_max : 1;
  const int kq = P->d_hdst + P->d_t, ke = P->d_hsrc + P->d_e + P->d_t, ko = P->d_model + P->d_hdst;
  const int dm = P->d_model;
  WsLayout L;
  const size_t oZq = L.take(4 * n1 * kq), oQ = L.take(4 * n1 * dm), oZe = L.take(4 * e1 * ke),
               oKV = L.take(4 * e1 * 2 * dm), oDT = L.take(4 * e1), oU = L.take(8 * e1),
               oA = L.take(8 * e1), oZo = L.take(4 * n1 * ko), oY = L.take(4 * n1 * dm),
               oGY = L.take(4 * n1 * dm), oGZo = L.take(4 * n1 * ko), oGA = L.take(8 * e1),
               oGKV = L.take(4 * e1 * 2 * dm), oGQ = L.take(4 * n1 * dm),
               oGZe = L.take(4 * e1 * ke), oGZq = L.take(4 * n1 * kq);
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  if (n_dst_max == 0) return TGL_OK;
  TGL_REQUIRE(seg_ptr && dst_t && hdst && hsrc && edge_t && grad_out, "null pointer");
  TGL_REQUIRE(P->d_e == 0 || (efeat && eid), "null efeat / eid with d_e > 0");
  TGL_REQUIRE(G->dWq && G->dbq && G->dWk && G->dbk && G->dWv && G->dbv && G->dWo && G->dbo &&
                  G->dgamma && G->dbeta && G->domega && G->dphi,
              "null gradient buffer");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  // zero-padded rows beyond the device counts must contribute nothing to the GEMMs
  TGL_TRY(cuda_check(cudaMemsetAsync(w, 0, L.off, s), "backward workspace memset"));
  BArgs a;
  a.P = *P;
  a.n_max = n_dst_max;
  a.e_max = n_edges_max;
  a.n_dev = n_dst_dev;
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
  a.gout = grad_out;
  a.ld_gout = ld_gout;
  a.G = *G;
  a.ghdst = grad_hdst;
  a.ld_ghdst = ld_ghdst;
  a.ghsrc = grad_hsrc;
  a.ld_ghsrc = ld_ghsrc;
  auto F = [&](size_t o) { return reinterpret_cast<float*>(w + o); };
  a.Zq = F(oZq); a.Q = F(oQ); a.Ze = F(oZe); a.KV = F(oKV); a.DT = F(oDT); a.U = F(oU);
  a.A = F(oA); a.Zo = F(oZo); a.Y = F(oY); a.GY = F(oGY); a.GZo = F(oGZo); a.GA = F(oGA);
  a.GKV = F(oGKV); a.GQ = F(oGQ); a.GZe = F(oGZe); a.GZq = F(oGZq);
  a.kq = kq; a.ke = ke; a.ko = ko;
  const int64_t N = n_dst_max, E = n_edges_max;
  const unsigned gw = (unsigned)(ceil_div(N, 8) < kNumSMs * 8 ? ceil_div(N, 8) : kNumSMs * 8);
  const unsigned gr = (unsigned)(kNumSMs * 4);
  bw_gather_kernel<<<gw, 256, 0, s>>>(a);
  TGL_TRY(launch_check("bw_gather"));
  // forward GEMMs (fp32): Q = Zq Wq^T (bq added per row), K|V = Ze [Wk ; Wv]^T, Y = Zo Wo^T
  TGL_TRY(cuda_check(sgemm(s, N, dm, kq, a.Zq, kq, 1, P->Wq, 1, kq, 0.f, a.Q, dm), "gemm Q"));
  TGL_TRY(cuda_check(sgemm(s, E, dm, ke, a.Ze, ke, 1, P->Wk, 1, ke, 0.f, a.KV, 2 * dm), "gemm K"));
  TGL_TRY(cuda_check(sgemm(s, E, dm, ke, a.Ze, ke, 1, P->Wv, 1, ke, 0.f, a.KV + dm, 2 * dm),
                     "gemm V"));
  bw_attn_fwd_kernel<<<gw, 256, 0, s>>>(a);
  TGL_TRY(launch_check("bw_attn_fwd"));
  TGL_TRY(cuda_check(sgemm(s, N, dm, ko, a.Zo, ko, 1, P->Wo, 1, ko, 0.f, a.Y, dm), "gemm Y"));
  bw_ln_kernel<<<gw, 256, 0, s>>>(a);
  TGL_TRY(launch_check("bw_ln"));
  // output projection: dWo += dY^T Zo, dbo += colsum dY, dZo = dY Wo
  TGL_TRY(cuda_check(sgemm(s, dm, ko, N, a.GY, 1, dm, a.Zo, ko, 1, 1.f, G->dWo, ko), "gemm dWo"));
  colsum_kernel<<<gr, 128, 0, s>>>(N, dm, a.GY, dm, G->dbo);
  TGL_TRY(launch_check("colsum dbo"));
  TGL_TRY(cuda_check(sgemm(s, N, ko, dm, a.GY, dm, 1, P->Wo, ko, 1, 0.f, a.GZo, ko), "gemm dZo"));
  bw_attn_bwd_kernel<<<gw, 256, 0, s>>>(a);
  TGL_TRY(launch_check("bw_attn_bwd"));
  // K / V projections: dWk += dK^T Ze, dWv += dV^T Ze, dbk / dbv, dZe = dK Wk + dV Wv
  TGL_TRY(cuda_check(sgemm(s, dm, ke, E, a.GKV, 1, 2 * dm, a.Ze, ke, 1, 1.f, G->dWk, ke),
                     "gemm dWk"));
  TGL_TRY(cuda_check(sgemm(s, dm, ke, E, a.GKV + dm, 1, 2 * dm, a.Ze, ke, 1, 1.f, G->dWv, ke),
                     "gemm dWv"));
  colsum_kernel<<<gr, 128, 0, s>>>(E, dm, a.GKV, 2 * dm, G->dbk);
  colsum_kernel<<<gr, 128, 0, s>>>(E, dm, a.GKV + dm, 2 * dm, G->dbv);
  TGL_TRY(launch_check("colsum dbk/dbv"));
  TGL_TRY(cuda_check(sgemm(s, E, ke, dm, a.GKV, 2 * dm, 1, P->Wk, ke, 1, 0.f, a.GZe, ke),
                     "gemm dZe (K)"));
  TGL_TRY(cuda_check(sgemm(s, E, ke, dm, a.GKV + dm, 2 * dm, 1, P->Wv, ke, 1, 1.f, a.GZe, ke),
                     "gemm dZe (V)"));
  bw_edge_kernel<<<gr, 128, 0, s>>>(a, E);
  TGL_TRY(launch_check("bw_edge"));
  // query projection: dWq += dQ^T Zq, dbq += colsum dQ, dZq = dQ Wq
  TGL_TRY(cuda_check(sgemm(s, dm, kq, N, a.GQ, 1, dm, a.Zq, kq, 1, 1.f, G->dWq, kq), "gemm dWq"));
  colsum_kernel<<<gr, 128, 0, s>>>(N, dm, a.GQ, dm, G->dbq);
  TGL_TRY(launch_check("colsum dbq"));
  TGL_TRY(cuda_check(sgemm(s, N, kq, dm, a.GQ, dm, 1, P->Wq, kq, 1, 0.f, a.GZq, kq), "gemm dZq"));
  bw_dst_kernel<<<gr, 128, 0, s>>>(a);
  return launch_check("bw_dst");
}
