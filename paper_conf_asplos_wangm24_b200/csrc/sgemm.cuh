// sgemm.cuh -- a strided fp32 SIMT GEMM (64x64 tiles, exact fp32 products, fp32
// accumulation) for the small training-side GEMMs (N2 backward, N3 GRU memory update):
// tens of MFLOP per call, where a tensor-core kernel's split-precision passes and setup
// would not pay.
#pragma once
#include "common.cuh"

namespace tgl {

// ------------------------------------------------------------------ strided SGEMM
// C[m][n] = alpha * sum_k A(m, k) B(k, n) + beta * C[m][n], A(m,k) = A[m*sam + k*sak],
// B(k,n) = B[k*sbk + n*sbn], C row-major (ldc).
constexpr int kGB = 64, kGK = 16;
static __global__ void __launch_bounds__(256)
sgemm_kernel(int64_t M, int64_t N, int64_t K, float alpha, const float* __restrict__ A,
             int64_t sam, int64_t sak, const float* __restrict__ B, int64_t sbk, int64_t sbn,
             float beta, float* __restrict__ C, int64_t ldc) {
  __shared__ float As[kGK][kGB + 1];
  __shared__ float Bs[kGK][kGB + 1];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int64_t m0 = (int64_t)blockIdx.y * kGB, n0 = (int64_t)blockIdx.x * kGB;
  float acc[4][4] = {};
  for (int64_t k0 = 0; k0 < K; k0 += kGK) {
    for (int x = threadIdx.x; x < kGK * kGB; x += 256) {
      const int kk = x / kGB, mm = x % kGB;
      const int64_t gm = m0 + mm, gk = k0 + kk;
      As[kk][mm] = (gm < M && gk < K) ? A[gm * sam + gk * sak] : 0.f;
      const int64_t gn = n0 + mm;
      Bs[kk][mm] = (gn < N && gk < K) ? B[gk * sbk + gn * sbn] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < kGK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        a[u] = As[kk][ty * 4 + u];
        b[u] = Bs[kk][tx * 4 + u];
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(a[u], b[v], acc[u][v]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int64_t gm = m0 + ty * 4 + u;
    if (gm >= M) continue;
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int64_t gn = n0 + tx * 4 + v;
      if (gn >= N) continue;
      float* c = C + gm * ldc + gn;
      *c = alpha * acc[u][v] + (beta != 0.f ? beta * *c : 0.f);
    }
  }
}

static cudaError_t sgemm(cudaStream_t s, int64_t M, int64_t N, int64_t K, const float* A,
                         int64_t sam, int64_t sak, const float* B, int64_t sbk, int64_t sbn,
                         float beta, float* C, int64_t ldc) {
  if (M <= 0 || N <= 0) return cudaSuccess;
  dim3 grid((unsigned)ceil_div(N, kGB), (unsigned)ceil_div(M, kGB));
  sgemm_kernel<<<grid, 256, 0, s>>>(M, N, K, 1.f, A, sam, sak, B, sbk, sbn, beta, C, ldc);
  return cudaGetLastError();
}

}  // namespace tgl
