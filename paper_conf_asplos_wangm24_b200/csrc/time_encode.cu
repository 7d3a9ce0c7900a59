// time_encode.cu -- S6: tgl_time_precompute / tgl_time_encode (eq 8).
// HBM-bound elementwise kernels: one thread per output element, j fastest so the
// d_t-wide rows are written with coalesced stores; omega/phi are read through L1.
#include "common.cuh"
#include "tenc.cuh"

namespace tgl {

__global__ void time_precompute_kernel(int64_t window, int32_t d_t,
                                       const float* __restrict__ omega,
                                       const float* __restrict__ phi, float* __restrict__ table) {
  int64_t total = window * d_t;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    int64_t d = x / d_t;
    int j = (int)(x - d * d_t);
    table[x] = tenc_direct((float)d, omega[j], phi[j]);
  }
}

__global__ void time_encode_kernel(int64_t n, const float* __restrict__ dt, int32_t d_t,
                                   const float* __restrict__ omega, const float* __restrict__ phi,
                                   const float* __restrict__ table, int64_t window,
                                   float* __restrict__ out) {
  int64_t total = n * d_t;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    int64_t i = x / d_t;
    int j = (int)(x - i * d_t);
    float v = dt[i];
    int64_t row = tenc_table_row(v, table, window);
    out[x] = row >= 0 ? table[row * d_t + j] : tenc_direct(v, omega[j], phi[j]);
  }
}

static int grid_for(int64_t n, int threads) {
  int64_t g = ceil_div(n > 0 ? n : 1, threads);
  int64_t cap = (int64_t)kNumSMs * 16;
  return (int)(g < cap ? g : cap);
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_time_precompute(int64_t window, int32_t d_t, const float* omega,
                                          const float* phi, float* table, void* stream) {
  TGL_REQUIRE(window >= 0 && d_t > 0, "bad size");
  TGL_REQUIRE(omega && phi && (window == 0 || table), "null pointer");
  TGL_REQUIRE(window <= (int64_t)1 << 24, "window must be <= 2^24 (exact fp32 integers)");
  if (window == 0) return TGL_OK;
  time_precompute_kernel<<<grid_for(window * d_t, 256), 256, 0, as_stream(stream)>>>(
      window, d_t, omega, phi, table);
  return launch_check("time_precompute");
}

extern "C" tgl_status tgl_time_encode(int64_t n, const float* dt, int32_t d_t, const float* omega,
                                      const float* phi, const float* table, int64_t window,
                                      float* out, void* stream) {
  TGL_REQUIRE(n >= 0 && d_t > 0 && window >= 0, "bad size");
  TGL_REQUIRE(omega && phi, "null pointer");
  if (n == 0) return TGL_OK;
  TGL_REQUIRE(dt && out, "null pointer");
  time_encode_kernel<<<grid_for(n * d_t, 256), 256, 0, as_stream(stream)>>>(
      n, dt, d_t, omega, phi, window > 0 ? table : nullptr, window, out);
  return launch_check("time_encode");
}
