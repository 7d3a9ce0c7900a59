// tenc.cuh -- the time encoder Phi_j(dt) = cos(omega_j * dt + phi_j), eq (8) P:126,
// evaluated like the paper's fp32 code `torch.cos(ts * w + b)` (reading R10):
// round-to-nearest fp32 multiply, round-to-nearest fp32 add (no FMA contraction),
// then an accurate cosine of that fp32 argument (this file must not be built with
// fast-math).
#pragma once
#include "common.cuh"

namespace tgl {

__device__ __forceinline__ float tenc_direct(float dt, float omega, float phi) {
  return cosf(__fadd_rn(__fmul_rn(omega, dt), phi));
}

// Row index into the precompute table when dt is an integer in [0, window), else -1
// (reading R11).  Table rows were produced by tenc_direct((float)d, ...), so the
// table value equals the direct value bit for bit.
__device__ __forceinline__ int64_t tenc_table_row(float dt, const float* table, int64_t window) {
  if (table == nullptr) return -1;
  if (!(dt >= 0.0f) || !(dt < (float)window)) return -1;
  float f = truncf(dt);
  if (f != dt) return -1;
  return (int64_t)f;
}

}  // namespace tgl
