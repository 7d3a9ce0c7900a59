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

// Phi inside the fused attention kernels, where the contract is the 1e-3 embedding
// tolerance (not the 2-ulp contract of tgl_time_encode): the same fp32 argument
// b = fl(fl(omega*dt) + phi) (R10), reduced modulo 2*pi with two FMA Cody-Waite
// steps (C1 = fl32(2 pi), C2 = fl32(2 pi - C1); k*C1 is exact inside the FMA), then
// the SFU cosine (cos.approx, abs error 2^-20.5 on |x| <= 100 pi).  |error| < 2e-6 for
// |b| < 1e9, i.e. below the bf16 hi/lo operand split it feeds (2^-17); larger |b|
// take the accurate cosf.  Accurate cosf falls back to Payne-Hanek reduction for
// |b| > 105615 (REDDIT/LASTFM Delta t reach 1e6-1e8 with omega_0 = 1), which costs
// hundreds of instructions and local memory per element.
static __device__ __noinline__ float tenc_cos_slow(float b) { return cosf(b); }

// the reduction + SFU cosine alone (valid for |b| < 1e9; callers check)
__device__ __forceinline__ float tenc_cos_reduced(float b) {
  const float k = rintf(b * 0.159154943091895336f);
  float r = fmaf(-k, 6.28318548202514648f, b);
  r = fmaf(-k, -1.74845560007449713e-7f, r);
  return __cosf(r);
}

__device__ __forceinline__ float tenc_cos_fast(float b) {
  // out of line: an inlined cosf would drag its Payne-Hanek path (local-memory table
  // walk) into every call site, predicated on in the steady state
  if (!(fabsf(b) < 1e9f)) return tenc_cos_slow(b);
  const float k = rintf(b * 0.159154943091895336f);
  float r = fmaf(-k, 6.28318548202514648f, b);
  r = fmaf(-k, -1.74845560007449713e-7f, r);
  return __cosf(r);
}

__device__ __forceinline__ float tenc_fast(float dt, float omega, float phi) {
  return tenc_cos_fast(__fadd_rn(__fmul_rn(omega, dt), phi));
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
