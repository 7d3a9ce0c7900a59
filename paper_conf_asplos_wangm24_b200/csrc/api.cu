// api.cu -- error reporting, version, and the small S2/S5/S14 kernels.
#include <stdarg.h>
#include <string.h>

#include <cuda_bf16.h>

#include "common.cuh"

namespace tgl {

static thread_local char g_last_error[512] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_last_error, sizeof(g_last_error), fmt, ap);
  va_end(ap);
}

tgl_status cuda_check(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return TGL_OK;
  set_error("%s: %s", what, cudaGetErrorString(e));
  return TGL_ECUDA;
}

tgl_status launch_check(const char* what) { return cuda_check(cudaGetLastError(), what); }

// ---------------------------------------------------------------- S2 roots
__global__ void batch_roots_kernel(int64_t batch, int64_t num_edges, const int64_t* start_dev,
                                   const int32_t* __restrict__ src, const int32_t* __restrict__ dst,
                                   const float* __restrict__ t, const int32_t* __restrict__ neg,
                                   int32_t* __restrict__ qnode, float* __restrict__ qtime,
                                   int64_t* n_roots_dev) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  int64_t s = start_dev ? *start_dev : 0;
  int64_t b = num_edges - s;
  b = b < 0 ? 0 : (b < batch ? b : batch);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < b;
       i += (int64_t)gridDim.x * blockDim.x) {
    int64_t e = s + i;
    float te = t[e];
    qnode[i] = src[e];
    qnode[b + i] = dst[e];
    qnode[2 * b + i] = neg[e];
    qtime[i] = te;
    qtime[b + i] = te;
    qtime[2 * b + i] = te;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && n_roots_dev) *n_roots_dev = 3 * b;
}

// ---------------------------------------------------------------- S5 next block
__global__ void next_block_kernel(int64_t n_dst_max, const int64_t* n_dst_dev,
                                  const int32_t* __restrict__ dst_node,
                                  const float* __restrict__ dst_t, int64_t n_src_max,
                                  const int64_t* __restrict__ seg_ptr,
                                  const int32_t* __restrict__ src_node,
                                  const float* __restrict__ src_t, int32_t* __restrict__ out_node,
                                  float* __restrict__ out_t, int64_t* n_out_dev) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  int64_t nd = dev_count(n_dst_dev, n_dst_max);
  int64_t ns = seg_ptr[nd];
  ns = ns < n_src_max ? ns : n_src_max;
  int64_t n = nd + ns;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    if (i < nd) {
      out_node[i] = dst_node[i];
      out_t[i] = dst_t[i];
    } else {
      out_node[i] = src_node[i - nd];
      out_t[i] = src_t[i - nd];
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && n_out_dev) *n_out_dev = n;
}

// ---------------------------------------------------------------- S14 row gather
__global__ void gather_rows_kernel(int64_t n_max, const int64_t* n_dev,
                                   const int32_t* __restrict__ idx,
                                   const float* __restrict__ table, int64_t ld_table, int32_t d,
                                   float* __restrict__ out, int64_t ld_out) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  int64_t n = dev_count(n_dev, n_max);
  int64_t total = n * d;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    int64_t j = x / d;
    int c = (int)(x - j * d);
    out[j * ld_out + c] = table[(int64_t)idx[j] * ld_table + c];
  }
}

// ---------------------------------------------------------------- N2 row scatter-add
// out[idx[j]][:] += src[j][:] for j < n (the adjoint of the S14 gather); atomic adds.
__global__ void scatter_add_rows_kernel(int64_t n_max, const int64_t* n_dev,
                                        const int32_t* __restrict__ idx,
                                        const float* __restrict__ src, int64_t ld_src, int32_t d,
                                        float* __restrict__ out, int64_t ld_out) {
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const int64_t total = n * d;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = x / d;
    const int c = (int)(x - j * d);
    const int64_t r = idx ? (int64_t)idx[j] : j;
    atomicAdd(out + r * ld_out + c, src[j * ld_src + c]);
  }
}

// ---------------------------------------------------------------- N4 preload
// dst row j = src row idx[j] (row_bytes bytes) for j < n; src may be pinned host memory
// mapped into the device address space (the GPU reads it over the host link).  One warp
// per row, 16-byte vectors when every pitch and the row size allow.
__global__ void preload_rows_kernel(int64_t n_max, const int64_t* n_dev, const int64_t* n_at,
                                    const int32_t* __restrict__ idx, const uint8_t* src,
                                    int64_t src_pitch, int64_t row_bytes, uint8_t* dst,
                                    int64_t dst_pitch, bool vec16) {
  pdl_wait();
  pdl_trigger();
  int64_t n = n_max;
  if (n_dev != nullptr) n = n_dev[n_at ? *n_at : 0];
  n = n < n_max ? n : n_max;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); j < n; j += warps) {
    const int64_t r = idx ? (int64_t)idx[j] : j;
    const uint8_t* s = src + r * src_pitch;
    uint8_t* d = dst + j * dst_pitch;
    if (vec16) {
      for (int64_t b = 16 * lane; b < row_bytes; b += 16 * 32)
        *reinterpret_cast<uint4*>(d + b) = *reinterpret_cast<const uint4*>(s + b);
    } else {
      for (int64_t b = 4 * lane; b < row_bytes; b += 4 * 32)
        *reinterpret_cast<uint32_t*>(d + b) = *reinterpret_cast<const uint32_t*>(s + b);
    }
  }
}

// ---------------------------------------------------------------- split16 rows
// dst row r (pitch ld_dst 4-byte words): bf16 hi of columns [0, dp) then bf16 lo of the
// same columns, dp = d rounded up to 8 (zero columns past d); hi = RNE(x),
// lo = RNE(x - hi) -- the operand split of the 3-pass tensor-core path.  One thread per
// 8-column group: 16-byte stores.
__global__ void split_rows_kernel(int64_t n_rows, int32_t d, const float* __restrict__ src,
                                  int64_t ld_src, uint8_t* __restrict__ dst, int64_t ld_dst) {
  pdl_wait();
  pdl_trigger();
  const int dp = (d + 7) & ~7;
  const int groups = dp >> 3;
  const int64_t total = n_rows * groups;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = x / groups;
    const int g = (int)(x - r * groups);
    const float* sp = src + r * ld_src + 8 * g;
    uint32_t h[4], l[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int c = 8 * g + 2 * e;
      const float x0 = c < d ? sp[2 * e] : 0.f, x1 = c + 1 < d ? sp[2 * e + 1] : 0.f;
      __nv_bfloat162 hh = __floats2bfloat162_rn(x0, x1);
      __nv_bfloat162 ll = __floats2bfloat162_rn(x0 - __low2float(hh), x1 - __high2float(hh));
      h[e] = *reinterpret_cast<uint32_t*>(&hh);
      l[e] = *reinterpret_cast<uint32_t*>(&ll);
    }
    uint8_t* row = dst + r * ld_dst * 4;
    *reinterpret_cast<uint4*>(row + 16 * g) = make_uint4(h[0], h[1], h[2], h[3]);
    *reinterpret_cast<uint4*>(row + 2 * dp + 16 * g) = make_uint4(l[0], l[1], l[2], l[3]);
  }
}

static int grid_for(int64_t n, int threads) {
  int64_t g = ceil_div(n > 0 ? n : 1, threads);
  int64_t cap = (int64_t)kNumSMs * 16;
  return (int)(g < cap ? g : cap);
}

}  // namespace tgl

using namespace tgl;

extern "C" {

const char* tgl_version(void) { return "tgl-b200 0.1 (sm_100a)"; }

const char* tgl_status_string(tgl_status s) {
  switch (s) {
    case TGL_OK: return "TGL_OK";
    case TGL_EINVAL: return "TGL_EINVAL";
    case TGL_EWORKSPACE: return "TGL_EWORKSPACE";
    case TGL_ECUDA: return "TGL_ECUDA";
    case TGL_ERANGE: return "TGL_ERANGE";
    case TGL_EUNSUPPORTED: return "TGL_EUNSUPPORTED";
    default: return "TGL_UNKNOWN";
  }
}

const char* tgl_last_error(void) { return g_last_error; }

tgl_status tgl_batch_roots(int64_t batch, int64_t num_edges, const int64_t* start_dev,
                           const int32_t* src, const int32_t* dst, const float* t,
                           const int32_t* neg, int32_t* qnode, float* qtime,
                           int64_t* n_roots_dev, void* stream) {
  TGL_REQUIRE(batch >= 0 && num_edges >= 0, "negative size");
  TGL_REQUIRE(src && dst && t && neg && qnode && qtime, "null pointer");
  launch_pdl(batch_roots_kernel, dim3(grid_for(batch, 256)), dim3(256), 0, as_stream(stream), 
      batch, num_edges, start_dev, src, dst, t, neg, qnode, qtime, n_roots_dev);
  return launch_check("batch_roots");
}

tgl_status tgl_next_block(int64_t n_dst_max, const int64_t* n_dst_dev, const int32_t* dst_node,
                          const float* dst_t, int64_t n_src_max, const int64_t* seg_ptr,
                          const int32_t* src_node, const float* src_t, int32_t* out_node,
                          float* out_t, int64_t* n_out_dev, void* stream) {
  TGL_REQUIRE(n_dst_max >= 0 && n_src_max >= 0, "negative size");
  TGL_REQUIRE(seg_ptr && out_node && out_t, "null pointer");
  TGL_REQUIRE((n_dst_max == 0 || (dst_node && dst_t)) && (n_src_max == 0 || (src_node && src_t)),
              "null pointer");
  launch_pdl(next_block_kernel, dim3(grid_for(n_dst_max + n_src_max, 256)), dim3(256), 0, as_stream(stream), 
      n_dst_max, n_dst_dev, dst_node, dst_t, n_src_max, seg_ptr, src_node, src_t, out_node, out_t,
      n_out_dev);
  return launch_check("next_block");
}

tgl_status tgl_gather_rows(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                           const float* table, int64_t ld_table, int32_t d, float* out,
                           int64_t ld_out, void* stream) {
  TGL_REQUIRE(n_max >= 0 && d >= 0 && ld_table >= d && ld_out >= d, "bad size");
  if (n_max == 0 || d == 0) return TGL_OK;
  TGL_REQUIRE(idx && table && out, "null pointer");
  launch_pdl(gather_rows_kernel, dim3(grid_for(n_max * d, 256)), dim3(256), 0, as_stream(stream), 
      n_max, n_dev, idx, table, ld_table, d, out, ld_out);
  return launch_check("gather_rows");
}

tgl_status tgl_scatter_add_rows(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                                const float* src, int64_t ld_src, int32_t d, float* out,
                                int64_t ld_out, void* stream) {
  TGL_REQUIRE(n_max >= 0 && d >= 0 && ld_src >= d && ld_out >= d, "bad size");
  if (n_max == 0 || d == 0) return TGL_OK;
  TGL_REQUIRE(src && out, "null pointer");
  launch_pdl(scatter_add_rows_kernel, dim3(grid_for(n_max * d, 256)), dim3(256), 0,
             as_stream(stream), n_max, n_dev, idx, src, ld_src, d, out, ld_out);
  return launch_check("scatter_add_rows");
}

tgl_status tgl_preload_rows(int64_t n_max, const int64_t* n_dev, const int64_t* n_at,
                            const int32_t* idx, const void* src, int64_t src_pitch,
                            int64_t row_bytes, void* dst, int64_t dst_pitch, void* stream) {
  TGL_REQUIRE(n_max >= 0 && row_bytes >= 0 && src_pitch >= row_bytes && dst_pitch >= row_bytes,
              "bad size");
  TGL_REQUIRE(row_bytes % 4 == 0, "row_bytes must be a multiple of 4");
  if (n_max == 0 || row_bytes == 0) return TGL_OK;
  TGL_REQUIRE(src && dst, "null pointer");
  const bool vec16 = row_bytes % 16 == 0 && src_pitch % 16 == 0 && dst_pitch % 16 == 0 &&
                     (reinterpret_cast<uintptr_t>(src) & 15) == 0 &&
                     (reinterpret_cast<uintptr_t>(dst) & 15) == 0;
  int64_t g = ceil_div(n_max, 8);
  if (g > (int64_t)kNumSMs * 16) g = (int64_t)kNumSMs * 16;
  launch_pdl(preload_rows_kernel, dim3((unsigned)g), dim3(256), 0, as_stream(stream), n_max,
             n_dev, n_at, idx, static_cast<const uint8_t*>(src), src_pitch, row_bytes,
             static_cast<uint8_t*>(dst), dst_pitch, vec16);
  return launch_check("preload_rows");
}

tgl_status tgl_split_rows(int64_t n_rows, int32_t d, const float* src, int64_t ld_src,
                          void* dst, int64_t ld_dst, void* stream) {
  TGL_REQUIRE(n_rows >= 0 && d >= 0, "negative size");
  const int64_t dp = (d + 7) & ~7;
  TGL_REQUIRE(ld_src >= d && ld_dst >= dp && ld_dst % 4 == 0, "bad leading dim");
  if (n_rows == 0 || d == 0) return TGL_OK;
  TGL_REQUIRE(src && dst, "null pointer");
  TGL_REQUIRE((reinterpret_cast<uintptr_t>(dst) & 15) == 0, "dst must be 16-byte aligned");
  launch_pdl(split_rows_kernel, dim3(grid_for(n_rows * (dp / 8), 256)), dim3(256), 0,
             as_stream(stream), n_rows, d, src, ld_src, static_cast<uint8_t*>(dst), ld_dst);
  return launch_check("split_rows");
}

}  // extern "C"
