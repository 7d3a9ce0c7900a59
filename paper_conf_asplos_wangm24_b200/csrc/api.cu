// api.cu -- error reporting, version, and the small S2/S5/S14 kernels.
#include <stdarg.h>
#include <string.h>

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

}  // extern "C"
