// shard.cu -- S16: root sharding of one batch across G ranks.
//
// Every rank holds the whole graph, features and weights (replicated), computes the
// batch's roots (and their dedup, when enabled) redundantly, and runs S4-S15 for the
// contiguous slice [r*c, min((r+1)*c, U)) of the U unique roots, c = ceil(U / G).
// The slices' embeddings are all-gathered (NCCL, padded to c_max rows per rank) and
// every rank rebuilds the batch's root embeddings through the dedup inverse.  U lives
// on the device, so both kernels read it there (no host sync, CUDA-graph friendly).
#include "common.cuh"

namespace tgl {

__device__ __forceinline__ void shard_bounds(int64_t U, int32_t rank, int32_t world,
                                             int64_t& lo, int64_t& hi) {
  const int64_t c = (U + world - 1) / world;
  lo = (int64_t)rank * c;
  lo = lo < U ? lo : U;
  hi = lo + c < U ? lo + c : U;
}

__global__ void shard_slice_kernel(int64_t n_max, const int64_t* n_dev, const int32_t* __restrict__ node,
                                   const float* __restrict__ t, int32_t rank, int32_t world,
                                   int64_t out_max, int32_t* __restrict__ out_node,
                                   float* __restrict__ out_t, int64_t* out_n_dev) {
  pdl_wait();
  pdl_trigger();
  const int64_t U = dev_count(n_dev, n_max);
  int64_t lo, hi;
  shard_bounds(U, rank, world, lo, hi);
  int64_t m = hi - lo;
  m = m < out_max ? m : out_max;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    out_node[i] = node[lo + i];
    out_t[i] = t[lo + i];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && out_n_dev) *out_n_dev = m;
}

// out[j] = gathered[r * c_max + o] with i = idx ? idx[j] : j, r = i / c, o = i % c
// (one warp per row; rows are d floats)
__global__ void shard_gather_kernel(int64_t n_max, const int64_t* n_dev, const int32_t* __restrict__ idx,
                                    int64_t u_max, const int64_t* u_dev, int32_t world,
                                    const float* __restrict__ gathered, int64_t c_max, int32_t d,
                                    float* __restrict__ out, int64_t ld_out) {
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const int64_t U = dev_count(u_dev, u_max);
  const int64_t c = U > 0 ? (U + world - 1) / world : 1;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); j < n; j += warps) {
    const int64_t i = idx ? (int64_t)idx[j] : j;
    const int64_t src = (i / c) * c_max + (i % c);
    const float* row = gathered + src * d;
    for (int k = lane; k < d; k += 32) out[j * ld_out + k] = row[k];
  }
}

static int grid_for_rows(int64_t n, int rows_per_block) {
  int64_t g = ceil_div(n > 0 ? n : 1, rows_per_block);
  const int64_t cap = (int64_t)kNumSMs * 8;
  return (int)(g < cap ? g : cap);
}

}  // namespace tgl

using namespace tgl;

extern "C" {

tgl_status tgl_shard_slice(int64_t n_max, const int64_t* n_dev, const int32_t* node,
                           const float* t, int32_t rank, int32_t world, int32_t* out_node,
                           float* out_t, int64_t* out_n_dev, void* stream) {
  TGL_REQUIRE(n_max >= 0, "negative size");
  TGL_REQUIRE(world >= 1 && rank >= 0 && rank < world, "bad rank / world");
  TGL_REQUIRE(out_n_dev != nullptr, "null out_n_dev");
  TGL_REQUIRE(n_max == 0 || (node && t && out_node && out_t), "null pointer");
  const int64_t out_max = ceil_div(n_max, world);
  launch_pdl(shard_slice_kernel, dim3(grid_for_rows(out_max, 256)), dim3(256), 0,
             as_stream(stream), n_max, n_dev, node, t, rank, world, out_max, out_node, out_t,
             out_n_dev);
  return launch_check("shard_slice");
}

tgl_status tgl_shard_gather(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                            int64_t u_max, const int64_t* u_dev, int32_t world,
                            const float* gathered, int64_t c_max, int32_t d, float* out,
                            int64_t ld_out, void* stream) {
  TGL_REQUIRE(n_max >= 0 && u_max >= 0 && d >= 0 && ld_out >= d, "bad size");
  TGL_REQUIRE(world >= 1, "bad world");
  TGL_REQUIRE(c_max >= ceil_div(u_max, world), "c_max < ceil(u_max / world)");
  if (n_max == 0 || d == 0) return TGL_OK;
  TGL_REQUIRE(gathered && out, "null pointer");
  launch_pdl(shard_gather_kernel, dim3(grid_for_rows(n_max, 8)), dim3(256), 0, as_stream(stream),
             n_max, n_dev, idx, u_max, u_dev, world, gathered, c_max, d, out, ld_out);
  return launch_check("shard_gather");
}

}  // extern "C"
