// tcsr.cu -- S1 temporal CSR build (readings R2, R3).
//
// Entries j in [0, M): undirected j = 2e + dir (dir 1 = reverse), directed j = e.
// Their natural order is (eid, dir).  A stable LSD radix sort keyed first by the
// order-preserving bits of t (skipped with TGL_INPUT_TIME_SORTED, where the
// (eid, dir) order already is the (t, eid, dir) order) and then by the owner
// node yields (owner, t, eid, dir) -- the segment order R3 asks for.  Each
// 8-bit pass: per-tile digit histogram -> one single-pass look-back scan of the
// digit-major counts -> stable scatter (warp match_any ranks, striped rounds).
// indptr is filled from the owner boundaries of the sorted keys.
#include "common.cuh"

namespace tgl {

constexpr int kRadixThreads = 256;
constexpr int kRadixRounds = 16;
constexpr int kRadixTile = kRadixThreads * kRadixRounds;  // 4096
constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;

__device__ __forceinline__ uint32_t ordered_time_bits(float t) {
  uint32_t b = time_key_bits(t);  // -0 == +0 (R8)
  return b ^ ((b >> 31) ? 0xFFFFFFFFu : 0x80000000u);
}

__device__ __forceinline__ int32_t entry_owner(uint32_t j, bool undirected,
                                               const int32_t* __restrict__ src,
                                               const int32_t* __restrict__ dst) {
  if (!undirected) return __ldg(src + j);
  return (j & 1u) ? __ldg(dst + (j >> 1)) : __ldg(src + (j >> 1));
}

__global__ void tcsr_init_kernel(int64_t M, bool undirected, bool time_pass,
                                 const int32_t* __restrict__ src, const int32_t* __restrict__ dst,
                                 const float* __restrict__ t, uint32_t* __restrict__ keys,
                                 uint32_t* __restrict__ vals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M;
       i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t j = (uint32_t)i;
    vals[i] = j;
    if (time_pass) {
      uint32_t e = undirected ? (j >> 1) : j;
      keys[i] = ordered_time_bits(__ldg(t + e));
    } else {
      keys[i] = (uint32_t)entry_owner(j, undirected, src, dst);
    }
  }
}

__global__ void tcsr_owner_keys_kernel(int64_t M, bool undirected, const int32_t* __restrict__ src,
                                       const int32_t* __restrict__ dst,
                                       const uint32_t* __restrict__ vals,
                                       uint32_t* __restrict__ keys) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M;
       i += (int64_t)gridDim.x * blockDim.x)
    keys[i] = (uint32_t)entry_owner(vals[i], undirected, src, dst);
}

__global__ void __launch_bounds__(kRadixThreads)
radix_hist_kernel(int64_t M, int shift, const uint32_t* __restrict__ keys,
                  uint32_t* __restrict__ counts, int64_t tiles) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kRadixTile;
#pragma unroll 4
  for (int r = 0; r < kRadixRounds; ++r) {
    int64_t i = base + r * kRadixThreads + threadIdx.x;
    if (i < M) atomicAdd(&h[(keys[i] >> shift) & 0xFFu], 1u);
  }
  __syncthreads();
  counts[(int64_t)threadIdx.x * tiles + blockIdx.x] = h[threadIdx.x];
}

// exclusive scan of u32 counts (total < 2^32), single pass with look-back
__global__ void __launch_bounds__(kScanThreads)
scan_u32_kernel(int64_t n, uint32_t* __restrict__ data, unsigned long long* status,
                unsigned int* ticket) {
  __shared__ int64_t s_tile;
  __shared__ int64_t s_warp[kScanThreads / 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t base = tile * kScanTile + (int64_t)threadIdx.x * kScanItems;
  uint32_t v[kScanItems];
  int64_t sum = 0;
#pragma unroll
  for (int r = 0; r < kScanItems; ++r) {
    v[r] = (base + r < n) ? data[base + r] : 0u;
    sum += v[r];
  }
  int64_t incl = warp_inclusive_scan(sum, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int64_t wv = lane < kScanThreads / 32 ? s_warp[lane] : 0;
    int64_t wincl = warp_inclusive_scan(wv, lane);
    int64_t agg = __shfl_sync(0xffffffffu, wincl, 31);
    int64_t excl_tile = lookback(status, tile, agg, lane);
    if (lane < kScanThreads / 32) s_warp[lane] = excl_tile + wincl - wv;
  }
  __syncthreads();
  int64_t run = s_warp[warp] + incl - sum;
#pragma unroll
  for (int r = 0; r < kScanItems; ++r) {
    if (base + r < n) data[base + r] = (uint32_t)run;
    run += v[r];
  }
}

__global__ void __launch_bounds__(kRadixThreads)
radix_scatter_kernel(int64_t M, int shift, const uint32_t* __restrict__ keys_in,
                     const uint32_t* __restrict__ vals_in, uint32_t* __restrict__ keys_out,
                     uint32_t* __restrict__ vals_out, const uint32_t* __restrict__ offsets,
                     int64_t tiles) {
  __shared__ uint32_t s_base[256];
  __shared__ uint32_t s_run[256];
  __shared__ uint32_t s_wcnt[kRadixThreads / 32][256];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  s_base[threadIdx.x] = offsets[(int64_t)threadIdx.x * tiles + blockIdx.x];
  s_run[threadIdx.x] = 0;
  for (int w = 0; w < kRadixThreads / 32; ++w) s_wcnt[w][threadIdx.x] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kRadixTile;
  const unsigned lt_mask = (1u << lane) - 1u;
  for (int r = 0; r < kRadixRounds; ++r) {
    const int64_t i = base + r * kRadixThreads + threadIdx.x;
    const bool valid = i < M;
    uint32_t k = 0, v = 0, d = 0;
    if (valid) {
      k = keys_in[i];
      v = vals_in[i];
      d = (k >> shift) & 0xFFu;
    }
    // invalid lanes get a unique tag so they never join a digit group
    unsigned peers = __match_any_sync(0xffffffffu, valid ? d : (0x100u + lane));
    int rk = __popc(peers & lt_mask);
    if (valid && rk == 0) s_wcnt[warp][d] = __popc(peers);
    __syncthreads();
    if (valid) {
      uint32_t pre = 0;
      for (int w = 0; w < warp; ++w) pre += s_wcnt[w][d];
      uint32_t pos = s_base[d] + s_run[d] + pre + rk;
      keys_out[pos] = k;
      vals_out[pos] = v;
    }
    __syncthreads();
    {
      uint32_t tot = 0;
#pragma unroll
      for (int w = 0; w < kRadixThreads / 32; ++w) {
        tot += s_wcnt[w][threadIdx.x];
        s_wcnt[w][threadIdx.x] = 0;
      }
      s_run[threadIdx.x] += tot;
    }
    __syncthreads();
  }
}

__global__ void tcsr_emit_kernel(int64_t M, bool undirected, const int32_t* __restrict__ src,
                                 const int32_t* __restrict__ dst, const float* __restrict__ t,
                                 const uint32_t* __restrict__ vals, int32_t* __restrict__ nbr,
                                 int32_t* __restrict__ eid, float* __restrict__ ts) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < M;
       p += (int64_t)gridDim.x * blockDim.x) {
    uint32_t j = vals[p];
    uint32_t e = undirected ? (j >> 1) : j;
    bool rev = undirected && (j & 1u);
    nbr[p] = rev ? __ldg(src + e) : __ldg(dst + e);
    eid[p] = (int32_t)e;
    ts[p] = __ldg(t + e);
  }
}

// indptr[v] = first position whose owner >= v; keys sorted ascending.
__global__ void tcsr_indptr_kernel(int64_t M, int64_t N, const uint32_t* __restrict__ keys,
                                   int64_t* __restrict__ indptr) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p <= M;
       p += (int64_t)gridDim.x * blockDim.x) {
    int64_t lo = p == 0 ? 0 : (int64_t)keys[p - 1] + 1;   // owners (prev, cur] start at p
    int64_t hi = p == M ? N : (int64_t)keys[p];
    for (int64_t v = lo; v <= hi; ++v) indptr[v] = p;
  }
}

static int grid_for(int64_t n, int threads) {
  int64_t g = ceil_div(n > 0 ? n : 1, threads);
  int64_t cap = (int64_t)kNumSMs * 16;
  return (int)(g < cap ? g : cap);
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_build_tcsr(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                                     const int32_t* dst, const float* t, uint32_t flags,
                                     int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts,
                                     void* ws, size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(num_nodes >= 0 && num_edges >= 0, "negative size");
  TGL_REQUIRE((flags & ~(TGL_UNDIRECTED | TGL_INPUT_TIME_SORTED)) == 0, "unknown flags 0x%x",
              flags);
  const bool undirected = (flags & TGL_UNDIRECTED) != 0;
  const bool sorted = (flags & TGL_INPUT_TIME_SORTED) != 0;
  const int64_t M = undirected ? 2 * num_edges : num_edges;
  if (M >= ((int64_t)1 << 32) || num_nodes >= ((int64_t)1 << 31) ||
      num_edges >= ((int64_t)1 << 31)) {
    set_error("T-CSR supports < 2^32 entries, < 2^31 nodes and edges");
    return TGL_ERANGE;
  }
  const int64_t tiles = ceil_div(M > 0 ? M : 1, kRadixTile);
  const int64_t ncount = 256 * tiles;
  const int64_t scan_tiles = ceil_div(ncount, kScanTile);
  WsLayout L;
  const size_t o_k0 = L.take(sizeof(uint32_t) * (M > 0 ? M : 1));
  const size_t o_v0 = L.take(sizeof(uint32_t) * (M > 0 ? M : 1));
  const size_t o_k1 = L.take(sizeof(uint32_t) * (M > 0 ? M : 1));
  const size_t o_v1 = L.take(sizeof(uint32_t) * (M > 0 ? M : 1));
  const size_t o_cnt = L.take(sizeof(uint32_t) * ncount);
  const size_t o_status = L.take(sizeof(unsigned long long) * scan_tiles);
  const size_t o_ticket = L.take(sizeof(unsigned int));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(indptr != nullptr, "null indptr");
  TGL_REQUIRE(M == 0 || (src && dst && t && nbr && eid && ts), "null pointer");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  if (M == 0) {
    return cuda_check(cudaMemsetAsync(indptr, 0, sizeof(int64_t) * (num_nodes + 1), s),
                      "indptr memset");
  }
  uint32_t* k[2] = {reinterpret_cast<uint32_t*>(w + o_k0), reinterpret_cast<uint32_t*>(w + o_k1)};
  uint32_t* v[2] = {reinterpret_cast<uint32_t*>(w + o_v0), reinterpret_cast<uint32_t*>(w + o_v1)};
  uint32_t* counts = reinterpret_cast<uint32_t*>(w + o_cnt);
  auto status = reinterpret_cast<unsigned long long*>(w + o_status);
  auto ticket = reinterpret_cast<unsigned int*>(w + o_ticket);
  int cur = 0;
  auto run_pass = [&](int shift) -> tgl_status {
    radix_hist_kernel<<<(unsigned)tiles, kRadixThreads, 0, s>>>(M, shift, k[cur], counts, tiles);
    TGL_TRY(launch_check("radix_hist"));
    TGL_TRY(cuda_check(cudaMemsetAsync(w + o_status, 0, L.off - o_status, s), "scan memset"));
    scan_u32_kernel<<<(unsigned)scan_tiles, kScanThreads, 0, s>>>(ncount, counts, status, ticket);
    TGL_TRY(launch_check("radix_scan"));
    radix_scatter_kernel<<<(unsigned)tiles, kRadixThreads, 0, s>>>(
        M, shift, k[cur], v[cur], k[cur ^ 1], v[cur ^ 1], counts, tiles);
    TGL_TRY(launch_check("radix_scatter"));
    cur ^= 1;
    return TGL_OK;
  };
  tcsr_init_kernel<<<grid_for(M, 256), 256, 0, s>>>(M, undirected, !sorted, src, dst, t, k[0], v[0]);
  TGL_TRY(launch_check("tcsr_init"));
  if (!sorted) {
    for (int shift = 0; shift < 32; shift += 8) TGL_TRY(run_pass(shift));
    tcsr_owner_keys_kernel<<<grid_for(M, 256), 256, 0, s>>>(M, undirected, src, dst, v[cur], k[cur]);
    TGL_TRY(launch_check("tcsr_owner_keys"));
  }
  int bits = 1;
  while (bits < 31 && ((int64_t)1 << bits) < num_nodes) ++bits;
  for (int shift = 0; shift < bits; shift += 8) TGL_TRY(run_pass(shift));
  tcsr_emit_kernel<<<grid_for(M, 256), 256, 0, s>>>(M, undirected, src, dst, t, v[cur], nbr, eid, ts);
  TGL_TRY(launch_check("tcsr_emit"));
  tcsr_indptr_kernel<<<grid_for(M + 1, 256), 256, 0, s>>>(M, num_nodes, k[cur], indptr);
  return launch_check("tcsr_indptr");
}
