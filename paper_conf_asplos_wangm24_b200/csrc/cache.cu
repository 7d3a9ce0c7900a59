// cache.cu -- N1 embedding memoisation, the cache() operator (TGOpt
// cache_lookup / cache_store, Listing 1 L10-23 P:184-197; reading R22).
//
// Per-layer open-addressing table in HBM: u64 keys (node << 32 | ordered time
// bits, +1 so 0 = empty; the dedup packing, R8) and fp32 rows.  Lookup probes
// <= TGL_CACHE_PROBES slots and compacts the misses in input order with a
// single-pass look-back scan (one launch); store claims a slot with atomicCAS,
// one warp per pair copying the row; combine is one warp per output row.
#include "common.cuh"

namespace tgl {

constexpr int kCacheThreads = 256;
constexpr int kCacheItems = 2;
constexpr int kCacheTile = kCacheThreads * kCacheItems;

__device__ __forceinline__ unsigned long long cache_key(int32_t node, float t) {
  return ((((unsigned long long)(uint32_t)node) << 32) | time_key_bits(t)) + 1ull;
}

__device__ __forceinline__ uint64_t cache_hash(unsigned long long k, int log2cap) {
  return (k * 0x9E3779B97F4A7C15ull) >> (64 - log2cap);
}

// slot of key k, or -1 (an empty slot or TGL_CACHE_PROBES probes end the search)
__device__ __forceinline__ int64_t cache_find(const unsigned long long* keys, int log2cap,
                                              unsigned long long k) {
  const uint64_t mask = (1ull << log2cap) - 1ull;
  uint64_t h = cache_hash(k, log2cap);
  for (int p = 0; p < TGL_CACHE_PROBES; ++p) {
    const unsigned long long cur = keys[h];
    if (cur == k) return (int64_t)h;
    if (cur == 0ull) return -1;
    h = (h + 1) & mask;
  }
  return -1;
}

__global__ void __launch_bounds__(kCacheThreads)
cache_lookup_kernel(const unsigned long long* __restrict__ keys, int log2cap, int64_t n_max,
                    const int64_t* n_dev, const int32_t* __restrict__ node,
                    const float* __restrict__ t, int32_t* __restrict__ slot,
                    int32_t* __restrict__ miss_node, float* __restrict__ miss_t,
                    int64_t* num_miss_dev, unsigned long long* status, unsigned int* ticket) {
  pdl_wait();
  pdl_trigger();
  __shared__ int64_t s_tile;
  __shared__ int64_t s_warp[kCacheThreads / 32];
  __shared__ int64_t s_excl;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t n = dev_count(n_dev, n_max);
  const int64_t base = tile * kCacheTile;
  if (base >= n) {
    if (tile == 0 && threadIdx.x == 0) *num_miss_dev = 0;
    return;
  }
  int64_t hit[kCacheItems];
  int cnt = 0;
#pragma unroll
  for (int r = 0; r < kCacheItems; ++r) {        // blocked: thread owns base + tid*ITEMS + r
    const int64_t i = base + (int64_t)threadIdx.x * kCacheItems + r;
    hit[r] = -2;                                 // -2: out of range
    if (i < n) {
      const float ti = __ldg(t + i);
      hit[r] = (ti == ti) ? cache_find(keys, log2cap, cache_key(__ldg(node + i), ti)) : -1;
      cnt += hit[r] == -1;
    }
  }
  int64_t incl = warp_inclusive_scan((int64_t)cnt, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int64_t wv = lane < kCacheThreads / 32 ? s_warp[lane] : 0;
    int64_t wincl = warp_inclusive_scan(wv, lane);
    int64_t agg = __shfl_sync(0xffffffffu, wincl, 31);
    int64_t excl_tile = lookback(status, tile, agg, lane);
    if (lane < kCacheThreads / 32) s_warp[lane] = excl_tile + wincl - wv;
    if (lane == 0) s_excl = excl_tile + agg;
  }
  __syncthreads();
  int64_t pos = s_warp[warp] + incl - cnt;
#pragma unroll
  for (int r = 0; r < kCacheItems; ++r) {
    const int64_t i = base + (int64_t)threadIdx.x * kCacheItems + r;
    if (hit[r] >= 0) {
      slot[i] = (int32_t)hit[r];
    } else if (hit[r] == -1) {
      slot[i] = (int32_t)(-1 - pos);
      miss_node[pos] = node[i];
      miss_t[pos] = t[i];
      ++pos;
    }
  }
  if (threadIdx.x == 0 && base + kCacheTile >= n) *num_miss_dev = s_excl;
}

__global__ void cache_store_kernel(unsigned long long* keys, float* __restrict__ vals,
                                   int log2cap, int d, int64_t n_max, const int64_t* n_dev,
                                   const int32_t* __restrict__ node, const float* __restrict__ t,
                                   const float* __restrict__ emb, int64_t ld_emb) {
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  const uint64_t mask = (1ull << log2cap) - 1ull;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    int64_t h = -1;
    if (lane == 0) {
      const float ti = t[i];
      if (ti == ti) {
        const unsigned long long k = cache_key(node[i], ti);
        uint64_t p = cache_hash(k, log2cap);
        for (int q = 0; q < TGL_CACHE_PROBES; ++q) {
          const unsigned long long prev = atomicCAS(keys + p, 0ull, k);
          if (prev == 0ull || prev == k) {
            h = (int64_t)p;
            break;
          }
          p = (p + 1) & mask;
        }
      }
    }
    h = __shfl_sync(0xffffffffu, h, 0);
    if (h < 0) continue;                         // NaN time or no free slot: not stored
    const float* src = emb + i * ld_emb;
    float* dst = vals + h * (int64_t)d;
    for (int c = lane; c < d; c += 32) dst[c] = src[c];
  }
}

__global__ void cache_combine_kernel(const float* __restrict__ vals, int d, int64_t n_max,
                                     const int64_t* n_dev, const int32_t* __restrict__ slot,
                                     const float* __restrict__ computed, int64_t ld_computed,
                                     float* __restrict__ out, int64_t ld_out) {
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    const int32_t s = slot[i];
    const float* src = s >= 0 ? vals + (int64_t)s * d : computed + (int64_t)(-1 - s) * ld_computed;
    float* dst = out + i * ld_out;
    for (int c = lane; c < d; c += 32) dst[c] = src[c];
  }
}

__global__ void cache_merge_kernel(unsigned long long* keys, float* __restrict__ vals,
                                   int log2cap, int d, int64_t n_max, const int64_t* n_dev,
                                   const int32_t* __restrict__ idx,
                                   const int32_t* __restrict__ node, const float* __restrict__ t,
                                   const int32_t* __restrict__ slot,
                                   const float* __restrict__ computed, int64_t ld_computed,
                                   float* __restrict__ out, int64_t ld_out) {
  pdl_wait();
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  const uint64_t mask = (1ull << log2cap) - 1ull;
  for (int64_t j = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < n; j += warps) {
    const int64_t i = idx ? (int64_t)idx[j] : j;
    const int32_t s = slot[i];
    const float* src = s >= 0 ? vals + (int64_t)s * d : computed + (int64_t)(-1 - s) * ld_computed;
    float* dst = out + j * ld_out;
    int64_t h = -1;
    if (s < 0 && lane == 0) {                    // a miss: claim its slot (as cache_store)
      const float ti = t[i];
      if (ti == ti) {
        const unsigned long long k = cache_key(node[i], ti);
        uint64_t p = cache_hash(k, log2cap);
        for (int q = 0; q < TGL_CACHE_PROBES; ++q) {
          const unsigned long long prev = atomicCAS(keys + p, 0ull, k);
          if (prev == 0ull || prev == k) {
            h = (int64_t)p;
            break;
          }
          p = (p + 1) & mask;
        }
      }
    }
    h = __shfl_sync(0xffffffffu, h, 0);
    float* row = h >= 0 ? vals + h * (int64_t)d : nullptr;
    for (int c = lane; c < d; c += 32) {
      const float v = src[c];
      dst[c] = v;
      if (row) row[c] = v;
    }
  }
}

static tgl_status cache_check(const tgl_cache* c, int* log2cap) {
  TGL_REQUIRE(c != nullptr && c->keys != nullptr && c->vals != nullptr, "null cache");
  TGL_REQUIRE(c->capacity > 0 && (c->capacity & (c->capacity - 1)) == 0 &&
                  c->capacity <= ((int64_t)1 << 30),
              "cache capacity must be a power of two <= 2^30");
  TGL_REQUIRE(c->d > 0, "cache row width must be > 0");
  int l = 0;
  while (((int64_t)1 << l) < c->capacity) ++l;
  *log2cap = l < 1 ? 1 : l;
  TGL_REQUIRE(c->capacity >= 2, "cache capacity must be >= 2");
  return TGL_OK;
}

static unsigned warp_grid(int64_t n_max) {
  int64_t g = ceil_div(n_max > 0 ? n_max : 1, 8);   // 8 warps per 256-thread CTA
  if (g > (int64_t)kNumSMs * 16) g = (int64_t)kNumSMs * 16;
  return (unsigned)g;
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_cache_lookup(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                                       const int32_t* node, const float* t, int32_t* slot,
                                       int32_t* miss_node, float* miss_t, int64_t* num_miss_dev,
                                       void* ws, size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(n_max >= 0 && n_max < ((int64_t)1 << 31), "n_max out of range");
  const int64_t tiles = ceil_div(n_max > 0 ? n_max : 1, kCacheTile);
  WsLayout L;
  const size_t o_status = L.take(sizeof(unsigned long long) * tiles);
  const size_t o_ticket = L.take(sizeof(unsigned int));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  int l2 = 0;
  TGL_TRY(cache_check(c, &l2));
  TGL_REQUIRE(num_miss_dev != nullptr, "null num_miss_dev");
  TGL_REQUIRE(n_max == 0 || (node && t && slot && miss_node && miss_t), "null pointer");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  TGL_TRY(cuda_check(cudaMemsetAsync(w, 0, L.off, s), "cache memset"));
  launch_pdl(cache_lookup_kernel, dim3((unsigned)tiles), dim3(kCacheThreads), 0, s,
             (const unsigned long long*)c->keys, l2, n_max, n_dev, node, t, slot, miss_node,
             miss_t, num_miss_dev, reinterpret_cast<unsigned long long*>(w + o_status),
             reinterpret_cast<unsigned int*>(w + o_ticket));
  return launch_check("cache_lookup");
}

extern "C" tgl_status tgl_cache_store(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                                      const int32_t* node, const float* t, const float* emb,
                                      int64_t ld_emb, void* stream) {
  TGL_REQUIRE(n_max >= 0, "negative n_max");
  int l2 = 0;
  TGL_TRY(cache_check(c, &l2));
  TGL_REQUIRE(ld_emb >= c->d, "ld_emb < d");
  TGL_REQUIRE(n_max == 0 || (node && t && emb), "null pointer");
  launch_pdl(cache_store_kernel, dim3(warp_grid(n_max)), dim3(256), 0, as_stream(stream),
             c->keys, c->vals, l2, (int)c->d, n_max, n_dev, node, t, emb, ld_emb);
  return launch_check("cache_store");
}

extern "C" tgl_status tgl_cache_combine(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                                        const int32_t* slot, const float* computed,
                                        int64_t ld_computed, float* out, int64_t ld_out,
                                        void* stream) {
  TGL_REQUIRE(n_max >= 0, "negative n_max");
  int l2 = 0;
  TGL_TRY(cache_check(c, &l2));
  TGL_REQUIRE(ld_out >= c->d && ld_computed >= c->d, "row pitch < d");
  TGL_REQUIRE(n_max == 0 || (slot && computed && out), "null pointer");
  launch_pdl(cache_combine_kernel, dim3(warp_grid(n_max)), dim3(256), 0, as_stream(stream),
             (const float*)c->vals, (int)c->d, n_max, n_dev, slot, computed, ld_computed, out,
             ld_out);
  return launch_check("cache_combine");
}

extern "C" tgl_status tgl_cache_merge(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                                      const int32_t* idx, const int32_t* node, const float* t,
                                      const int32_t* slot, const float* computed,
                                      int64_t ld_computed, float* out, int64_t ld_out,
                                      void* stream) {
  TGL_REQUIRE(n_max >= 0, "negative n_max");
  int l2 = 0;
  TGL_TRY(cache_check(c, &l2));
  TGL_REQUIRE(ld_out >= c->d && ld_computed >= c->d, "row pitch < d");
  TGL_REQUIRE(n_max == 0 || (node && t && slot && computed && out), "null pointer");
  launch_pdl(cache_merge_kernel, dim3(warp_grid(n_max)), dim3(256), 0, as_stream(stream),
             c->keys, c->vals, l2, (int)c->d, n_max, n_dev, idx, node, t, slot, computed,
             ld_computed, out, ld_out);
  return launch_check("cache_merge");
}
