// dedup.cu -- S3 dedup of <node, time> pairs (readings R8, R9).
//
// Packed 64-bit key (node << 32 | time bits, -0 -> +0) inserted into an open-
// addressing table (next_pow2(2n) slots) with atomicCAS; each slot keeps the
// smallest input index that carries its key (atomicMax of ~i).  A single-pass
// look-back scan over "i is the first occurrence of its key" then emits the
// distinct pairs in first-occurrence order and records each slot's rank, and a
// last pass writes inv[i] = rank[slot(i)].  O(n) work, 3 launches + 1 memset,
// no host sync.  Memory-bound on the key/slot arrays (tiny next to S7).
#include "common.cuh"

namespace tgl {

constexpr int kDedupThreads = 256;
constexpr int kDedupItems = 2;   // 512-pair tiles: many CTAs in flight for the ~2k-20k pairs of a batch
constexpr int kDedupTile = kDedupThreads * kDedupItems;

__device__ __forceinline__ unsigned long long pair_key(int32_t node, float t) {
  // +1 so that the all-zero memset means "empty slot"
  return ((((unsigned long long)(uint32_t)node) << 32) | time_key_bits(t)) + 1ull;
}

__device__ __forceinline__ uint32_t slot_hash(unsigned long long k, int log2cap) {
  return (uint32_t)((k * 0x9E3779B97F4A7C15ull) >> (64 - log2cap));
}

__global__ void dedup_insert_kernel(int64_t n_max, const int64_t* n_dev,
                                    const int32_t* __restrict__ node, const float* __restrict__ t,
                                    unsigned long long* keys, unsigned int* first,
                                    uint32_t* __restrict__ slot_of, int log2cap) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  const uint32_t mask = (1u << log2cap) - 1u;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = pair_key(__ldg(node + i), __ldg(t + i));
    uint32_t h = slot_hash(k, log2cap);
    while (true) {
      unsigned long long prev = atomicCAS(keys + h, 0ull, k);
      if (prev == 0ull || prev == k) {
        atomicMax(first + h, ~(unsigned int)i);
        slot_of[i] = h;
        break;
      }
      h = (h + 1u) & mask;
    }
  }
}

__global__ void __launch_bounds__(kDedupThreads)
dedup_compact_kernel(int64_t n_max, const int64_t* n_dev, const int32_t* __restrict__ node,
                     const float* __restrict__ t, const unsigned int* __restrict__ first,
                     const uint32_t* __restrict__ slot_of, unsigned int* __restrict__ rank,
                     int32_t* __restrict__ uniq_node, float* __restrict__ uniq_t,
                     int64_t* num_uniq_dev, unsigned long long* status, unsigned int* ticket) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  __shared__ int64_t s_tile;
  __shared__ int64_t s_warp[kDedupThreads / 32];
  __shared__ int64_t s_excl;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t n = dev_count(n_dev, n_max);
  const int64_t base = tile * kDedupTile;
  if (base >= n) {
    if (tile == 0 && threadIdx.x == 0) *num_uniq_dev = 0;
    return;
  }
  // blocked arrangement: thread owns items base + tid*ITEMS + [0, ITEMS)
  bool isfirst[kDedupItems];
  uint32_t slot[kDedupItems];
  int cnt = 0;
#pragma unroll
  for (int r = 0; r < kDedupItems; ++r) {
    const int64_t i = base + (int64_t)threadIdx.x * kDedupItems + r;
    isfirst[r] = false;
    slot[r] = 0;
    if (i < n) {
      slot[r] = slot_of[i];
      isfirst[r] = (first[slot[r]] == ~(unsigned int)i);
      cnt += isfirst[r];
    }
  }
  int64_t incl = warp_inclusive_scan((int64_t)cnt, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int64_t wv = lane < kDedupThreads / 32 ? s_warp[lane] : 0;
    int64_t wincl = warp_inclusive_scan(wv, lane);
    int64_t agg = __shfl_sync(0xffffffffu, wincl, 31);
    int64_t excl_tile = lookback(status, tile, agg, lane);
    if (lane < kDedupThreads / 32) s_warp[lane] = excl_tile + wincl - wv;  // warp exclusive
    if (lane == 0) s_excl = excl_tile + agg;
  }
  __syncthreads();
  int64_t pos = s_warp[warp] + incl - cnt;
#pragma unroll
  for (int r = 0; r < kDedupItems; ++r) {
    if (isfirst[r]) {
      const int64_t i = base + (int64_t)threadIdx.x * kDedupItems + r;
      uniq_node[pos] = node[i];
      uniq_t[pos] = t[i];
      rank[slot[r]] = (unsigned int)pos;
      ++pos;
    }
  }
  if (threadIdx.x == 0 && base + kDedupTile >= n) *num_uniq_dev = s_excl;
}

__global__ void dedup_inverse_kernel(int64_t n_max, const int64_t* n_dev,
                                     const uint32_t* __restrict__ slot_of,
                                     const unsigned int* __restrict__ rank,
                                     int32_t* __restrict__ inv) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  const int64_t n = dev_count(n_dev, n_max);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    inv[i] = (int32_t)rank[slot_of[i]];
}

// Small batches (n_max <= kSmallN, e.g. the 3*batch roots of a step): the whole dedup in
// ONE CTA -- hash table in shared memory, blocked first-occurrence scan, inverse -- one
// launch instead of two memsets and three kernels.  Same keys, same order (R9).
constexpr int kSmallThreads = 1024;
constexpr int kSmallItems = 4;
constexpr int kSmallN = kSmallThreads * kSmallItems;   // 4096
constexpr int kSmallLog2Cap = 13;                       // 8192 slots (load <= 1/2)
constexpr int kSmallSmem = (1 << kSmallLog2Cap) * (8 + 4 + 4);   // keys, first, rank

__global__ void __launch_bounds__(kSmallThreads)
dedup_small_kernel(int64_t n_max, const int64_t* n_dev, const int32_t* __restrict__ node,
                   const float* __restrict__ t, int32_t* __restrict__ uniq_node,
                   float* __restrict__ uniq_t, int64_t* num_uniq_dev, int32_t* __restrict__ inv) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  extern __shared__ unsigned long long s_keys[];
  unsigned int* s_first = reinterpret_cast<unsigned int*>(s_keys + (1 << kSmallLog2Cap));
  unsigned int* s_rank = s_first + (1 << kSmallLog2Cap);
  __shared__ int s_warp[kSmallThreads / 32];
  constexpr uint32_t mask = (1u << kSmallLog2Cap) - 1u;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int n = (int)dev_count(n_dev, n_max);
  for (int j = tid; j < (1 << kSmallLog2Cap); j += kSmallThreads) {
    s_keys[j] = 0ull;
    s_first[j] = 0u;
  }
  __syncthreads();
  uint32_t slot[kSmallItems];
#pragma unroll
  for (int r = 0; r < kSmallItems; ++r) {        // blocked: thread owns items tid*4 + r
    const int i = tid * kSmallItems + r;
    slot[r] = 0;
    if (i < n) {
      const unsigned long long k = pair_key(__ldg(node + i), __ldg(t + i));
      uint32_t h = slot_hash(k, kSmallLog2Cap);
      while (true) {
        const unsigned long long prev = atomicCAS(s_keys + h, 0ull, k);
        if (prev == 0ull || prev == k) {
          atomicMax(s_first + h, ~(unsigned int)i);
          slot[r] = h;
          break;
        }
        h = (h + 1u) & mask;
      }
    }
  }
  __syncthreads();
  bool isfirst[kSmallItems];
  int cnt = 0;
#pragma unroll
  for (int r = 0; r < kSmallItems; ++r) {
    const int i = tid * kSmallItems + r;
    isfirst[r] = i < n && s_first[slot[r]] == ~(unsigned int)i;
    cnt += isfirst[r];
  }
  const int incl = (int)warp_inclusive_scan((int64_t)cnt, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const int wv = s_warp[lane];
    const int wincl = (int)warp_inclusive_scan((int64_t)wv, lane);
    s_warp[lane] = wincl - wv;                    // exclusive offset of each warp
    if (lane == 31) *num_uniq_dev = wincl;
  }
  __syncthreads();
  int pos = s_warp[warp] + incl - cnt;
#pragma unroll
  for (int r = 0; r < kSmallItems; ++r) {
    if (isfirst[r]) {
      const int i = tid * kSmallItems + r;
      uniq_node[pos] = node[i];
      uniq_t[pos] = t[i];
      s_rank[slot[r]] = (unsigned int)pos;
      ++pos;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kSmallItems; ++r) {
    const int i = tid * kSmallItems + r;
    if (i < n) inv[i] = (int32_t)s_rank[slot[r]];
  }
}

static int log2_capacity(int64_t n_max) {
  int64_t want = 2 * (n_max > 32 ? n_max : 32);
  int l = 6;
  while (((int64_t)1 << l) < want) ++l;
  return l;
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_dedup(int64_t n_max, const int64_t* n_dev, const int32_t* node,
                                const float* t, int32_t* uniq_node, float* uniq_t,
                                int64_t* num_uniq_dev, int32_t* inv, void* ws, size_t* ws_bytes,
                                void* stream) {
  TGL_REQUIRE(n_max >= 0, "negative n_max");
  if (n_max >= ((int64_t)1 << 31)) {
    set_error("dedup supports n < 2^31");
    return TGL_ERANGE;
  }
  const int l2 = log2_capacity(n_max);
  const int64_t cap = (int64_t)1 << l2;
  const int64_t tiles = ceil_div(n_max > 0 ? n_max : 1, kDedupTile);
  WsLayout L;
  const size_t o_keys = L.take(sizeof(unsigned long long) * cap);
  const size_t o_first = L.take(sizeof(unsigned int) * cap);
  const size_t o_rank = L.take(sizeof(unsigned int) * cap);
  const size_t o_slot = L.take(sizeof(uint32_t) * (n_max > 0 ? n_max : 1));
  const size_t o_status = L.take(sizeof(unsigned long long) * tiles);
  const size_t o_ticket = L.take(sizeof(unsigned int));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(num_uniq_dev != nullptr, "null num_uniq_dev");
  TGL_REQUIRE(n_max == 0 || (node && t && uniq_node && uniq_t && inv), "null pointer");
  cudaStream_t s = as_stream(stream);
  if (n_max <= kSmallN) {                        // one CTA, shared-memory table
    static PerDeviceOnce attr;
    TGL_TRY(cuda_check(attr.run([] {
                         return cudaFuncSetAttribute(dedup_small_kernel,
                                                     cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                     kSmallSmem);
                       }), "dedup attr"));
    launch_pdl(dedup_small_kernel, dim3(1), dim3(kSmallThreads), kSmallSmem, s, n_max, n_dev, node, t, uniq_node,
                                                            uniq_t, num_uniq_dev, inv);
    return launch_check("dedup_small");
  }
  char* w = static_cast<char*>(ws);
  // keys/first/rank must start at 0; slot_of is fully overwritten -> clear only what matters
  TGL_TRY(cuda_check(cudaMemsetAsync(w + o_keys, 0, o_slot - o_keys, s), "dedup memset"));
  TGL_TRY(cuda_check(cudaMemsetAsync(w + o_status, 0, L.off - o_status, s), "dedup memset"));
  auto keys = reinterpret_cast<unsigned long long*>(w + o_keys);
  auto first = reinterpret_cast<unsigned int*>(w + o_first);
  auto rank = reinterpret_cast<unsigned int*>(w + o_rank);
  auto slot = reinterpret_cast<uint32_t*>(w + o_slot);
  int64_t g1 = ceil_div(n_max > 0 ? n_max : 1, 256);
  if (g1 > kNumSMs * 8) g1 = kNumSMs * 8;
  launch_pdl(dedup_insert_kernel, dim3((unsigned)g1), dim3(256), 0, s, n_max, n_dev, node, t, keys, first, slot, l2);
  TGL_TRY(launch_check("dedup_insert"));
  launch_pdl(dedup_compact_kernel, dim3((unsigned)tiles), dim3(kDedupThreads), 0, s, 
      n_max, n_dev, node, t, first, slot, rank, uniq_node, uniq_t, num_uniq_dev,
      reinterpret_cast<unsigned long long*>(w + o_status),
      reinterpret_cast<unsigned int*>(w + o_ticket));
  TGL_TRY(launch_check("dedup_compact"));
  launch_pdl(dedup_inverse_kernel, dim3((unsigned)g1), dim3(256), 0, s, n_max, n_dev, slot, rank, inv);
  return launch_check("dedup_inverse");
}
