// tcsr.cu -- S1 temporal CSR build (readings R2, R3).
//
// Two implementations of the same stable LSD sort: the one-sweep record path below (M <
// 2^30 entries: every product config but MAG) and the index-sort path (any size).
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


// ------------------------------------------------------------------ one-sweep path (M < 2^30)
// The same stable LSD digit sequence, but the entries travel as 16-byte records
// {owner, nbr, eid, bits(t)} built from the COO in the first pass, so the last pass writes
// the T-CSR arrays (and the sampler indexes) directly -- no index gather afterwards.  One
// kernel per pass (Merrill & Garland "onesweep"): per-pass global digit counts come from one
// histogram sweep over the COO; a tile ranks its 4,096 records with warp ballots (8 per round,
// an exact multi-split), publishes its 256 digit counts and looks back over earlier tiles per
// digit (decoupled look-back) for its offsets.  Warp w of a tile owns entries
// [w*512, (w+1)*512) of it, so ranks need no block barrier until the tile's totals.
constexpr int kSwThreads = 256;
constexpr int kSwWarps = kSwThreads / 32;
constexpr int kSwIPT = 16;
constexpr int kSwTile = kSwThreads * kSwIPT;  // 4096
constexpr uint32_t kSwAgg = 1u << 30, kSwPre = 2u << 30, kSwVal = (1u << 30) - 1;
constexpr int kSwMaxPasses = 8;
constexpr int kSwWindow = 8;
constexpr int64_t kSwDegSmemNodes = 40960;   // degree histogram in shared memory (160 KB)

struct SwArgs {
  int64_t M, N;
  bool undirected;
  const int32_t* src;
  const int32_t* dst;
  const float* t;
  int npass;
  int field[kSwMaxPasses];  // 0 = ordered bits of t, 1 = owner
  int shift[kSwMaxPasses];
  uint32_t* ghist;          // [npass][256]: counts, then exclusive bases
  uint32_t* deg;            // [N] (N <= kSwDegSmemNodes) or NULL
  int64_t* indptr;
};

__device__ __forceinline__ uint4 sw_make_record(const SwArgs& a, int64_t i) {
  const int64_t e = a.undirected ? (i >> 1) : i;
  const bool rev = a.undirected && (i & 1);
  const int32_t s = __ldg(a.src + e), d = __ldg(a.dst + e);
  return make_uint4((uint32_t)(rev ? d : s), (uint32_t)(rev ? s : d), (uint32_t)e,
                    __float_as_uint(__ldg(a.t + e)));
}

__device__ __forceinline__ uint32_t sw_digit(const uint4& r, int field, int shift) {
  const uint32_t k = field == 0 ? ordered_time_bits(__uint_as_float(r.w)) : r.x;
  return (k >> shift) & 0xFFu;
}

__device__ __forceinline__ void sw_count(const SwArgs& a, uint32_t (*h)[256], uint32_t* s_deg,
                                         uint32_t owner, uint32_t tb) {
  for (int p = 0; p < a.npass; ++p)
    atomicAdd(&h[p][((a.field[p] == 0 ? tb : owner) >> a.shift[p]) & 0xFFu], 1u);
  if (s_deg) atomicAdd(&s_deg[owner], 1u);
}

// grid-stride over EDGES, 4 per thread per step (12 independent loads in flight)
__global__ void __launch_bounds__(1024) sw_hist_kernel(SwArgs a, int64_t E) {
  extern __shared__ uint32_t s_deg_dyn[];
  __shared__ uint32_t h[kSwMaxPasses][256];
  uint32_t* s_deg = a.deg != nullptr ? s_deg_dyn : nullptr;
  for (int x = threadIdx.x; x < a.npass * 256; x += blockDim.x) h[x / 256][x % 256] = 0;
  if (s_deg)
    for (int64_t v = threadIdx.x; v < a.N; v += blockDim.x) s_deg[v] = 0;
  __syncthreads();
  const bool need_t = a.field[0] == 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * 4;
  for (int64_t e0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 4; e0 < E; e0 += stride) {
    int32_t sv[4], dv[4];
    float tv[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t e = e0 + u;
      sv[u] = e < E ? __ldg(a.src + e) : 0;
      dv[u] = e < E ? __ldg(a.dst + e) : 0;
      tv[u] = (need_t && e < E) ? __ldg(a.t + e) : 0.f;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      if (e0 + u >= E) break;
      const uint32_t tb = need_t ? ordered_time_bits(tv[u]) : 0u;
      sw_count(a, h, s_deg, (uint32_t)sv[u], tb);
      if (a.undirected) sw_count(a, h, s_deg, (uint32_t)dv[u], tb);
    }
  }
  __syncthreads();
  for (int x = threadIdx.x; x < a.npass * 256; x += blockDim.x)
    if (h[x / 256][x % 256]) atomicAdd(a.ghist + x, h[x / 256][x % 256]);
  if (s_deg)
    for (int64_t v = threadIdx.x; v < a.N; v += blockDim.x)
      if (s_deg[v]) atomicAdd(a.deg + v, s_deg[v]);
}

// one CTA of 1024: exclusive digit bases per pass; indptr = exclusive scan of the degrees
__global__ void __launch_bounds__(1024) sw_bases_kernel(SwArgs a) {
  __shared__ int64_t s_warp[32];
  __shared__ int64_t s_carry;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x < a.npass) {
    uint32_t run = 0;
    uint32_t* g = a.ghist + threadIdx.x * 256;
    for (int d = 0; d < 256; ++d) {
      const uint32_t c = g[d];
      g[d] = run;
      run += c;
    }
  }
  if (a.deg == nullptr) return;
  if (threadIdx.x == 0) s_carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < a.N; base += 1024) {
    const int64_t v = base + threadIdx.x;
    const int64_t c = v < a.N ? (int64_t)a.deg[v] : 0;
    const int64_t incl = warp_inclusive_scan(c, lane);
    if (lane == 31) s_warp[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      const int64_t x = s_warp[lane];
      const int64_t xi = warp_inclusive_scan(x, lane);
      s_warp[lane] = xi - x;
    }
    __syncthreads();
    const int64_t carry = s_carry;
    if (v < a.N) a.indptr[v] = carry + s_warp[warp] + incl - c;
    __syncthreads();
    if (threadIdx.x == 1023) s_carry = carry + s_warp[warp] + incl;
    __syncthreads();
  }
  if (threadIdx.x == 0) a.indptr[a.N] = a.M;
}

struct SwOut {
  uint4* rec;            // next pass's input (not last)
  int32_t* nbr;          // last pass
  int32_t* eid;
  float* ts;
  uint32_t* keys;        // owners in T-CSR order (for indptr when deg is not kept) or NULL
  float* coarse;         // optional sampler indexes
  int4* entries;
};

template <bool kFirst, bool kLast>
__global__ void __launch_bounds__(kSwThreads, 2)
sw_scatter_kernel(SwArgs a, int p, const uint4* __restrict__ in, SwOut o,
                  uint32_t* __restrict__ status, unsigned int* ticket) {
  // the tile's records are staged in shared memory in (digit, rank) order, then written
  // out by consecutive threads: each digit's run of the tile lands as one contiguous,
  // coalesced stretch (instead of 16-byte / 4-byte stores scattered over 256 buckets)
  extern __shared__ uint4 s_rec[];              // [kSwTile]
  __shared__ uint32_t s_wrun[kSwWarps][256];
  __shared__ uint32_t s_base[256];
  __shared__ uint32_t s_loff[256];              // tile-local start of each digit's run
  __shared__ uint32_t s_wsum[kSwWarps];
  __shared__ int64_t s_tile;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int w = 0; w < kSwWarps; ++w) s_wrun[w][threadIdx.x] = 0;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t wbase = tile * kSwTile + warp * (32 * kSwIPT);
  const int field = a.field[p], shift = a.shift[p];
  uint4 rec[kSwIPT];
#pragma unroll
  for (int r = 0; r < kSwIPT; ++r) {
    const int64_t i = wbase + r * 32 + lane;
    if (i < a.M) rec[r] = kFirst ? sw_make_record(a, i) : in[i];
  }
  const unsigned lt = (1u << lane) - 1u;
  uint32_t rank[kSwIPT];
#pragma unroll
  for (int r = 0; r < kSwIPT; ++r) {
    const int64_t i = wbase + r * 32 + lane;
    const bool valid = i < a.M;
    const uint32_t d = valid ? sw_digit(rec[r], field, shift) : 0u;
    unsigned peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < 8; ++b) {
      const bool bit = (d >> b) & 1u;
      const unsigned bb = __ballot_sync(0xffffffffu, bit);
      peers &= bit ? bb : ~bb;
    }
    const uint32_t old = valid ? s_wrun[warp][d] : 0u;
    const uint32_t rk = __popc(peers & lt);
    __syncwarp();
    if (valid && rk == 0) s_wrun[warp][d] = old + __popc(peers);
    __syncwarp();
    rank[r] = old + rk;
  }
  __syncthreads();
  {
    const int d = threadIdx.x;
    uint32_t tot = 0;
#pragma unroll
    for (int w = 0; w < kSwWarps; ++w) {
      const uint32_t x = s_wrun[w][d];
      s_wrun[w][d] = tot;
      tot += x;
    }
    {   // exclusive scan of the tile's digit totals (one digit per thread)
      uint32_t v = tot;
#pragma unroll
      for (int o2 = 1; o2 < 32; o2 <<= 1) {
        const uint32_t n = __shfl_up_sync(0xffffffffu, v, o2);
        if (lane >= o2) v += n;
      }
      if (lane == 31) s_wsum[warp] = v;
      __syncthreads();
      uint32_t wo = 0;
      for (int w = 0; w < warp; ++w) wo += s_wsum[w];
      s_loff[d] = wo + v - tot;
    }
    uint32_t* st = status + tile * 256 + d;
    uint32_t excl = 0;
    if (tile == 0) {
      atomicExch(st, kSwPre | tot);
    } else {
      asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(st), "r"(kSwAgg | tot) : "memory");
      // walk back kSwWindow predecessors per step (independent loads in flight), consuming
      // published aggregates in order until an inclusive prefix; re-poll from the first
      // tile that has not published yet
      int64_t j = tile - 1;
      bool done = false;
      while (!done) {
        uint32_t v[kSwWindow];
#pragma unroll
        for (int u = 0; u < kSwWindow; ++u) {
          if (j - u >= 0) {
            asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];"
                         : "=r"(v[u]) : "l"(status + (j - u) * 256 + d) : "memory");
          } else {
            v[u] = kSwPre;
          }
        }
        int used = 0;
#pragma unroll
        for (int u = 0; u < kSwWindow; ++u) {
          if (done || used < u) continue;       // stopped at an earlier slot
          const uint32_t f = v[u] >> 30;
          if (f == 0) continue;                 // not published: re-poll from here
          excl += v[u] & kSwVal;
          used = u + 1;
          if (f == 2) done = true;
        }
        j -= used;
      }
      asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(st), "r"(kSwPre | (excl + tot))
                   : "memory");
    }
    s_base[d] = a.ghist[p * 256 + d] + excl;
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kSwIPT; ++r) {
    const int64_t i = wbase + r * 32 + lane;
    if (i >= a.M) continue;
    const uint32_t d = sw_digit(rec[r], field, shift);
    s_rec[s_loff[d] + s_wrun[warp][d] + rank[r]] = rec[r];
  }
  __syncthreads();
  const int64_t t0 = tile * kSwTile;
  const int nv = (int)((a.M - t0) < kSwTile ? (a.M - t0) : kSwTile);
  for (int x = threadIdx.x; x < nv; x += kSwThreads) {
    const uint4 rr = s_rec[x];
    const uint32_t d = sw_digit(rr, field, shift);
    const int64_t pos = (int64_t)s_base[d] + (uint32_t)(x - (int)s_loff[d]);
    if (!kLast) {
      o.rec[pos] = rr;
    } else {
      o.nbr[pos] = (int32_t)rr.y;
      o.eid[pos] = (int32_t)rr.z;
      o.ts[pos] = __uint_as_float(rr.w);
      if (o.keys) o.keys[pos] = rr.x;
      if (o.coarse && (pos & 31) == 0) o.coarse[pos >> 5] = __uint_as_float(rr.w);
      if (o.entries) o.entries[pos] = make_int4((int)rr.y, (int)rr.z, (int)rr.w, 0);
    }
  }
}

static int grid_for(int64_t n, int threads) {
  int64_t g = ceil_div(n > 0 ? n : 1, threads);
  int64_t cap = (int64_t)kNumSMs * 16;
  return (int)(g < cap ? g : cap);
}

}  // namespace tgl

using namespace tgl;

static tgl_status build_onesweep(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                                 const int32_t* dst, const float* t, bool undirected, bool sorted,
                                 int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts,
                                 float* ts_coarse, void* entries, void* ws, size_t* ws_bytes,
                                 cudaStream_t s) {
  const int64_t M = undirected ? 2 * num_edges : num_edges;
  SwArgs a{};
  a.M = M;
  a.N = num_nodes;
  a.undirected = undirected;
  a.src = src;
  a.dst = dst;
  a.t = t;
  int np = 0;
  if (!sorted)
    for (int sh = 0; sh < 32; sh += 8) a.field[np] = 0, a.shift[np++] = sh;
  int bits = 1;
  while (bits < 31 && ((int64_t)1 << bits) < num_nodes) ++bits;
  for (int sh = 0; sh < bits; sh += 8) a.field[np] = 1, a.shift[np++] = sh;
  a.npass = np;
  const bool deg = num_nodes <= kSwDegSmemNodes;
  const int64_t tiles = ceil_div(M > 0 ? M : 1, kSwTile);
  const int nbuf = np >= 3 ? 2 : (np == 2 ? 1 : 0);
  WsLayout L;
  const size_t o_rec0 = nbuf >= 1 ? L.take(16 * (size_t)M) : 0;
  const size_t o_rec1 = nbuf >= 2 ? L.take(16 * (size_t)M) : 0;
  const size_t o_keys = deg ? 0 : L.take(4 * (size_t)M);
  const size_t o_zero = L.take(0);
  const size_t o_status = L.take(4ull * 256 * tiles * np);
  const size_t o_ticket = L.take(4 * kSwMaxPasses);
  const size_t o_ghist = L.take(4 * 256 * kSwMaxPasses);
  const size_t o_deg = deg ? L.take(4 * (size_t)(num_nodes > 0 ? num_nodes : 1)) : L.off;
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  char* w = static_cast<char*>(ws);
  TGL_TRY(cuda_check(cudaMemsetAsync(w + o_zero, 0, L.off - o_zero, s), "tcsr workspace memset"));
  a.ghist = reinterpret_cast<uint32_t*>(w + o_ghist);
  a.deg = deg ? reinterpret_cast<uint32_t*>(w + o_deg) : nullptr;
  a.indptr = indptr;
  const size_t dsmem = deg ? 4 * (size_t)(num_nodes > 0 ? num_nodes : 1) : 0;
  {  // the default cap is 48 KB minus the static shared memory: always opt in
    static PerDeviceOnce once;
    TGL_TRY(cuda_check(once.run([] {
                         return cudaFuncSetAttribute(sw_hist_kernel,
                                                     cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                     (int)(kSwDegSmemNodes * 4));
                       }), "sw_hist smem attr"));
  }
  {
    static PerDeviceOnce once2;
    TGL_TRY(cuda_check(once2.run([] {
                         const int b = (int)(sizeof(uint4) * kSwTile);
                         cudaError_t e = cudaFuncSetAttribute(
                             sw_scatter_kernel<true, true>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, b);
                         if (e == cudaSuccess)
                           e = cudaFuncSetAttribute(sw_scatter_kernel<true, false>,
                                                    cudaFuncAttributeMaxDynamicSharedMemorySize, b);
                         if (e == cudaSuccess)
                           e = cudaFuncSetAttribute(sw_scatter_kernel<false, true>,
                                                    cudaFuncAttributeMaxDynamicSharedMemorySize, b);
                         if (e == cudaSuccess)
                           e = cudaFuncSetAttribute(sw_scatter_kernel<false, false>,
                                                    cudaFuncAttributeMaxDynamicSharedMemorySize, b);
                         return e;
                       }), "sw_scatter smem attr"));
  }
  const int hist_ctas = dsmem <= 100 * 1024 ? 2 * kNumSMs : kNumSMs;
  sw_hist_kernel<<<hist_ctas, 1024, dsmem, s>>>(a, num_edges);
  TGL_TRY(launch_check("tcsr sw_hist"));
  sw_bases_kernel<<<1, 1024, 0, s>>>(a);
  TGL_TRY(launch_check("tcsr sw_bases"));
  uint4* rec[2] = {reinterpret_cast<uint4*>(w + o_rec0), reinterpret_cast<uint4*>(w + o_rec1)};
  SwOut o{};
  for (int p = 0; p < np; ++p) {
    const bool first = p == 0, last = p == np - 1;
    const uint4* in = first ? nullptr : rec[(p - 1) & 1];
    o.rec = last ? nullptr : rec[p & 1];
    if (last) {
      o.nbr = nbr;
      o.eid = eid;
      o.ts = ts;
      o.keys = deg ? nullptr : reinterpret_cast<uint32_t*>(w + o_keys);
      o.coarse = ts_coarse;
      o.entries = static_cast<int4*>(entries);
    }
    uint32_t* status = reinterpret_cast<uint32_t*>(w + o_status) + (size_t)p * 256 * tiles;
    unsigned int* ticket = reinterpret_cast<unsigned int*>(w + o_ticket) + p;
    const dim3 grid((unsigned)tiles);
    const size_t rsm = sizeof(uint4) * kSwTile;    // the staged tile (64 KB)
    if (first && last)
      sw_scatter_kernel<true, true><<<grid, kSwThreads, rsm, s>>>(a, p, in, o, status, ticket);
    else if (first)
      sw_scatter_kernel<true, false><<<grid, kSwThreads, rsm, s>>>(a, p, in, o, status, ticket);
    else if (last)
      sw_scatter_kernel<false, true><<<grid, kSwThreads, rsm, s>>>(a, p, in, o, status, ticket);
    else
      sw_scatter_kernel<false, false><<<grid, kSwThreads, rsm, s>>>(a, p, in, o, status, ticket);
    TGL_TRY(launch_check("tcsr sw_scatter"));
  }
  if (!deg) {
    tcsr_indptr_kernel<<<grid_for(M + 1, 256), 256, 0, s>>>(
        M, num_nodes, reinterpret_cast<uint32_t*>(w + o_keys), indptr);
    TGL_TRY(launch_check("tcsr_indptr"));
  }
  return TGL_OK;
}

static tgl_status build_radix(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                              const int32_t* dst, const float* t, bool undirected, bool sorted,
                              int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts, void* ws,
                              size_t* ws_bytes, cudaStream_t s) {
  const int64_t M = undirected ? 2 * num_edges : num_edges;
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
  char* w = static_cast<char*>(ws);
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

extern "C" tgl_status tgl_build_tcsr_ex(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                                        const int32_t* dst, const float* t, uint32_t flags,
                                        int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts,
                                        float* ts_coarse, void* entries, void* ws,
                                        size_t* ws_bytes, void* stream) {
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
  TGL_REQUIRE(entries == nullptr || (reinterpret_cast<uintptr_t>(entries) & 15) == 0,
              "entries must be 16-byte aligned");
  cudaStream_t s = as_stream(stream);
  const bool onesweep = M < kSwVal;   // look-back counts carry 30 bits
  if (ws != nullptr) {
    TGL_REQUIRE(indptr != nullptr, "null indptr");
    TGL_REQUIRE(M == 0 || (src && dst && t && nbr && eid && ts), "null pointer");
    if (M == 0) {
      return cuda_check(cudaMemsetAsync(indptr, 0, sizeof(int64_t) * (num_nodes + 1), s),
                        "indptr memset");
    }
  }
  if (onesweep)
    return build_onesweep(num_nodes, num_edges, src, dst, t, undirected, sorted, indptr, nbr, eid,
                          ts, ts_coarse, entries, ws, ws_bytes, s);
  TGL_TRY(build_radix(num_nodes, num_edges, src, dst, t, undirected, sorted, indptr, nbr, eid, ts,
                      ws, ws_bytes, s));
  if (ws == nullptr || (ts_coarse == nullptr && entries == nullptr)) return TGL_OK;
  tgl_tcsr g{num_nodes, M, indptr, nbr, eid, ts, nullptr, nullptr};
  return tgl_tcsr_index(&g, ts_coarse, entries, stream);
}

extern "C" tgl_status tgl_build_tcsr(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                                     const int32_t* dst, const float* t, uint32_t flags,
                                     int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts,
                                     void* ws, size_t* ws_bytes, void* stream) {
  return tgl_build_tcsr_ex(num_nodes, num_edges, src, dst, t, flags, indptr, nbr, eid, ts,
                           nullptr, nullptr, ws, ws_bytes, stream);
}
