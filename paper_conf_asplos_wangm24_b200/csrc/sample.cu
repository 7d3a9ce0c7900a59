// sample.cu -- S4 temporal neighbourhood sampling (readings R1, R4-R7).
//
// Two launches, neither of which waits on another CTA:
//  1. sample_count: one CTA = a tile of 8 warps x Q queries searched in lockstep (each
//     round of dependent probes has Q independent loads per lane).  Per query a warp
//     runs a 32-ary search for the first segment entry with !(ts < t) (monotone
//     predicate, so NaN t -> 0 candidates) and writes (start, n, min(n, k)); the tile
//     writes the sum of its min(n, k).  Entry indices are 32-bit (the T-CSR holds < 2^32
//     entries), which keeps Q = 8 queries per warp in registers.
//  2. sample_pick: one CTA per count tile.  Its output offset is the sum of the earlier
//     tiles' sums (read straight from L2: <= a few thousand words, no look-back chain and
//     no scan launch); it writes seg_ptr for its queries, then picks -- recent picks are
//     contiguous loads, uniform picks use Philox4x32-10 keyed by the query content
//     (v, bits(t), layer, slot/4) so dedup / sharding cannot change them (R6).
// (Round 1 fused the search with a look-back scan: every wave of tiles finished its
// searches together and then walked the look-back 32 tiles per L2 round trip -- 186 us for
// GDELT's 132k queries.  Round 2 split it into count / scan / pick launches.)
#include "common.cuh"

namespace tgl {

constexpr int kSampleWarps = 8;
#ifndef TGL_SAMPLE_Q
#define TGL_SAMPLE_Q 4
#endif
#ifndef TGL_SAMPLE_MINB
#define TGL_SAMPLE_MINB 6
#endif
constexpr int kQueriesPerWarp = TGL_SAMPLE_Q;
constexpr int kSampleTile = kSampleWarps * kQueriesPerWarp;  // 32
constexpr int kPickTile = 64;      // queries per pick CTA (a whole number of count tiles)
static_assert(kPickTile % kSampleTile == 0 && kPickTile <= 64, "pick tile: <= 2 warps of counts");
constexpr int kSuperTiles = 64;    // agg2[j] = sum of agg over tiles [64 j, 64 j + 64)

// 32-ary lockstep narrowing of the warp's queries over a sorted array slice: every
// window [lo, hi) shrinks (one round of 32 probes per query, the queries' probes
// independent) until it holds <= 32 entries; pos = first index with !(arr < t) stays
// inside the window (monotone predicate, so NaN t -> pos = lo).
template <int Q>
__device__ __forceinline__ void narrow32(const float* __restrict__ arr, uint32_t (&lo)[Q],
                                         uint32_t (&hi)[Q], const float (&tq)[Q], int lane) {
  while (true) {
    bool any = false;
    float pv[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) {                    // issue this round's probes
      pv[j] = 0.f;
      if (hi[j] - lo[j] > 32) {
        any = true;
        const uint32_t step = (hi[j] - lo[j] + 31) >> 5;
        const uint32_t jj = lo[j] + (uint32_t)lane * step;
        if (jj < hi[j]) pv[j] = __ldg(arr + jj);
      }
    }
    if (!any) break;
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      if (hi[j] - lo[j] <= 32) continue;
      const uint32_t step = (hi[j] - lo[j] + 31) >> 5;
      const uint32_t jj = lo[j] + (uint32_t)lane * step;
      const bool p = (jj < hi[j]) && (pv[j] < tq[j]);
      const uint32_t c = __popc(__ballot_sync(0xffffffffu, p));
      if (c == 0) {
        hi[j] = lo[j];                               // pos = lo
        continue;
      }
      const uint64_t next = (uint64_t)lo[j] + (uint64_t)c * step;
      const uint32_t new_lo = lo[j] + (c - 1) * step + 1;
      hi[j] = (c < 32 && next < hi[j]) ? (uint32_t)next : hi[j];
      lo[j] = new_lo;
    }
  }
}

// pos = lo + #{entries < t} of windows of <= 32 entries (one probe per lane)
template <int Q>
__device__ __forceinline__ void final32(const float* __restrict__ arr, uint32_t (&lo)[Q],
                                        const uint32_t (&hi)[Q], const float (&tq)[Q], int lane) {
  float fv[Q];
#pragma unroll
  for (int j = 0; j < Q; ++j) fv[j] = (lo[j] + lane < hi[j]) ? __ldg(arr + lo[j] + lane) : 0.f;
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    const bool p = (lo[j] + lane < hi[j]) && (fv[j] < tq[j]);
    lo[j] += __popc(__ballot_sync(0xffffffffu, p));
  }
}

__global__ void __launch_bounds__(kSampleWarps * 32, TGL_SAMPLE_MINB)
sample_count_kernel(const int64_t* __restrict__ indptr, const float* __restrict__ ts,
                    const float* __restrict__ coarse, int64_t nq_max, const int64_t* nq_dev,
                    const int32_t* __restrict__ qnode, const float* __restrict__ qtime, int k,
                    uint32_t* __restrict__ qstart, uint32_t* __restrict__ qn,
                    uint32_t* __restrict__ cnt, unsigned long long* __restrict__ agg,
                    unsigned long long* __restrict__ agg2) {
  __shared__ unsigned long long s_agg[kSampleWarps];
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nq = dev_count(nq_dev, nq_max);
  const int64_t q0 = (int64_t)blockIdx.x * kSampleTile;
  if (q0 >= nq) return;
  constexpr int Q = kQueriesPerWarp;
  uint32_t lo[Q], hi[Q], st[Q], en[Q];
  float tq[Q];
  int32_t vq[Q];
#pragma unroll
  for (int j = 0; j < Q; ++j) {                      // node / time loads first (independent)
    const int64_t q = q0 + warp * Q + j;
    vq[j] = q < nq ? __ldg(qnode + q) : -1;
    tq[j] = q < nq ? __ldg(qtime + q) : 0.f;
  }
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    lo[j] = vq[j] >= 0 ? (uint32_t)__ldg(indptr + vq[j]) : 0u;
    hi[j] = vq[j] >= 0 ? (uint32_t)__ldg(indptr + vq[j] + 1) : 0u;
    st[j] = lo[j];
    en[j] = hi[j];
  }
  if (coarse != nullptr) {
    // coarse phase over ts_coarse[p] = ts[32 p] (1/32 of the entries, mostly L2-resident):
    // the segment's coarse slice is p in [cs, ce) = [ceil(s/32), ceil(e/32)); with
    // c = first p there with !(coarse[p] < t), pos lies in (32 (c-1), 32 c] -- one
    // 32-entry (128-byte aligned) window of the segment
    uint32_t clo[Q], chi[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      const bool big = en[j] - st[j] > 32;
      clo[j] = big ? (uint32_t)(((uint64_t)st[j] + 31) >> 5) : 0u;
      chi[j] = big ? (uint32_t)(((uint64_t)en[j] + 31) >> 5) : 0u;
    }
    uint32_t cs[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) cs[j] = clo[j];
    narrow32<Q>(coarse, clo, chi, tq, lane);
    final32<Q>(coarse, clo, chi, tq, lane);
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      if (en[j] - st[j] <= 32) continue;
      const uint32_t c = clo[j];
      const uint32_t ce = (uint32_t)(((uint64_t)en[j] + 31) >> 5);
      const uint64_t l = c > cs[j] ? 32ull * (c - 1) + 1 : st[j];
      const uint64_t h = c < ce ? 32ull * c : en[j];
      lo[j] = l < st[j] ? st[j] : (uint32_t)l;
      hi[j] = h > en[j] ? en[j] : (uint32_t)h;
    }
  }
  narrow32<Q>(ts, lo, hi, tq, lane);                 // no-op after the coarse phase
  final32<Q>(ts, lo, hi, tq, lane);
  // per-query results for the pick kernel, and the tile's sum of min(n, k)
  unsigned long long wsum = 0;
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    const uint32_t n = lo[j] - st[j];
    const uint32_t c = n < (uint32_t)k ? n : (uint32_t)k;
    const int64_t q = q0 + warp * Q + j;
    if (q < nq) {
      wsum += c;
      if (lane == 0) {
        qstart[q] = st[j];
        qn[q] = n;
        cnt[q] = c;
      }
    }
  }
  if (lane == 0) s_agg[warp] = wsum;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
#pragma unroll
    for (int w = 0; w < kSampleWarps; ++w) t += s_agg[w];
    agg[blockIdx.x] = t;
    atomicAdd(agg2 + blockIdx.x / kSuperTiles, t);
  }
}

// Picks: CTA b takes count tile b.  Offset of the tile = sum of agg[0, b) (coalesced L2
// reads, block reduction); the tile's 64 offsets by a two-warp scan; seg_ptr written here.
// A group of G lanes per query (G = the power of two >= max(k, 4), <= 32; lane s of the
// group takes slot s, s + G, ...), so a query's outputs are written by consecutive lanes.
// Recent picks are the last cnt candidates in CSR order; uniform picks use
// Philox4x32-10 keyed by the query content (v, bits(t), layer, slot/4) (R6): the lane
// holding slot 4b computes block b and hands words 1-3 to its 3 neighbours.  With the
// packed entry array (tgl_tcsr.entries) one 16-byte load fetches nbr, eid and ts of a
// picked entry (one DRAM sector instead of three).
template <int G>
__global__ void __launch_bounds__(256)
sample_pick_kernel(const int32_t* __restrict__ nbr, const int32_t* __restrict__ eid,
                   const float* __restrict__ ts, const int4* __restrict__ entries,
                   int64_t nq_max, const int64_t* nq_dev, const int32_t* __restrict__ qnode,
                   const float* __restrict__ qtime, int k, int strategy, uint2 key,
                   uint32_t layer, const unsigned long long* __restrict__ agg,
                   const unsigned long long* __restrict__ agg2,
                   const uint32_t* __restrict__ qstart, const uint32_t* __restrict__ qn,
                   const uint32_t* __restrict__ cnt, int64_t* __restrict__ seg_ptr,
                   int32_t* __restrict__ out_nbr, int32_t* __restrict__ out_eid,
                   float* __restrict__ out_ts) {
  __shared__ unsigned long long s_red[8];
  __shared__ int64_t s_off[kPickTile];
  __shared__ int64_t s_w0;
  pdl_wait();
  pdl_trigger();
  const int64_t nq = dev_count(nq_dev, nq_max);
  const int64_t q0 = (int64_t)blockIdx.x * kPickTile;
  if (nq == 0) {
    if (blockIdx.x == 0 && threadIdx.x == 0) seg_ptr[0] = 0;
    return;
  }
  if (q0 >= nq) return;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  {
    // tiles before this one: whole super-tiles from agg2, the rest of this super-tile
    // from agg (<= 64 + 63 words, whatever the number of tiles)
    unsigned long long part = 0;
    const int64_t ct = (int64_t)blockIdx.x * (kPickTile / kSampleTile);   // first count tile
    const int64_t sup = ct / kSuperTiles, t0 = sup * kSuperTiles;
    for (int64_t i = threadIdx.x; i < sup; i += blockDim.x) part += agg2[i];
    for (int64_t i = t0 + threadIdx.x; i < ct; i += blockDim.x) part += agg[i];
    part = warp_sum(part);
    if (lane == 0) s_red[warp] = part;
  }
  int64_t c_own = 0, incl = 0;
  if (threadIdx.x < kPickTile) {                      // warps 0-1: the tile's counts
    const int64_t q = q0 + threadIdx.x;
    c_own = q < nq ? (int64_t)cnt[q] : 0;
    incl = warp_inclusive_scan(c_own, lane);
    if (threadIdx.x == 31) s_w0 = incl;               // warp 0's total
  }
  __syncthreads();
  if (threadIdx.x < kPickTile) {
    int64_t base = warp == 1 ? s_w0 : 0;
#pragma unroll
    for (int w = 0; w < 8; ++w) base += (int64_t)s_red[w];
    s_off[threadIdx.x] = base + incl - c_own;
  }
  __syncthreads();
  if (threadIdx.x < kPickTile) {
    const int64_t q = q0 + threadIdx.x;
    if (q < nq) {
      seg_ptr[q] = s_off[threadIdx.x];
      if (q == nq - 1) seg_ptr[nq] = s_off[threadIdx.x] + c_own;
    }
  }
  const int s0 = lane & (G - 1);
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  // (measured: issuing the loads of 2 or 4 queries per group ahead raised registers to
  // 64 / 127 and lost more occupancy than it gained ILP: 38 / 50 us vs 33 us on GDELT)
  for (int qi = threadIdx.x / G; qi < kPickTile; qi += blockDim.x / G) {
    const int64_t q = q0 + qi;                        // (q is uniform in a lane group)
    if (q >= nq) break;
    const int64_t start = qstart[q], n = qn[q], o = s_off[qi];
    const int c = (int)(n < k ? n : k);
    const bool draw = strategy == TGL_UNIFORM && n > k;
    uint32_t v = 0, tb = 0;
    if (draw) {
      v = (uint32_t)__ldg(qnode + q);
      tb = time_key_bits(__ldg(qtime + q));
    }
    for (int sb = 0; sb < c; sb += G) {              // warp-uniform within the group
      const int s = sb + s0;
      int64_t jj;
      if (!draw) {
        jj = start + (n - c) + s;
      } else {
        uint4 r4 = make_uint4(0, 0, 0, 0);
        if ((s & 3) == 0) r4 = philox4x32_10(make_uint4(v, tb, layer, (uint32_t)(s >> 2)), key);
        const int src = lane & ~3;                   // the group's lane holding slot 4b
        const uint32_t w1 = __shfl_sync(gmask, r4.y, src);
        const uint32_t w2 = __shfl_sync(gmask, r4.z, src);
        const uint32_t w3 = __shfl_sync(gmask, r4.w, src);
        const uint32_t r = (s & 3) == 0 ? r4.x : (s & 3) == 1 ? w1 : (s & 3) == 2 ? w2 : w3;
        jj = start + (int64_t)(((uint64_t)r * (uint64_t)n) >> 32);
      }
      if (s < c) {
        if (entries != nullptr) {
          const int4 e = __ldg(entries + jj);
          out_nbr[o + s] = e.x;
          out_eid[o + s] = e.y;
          out_ts[o + s] = __int_as_float(e.z);
        } else {
          out_nbr[o + s] = __ldg(nbr + jj);
          out_eid[o + s] = __ldg(eid + jj);
          out_ts[o + s] = __ldg(ts + jj);
        }
      }
    }
  }
}

__global__ void tcsr_index_kernel(int64_t M, const int32_t* __restrict__ nbr,
                                  const int32_t* __restrict__ eid, const float* __restrict__ ts,
                                  float* __restrict__ coarse, int4* __restrict__ entries) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < M;
       p += (int64_t)gridDim.x * blockDim.x) {
    const float t = __ldg(ts + p);
    if (coarse != nullptr && (p & 31) == 0) coarse[p >> 5] = t;
    if (entries != nullptr)
      entries[p] = make_int4(__ldg(nbr + p), __ldg(eid + p), __float_as_int(t), 0);
  }
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_tcsr_index(const tgl_tcsr* g, float* ts_coarse, void* entries,
                                     void* stream) {
  TGL_REQUIRE(g != nullptr && g->num_entries >= 0, "bad graph");
  const int64_t M = g->num_entries;
  if (M == 0 || (ts_coarse == nullptr && entries == nullptr)) return TGL_OK;
  TGL_REQUIRE(g->nbr && g->eid && g->ts, "null graph array");
  TGL_REQUIRE(entries == nullptr || (reinterpret_cast<uintptr_t>(entries) & 15) == 0,
              "entries must be 16-byte aligned");
  int64_t gr = ceil_div(M, 256);
  if (gr > (int64_t)kNumSMs * 16) gr = (int64_t)kNumSMs * 16;
  tcsr_index_kernel<<<(unsigned)gr, 256, 0, as_stream(stream)>>>(
      M, g->nbr, g->eid, g->ts, ts_coarse, static_cast<int4*>(entries));
  return launch_check("tcsr_index");
}

extern "C" tgl_status tgl_sample(const tgl_tcsr* g, int64_t nq_max, const int64_t* nq_dev,
                                 const int32_t* qnode, const float* qtime, int32_t k,
                                 int32_t strategy, uint64_t seed, uint32_t layer,
                                 int64_t* seg_ptr, int32_t* out_nbr, int32_t* out_eid,
                                 float* out_ts, void* ws, size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(g != nullptr, "null graph");
  TGL_REQUIRE(nq_max >= 0, "negative nq_max");
  TGL_REQUIRE(k > 0, "k must be > 0");
  TGL_REQUIRE(strategy == TGL_RECENT || strategy == TGL_UNIFORM, "unknown strategy %d", strategy);
  TGL_REQUIRE(g->num_entries < ((int64_t)1 << 32), "T-CSR with >= 2^32 entries");
  const int64_t nq1 = nq_max > 0 ? nq_max : 1;
  const int64_t tiles = ceil_div(nq1, kSampleTile);
  WsLayout L;
  const size_t o_start = L.take(sizeof(uint32_t) * nq1);
  const size_t o_n = L.take(sizeof(uint32_t) * nq1);
  const size_t o_cnt = L.take(sizeof(uint32_t) * nq1);
  const size_t o_agg = L.take(sizeof(unsigned long long) * tiles);
  const size_t o_agg2 = L.take(sizeof(unsigned long long) * ceil_div(tiles, kSuperTiles));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(seg_ptr != nullptr, "null seg_ptr");
  TGL_REQUIRE(nq_max == 0 || (qnode && qtime && out_nbr && out_eid && out_ts), "null pointer");
  TGL_REQUIRE(g->indptr && (g->num_entries == 0 || (g->nbr && g->eid && g->ts)), "null graph array");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  auto qstart = reinterpret_cast<uint32_t*>(w + o_start);
  auto qn = reinterpret_cast<uint32_t*>(w + o_n);
  auto cnt = reinterpret_cast<uint32_t*>(w + o_cnt);
  auto agg = reinterpret_cast<unsigned long long*>(w + o_agg);
  auto agg2 = reinterpret_cast<unsigned long long*>(w + o_agg2);
  TGL_TRY(cuda_check(cudaMemsetAsync(agg2, 0, L.off - o_agg2, s), "sample agg2 memset"));
  uint2 key = make_uint2((uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32));
  launch_pdl(sample_count_kernel, dim3((unsigned)tiles), dim3(kSampleWarps * 32), 0, s,
             g->indptr, g->ts, g->ts_coarse, nq_max, nq_dev, qnode, qtime, k, qstart, qn, cnt,
             agg, agg2);
  TGL_TRY(launch_check("sample_count"));
  const int G = k <= 4 ? 4 : k <= 8 ? 8 : k <= 16 ? 16 : 32;
  auto pick = G == 4 ? sample_pick_kernel<4> : G == 8 ? sample_pick_kernel<8>
            : G == 16 ? sample_pick_kernel<16> : sample_pick_kernel<32>;
  launch_pdl(pick, dim3((unsigned)ceil_div(nq1, kPickTile)), dim3(256), 0, s, g->nbr, g->eid,
             g->ts,
             reinterpret_cast<const int4*>(g->entries), nq_max, nq_dev, qnode, qtime, k,
             strategy, key, layer, (const unsigned long long*)agg,
             (const unsigned long long*)agg2, (const uint32_t*)qstart,
             (const uint32_t*)qn, (const uint32_t*)cnt, seg_ptr, out_nbr, out_eid, out_ts);
  return launch_check("sample_pick");
}
