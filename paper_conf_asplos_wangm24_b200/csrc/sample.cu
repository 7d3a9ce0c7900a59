// sample.cu -- S4 temporal neighbourhood sampling (readings R1, R4-R7).
//
// Three launches, none of which waits on another CTA:
//  1. sample_count: one CTA = 32 queries (8 warps x 4 queries searched in lockstep, so
//     each round of dependent probes has 4 independent loads per lane).  Per query a
//     warp runs a 32-ary search for the first segment entry with !(ts < t) (monotone
//     predicate, so NaN t -> 0 candidates) and writes (start, n, min(n, k)).
//  2. sample_scan: exclusive scan of the counts into seg_ptr (decoupled look-back over
//     a few 2048-count tiles).
//  3. sample_pick: one thread per query; recent picks are contiguous loads, uniform
//     picks use Philox4x32-10 keyed by the query content (v, bits(t), layer, slot/4) so
//     dedup / sharding cannot change them (R6).
// (Round 1 fused the three with a look-back inside the search kernel: every wave of
// tiles finished its searches together and then walked the look-back 32 tiles per L2
// round trip -- 186 us for GDELT's 132k queries, ~3.5x the search itself.)
#include "common.cuh"

namespace tgl {

constexpr int kSampleWarps = 8;
constexpr int kQueriesPerWarp = 4;
constexpr int kSampleTile = kSampleWarps * kQueriesPerWarp;  // 32


// 32-ary lockstep narrowing of the warp's queries over a sorted array slice: every
// window [lo, hi) shrinks (one round of 32 probes per query, the queries' probes
// independent) until it holds <= 32 entries; pos = first index with !(arr < t) stays
// inside the window (monotone predicate, so NaN t -> pos = lo).
template <int Q>
__device__ __forceinline__ void narrow32(const float* __restrict__ arr, int64_t (&lo)[Q],
                                         int64_t (&hi)[Q], const float (&tq)[Q], int lane) {
  while (true) {
    bool any = false;
    float pv[Q];
    int64_t stepv[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) {                    // issue this round's probes
      stepv[j] = 0;
      pv[j] = 0.f;
      if (hi[j] - lo[j] > 32) {
        any = true;
        stepv[j] = (hi[j] - lo[j] + 31) >> 5;
        const int64_t jj = lo[j] + (int64_t)lane * stepv[j];
        if (jj < hi[j]) pv[j] = __ldg(arr + jj);
      }
    }
    if (!any) break;
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      if (stepv[j] == 0) continue;
      const int64_t jj = lo[j] + (int64_t)lane * stepv[j];
      const bool p = (jj < hi[j]) && (pv[j] < tq[j]);
      const int c = __popc(__ballot_sync(0xffffffffu, p));
      if (c == 0) {
        hi[j] = lo[j];                               // pos = lo
        continue;
      }
      const int64_t next = lo[j] + (int64_t)c * stepv[j];
      const int64_t new_lo = lo[j] + (int64_t)(c - 1) * stepv[j] + 1;
      hi[j] = (c < 32 && next < hi[j]) ? next : hi[j];
      lo[j] = new_lo;
    }
  }
}

// pos = lo + #{entries < t} of windows of <= 32 entries (one probe per lane)
template <int Q>
__device__ __forceinline__ void final32(const float* __restrict__ arr, int64_t (&lo)[Q],
                                        const int64_t (&hi)[Q], const float (&tq)[Q], int lane) {
  float fv[Q];
#pragma unroll
  for (int j = 0; j < Q; ++j) fv[j] = (lo[j] + lane < hi[j]) ? __ldg(arr + lo[j] + lane) : 0.f;
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    const bool p = (lo[j] + lane < hi[j]) && (fv[j] < tq[j]);
    lo[j] += __popc(__ballot_sync(0xffffffffu, p));
  }
}

__global__ void __launch_bounds__(kSampleWarps * 32, 4)
sample_count_kernel(const int64_t* __restrict__ indptr, const float* __restrict__ ts,
                    const float* __restrict__ coarse, int64_t nq_max, const int64_t* nq_dev,
                    const int32_t* __restrict__ qnode, const float* __restrict__ qtime, int k,
                    int64_t* __restrict__ qstart, int64_t* __restrict__ qn,
                    uint32_t* __restrict__ cnt) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nq = dev_count(nq_dev, nq_max);
  const int64_t q0 = (int64_t)blockIdx.x * kSampleTile;
  if (q0 >= nq) return;
  constexpr int Q = kQueriesPerWarp;
  int64_t lo[Q], hi[Q], st[Q], en[Q];
  float tq[Q];
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    const int64_t q = q0 + warp * Q + j;
    lo[j] = hi[j] = 0;
    tq[j] = 0.f;
    if (q < nq) {
      const int32_t v = __ldg(qnode + q);
      tq[j] = __ldg(qtime + q);
      lo[j] = __ldg(indptr + v);
      hi[j] = __ldg(indptr + v + 1);
    }
    st[j] = lo[j];
    en[j] = hi[j];
  }
  if (coarse != nullptr) {
    // coarse phase over ts_coarse[p] = ts[32 p] (1/32 of the entries, mostly L2-resident):
    // the segment's coarse slice is p in [cs, ce) = [ceil(s/32), ceil(e/32)); with
    // c = first p there with !(coarse[p] < t), pos lies in (32 (c-1), 32 c] -- one
    // 32-entry (128-byte aligned) window of the segment
    int64_t clo[Q], chi[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      const bool big = en[j] - st[j] > 32;
      clo[j] = big ? (st[j] + 31) >> 5 : 0;
      chi[j] = big ? (en[j] + 31) >> 5 : 0;
    }
    int64_t cs[Q], ce[Q];
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      cs[j] = clo[j];
      ce[j] = chi[j];
    }
    narrow32<Q>(coarse, clo, chi, tq, lane);
    final32<Q>(coarse, clo, chi, tq, lane);
#pragma unroll
    for (int j = 0; j < Q; ++j) {
      if (en[j] - st[j] <= 32) continue;
      const int64_t c = clo[j];
      lo[j] = c > cs[j] ? 32 * (c - 1) + 1 : st[j];
      hi[j] = c < ce[j] ? 32 * c : en[j];
      lo[j] = lo[j] < st[j] ? st[j] : lo[j];
      hi[j] = hi[j] > en[j] ? en[j] : hi[j];
    }
  }
  narrow32<Q>(ts, lo, hi, tq, lane);                 // no-op after the coarse phase
  final32<Q>(ts, lo, hi, tq, lane);
  // per-query results for the scan and the pick kernels
#pragma unroll
  for (int j = 0; j < Q; ++j) {
    const int64_t n = lo[j] - st[j];
    const int64_t q = q0 + warp * Q + j;
    if (lane == 0 && q < nq) {
      qstart[q] = st[j];
      qn[q] = n;
      cnt[q] = (uint32_t)(n < k ? n : k);
    }
  }
}

// Exclusive scan of the per-query counts into seg_ptr (int64), total in seg_ptr[nq]: single
// pass, decoupled look-back over tiles of kScanQ counts (a few tiles: short chains).
constexpr int kScanQThreads = 256, kScanQItems = 32, kScanQ = kScanQThreads * kScanQItems;

__global__ void __launch_bounds__(kScanQThreads)
sample_scan_kernel(int64_t nq_max, const int64_t* nq_dev, const uint32_t* __restrict__ cnt,
                   int64_t* __restrict__ seg_ptr, unsigned long long* status,
                   unsigned int* ticket) {
  pdl_wait();
  pdl_trigger();
  __shared__ int64_t s_tile;
  __shared__ int64_t s_warp[kScanQThreads / 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nq = dev_count(nq_dev, nq_max);
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  if (tile * kScanQ >= nq && !(tile == 0)) return;
  const int64_t base = tile * kScanQ + (int64_t)threadIdx.x * kScanQItems;
  uint32_t v[kScanQItems];
  int64_t sum = 0;
#pragma unroll
  for (int r = 0; r < kScanQItems; ++r) {
    v[r] = (base + r < nq) ? cnt[base + r] : 0u;
    sum += v[r];
  }
  const int64_t incl = warp_inclusive_scan(sum, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const int64_t wv = lane < kScanQThreads / 32 ? s_warp[lane] : 0;
    const int64_t wincl = warp_inclusive_scan(wv, lane);
    const int64_t agg = __shfl_sync(0xffffffffu, wincl, 31);
    const int64_t excl_tile = lookback(status, tile, agg, lane);
    if (lane < kScanQThreads / 32) s_warp[lane] = excl_tile + wincl - wv;
  }
  __syncthreads();
  int64_t run = s_warp[warp] + incl - sum;
#pragma unroll
  for (int r = 0; r < kScanQItems; ++r) {
    if (base + r < nq) seg_ptr[base + r] = run;
    run += v[r];
    if (base + r == nq - 1) seg_ptr[nq] = run;
  }
  if (nq == 0 && tile == 0 && threadIdx.x == 0) seg_ptr[0] = 0;
}

// Picks: a group of G lanes per query (G = the power of two >= max(k, 4), <= 32; lane s
// of the group takes slot s, s + G, ...), so a query's outputs are written by
// consecutive lanes.  Recent picks are the last cnt candidates in CSR order; uniform
// picks use Philox4x32-10 keyed by the query content (v, bits(t), layer, slot/4) (R6):
// the lane holding slot 4b computes block b and hands words 1-3 to its 3 neighbours.
// With the packed entry array (tgl_tcsr.entries) one 16-byte load fetches nbr, eid
// and ts of a picked entry (one DRAM sector instead of three).
template <int G>
__global__ void __launch_bounds__(256)
sample_pick_kernel(const int32_t* __restrict__ nbr, const int32_t* __restrict__ eid,
                   const float* __restrict__ ts, const int4* __restrict__ entries,
                   int64_t nq_max, const int64_t* nq_dev, const int32_t* __restrict__ qnode,
                   const float* __restrict__ qtime, int k, int strategy, uint2 key,
                   uint32_t layer, const int64_t* __restrict__ seg_ptr,
                   const int64_t* __restrict__ qstart, const int64_t* __restrict__ qn,
                   int32_t* __restrict__ out_nbr, int32_t* __restrict__ out_eid,
                   float* __restrict__ out_ts) {
  pdl_wait();
  pdl_trigger();
  const int64_t nq = dev_count(nq_dev, nq_max);
  const int lane = threadIdx.x & 31;
  const int s0 = lane & (G - 1);
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t groups = (int64_t)gridDim.x * (blockDim.x / G);
  for (int64_t q = blockIdx.x * (int64_t)(blockDim.x / G) + threadIdx.x / G; q < nq;
       q += groups) {                                 // (q is uniform in a lane group)
    const int64_t start = qstart[q], n = qn[q], o = seg_ptr[q];
    const int cnt = (int)(n < k ? n : k);
    const bool draw = strategy == TGL_UNIFORM && n > k;
    uint32_t v = 0, tb = 0;
    if (draw) {
      v = (uint32_t)__ldg(qnode + q);
      tb = time_key_bits(__ldg(qtime + q));
    }
    for (int sb = 0; sb < cnt; sb += G) {            // warp-uniform within the group
      const int s = sb + s0;
      int64_t jj;
      if (!draw) {
        jj = start + (n - cnt) + s;
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
      if (s < cnt) {
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
  const int64_t nq1 = nq_max > 0 ? nq_max : 1;
  const int64_t tiles = ceil_div(nq1, kSampleTile);
  const int64_t scan_tiles = ceil_div(nq1, kScanQ);
  WsLayout L;
  const size_t o_start = L.take(sizeof(int64_t) * nq1);
  const size_t o_n = L.take(sizeof(int64_t) * nq1);
  const size_t o_cnt = L.take(sizeof(uint32_t) * nq1);
  const size_t o_status = L.take(sizeof(unsigned long long) * scan_tiles);
  const size_t o_ticket = L.take(sizeof(unsigned int));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(seg_ptr != nullptr, "null seg_ptr");
  TGL_REQUIRE(nq_max == 0 || (qnode && qtime && out_nbr && out_eid && out_ts), "null pointer");
  TGL_REQUIRE(g->indptr && (g->num_entries == 0 || (g->nbr && g->eid && g->ts)), "null graph array");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  auto qstart = reinterpret_cast<int64_t*>(w + o_start);
  auto qn = reinterpret_cast<int64_t*>(w + o_n);
  auto cnt = reinterpret_cast<uint32_t*>(w + o_cnt);
  TGL_TRY(cuda_check(cudaMemsetAsync(w + o_status, 0, L.off - o_status, s), "sample memset"));
  uint2 key = make_uint2((uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32));
  launch_pdl(sample_count_kernel, dim3((unsigned)tiles), dim3(kSampleWarps * 32), 0, s,
             g->indptr, g->ts, g->ts_coarse, nq_max, nq_dev, qnode, qtime, k, qstart, qn, cnt);
  TGL_TRY(launch_check("sample_count"));
  launch_pdl(sample_scan_kernel, dim3((unsigned)scan_tiles), dim3(kScanQThreads), 0, s, nq_max,
             nq_dev, cnt, seg_ptr, reinterpret_cast<unsigned long long*>(w + o_status),
             reinterpret_cast<unsigned int*>(w + o_ticket));
  TGL_TRY(launch_check("sample_scan"));
  const int G = k <= 4 ? 4 : k <= 8 ? 8 : k <= 16 ? 16 : 32;
  int64_t gp = ceil_div(nq1, 256 / G);
  if (gp > (int64_t)kNumSMs * 16) gp = (int64_t)kNumSMs * 16;
  auto pick = G == 4 ? sample_pick_kernel<4> : G == 8 ? sample_pick_kernel<8>
            : G == 16 ? sample_pick_kernel<16> : sample_pick_kernel<32>;
  launch_pdl(pick, dim3((unsigned)gp), dim3(256), 0, s, g->nbr, g->eid, g->ts,
             reinterpret_cast<const int4*>(g->entries), nq_max, nq_dev, qnode, qtime, k,
             strategy, key, layer, seg_ptr, qstart, qn, out_nbr, out_eid, out_ts);
  return launch_check("sample_pick");
}
