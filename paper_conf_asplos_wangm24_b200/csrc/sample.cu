// sample.cu -- S4 temporal neighbourhood sampling (readings R1, R4-R7).
//
// One CTA = one tile of 32 queries (8 warps x 4 queries searched in lockstep, so
// each round of dependent probes has 4 independent loads per lane), tiles taken from an
// atomic ticket.  Per query a warp runs a 32-ary search for the first segment
// entry with !(ts < t) (monotone predicate, so NaN t -> 0 candidates), then the
// tile's counts are prefix-summed with a decoupled look-back so `seg_ptr` and
// the compact outputs are produced in ONE launch (no count pass, no host sync).
// Recent picks are contiguous loads; uniform picks use Philox4x32-10 keyed by
// the query content (v, bits(t), layer, slot/4) so dedup / sharding cannot
// change them (R6).  The kernel is latency-bound (dependent probes): many
// independent queries in flight per SM is what matters.
#include "common.cuh"

namespace tgl {

constexpr int kSampleWarps = 8;
constexpr int kQueriesPerWarp = 4;
constexpr int kSampleTile = kSampleWarps * kQueriesPerWarp;  // 32

__device__ __forceinline__ int64_t warp_lower_time(const float* __restrict__ ts, int64_t lo,
                                                   int64_t hi, float t, int lane) {
  // returns pos = lo + #{j in [lo,hi): ts[j] < t}  (ts sorted inside the segment)
  while (hi - lo > 32) {
    int64_t step = (hi - lo + 31) >> 5;
    int64_t j = lo + (int64_t)lane * step;
    bool p = (j < hi) && (__ldg(ts + j) < t);
    unsigned b = __ballot_sync(0xffffffffu, p);
    int c = __popc(b);
    if (c == 0) return lo;
    int64_t next = lo + (int64_t)c * step;
    int64_t new_lo = lo + (int64_t)(c - 1) * step + 1;
    hi = (c < 32 && next < hi) ? next : hi;
    lo = new_lo;
  }
  bool p = (lo + lane < hi) && (__ldg(ts + lo + lane) < t);
  return lo + __popc(__ballot_sync(0xffffffffu, p));
}

__global__ void __launch_bounds__(kSampleWarps * 32)
sample_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ nbr,
              const int32_t* __restrict__ eid, const float* __restrict__ ts, int64_t nq_max,
              const int64_t* nq_dev, const int32_t* __restrict__ qnode,
              const float* __restrict__ qtime, int k, int strategy, uint2 key, uint32_t layer,
              int64_t* __restrict__ seg_ptr, int32_t* __restrict__ out_nbr,
              int32_t* __restrict__ out_eid, float* __restrict__ out_ts,
              unsigned long long* status, unsigned int* ticket) {
  pdl_wait();     // PDL: predecessor grid complete, its writes visible
  pdl_trigger();
  __shared__ int64_t s_tile;
  __shared__ int64_t s_start[kSampleTile];
  __shared__ int64_t s_n[kSampleTile];
  __shared__ int64_t s_off[kSampleTile];
  __shared__ int32_t s_cnt[kSampleTile];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t nq = dev_count(nq_dev, nq_max);
  const int64_t q0 = tile * kSampleTile;
  if (q0 >= nq) {
    if (tile == 0 && threadIdx.x == 0) seg_ptr[0] = 0;  // nq == 0
    return;
  }

  // phase 1: search -- the warp's 4 queries advance together (one 32-ary narrowing
  // round per iteration, the 4 probes of a round independent), then the final window
  int64_t lo[kQueriesPerWarp], hi[kQueriesPerWarp], st[kQueriesPerWarp];
  float tq[kQueriesPerWarp];
#pragma unroll
  for (int j = 0; j < kQueriesPerWarp; ++j) {
    const int64_t q = q0 + warp * kQueriesPerWarp + j;
    lo[j] = hi[j] = 0;
    tq[j] = 0.f;
    if (q < nq) {
      const int32_t v = __ldg(qnode + q);
      tq[j] = __ldg(qtime + q);
      lo[j] = __ldg(indptr + v);
      hi[j] = __ldg(indptr + v + 1);
    }
    st[j] = lo[j];
  }
  while (true) {
    bool any = false;
    float pv[kQueriesPerWarp];
    int64_t stepv[kQueriesPerWarp];
#pragma unroll
    for (int j = 0; j < kQueriesPerWarp; ++j) {      // issue this round's probes
      stepv[j] = 0;
      pv[j] = 0.f;
      if (hi[j] - lo[j] > 32) {
        any = true;
        stepv[j] = (hi[j] - lo[j] + 31) >> 5;
        const int64_t jj = lo[j] + (int64_t)lane * stepv[j];
        if (jj < hi[j]) pv[j] = __ldg(ts + jj);
      }
    }
    if (!any) break;
#pragma unroll
    for (int j = 0; j < kQueriesPerWarp; ++j) {
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
  float fv[kQueriesPerWarp];
#pragma unroll
  for (int j = 0; j < kQueriesPerWarp; ++j)          // final windows (<= 32 entries)
    fv[j] = (lo[j] + lane < hi[j]) ? __ldg(ts + lo[j] + lane) : 0.f;
#pragma unroll
  for (int j = 0; j < kQueriesPerWarp; ++j) {
    const bool p = (lo[j] + lane < hi[j]) && (fv[j] < tq[j]);
    const int64_t n = lo[j] + __popc(__ballot_sync(0xffffffffu, p)) - st[j];
    const int lq = warp * kQueriesPerWarp + j;
    if (lane == 0) {
      s_start[lq] = st[j];
      s_n[lq] = n;
      s_cnt[lq] = (int32_t)(n < k ? n : k);
    }
  }
  __syncthreads();

  // phase 2: tile prefix (warp 0) + decoupled look-back across tiles
  if (warp == 0) {
    int64_t c = s_cnt[lane];
    int64_t incl = warp_inclusive_scan(c, lane);
    int64_t agg = __shfl_sync(0xffffffffu, incl, 31);
    int64_t excl_tile = lookback(status, tile, agg, lane);
    int64_t off = excl_tile + incl - c;
    s_off[lane] = off;
    const int64_t q = q0 + lane;
    if (q < nq) seg_ptr[q] = off;
    if (q == nq - 1) seg_ptr[nq] = off + c;
  }
  __syncthreads();

  // phase 3: picks
#pragma unroll 1
  for (int j = 0; j < kQueriesPerWarp; ++j) {
    const int lq = warp * kQueriesPerWarp + j;
    const int64_t q = q0 + lq;
    if (q >= nq) break;
    const int cnt = s_cnt[lq];
    const int64_t start = s_start[lq], n = s_n[lq], o = s_off[lq];
    const bool draw = (strategy == TGL_UNIFORM) && (n > k);
    uint32_t v = 0, tb = 0;
    if (draw) {
      v = (uint32_t)__ldg(qnode + q);
      tb = time_key_bits(__ldg(qtime + q));
    }
    for (int s = lane; s < cnt; s += 32) {
      int64_t jj;
      if (!draw) {
        jj = start + (n - cnt) + s;
      } else {
        uint4 r4 = philox4x32_10(make_uint4(v, tb, layer, (uint32_t)(s >> 2)), key);
        uint32_t r = (s & 3) == 0 ? r4.x : (s & 3) == 1 ? r4.y : (s & 3) == 2 ? r4.z : r4.w;
        jj = start + (int64_t)(((uint64_t)r * (uint64_t)n) >> 32);
      }
      out_nbr[o + s] = __ldg(nbr + jj);
      out_eid[o + s] = __ldg(eid + jj);
      out_ts[o + s] = __ldg(ts + jj);
    }
  }
}

}  // namespace tgl

using namespace tgl;

extern "C" tgl_status tgl_sample(const tgl_tcsr* g, int64_t nq_max, const int64_t* nq_dev,
                                 const int32_t* qnode, const float* qtime, int32_t k,
                                 int32_t strategy, uint64_t seed, uint32_t layer,
                                 int64_t* seg_ptr, int32_t* out_nbr, int32_t* out_eid,
                                 float* out_ts, void* ws, size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(g != nullptr, "null graph");
  TGL_REQUIRE(nq_max >= 0, "negative nq_max");
  TGL_REQUIRE(k > 0, "k must be > 0");
  TGL_REQUIRE(strategy == TGL_RECENT || strategy == TGL_UNIFORM, "unknown strategy %d", strategy);
  const int64_t tiles = ceil_div(nq_max > 0 ? nq_max : 1, kSampleTile);
  WsLayout L;
  const size_t o_status = L.take(sizeof(unsigned long long) * tiles);
  const size_t o_ticket = L.take(sizeof(unsigned int));
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(seg_ptr != nullptr, "null seg_ptr");
  TGL_REQUIRE(nq_max == 0 || (qnode && qtime && out_nbr && out_eid && out_ts), "null pointer");
  TGL_REQUIRE(g->indptr && (g->num_entries == 0 || (g->nbr && g->eid && g->ts)), "null graph array");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  TGL_TRY(cuda_check(cudaMemsetAsync(w, 0, L.off, s), "sample memset"));
  uint2 key = make_uint2((uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32));
  launch_pdl(sample_kernel, dim3((unsigned)tiles), dim3(kSampleWarps * 32), 0, s, 
      g->indptr, g->nbr, g->eid, g->ts, nq_max, nq_dev, qnode, qtime, k, strategy, key, layer,
      seg_ptr, out_nbr, out_eid, out_ts, reinterpret_cast<unsigned long long*>(w + o_status),
      reinterpret_cast<unsigned int*>(w + o_ticket));
  return launch_check("sample");
}
