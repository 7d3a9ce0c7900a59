// memory.cu -- §8(f) N3: the TGN node-memory path (eqs 9-11; the TGN
// case study, Listings 3-4).  Oracle: oracle/memory.py.
//
//   tgl_mailbox_store  (save_raw_msgs, Listing 4 L20-25)
//     insert   thread per message position j < 2B: open-addressing hash on the node id;
//              atomicMin(first position), atomicMax(latest = ordered t bits << 32 | j)
//              (coalesce by='latest', eq 10, ties -> larger j, R26)
//     compact  one CTA scans the 2B positions in order: a position that is its node's
//              first occurrence gets the next rank -> uniq[rank], pick[rank]
//     store    warp per unique node: mail[v] = [mem[v] ; mem[other] ; efeat[eid]] (eq 9),
//              mail_ts[v] = t  (coalesced float4-free row copies; rows are short)
//   tgl_memory_update  (update_memory, Listing 4 L11-17, eq 11)
//     gather   warp per node: X = [mail[v] ; Phi(mail_ts[v] - mem_ts[v])], H = mem[v]
//     GEMM     GI = X W_ih^T, GH = H W_hh^T   (strided fp32 SIMT GEMM, sgemm.cuh)
//     gate     thread per (node, unit): PyTorch GRUCell gates, writes mem[v], mem_ts[v]
//
// Sizes: a TGN batch is B = 600 edges (REDDIT/WIKI) -> 1200 messages and ~1-2k
// nodes to update; the whole path moves a few MB, so it is launch-bound rather than
// HBM-bound.
#include "common.cuh"
#include "sgemm.cuh"
#include "tenc.cuh"

namespace tgl {
namespace mem {

constexpr int kCompactThreads = 1024;

__device__ __forceinline__ uint32_t ordered_bits(float t) {
  // monotone map fp32 -> u32 (t1 < t2  <=>  bits(t1) < bits(t2)); -0 == +0 (R8)
  uint32_t u = time_key_bits(t);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

struct StoreArgs {
  tgl_memory M;
  int64_t B_max;
  const int64_t* B_dev;
  const int32_t *src, *dst, *eid;
  const float* t;
  int64_t eid0;
  const float* efeat;
  int64_t ld_e;
  int32_t* uniq;
  int64_t* pick;
  int64_t* n_uniq_dev;
  // workspace
  int32_t* keys;       // node + 1 (0 = empty)
  int32_t* first;      // first position (init INT32_MAX)
  unsigned long long* best;
  int32_t* slot_of;    // [2 B_max]
  uint32_t mask;       // capacity - 1
};

__device__ __forceinline__ int32_t node_at(const StoreArgs& a, int64_t j, int64_t B) {
  return j < B ? a.src[j] : a.dst[j - B];
}

__global__ void __launch_bounds__(256) insert_kernel(StoreArgs a) {
  const int64_t B = dev_count(a.B_dev, a.B_max);
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= 2 * a.B_max) return;
  if (j >= 2 * B) return;
  const int32_t v = node_at(a, j, B);
  if (v < 0 || (int64_t)v >= a.M.n_nodes) {
    a.slot_of[j] = -1;
    return;
  }
  uint32_t h = ((uint32_t)v * 0x9E3779B1u) & a.mask;
  while (true) {
    const int32_t prev = atomicCAS(a.keys + h, 0, v + 1);
    if (prev == 0 || prev == v + 1) break;
    h = (h + 1) & a.mask;
  }
  atomicMin(a.first + h, (int32_t)j);
  const float tj = a.t[j < B ? j : j - B];
  atomicMax(a.best + h, ((unsigned long long)ordered_bits(tj) << 32) | (unsigned long long)j);
  a.slot_of[j] = (int32_t)h;
}

__global__ void __launch_bounds__(kCompactThreads) compact_kernel(StoreArgs a) {
  __shared__ int64_t warp_tot[kCompactThreads / 32];
  __shared__ int64_t carry_s;
  const int64_t B = dev_count(a.B_dev, a.B_max);
  const int64_t n2 = 2 * B;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (int64_t base = 0; base < n2; base += kCompactThreads) {
    const int64_t j = base + threadIdx.x;
    int32_t h = -1;
    bool f = false;
    if (j < n2) {
      h = a.slot_of[j];
      f = h >= 0 && a.first[h] == (int32_t)j;
    }
    const int64_t incl = warp_inclusive_scan<int64_t>(f ? 1 : 0, lane);
    if (lane == 31) warp_tot[wid] = incl;
    __syncthreads();
    int64_t woff = 0, total = 0;
    for (int w = 0; w < kCompactThreads / 32; ++w) {
      const int64_t x = warp_tot[w];
      if (w < wid) woff += x;
      total += x;
    }
    const int64_t carry = carry_s;
    if (f) {
      const int64_t r = carry + woff + incl - 1;
      a.uniq[r] = node_at(a, j, B);
      a.pick[r] = (int64_t)(a.best[h] & 0xffffffffull);
    }
    __syncthreads();
    if (threadIdx.x == 0) carry_s = carry + total;
    __syncthreads();
  }
  if (threadIdx.x == 0) *a.n_uniq_dev = carry_s;
}

__global__ void __launch_bounds__(256) store_kernel(StoreArgs a) {
  const int64_t B = dev_count(a.B_dev, a.B_max);
  const int64_t n = *a.n_uniq_dev;
  const int lane = threadIdx.x & 31;
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (i >= n) return;
  const int64_t j = a.pick[i];
  const int64_t e = j < B ? j : j - B;
  const int32_t me = j < B ? a.src[e] : a.dst[e];
  const int32_t other = j < B ? a.dst[e] : a.src[e];
  const int dm = a.M.d_mem, de = a.M.d_e;
  const int64_t dmail = 2 * (int64_t)dm + de;
  float* out = a.M.mail + (int64_t)me * dmail;
  const float* sm = a.M.mem + (int64_t)me * dm;
  const float* so = a.M.mem + (int64_t)other * dm;
  for (int c = lane; c < dm; c += 32) {
    out[c] = sm[c];
    out[dm + c] = so[c];
  }
  if (de > 0) {
    const int64_t id = a.eid ? (int64_t)a.eid[e] : a.eid0 + e;
    const float* ef = a.efeat + id * a.ld_e;
    for (int c = lane; c < de; c += 32) out[2 * dm + c] = ef[c];
  }
  if (lane == 0) a.M.mail_ts[me] = a.t[e];
}

struct UpdArgs {
  tgl_memory M;
  tgl_gru_params G;
  int64_t n_max;
  const int64_t* n_dev;
  const int32_t* nodes;
  float *X, *H, *GI, *GH;
  int dx;
};

__global__ void __launch_bounds__(256) upd_gather_kernel(UpdArgs a) {
  const int64_t n = dev_count(a.n_dev, a.n_max);
  const int lane = threadIdx.x & 31;
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (i >= n) return;
  const int64_t v = a.nodes[i];
  const int dm = a.M.d_mem;
  const int dmail = 2 * dm + a.M.d_e;
  const float* mail = a.M.mail + v * dmail;
  float* x = a.X + i * a.dx;
  for (int c = lane; c < dmail; c += 32) x[c] = mail[c];
  const float dt = __fsub_rn(a.M.mail_ts[v], a.M.mem_ts[v]);
  for (int c = lane; c < a.G.d_t; c += 32) x[dmail + c] = tenc_direct(dt, a.G.omega[c], a.G.phi[c]);
  const float* h = a.M.mem + v * dm;
  for (int c = lane; c < dm; c += 32) a.H[i * dm + c] = h[c];
}

__device__ __forceinline__ float sigmoid_acc(float x) { return 1.f / (1.f + expf(-x)); }

__global__ void __launch_bounds__(256) upd_gate_kernel(UpdArgs a) {
  const int64_t n = dev_count(a.n_dev, a.n_max);
  const int dm = a.M.d_mem;
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= n * dm) return;
  const int64_t i = idx / dm;
  const int c = (int)(idx % dm);
  const float* gi = a.GI + i * 3 * dm;
  const float* gh = a.GH + i * 3 * dm;
  const float r = sigmoid_acc(gi[c] + a.G.b_ih[c] + gh[c] + a.G.b_hh[c]);
  const float z = sigmoid_acc(gi[dm + c] + a.G.b_ih[dm + c] + gh[dm + c] + a.G.b_hh[dm + c]);
  const float nn = tanhf(gi[2 * dm + c] + a.G.b_ih[2 * dm + c] +
                         r * (gh[2 * dm + c] + a.G.b_hh[2 * dm + c]));
  const float hp = (1.f - z) * nn + z * a.H[i * dm + c];
  const int64_t v = a.nodes[i];
  a.M.mem[v * dm + c] = hp;
  if (c == 0) a.M.mem_ts[v] = a.M.mail_ts[v];
}

}  // namespace mem
}  // namespace tgl

using namespace tgl;
using namespace tgl::mem;

static uint32_t pow2_at_least(int64_t x) {
  uint32_t c = 64;
  while ((int64_t)c < x) c <<= 1;
  return c;
}

extern "C" tgl_status tgl_mailbox_store(const tgl_memory* M, int64_t B_max, const int64_t* B_dev,
                                        const int32_t* src, const int32_t* dst, const float* t,
                                        const int32_t* eid, int64_t eid0, const float* efeat,
                                        int64_t ld_e, int32_t* uniq, int64_t* pick,
                                        int64_t* n_uniq_dev, void* ws, size_t* ws_bytes,
                                        void* stream) {
  TGL_REQUIRE(M != nullptr, "null memory");
  TGL_REQUIRE(B_max >= 0 && B_max < (1ll << 29), "B_max out of range");
  TGL_REQUIRE(M->d_mem >= 1 && M->d_e >= 0, "bad widths");
  const uint32_t cap = pow2_at_least(4 * B_max);
  const int64_t n2 = 2 * (B_max > 0 ? B_max : 1);
  WsLayout L;
  const size_t okeys = L.take(4ull * cap), ofirst = L.take(4ull * cap), obest = L.take(8ull * cap),
               oslot = L.take(4 * n2);
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  TGL_REQUIRE(M->mem && M->mail && M->mail_ts && uniq && pick && n_uniq_dev, "null pointer");
  TGL_REQUIRE(B_max == 0 || (src && dst && t), "null batch");
  TGL_REQUIRE(M->d_e == 0 || (efeat && ld_e >= M->d_e), "d_e > 0 needs efeat, ld_e >= d_e");
  cudaStream_t s = as_stream(stream);
  if (B_max == 0) return cuda_check(cudaMemsetAsync(n_uniq_dev, 0, 8, s), "memset n_uniq");
  char* w = static_cast<char*>(ws);
  StoreArgs a;
  a.M = *M;
  a.B_max = B_max;
  a.B_dev = B_dev;
  a.src = src;
  a.dst = dst;
  a.eid = eid;
  a.t = t;
  a.eid0 = eid0;
  a.efeat = efeat;
  a.ld_e = ld_e;
  a.uniq = uniq;
  a.pick = pick;
  a.n_uniq_dev = n_uniq_dev;
  a.keys = reinterpret_cast<int32_t*>(w + okeys);
  a.first = reinterpret_cast<int32_t*>(w + ofirst);
  a.best = reinterpret_cast<unsigned long long*>(w + obest);
  a.slot_of = reinterpret_cast<int32_t*>(w + oslot);
  a.mask = cap - 1;
  TGL_TRY(cuda_check(cudaMemsetAsync(w + okeys, 0, 4ull * cap, s), "memset keys"));
  TGL_TRY(cuda_check(cudaMemsetAsync(w + ofirst, 0x7f, 4ull * cap, s), "memset first"));
  TGL_TRY(cuda_check(cudaMemsetAsync(w + obest, 0, 8ull * cap, s), "memset best"));
  insert_kernel<<<(unsigned)ceil_div(2 * B_max, 256), 256, 0, s>>>(a);
  TGL_TRY(launch_check("mailbox insert"));
  compact_kernel<<<1, kCompactThreads, 0, s>>>(a);
  TGL_TRY(launch_check("mailbox compact"));
  store_kernel<<<(unsigned)ceil_div(2 * B_max * 32, 256), 256, 0, s>>>(a);
  return launch_check("mailbox store");
}

extern "C" tgl_status tgl_memory_update(const tgl_memory* M, const tgl_gru_params* G,
                                        int64_t n_max, const int64_t* n_dev, const int32_t* nodes,
                                        void* ws, size_t* ws_bytes, void* stream) {
  TGL_REQUIRE(M != nullptr && G != nullptr, "null memory / params");
  TGL_REQUIRE(n_max >= 0 && M->d_mem >= 1 && M->d_e >= 0 && G->d_t >= 0, "bad sizes");
  const int dm = M->d_mem, dx = 2 * dm + M->d_e + G->d_t;
  const int64_t n1 = n_max > 0 ? n_max : 1;
  WsLayout L;
  const size_t oX = L.take(4 * n1 * dx), oH = L.take(4 * n1 * dm), oGI = L.take(4 * n1 * 3 * dm),
               oGH = L.take(4 * n1 * 3 * dm);
  bool query = false;
  TGL_TRY(ws_protocol(ws, ws_bytes, L.off, &query));
  if (query) return TGL_OK;
  if (n_max == 0) return TGL_OK;
  TGL_REQUIRE(M->mem && M->mem_ts && M->mail && M->mail_ts && nodes, "null pointer");
  TGL_REQUIRE(G->W_ih && G->W_hh && G->b_ih && G->b_hh && (G->d_t == 0 || (G->omega && G->phi)),
              "null GRU parameter");
  cudaStream_t s = as_stream(stream);
  char* w = static_cast<char*>(ws);
  UpdArgs a;
  a.M = *M;
  a.G = *G;
  a.n_max = n_max;
  a.n_dev = n_dev;
  a.nodes = nodes;
  a.X = reinterpret_cast<float*>(w + oX);
  a.H = reinterpret_cast<float*>(w + oH);
  a.GI = reinterpret_cast<float*>(w + oGI);
  a.GH = reinterpret_cast<float*>(w + oGH);
  a.dx = dx;
  // rows beyond the device count stay zero (the GEMMs run over n_max rows)
  TGL_TRY(cuda_check(cudaMemsetAsync(w, 0, oGI, s), "memory_update workspace memset"));
  upd_gather_kernel<<<(unsigned)ceil_div(n_max * 32, 256), 256, 0, s>>>(a);
  TGL_TRY(launch_check("memory gather"));
  TGL_TRY(cuda_check(sgemm(s, n_max, 3 * dm, dx, a.X, dx, 1, G->W_ih, 1, dx, 0.f, a.GI, 3 * dm),
                     "gemm GI"));
  TGL_TRY(cuda_check(sgemm(s, n_max, 3 * dm, dm, a.H, dm, 1, G->W_hh, 1, dm, 0.f, a.GH, 3 * dm),
                     "gemm GH"));
  upd_gate_kernel<<<(unsigned)ceil_div(n_max * dm, 256), 256, 0, s>>>(a);
  return launch_check("memory gate");
}
