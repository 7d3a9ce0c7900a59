/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for the TBlock hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py
 * (its cpu_baseline leg and `--impl reference`) may load this library.  It
 * shares no code, header or constant with the CUDA path
 * (paper_conf_asplos_wangm24_b200/csrc); neither includes the other.
 *
 * Reference: Wang & Mendis, "TGLite", ASPLOS'24 -- /root/reference/PAPER.md,
 * cited as P:<line>.  Readings of silent/garbled passages are DESIGN.md §2
 * (ids R1..).  Every function below follows either a plain definition or the
 * paper's equations step by step, in the paper's order; floating point is
 * carried in fp64 except where the paper's code fixes fp32 (the time encoder,
 * `torch.cos(ts * self.weight + self.bias)`, P:219 / P:247, and the fp32
 * timestamps of the dataset).
 *
 * Pin status (tests/test_oracle_pins.py): every function here is pinned
 * (brute force over all edges, library routines, closed forms, invariants,
 * Random123 / cuRAND known answers).  The numeric values of the paper itself
 * are "parity unpinned": the paper prints no worked example.
 *
 * Build: gcc -O2 -fno-fast-math -ffp-contract=off -fopenmp -shared -fPIC
 * (OpenMP only over independent queries / destinations).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

/* ---------------------------------------------------------------------- */
/* misc                                                                    */
/* ---------------------------------------------------------------------- */

int or_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

void or_set_num_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}

/* Bit pattern of a timestamp used as a key: -0.0 and +0.0 are the same
 * time (they compare equal), so both map to +0.0 (reading R8). */
static uint32_t time_key_bits(float t) {
  uint32_t b;
  if (t == 0.0f) t = 0.0f;
  memcpy(&b, &t, 4);
  return b;
}

/* ---------------------------------------------------------------------- */
/* S1. Temporal CSR ("edges in COO, sorted by timestamp"; "a CSR    */
/* format for faster lookups" for sampling).                               */
/*                                                                         */
/* Definition (reading R2, R3): for edge e (eid = e) emit the entry         */
/* (owner=src_e, nbr=dst_e, e, t_e) and, if undirected, (owner=dst_e,       */
/* nbr=src_e, e, t_e).  indptr = exclusive prefix sum of entries per owner; */
/* inside an owner's segment entries are ordered by (t asc, eid asc,        */
/* forward-before-reverse).                                                 */
/* ---------------------------------------------------------------------- */

typedef struct {
  int32_t owner, nbr, eid, dir;
  float t;
} or_entry;

static int cmp_entry(const void* a, const void* b) {
  const or_entry* x = (const or_entry*)a;
  const or_entry* y = (const or_entry*)b;
  if (x->owner != y->owner) return x->owner < y->owner ? -1 : 1;
  if (x->t != y->t) return x->t < y->t ? -1 : 1;
  if (x->eid != y->eid) return x->eid < y->eid ? -1 : 1;
  if (x->dir != y->dir) return x->dir < y->dir ? -1 : 1;
  return 0;
}

int64_t or_tcsr_num_entries(int64_t num_edges, int undirected) {
  return undirected ? 2 * num_edges : num_edges;
}

/* returns 0 on success, -1 on a node id out of range */
int or_build_tcsr(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                  const int32_t* dst, const float* t, int undirected,
                  int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts) {
  int64_t M = or_tcsr_num_entries(num_edges, undirected);
  or_entry* ent = (or_entry*)malloc(sizeof(or_entry) * (size_t)(M > 0 ? M : 1));
  int64_t m = 0;
  for (int64_t e = 0; e < num_edges; ++e) {
    if (src[e] < 0 || src[e] >= num_nodes || dst[e] < 0 || dst[e] >= num_nodes) {
      free(ent);
      return -1;
    }
    ent[m].owner = src[e]; ent[m].nbr = dst[e]; ent[m].eid = (int32_t)e;
    ent[m].dir = 0; ent[m].t = t[e]; ++m;
    if (undirected) {
      ent[m].owner = dst[e]; ent[m].nbr = src[e]; ent[m].eid = (int32_t)e;
      ent[m].dir = 1; ent[m].t = t[e]; ++m;
    }
  }
  qsort(ent, (size_t)M, sizeof(or_entry), cmp_entry);
  for (int64_t v = 0; v <= num_nodes; ++v) indptr[v] = 0;
  for (int64_t j = 0; j < M; ++j) indptr[ent[j].owner + 1] += 1;
  for (int64_t v = 0; v < num_nodes; ++v) indptr[v + 1] += indptr[v];
  for (int64_t j = 0; j < M; ++j) {
    nbr[j] = ent[j].nbr;
    eid[j] = ent[j].eid;
    ts[j] = ent[j].t;
  }
  free(ent);
  return 0;
}

/* ---------------------------------------------------------------------- */
/* Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11 -- "Random123").        */
/* Used for uniform temporal sampling (reading R6: the paper only says     */
/* "uniform"; the counter-based generator keyed by query content     */
/* keeps dedup semantics-preserving).                          */
/* ---------------------------------------------------------------------- */

void or_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
  uint32_t k0 = key_in[0], k1 = key_in[1];
  for (int round = 0; round < 10; ++round) {
    uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* ---------------------------------------------------------------------- */
/* S4. Temporal neighbourhood sampling.                                    */
/* N(i,t): neighbours over edges with timestamp less than t, then sampled   */
/* by a strategy such as most-recent; TSampler does uniform or       */
/* most-recent.                                                     */
/*                                                                         */
/* For query (v, t): the candidates are the entries of v's segment with     */
/* ts < t (a prefix, the segment being time-sorted); n = their number.      */
/* RECENT (0): the last min(n, k) candidates in segment order (R4).         */
/* UNIFORM (1): n <= k -> all n candidates in segment order; otherwise k    */
/* draws with replacement, slot s = 0..k-1 in slot order (R5), entry        */
/* start + floor(r * n / 2^32) with r = Philox(ctr = {v, bits(t), layer,    */
/* s/4}, key = {lo32(seed), hi32(seed)})[s % 4] (R6).                       */
/* seg_ptr = exclusive prefix sum of the per-query output counts (R7).      */
/* ---------------------------------------------------------------------- */

static int64_t sample_count(const int64_t* indptr, const float* ts, int32_t v, float t,
                            int32_t k, int64_t* start_out, int64_t* n_out) {
  int64_t start = indptr[v], end = indptr[v + 1];
  int64_t n = 0;
  while (start + n < end && ts[start + n] < t) ++n; /* plain linear scan */
  *start_out = start;
  *n_out = n;
  return n < k ? n : k;
}

/* qkey[q] is the node id that keys the Philox counter (R6); it equals qnode[q]
 * except when the CSR is a sub-graph with locally renumbered owners (the large-config
 * checks build one per queried node).  returns 0, or -1 on a query node out of
 * range / bad k / bad strategy */
int or_sample_keyed(int64_t num_nodes, const int64_t* indptr, const int32_t* nbr,
                    const int32_t* eid, const float* ts, int64_t nq, const int32_t* qnode,
                    const int32_t* qkey, const float* qtime, int32_t k, int32_t strategy,
                    uint64_t seed, uint32_t layer, int64_t* seg_ptr, int32_t* out_nbr,
                    int32_t* out_eid, float* out_ts) {
  if (k <= 0 || (strategy != 0 && strategy != 1)) return -1;
  for (int64_t q = 0; q < nq; ++q)
    if (qnode[q] < 0 || qnode[q] >= num_nodes) return -1;
  /* pass 1: counts -> seg_ptr */
  seg_ptr[0] = 0;
  for (int64_t q = 0; q < nq; ++q) {
    int64_t start, n;
    seg_ptr[q + 1] = seg_ptr[q] + sample_count(indptr, ts, qnode[q], qtime[q], k, &start, &n);
  }
  /* pass 2: picks */
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t q = 0; q < nq; ++q) {
    int64_t start, n;
    int64_t m = sample_count(indptr, ts, qnode[q], qtime[q], k, &start, &n);
    int64_t o = seg_ptr[q];
    for (int64_t s = 0; s < m; ++s) {
      int64_t j;
      if (strategy == 0 || n <= k) {
        j = start + (n - m) + s;
      } else {
        uint32_t ctr[4] = {(uint32_t)qkey[q], time_key_bits(qtime[q]), layer,
                           (uint32_t)(s >> 2)};
        uint32_t key[2] = {(uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)};
        uint32_t r[4];
        or_philox4x32_10(ctr, key, r);
        j = start + (int64_t)(((uint64_t)r[s & 3] * (uint64_t)n) >> 32);
      }
      out_nbr[o + s] = nbr[j];
      out_eid[o + s] = eid[j];
      out_ts[o + s] = ts[j];
    }
  }
  return 0;
}

int or_sample(int64_t num_nodes, const int64_t* indptr, const int32_t* nbr,
              const int32_t* eid, const float* ts, int64_t nq, const int32_t* qnode,
              const float* qtime, int32_t k, int32_t strategy, uint64_t seed,
              uint32_t layer, int64_t* seg_ptr, int32_t* out_nbr, int32_t* out_eid,
              float* out_ts) {
  return or_sample_keyed(num_nodes, indptr, nbr, eid, ts, nq, qnode, qnode, qtime, k, strategy,
                         seed, layer, seg_ptr, out_nbr, out_eid, out_ts);
}

/* ---------------------------------------------------------------------- */
/* S3. Deduplication of <node, time> pairs ("embeddings are only     */
/* computed for unique node-time pairs"; dedup() filters a block's          */
/* destination pairs in place and registers an inverting hook;       */
/* TGOpt form dedup_filter / dedup_invert).                      */
/*                                                                         */
/* Definition (reading R9): uniq = the distinct (node, time) pairs in order */
/* of first occurrence; inv[i] = position of pair i in uniq.  Two times are */
/* the same when they compare equal (so -0 == +0, R8).                      */
/* ---------------------------------------------------------------------- */

typedef struct {
  uint64_t key;
  int64_t idx;
} or_keyidx;

static int cmp_keyidx(const void* a, const void* b) {
  const or_keyidx* x = (const or_keyidx*)a;
  const or_keyidx* y = (const or_keyidx*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  if (x->idx != y->idx) return x->idx < y->idx ? -1 : 1;
  return 0;
}

static int cmp_first(const void* a, const void* b) {
  const or_keyidx* x = (const or_keyidx*)a;
  const or_keyidx* y = (const or_keyidx*)b;
  return x->idx < y->idx ? -1 : (x->idx > y->idx ? 1 : 0);
}

/* returns U */
int64_t or_dedup(int64_t n, const int32_t* node, const float* t, int32_t* uniq_node,
                 float* uniq_t, int32_t* inv) {
  if (n <= 0) return 0;
  or_keyidx* a = (or_keyidx*)malloc(sizeof(or_keyidx) * (size_t)n);
  for (int64_t i = 0; i < n; ++i) {
    a[i].key = ((uint64_t)(uint32_t)node[i] << 32) | time_key_bits(t[i]);
    a[i].idx = i;
  }
  /* group equal keys; within a group the smallest index is the first occurrence */
  qsort(a, (size_t)n, sizeof(or_keyidx), cmp_keyidx);
  int64_t* first_of = (int64_t*)malloc(sizeof(int64_t) * (size_t)n); /* per input i */
  or_keyidx* firsts = (or_keyidx*)malloc(sizeof(or_keyidx) * (size_t)n);
  int64_t U = 0;
  for (int64_t j = 0; j < n; ++j) {
    if (j == 0 || a[j].key != a[j - 1].key) {
      firsts[U].key = a[j].key;
      firsts[U].idx = a[j].idx;
      ++U;
    }
    first_of[a[j].idx] = firsts[U - 1].idx;
  }
  /* order the distinct pairs by first occurrence */
  qsort(firsts, (size_t)U, sizeof(or_keyidx), cmp_first);
  int64_t* rank_of_first = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  for (int64_t u = 0; u < U; ++u) {
    int64_t f = firsts[u].idx;
    rank_of_first[f] = u;
    uniq_node[u] = node[f];
    uniq_t[u] = t[f];
  }
  for (int64_t i = 0; i < n; ++i) inv[i] = (int32_t)rank_of_first[first_of[i]];
  free(a);
  free(first_of);
  free(firsts);
  free(rank_of_first);
  return U;
}

/* ---------------------------------------------------------------------- */
/* S6. Time encoding, eq (8): Phi(dt) = cos(omega * dt + phi), as the */
/* paper's code computes it in fp32 tensors: torch.cos(ts * w + b)          */
/* (P:219).  Reading R10: two fp32 roundings (multiply, then add),   */
/* then the cosine of that fp32 argument, rounded once to fp32.             */
/* ---------------------------------------------------------------------- */

static float time_encode_one(float dt, float omega, float phi) {
  volatile float a = omega * dt; /* fp32 product (no contraction: -ffp-contract=off) */
  volatile float b = a + phi;    /* fp32 sum */
  return (float)cos((double)b);
}

void or_time_encode(int64_t n, const float* dt, int32_t d_t, const float* omega,
                    const float* phi, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int32_t j = 0; j < d_t; ++j)
      out[i * d_t + j] = time_encode_one(dt[i], omega[j], phi[j]);
}

/* Time precomputation (reading R11): the table row for an     */
/* integer dt = d is Phi((float)d); it equals the direct value bit for bit. */
void or_time_precompute(int64_t window, int32_t d_t, const float* omega, const float* phi,
                        float* table) {
  for (int64_t d = 0; d < window; ++d)
    for (int32_t j = 0; j < d_t; ++j)
      table[d * d_t + j] = time_encode_one((float)d, omega[j], phi[j]);
}

/* ---------------------------------------------------------------------- */
/* S7-S13. One TBlock of TGAT temporal attention (eqs 4-7;       */
/* Listing 2 TemporalAttnLayer.forward).                          */
/*                                                                         */
/*   z_i = h_i || Phi(0)                                (eq 4, L2.27,29)    */
/*   z_j = h_j || e_ij || Phi(t - t_j)                  (eq 5, L2.28,30-31) */
/*   q = Wq z_i + bq ; k_j = Wk z_j + bk ; v_j = Wv z_j + bv                */
/*   s_j^h = LeakyReLU_slope(scale * sum_{c in head h} q_c k_jc)  (L2.33, R12) */
/*   alpha^h = edge_softmax over i's segment                       (L2.34)  */
/*   r_i^h = sum_j alpha_j^h v_j^h ; empty segment -> r_i = 0      (L2.36)  */
/*   h_i' = LayerNorm(ReLU(Wo [r_i || h_i] + bo))                  (eq 7, R13) */
/* Weights are [out, in] row-major (PyTorch Linear layout).                 */
/* All arithmetic after the fp32 time encoder is fp64.                      */
/* ---------------------------------------------------------------------- */

typedef struct {
  int32_t d_hdst, d_hsrc, d_e, d_t, d_model, n_heads, d_out;
  const float *Wq, *bq, *Wk, *bk, *Wv, *bv, *Wo, *bo, *ln_gamma, *ln_beta;
  float ln_eps;
  const float *omega, *phi;
  float leaky_slope; /* < 0 -> identity */
  float logit_scale;
} or_attn_params;

static void linear64(const float* W, const float* b, int out_f, int in_f, const double* x,
                     double* y) {
  for (int o = 0; o < out_f; ++o) {
    double acc = 0.0;
    for (int c = 0; c < in_f; ++c) acc += (double)W[(int64_t)o * in_f + c] * x[c];
    y[o] = acc + (double)b[o];
  }
}

/* one destination; returns into out[d_out] */
static void attn_one_dst(const or_attn_params* P, int64_t e0, int64_t e1, float t_dst,
                         const float* h_dst, const float* hsrc, const int32_t* hsrc_idx,
                         int64_t ld_hsrc, const float* efeat, const int32_t* eid,
                         int64_t ld_e, const float* edge_t, double* out) {
  const int dq = P->d_hdst + P->d_t;
  const int dk = P->d_hsrc + P->d_e + P->d_t;
  const int dm = P->d_model, H = P->n_heads, dh = dm / H;
  double* zq = (double*)malloc(sizeof(double) * (size_t)dq);
  double* q = (double*)malloc(sizeof(double) * (size_t)dm);
  double* zk = (double*)malloc(sizeof(double) * (size_t)dk);
  double* kk = (double*)malloc(sizeof(double) * (size_t)dm);
  double* vv = (double*)malloc(sizeof(double) * (size_t)dm);
  int64_t m = e1 - e0;
  double* s = (double*)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1) * H);
  double* V = (double*)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1) * dm);
  double* r = (double*)calloc((size_t)dm, sizeof(double));
  double* zo = (double*)malloc(sizeof(double) * (size_t)(dm + P->d_hdst));
  double* o = (double*)malloc(sizeof(double) * (size_t)P->d_out);

  /* eq 4: z_i = h_i || Phi(0) */
  for (int c = 0; c < P->d_hdst; ++c) zq[c] = h_dst[c];
  for (int j = 0; j < P->d_t; ++j)
    zq[P->d_hdst + j] = time_encode_one(0.0f, P->omega[j], P->phi[j]);
  linear64(P->Wq, P->bq, dm, dq, zq, q);

  for (int64_t e = 0; e < m; ++e) {
    int64_t ge = e0 + e;
    /* eq 5: z_j = h_j || e_ij || Phi(t - t_j) */
    const float* hs = hsrc + (int64_t)hsrc_idx[ge] * ld_hsrc;
    for (int c = 0; c < P->d_hsrc; ++c) zk[c] = hs[c];
    if (P->d_e > 0) {
      const float* ef = efeat + (int64_t)eid[ge] * ld_e;
      for (int c = 0; c < P->d_e; ++c) zk[P->d_hsrc + c] = ef[c];
    }
    float dt = t_dst - edge_t[ge]; /* fp32 delta of fp32 timestamps */
    for (int j = 0; j < P->d_t; ++j)
      zk[P->d_hsrc + P->d_e + j] = time_encode_one(dt, P->omega[j], P->phi[j]);
    linear64(P->Wk, P->bk, dm, dk, zk, kk);
    linear64(P->Wv, P->bv, dm, dk, zk, vv);
    for (int h = 0; h < H; ++h) {
      double acc = 0.0;
      for (int c = h * dh; c < (h + 1) * dh; ++c) acc += q[c] * kk[c];
      acc *= (double)P->logit_scale;
      if (P->leaky_slope >= 0.0f && acc < 0.0) acc *= (double)P->leaky_slope;
      s[e * H + h] = acc;
    }
    for (int c = 0; c < dm; ++c) V[e * dm + c] = vv[c];
  }
  /* edge_softmax + edge_reduce(sum) per head */
  for (int h = 0; h < H; ++h) {
    if (m == 0) break;
    double mx = s[h];
    for (int64_t e = 1; e < m; ++e)
      if (s[e * H + h] > mx) mx = s[e * H + h];
    double den = 0.0;
    for (int64_t e = 0; e < m; ++e) den += exp(s[e * H + h] - mx);
    for (int64_t e = 0; e < m; ++e) {
      double a = exp(s[e * H + h] - mx) / den;
      for (int c = h * dh; c < (h + 1) * dh; ++c) r[c] += a * V[e * dm + c];
    }
  }
  /* eq 7: FFN(r || h) = LayerNorm(ReLU(Wo [r || h] + bo)) */
  for (int c = 0; c < dm; ++c) zo[c] = r[c];
  for (int c = 0; c < P->d_hdst; ++c) zo[dm + c] = h_dst[c];
  linear64(P->Wo, P->bo, P->d_out, dm + P->d_hdst, zo, o);
  double mean = 0.0, var = 0.0;
  for (int c = 0; c < P->d_out; ++c) {
    if (o[c] < 0.0) o[c] = 0.0;
    mean += o[c];
  }
  mean /= P->d_out;
  for (int c = 0; c < P->d_out; ++c) var += (o[c] - mean) * (o[c] - mean);
  var /= P->d_out;
  double inv_std = 1.0 / sqrt(var + (double)P->ln_eps);
  for (int c = 0; c < P->d_out; ++c)
    out[c] = (o[c] - mean) * inv_std * (double)P->ln_gamma[c] + (double)P->ln_beta[c];

  free(zq); free(q); free(zk); free(kk); free(vv); free(s); free(V); free(r);
  free(zo); free(o);
}

/* hdst_idx == NULL means identity (row i of hdst). out: fp64 [n_dst, d_out]. */
int or_tblock_attn(const or_attn_params* P, int64_t n_dst, const int64_t* seg_ptr,
                   const float* dst_t, const float* hdst, const int32_t* hdst_idx,
                   int64_t ld_hdst, const float* hsrc, const int32_t* hsrc_idx,
                   int64_t ld_hsrc, const float* efeat, const int32_t* eid, int64_t ld_e,
                   const float* edge_t, double* out) {
  if (P->n_heads <= 0 || P->d_model % P->n_heads != 0) return -1;
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t i = 0; i < n_dst; ++i) {
    int64_t row = hdst_idx ? (int64_t)hdst_idx[i] : i;
    attn_one_dst(P, seg_ptr[i], seg_ptr[i + 1], dst_t[i], hdst + row * ld_hdst, hsrc,
                 hsrc_idx, ld_hsrc, efeat, eid, ld_e, edge_t, out + i * P->d_out);
  }
  return 0;
}

/* ---------------------------------------------------------------------- */
/* S15 cross-check: the recursive formulation of Listing 1.    */
/* embed(v, t, depth): depth == L -> raw node features (L1.8-9); otherwise  */
/* sample N(v, t) with RNG layer = depth (L1.14), recurse on every sampled  */
/* neighbour (L1.15) and on (v, t) itself (L1.16), then run the attention   */
/* of block `depth` (L1.22).  No dedup, no block bookkeeping.               */
/* params[depth] are the weights of block `depth` (0 = head).               */
/* ---------------------------------------------------------------------- */

typedef struct {
  int64_t num_nodes;
  const int64_t* indptr;
  const int32_t* nbr;
  const int32_t* eid;
  const float* ts;
  const float* nfeat;
  int64_t d_v;
  const float* efeat;
  int64_t d_e;
  int32_t k, strategy, n_layers;
  uint64_t seed;
  const or_attn_params* params; /* [n_layers] */
} or_model;

static void embed_rec(const or_model* M, int32_t v, float t, int depth, double* out) {
  if (depth == M->n_layers) {
    for (int64_t c = 0; c < M->d_v; ++c) out[c] = M->nfeat[(int64_t)v * M->d_v + c];
    return;
  }
  const or_attn_params* P = &M->params[depth];
  int64_t seg[2];
  int32_t* snbr = (int32_t*)malloc(sizeof(int32_t) * (size_t)M->k);
  int32_t* seid = (int32_t*)malloc(sizeof(int32_t) * (size_t)M->k);
  float* sts = (float*)malloc(sizeof(float) * (size_t)M->k);
  or_sample(M->num_nodes, M->indptr, M->nbr, M->eid, M->ts, 1, &v, &t, M->k, M->strategy,
            M->seed, (uint32_t)depth, seg, snbr, seid, sts);
  int64_t m = seg[1];
  int dh_in = P->d_hdst; /* == width of embed(., ., depth+1) */
  double* hd = (double*)malloc(sizeof(double) * (size_t)dh_in);
  embed_rec(M, v, t, depth + 1, hd);
  float* hdf = (float*)malloc(sizeof(float) * (size_t)dh_in);
  float* hsf = (float*)malloc(sizeof(float) * (size_t)(m > 0 ? m : 1) * P->d_hsrc);
  double* tmp = (double*)malloc(sizeof(double) * (size_t)P->d_hsrc);
  for (int c = 0; c < dh_in; ++c) hdf[c] = (float)hd[c];
  for (int64_t j = 0; j < m; ++j) {
    embed_rec(M, snbr[j], sts[j], depth + 1, tmp);
    for (int c = 0; c < P->d_hsrc; ++c) hsf[j * P->d_hsrc + c] = (float)tmp[c];
  }
  int32_t* ident = (int32_t*)malloc(sizeof(int32_t) * (size_t)(m > 0 ? m : 1));
  for (int64_t j = 0; j < m; ++j) ident[j] = (int32_t)j;
  attn_one_dst(P, 0, m, t, hdf, hsf, ident, P->d_hsrc, M->efeat, seid, M->d_e, sts, out);
  free(snbr); free(seid); free(sts); free(hd); free(hdf); free(hsf); free(tmp); free(ident);
}

/* Intermediate layer outputs are rounded to fp32 between layers, as the
 * iterative path stores them (fp32 tensors between blocks). */
void or_embed_recursive(const or_model* M, int64_t n, const int32_t* node, const float* t,
                        double* out) {
  int64_t d_out = M->params[0].d_out;
#pragma omp parallel for schedule(dynamic, 4)
  for (int64_t i = 0; i < n; ++i) embed_rec(M, node[i], t[i], 0, out + i * d_out);
}
