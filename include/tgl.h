/*
 * tgl.h -- C ABI of the B200-native TBlock hot path (libtgl.so, sm_100a).
 *
 * Method: TGLite (Wang & Mendis, ASPLOS'24).  "P:n" cites line n of the paper
 * text; "R<n>" cites a reading in DESIGN.md §2.
 *
 * Conventions (all entry points):
 *  - Every array argument is a DEVICE pointer unless stated otherwise.  The
 *    parameter structs (tgl_tcsr, tgl_attn_params) are HOST structs holding
 *    device pointers; they are read during the call only.
 *  - The caller owns every buffer.  The library never allocates or frees device
 *    memory, never synchronises the stream, and keeps no mutable global state.
 *    Calls on different streams may run concurrently.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *  - Workspace (CUB style): `ws == NULL` writes the required byte count to
 *    *ws_bytes and returns TGL_OK without launching; a non-NULL `ws` smaller
 *    than *ws_bytes' requirement returns TGL_EWORKSPACE.  Workspace must be
 *    256-byte aligned and is clobbered.
 *  - Data-dependent sizes stay on the device: outputs are capacity-bounded and
 *    the true count is written to a device int64 (`*_dev`).  Every consumer
 *    takes a HOST upper bound `*_max` (sizes the launch) plus the DEVICE count
 *    `*_dev` (NULL = the host bound is exact).  No call needs a host sync, so a
 *    batch is a fixed launch sequence a CUDA graph can capture.
 *  - Errors: host-side validation is synchronous and enqueues nothing.
 *    TGL_ECUDA reports a launch error; tgl_last_error() gives a thread-local
 *    message.  Device-side faults surface at the caller's next sync.
 *  - Dtypes: node ids int32, edge ids int32 (< 2^31 edges), CSR / segment
 *    offsets int64, times fp32, features / weights / outputs fp32 row-major
 *    with explicit leading dimensions (in elements).
 */
#ifndef TGL_H_
#define TGL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t tgl_status;
#define TGL_OK 0
#define TGL_EINVAL (-1)       /* null pointer, negative size, k <= 0, bad flags, ... */
#define TGL_EWORKSPACE (-2)   /* workspace too small */
#define TGL_ECUDA (-3)        /* CUDA launch / API error (see tgl_last_error) */
#define TGL_ERANGE (-4)       /* value out of representable range (e.g. > 2^31 entries) */
#define TGL_EUNSUPPORTED (-5) /* shape the kernels do not take (message says which) */

/* tgl_build_tcsr flags */
#define TGL_UNDIRECTED 1u        /* R2: both endpoints own an entry (default for TGNN data) */
#define TGL_INPUT_TIME_SORTED 2u /* COO already sorted by t: skips the time passes */

/* tgl_sample strategies */
#define TGL_RECENT 0
#define TGL_UNIFORM 1

/* tgl_attn_params.precision */
#define TGL_FP32 0 /* fp32 operands, fp32 accumulate (max abs err 1e-3 vs oracle) */
#define TGL_BF16 1 /* bf16-rounded projection operands, fp32 accumulate (5e-2) */
#define TGL_FP32_SIMT 2 /* fp32 FFMA on CUDA cores (exact fp32 products; slow reference mode) */

const char* tgl_version(void);
const char* tgl_status_string(tgl_status s);
const char* tgl_last_error(void); /* thread-local; "" if none */

/* ---------------------------------------------------------------------------
 * S1  T-CSR build.  P:311: "TGLITE initially stores temporal edges in COO
 * format, sorting based on timestamp ... it is best to use a CSR format for
 * faster lookups".
 *
 * Input COO (src, dst, t)[num_edges]; the edge id of edge e is e.  Output: for
 * every node v the segment [indptr[v], indptr[v+1]) of entries (nbr, eid, ts)
 * whose owner is v: (owner=src_e, nbr=dst_e) and, with TGL_UNDIRECTED,
 * (owner=dst_e, nbr=src_e).  Inside a segment entries are ordered by
 * (t asc, eid asc, forward-before-reverse) (R3).  num_entries M = E or 2E.
 * Capacities: indptr[num_nodes+1], nbr/eid/ts[M].  TGL_INPUT_TIME_SORTED is a
 * promise (t non-decreasing); the result is the same either way.
 * Errors: EINVAL (null, negative size, unknown flag), ERANGE (M >= 2^32 or
 * num_nodes >= 2^31).  Node ids must lie in [0, num_nodes) (unchecked on device).
 * ------------------------------------------------------------------------- */
tgl_status tgl_build_tcsr(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                          const int32_t* dst, const float* t, uint32_t flags,
                          int64_t* indptr, int32_t* nbr, int32_t* eid, float* ts,
                          void* ws, size_t* ws_bytes, void* stream);

typedef struct {
  int64_t num_nodes;
  int64_t num_entries;
  const int64_t* indptr; /* [num_nodes+1] */
  const int32_t* nbr;    /* [num_entries] */
  const int32_t* eid;    /* [num_entries] */
  const float* ts;       /* [num_entries], sorted inside each segment */
  const float* ts_coarse; /* optional (NULL): ts_coarse[p] = ts[32 p], p < ceil(M / 32) -- a
                             1/32 fence index the sampler searches first, so a query's
                             DRAM probes shrink to one 128-byte window of its segment */
  const void* entries;    /* optional (NULL): int32x4 {nbr, eid, bits(ts), 0} per entry --
                             the sampler's picks fetch one 16-byte record (one DRAM
                             sector) instead of three arrays */
} tgl_tcsr;

/* Sampler indexes of a T-CSR (once per graph, after tgl_build_tcsr; either output may be
 * NULL): ts_coarse [ceil(M/32)] floats as above, entries [M] x 16 bytes (16-byte
 * aligned).  The caller owns both and stores them in the tgl_tcsr it passes to
 * tgl_sample; results are bit-identical with or without them. */
tgl_status tgl_tcsr_index(const tgl_tcsr* g, float* ts_coarse, void* entries, void* stream);

/* tgl_build_tcsr that also writes the sampler indexes above (ts_coarse / entries, either
 * may be NULL) in the same sweep: the arrays equal tgl_build_tcsr + tgl_tcsr_index bit for
 * bit.  For M < 2^30 entries the build moves each entry as one 16-byte record through a
 * stable LSD digit sort (one kernel per 8-bit digit of the owner, plus four of t without
 * TGL_INPUT_TIME_SORTED), so no output is gathered afterwards; larger graphs take the
 * index-sort path and then tgl_tcsr_index.  Same arguments, errors and workspace protocol
 * as tgl_build_tcsr (the workspace holds the records: 16 B per entry for <= 2 passes). */
tgl_status tgl_build_tcsr_ex(int64_t num_nodes, int64_t num_edges, const int32_t* src,
                             const int32_t* dst, const float* t, uint32_t flags, int64_t* indptr,
                             int32_t* nbr, int32_t* eid, float* ts, float* ts_coarse,
                             void* entries, void* ws, size_t* ws_bytes, void* stream);

/* ---------------------------------------------------------------------------
 * S2  Roots of a batch (head TBlock).  P:235 (L2.8) `head = batch.block(ctx)`;
 * roots are the batch's source and destination nodes plus one negative
 * per edge (R15), all at the edge time.
 *
 * Batch = edges [s, s + min(batch, num_edges - s)), s = *start_dev (device
 * int64; NULL -> 0).  qnode = [src; dst; neg], qtime = [t; t; t]; neg is
 * indexed like src.  Capacity 3*batch; *n_roots_dev = 3 * (edges in batch).
 * ------------------------------------------------------------------------- */
tgl_status tgl_batch_roots(int64_t batch, int64_t num_edges, const int64_t* start_dev,
                           const int32_t* src, const int32_t* dst, const float* t,
                           const int32_t* neg, int32_t* qnode, float* qtime,
                           int64_t* n_roots_dev, void* stream);

/* ---------------------------------------------------------------------------
 * S3  Dedup of <node, time> pairs.  P:149 "embeddings are only computed for
 * unique node-time pairs"; dedup() filters a block's destinations in place and
 * registers an inverting hook (TGOpt dedup_filter/dedup_invert P:177-179).
 *
 * uniq = distinct pairs in order of first occurrence (R9); two times are equal
 * when they compare equal (-0 == +0, R8).  inv[i] = position of pair i in uniq,
 * so uniq[inv[i]] == (node[i], t[i]).  n = *n_dev (NULL -> n_max).
 * Capacities: uniq_node/uniq_t/inv[n_max]; *num_uniq_dev = U.
 * Workspace: O(n_max) (hash table of next_pow2(2 n_max) slots + scan state).
 * ------------------------------------------------------------------------- */
tgl_status tgl_dedup(int64_t n_max, const int64_t* n_dev, const int32_t* node,
                     const float* t, int32_t* uniq_node, float* uniq_t,
                     int64_t* num_uniq_dev, int32_t* inv, void* ws, size_t* ws_bytes,
                     void* stream);

/* ---------------------------------------------------------------------------
 * S4  Temporal neighbourhood sampling.  P:92: N(i,t) = neighbours over edges
 * with timestamp less than t (strict, R1), "further sampled based on a strategy
 * such as most-recent"; TSampler: uniform or most-recent, used as a
 * block operator `sampler.sample(tail)`.
 *
 * For query q = (v, t): candidates = entries of v's segment with ts < t (a
 * prefix; n of them).  TGL_RECENT: the last min(n,k) candidates in CSR order
 * (R4).  TGL_UNIFORM: n <= k -> all n in CSR order; else k draws with
 * replacement in slot order, slot s picks start + floor(r*n/2^32) with
 * r = Philox4x32-10(ctr={v, bits(t), layer, s/4}, key={lo32(seed),hi32(seed)})
 * word s%4 (R5, R6).  Output segments are compact: seg_ptr[q] = exclusive
 * prefix of per-query counts, seg_ptr[nq] = total (R7).  nq = *nq_dev (NULL ->
 * nq_max).  Capacities: seg_ptr[nq_max+1], out_*[nq_max*k].
 * Errors: EINVAL (k <= 0, bad strategy, null).  Workspace: scan state.
 * ------------------------------------------------------------------------- */
tgl_status tgl_sample(const tgl_tcsr* g, int64_t nq_max, const int64_t* nq_dev,
                      const int32_t* qnode, const float* qtime, int32_t k, int32_t strategy,
                      uint64_t seed, uint32_t layer, int64_t* seg_ptr, int32_t* out_nbr,
                      int32_t* out_eid, float* out_ts, void* ws, size_t* ws_bytes,
                      void* stream);

/* ---------------------------------------------------------------------------
 * S5  Next block.  P:237-238 (L2.10-11) `tail.next_block(...)`; reading R14:
 * dst' = [dst ; sampled src], t' = [t_dst ; edge t].
 * n_dst = *n_dst_dev (NULL -> n_dst_max); the source count is seg_ptr[n_dst].
 * Capacities: out_node/out_t[n_dst_max + n_src_max]; *n_out_dev = n_dst + n_src.
 * ------------------------------------------------------------------------- */
tgl_status tgl_next_block(int64_t n_dst_max, const int64_t* n_dst_dev, const int32_t* dst_node,
                          const float* dst_t, int64_t n_src_max, const int64_t* seg_ptr,
                          const int32_t* src_node, const float* src_t, int32_t* out_node,
                          float* out_t, int64_t* n_out_dev, void* stream);

/* ---------------------------------------------------------------------------
 * S6  Time encoding, eq (8): Phi(dt) = cos(omega*dt + phi), computed as
 * the paper's code does in fp32 (`torch.cos(ts * w + b)`): fp32
 * multiply, fp32 add, accurate cosine of that fp32 argument (R10).
 *
 * tgl_time_precompute: table[d][j] = Phi_j((float)d), d in [0, window) -- the
 * time-precomputation optimisation (R11).
 * tgl_time_encode: out[i][j] = Phi_j(dt[i]); when table != NULL and dt[i] is an
 * integer in [0, window) the row is read from the table (bit-identical).
 * ------------------------------------------------------------------------- */
tgl_status tgl_time_precompute(int64_t window, int32_t d_t, const float* omega,
                               const float* phi, float* table, void* stream);
tgl_status tgl_time_encode(int64_t n, const float* dt, int32_t d_t, const float* omega,
                           const float* phi, const float* table, int64_t window, float* out,
                           void* stream);

/* ---------------------------------------------------------------------------
 * S7-S13  One TBlock of TGAT temporal attention, eqs (4)-(7) P:104-119 as in
 * Listing 2 `TemporalAttnLayer.forward`:
 *   q_i   = Wq [h_i ; Phi(0)] + bq                              (eq 4; L2.27,29)
 *   k_e,v_e = W{k,v} [h_src(e) ; efeat(eid_e) ; Phi(t_i - t_e)] + b{k,v}
 *                                                               (eq 5; L2.28,30-31)
 *   s_e^h = LeakyReLU(logit_scale * <q_i^h, k_e^h>)             (L2.33; R12)
 *   alpha = edge_softmax over i's segment, per head              (L2.34)
 *   r_i   = sum_e alpha_e v_e  (0 for an empty segment)          (L2.36; R19)
 *   out_i = LayerNorm(ReLU(Wo [r_i ; h_i] + bo))                 (eq 7; R13)
 * Weights are [out, in] row-major (PyTorch Linear layout); concat orders are
 * exactly as written.  Heads split d_model into n_heads contiguous slices.
 *
 * Destinations i in [0, n_dst), n_dst = *n_dst_dev (NULL -> n_dst_max), with
 * time dst_t[i] and segment [seg_ptr[i], seg_ptr[i+1]) of edges.
 * Row of h_i: hdst_idx ? hdst_idx[i] : i, in table hdst (leading dim ld_hdst).
 * Row of h_src(e): hsrc_idx ? hsrc_idx[o + e] : o + e, o = *hsrc_off_dev
 * (NULL -> 0) -- the dedup inverse hook of the next block (S14).
 * efeat row eid[e] (ld_e); unused when d_e == 0.  edge_t[e] = edge time.
 * tenc_table (NULL = direct) as in tgl_time_encode.  max_seg = an upper bound on
 * every segment length (the sampler's k).  With max_seg <= 32 the tensor-core path
 * packs whole segments into 32-row bins; a segment longer than max_seg there is a
 * caller error and its output row is NaN.  max_seg > 32 (or <= 0: unknown) selects
 * the general path that takes any segment length.
 * Output out[n_dst_max][d_out] (rows >= n_dst untouched).
 * Limits: d_model == d_out, d_model % n_heads == 0, n_heads <= 2, d_t <= 256;
 * TGL_FP32 / TGL_BF16 run on the tensor cores (tcgen05) and need d_model == 100;
 * TGL_FP32_SIMT takes any d_model <= 128.
 * Precision: TGL_FP32 splits every fp32 operand into bf16 hi + lo and runs three
 * MMA passes (hi*hi + lo*hi + hi*lo) with fp32 accumulation; TGL_BF16 one pass.
 * ------------------------------------------------------------------------- */
/* Which K|V attention kernel runs (S6, S7, S9-S12; the dominant kernel).  AUTO picks
 * SPLIT when every row table has a 16-byte pitch and max_seg <= 32, BIN for other
 * pitches, GENERAL for max_seg > 32.  The others are kept as tested baselines. */
#define TGL_KV_AUTO 0
#define TGL_KV_SPLIT 1        /* split-role tcgen05 kernel; K chunks cut contiguously over
                                 [h | e | Phi] when d_hsrc, d_e are multiples of 4, else
                                 per-segment padded (reported as TGL_KV_SPLIT_PAD) */
#define TGL_KV_SPLIT_PAD 2    /* split-role, per-segment padded K chunks */
#define TGL_KV_ASYNC 3        /* single-role cp.async producers */
#define TGL_KV_BIN 4          /* register-gather producers (any row pitch) */
#define TGL_KV_GENERAL 5      /* any segment length */
#define TGL_KV_SIMT 6         /* (reported only) the TGL_FP32_SIMT kernel */
#define TGL_KV_PRE2 8         /* kv_pre on a CTA pair: one tcgen05.mma.cta_group::2 (M = 256)
                                 per K step, each SM streams half of the weights */
#define TGL_KV_PRE 7          /* pre-split h_src / e tables (tgl_split_rows): loaders move
                                 the bf16 hi / lo operands straight into the MMA's shared-
                                 memory stages, no conversion in the SM (AUTO picks it
                                 whenever input_layout marks the gathered tables split) */

/* tgl_attn_params.input_layout bits: the table is in the split16 layout of
 * tgl_split_rows (its leading dimension still counts 4-byte words). */
#define TGL_SPLIT_HSRC 1
#define TGL_SPLIT_E 2
#define TGL_SPLIT_TABLE 4   /* tenc_table is split16 [window, round_up(d_t, 8)] (kv_pre only) */
#define TGL_SPLIT_HDST 8    /* hdst is split16 too: the Q / FFN projections gather converter-
                               free operands (Phi(0) folded into the Q bias); needs the
                               pre-split K|V path and d_model == 100 */
#define TGL_NODE_PROJ 16    /* node projections: P->node_proj holds tgl_node_proj's Z for the
                               node table that h_src and h_dst both index (the tail block of
                               a chain, whose inputs are node features); hsrc_idx / hdst_idx
                               index Z rows, hsrc / hdst are not read.  Needs d_hsrc ==
                               d_hdst, split16 e (TGL_SPLIT_E), kv_kernel AUTO / PRE */

/* Layout of the node-projection table Z [n_nodes][TGL_NODE_PROJ_LD] fp32 (tgl_node_proj):
 * columns [K, K+d_model) = Wk[:, :d_h] h_v, [V, V+d_model) = Wv[:, :d_h] h_v,
 * [Q, Q+d_model) = Wq [h_v ; Phi(0)] + bq and Q+d_model+hd = q^hd . bk^hd (per head),
 * [O, O+d_model) = Wo[:, d_model:] h_v. */
#define TGL_NODE_PROJ_LD 512
#define TGL_NODE_PROJ_K 0
#define TGL_NODE_PROJ_V 100
#define TGL_NODE_PROJ_Q 256
#define TGL_NODE_PROJ_O 384

/* Measurement record (bench.py): when tgl_attn_params.probe != NULL the call records
 * ev_start / ev_stop (cudaEvent_t, created by the caller) on its stream immediately
 * before and after the K|V kernel and writes the TGL_KV_* id of the kernel that ran to
 * `kernel`.  Never set it while capturing a CUDA graph. */
typedef struct {
  void* ev_start;
  void* ev_stop;
  int32_t kernel;
} tgl_kv_probe;

typedef struct {
  int32_t d_hdst, d_hsrc, d_e, d_t, d_model, n_heads, d_out;
  const float *Wq, *bq;           /* [d_model][d_hdst + d_t]          */
  const float *Wk, *bk, *Wv, *bv; /* [d_model][d_hsrc + d_e + d_t]   */
  const float *Wo, *bo;           /* [d_out][d_model + d_hdst]        */
  const float *ln_gamma, *ln_beta;
  float ln_eps;                   /* 1e-5 */
  const float *omega, *phi;       /* [d_t] */
  float leaky_slope;              /* 0.2; < 0 -> identity */
  float logit_scale;              /* 1.0 */
  int32_t precision;              /* TGL_FP32 | TGL_BF16 | TGL_FP32_SIMT */
  const void* packed;             /* optional tgl_attn_pack() output for these weights and
                                     this precision; NULL = pack inside every call */
  int32_t kv_kernel;              /* TGL_KV_AUTO (0) or a specific K|V kernel (TGL_KV_*);
                                     a kernel that cannot take the call -> EUNSUPPORTED */
  tgl_kv_probe* probe;            /* optional (NULL): caller-owned measurement record */
  int32_t input_layout;           /* TGL_SPLIT_* bits: hsrc / efeat / tenc_table are
                                     split16 tables (tensor-core precisions, max_seg <= 32,
                                     2 heads); TGL_NODE_PROJ */
  const float* node_proj;         /* TGL_NODE_PROJ: Z of tgl_node_proj (else unused) */
} tgl_attn_params;

/* Weight layout transform for the tensor-core path, done once per layer (the
 * weights are constant across batches): Wq, [Wk;Wv], Wo -> bf16 hi/lo pairs in the
 * swizzled shared-memory image the kernels stream with bulk copies.  `packed`
 * (device, >= tgl_attn_packed_bytes(P) bytes, 256-aligned) is owned by the caller
 * and must be re-packed if the weights change.  EUNSUPPORTED for shapes the
 * tensor-core path does not take. */
size_t tgl_attn_packed_bytes(const tgl_attn_params* P);
tgl_status tgl_attn_pack(const tgl_attn_params* P, void* packed, size_t bytes, void* stream);

/* Node projections (the TBlock layer of eqs 4, 5, 7 is linear in h before the logits:
 * q_i = Wq [h_i ; Phi(0)] + bq, k_e = Wk [h_src ; e ; Phi] + bk = Wk[:, :d_h] h_src + ...,
 * FFN input Wo [r ; h_i] = Wo[:, :d_model] r + Wo[:, d_model:] h_i).  When h_src and h_dst
 * are rows of one node table with far fewer rows than the block gathers (the tail block:
 * GDELT 16,682 nodes vs 1.32M sampled edges per batch), the h terms are computed once per
 * node and gathered, so the per-edge MMAs cover [e | Phi] only.  Writes Z (layout above)
 * for rows v < n_nodes of hnode (split16, tgl_split_rows; ld >= round_up(d_hsrc, 8) words,
 * 16-byte aligned).  Same precision modes as tgl_tblock_attn (3-pass fp32 / bf16); Z is
 * fp32.  Needs P->packed (tgl_attn_pack), d_hsrc == d_hdst, 2 heads.  Z is owned by the
 * caller, valid until the weights change.  Errors: EINVAL, EUNSUPPORTED. */
tgl_status tgl_node_proj(const tgl_attn_params* P, int64_t n_nodes, const void* hnode,
                         int64_t ld, float* Z, void* stream);

tgl_status tgl_tblock_attn(const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev,
                           const int64_t* seg_ptr, const float* dst_t, const float* hdst,
                           const int32_t* hdst_idx, int64_t ld_hdst, const float* hsrc,
                           const int32_t* hsrc_idx, const int64_t* hsrc_off_dev, int64_t ld_hsrc,
                           const float* efeat, const int32_t* eid, int64_t ld_e,
                           const float* edge_t, const float* tenc_table, int64_t window,
                           int32_t max_seg, float* out, void* ws, size_t* ws_bytes,
                           void* stream);

/* Split16 feature layout for the gathered operands of the tensor-core K|V path: row r
 * of dst (pitch ld_dst 4-byte words, 16-byte aligned rows) holds bf16 RNE(x) for the
 * dp = round_up(d, 8) columns (zeros past d), then bf16 RNE(x - hi) for the same
 * columns -- 4 bytes per column like fp32, written once per table (features) or per
 * layer output, so the K|V kernel gathers MMA operands without converting them.
 * hi + lo equals x to 2^-17 relative; the 3-pass product is the fp32 mode's.  Errors:
 * EINVAL (ld_dst < dp, ld_dst % 4 != 0, unaligned dst). */
tgl_status tgl_split_rows(int64_t n_rows, int32_t d, const float* src, int64_t ld_src,
                          void* dst, int64_t ld_dst, void* stream);

/* ---------------------------------------------------------------------------
 * N2  Backward of one TBlock attention layer (training is the paper's
 * headline workload).  Given dL/d(out) for the n = *n_dst_dev destinations
 * of a tgl_tblock_attn call (same arguments, but fp32 row tables for h_dst, h_src and e:
 * P->input_layout and P->kv_kernel are ignored), adds
 * (+=) dL/dtheta for every parameter of the layer into G (shapes of the weights) and,
 * when the pointers are non-NULL, dL/dh into grad_hdst (row hdst_idx[i]) and grad_hsrc
 * (row hsrc_idx[o + e]) -- the rows the forward gathered; several destinations / edges
 * may hit one row (atomic adds).  The time encoder Phi_j(dt) = cos(omega_j dt + phi_j)
 * (R10 fp32 argument b) contributes domega_j = sum -sin(b) dt dPhi, dphi_j = sum -sin(b)
 * dPhi (including Phi(0) of eq 4).  The forward is recomputed in fp32 (exact fp32
 * products); n_edges_max bounds seg_ptr[n].  Workspace: O(n_dst_max * (d_hdst + d_t +
 * d_model) + n_edges_max * (d_hsrc + d_e + d_t + d_model)) floats.
 * Errors: EINVAL (d_out != d_model, d_model > 128, > 2 heads, nulls).
 * ------------------------------------------------------------------------- */
typedef struct {
  float *dWq, *dbq, *dWk, *dbk, *dWv, *dbv, *dWo, *dbo, *dgamma, *dbeta, *domega, *dphi;
} tgl_attn_grads;

/* Adjoint of the S14 gather (the dedup inverse hook in the backward): out[idx[j]][:] +=
 * src[j][:] for j < n = *n_dev (NULL -> n_max); idx NULL = identity; atomic adds. */
tgl_status tgl_scatter_add_rows(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                                const float* src, int64_t ld_src, int32_t d, float* out,
                                int64_t ld_out, void* stream);

tgl_status tgl_tblock_attn_backward(
    const tgl_attn_params* P, int64_t n_dst_max, const int64_t* n_dst_dev, int64_t n_edges_max,
    const int64_t* seg_ptr, const float* dst_t, const float* hdst, const int32_t* hdst_idx,
    int64_t ld_hdst, const float* hsrc, const int32_t* hsrc_idx, const int64_t* hsrc_off_dev,
    int64_t ld_hsrc, const float* efeat, const int32_t* eid, int64_t ld_e, const float* edge_t,
    const float* grad_out, int64_t ld_gout, const tgl_attn_grads* G, float* grad_hdst,
    int64_t ld_ghdst, float* grad_hsrc, int64_t ld_ghsrc, void* ws, size_t* ws_bytes,
    void* stream);

/* ---------------------------------------------------------------------------
 * N4  preload(): feature tables that live in host memory (graphs whose
 * features exceed HBM: GDELT's edge features are 142 GB) are read by the GPU
 * directly from pinned memory, one block at a time: dst row j = src row idx[j]
 * (row_bytes bytes, any layout: fp32 or split16) for j < n, n = n_dev[n_at ? *n_at : 0]
 * (NULL n_dev -> n_max; n_at lets n be seg_ptr[U] of a block, both on the device).  src
 * may be pinned host memory (cudaHostAlloc / cudaHostRegister; the pointer is valid on
 * the device under UVA) or device memory; dst is device memory; idx NULL = identity.
 * The TBlock chain then gathers from dst with identity indices.  Errors: EINVAL. */
tgl_status tgl_preload_rows(int64_t n_max, const int64_t* n_dev, const int64_t* n_at,
                            const int32_t* idx, const void* src, int64_t src_pitch,
                            int64_t row_bytes, void* dst, int64_t dst_pitch, void* stream);

/* ---------------------------------------------------------------------------
 * N3  TGN node memory (eqs 9-11, and the TGN case
 * study, Listings 3-4).  Reading R25-R27.  The caller owns the
 * state, all device fp32 row-major:
 *   mem [n_nodes, d_mem] (s_v), mem_ts [n_nodes] (time of s_v's last update),
 *   mail [n_nodes, d_mail] with d_mail = 2 d_mem + d_e (the one-slot mailbox: TGN keeps
 *   only the latest message per node), mail_ts [n_nodes].
 * ------------------------------------------------------------------------- */
typedef struct {
  int64_t n_nodes;
  int32_t d_mem, d_e;
  float* mem;
  float* mem_ts;
  float* mail;
  float* mail_ts;
} tgl_memory;

/* GRU memory updater (eq 11; Listing 4 GRUMemoryUpdater): PyTorch GRUCell
 * layout, gates (r, z, n) stacked along rows: W_ih [3 d_mem, d_mail + d_t], W_hh
 * [3 d_mem, d_mem], b_ih / b_hh [3 d_mem]; the time encoder omega / phi [d_t]. */
typedef struct {
  int32_t d_t;
  const float *W_ih, *W_hh, *b_ih, *b_hh, *omega, *phi;
} tgl_gru_params;

/* save_raw_msgs + mailbox.store (Listing 4 L20-25).  The batch: edges j < B = *B_dev
 * (NULL -> B_max) with endpoints src[j], dst[j], time t[j] and edge id eid[j] (NULL ->
 * eid0 + j: consecutive rows of the time-sorted edge list).  Edge j gives src[j] the
 * message [mem[src] ; mem[dst] ; efeat[eid]] (position j) and dst[j] the message
 * [mem[dst] ; mem[src] ; efeat[eid]] (position B + j) (eq 9).  coalesce(by='latest')
 * (eq 10): per node, the message with the largest t, ties -> the larger position (R26);
 * it is written to mail[node], its t to mail_ts[node].  Outputs (device, capacity
 * 2 B_max): uniq[i] = the distinct nodes in order of first position, pick[i] = the
 * position of the kept message, *n_uniq_dev = their count.  mem is only read.
 * Workspace: a hash table of O(B_max) slots plus scan state.  Errors: EINVAL (nulls,
 * d_e > 0 without efeat, node ids outside [0, n_nodes) are skipped, not errors). */
tgl_status tgl_mailbox_store(const tgl_memory* M, int64_t B_max, const int64_t* B_dev,
                             const int32_t* src, const int32_t* dst, const float* t,
                             const int32_t* eid, int64_t eid0, const float* efeat,
                             int64_t ld_e, int32_t* uniq, int64_t* pick, int64_t* n_uniq_dev,
                             void* ws, size_t* ws_bytes, void* stream);

/* update_memory (Listing 4 L11-17, eq 11) for the n = *n_dev (NULL -> n_max) nodes[i],
 * which must be distinct (the dedup'ed nodes of a block): dt = fl(mail_ts[v] - mem_ts[v]),
 * x = [mail[v] ; Phi(dt)] (R10), mem[v] = GRUCell(x, mem[v]), mem_ts[v] = mail_ts[v].
 * fp32 GEMMs (exact products, fp32 sums).  Workspace: O(n_max (d_mail + d_t + 7 d_mem))
 * floats.  Errors: EINVAL (nulls, d_mem < 1). */
tgl_status tgl_memory_update(const tgl_memory* M, const tgl_gru_params* G, int64_t n_max,
                             const int64_t* n_dev, const int32_t* nodes, void* ws,
                             size_t* ws_bytes, void* stream);

/* ---------------------------------------------------------------------------
 * S14  Dedup inverse applied to rows (the hook of P:279 / TGOpt dedup_invert
 * P:179): out[j][:] = table[idx[j]][:] for j < n, n = *n_dev (NULL -> n_max).
 * ------------------------------------------------------------------------- */
tgl_status tgl_gather_rows(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                           const float* table, int64_t ld_table, int32_t d, float* out,
                           int64_t ld_out, void* stream);

/* ---------------------------------------------------------------------------
 * S16  Root sharding across G ranks (the paper is single-GPU, P:424,
 * and TGL's multi-GPU training is the contrast it names).  Every rank holds the
 * whole graph, features and weights, forms the batch's roots (and dedups them when
 * enabled) redundantly, and computes S4-S15 for the contiguous slice
 * [r*c, min((r+1)*c, U)) of the U unique roots, c = ceil(U / world); embeddings
 * depend only on <node, t> (content-keyed sampling, R6), so the slices compose.
 *
 * tgl_shard_slice: out[i] = (node, t)[lo + i] for the slice of `rank`; U = *n_dev
 * (NULL -> n_max); capacities out_node/out_t[ceil(n_max / world)]; *out_n_dev = its
 * length (device).
 * tgl_shard_gather: after an all-gather of every rank's slice outputs padded to c_max
 * rows (`gathered` = [world * c_max, d], rank-major), rebuild row j < n = *n_dev (NULL
 * -> n_max): i = idx ? idx[j] : j (idx = the roots' dedup inverse, S14), out[j] =
 * gathered[(i / c) * c_max + i % c] with c = ceil(U / world), U = *u_dev (NULL ->
 * u_max).  Requires c_max >= ceil(u_max / world).  Errors: EINVAL.
 * ------------------------------------------------------------------------- */
tgl_status tgl_shard_slice(int64_t n_max, const int64_t* n_dev, const int32_t* node,
                           const float* t, int32_t rank, int32_t world, int32_t* out_node,
                           float* out_t, int64_t* out_n_dev, void* stream);
tgl_status tgl_shard_gather(int64_t n_max, const int64_t* n_dev, const int32_t* idx,
                            int64_t u_max, const int64_t* u_dev, int32_t world,
                            const float* gathered, int64_t c_max, int32_t d, float* out,
                            int64_t ld_out, void* stream);

/* ---------------------------------------------------------------------------
 * N1  Embedding memoisation: the cache() operator ("previously computed
 * embeddings could be reused and cached"; "cache() will filter destination
 * node-time pairs to ones that have not been cached and register a hook to
 * combine computed outputs with cached results"; TGOpt cache_lookup /
 * cache_store, Listing 1 lines 10-23).  One table per layer (the
 * listing keys the store by layer); the caller owns it.
 *
 * Table: `capacity` slots (a power of two, <= 2^30), keys u64 [capacity] that
 * the caller zeroes once (0 = empty), vals fp32 [capacity, d] row-major.  A pair
 * (v, t) is keyed like dedup (node << 32 | raw fp32 bits of t with -0 canonicalised
 * to +0, R8); a NaN t never hits and is never stored (NaN != NaN).  Linear probing over
 * at most TGL_CACHE_PROBES slots: a pair that finds no free slot is not stored,
 * so a full table only costs recomputation, never a wrong row (reading R22).
 * ------------------------------------------------------------------------- */
#define TGL_CACHE_PROBES 64
typedef struct {
  int64_t capacity;
  int32_t d;
  unsigned long long* keys;   /* device [capacity] */
  float* vals;                /* device [capacity, d] */
} tgl_cache;

/* Lookup + filter (the pre-processing half of cache()).  For i < n = *n_dev
 * (NULL -> n_max): slot[i] = the table slot holding (node[i], t[i]) if cached,
 * else -(1 + j) where j is the rank of i among the misses in input order.  The
 * misses are compacted, stable: miss_node[j], miss_t[j]; *num_miss_dev = count.
 * Capacities n_max.  Workspace: scan state (CUB-style protocol). */
tgl_status tgl_cache_lookup(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                            const int32_t* node, const float* t, int32_t* slot,
                            int32_t* miss_node, float* miss_t, int64_t* num_miss_dev,
                            void* ws, size_t* ws_bytes, void* stream);

/* Store (Listing 1 cache_store): for i < n = *n_dev (NULL -> n_max) insert
 * (node[i], t[i]) -> emb[i][0:d) (row pitch ld_emb floats).  A pair already
 * present keeps its slot and gets the row rewritten; duplicate pairs inside one
 * call must carry equal rows (true for dedup'ed or deterministic outputs). */
tgl_status tgl_cache_store(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                           const int32_t* node, const float* t, const float* emb,
                           int64_t ld_emb, void* stream);

/* Combine hook (the post-processing half of cache()): for i < n = *n_dev
 * (NULL -> n_max): out[i] = slot[i] >= 0 ? vals[slot[i]] : computed[-(1 + slot[i])]
 * (rows of d floats; pitches ld_computed, ld_out). */
tgl_status tgl_cache_combine(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                             const int32_t* slot, const float* computed, int64_t ld_computed,
                             float* out, int64_t ld_out, void* stream);

/* Store + combine in one pass (what the TBlock chain launches).  The pairs are
 * indexed in "dedup space": node[i], t[i], slot[i] as written by tgl_cache_lookup.
 * For j < n = *n_dev (NULL -> n_max), i = idx ? idx[j] : j:
 * out[j] = slot[i] >= 0 ? vals[slot[i]] : computed[-(1 + slot[i])], and a miss's
 * row is inserted under (node[i], t[i]) exactly as tgl_cache_store would.  idx lets
 * the dedup inverse hook (S14) read the merged rows directly: several j
 * may share one i; they then store the same row under the same key.  Only the
 * misses some j reads are stored: idx must be onto [0, U) (the dedup inverse is)
 * for the table to receive every computed row. */
tgl_status tgl_cache_merge(const tgl_cache* c, int64_t n_max, const int64_t* n_dev,
                           const int32_t* idx, const int32_t* node, const float* t,
                           const int32_t* slot, const float* computed, int64_t ld_computed,
                           float* out, int64_t ld_out, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* TGL_H_ */
