/*
 * tg.h -- C ABI of the B200-native TGOpt hot path (libtg.so).
 *
 * Redundancy-aware batched TGAT inference (TGOpt, PPoPP'23): dedup of
 * (node, t) targets (Sec. 4.1, Alg. 2), memoization of layer embeddings in a
 * device-resident FIFO cache (Sec. 4.2, Alg. 3), precomputed time encoding
 * (Sec. 4.3), most-recent-k temporal sampling and the TGAT attention M
 * (Eqs. 4-8) -- the embedding function Embed(l, ns, ts) of Alg. 1
 * -- plus the link-prediction score.
 * "P:Lnnn" cites a line of the paper text; "Rnn" a reading in
 * DESIGN.md.
 *
 * Conventions
 *  - Every call returns tg_status (0 = TG_OK, < 0 = error); nothing throws
 *    across the ABI. tg_strerror() gives a static message.
 *  - "host" pointers are plain CPU memory; "device" pointers are CUDA global
 *    memory of the device the context was created on. Calls marked "either"
 *    accept both (detected with cudaPointerGetAttributes; host buffers are
 *    staged through the context's pinned buffers inside the call).
 *  - The context owns every device copy it makes (graph, features, weights,
 *    tables, cache, workspaces). The caller keeps ownership of all argument
 *    buffers; the library never frees or retains them past the call.
 *  - Hot-path calls are stream-ordered on the given cudaStream_t (NULL = the
 *    legacy default stream) and asynchronous w.r.t. the host when all
 *    buffers are device memory: outputs are valid once the stream reaches the
 *    point after the call. They must not be issued concurrently on two
 *    streams for the same context.
 *  - After TG_ECUDA the context is unusable except for tg_free().
 */
#ifndef TG_H_
#define TG_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TG_OK = 0,
  TG_EINVAL = -1,   /* bad argument (size, null pointer, range)                 */
  TG_ENOMEM = -2,   /* device or pinned allocation failed                        */
  TG_ECUDA = -3,    /* CUDA runtime error (context now unusable)                 */
  TG_ESTATE = -4,   /* call out of order (e.g. embed before tg_model_load)       */
  TG_EORDER = -5,   /* timestamps not non-decreasing                     */
  TG_EDEVICE = -6   /* sticky device-side error (out-of-range id seen in a kernel) */
} tg_status;

typedef struct tg_ctx tg_ctx; /* opaque; one per device */

/* Optimisation toggles (the ablation of P:L408, Fig. 6). Outputs never depend
 * on them (semantic-preserving, P:L37/P:L176/P:L384); counters do. */
#define TG_OPT_DEDUP  1u  /* DedupFilter at layers l > 0 (Sec. 4.1)            */
#define TG_OPT_CACHE  2u  /* memo cache at layers 1..L-1 (Sec. 4.2)    */
#define TG_OPT_TTABLE 4u  /* precomputed Phi(dt) window [0, W) (Sec. 4.3)      */
#define TG_OPT_ALL    7u
/* Storage location of the memo cache (NEXT-2; the paper's design choice, Table 5):
 * the FIFO payload ring of every cached layer lives in pinned, mapped host memory (read
 * and written by the kernels over PCIe / C2C); the index stays in HBM. Outputs and counters
 * are unchanged; only speed and bytes moved differ. Not part of TG_OPT_ALL. */
#define TG_OPT_HOST_CACHE 8u

/* Arithmetic of the dense projections. */
#define TG_PREC_FP32  0   /* fp32 FFMA (CUDA cores): rtol 1e-4 / atol 1e-5 vs oracle */
#define TG_PREC_TF32X3 1  /* tcgen05 kind::tf32, 3-term hi/lo split: fp32-level error */
#define TG_PREC_BF16  2   /* tcgen05 kind::f16 bf16 operands, fp32 accumulate: rtol 2e-2 */
#define TG_PREC_TF32  3   /* tcgen05 kind::tf32 one pass (A streamed raw fp32, B rna-tf32): rtol 2e-2 class */
#define TG_PREC_F16X3 4   /* tcgen05 kind::f16, fp16 operands with the 3-term hi/lo split (11 + 11 bits, as
                           * TF32X3) at twice the tf32 rate: fp32-level error (parity 1e-5 + 1e-4|ref|).
                           * Weights are scaled per row by exact powers of two; activations entering a
                           * projection must satisfy |a| < 65504, else the sticky device error bit 32 is set
                           * (tg_counters_read returns TG_EDEVICE) -- use TG_PREC_TF32X3 for such data. */
#define TG_PREC_LAST  TG_PREC_F16X3

/* ------------------------------------------------------------------------ */
/* Graph: a CTDG edge stream with static node/edge features.        */
/* ------------------------------------------------------------------------ */
typedef struct {
  int64_t n_nodes;          /* |V|; node ids are 1..n_nodes, 0 = padding */
  int64_t n_edges;          /* |E|; edge i (0-based) has edge id i+1                  */
  const int32_t* src;       /* host [n_edges]                                          */
  const int32_t* dst;       /* host [n_edges]                                          */
  const uint32_t* ts;       /* host [n_edges], non-decreasing, integer seconds (R4) */
  const float* node_feat;   /* host [(n_nodes+1) x d_n] row-major; row 0 is forced to 0 */
  int32_t d_n;
  const float* edge_feat;   /* host [(n_edges+1) x d_e] row-major; row 0 is forced to 0 */
  int32_t d_e;
} tg_graph_desc;

/* Builds the device T-CSR (per-node adjacency sorted by (t, edge id), both
 * directions of every edge: graphs are undirected) and uploads the
 * padded feature tables. Synchronous. Errors: TG_EINVAL (sizes, ids out of
 * range, d < 1), TG_EORDER (ts decreasing), TG_ENOMEM, TG_ECUDA. */
tg_status tg_graph_load(int device, const tg_graph_desc* graph, tg_ctx** out);

/* ------------------------------------------------------------------------ */
/* Model: L-layer TGAT (Eqs. 4-8; M per TGAT [37], reading R1).             */
/* ------------------------------------------------------------------------ */
typedef struct {
  int32_t n_layers;           /* L >= 1 (2)                                  */
  int32_t n_heads;            /* H >= 1, D % H == 0 (2)                      */
  int32_t n_neighbors;        /* k >= 1, <= 32 (20)                          */
  int32_t d_t;                /* time-encoding dim (R2: d_n)                         */
  int32_t max_batch_targets;  /* workspace bound on n of tg_embed_batch (2 x edges)  */
  int64_t cache_limit;        /* items per cached layer (2,000,000)          */
  int32_t time_window;        /* W of the precomputed Phi table (10,000)     */
  uint32_t opts;              /* TG_OPT_* bits                                        */
  int32_t precision;          /* TG_PREC_*                                            */
  int32_t superbatch;         /* S: batches per launch sequence in tg_score_stream (0 = 64,
                               * 1 = one batch at a time, <= 128). Semantics per batch are
                               * unchanged: dedup scope, cache lookups and FIFO inserts stay per
                               * batch and in batch order, so outputs and counters do not depend
                               * on S. Both cache passes (grid-wide eviction-free pass, ordered
                               * pass) keep their superbatch hash in global memory, so S is bounded
                               * only by a ~40 GB budget for the S-proportional workspaces.
                               * tg_superbatch() returns the S in use. */
} tg_model_cfg;

/* params: host float32 [n_params] in this order (row-major, Linear = [out x in]),
 * D = d_n + d_e + d_t:
 *   for l = 1..L: W_q[D*D], W_k[D*D], W_v[D*D], W_fc[D*D], b_fc[D], ln_g[D], ln_b[D],
 *                 W_m1[d_n*(D+d_n)], b_m1[d_n], W_m2[d_n*d_n], b_m2[d_n]
 *   shared:       omega[d_t], phi[d_t], W_a1[d_n*2d_n], b_a1[d_n], W_a2[d_n], b_a2[1]
 * Uploads/prepares weights, builds Phi table and Phi(0),
 * allocates workspaces and the cache, and resets it. Synchronous.
 * Errors: TG_ESTATE (no graph), TG_EINVAL (n_params mismatch, bad cfg, or a time
 * encoder with |omega_c| * 2^32 + |phi_c| >= 1e15, beyond the device cosine's fp64
 * argument reduction), TG_ENOMEM, TG_ECUDA. May be called again to replace the model. */
tg_status tg_model_load(tg_ctx* ctx, const tg_model_cfg* cfg, const float* params, int64_t n_params);

/* ------------------------------------------------------------------------ */
/* Hot path                                                                  */
/* ------------------------------------------------------------------------ */
/* H = Embed(L, ns, ts) (Alg. 1 invoked at l = L): out[i] is the
 * layer-L embedding of target <nodes[i], ts[i]>. n <= max_batch_targets.
 * nodes/ts/out: either (device for the asynchronous path); out is [n x d_n]
 * float32 row-major. Updates the memo cache and the counters.
 * Errors: TG_EINVAL (n < 0, n > bound, null), TG_ESTATE. */
tg_status tg_embed_batch(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n,
                         float* out, void* cuda_stream);

/* One chronological batch: embeds src || dst at the edge times as
 * one deduplicated target list and writes
 * scores[e] = sigmoid(MLP(h_src, h_dst)) (R10). 2*n_edges <= max_batch_targets.
 * src/dst/ts/scores: either. Errors as tg_embed_batch. */
tg_status tg_score_edges(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts,
                         int64_t n_edges, float* scores, void* cuda_stream);

/* Link prediction with negatives (NEXT-3; the TGAT evaluation the paper's task
 * follows, [37]): embeds nodes/ts as ONE chronological batch (one
 * deduplicated target list, P:L239 -- e.g. src || dst || negatives, 3 x edges)
 * and writes scores[p] = sigmoid(MLP(h[pair_a[p]], h[pair_b[p]])) (R10) for
 * every pair of target indices (0 <= pair_a[p], pair_b[p] < n_targets).
 * n_targets <= max_batch_targets; n_pairs <= max_batch_targets.
 * nodes/ts/pair_a/pair_b: all host or all device (a mix is TG_EINVAL); scores: either.
 * Updates the memo cache and the counters like tg_embed_batch.
 * Errors: TG_EINVAL (sizes, null, host pair index out of range), TG_ESTATE;
 * a device pair index out of range sets the sticky device error bit 16
 * (reported by tg_counters_read as TG_EDEVICE) and that pair's score is not written. */
tg_status tg_score_pairs(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n_targets,
                         const int32_t* pair_a, const int32_t* pair_b, int64_t n_pairs, float* scores,
                         void* cuda_stream);

/* The paper's inference task: the whole edge range [0, n_edges) in
 * chronological batches of `batch` edges (the last one partial, R13), with the
 * per-batch semantics of tg_score_edges, issued from native code as superbatches
 * of S batches (tg_superbatch) on two internal streams without host sync.
 * src/dst/ts: all host or all device (a mix is TG_EINVAL), [n_edges]; scores:
 * either, [n_edges].
 * batch_counters: optional device int64 [n_batches x TG_NCOUNTERS] that
 * receives each batch's counters (NULL = not recorded). */
tg_status tg_score_stream(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts,
                          int64_t n_edges, int32_t batch, float* scores, int64_t* batch_counters,
                          void* cuda_stream);

/* Link-prediction evaluation with negatives over the whole stream (NEXT-3; the TGAT
 * evaluation protocol the paper's task follows, [37]): like tg_score_stream, but
 * batch b's target list is src || dst || neg at the edge times (3 x batch targets, ONE
 * deduplicated Alg. 1 batch) and it writes scores[e] = p(src_e, dst_e) and
 * scores[n_edges + e] = p(src_e, neg_e) (R10). neg[e] (1..n_nodes) is the caller's seeded
 * negative destination of edge e -- an input, not part of the method. Requires
 * 3 x batch <= max_batch_targets. src/dst/ts/neg: all host or all device (a mix is
 * TG_EINVAL); scores: either, [2 x n_edges]. Errors as tg_score_stream. */
tg_status tg_score_stream_neg(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts,
                              const int32_t* neg, int64_t n_edges, int32_t batch, float* scores,
                              int64_t* batch_counters, void* cuda_stream);

/* Empties the memo cache (all layers) and zeroes the counters; new_limit >= 0
 * replaces the item limit (must be <= the limit given to tg_model_load), < 0
 * keeps it. Synchronous. Errors: TG_ESTATE, TG_EINVAL. */
tg_status tg_cache_reset(tg_ctx* ctx, int64_t new_limit);

/* ------------------------------------------------------------------------ */
/* Counters, debug and hygiene                                               */
/* ------------------------------------------------------------------------ */
/* Counter vector layout (int64): for l = 0..TG_MAX_LAYERS:
 *   [l*6 + 0] n        inputs entering Embed(l)
 *   [l*6 + 1] unique   after DedupFilter (= n when dedup is off)
 *   [l*6 + 2] lookups  cache probes (cached layers only)
 *   [l*6 + 3] hits
 *   [l*6 + 4] misses   embeddings computed at layer l (l >= 1)
 *   [l*6 + 5] evicted  live cache items evicted (FIFO, R11)
 * then [TG_CNT_TTABLE] Phi(dt) served from the table, [TG_CNT_TDIRECT] computed. */
#define TG_MAX_LAYERS 4
#define TG_CNT_PER_LAYER 6
#define TG_CNT_TTABLE ((TG_MAX_LAYERS + 1) * TG_CNT_PER_LAYER)
#define TG_CNT_TDIRECT (TG_CNT_TTABLE + 1)
#define TG_NCOUNTERS (TG_CNT_TDIRECT + 1)

/* Synchronises the context's work, copies min(n, TG_NCOUNTERS) cumulative
 * counters into host_out, and reports a sticky device error as TG_EDEVICE. */
tg_status tg_counters_read(tg_ctx* ctx, int64_t* host_out, int32_t n);

/* Unit entry points for parity tests of single steps (device pointers,
 * stream-ordered). They do not touch the cache or the counters. */
/* DedupFilter (Alg. 2): uniq_nodes/uniq_ts[n] get the unique targets in
 * first-occurrence order, inv[n] the inverse index, *n_uniq (device int32)
 * the count. n <= max_batch_targets * (k+1). */
tg_status tg_dedup(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n,
                   int32_t* uniq_nodes, uint32_t* uniq_ts, int32_t* inv, int32_t* n_uniq,
                   void* cuda_stream);
/* NghLookup: k most-recent neighbours with t_j < t (R6, R7),
 * right-aligned, zero-padded; nbr/eid/nts are [n x k]. */
tg_status tg_sample(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n,
                    int32_t* nbr, int32_t* eid, uint32_t* nts, void* cuda_stream);
/* TimeEncode (Eq. 8): out[n x d_t] = Phi(delta[i]); use_table selects the
 * precomputed window for delta < W (bit-identical to the direct path). */
tg_status tg_time_encode(tg_ctx* ctx, const int64_t* delta, int64_t n, int32_t use_table,
                         float* out, void* cuda_stream);

/* Dense projection GEMM unit entry point (the kernels of the M/FFN stages):
 * C[M x N] = A[M x K] . B[N x K]^T (+ bias[N] if non-null, then ReLU if relu),
 * all device float32 row-major; precision TG_PREC_* selects SIMT fp32,
 * tcgen05 tf32x3 / tf32 / bf16. K, N multiples of 4. Stream-ordered (asynchronous). */
tg_status tg_gemm(tg_ctx* ctx, int32_t precision, int32_t M, int32_t N, int32_t K, const float* A,
                  const float* B, const float* bias, int32_t relu, float* C, void* cuda_stream);

/* Library/launch statistics for the bench: number of kernels launched by the
 * hot-path calls since the last tg_cache_reset (host-side count). */
int64_t tg_kernel_launches(tg_ctx* ctx);
/* Batches per launch sequence actually used by tg_score_stream (tg_model_cfg.superbatch after
 * the default and the cache-pass capacity clamp); 0 before tg_model_load or for a null ctx. */
int32_t tg_superbatch(tg_ctx* ctx);

/* Per-stage device timing (the operation breakdown of Table 3):
 * when enabled, every hot-path launch is bracketed by CUDA events on its
 * stream (adds host overhead; use a separate pass from throughput timing).
 * tg_profile_read synchronises and returns, per stage id (TG_ST_*), the
 * summed device milliseconds and the launch count since enabling. */
#define TG_ST_PREP 0
#define TG_ST_DEDUP 1
#define TG_ST_LOOKUP 2
#define TG_ST_SAMPLE 3
#define TG_ST_RESOLVE 4
#define TG_ST_PROJ_K 5   /* G1: target-side key projection u = P h + b   */
#define TG_ST_ATTN 6     /* gather + time encode + scores + softmax + sums */
#define TG_ST_PROJ_V 7   /* G2: value/output projection + residual         */
#define TG_ST_LNORM 8
#define TG_ST_FFN1 9
#define TG_ST_FFN2 10    /* includes the CacheStore payload write          */
#define TG_ST_SCORE 11
#define TG_ST_OTHER 12
#define TG_ST_PHI 13     /* TimeEncode of dt >= W rows (front stream, Eq. 8) */
#define TG_NSTAGES 14
tg_status tg_profile_enable(tg_ctx* ctx, int32_t on);
tg_status tg_profile_read(tg_ctx* ctx, double* ms, int64_t* launches, int32_t n);

void tg_free(tg_ctx* ctx);
const char* tg_strerror(tg_status s);
/* Build/version string (arch, precision modes compiled). */
const char* tg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TG_H_ */
