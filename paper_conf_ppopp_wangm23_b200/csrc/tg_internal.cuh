// Internal declarations of libtg (B200 / sm_100a). Not part of the ABI.
//
// Data layout in HBM:
//   T-CSR      rowptr[V+2] int32, adj_nbr/adj_eid int32 [2E], adj_t uint32 [2E]
//              per node sorted by (t, edge id) (R6); both directions
//   X          float [(V+1) x ldn]   ldn = round4(d_n), zero padded, row 0 = 0
//   Ef         float [(E+1) x lde]   lde = round4(d_e)
//   kv rows    [hn (dnp) | ef (dep) | Phi (dtp)] = Dp floats, dXp = round4(dX)
//   ring_l     float [C x ldn] FIFO ring of cached layer-l embeddings
//   index_l    {u64 key, i64 logical pos} open addressing, linear probing
//
// Superbatch: S consecutive batches share one launch
// sequence. Per recursion level l the *dedup lists* (I_l, U_l, inv_l, slot_l)
// are batch-segmented with a fixed per-batch stride `cap`; the *compute list*
// C_l (targets whose embedding is computed at layer l) is compacted over the
// superbatch in (batch, unique-list) order, with its neighbour slots stored
// compute-centric at [q*k + m].
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/tg.h"

namespace tg {

constexpr unsigned long long kEmptyKey = 0xFFFFFFFFFFFFFFFFull;
constexpr unsigned long long kLockedKey = 0xFFFFFFFFFFFFFFFEull;
constexpr int kMaxK = 32;          // neighbours per target (warp lanes)
constexpr int kMaxS = 128;         // batches per superbatch
constexpr int kDedupThreads = 1024;
constexpr int kDedupIPT = 16;      // items per thread per CTA (ordered scan)
constexpr int kDedupSlots = 16384; // smem hash slots per CTA (load <= ~0.6)
constexpr int kProbeIPT = 16;
constexpr int kSeqCLMax = 16;        // cluster CTAs of the ordered cache passes
constexpr int kSeqSlotsPerCTA = 16384; // their DSMEM hash slots per CTA

// ---- programmatic dependent launch (PDL). Every kernel of the hot path is
// launched with programmatic stream serialization, so its CTAs may become
// resident while the previous kernel of the same stream drains. Each kernel
// calls pdl_wait() before its first global-memory access (read OR write: the
// predecessor may still read what this kernel overwrites) -- it returns once
// the predecessor grid has completed and its writes are visible -- and then
// pdl_trigger(), which lets the *next* kernel start its own prologue. Only
// shared-memory / TMEM / barrier setup and kernel parameters are touched
// before pdl_wait(). Without a programmatic predecessor both are no-ops.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory"); }
__device__ __forceinline__ void pdl_enter() {
  pdl_wait();
  pdl_trigger();
}
bool pdl_enabled();  // TG_PDL=0 disables (A/B measurement)

// cudaLaunchKernelEx with the PDL attribute (+ an optional cluster size)
template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                            Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_k_cluster(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                                    int cluster_x, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = cluster_x;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

// device error bits (sticky)
enum : int { kErrNodeRange = 1, kErrIndexFull = 2, kErrDedupFull = 4, kErrEidRange = 8, kErrPairIndex = 16,
             kErrF16Range = 32 };

__host__ __device__ inline int round4(int x) { return (x + 3) & ~3; }

__device__ __forceinline__ unsigned long long mix64(unsigned long long k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdull;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ull;
  k ^= k >> 33;
  return k;
}

// Hash(n, t) of P:L282: node in the high 32 bits, time in the low 32 (R4).
__device__ __forceinline__ unsigned long long tkey(int32_t n, uint32_t t) {
  return ((unsigned long long)(uint32_t)n << 32) | (unsigned long long)t;
}

struct GraphDev {
  int64_t V, E;
  const int32_t* rowptr;
  const int32_t* adj_nbr;
  const int32_t* adj_eid;
  const uint32_t* adj_t;
  const float* X;
  const float* Ef;
  int d_n, d_e, ldn, lde;
};

struct CacheDev {
  unsigned long long* ikey;  // [icap]
  long long* ipos;           // [icap]
  unsigned long long imask;
  float* ring;               // [rcap x ldn]
  long long rcap;
  long long* state;          // device [8]: head, size, limit, occupied index slots, head at SB start,
                             // grid-wide pass valid (1) / ordered pass (0), min position of the
                             // superbatch's first-occurrence hits, slots filled by an index rebuild
  unsigned long long* rkey;  // [rcap] key stored at each ring slot (index rebuild)
  // host-mapped report word: ((superbatch + 1) << 40) | occupied slots, written by
  // k_probe_pre, read by the host without synchronising (rebuild trigger bound)
  unsigned long long* occ_report;
  long long report_sb;       // superbatch number of this launch (set per launch)
  // superbatch-scoped lookup hash in global memory (L2-resident), grid-wide eviction-free
  // CacheLookup pass (k_sbh_*): key -> min concatenated position j, then the ring slot of
  // the key's first occurrence. T = sb_mask + 1 >= 2 x (S x cap) slots.
  unsigned long long* sb_key;  // [T]
  unsigned* sb_val;            // [T] min j
  long long* sb_slot;          // [T] ring slot of the first occurrence
  int* sb_h;                   // [S x cap] table slot of each unique-list entry
  int* sb_blk;                 // [kSbhMaxBlocks] misses per scan block
  unsigned long long sb_mask;
};
constexpr int kSbhItems = 8, kSbhThreads = 1024, kSbhChunk = kSbhItems * kSbhThreads;
constexpr int kSbhMaxBlocks = 1024;  // S x cap <= 8.4M entries per cached level
// Index maintenance: the index never deletes, so FIFO churn (small limits) fills it with
// dead keys and absent-key probes lengthen; when more than half of the slots are occupied
// the index is rebuilt from the live ring window (clear, then re-insert keys of positions
// [head - size, head), newest position per key). Returns launches issued.
int launch_index_maint(const CacheDev& c, cudaStream_t st, int* err);
void launch_index_check(const CacheDev& c, int* err, cudaStream_t st);
constexpr int kIndexRebuildNum = 1, kIndexRebuildDen = 2;  // rebuild above 1/2 occupancy

// One recursion level l >= 1 of a superbatch.
struct LevelDev {
  int cap;                   // per-batch stride of the segmented lists
  // batch-segmented (stride cap): input I_l, unique U_l, inverse, ring slot per U entry
  int32_t* in_node;
  uint32_t* in_ts;
  int* n_in;                 // [S]
  int32_t* u_node;
  uint32_t* u_ts;
  int* n_u;                  // [S]
  int32_t* inv;
  long long* slot;
  long long* p0;             // index position of each U entry at superbatch start (-1: absent)
  // compute list C_l, compacted over the superbatch (q = 0..n_c_total-1)
  int32_t* c_b;              // batch of q
  int32_t* c_u;              // unique-list index of q inside its batch
  int32_t* c_node;
  uint32_t* c_ts;
  int* c_base;               // [S] first q of each batch
  int* n_c;                  // [S]
  int* n_c_total;            // [1]
  int c_cap;                 // S * cap
  unsigned char* sup;        // [S*cap] miss q superseded by a later re-miss of its key in the SB
  // sampled neighbours of each q (compute-centric [q*k + m])
  int32_t* nb_node;
  uint32_t* nb_ts;
  int32_t* nb_eid;
  // row addresses resolved for the layer-l compute
  const float** hs_row;      // [c_cap]     h^(l-1) of the target
  float* hs_dense;           // [c_cap x ldn] the same rows gathered densely (G1's A; may be null)
  const float** nb_row;      // [c_cap * k] h^(l-1) of each neighbour
  int32_t* nb_hidx;          // [c_cap * k] its row in the level's h tensor (X at l = 1, else ring l-1)
  float** dst_row;           // [c_cap]     where h^(l) goes (ring slot or H_L)
};

// per-superbatch counter rows: cnt[b * TG_NCOUNTERS + c]
__device__ __forceinline__ void cnt_add(long long* cnt, int b, int c, long long v) {
  if (cnt && v) atomicAdd((unsigned long long*)(cnt + (size_t)b * TG_NCOUNTERS + c), (unsigned long long)v);
}

// -------------------------------------------------------------- launchers
struct EdgeSrc {            // batch b of the superbatch = edges [e0 + b*B, +B) clipped to n_edges
  const int32_t* src;
  const int32_t* dst;
  const uint32_t* ts;
  const int32_t* neg;       // optional negative destinations (NEXT-3): targets src || dst || neg
  int64_t n_edges;
  int64_t e0;
  int B;
};

// DedupFilter (Alg. 2) of every batch segment of level `lv`, one cluster per batch.
// edge_mode: the level-L input is src || dst of the batch, read from `es`.
void launch_dedup(LevelDev lv, int S, int n_max, bool edge_mode, EdgeSrc es, long long* cnt, int layer,
                  bool dedup_on, int* err, cudaStream_t st);

// CacheLookup + compaction + slot assignment + index insert, sequential over
// the S batches (Alg. 1 l.7-10 and CacheStore, Alg. 3, in batch order).
// cache == nullptr: no lookup (top layer, R9, or cache disabled).
int launch_probe(LevelDev lv, int S, const CacheDev* cache, long long* cnt, int layer, int* err,
                 cudaStream_t st);  // returns the number of kernels launched

// NghLookup for every q of level `lv`; writes lv.nb_* and,
// if next != nullptr, the batch-segmented input list of level l-1 (Alg. 1 l.12).
void launch_sample(const GraphDev& g, LevelDev lv, int S, int k, const LevelDev* next, int W, int use_table,
                   long long* cnt, int layer, int* err, cudaStream_t st);

// Row addresses for the layer-l compute of every level (one launch).
struct ResolveArgs {
  LevelDev lv[TG_MAX_LAYERS + 1];
  float* ring[TG_MAX_LAYERS + 1];   // ring of level l (null for l = L)
  float* HL;
  const float* X;
  int ldn, k, L;
  int c_cap_max;
};
void launch_resolve(const ResolveArgs& a, int* err, cudaStream_t st);
// hs_dense[q] = *hs_row[q] for every computed target of levels l0..l1 (warp per row), so the
// key projection G1 reads a dense A operand (TMA tiles) instead of gathering rows. Level 1
// reads node features (front stream); level l >= 2 reads layer l-1 embeddings of the same
// superbatch, so it runs on the layer stream after layer l-1
void launch_gather_hs(const ResolveArgs& a, int l0, int l1, cudaStream_t st);

// Phi table [W x dtp] built on device with the same function as the direct path.
void launch_time_table(const float* omega, const float* phi, int d_t, int dtp, int W, float* table,
                       cudaStream_t st);
void launch_time_encode(const float* omega, const float* phi, const float* table, int d_t, int dtp, int W,
                        int use_table, const int64_t* delta, int64_t n, float* out, cudaStream_t st);

struct AttnArgs {
  const float* u;          // [nc x H*Dp], or [V+1 x H*Dp] rows selected by u_row
  const int32_t* u_row;    // if non-null: target p reads u row u_row[p] (level 1: node id, per-node table)
  float* c;                // [nc x H*Dp]
  const float* const* nb_row;
  const int32_t* nb_node;  // mask: node == 0 (R7)
  const uint32_t* nb_ts;
  const int32_t* nb_eid;
  const uint32_t* c_ts;
  const float* Ef;
  int lde;
  const float* omega;
  const float* phi;
  const float* table;
  int W, use_table;
  int dnp, dep, dtp, d_t, Dp, H, k;
  const int* nc_dev;
  int nc_max;
  unsigned short* c_h;     // if non-null: c written as bf16 [nc x ldc_h] (zero padded) instead of fp32
  int ldc_h;
  const int32_t* nb_hidx;  // row indices of nb_row in maps.h (gather path)
  long long phi_row0;      // >= 0: Phi rows of dt >= W precomputed at rows phi_row0 + p*k + m of maps.t
  const float* trows;      // base of the maps.t rows (table, or table + precomputed rows)
  // if rh_h: the target's own h^(l-1) row (hs_row[p], dnp floats) is also written as bf16 to
  // rh_h[p][rh_off : rh_off+dnp] (rh_off 16-byte aligned, >= Dp) and zeros to the rest of
  // [Dp, ld_rh): the h block of the merge-FFN input [LN(y) | h] (Eq. 7), read by G2 (residual
  // q, Eq. 4/6, TMA at column rh_off) and G3
  const float* const* hs_row;
  unsigned short* rh_h;
  int ld_rh, rh_off;
};
// TMA row-gather maps of the attention sources: h rows of the level, E rows, Phi table rows.
struct AttnMaps {
  CUtensorMap h, e, t;
  int valid;
};
tg_status attn_make_rows_map(const float* base, int row_elems, int ld, long long rows, CUtensorMap* out);

// Phi(t - t_j) rows of every (target, neighbour) pair with dt >= W (or no
// table) of levels 1..L, written to out + (row0[l] + q*k + m) * dtp (Eq. 8).
struct PhiRowsArgs {
  LevelDev lv[TG_MAX_LAYERS + 1];
  long long row0[TG_MAX_LAYERS + 1];
  float* out;
  const float* omega;
  const float* phi;
  int L, k, W, use_table, d_t, dtp;
};
void launch_phi_rows(const PhiRowsArgs& a, cudaStream_t st);
void launch_attn(const AttnArgs& a, const AttnMaps* maps, cudaStream_t st);

// C[M x N] = A[M x K] B^T + epilogue, fp32 CUDA cores (TG_PREC_FP32).
// A row p = seg0[p][0:K0] || seg1[p][0:K-K0] (seg pointers from arrays or dense bases).
struct GemmArgs {
  const float* const* a_rows0;  // if non-null: per-row pointers for segment 0
  const float* a_base0;         // else dense base
  int lda0;
  int K0;
  const float* const* a_rows1;  // segment 1 (K - K0 columns), may be null if K0 == K
  const float* a_base1;
  int lda1;
  const float* B;               // [N x K] row-major
  int N, K;
  const float* bias;            // [N] or null
  int relu;
  // output: dense C (ldc) or per-row destinations (either may be null)
  float* C;
  int ldc;
  float* const* c_rows;
  const int* m_dev;
  int m_max;
  // bf16 activation path (TG_PREC_BF16, tensor-core kernel only):
  //   a_h  : dense bf16 A [M x lda_h] covering all K columns (zero padded to lda_h);
  //          streamed into shared memory with cp.async instead of the row segments
  //   c_h  : bf16 copy of the output [M x ldc_h], columns [N, ldc_h) written as 0
  const unsigned short* a_h;
  int lda_h;
  unsigned short* c_h;
  int ldc_h;
  // fused LayerNorm epilogue (G2 in TG_PREC_BF16, tensor-core kernel only):
  //   x = acc + bias;  r = LN(x; ln_g, ln_b) over the valid columns
  //   c < ln_dn | ln_s1 <= c < ln_s1 + ln_de | ln_s2 <= c < ln_s2 + ln_dt (Eq. 6, R1),
  //   written as bf16 to c_h[:, 0:N] only. Row statistics are exchanged between the ntn
  //   CTAs of a thread-block cluster (DSMEM).
  int ln;
  const float* ln_g;
  const float* ln_b;
  int ln_dn, ln_de, ln_dt, ln_s1, ln_s2;
  int* err;                     // sticky device error word (F16X3 range check), may be null
};
void launch_gemm_simt(const GemmArgs& g, cudaStream_t st);

// LayerNorm over the true (unpadded) columns of each row (R1: eps 1e-5, biased var)
// of y + q, with the attention residual q = [h^(l-1) || 0 || Phi(0)] (Eq. 4)
// added on load (y = F c + b_fc comes from G2). r (fp32 [M x (Dp + dnp)] = [LN | h]) and/or rh
// (bf16 [M x ldrh] = [LN(y+q) | h^(l-1) | 0-pad], the A operand of the merge
// FFN) are written when non-null.
void launch_layernorm(const float* y, float* r, int Dp, int dn, int dnp, int de, int dep, int dt,
                      const float* gamma, const float* beta, const int* m_dev, int m_max,
                      const float* const* hs_rows, const float* phi0, unsigned short* rh, int ldrh, int rh_off,
                      cudaStream_t st);

// Scores p_e = sigmoid(MLP(h_src, h_dst)) (R10) for every edge of the superbatch:
// row resolution, hidden layer as a projection GEMM, then the W_a2 head.
void launch_score_rows(const float* HL, int ldh, LevelDev top, int S, EdgeSrc es, const float** rs,
                       const float** rd, long long* oidx, int* m_dev, cudaStream_t st);
void launch_score_head(const float* z, int ldz, const long long* oidx, int M, const float* Wa2, float ba2, int dn,
                       float* scores, cudaStream_t st);
// Row pointers of target pairs (pa[p], pb[p]) of a single-batch target list (tg_score_pairs).
void launch_pair_rows(const float* HL, int ldh, LevelDev top, int n_targets, const int32_t* pa, const int32_t* pb,
                      int n_pairs, const float** rs, const float** rd, long long* oidx, int* m_dev, int* err,
                      cudaStream_t st);
// out[i] = H_L[q(i)] for a single-batch embed call (DedupInvert, Alg. 1 l.20).
void launch_invert(const float* HL, int ldh, LevelDev top, int n, int dn, float* out, cudaStream_t st);
void launch_prep_nodes(const int32_t* nodes, const uint32_t* ts, int n, LevelDev top, cudaStream_t st);

void launch_set_int(int* p, int v, cudaStream_t st);

// fold the superbatch counter rows into the totals and the per-batch log
void launch_finish(long long* cnt_sb, int S, long long* total, long long* log, int64_t log_row0,
                   cudaStream_t st);

}  // namespace tg
