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
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/tg.h"

namespace tg {

constexpr unsigned long long kEmptyKey = 0xFFFFFFFFFFFFFFFFull;
constexpr unsigned long long kLockedKey = 0xFFFFFFFFFFFFFFFEull;
constexpr int kMaxK = 32;          // neighbours per target (warp lanes)
constexpr int kDedupThreads = 1024;
constexpr int kDedupIPT = 16;      // items per thread per CTA (ordered scan)
constexpr int kDedupSlots = 16384; // smem hash slots per CTA (load <= 0.5 target)

// device error bits (sticky)
enum : int { kErrNodeRange = 1, kErrIndexFull = 2, kErrDedupFull = 4, kErrEidRange = 8 };

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

// Target list of one recursion level: I_l = [C_{l+1} ; N(C_{l+1})] (Alg. 1 l.12).
struct Level {
  int32_t* node;   // [cap]
  uint32_t* ts;    // [cap]
  int cap;
};

struct CacheDev {
  unsigned long long* ikey;  // [icap]
  long long* ipos;           // [icap]
  unsigned long long imask;
  float* ring;               // [rcap x ldn]
  long long rcap;
  long long* state;          // device [4]: head, size, limit, occupied index slots
};

// -------------------------------------------------------------- launchers
// All launchers are stream-ordered; counts marked *_dev are device scalars.

// targets = src || dst at the batch's edge times; batch picked by *bidx
void launch_prep_edges(const int32_t* src, const int32_t* dst, const uint32_t* ts, int64_t n_edges,
                       int batch, const int* bidx, Level out, int* n_out_dev, cudaStream_t st);
void launch_prep_nodes(const int32_t* nodes, const uint32_t* ts, int n, Level out, int* n_out_dev,
                       cudaStream_t st);

// DedupFilter (Alg. 2); n from *n_dev (<= n_max). Writes U, inv, *nu_dev; adds counters.
void launch_dedup(Level in, const int* n_dev, int n_max, Level uniq, int32_t* inv, int* nu_dev,
                  long long* cnt_n, long long* cnt_u, bool dedup_on, int* err, cudaStream_t st);

// CacheLookup + slot assignment + index insert (Alg. 1 l.7-10, 17; Alg. 3).
// Writes the miss list C (as U indices and node/ts), slot[u] for every u.
void launch_probe(Level uniq, const int* nu_dev, int nu_max, CacheDev cache, bool cache_on,
                  int32_t* c_uidx, Level C, int* nc_dev, long long* slot, long long* cnt_layer,
                  int* err, cudaStream_t st);

// C_L = U_L (top layer: no lookup): identity miss list.
void launch_copy_level(Level in, const int* n_dev, int n_max, Level out, int32_t* c_uidx, int* n_out_dev,
                       long long* cnt_lookup_miss, cudaStream_t st);

// NghLookup: k most recent with t_j < t; writes I_{l-1} =
// [C ; N(C)] plus eid[p*k+m]; *n_next_dev = nC*(k+1).
void launch_sample(const GraphDev& g, Level C, const int* nc_dev, int nc_max, int k, Level next,
                   int32_t* eid, int* n_next_dev, int* err, cudaStream_t st);

// Row addresses for layer l: rows[j] for j in I_{l-1}; dst[p] for p in C_l.
void launch_resolve(const GraphDev& g, int lm1_is_zero, Level prev, const int* nprev_dev, int nprev_max,
                    const int32_t* inv_prev, const long long* slot_prev, const float* ring_prev,
                    long long rcap_prev, int ld, const int* nc_dev, int nc_max, const int32_t* c_uidx,
                    const long long* slot_cur, float* ring_cur, long long rcap_cur, float* hl_out,
                    const float** rows, float** dst, int* err, cudaStream_t st);

// Phi table [W x dtp] built on device with the same function as the direct path.
void launch_time_table(const float* omega, const float* phi, int d_t, int dtp, int W, float* table,
                       cudaStream_t st);
void launch_time_encode(const float* omega, const float* phi, const float* table, int d_t, int dtp, int W,
                        int use_table, const int64_t* delta, int64_t n, float* out, cudaStream_t st);

struct AttnArgs {
  const float* u;          // [nc x 2Dp] (H*Dp)
  float* c;                // [nc x H*Dp]
  const float** rows;      // I_{l-1} row addresses
  const int32_t* prev_node;   // I_{l-1} nodes (mask: node == 0)
  const uint32_t* prev_ts;    // I_{l-1} times
  const int32_t* eid;      // [nc x k]
  const float* Ef;
  int lde;
  const float* omega;
  const float* phi;
  const float* table;
  int W, use_table;
  int dnp, dep, dtp, d_t, Dp, H, k;
  const int* nc_dev;
  int nc_max;
  long long* cnt_ttable;   // [2] table, direct
};
void launch_attn(const AttnArgs& a, cudaStream_t st);

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
  // residual q = [hs || 0 || Phi0] added in the epilogue (G2), if q_rows != null
  const float* const* q_rows;
  int q_dnp, q_dep;
  const float* q_phi0;          // [dtp]
  // output: dense C (ldc) or per-row destinations
  float* C;
  int ldc;
  float* const* c_rows;
  const int* m_dev;
  int m_max;
};
void launch_gemm_simt(const GemmArgs& g, cudaStream_t st);

// LayerNorm over the true (unpadded) columns of each row (R1: eps 1e-5, biased var).
void launch_layernorm(const float* y, float* r, int Dp, int dn, int dnp, int de, int dep, int dt,
                      const float* gamma, const float* beta, const int* m_dev, int m_max, cudaStream_t st);

// Scores p_e = sigmoid(MLP(h_src, h_dst)) (R10) and inversion out[i] = H_L[inv[i]].
void launch_score(const float* HL, int ldh, const int32_t* inv, int n_edges, int batch, const int* bidx,
                  const float* Wa1, const float* ba1, const float* Wa2, float ba2, int dn, int dnp,
                  float* scores, cudaStream_t st);
void launch_invert(const float* HL, int ldh, const int32_t* inv, int n, int dn, float* out, cudaStream_t st);

void launch_bump(int* bidx, cudaStream_t st);
void launch_add_counters(const long long* src, long long* dst, int n, cudaStream_t st);

}  // namespace tg
