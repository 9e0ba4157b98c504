// C ABI of libtg (include/tg.h): context, loading, and the orchestration of
// Alg. 1 over a superbatch of S chronological batches as one
// chain of stream-ordered sm_100a kernels with device-resident counts (no
// host sync inside the chain).
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include "tg_internal.cuh"
#include "tg_tc.cuh"

using namespace tg;

bool tg::pdl_enabled() {
  static const bool on = [] {
    const char* e = getenv("TG_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

namespace {

struct LayerW {
  float *P = nullptr, *bu = nullptr, *F = nullptr, *bfc = nullptr, *lng = nullptr, *lnb = nullptr;
  float* bfcq = nullptr;  // b_fc + [0 | 0 | Phi(0)]: the constant part of the residual q (fused LN epilogue)
  float *W1 = nullptr, *b1 = nullptr, *W2 = nullptr, *b2 = nullptr;
  TcWeights tcP, tcF, tcW1, tcW2;  // tensor-core operand copies (TG_PREC_TF32X3 / BF16)
  TcWeights tcFa;  // BF16: [F | I_h] -- G2 with the residual h^(l-1) as extra K (identity block)
  int fa_kb0 = 0;  // first k-block of the identity block
};

}  // namespace

struct tg_ctx {
  int device = 0;
  bool broken = false;
  // graph
  GraphDev g{};
  int32_t *rowptr = nullptr, *adj_nbr = nullptr, *adj_eid = nullptr;
  uint32_t* adj_t = nullptr;
  float *X = nullptr, *Ef = nullptr;
  // model
  bool loaded = false;
  tg_model_cfg cfg{};
  int L = 0, H = 0, k = 0, d_n = 0, d_e = 0, d_t = 0, dnp = 0, dep = 0, dtp = 0, Dp = 0, W = 0, S = 1;
  // Wt: rows of the device Phi table. The paper's window W fixes which dt count as
  // served by the precomputed table (the t_table / t_direct counters, the ablation); the table
  // itself extends to Wt = min(max t + 1, 4M) rows (same bits as the direct path, R5), so the
  // kernels gather Phi(dt) for every dt < Wt instead of recomputing it
  int Wt = 0;
  uint32_t max_ts = 0;
  LayerW lw[TG_MAX_LAYERS];
  float *omega = nullptr, *phi = nullptr, *table = nullptr;
  float *Wa1 = nullptr, *ba1 = nullptr, *Wa2 = nullptr;
  float ba2 = 0.f;
  TcWeights tcWa1;
  TcWeights tcWa1g;  // BF16 config: W_a1 as a 1-pass tf32 image (gathered fp32 H_L rows)
  // score workspace (S * B edges)
  const float** sc_rs = nullptr;
  const float** sc_rd = nullptr;
  long long* sc_oidx = nullptr;
  float* sc_z = nullptr;
  int* sc_m = nullptr;
  // recursion levels (index l = 1..L), caches for l = 1..L-1. Two sets: the
  // front half of superbatch i+1 (dedup, lookup, sampling, resolve) fills one
  // set on the front stream while the layers of superbatch i read the other.
  LevelDev lvs[2][TG_MAX_LAYERS + 1]{};
  LevelDev* lv = lvs[0];
  int cap[TG_MAX_LAYERS + 1]{};
  CacheDev cache[TG_MAX_LAYERS]{};
  long long* cache_state = nullptr;
  int64_t limit0 = 0;
  long long idx_bound[TG_MAX_LAYERS + 1]{};  // host upper bound on occupied index slots (rebuild trigger)
  unsigned long long* occ_h = nullptr;       // host-mapped [TG_MAX_LAYERS + 1] occupancy reports
  long long sb_count = 0;                    // superbatches issued since the last cache reset
  long long targets_issued = 0;              // layer-L targets issued since the last cache reset
  // compute workspace
  int maxC = 0;
  float *u = nullptr, *c = nullptr, *y = nullptr, *r = nullptr, *z = nullptr, *HL = nullptr;
  // U1 [(V+1) x H*Dp]: the layer-1 query side u = P x_i + b_u of every node (R27). Layer-1
  // targets' h^(0) is the node's static feature row, so u is a function of the node
  // alone: computed once at tg_model_load by the same GEMM (row-invariant: the bits G1 would
  // produce per target); null when it would exceed the budget (G1 per target then)
  float* u1 = nullptr;
  int* u1_m = nullptr;
  // bf16 activations (TG_PREC_BF16): c, [LN(y) | h], z with row strides padded to 8
  unsigned short *c_h = nullptr, *rh_h = nullptr, *z_h = nullptr;
  int ld_ch = 0, ld_rh = 0, ld_z = 0;
  int dpa = 0;  // BF16 merge-FFN input row [LN(y) (Dp) | 0 | h at dpa = round8(Dp) (16-byte aligned) | 0]
  TcTensorA ta_c, ta_rh, ta_z;  // TMA tensor maps of the bf16 activations (dense GEMM A operands)
  TcTensorA ta_c32, ta_z32, ta_r32;  // fp32-level modes: fp32 c, z and [LN | h], feeding the GEMM staging
  TcTensorA ta_hs[2][TG_MAX_LAYERS + 1];  // fp32-level modes: dense h^(l-1) rows of each set / level (G1)
  AttnMaps am[2][TG_MAX_LAYERS + 1]{};  // per set and level l: TMA row-gather maps (h rows, E rows, Phi rows)
  int cur_set = 0;
  // Phi rows per set: [table (W rows) | direct rows of level 1 | level 2 | ...] (k_phi_rows, front stream)
  float* phi_buf[2] = {nullptr, nullptr};
  long long phi_row0[TG_MAX_LAYERS + 1]{};
  bool phi_pre = false;
  // counters / flags
  long long* cnt_total = nullptr;
  long long* cnt_sb = nullptr;  // [kMaxS x TG_NCOUNTERS] of the current set
  long long* cnt_sbs[2] = {nullptr, nullptr};
  // front stream + events of the two-set pipeline (stream_edges)
  cudaStream_t fst = nullptr;
  cudaStream_t lst = nullptr;      // layer stream at the highest priority (TG_LAYER_PRIO=1)
  cudaEvent_t ev_lend = nullptr;
  cudaEvent_t ev_front[2] = {nullptr, nullptr}, ev_back[2] = {nullptr, nullptr}, ev_in = nullptr, ev_fend = nullptr;
  int* err = nullptr;
  int64_t launches = 0;
  // per-stage profiling (events around launches)
  bool prof = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<int> ev_stage;
  size_t ev_used = 0;
  // tg_gemm unit entry: device M and prepared-weight cache
  int* gemm_m = nullptr;
  struct GemmCacheEntry {
    const float* B;
    int N, K, prec;
    TcWeights w;
  };
  std::vector<GemmCacheEntry> gemm_cache;
  // staging for host buffers
  void* stage = nullptr;
  size_t stage_bytes = 0;
  std::vector<void*> owned;
  std::vector<void*> owned_host;  // pinned host allocations (TG_OPT_HOST_CACHE rings)
};

namespace {

#define CK(x)                                                                                         \
  do {                                                                                                \
    cudaError_t e_ = (x);                                                                             \
    if (e_ != cudaSuccess) {                                                                          \
      fprintf(stderr, "libtg: CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      return e_ == cudaErrorMemoryAllocation ? TG_ENOMEM : TG_ECUDA;                                  \
    }                                                                                                 \
  } while (0)

#define TRY(x)                  \
  do {                          \
    tg_status s_ = (x);         \
    if (s_ != TG_OK) return s_; \
  } while (0)

template <class T>
tg_status dalloc(tg_ctx* ctx, T** p, size_t n) {
  void* q = nullptr;
  if (n == 0) n = 1;
  cudaError_t e = cudaMalloc(&q, n * sizeof(T));
  if (e != cudaSuccess) {
    cudaGetLastError();
    return TG_ENOMEM;
  }
  ctx->owned.push_back(q);
  *p = reinterpret_cast<T*>(q);
  return TG_OK;
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Bracket a launch with an event pair when profiling is on (Table 3 style breakdown).
struct Prof {
  tg_ctx* ctx;
  cudaEvent_t e1 = nullptr;
  cudaStream_t stream = nullptr;
  Prof(tg_ctx* c, int stage, cudaStream_t st) : ctx(c) {
    if (!c->prof) return;
    if (c->ev_used * 2 + 2 > c->ev_pool.size()) {
      for (int i = 0; i < 256; ++i) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        c->ev_pool.push_back(e);
      }
    }
    cudaEvent_t e0 = c->ev_pool[2 * c->ev_used];
    e1 = c->ev_pool[2 * c->ev_used + 1];
    if (c->ev_stage.size() <= c->ev_used) c->ev_stage.resize(c->ev_used + 1);
    c->ev_stage[c->ev_used] = stage;
    ++c->ev_used;
    stream = st;
    cudaEventRecord(e0, st);
  }
  ~Prof() {
    if (e1) cudaEventRecord(e1, stream);
  }
};

tg_status launched(tg_ctx* ctx, int n = 1) {
  ctx->launches += n;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    fprintf(stderr, "libtg: launch error %s\n", cudaGetErrorString(e));
    ctx->broken = true;
    return TG_ECUDA;
  }
  return TG_OK;
}

tg_status ensure_stage(tg_ctx* ctx, size_t bytes) {
  if (ctx->stage_bytes >= bytes) return TG_OK;
  if (ctx->stage) cudaFree(ctx->stage);
  ctx->stage = nullptr;
  ctx->stage_bytes = 0;
  CK(cudaMalloc(&ctx->stage, bytes));
  ctx->stage_bytes = bytes;
  return TG_OK;
}

inline int pc(const tg_ctx* ctx, int a) {  // D-space index -> padded kv index
  if (a < ctx->d_n) return a;
  if (a < ctx->d_n + ctx->d_e) return ctx->dnp + (a - ctx->d_n);
  return ctx->dnp + ctx->dep + (a - ctx->d_n - ctx->d_e);
}

// ------------------------------------------------------------------------
// Dense stages of layer l over its compute list (Eqs. 4-7).
// ------------------------------------------------------------------------
tg_status run_layer(tg_ctx* ctx, int l, cudaStream_t st) {
  const LayerW& w = ctx->lw[l - 1];
  const LevelDev& lv = ctx->lv[l];
  const int HDp = ctx->H * ctx->Dp;
  const int mmax = lv.c_cap;
  const bool tc = ctx->cfg.precision != TG_PREC_FP32;
  const int* m_dev = lv.n_c_total;
  // G1: u = P h^(l-1) + bu  (target-side K projection with W_q and 1/sqrt(d_k) folded)
  // level 1: the node-feature rows were gathered densely on the front stream (TMA-fed A);
  // levels >= 2 read layer l-1 embeddings of this superbatch through their row pointers
  // (densifying them here on the layer stream measured no faster: 9.31 vs 9.35 M edges/s)
  const bool u1 = l == 1 && ctx->u1;  // layer 1: u rows from the per-node table (no G1)
  const bool dense_hs = lv.hs_dense && l == 1;
  GemmArgs g1{};
  g1.err = ctx->err;
  g1.a_rows0 = dense_hs ? nullptr : lv.hs_row;
  g1.a_base0 = dense_hs ? lv.hs_dense : nullptr;
  g1.lda0 = ctx->dnp;
  g1.K0 = g1.K = ctx->dnp;
  g1.B = w.P;
  g1.N = HDp;
  g1.bias = w.bu;
  g1.C = ctx->u;
  g1.ldc = HDp;
  g1.m_dev = m_dev;
  g1.m_max = mmax;
  if (!u1) {
    {
      Prof pf(ctx, TG_ST_PROJ_K, st);
      if (tc) launch_gemm_tc(g1, w.tcP, ctx->cfg.precision, st, dense_hs ? &ctx->ta_hs[ctx->cur_set][l] : nullptr);
      else launch_gemm_simt(g1, st);
    }
    TRY(launched(ctx));
  }
  // attention over the k sampled neighbours
  AttnArgs a{};
  a.u = u1 ? ctx->u1 : ctx->u;
  a.u_row = u1 ? lv.c_node : nullptr;
  a.c = ctx->c;
  a.nb_row = lv.nb_row;
  a.nb_node = lv.nb_node;
  a.nb_ts = lv.nb_ts;
  a.nb_eid = lv.nb_eid;
  a.c_ts = lv.c_ts;
  a.Ef = ctx->Ef;
  a.lde = ctx->g.lde;
  a.omega = ctx->omega;
  a.phi = ctx->phi;
  a.table = ctx->table;
  a.W = ctx->Wt;
  a.use_table = (ctx->cfg.opts & TG_OPT_TTABLE) ? 1 : 0;
  a.dnp = ctx->dnp;
  a.dep = ctx->dep;
  a.dtp = ctx->dtp;
  a.d_t = ctx->d_t;
  a.Dp = ctx->Dp;
  a.H = ctx->H;
  a.k = ctx->k;
  a.nc_dev = m_dev;
  a.nc_max = mmax;
  a.nb_hidx = lv.nb_hidx;
  a.phi_row0 = ctx->phi_pre ? ctx->phi_row0[l] : -1;
  a.trows = ctx->phi_pre ? ctx->phi_buf[ctx->cur_set] : ctx->table;
  const bool bfa = ctx->cfg.precision == TG_PREC_BF16;  // bf16 activations between the GEMMs
  const bool x3 = ctx->cfg.precision == TG_PREC_TF32X3 || ctx->cfg.precision == TG_PREC_F16X3;
  // TG_LN_FUSE=1: LayerNorm in G2's epilogue (thread-block clusters, DSMEM statistics);
  // measured slower end to end than G2 + k_layernorm, so off by default
  static const bool ln_fuse_env = [] {
    const char* e = getenv("TG_LN_FUSE");
    return e && e[0] == '1';
  }();
  const bool fuse = bfa && ln_fuse_env;
  if (bfa) {
    a.c = nullptr;
    a.c_h = ctx->c_h;
    a.ldc_h = ctx->ld_ch;
  }
  if (fuse) {
    a.hs_row = lv.hs_row;  // h block of the merge-FFN input, also G2's identity-block operand
    a.rh_h = ctx->rh_h;
    a.ld_rh = ctx->ld_rh;
    a.rh_off = ctx->dpa;
  }
  {
    Prof pf(ctx, TG_ST_ATTN, st);
    launch_attn(a, &ctx->am[ctx->cur_set][l], st);
  }
  static const bool attn_sync = getenv("TG_ATTN_SYNC") != nullptr;  // debug
  if (attn_sync) cudaStreamSynchronize(st);
  static const bool attn_check = getenv("TG_ATTN_CHECK") != nullptr;  // debug: gather vs CTA kernel
  if (attn_check && !bfa) {
    int nc = 0;
    cudaStreamSynchronize(st);
    cudaMemcpy(&nc, m_dev, sizeof(int), cudaMemcpyDeviceToHost);
    float* ref = nullptr;
    cudaMalloc(&ref, (size_t)std::max(nc, 1) * HDp * sizeof(float));
    AttnArgs b = a;
    b.c = ref;
    b.nb_hidx = nullptr;  // forces the CTA kernel
    launch_attn(b, nullptr, st);
    cudaStreamSynchronize(st);
    std::vector<float> x((size_t)nc * HDp), y((size_t)nc * HDp);
    cudaMemcpy(x.data(), ctx->c, x.size() * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(y.data(), ref, y.size() * 4, cudaMemcpyDeviceToHost);
    if (getenv("TG_ATTN_USE_REF")) cudaMemcpy(ctx->c, ref, y.size() * 4, cudaMemcpyDeviceToDevice);
    cudaFree(ref);
    int bad = 0;
    float gmd = 0.f;
    for (int p = 0; p < nc; ++p) {
      float md = 0.f, mag = 0.f;
      int jw = 0;
      for (int j = 0; j < HDp; ++j) mag = std::max(mag, std::fabs(y[(size_t)p * HDp + j]));
      for (int j = 0; j < HDp; ++j) {
        const float d = std::fabs(x[(size_t)p * HDp + j] - y[(size_t)p * HDp + j]) / (1e-20f + mag);
        if (d > md) {
          md = d;
          jw = j;
        }
      }
      gmd = std::max(gmd, md);
      if (md > 1e-5f && bad++ < 8)
        fprintf(stderr, "attn check: level %d target %d/%d max diff/rowmax %g at col %d (got %g ref %g)\n", l, p, nc,
                md, jw, x[(size_t)p * HDp + jw], y[(size_t)p * HDp + jw]);
    }
    fprintf(stderr, "attn check: level %d: %d of %d targets differ (max rel %g)\n", l, bad, nc, gmd);
    {
      const size_t nr = (size_t)nc * ctx->k;
      std::vector<const float*> rp(nr);
      std::vector<int32_t> hi(nr);
      cudaMemcpy(rp.data(), lv.nb_row, nr * sizeof(void*), cudaMemcpyDeviceToHost);
      cudaMemcpy(hi.data(), lv.nb_hidx, nr * 4, cudaMemcpyDeviceToHost);
      const float* hb = l == 1 ? ctx->X : ctx->cache[l - 1].ring;
      int nbad = 0;
      for (size_t i = 0; i < nr; ++i)
        if (rp[i] != hb + (size_t)hi[i] * ctx->g.ldn && nbad++ < 4)
          fprintf(stderr, "attn check: row %zu ptr off %td vs idx %d\n", i, (rp[i] - hb), hi[i]);
      fprintf(stderr, "attn check: level %d: %d of %zu row indices inconsistent\n", l, nbad, nr);
    }
  }
  TRY(launched(ctx));
  // G2: y = F c + b_fc  (W_v and W_fc folded; the residual q of Eq. 4 is added by the LayerNorm)
  GemmArgs g2{};
  g2.err = ctx->err;
  g2.a_base0 = ctx->c;
  g2.lda0 = HDp;
  g2.K0 = g2.K = HDp;
  g2.B = w.F;
  g2.N = ctx->Dp;
  g2.bias = w.bfc;
  g2.C = ctx->y;
  g2.ldc = ctx->Dp;
  g2.m_dev = m_dev;
  g2.m_max = mmax;
  if (bfa) {
    g2.a_h = ctx->c_h;
    g2.lda_h = ctx->ld_ch;
  }
  if (fuse) {
    // residual q (h through the identity block of tcFa, Phi(0) in bfcq) + LayerNorm fused
    // into the epilogue, which writes the bf16 LN(y) block of the merge-FFN input
    g2.ln = 1;
    g2.bias = w.bfcq;
    g2.ln_g = w.lng;
    g2.ln_b = w.lnb;
    g2.ln_dn = ctx->d_n;
    g2.ln_de = ctx->d_e;
    g2.ln_dt = ctx->d_t;
    g2.ln_s1 = ctx->dnp;
    g2.ln_s2 = ctx->dnp + ctx->dep;
    g2.C = nullptr;
    g2.c_h = ctx->rh_h;
    g2.ldc_h = ctx->ld_rh;
  }
  {
    Prof pf(ctx, TG_ST_PROJ_V, st);
    if (fuse) launch_gemm_tc(g2, w.tcFa, ctx->cfg.precision, st, &ctx->ta_c, &ctx->ta_rh, w.fa_kb0, ctx->dpa);
    else if (tc) launch_gemm_tc(g2, w.tcF, ctx->cfg.precision, st, bfa ? &ctx->ta_c : (x3 ? &ctx->ta_c32 : nullptr));
    else launch_gemm_simt(g2, st);
  }
  TRY(launched(ctx));
  if (!fuse) {
    Prof pf(ctx, TG_ST_LNORM, st);
    launch_layernorm(ctx->y, bfa ? nullptr : ctx->r, ctx->Dp, ctx->d_n, ctx->dnp, ctx->d_e, ctx->dep, ctx->d_t,
                     w.lng, w.lnb, m_dev, mmax, lv.hs_row, ctx->table /* Phi(0): row 0 */,
                     bfa ? ctx->rh_h : nullptr, ctx->ld_rh, ctx->dpa, st);
    TRY(launched(ctx));
  }
  // G3: z = ReLU(W1 [r || h^(l-1)] + b1)  (Eq. 7); the LayerNorm wrote the dense row [r | h]
  GemmArgs g3{};
  g3.err = ctx->err;
  g3.a_base0 = ctx->r;
  g3.lda0 = ctx->Dp + ctx->dnp;
  g3.K0 = g3.K = ctx->Dp + ctx->dnp;
  g3.B = w.W1;
  g3.N = ctx->dnp;
  g3.bias = w.b1;
  g3.relu = 1;
  g3.C = ctx->z;
  g3.ldc = ctx->dnp;
  g3.m_dev = m_dev;
  g3.m_max = mmax;
  if (bfa) {
    g3.a_h = ctx->rh_h;
    g3.lda_h = ctx->ld_rh;
    g3.C = nullptr;
    g3.c_h = ctx->z_h;
    g3.ldc_h = ctx->ld_z;
  }
  {
    Prof pf(ctx, TG_ST_FFN1, st);
    if (tc) launch_gemm_tc(g3, w.tcW1, ctx->cfg.precision, st, bfa ? &ctx->ta_rh : (x3 ? &ctx->ta_r32 : nullptr));
    else launch_gemm_simt(g3, st);
  }
  TRY(launched(ctx));
  // G4: h = W2 z + b2 -> ring slot (CacheStore payload, Alg. 3 l.8-10) or H_L
  GemmArgs g4{};
  g4.err = ctx->err;
  g4.a_base0 = ctx->z;
  g4.lda0 = ctx->dnp;
  g4.K0 = g4.K = ctx->dnp;
  g4.B = w.W2;
  g4.N = ctx->dnp;
  g4.bias = w.b2;
  g4.c_rows = lv.dst_row;
  g4.m_dev = m_dev;
  g4.m_max = mmax;
  if (bfa) {
    g4.a_h = ctx->z_h;
    g4.lda_h = ctx->ld_z;
  }
  {
    Prof pf(ctx, TG_ST_FFN2, st);
    if (tc) launch_gemm_tc(g4, w.tcW2, ctx->cfg.precision, st, bfa ? &ctx->ta_z : (x3 ? &ctx->ta_z32 : nullptr));
    else launch_gemm_simt(g4, st);
  }
  return launched(ctx);
}

// ------------------------------------------------------------------------
// Embed(L, .) for S batches (Alg. 1): edge_mode -> batches of the stream
// (targets src || dst), else one batch of explicit targets (prepared in lv[L]).
// ------------------------------------------------------------------------
void select_set(tg_ctx* ctx, int s) {
  ctx->cur_set = s;
  ctx->lv = ctx->lvs[s];
  ctx->cnt_sb = ctx->cnt_sbs[s];
}

// Top-down half (Alg. 1 l.5-12) and row resolution: reads only the inputs, the
// graph and the cache index, writes the current level set.
tg_status run_front(tg_ctx* ctx, int S, bool edge_mode, const EdgeSrc& es, int n_max_top, cudaStream_t st) {
  const int L = ctx->L, k = ctx->k;
  const bool dedup = ctx->cfg.opts & TG_OPT_DEDUP;
  const bool cache_on = ctx->cfg.opts & TG_OPT_CACHE;
  const int use_table = (ctx->cfg.opts & TG_OPT_TTABLE) ? 1 : 0;
  long long* cnt = ctx->cnt_sb;
  ctx->targets_issued += edge_mode ? (es.neg ? 3 : 2) * std::min<int64_t>((int64_t)S * es.B, es.n_edges - es.e0)
                                   : (long long)S * n_max_top;
  // ---- top-down (Alg. 1 l.5-12): dedup, lookup/compaction, sampling
  {
    Prof pf(ctx, TG_ST_DEDUP, st);
    launch_dedup(ctx->lv[L], S, n_max_top, edge_mode, es, cnt, L, dedup, ctx->err, st);
  }
  TRY(launched(ctx));
  int nl;
  {
    Prof pf(ctx, TG_ST_LOOKUP, st);
    nl = launch_probe(ctx->lv[L], S, nullptr, cnt, L, ctx->err, st);  // no lookup at l = L
  }
  TRY(launched(ctx, nl));
  for (int l = L; l >= 1; --l) {
    {
      Prof pf(ctx, TG_ST_SAMPLE, st);
      launch_sample(ctx->g, ctx->lv[l], S, k, l >= 2 ? &ctx->lv[l - 1] : nullptr, ctx->W, use_table, cnt, l,
                    ctx->err, st);
    }
    TRY(launched(ctx));
    if (l >= 2) {
      {
        Prof pf(ctx, TG_ST_DEDUP, st);
        launch_dedup(ctx->lv[l - 1], S, ctx->cap[l - 1], false, es, cnt, l - 1, dedup, ctx->err, st);
      }
      TRY(launched(ctx));
      CacheDev cd = ctx->cache[l - 1];
      if (!cache_on) cd.ikey = nullptr;  // ring used as scratch only
      if (cache_on) {  // index rebuild when it may exceed half occupancy (host upper bound)
        const long long slots = (long long)cd.imask + 1, per_sb = (long long)S * ctx->cap[l - 1];
        ctx->idx_bound[l - 1] += per_sb;
        // tighter bound from the latest device report (occupancy before superbatch sb_obs's
        // inserts): + at most per_sb for each superbatch since (rebuilds only lower it)
        // key universe: every cached-level key is a graph edge endpoint (node, t_e), a
        // layer-L target, or <0, 0>; and a re-inserted (evicted) key reuses its own slot or an
        // earlier dead one, never an empty slot -> occupied slots <= distinct keys inserted
        const long long universe = 2 * ctx->g.E + 1 + ctx->targets_issued;
        if (universe < ctx->idx_bound[l - 1]) ctx->idx_bound[l - 1] = universe;
        const unsigned long long rep = ctx->occ_h ? *(volatile unsigned long long*)&ctx->occ_h[l - 1] : 0ull;
        const long long sb_obs = (long long)(rep >> 40) - 1;
        if (sb_obs >= 0 && sb_obs <= ctx->sb_count) {
          const long long b = (long long)(rep & ((1ull << 40) - 1)) + (ctx->sb_count - sb_obs + 1) * per_sb;
          if (b < ctx->idx_bound[l - 1]) ctx->idx_bound[l - 1] = b;
        }
        cd.occ_report = ctx->occ_h ? ctx->occ_h + (l - 1) : nullptr;
        cd.report_sb = ctx->sb_count;
        if (ctx->idx_bound[l - 1] * kIndexRebuildDen > slots * kIndexRebuildNum) {
          Prof pf(ctx, TG_ST_LOOKUP, st);
          TRY(launched(ctx, launch_index_maint(cd, st, ctx->err)));
          ctx->idx_bound[l - 1] = slots * kIndexRebuildNum / kIndexRebuildDen;  // <= threshold afterwards
        }
      }
      {
        Prof pf(ctx, TG_ST_LOOKUP, st);
        nl = launch_probe(ctx->lv[l - 1], S, &cd, cnt, l - 1, ctx->err, st);
        static const bool dbg_check = getenv("TG_DBG_INDEX_CHECK") != nullptr;
        if (dbg_check && cache_on) launch_index_check(cd, ctx->err, st);
      }
      TRY(launched(ctx, nl));
    }
  }
  ++ctx->sb_count;
  // ---- row addresses for every layer
  ResolveArgs ra{};
  for (int l = 0; l <= L; ++l) ra.lv[l] = ctx->lv[l];
  for (int l = 1; l < L; ++l) ra.ring[l] = ctx->cache[l].ring;
  ra.HL = ctx->HL;
  ra.X = ctx->X;
  ra.ldn = ctx->dnp;
  ra.k = k;
  ra.L = L;
  ra.c_cap_max = ctx->maxC;
  {
    Prof pf(ctx, TG_ST_RESOLVE, st);
    launch_resolve(ra, ctx->err, st);
  }
  TRY(launched(ctx));
  if (ctx->lv[1].hs_dense && !ctx->u1) {  // fp32-level modes: G1's A rows of level 1 (node features) made dense
    Prof pf(ctx, TG_ST_RESOLVE, st);
    launch_gather_hs(ra, 1, 1, st);
    TRY(launched(ctx));
  }
  if (ctx->phi_pre && ctx->am[ctx->cur_set][1].valid) {  // TimeEncode of the dt >= W rows (Eq. 8)
    PhiRowsArgs pa{};
    for (int l = 0; l <= L; ++l) {
      pa.lv[l] = ctx->lv[l];
      pa.row0[l] = ctx->phi_row0[l];
    }
    pa.out = ctx->phi_buf[ctx->cur_set];
    pa.omega = ctx->omega;
    pa.phi = ctx->phi;
    pa.L = L;
    pa.k = k;
    pa.W = ctx->Wt;
    pa.use_table = use_table;
    pa.d_t = ctx->d_t;
    pa.dtp = ctx->dtp;
    {
      Prof pf(ctx, TG_ST_PHI, st);
      launch_phi_rows(pa, st);
    }
    TRY(launched(ctx));
  }
  return TG_OK;
}

// Bottom-up half (Alg. 1 l.13-18): M and FFN, layer by layer over all S batches.
tg_status run_back(tg_ctx* ctx, cudaStream_t st) {
  for (int l = 1; l <= ctx->L; ++l) TRY(run_layer(ctx, l, st));
  return TG_OK;
}

tg_status run_superbatch(tg_ctx* ctx, int S, bool edge_mode, const EdgeSrc& es, int n_max_top, cudaStream_t st) {
  TRY(run_front(ctx, S, edge_mode, es, n_max_top, st));
  return run_back(ctx, st);
}

tg_status finish(tg_ctx* ctx, int S, long long* log, int64_t row0, cudaStream_t st) {
  {
    Prof pf(ctx, TG_ST_OTHER, st);
    launch_finish(ctx->cnt_sb, S, ctx->cnt_total, log, row0, st);
  }
  return launched(ctx);
}

tg_status stream_edges(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts, const int32_t* neg,
                       int64_t n_edges, int batch, float* scores, long long* log, cudaStream_t st_in) {
  const int64_t nb = (n_edges + batch - 1) / batch;
  static const bool prio = [] {  // experiment: layers on a high-priority stream, front on the lowest
    const char* e = getenv("TG_LAYER_PRIO");
    return e && e[0] == '1';
  }();
  cudaStream_t st = st_in;
  // Two-set pipeline: superbatch i's front half runs on ctx->fst into level set
  // i % 2 as soon as superbatch i-2's layers released that set, overlapping the
  // layers of superbatch i-1 on st. The cache index is only touched by front
  // halves (in order on fst) and ring rows only by layers (in order on st), so
  // every kernel sees the same data as in the serial order.
  CK(cudaEventRecord(ctx->ev_in, st));
  CK(cudaStreamWaitEvent(ctx->fst, ctx->ev_in, 0));
  if (prio) {
    st = ctx->lst;
    CK(cudaStreamWaitEvent(st, ctx->ev_in, 0));
  }
  int64_t sb = 0;
  for (int64_t b0 = 0, S = 0; b0 < nb; b0 += S, ++sb) {
    S = std::min<int64_t>(ctx->S, nb - b0);
    const int set = (int)(sb & 1);
    EdgeSrc es{src, dst, ts, neg, n_edges, b0 * batch, batch};
    const int per_edge = neg ? 3 : 2;  // targets per edge: src || dst (|| neg, NEXT-3)
    select_set(ctx, set);
    if (sb >= 2) CK(cudaStreamWaitEvent(ctx->fst, ctx->ev_back[set], 0));
    static const bool one_stream = getenv("TG_ONE_STREAM") != nullptr;  // debug: no overlap
    TRY(run_front(ctx, S, true, es, per_edge * batch, one_stream ? st : ctx->fst));
    if (one_stream) CK(cudaEventRecord(ctx->ev_front[set], st));
    CK(cudaEventRecord(ctx->ev_front[set], ctx->fst));
    CK(cudaStreamWaitEvent(st, ctx->ev_front[set], 0));
    TRY(run_back(ctx, st));
    {
      Prof pf(ctx, TG_ST_SCORE, st);
      launch_score_rows(ctx->HL, ctx->dnp, ctx->lv[ctx->L], S, es, ctx->sc_rs, ctx->sc_rd, ctx->sc_oidx, ctx->sc_m,
                        st);
      GemmArgs g{};  // hidden layer of the affinity MLP: ReLU(W_a1 [h_src || h_dst] + b_a1)
      g.err = ctx->err;
      g.a_rows0 = ctx->sc_rs;
      g.K0 = ctx->dnp;
      g.a_rows1 = ctx->sc_rd;
      g.K = 2 * ctx->dnp;
      g.B = ctx->Wa1;
      g.N = ctx->dnp;
      g.bias = ctx->ba1;
      g.relu = 1;
      g.C = ctx->sc_z;
      g.ldc = ctx->dnp;
      g.m_dev = ctx->sc_m;
      g.m_max = (neg ? 2 : 1) * S * batch;
      if (ctx->cfg.precision == TG_PREC_BF16) launch_gemm_tc(g, ctx->tcWa1g, TG_PREC_TF32, st);
      else if (ctx->cfg.precision != TG_PREC_FP32) launch_gemm_tc(g, ctx->tcWa1, ctx->cfg.precision, st);
      else launch_gemm_simt(g, st);
      launch_score_head(ctx->sc_z, ctx->dnp, ctx->sc_oidx, g.m_max, ctx->Wa2, ctx->ba2, ctx->d_n, scores, st);
    }
    TRY(launched(ctx, 3));
    TRY(finish(ctx, S, log, b0, st));
    CK(cudaEventRecord(ctx->ev_back[set], st));

  }
  CK(cudaEventRecord(ctx->ev_fend, ctx->fst));  // join the front stream into st
  CK(cudaStreamWaitEvent(st_in, ctx->ev_fend, 0));
  if (prio) {
    CK(cudaEventRecord(ctx->ev_lend, st));
    CK(cudaStreamWaitEvent(st_in, ctx->ev_lend, 0));
  }
  select_set(ctx, 0);
  return TG_OK;
}

struct Staged {
  const int32_t *src = nullptr, *dst = nullptr, *neg = nullptr;
  const uint32_t* ts = nullptr;
  float* out = nullptr;
  bool host_out = false;
};

}  // namespace

// =========================================================================
extern "C" {

const char* tg_strerror(tg_status s) {
  switch (s) {
    case TG_OK: return "ok";
    case TG_EINVAL: return "invalid argument";
    case TG_ENOMEM: return "out of memory";
    case TG_ECUDA: return "CUDA error";
    case TG_ESTATE: return "call out of order";
    case TG_EORDER: return "timestamps not non-decreasing";
    case TG_EDEVICE: return "device-side error flag set (id out of range or table full)";
  }
  return "unknown";
}

const char* tg_version(void) { return "libtg 0.2 sm_100a (fp32 SIMT, tf32x3/bf16 tcgen05; superbatch schedule)"; }

int64_t tg_kernel_launches(tg_ctx* ctx) { return ctx ? ctx->launches : 0; }
int32_t tg_superbatch(tg_ctx* ctx) { return (ctx && ctx->loaded) ? ctx->S : 0; }

tg_status tg_graph_load(int device, const tg_graph_desc* gd, tg_ctx** out) {
  if (!gd || !out) return TG_EINVAL;
  *out = nullptr;
  if (gd->n_nodes < 0 || gd->n_edges < 0 || gd->d_n < 1 || gd->d_e < 1) return TG_EINVAL;
  if (gd->n_edges > 0 && (!gd->src || !gd->dst || !gd->ts)) return TG_EINVAL;
  if (!gd->node_feat || !gd->edge_feat) return TG_EINVAL;
  if (2 * gd->n_edges >= (int64_t)INT32_MAX || gd->n_nodes >= (int64_t)INT32_MAX) return TG_EINVAL;
  const int64_t V = gd->n_nodes, E = gd->n_edges;
  for (int64_t i = 0; i < E; ++i) {
    if (gd->src[i] < 1 || gd->src[i] > V || gd->dst[i] < 1 || gd->dst[i] > V) return TG_EINVAL;
    if (i && gd->ts[i] < gd->ts[i - 1]) return TG_EORDER;
  }
  if (cudaSetDevice(device) != cudaSuccess) return TG_ECUDA;
  tg_ctx* ctx = new (std::nothrow) tg_ctx();
  if (!ctx) return TG_ENOMEM;
  ctx->device = device;
  // T-CSR on the host: counting sort by node; edges are already in (t, edge
  // id) order, so appending keeps each adjacency sorted (R6).
  std::vector<int32_t> rowptr(V + 2, 0);
  for (int64_t i = 0; i < E; ++i) {
    rowptr[gd->src[i] + 1]++;
    rowptr[gd->dst[i] + 1]++;
  }
  for (int64_t v = 0; v <= V; ++v) rowptr[v + 1] += rowptr[v];
  std::vector<int32_t> fill(rowptr.begin(), rowptr.end() - 1);
  std::vector<int32_t> nbr(2 * E), eid(2 * E);
  std::vector<uint32_t> tt(2 * E);
  for (int64_t i = 0; i < E; ++i) {
    const int32_t s = gd->src[i], d = gd->dst[i];
    int32_t p = fill[s]++;
    nbr[p] = d;
    eid[p] = (int32_t)(i + 1);
    tt[p] = gd->ts[i];
    p = fill[d]++;
    nbr[p] = s;
    eid[p] = (int32_t)(i + 1);
    tt[p] = gd->ts[i];
  }
  tg_status s;
#define TRYF(x)       \
  do {                \
    s = (x);          \
    if (s != TG_OK) { \
      tg_free(ctx);   \
      return s;       \
    }                 \
  } while (0)
  TRYF(dalloc(ctx, &ctx->rowptr, V + 2));
  TRYF(dalloc(ctx, &ctx->adj_nbr, 2 * E));
  TRYF(dalloc(ctx, &ctx->adj_eid, 2 * E));
  TRYF(dalloc(ctx, &ctx->adj_t, 2 * E));
  cudaMemcpy(ctx->rowptr, rowptr.data(), (V + 2) * 4, cudaMemcpyHostToDevice);
  if (E) {
    cudaMemcpy(ctx->adj_nbr, nbr.data(), 2 * E * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(ctx->adj_eid, eid.data(), 2 * E * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(ctx->adj_t, tt.data(), 2 * E * 4, cudaMemcpyHostToDevice);
  }
  const int ldn = round4(gd->d_n), lde = round4(gd->d_e);
  TRYF(dalloc(ctx, &ctx->X, (size_t)(V + 1) * ldn));
  TRYF(dalloc(ctx, &ctx->Ef, (size_t)(E + 1) * lde));
  cudaMemset(ctx->X, 0, (size_t)(V + 1) * ldn * 4);
  cudaMemset(ctx->Ef, 0, (size_t)(E + 1) * lde * 4);
  if (V > 0)
    cudaMemcpy2D(ctx->X + ldn, ldn * 4, gd->node_feat + gd->d_n, gd->d_n * 4, gd->d_n * 4, V, cudaMemcpyHostToDevice);
  if (E > 0)
    cudaMemcpy2D(ctx->Ef + lde, lde * 4, gd->edge_feat + gd->d_e, gd->d_e * 4, gd->d_e * 4, E,
                 cudaMemcpyHostToDevice);
  if (cudaDeviceSynchronize() != cudaSuccess) {
    tg_free(ctx);
    return TG_ECUDA;
  }
  GraphDev& g = ctx->g;
  g.V = V;
  g.E = E;
  g.rowptr = ctx->rowptr;
  g.adj_nbr = ctx->adj_nbr;
  g.adj_eid = ctx->adj_eid;
  g.adj_t = ctx->adj_t;
  g.X = ctx->X;
  g.Ef = ctx->Ef;
  g.d_n = gd->d_n;
  g.d_e = gd->d_e;
  g.ldn = ldn;
  for (int64_t i = 0; i < E; ++i) ctx->max_ts = std::max(ctx->max_ts, gd->ts[i]);
  g.lde = lde;
  TRYF(dalloc(ctx, &ctx->err, 2));  // [0] sticky error bits, [1] debug index-check mismatches
  cudaMemset(ctx->err, 0, 2 * sizeof(int));
  *out = ctx;
  return TG_OK;
#undef TRYF
}

tg_status tg_model_load(tg_ctx* ctx, const tg_model_cfg* cfg, const float* params, int64_t n_params) {
  if (!ctx || !cfg || !params) return TG_EINVAL;
  if (ctx->broken) return TG_ECUDA;
  if (ctx->loaded) return TG_ESTATE;  // one model per context
  const int L = cfg->n_layers, H = cfg->n_heads, k = cfg->n_neighbors, d_t = cfg->d_t;
  const int d_n = ctx->g.d_n, d_e = ctx->g.d_e;
  const int D = d_n + d_e + d_t;
  if (L < 1 || L > TG_MAX_LAYERS || H < 1 || H > 8 || k < 1 || k > kMaxK || d_t < 1 || D % H) return TG_EINVAL;
  if (cfg->max_batch_targets < 1 || cfg->cache_limit < 0 || cfg->time_window < 0) return TG_EINVAL;
  if (cfg->precision < TG_PREC_FP32 || cfg->precision > TG_PREC_LAST) return TG_EINVAL;
  if (cfg->superbatch < 0 || cfg->superbatch > kMaxS) return TG_EINVAL;
  if (round4(d_n) + round4(d_e) + round4(d_t) > 1024) return TG_EINVAL;  // LayerNorm row in registers
  const int64_t per_layer = 4LL * D * D + 3LL * D + (int64_t)d_n * (D + d_n) + d_n + (int64_t)d_n * d_n + d_n;
  const int64_t expect = L * per_layer + 2LL * d_t + 2LL * d_n * d_n + d_n + d_n + 1;
  if (n_params != expect) return TG_EINVAL;
  static const int s_default = [] {
    const char* e = getenv("TG_SB_DEFAULT");  // experiments: default superbatch
    const int v = e ? atoi(e) : 0;
    return v > 0 && v <= kMaxS ? v : 64;
  }();
  // default S: the cost model below picks it in [smax / 8, smax] (smax: the workspace budget);
  // TG_SB_DEFAULT or cfg->superbatch fix it
  const bool s_auto = cfg->superbatch == 0 && !getenv("TG_SB_DEFAULT") && cfg->precision != TG_PREC_FP32;
  int S = cfg->superbatch ? cfg->superbatch : (s_auto ? kMaxS : s_default);
  // per-batch capacities: I_L = targets; I_{l-1} = C_l (k+1) <= I_l (k+1)
  int cap[TG_MAX_LAYERS + 1];
  int64_t cc = cfg->max_batch_targets;
  cap[L] = (int)cc;
  for (int l = L - 1; l >= 1; --l) {
    cc = cc * (k + 1);
    if (cc > ((int64_t)1 << 26)) return TG_EINVAL;
    cap[l] = (int)cc;
  }
  for (int l = 1; l <= L; ++l) {
    if (cap[l] > 16 * 10000) return TG_EINVAL;                   // dedup cluster bound
    if (cap[l] > kSeqCLMax * 1024 * kProbeIPT) return TG_EINVAL; // ordered cache pass bound
  }
  // Both cache passes keep their superbatch hash in global memory (r1: DSMEM, which capped
  // S at 28 for batch 200 / k = 20 and at 1 for batch 2,000): S is bounded only by the
  // grid-wide pass's block count and a ~40 GB budget for the S-proportional workspaces.
  {
    const int64_t HDp_ = (int64_t)H * (round4(d_n) + round4(d_e) + round4(d_t)), Dp_ = HDp_ / H;
    auto ws = [&](int64_t s) {  // device bytes that grow with S (both level sets)
      int64_t b = 0, mx = 0;
      for (int l = 1; l <= L; ++l) {
        b += 2 * s * cap[l] * (72 + 24 * (int64_t)k);
        mx = std::max<int64_t>(mx, s * cap[l]);
        if (l < L) b += s * cap[l] * 8 * 20 + s * cap[l] * 4;  // superbatch lookup table (4x pow2) + slots
      }
      return b + mx * 4 * (2 * HDp_ + 2 * Dp_ + round4(d_n)) + mx * 2 * (HDp_ + Dp_ + 2 * round4(d_n));
    };
    while (S > 1 && (ws(S) > (40ll << 30) || (int64_t)cap[1] * S > (int64_t)kSbhMaxBlocks * kSbhChunk)) --S;
  }
  const int smax = S;
  if ((int64_t)cap[1] * S > ((int64_t)1 << 26)) return TG_EINVAL;
  if (cudaSetDevice(ctx->device) != cudaSuccess) return TG_ECUDA;
  ctx->cfg = *cfg;
  ctx->S = S;
  ctx->L = L;
  ctx->H = H;
  ctx->k = k;
  ctx->d_n = d_n;
  ctx->d_e = d_e;
  ctx->d_t = d_t;
  ctx->dnp = round4(d_n);
  ctx->dep = round4(d_e);
  ctx->dtp = round4(d_t);
  ctx->Dp = ctx->dnp + ctx->dep + ctx->dtp;
  ctx->W = cfg->time_window;
  const int dnp = ctx->dnp, Dp = ctx->Dp, dk = D / H;
  const int HDp = H * Dp;
  // ---- time encoder: Phi table [max(W,1) x dtp] on device; Phi(0) = row 0
  const float* om = params + L * per_layer;
  const float* ph = om + d_t;
  // The device cosine reduces its argument in fp64 (two-term Cody-Waite), accurate for
  // |dt * omega + phi| < 1e15; dt < 2^32 (R4), so bound |omega| and |phi| accordingly.
  for (int c = 0; c < d_t; ++c)
    if (!(std::fabs((double)om[c]) * 4294967296.0 + std::fabs((double)ph[c]) < 1e15)) return TG_EINVAL;
  TRY(dalloc(ctx, &ctx->omega, d_t));
  TRY(dalloc(ctx, &ctx->phi, d_t));
  {
    static const int wt_env = [] {  // TG_PHI_TABLE=0: table of the paper's window only (A/B)
      const char* e = getenv("TG_PHI_TABLE");
      return e ? atoi(e) : 1;
    }();
    const long long want = (long long)ctx->max_ts + 1;
    ctx->Wt = (ctx->W > 0 && wt_env) ? (int)std::min<long long>(std::max<long long>(want, ctx->W), 1ll << 22) : ctx->W;
  }
  const int Wrows = std::max(ctx->Wt, 1);
  TRY(dalloc(ctx, &ctx->table, (size_t)Wrows * ctx->dtp));
  CK(cudaMemcpy(ctx->omega, om, d_t * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(ctx->phi, ph, d_t * 4, cudaMemcpyHostToDevice));
  launch_time_table(ctx->omega, ctx->phi, d_t, ctx->dtp, Wrows, ctx->table, 0);
  CK(cudaGetLastError());
  std::vector<float> phi0(ctx->dtp);
  CK(cudaMemcpy(phi0.data(), ctx->table, ctx->dtp * 4, cudaMemcpyDeviceToHost));
  // ---- per-layer weights, folded in float64 on the host (load time only)
  const double isq = 1.0 / std::sqrt((double)dk);
  for (int l = 0; l < L; ++l) {
    const float* base = params + l * per_layer;
    const float* Wq = base;
    const float* Wk = Wq + (size_t)D * D;
    const float* Wv = Wk + (size_t)D * D;
    const float* Wfc = Wv + (size_t)D * D;
    const float* bfc = Wfc + (size_t)D * D;
    const float* lng = bfc + D;
    const float* lnb = lng + D;
    const float* Wm1 = lnb + D;
    const float* bm1 = Wm1 + (size_t)d_n * (D + d_n);
    const float* Wm2 = bm1 + d_n;
    const float* bm2 = Wm2 + (size_t)d_n * d_n;
    std::vector<double> P((size_t)HDp * dnp, 0.0), bu(HDp, 0.0), F((size_t)Dp * HDp, 0.0);
    std::vector<double> qc(D, 0.0);  // W_q[:, Phi block] Phi(0)
    for (int r = 0; r < D; ++r)
      for (int c = d_n + d_e; c < D; ++c) qc[r] += (double)Wq[(size_t)r * D + c] * phi0[c - d_n - d_e];
    for (int h = 0; h < H; ++h) {
      for (int r = h * dk; r < (h + 1) * dk; ++r) {
        const float* wq = Wq + (size_t)r * D;
        const float* wk = Wk + (size_t)r * D;
        for (int a = 0; a < D; ++a) {
          const double wka = wk[a];
          double* prow = &P[((size_t)h * Dp + pc(ctx, a)) * dnp];
          for (int b = 0; b < d_n; ++b) prow[b] += wka * wq[b];
          bu[(size_t)h * Dp + pc(ctx, a)] += wka * qc[r];
        }
      }
    }
    for (auto& v : P) v *= isq;
    for (auto& v : bu) v *= isq;
    for (int o = 0; o < D; ++o) {
      double* frow = &F[(size_t)pc(ctx, o) * HDp];
      for (int h = 0; h < H; ++h)
        for (int r = h * dk; r < (h + 1) * dk; ++r) {
          const double w = Wfc[(size_t)o * D + r];
          const float* wv = Wv + (size_t)r * D;
          for (int a = 0; a < D; ++a) frow[(size_t)h * Dp + pc(ctx, a)] += w * wv[a];
        }
    }
    std::vector<float> Pf(P.begin(), P.end()), buf(bu.begin(), bu.end()), Ff(F.begin(), F.end());
    std::vector<float> bfcp(Dp, 0.f), lngp(Dp, 0.f), lnbp(Dp, 0.f);
    for (int a = 0; a < D; ++a) {
      bfcp[pc(ctx, a)] = bfc[a];
      lngp[pc(ctx, a)] = lng[a];
      lnbp[pc(ctx, a)] = lnb[a];
    }
    const int K3 = Dp + dnp;
    std::vector<float> W1p((size_t)dnp * K3, 0.f), b1p(dnp, 0.f), W2p((size_t)dnp * dnp, 0.f), b2p(dnp, 0.f);
    for (int j = 0; j < d_n; ++j) {
      for (int a = 0; a < D; ++a) W1p[(size_t)j * K3 + pc(ctx, a)] = Wm1[(size_t)j * (D + d_n) + a];
      for (int b = 0; b < d_n; ++b) W1p[(size_t)j * K3 + Dp + b] = Wm1[(size_t)j * (D + d_n) + D + b];
      b1p[j] = bm1[j];
      for (int b = 0; b < d_n; ++b) W2p[(size_t)j * dnp + b] = Wm2[(size_t)j * d_n + b];
      b2p[j] = bm2[j];
    }
    LayerW& w = ctx->lw[l];
    auto up = [&](float** dptr, const std::vector<float>& v) -> tg_status {
      TRY(dalloc(ctx, dptr, v.size()));
      CK(cudaMemcpy(*dptr, v.data(), v.size() * 4, cudaMemcpyHostToDevice));
      return TG_OK;
    };
    TRY(up(&w.P, Pf));
    TRY(up(&w.bu, buf));
    TRY(up(&w.F, Ff));
    TRY(up(&w.bfc, bfcp));
    {
      std::vector<float> bq(bfcp);
      for (int c = 0; c < d_t; ++c) bq[dnp + ctx->dep + c] += phi0[c];
      TRY(up(&w.bfcq, bq));
    }
    TRY(up(&w.lng, lngp));
    TRY(up(&w.lnb, lnbp));
    TRY(up(&w.W1, W1p));
    TRY(up(&w.b1, b1p));
    TRY(up(&w.W2, W2p));
    TRY(up(&w.b2, b2p));
    if (cfg->precision != TG_PREC_FP32) {
      TRY(tc_prepare_weights(w.P, HDp, dnp, cfg->precision, &w.tcP, ctx->owned));
      TRY(tc_prepare_weights(w.F, Dp, HDp, cfg->precision, &w.tcF, ctx->owned));
      if (cfg->precision == TG_PREC_BF16) {  // h block at column dpa (see tg_ctx::dpa)
        const int dpa = (Dp + 7) & ~7, K3b = dpa + dnp;
        std::vector<float> W1b((size_t)dnp * K3b, 0.f);
        for (int j = 0; j < dnp; ++j) {
          for (int a = 0; a < Dp; ++a) W1b[(size_t)j * K3b + a] = W1p[(size_t)j * K3 + a];
          for (int b = 0; b < dnp; ++b) W1b[(size_t)j * K3b + dpa + b] = W1p[(size_t)j * K3 + Dp + b];
        }
        float* dW1b = nullptr;
        TRY(up(&dW1b, W1b));
        TRY(tc_prepare_weights(dW1b, dnp, K3b, cfg->precision, &w.tcW1, ctx->owned));
      } else {
        TRY(tc_prepare_weights(w.W1, dnp, K3, cfg->precision, &w.tcW1, ctx->owned));
      }
      TRY(tc_prepare_weights(w.W2, dnp, dnp, cfg->precision, &w.tcW2, ctx->owned));
    }
    if (cfg->precision == TG_PREC_BF16) {
      // y + q_h = [F | I] [c ; h]: k-blocks [0, kb0) read c (attention output), the last
      // ceil(dnp / 64) read h^(l-1) (bf16, the h block of the merge-FFN input row)
      const int kb0 = (HDp + 63) / 64;
      const int Ka = kb0 * 64 + dnp;
      std::vector<float> Fa((size_t)Dp * Ka, 0.f);
      for (int n = 0; n < Dp; ++n) {
        for (int j = 0; j < HDp; ++j) Fa[(size_t)n * Ka + j] = Ff[(size_t)n * HDp + j];
        if (n < dnp) Fa[(size_t)n * Ka + kb0 * 64 + n] = 1.f;
      }
      float* dFa = nullptr;
      TRY(up(&dFa, Fa));
      TRY(tc_prepare_weights(dFa, Dp, Ka, cfg->precision, &w.tcFa, ctx->owned));
      w.fa_kb0 = kb0;
    }
  }
  // ---- superbatch size from a wave-quantised cost model (default S only): per superbatch, every
  // projection GEMM of every layer runs ceil(tiles / 148) waves of tiles that each cost nkb k-blocks
  // of ~0.08 us per MMA instruction (6 per k-block in the fp32-level modes: 0.47 us, clock64 traces;
  // N <= 176 costs the same as wider tiles), the attention + LayerNorm cost ~8 ns per target and
  // layer at k = 20, D = 516 (scaled by k D), and ~140 us per superbatch is fixed (front-stream
  // overlap, launch ramps); rows per layer ~ S x max_batch_targets. S minimises cost / S over
  // [smax / 8, smax] -- Reddit: S = 94 (G2 882 tiles = 5.96 waves, G3/G4 294 tiles = 1.99 waves),
  // 51 ms per pass against 54 ms at S = 63 and 64
  if (cfg->superbatch == 0 && !getenv("TG_SB_DEFAULT") && cfg->precision != TG_PREC_FP32 && ctx->lw[L - 1].tcF.ntn > 0) {
    const int64_t T = cfg->max_batch_targets;
    const bool x3 = cfg->precision == TG_PREC_TF32X3 || cfg->precision == TG_PREC_F16X3;
    const double t_kb = 0.08 * (x3 ? 6 : 4);  // us per k-block
    static const bool u1_on = [] {
      const char* e = getenv("TG_U1");
      return !(e && e[0] == '0');
    }();
    const bool u1_will = u1_on && ((long long)ctx->g.V + 1) * HDp * 4 <= (8ll << 30);
    const double c_t = 8e-3 * ((double)k * Dp) / (20.0 * 516.0);  // us per target and layer
    auto waves = [](int64_t tiles) { return (double)((tiles + 147) / 148); };
    int best = S;
    double best_c = 1e300;
    for (int s2 = smax; s2 >= std::max(1, smax / 8); --s2) {
      const int64_t mt = ((int64_t)s2 * T + 127) / 128;
      double c = 140.0 + (double)L * s2 * T * c_t;
      for (int l = 0; l < L; ++l) {
        const LayerW& w = ctx->lw[l];
        if (!(l == 0 && u1_will)) c += waves(mt * w.tcP.ntn) * w.tcP.nkb * t_kb;
        c += waves(mt * w.tcF.ntn) * w.tcF.nkb * t_kb;
        c += waves(mt * w.tcW1.ntn) * w.tcW1.nkb * t_kb;
        c += waves(mt * w.tcW2.ntn) * w.tcW2.nkb * t_kb;
      }
      c /= s2;
      if (c < best_c * 0.9999) {
        best_c = c;
        best = s2;
      }
    }
    S = best;
    ctx->S = S;
  }
  // ---- affinity score MLP (R10), padded
  {
    const float* Wa1 = ph + d_t;
    const float* ba1 = Wa1 + (size_t)d_n * 2 * d_n;
    const float* Wa2 = ba1 + d_n;
    const float* ba2 = Wa2 + d_n;
    std::vector<float> Wv((size_t)dnp * 2 * dnp, 0.f), b(dnp, 0.f), w2(dnp, 0.f);
    for (int j = 0; j < d_n; ++j) {
      for (int a = 0; a < d_n; ++a) {
        Wv[(size_t)j * 2 * dnp + a] = Wa1[(size_t)j * 2 * d_n + a];
        Wv[(size_t)j * 2 * dnp + dnp + a] = Wa1[(size_t)j * 2 * d_n + d_n + a];
      }
      b[j] = ba1[j];
      w2[j] = Wa2[j];
    }
    TRY(dalloc(ctx, &ctx->Wa1, Wv.size()));
    TRY(dalloc(ctx, &ctx->ba1, b.size()));
    TRY(dalloc(ctx, &ctx->Wa2, w2.size()));
    CK(cudaMemcpy(ctx->Wa1, Wv.data(), Wv.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(ctx->ba1, b.data(), b.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(ctx->Wa2, w2.data(), w2.size() * 4, cudaMemcpyHostToDevice));
    ctx->ba2 = ba2[0];
    if (cfg->precision != TG_PREC_FP32)
      TRY(tc_prepare_weights(ctx->Wa1, dnp, 2 * dnp, cfg->precision, &ctx->tcWa1, ctx->owned));
      if (cfg->precision == TG_PREC_BF16)
        TRY(tc_prepare_weights(ctx->Wa1, dnp, 2 * dnp, TG_PREC_TF32, &ctx->tcWa1g, ctx->owned));
    // score rows of a superbatch: S x batch positive (+ S x batch negative) pairs, batch <= targets / 2
    const size_t ne = (size_t)S * cfg->max_batch_targets;
    TRY(dalloc(ctx, &ctx->sc_rs, ne));
    TRY(dalloc(ctx, &ctx->sc_rd, ne));
    TRY(dalloc(ctx, &ctx->sc_oidx, ne));
    TRY(dalloc(ctx, &ctx->sc_z, ne * dnp));
    TRY(dalloc(ctx, &ctx->sc_m, 1));
  }
  // ---- recursion levels: batch-segmented lists + superbatch compute lists
  int maxC = 0;
  for (int set = 0; set < 2; ++set)
  for (int l = 1; l <= L; ++l) {
    LevelDev& v = ctx->lvs[set][l];
    const size_t n = (size_t)S * cap[l];
    ctx->cap[l] = cap[l];
    v.cap = cap[l];
    v.c_cap = (int)n;
    maxC = std::max(maxC, (int)n);
    TRY(dalloc(ctx, &v.in_node, n));
    TRY(dalloc(ctx, &v.in_ts, n));
    TRY(dalloc(ctx, &v.n_in, kMaxS));
    TRY(dalloc(ctx, &v.u_node, n));
    TRY(dalloc(ctx, &v.u_ts, n));
    TRY(dalloc(ctx, &v.n_u, kMaxS));
    TRY(dalloc(ctx, &v.inv, n));
    TRY(dalloc(ctx, &v.slot, n));
    TRY(dalloc(ctx, &v.p0, n));
    TRY(dalloc(ctx, &v.sup, n));
    TRY(dalloc(ctx, &v.c_b, n));
    TRY(dalloc(ctx, &v.c_u, n));
    TRY(dalloc(ctx, &v.c_node, n));
    TRY(dalloc(ctx, &v.c_ts, n));
    TRY(dalloc(ctx, &v.c_base, kMaxS));
    TRY(dalloc(ctx, &v.n_c, kMaxS));
    TRY(dalloc(ctx, &v.n_c_total, 1));
    TRY(dalloc(ctx, &v.nb_node, n * k));
    TRY(dalloc(ctx, &v.nb_ts, n * k));
    TRY(dalloc(ctx, &v.nb_eid, n * k));
    TRY(dalloc(ctx, &v.hs_row, n));
    if ((cfg->precision == TG_PREC_TF32X3 || cfg->precision == TG_PREC_F16X3) && l == 1)
      TRY(dalloc(ctx, &v.hs_dense, n * round4(d_n)));
    TRY(dalloc(ctx, &v.nb_row, n * k));
    TRY(dalloc(ctx, &v.nb_hidx, n * k));
    TRY(dalloc(ctx, &v.dst_row, n));
    CK(cudaMemset(v.n_c_total, 0, sizeof(int)));
    CK(cudaMemset(v.n_in, 0, kMaxS * sizeof(int)));
  }
  ctx->maxC = maxC;
  // ---- caches for layers 1..L-1: index (load <= 1/4 of live items) + FIFO ring.
  // Ring capacity limit + (S+2) cap: a superbatch never overwrites a slot that
  // one of its own batches still reads.
  TRY(dalloc(ctx, &ctx->cache_state, 8 * TG_MAX_LAYERS));
  ctx->limit0 = cfg->cache_limit;
  for (int l = 1; l < L; ++l) {
    CacheDev& cd = ctx->cache[l];
    const long long rcap = cfg->cache_limit + (long long)(S + 2) * cap[l] + 16;
    unsigned long long icap = 1024;
    while (icap < 4ull * (unsigned long long)(cfg->cache_limit + (long long)S * cap[l])) icap <<= 1;
    TRY(dalloc(ctx, &cd.ikey, icap));
    TRY(dalloc(ctx, &cd.ipos, icap));
    if (cfg->opts & TG_OPT_HOST_CACHE) {  // NEXT-2: payload ring in pinned, mapped host memory
      void* hp = nullptr;
      if (cudaHostAlloc(&hp, (size_t)rcap * dnp * sizeof(float), cudaHostAllocMapped) != cudaSuccess) {
        cudaGetLastError();
        return TG_ENOMEM;
      }
      ctx->owned_host.push_back(hp);
      void* dp = nullptr;
      CK(cudaHostGetDevicePointer(&dp, hp, 0));
      cd.ring = reinterpret_cast<float*>(dp);
    } else {
      TRY(dalloc(ctx, &cd.ring, (size_t)rcap * dnp));
    }
    TRY(dalloc(ctx, &cd.rkey, (size_t)rcap));
    {  // grid-wide eviction-free lookup pass: superbatch-scoped hash, >= 2x its entries
      unsigned long long T = 1024;
      while (T < 4ull * (unsigned long long)S * cap[l]) T <<= 1;  // grid-wide + ordered pass keys
      TRY(dalloc(ctx, &cd.sb_key, T));
      TRY(dalloc(ctx, &cd.sb_val, T));
      TRY(dalloc(ctx, &cd.sb_slot, T));
      TRY(dalloc(ctx, &cd.sb_h, (size_t)S * cap[l]));
      TRY(dalloc(ctx, &cd.sb_blk, kSbhMaxBlocks));
      cd.sb_mask = T - 1;
    }
    cd.imask = icap - 1;
    cd.rcap = rcap;
    cd.state = ctx->cache_state + 8 * l;
  }
  // ---- compute workspace
  TRY(dalloc(ctx, &ctx->u, (size_t)maxC * HDp));
  TRY(dalloc(ctx, &ctx->c, (size_t)maxC * HDp));
  TRY(dalloc(ctx, &ctx->y, (size_t)maxC * Dp));
  TRY(dalloc(ctx, &ctx->r, (size_t)maxC * (Dp + dnp)));  // [LN(y) | h^(l-1)] rows (G3's A)
  TRY(dalloc(ctx, &ctx->z, (size_t)maxC * dnp));
  TRY(dalloc(ctx, &ctx->HL, (size_t)S * cap[L] * dnp));
  if (cfg->precision == TG_PREC_BF16) {
    ctx->ld_ch = (HDp + 7) & ~7;
    ctx->dpa = (Dp + 7) & ~7;
    ctx->ld_rh = (ctx->dpa + dnp + 7) & ~7;
    ctx->ld_z = (dnp + 7) & ~7;
    TRY(dalloc(ctx, &ctx->c_h, (size_t)maxC * ctx->ld_ch));
    TRY(dalloc(ctx, &ctx->rh_h, (size_t)maxC * ctx->ld_rh));
    TRY(dalloc(ctx, &ctx->z_h, (size_t)maxC * ctx->ld_z));
    TRY(tc_make_tensor_a(ctx->c_h, 2, ctx->ld_ch, maxC, &ctx->ta_c));
    TRY(tc_make_tensor_a(ctx->rh_h, 2, ctx->ld_rh, maxC, &ctx->ta_rh));
    TRY(tc_make_tensor_a(ctx->z_h, 2, ctx->ld_z, maxC, &ctx->ta_z));
  }
  if (cfg->precision == TG_PREC_TF32X3 || cfg->precision == TG_PREC_F16X3) {
    TRY(tc_make_tensor_a(ctx->c, 4, HDp, maxC, &ctx->ta_c32));
    TRY(tc_make_tensor_a(ctx->z, 4, dnp, maxC, &ctx->ta_z32));
    TRY(tc_make_tensor_a(ctx->r, 4, Dp + dnp, maxC, &ctx->ta_r32));
    for (int set = 0; set < 2; ++set)
      TRY(tc_make_tensor_a(ctx->lvs[set][1].hs_dense, 4, dnp, ctx->lvs[set][1].c_cap, &ctx->ta_hs[set][1]));
  }
  // Phi rows of dt >= W computed ahead on the front stream into a per-set buffer that follows a
  // copy of the table, so the attention gathers every Phi row from one tensor (dense row index
  // W + q*k + m per level; skipped when the buffers would exceed 16 GB: in-kernel Phi instead)
  {
    long long rows = Wrows;
    for (int l = 1; l <= L; ++l) {
      ctx->phi_row0[l] = rows;
      rows += (long long)ctx->lvs[0][l].c_cap * k;
    }
    const size_t bytes = (size_t)rows * ctx->dtp * sizeof(float);
    static const bool phi_pre_env = [] {  // TG_PHI_PRE=0: Phi of dt >= W inside the attention (A/B)
      const char* e = getenv("TG_PHI_PRE");
      return !(e && e[0] == '0');
    }();
    ctx->phi_pre = phi_pre_env && 2 * bytes <= (16ull << 30) && rows < (1ll << 31);
    if (ctx->phi_pre)
      for (int set = 0; set < 2; ++set) {
        TRY(dalloc(ctx, &ctx->phi_buf[set], (size_t)rows * ctx->dtp));
        CK(cudaMemcpy(ctx->phi_buf[set], ctx->table, (size_t)Wrows * ctx->dtp * sizeof(float),
                      cudaMemcpyDeviceToDevice));
      }
    // TMA row-gather maps for the attention (feature rows <= 256 fp32; else the CTA kernel gathers)
    for (int set = 0; set < 2; ++set)
      for (int l = 1; l <= L; ++l) {
        AttnMaps& m = ctx->am[set][l];
        m.valid = 0;
        const float* hb = l == 1 ? ctx->X : ctx->cache[l - 1].ring;
        const long long hrows = l == 1 ? ctx->g.V + 1 : ctx->cache[l - 1].rcap;
        const float* tb = ctx->phi_pre ? ctx->phi_buf[set] : ctx->table;
        const long long trows = ctx->phi_pre ? rows : Wrows;
        // host-resident cache rings are read with per-thread loads (CTA attention kernel), not TMA
        const bool host_rows = l > 1 && (cfg->opts & TG_OPT_HOST_CACHE);
        if (!host_rows && attn_make_rows_map(hb, dnp, ctx->g.ldn, hrows, &m.h) == TG_OK &&
            attn_make_rows_map(ctx->Ef, ctx->dep, ctx->g.lde, ctx->g.E + 1, &m.e) == TG_OK &&
            attn_make_rows_map(tb, ctx->dtp, ctx->dtp, trows, &m.t) == TG_OK)
          m.valid = 1;
      }
  }
  // ---- U1: layer-1 query side of every node, u = P x_i + b_u (R27), by the layer-1 G1 kernel
  {
    static const bool u1_env = [] {  // TG_U1=0: G1 per layer-1 target instead (A/B)
      const char* e = getenv("TG_U1");
      return !(e && e[0] == '0');
    }();
    const long long nv = (long long)ctx->g.V + 1;
    if (u1_env && nv * HDp * 4 <= (8ll << 30) && nv < (1ll << 31)) {
      TRY(dalloc(ctx, &ctx->u1, (size_t)nv * HDp));
      TRY(dalloc(ctx, &ctx->u1_m, 1));
      launch_set_int(ctx->u1_m, (int)nv, 0);
      const LayerW& w = ctx->lw[0];
      GemmArgs g{};
      g.err = ctx->err;
      g.a_base0 = ctx->X;
      g.lda0 = ctx->g.ldn;
      g.K0 = g.K = dnp;
      g.B = w.P;
      g.N = HDp;
      g.bias = w.bu;
      g.C = ctx->u1;
      g.ldc = HDp;
      g.m_dev = ctx->u1_m;
      g.m_max = (int)nv;
      if (cfg->precision == TG_PREC_FP32) {
        launch_gemm_simt(g, 0);
      } else {
        TcTensorA ta;  // fp32-level modes: dense rows staged by TMA, as for the per-target G1
        if (cfg->precision == TG_PREC_TF32X3 || cfg->precision == TG_PREC_F16X3)
          TRY(tc_make_tensor_a(ctx->X, 4, ctx->g.ldn, (int)nv, &ta));
        launch_gemm_tc(g, w.tcP, cfg->precision, 0, ta.valid ? &ta : nullptr);
      }
      CK(cudaGetLastError());
    }
  }
  TRY(dalloc(ctx, &ctx->cnt_total, TG_NCOUNTERS));
  for (int set = 0; set < 2; ++set) {
    TRY(dalloc(ctx, &ctx->cnt_sbs[set], (size_t)kMaxS * TG_NCOUNTERS));
    CK(cudaMemset(ctx->cnt_sbs[set], 0, (size_t)kMaxS * TG_NCOUNTERS * sizeof(long long)));
  }
  select_set(ctx, 0);
  if (!ctx->fst) {
    int plo = 0, phi = 0;
    CK(cudaDeviceGetStreamPriorityRange(&plo, &phi));
    CK(cudaStreamCreateWithPriority(&ctx->fst, cudaStreamNonBlocking, plo));
    CK(cudaStreamCreateWithPriority(&ctx->lst, cudaStreamNonBlocking, phi));
    CK(cudaEventCreateWithFlags(&ctx->ev_lend, cudaEventDisableTiming));
    for (int i = 0; i < 2; ++i) {
      CK(cudaEventCreateWithFlags(&ctx->ev_front[i], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&ctx->ev_back[i], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&ctx->ev_in, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ctx->ev_fend, cudaEventDisableTiming));
  }
  if (!ctx->occ_h) {
    CK(cudaHostAlloc(&ctx->occ_h, (TG_MAX_LAYERS + 1) * sizeof(unsigned long long), cudaHostAllocMapped));
    memset(ctx->occ_h, 0, (TG_MAX_LAYERS + 1) * sizeof(unsigned long long));
  }
  CK(cudaDeviceSynchronize());
  ctx->loaded = true;
  return tg_cache_reset(ctx, -1);
}

tg_status tg_cache_reset(tg_ctx* ctx, int64_t new_limit) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  if (new_limit > ctx->limit0) return TG_EINVAL;
  if (new_limit >= 0) ctx->cfg.cache_limit = new_limit;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  for (int l = 1; l < ctx->L; ++l) {
    CacheDev& cd = ctx->cache[l];
    CK(cudaMemset(cd.ikey, 0xFF, (cd.imask + 1) * sizeof(unsigned long long)));
    long long st[8] = {0, 0, ctx->cfg.cache_limit, 0, 0, 0, 0, 0};
    CK(cudaMemcpy(cd.state, st, sizeof(st), cudaMemcpyHostToDevice));
    ctx->idx_bound[l] = 0;
    if (ctx->occ_h) ctx->occ_h[l] = 0;
  }
  ctx->sb_count = 0;
  ctx->targets_issued = 0;
  CK(cudaMemset(ctx->cnt_total, 0, TG_NCOUNTERS * sizeof(long long)));
  CK(cudaMemset(ctx->cnt_sb, 0, (size_t)kMaxS * TG_NCOUNTERS * sizeof(long long)));
  CK(cudaMemset(ctx->err, 0, 2 * sizeof(int)));
  CK(cudaDeviceSynchronize());
  ctx->launches = 0;
  return TG_OK;
}

tg_status tg_embed_batch(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n, float* out,
                         void* cuda_stream) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  if (n < 0 || n > ctx->cap[ctx->L] || (n > 0 && (!nodes || !ts || !out))) return TG_EINVAL;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  const bool dev_in = n == 0 || is_device_ptr(nodes);
  const bool dev_out = n == 0 || is_device_ptr(out);
  const int32_t* dn = nodes;
  const uint32_t* dt = ts;
  float* dout = out;
  const size_t need = (size_t)n * 8 + (size_t)n * ctx->d_n * 4 + 64;
  if (!dev_in || !dev_out) TRY(ensure_stage(ctx, need));
  char* stg = (char*)ctx->stage;
  if (!dev_in) {
    CK(cudaMemcpyAsync(stg, nodes, n * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(stg + n * 4, ts, n * 4, cudaMemcpyHostToDevice, st));
    dn = (const int32_t*)stg;
    dt = (const uint32_t*)(stg + n * 4);
  }
  if (!dev_out) dout = (float*)(stg + ((n * 8 + 15) & ~15));
  launch_prep_nodes(dn, dt, (int)n, ctx->lv[ctx->L], st);
  TRY(launched(ctx));
  EdgeSrc none{};
  TRY(run_superbatch(ctx, 1, false, none, (int)std::max<int64_t>(n, 1), st));
  launch_invert(ctx->HL, ctx->dnp, ctx->lv[ctx->L], (int)n, ctx->d_n, dout, st);
  TRY(launched(ctx));
  TRY(finish(ctx, 1, nullptr, 0, st));
  if (!dev_out) {
    CK(cudaMemcpyAsync(out, dout, (size_t)n * ctx->d_n * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return TG_OK;
}

// Host buffers are staged through the context's device buffer; every array is checked
// separately (all inputs host or all device: a mix is rejected with TG_EINVAL).
static tg_status stage_edges(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts,
                             const int32_t* neg, int64_t n_edges, float* scores, cudaStream_t st, Staged& o) {
  const bool dev_in = is_device_ptr(src);
  if (is_device_ptr(dst) != dev_in || is_device_ptr(ts) != dev_in || (neg && is_device_ptr(neg) != dev_in))
    return TG_EINVAL;
  const bool dev_out = is_device_ptr(scores);
  const int64_t n_out = (neg ? 2 : 1) * n_edges;
  o.src = src;
  o.dst = dst;
  o.ts = ts;
  o.neg = neg;
  o.out = scores;
  o.host_out = !dev_out;
  if (dev_in && dev_out) return TG_OK;
  TRY(ensure_stage(ctx, (size_t)n_edges * 16 + (size_t)n_out * 4 + 64));
  char* stg = (char*)ctx->stage;
  if (!dev_in) {  // host -> device copies of this call's inputs (H2D)
    CK(cudaMemcpyAsync(stg, src, n_edges * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(stg + n_edges * 4, dst, n_edges * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(stg + n_edges * 8, ts, n_edges * 4, cudaMemcpyHostToDevice, st));
    o.src = (const int32_t*)stg;
    o.dst = (const int32_t*)(stg + n_edges * 4);
    o.ts = (const uint32_t*)(stg + n_edges * 8);
    if (neg) {
      CK(cudaMemcpyAsync(stg + n_edges * 12, neg, n_edges * 4, cudaMemcpyHostToDevice, st));
      o.neg = (const int32_t*)(stg + n_edges * 12);
    }
  }
  if (!dev_out) o.out = (float*)(stg + n_edges * 16);
  return TG_OK;
}

tg_status tg_score_edges(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts, int64_t n_edges,
                         float* scores, void* cuda_stream) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  if (n_edges < 0 || 2 * n_edges > ctx->cap[ctx->L] || (n_edges > 0 && (!src || !dst || !ts || !scores)))
    return TG_EINVAL;
  if (n_edges == 0) return TG_OK;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  Staged o;
  TRY(stage_edges(ctx, src, dst, ts, nullptr, n_edges, scores, st, o));
  TRY(stream_edges(ctx, o.src, o.dst, o.ts, nullptr, n_edges, (int)n_edges, o.out, nullptr, st));
  if (o.host_out) {
    CK(cudaMemcpyAsync(scores, o.out, n_edges * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return TG_OK;
}

tg_status tg_score_pairs(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n_targets,
                         const int32_t* pair_a, const int32_t* pair_b, int64_t n_pairs, float* scores,
                         void* cuda_stream) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  const int64_t ne = (int64_t)ctx->cfg.max_batch_targets;  // the score workspace holds at least this many
  if (n_targets < 0 || n_targets > ctx->cap[ctx->L] || n_pairs < 0 || n_pairs > ne ||
      (n_targets > 0 && (!nodes || !ts)) || (n_pairs > 0 && (!pair_a || !pair_b || !scores)))
    return TG_EINVAL;
  if (n_pairs == 0 && n_targets == 0) return TG_OK;
  if (n_pairs > 0 && n_targets == 0) return TG_EINVAL;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  const bool dev_in = is_device_ptr(nodes);
  // every input array is checked: a host/device mix would make a kernel dereference host memory
  if (is_device_ptr(ts) != dev_in || (n_pairs > 0 && (is_device_ptr(pair_a) != dev_in || is_device_ptr(pair_b) != dev_in)))
    return TG_EINVAL;
  const bool dev_out = n_pairs == 0 || is_device_ptr(scores);
  if (!dev_in && n_pairs > 0) {  // host pairs: range-checked here, before any launch
    for (int64_t p = 0; p < n_pairs; ++p)
      if (pair_a[p] < 0 || pair_a[p] >= n_targets || pair_b[p] < 0 || pair_b[p] >= n_targets) return TG_EINVAL;
  }
  const int32_t* dn = nodes;
  const uint32_t* dt = ts;
  const int32_t* da = pair_a;
  const int32_t* db = pair_b;
  float* dout = scores;
  if (!dev_in || !dev_out) {
    const size_t n8 = ((size_t)n_targets * 8 + 15) & ~(size_t)15, p8 = ((size_t)n_pairs * 8 + 15) & ~(size_t)15;
    TRY(ensure_stage(ctx, n8 + p8 + (size_t)n_pairs * 4 + 64));
    char* stg = (char*)ctx->stage;
    if (!dev_in) {
      CK(cudaMemcpyAsync(stg, nodes, n_targets * 4, cudaMemcpyHostToDevice, st));
      CK(cudaMemcpyAsync(stg + n_targets * 4, ts, n_targets * 4, cudaMemcpyHostToDevice, st));
      CK(cudaMemcpyAsync(stg + n8, pair_a, n_pairs * 4, cudaMemcpyHostToDevice, st));
      CK(cudaMemcpyAsync(stg + n8 + n_pairs * 4, pair_b, n_pairs * 4, cudaMemcpyHostToDevice, st));
      dn = (const int32_t*)stg;
      dt = (const uint32_t*)(stg + n_targets * 4);
      da = (const int32_t*)(stg + n8);
      db = (const int32_t*)(stg + n8 + n_pairs * 4);
    }
    if (!dev_out) dout = (float*)(stg + n8 + p8);
  }
  // embeddings of the (deduplicated) target list: one Alg. 1 batch, cache on
  launch_prep_nodes(dn, dt, (int)n_targets, ctx->lv[ctx->L], st);
  TRY(launched(ctx));
  EdgeSrc none{};
  TRY(run_superbatch(ctx, 1, false, none, (int)n_targets, st));
  if (n_pairs > 0) {
    Prof pf(ctx, TG_ST_SCORE, st);
    launch_pair_rows(ctx->HL, ctx->dnp, ctx->lv[ctx->L], (int)n_targets, da, db, (int)n_pairs, ctx->sc_rs,
                     ctx->sc_rd, ctx->sc_oidx, ctx->sc_m, ctx->err, st);
    GemmArgs g{};  // hidden layer of the affinity MLP over the pairs (R10)
    g.err = ctx->err;
    g.a_rows0 = ctx->sc_rs;
    g.K0 = ctx->dnp;
    g.a_rows1 = ctx->sc_rd;
    g.K = 2 * ctx->dnp;
    g.B = ctx->Wa1;
    g.N = ctx->dnp;
    g.bias = ctx->ba1;
    g.relu = 1;
    g.C = ctx->sc_z;
    g.ldc = ctx->dnp;
    g.m_dev = ctx->sc_m;
    g.m_max = (int)n_pairs;
    if (ctx->cfg.precision == TG_PREC_BF16) launch_gemm_tc(g, ctx->tcWa1g, TG_PREC_TF32, st);
    else if (ctx->cfg.precision != TG_PREC_FP32) launch_gemm_tc(g, ctx->tcWa1, ctx->cfg.precision, st);
    else launch_gemm_simt(g, st);
    launch_score_head(ctx->sc_z, ctx->dnp, ctx->sc_oidx, (int)n_pairs, ctx->Wa2, ctx->ba2, ctx->d_n, dout, st);
    TRY(launched(ctx, 3));
  }
  TRY(finish(ctx, 1, nullptr, 0, st));
  if (!dev_out) {
    CK(cudaMemcpyAsync(scores, dout, n_pairs * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return TG_OK;
}

tg_status tg_score_stream(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts, int64_t n_edges,
                          int32_t batch, float* scores, int64_t* batch_counters, void* cuda_stream) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  if (n_edges < 0 || batch < 1 || 2 * batch > ctx->cap[ctx->L] || (n_edges > 0 && (!src || !dst || !ts || !scores)))
    return TG_EINVAL;
  if (n_edges == 0) return TG_OK;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  Staged o;
  TRY(stage_edges(ctx, src, dst, ts, nullptr, n_edges, scores, st, o));
  TRY(stream_edges(ctx, o.src, o.dst, o.ts, nullptr, n_edges, batch, o.out, (long long*)batch_counters, st));
  if (o.host_out) {  // device -> host read of the results (D2H)
    CK(cudaMemcpyAsync(scores, o.out, n_edges * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return TG_OK;
}

tg_status tg_score_stream_neg(tg_ctx* ctx, const int32_t* src, const int32_t* dst, const uint32_t* ts,
                              const int32_t* neg, int64_t n_edges, int32_t batch, float* scores,
                              int64_t* batch_counters, void* cuda_stream) {
  if (!ctx) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (ctx->broken) return TG_ECUDA;
  if (n_edges < 0 || batch < 1 || 3 * batch > ctx->cap[ctx->L] ||
      (n_edges > 0 && (!src || !dst || !ts || !neg || !scores)))
    return TG_EINVAL;
  if (n_edges == 0) return TG_OK;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  Staged o;
  TRY(stage_edges(ctx, src, dst, ts, neg, n_edges, scores, st, o));
  TRY(stream_edges(ctx, o.src, o.dst, o.ts, o.neg, n_edges, batch, o.out, (long long*)batch_counters, st));
  if (o.host_out) {  // device -> host read of the results (D2H)
    CK(cudaMemcpyAsync(scores, o.out, 2 * n_edges * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return TG_OK;
}

tg_status tg_profile_enable(tg_ctx* ctx, int32_t on) {
  if (!ctx) return TG_EINVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  ctx->prof = on != 0;
  ctx->ev_used = 0;
  return TG_OK;
}

tg_status tg_profile_read(tg_ctx* ctx, double* ms, int64_t* launches, int32_t n) {
  if (!ctx || n < 0) return TG_EINVAL;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  std::vector<double> acc(TG_NSTAGES, 0.0);
  std::vector<int64_t> cnt(TG_NSTAGES, 0);
  for (size_t i = 0; i < ctx->ev_used; ++i) {
    float t = 0.f;
    if (cudaEventElapsedTime(&t, ctx->ev_pool[2 * i], ctx->ev_pool[2 * i + 1]) != cudaSuccess) {
      cudaGetLastError();
      continue;
    }
    acc[ctx->ev_stage[i]] += t;
    cnt[ctx->ev_stage[i]] += 1;
  }
  for (int i = 0; i < n && i < TG_NSTAGES; ++i) {
    if (ms) ms[i] = acc[i];
    if (launches) launches[i] = cnt[i];
  }
  return TG_OK;
}

tg_status tg_counters_read(tg_ctx* ctx, int64_t* host_out, int32_t n) {
  if (!ctx || !host_out || n < 0) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  CK(cudaSetDevice(ctx->device));
  CK(cudaDeviceSynchronize());
  long long tmp[TG_NCOUNTERS];
  CK(cudaMemcpy(tmp, ctx->cnt_total, sizeof(tmp), cudaMemcpyDeviceToHost));
  for (int i = 0; i < n && i < TG_NCOUNTERS; ++i) host_out[i] = tmp[i];
  int e = 0;
  CK(cudaMemcpy(&e, ctx->err, sizeof(int), cudaMemcpyDeviceToHost));
  return e ? TG_EDEVICE : TG_OK;
}

tg_status tg_dedup(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n, int32_t* uniq_nodes,
                   uint32_t* uniq_ts, int32_t* inv, int32_t* n_uniq, void* cuda_stream) {
  if (!ctx || n < 0 || n > 16 * 10000) return TG_EINVAL;
  if (n > 0 && (!nodes || !ts || !uniq_nodes || !uniq_ts || !inv || !n_uniq)) return TG_EINVAL;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  int* ndev = nullptr;
  CK(cudaMalloc(&ndev, sizeof(int)));
  int nn = (int)n;
  CK(cudaMemcpyAsync(ndev, &nn, sizeof(int), cudaMemcpyHostToDevice, st));
  LevelDev v{};
  v.cap = (int)std::max<int64_t>(n, 1);
  v.in_node = const_cast<int32_t*>(nodes);
  v.in_ts = const_cast<uint32_t*>(ts);
  v.n_in = ndev;
  v.u_node = uniq_nodes;
  v.u_ts = uniq_ts;
  v.n_u = n_uniq;
  v.inv = inv;
  EdgeSrc none{};
  launch_dedup(v, 1, v.cap, false, none, nullptr, 0, true, ctx->err, st);
  cudaError_t e = cudaGetLastError();
  cudaStreamSynchronize(st);
  cudaFree(ndev);
  return e == cudaSuccess ? TG_OK : TG_ECUDA;
}

tg_status tg_sample(tg_ctx* ctx, const int32_t* nodes, const uint32_t* ts, int64_t n, int32_t* nbr, int32_t* eid,
                    uint32_t* nts, void* cuda_stream) {
  if (!ctx || n < 0) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (n == 0) return TG_OK;
  if (!nodes || !ts || !nbr || !eid || !nts) return TG_EINVAL;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  // a one-batch compute list over the caller's targets
  int* meta = nullptr;
  int32_t* cb = nullptr;
  CK(cudaMalloc(&meta, 4 * sizeof(int)));
  CK(cudaMalloc(&cb, (size_t)n * sizeof(int32_t)));
  CK(cudaMemsetAsync(cb, 0, (size_t)n * sizeof(int32_t), st));
  int h[4] = {0, (int)n, (int)n, 0};  // c_base[0], n_c[0], n_c_total
  CK(cudaMemcpyAsync(meta, h, sizeof(h), cudaMemcpyHostToDevice, st));
  LevelDev v{};
  v.cap = (int)n;
  v.c_cap = (int)n;
  v.c_b = cb;
  v.c_node = const_cast<int32_t*>(nodes);
  v.c_ts = const_cast<uint32_t*>(ts);
  v.c_base = meta;
  v.n_c = meta + 1;
  v.n_c_total = meta + 2;
  v.nb_node = nbr;
  v.nb_ts = nts;
  v.nb_eid = eid;
  launch_sample(ctx->g, v, 1, ctx->k, nullptr, ctx->W, 0, nullptr, 0, ctx->err, st);
  cudaError_t e = cudaGetLastError();
  cudaStreamSynchronize(st);
  cudaFree(meta);
  cudaFree(cb);
  return e == cudaSuccess ? TG_OK : TG_ECUDA;
}

tg_status tg_time_encode(tg_ctx* ctx, const int64_t* delta, int64_t n, int32_t use_table, float* out,
                         void* cuda_stream) {
  if (!ctx || n < 0) return TG_EINVAL;
  if (!ctx->loaded) return TG_ESTATE;
  if (n > 0 && (!delta || !out)) return TG_EINVAL;
  CK(cudaSetDevice(ctx->device));
  launch_time_encode(ctx->omega, ctx->phi, ctx->table, ctx->d_t, ctx->dtp, ctx->W, use_table, delta, n, out,
                     (cudaStream_t)cuda_stream);
  CK(cudaGetLastError());
  return TG_OK;
}

tg_status tg_gemm(tg_ctx* ctx, int32_t precision, int32_t M, int32_t N, int32_t K, const float* A,
                  const float* B, const float* bias, int32_t relu, float* C, void* cuda_stream) {
  if (!ctx || M < 0 || N < 4 || K < 4 || (N & 3) || (K & 3) || !A || !B || !C) return TG_EINVAL;
  if (precision < TG_PREC_FP32 || precision > TG_PREC_LAST) return TG_EINVAL;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  CK(cudaSetDevice(ctx->device));
  if (!ctx->gemm_m) TRY(dalloc(ctx, &ctx->gemm_m, 1));
  launch_set_int(ctx->gemm_m, M, st);  // stream-ordered (device count as on the hot path)
  GemmArgs g{};
  g.err = ctx->err;
  g.a_base0 = A;
  g.lda0 = K;
  g.K0 = g.K = K;
  g.B = B;
  g.N = N;
  g.bias = bias;
  g.relu = relu;
  g.C = C;
  g.ldc = N;
  g.m_dev = ctx->gemm_m;
  g.m_max = std::max(M, 1);
  if (precision == TG_PREC_FP32) {
    launch_gemm_simt(g, st);
  } else {
    // weights re-tiled once per (B, N, K, precision) and cached in the context
    const TcWeights* w = nullptr;
    for (auto& e : ctx->gemm_cache)
      if (e.B == B && e.N == N && e.K == K && e.prec == precision) w = &e.w;
    if (!w) {
      tg_ctx::GemmCacheEntry e{B, N, K, precision, {}};
      TRY(tc_prepare_weights(B, N, K, precision, &e.w, ctx->owned));
      ctx->gemm_cache.push_back(e);
      w = &ctx->gemm_cache.back().w;
    }
    TcTensorA ta;  // dense fp32 A via TMA in the one-pass tf32 mode
    if ((precision == TG_PREC_TF32 || precision == TG_PREC_TF32X3 || precision == TG_PREC_F16X3) && M > 0)
      TRY(tc_make_tensor_a(A, 4, K, M, &ta));  // tf32: the MMA's A; fp32-level: the producers' staging
    launch_gemm_tc(g, *w, precision, st, ta.valid ? &ta : nullptr);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    fprintf(stderr, "libtg: tg_gemm %s\n", cudaGetErrorString(e));
    return TG_ECUDA;
  }
  return TG_OK;  // stream-ordered; the caller synchronises
}

void tg_free(tg_ctx* ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->device);
  cudaDeviceSynchronize();
  if (getenv("TG_DBG_INDEX_CHECK") && ctx->err) {
    int e[2] = {0, 0};
    cudaMemcpy(e, ctx->err, sizeof(e), cudaMemcpyDeviceToHost);
    fprintf(stderr, "libtg: index check mismatches %d (err bits %d)\n", e[1], e[0]);
  }
  for (void* p : ctx->owned) cudaFree(p);
  for (void* p : ctx->owned_host) cudaFreeHost(p);
  for (cudaEvent_t e : ctx->ev_pool) cudaEventDestroy(e);
  for (cudaEvent_t e : {ctx->ev_front[0], ctx->ev_front[1], ctx->ev_back[0], ctx->ev_back[1], ctx->ev_in, ctx->ev_fend,
                        ctx->ev_lend})
    if (e) cudaEventDestroy(e);
  if (ctx->fst) cudaStreamDestroy(ctx->fst);
  if (ctx->lst) cudaStreamDestroy(ctx->lst);
  if (ctx->occ_h) cudaFreeHost(ctx->occ_h);
  if (ctx->stage) cudaFree(ctx->stage);
  delete ctx;
}

}  // extern "C"
