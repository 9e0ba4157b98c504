// tcgen05 tensor-core GEMM for the dense per-target projections (sm_100a):
//   C[M x N] = epilogue(A[M x K] . B[N x K]^T)
//
// Persistent, warp-specialized, mbarrier-pipelined:
//   warps 0-3  A producers: thread t owns row m0+t of the tile; gathers the
//              row through its row pointer(s) (or dense), converts it (tf32
//              hi/lo split or bf16) and writes it into shared memory in the
//              canonical K-major 128B-swizzled UMMA layout;
//   warp 4     B producer: one lane issues TMA bulk copies (cp.async.bulk,
//              mbarrier complete_tx) of the pre-tiled weight images;
//   warp 5     MMA issuer: one lane issues tcgen05.mma (M = 128, N = BN) into a
//              double-buffered TMEM accumulator and commits to mbarriers;
//   warps 6-13 epilogue, two warps per TMEM lane quadrant splitting the
//              columns: tcgen05.ld (32x32b) -> per-warp shared transpose ->
//              bias / ReLU on float4 -> coalesced row stores (dense or
//              gathered destinations, fp32 and/or bf16).
// `stages` shared-memory stages decouple the producers from the tensor core.
//
// TG_PREC_TF32X3: kind::tf32 with the 3-term split a.b ~ ah.bh + ah.bl + al.bh
// (ah = rna_tf32(a), al = rna_tf32(a - ah)): fp32-level accuracy on tensor
// cores. TG_PREC_BF16: kind::f16 with bf16 operands, fp32 accumulation.
// TG_PREC_F16X3: kind::f16 with fp16 operands and the same 3-term split
// (ah = rn_f16(a), al = rn_f16(a - ah); 11 + 11 significant bits like tf32 hi/lo)
// at twice the tf32 MMA rate and half the shared-memory bytes per product. fp16's
// exponent range is handled by an exact power-of-two scale per weight row (host,
// undone per output column in the epilogue); activations must satisfy |a| < 65504
// (checked by the producers: sticky device error kErrF16Range otherwise).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "tg_tc.cuh"

namespace tg {

constexpr int TC_BM = 128;
// warp roles: [0, 8) A producers, 8 TMA (B and dense A tiles), 9 MMA issuer, [10, 14)
// epilogue (one per TMEM lane quadrant: warp w may only access lanes 32 (w % 4) .. + 31)
constexpr int TC_PROD_WARPS = 8;
constexpr int TC_EPI_WARPS = 4;
constexpr int TC_EPI_HALVES = TC_EPI_WARPS / 4;  // epilogue warps per lane quadrant (column split)
constexpr int TC_TMA_WARP = TC_PROD_WARPS, TC_MMA_WARP = TC_PROD_WARPS + 1, TC_EPI_WARP0 = TC_PROD_WARPS + 2;
// + one staging warp: refills the fp32-level producers' staging ring by TMA (stage_tma)
constexpr int TC_STG_WARP = TC_EPI_WARP0 + TC_EPI_WARPS;
constexpr int TC_WARPS = TC_PROD_WARPS + 2 + TC_EPI_WARPS + 1;
constexpr int TC_THREADS = TC_WARPS * 32;
constexpr int TC_MAXSTAGES = 8;
// TMEM: two accumulator buffers of 256 columns (all 512 columns; one CTA per
// SM). Two CTAs per SM with 2 x 128 columns each was measured slower.
__host__ __device__ constexpr int tc_acc_cols(int) { return 256; }
__host__ __device__ constexpr int tc_ctas_per_sm(int) { return 1; }

__host__ __device__ inline int tc_epc(int prec) {  // elements per 128 B
  return (prec == TG_PREC_BF16 || prec == TG_PREC_F16X3) ? 64 : 32;
}
__host__ __device__ inline int tc_planes(int prec) { return (prec == TG_PREC_TF32X3 || prec == TG_PREC_F16X3) ? 2 : 1; }
// TMEM plan of the fp32-level modes (A in TMEM): accumulator buffers of [big | small]
// (2 x round32(BN) columns) -- two (the epilogue drains one while the MMA fills the other)
// when they leave room for >= 2 A stages of 64 columns, else one; returns the A stages that fit
#ifndef TG_X3_NBUF_MAX
#define TG_X3_NBUF_MAX 2
#endif
__host__ __device__ inline int tc_tmem_nbuf(int BN) {
  const int buf = 2 * ((BN + 31) & ~31);
  return (TG_X3_NBUF_MAX > 1 && 2 * buf + 4 * 32 <= 512) ? 2 : 1;
}
__host__ __device__ inline int tc_tmem_astages(int BN) {  // A stages of 32 columns (64-byte k-blocks)
  const int buf = 2 * ((BN + 31) & ~31);
  return (512 - tc_tmem_nbuf(BN) * buf) / 32;
}

// offset of 16-byte chunk c of row r inside a 128B-swizzled K-major tile
__host__ __device__ inline unsigned sw128(int r, int c) {
  return (unsigned)((r >> 3) * 1024 + (r & 7) * 128 + ((c ^ (r & 7)) << 4));
}
// ... inside a 64B-swizzled K-major tile (8-row atoms of 512 B; chunk c in [0, 4))
__host__ __device__ inline unsigned sw64(int r, int c) {
  return (unsigned)((r >> 3) * 512 + (r & 7) * 64 + ((c ^ ((r >> 1) & 3)) << 4));
}
// The fp32-level modes (A in TMEM) stage B in 64-byte k-blocks (tf32: 16, f16: 32 elements):
// twice the pipeline stages in the same TMEM / shared memory as 128-byte k-blocks
__host__ __device__ inline int tc_kb_bytes(int prec) {
  return (prec == TG_PREC_TF32X3 || prec == TG_PREC_F16X3) ? 64 : 128;
}

// shared memory after the stages: barriers, then a 32 x 16 fp32 transpose
// buffer per epilogue warp
constexpr int TC_BAR_BYTES = 256;
constexpr int TC_STG_LD = 20;  // floats per staged row (16 columns + pad)
// + per-tile bias / column-scale staging, double-buffered by tile parity: [2][bias 256 | scale 256]
constexpr int TC_EPI_XPOSE_BYTES = TC_EPI_WARPS * 32 * TC_STG_LD * 4;
constexpr int TC_EPI_BYTES = TC_EPI_XPOSE_BYTES + 2 * 2 * 256 * 4;

// fused-LayerNorm epilogue (g.ln): per-row partial statistics of the two
// column halves [2][128] and the cluster exchange buffers [2 parities][4 N tiles][128]
constexpr int TC_LN_MAXTN = 4;
constexpr int TC_LN_BYTES = (2 * 128 + 2 * TC_LN_MAXTN * 128) * 16 + 4 * 256 * 4;  // + bias, gamma, beta, valid

// Shared-memory plan: `stages` operand stages plus, when the generic fp32 A producer runs,
// `stg` staging units of 16 KB (its cp.async look-ahead ring, up to 4 units) -- as many
// staging units as fit beside 2 stages, then as many stages as fit beside those.
constexpr int TC_STG_UNIT = TC_BM * 128;
constexpr int TC_PTR_BYTES = 2 * TC_BM * 8 + 64;  // the producers' row-pointer table + staging mbarriers [2][4]
static inline bool tc_atmem(int prec) { return tc_planes(prec) == 2; }  // A operand in TMEM
static inline void tc_plan(int prec, int BN, int ln, bool generic, int* stages, int* stg) {
  const size_t st = (size_t)tc_planes(prec) * ((tc_atmem(prec) ? 0 : (size_t)TC_BM * 128) + (size_t)BN * tc_kb_bytes(prec));
  const size_t budget = (tc_ctas_per_sm(prec) == 1 ? 205 * 1024 : 100 * 1024) - (ln ? TC_LN_BYTES : 0) -
                        (generic ? TC_PTR_BYTES + 1024 : 0);
  int d = 0;  // 0: no room beside 2 stages -> the producers load synchronously
  static const int d_env = [] {  // TG_GEMM_STG: cap on staging units (A/B experiments)
    const char* e = getenv("TG_GEMM_STG");
    return e ? atoi(e) : 4;
  }();
  if (generic) {
    d = budget > 2 * st ? (int)((budget - 2 * st) / TC_STG_UNIT) : 0;
    d = d > d_env ? d_env : d;
    if (d_env < 0) d = -1;  // TG_GEMM_STG=-1: register prefetch, no staging ring
  }
  int s = (int)((budget - (size_t)(d > 0 ? d : 0) * TC_STG_UNIT) / st);
  if (s > TC_MAXSTAGES) s = TC_MAXSTAGES;
  if (tc_atmem(prec)) {  // TMEM: [big | small] accumulator buffer(s) + 64 columns of A per stage
    const int sa = tc_tmem_astages(BN);
    if (s > sa) s = sa;
  }
  *stages = s < 2 ? 2 : s;
  *stg = d;
}

// ------------------------------------------------------------ host: weights
static inline uint32_t f2u(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  return u;
}
static inline float u2f(uint32_t u) {
  float f;
  memcpy(&f, &u, 4);
  return f;
}
static inline float tf32_rna(float x) {  // round to nearest (ties away) on the 10-bit mantissa
  uint32_t u = f2u(x);
  if ((u & 0x7f800000u) == 0x7f800000u) return x;
  u = (u + 0x1000u) & 0xffffe000u;
  return u2f(u);
}
static inline uint16_t bf16_rn(float x) {
  uint32_t u = f2u(x);
  u += 0x7fffu + ((u >> 16) & 1u);
  return (uint16_t)(u >> 16);
}

tg_status tc_prepare_weights(const float* W, int N, int K, int precision, TcWeights* out,
                             std::vector<void*>& owned) {
  // N tiles of <= 256 columns: each A tile is re-read once per N tile, and the
  // kernel is bound by L2 -> SM operand traffic at these sizes
  // (narrow GEMMs, N <= 256, keep two N tiles for parallelism instead)
  int ntn = (N > 256 && tc_acc_cols(precision) == 256) ? (N + 255) / 256 : (N + 127) / 128;
  // tf32x3 keeps a [big | small] accumulator pair per buffer: N tiles <= 128 keep the
  // epilogue double-buffered (4 x 128 TMEM columns); wider tiles run single-buffered
  // fp32-level modes keep A in TMEM beside a [big | small] accumulator pair: wide N tiles are
  // capped at 192 columns so that >= 2 A stages (64 columns each) fit in the 512 TMEM columns
  static const int x3_bn = [] {
    const char* e = getenv("TG_X3_BN");
    return e ? atoi(e) : 192;
  }();
  if ((precision == TG_PREC_TF32X3 || precision == TG_PREC_F16X3) && x3_bn > 0 && x3_bn < 256 && N > 256)
    ntn = (N + x3_bn - 1) / x3_bn;
  // narrow fp32-level GEMMs (N <= 192: G3, G4, the score MLP) run ONE N tile of round16(N) columns
  // (single-buffered [big | small]): a tf32x3 k-block of 16 K costs about the same (~0.47 us, six
  // MMAs) at N = 96 and N = 176 (clock64 traces), so two 96-column tiles cost twice the MMA time
  // and convert A twice (measured: G3 68 -> 55 us, G4 42 -> 36 us per launch; TG_X3_NARROW=2: two)
  static const int x3_narrow = [] {
    const char* e = getenv("TG_X3_NARROW");
    return e ? atoi(e) : 1;
  }();
  if ((precision == TG_PREC_TF32X3 || precision == TG_PREC_F16X3) && N <= 256 && N <= x3_bn && x3_narrow >= 1)
    ntn = std::min(ntn, x3_narrow);
  int BN = (N + ntn - 1) / ntn;
  BN = (BN + 15) & ~15;
  const int kbb = tc_kb_bytes(precision);          // bytes of K per k-block row
  const int epc = tc_epc(precision) * kbb / 128;   // elements per k-block row
  const int nkb = (K + epc - 1) / epc;
  const int planes = tc_planes(precision);
  const size_t plane_bytes = (size_t)BN * kbb;
  const size_t total = (size_t)ntn * nkb * planes * plane_bytes;
  std::vector<float> w((size_t)N * K);
  if (cudaMemcpy(w.data(), W, w.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) return TG_ECUDA;
  std::vector<unsigned char> img(total, 0);
  // F16X3: exact power-of-two scale per weight row n so that max_k |W[n,k]| 2^e lies in
  // [2^14, 2^15) -- the hi and lo fp16 parts then stay normal for every element within
  // 2^-14 of the row maximum; the epilogue multiplies output column n by 2^-e
  std::vector<float> colscale;
  if (precision == TG_PREC_F16X3) {
    colscale.assign((size_t)ntn * BN, 1.f);
    for (int n = 0; n < N; ++n) {
      float mx = 0.f;
      for (int k = 0; k < K; ++k) mx = std::max(mx, std::fabs(w[(size_t)n * K + k]));
      if (mx > 0.f && std::isfinite(mx)) {
        int e = 0;
        std::frexp(mx, &e);  // mx = f 2^e, f in [0.5, 1): mx 2^(15 - e) in [2^14, 2^15)
        const int s = 15 - e;
        for (int k = 0; k < K; ++k) w[(size_t)n * K + k] = std::ldexp(w[(size_t)n * K + k], s);
        colscale[n] = std::ldexp(1.f, -s);
      }
    }
  }
  for (int tn = 0; tn < ntn; ++tn)
    for (int kb = 0; kb < nkb; ++kb) {
      unsigned char* base = img.data() + ((size_t)tn * nkb + kb) * planes * plane_bytes;
      for (int r = 0; r < BN; ++r) {
        const int n = tn * BN + r;
        for (int c = 0; c < kbb / 16; ++c) {
          unsigned char* dst0 = base + (kbb == 64 ? sw64(r, c) : sw128(r, c));
          if (precision == TG_PREC_F16X3) {
            uint16_t vh[8], vl[8];
            for (int e = 0; e < 8; ++e) {
              const int kk = kb * epc + c * 8 + e;
              const float x = (n < N && kk < K) ? w[(size_t)n * K + kk] : 0.f;
              const __half h = __float2half_rn(x);
              const __half l = __float2half_rn(x - __half2float(h));
              memcpy(&vh[e], &h, 2);
              memcpy(&vl[e], &l, 2);
            }
            memcpy(dst0, vh, 16);
            memcpy(dst0 + plane_bytes, vl, 16);
          } else if (precision == TG_PREC_BF16) {
            uint16_t v[8];
            for (int e = 0; e < 8; ++e) {
              const int kk = kb * epc + c * 8 + e;
              v[e] = (n < N && kk < K) ? bf16_rn(w[(size_t)n * K + kk]) : 0;
            }
            memcpy(dst0, v, 16);
          } else {
            float hi[4], lo[4];
            for (int e = 0; e < 4; ++e) {
              const int kk = kb * epc + c * 4 + e;
              const float x = (n < N && kk < K) ? w[(size_t)n * K + kk] : 0.f;
              hi[e] = tf32_rna(x);
              lo[e] = tf32_rna(x - hi[e]);
            }
            memcpy(dst0, hi, 16);
            if (planes == 2) memcpy(dst0 + plane_bytes, lo, 16);
          }
        }
      }
    }
  void* d = nullptr;
  if (cudaMalloc(&d, total) != cudaSuccess) return TG_ENOMEM;
  owned.push_back(d);
  if (cudaMemcpy(d, img.data(), total, cudaMemcpyHostToDevice) != cudaSuccess) return TG_ECUDA;
  out->hi = d;
  out->lo = nullptr;
  out->colscale = nullptr;
  if (!colscale.empty()) {
    void* cs = nullptr;
    if (cudaMalloc(&cs, colscale.size() * 4) != cudaSuccess) return TG_ENOMEM;
    owned.push_back(cs);
    if (cudaMemcpy(cs, colscale.data(), colscale.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) return TG_ECUDA;
    out->colscale = reinterpret_cast<float*>(cs);
  }
  out->N = N;
  out->K = K;
  out->Np = ntn * BN;
  out->Kp = nkb * epc;
  out->BN = BN;
  out->ntn = ntn;
  out->nkb = nkb;
  return TG_OK;
}

// ------------------------------------------------------------ device helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
  // K-major, SWIZZLE_128B: LBO unused (1), SBO = 1024 B between 8-row groups,
  // version 1 (sm_100), layout type 2 at bits [61,64)
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

__device__ __forceinline__ uint64_t umma_desc64(uint32_t saddr) {
  // K-major, SWIZZLE_64B: SBO = 512 B between 8-row groups, layout type 4
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)4 << 61;
  return d;
}

__device__ __forceinline__ uint32_t umma_idesc(int prec, int N) {
  uint32_t d = 0;
  d |= 1u << 4;                                         // D = f32
  const uint32_t fmt = prec == TG_PREC_BF16 ? 1u : prec == TG_PREC_F16X3 ? 0u : 2u;  // bf16 : f16 : tf32
  d |= fmt << 7;                                        // A format
  d |= fmt << 10;                                       // B format
  d |= (uint32_t)(N >> 3) << 17;                        // N / 8
  d |= (uint32_t)(TC_BM >> 4) << 24;                    // M / 16
  return d;
}

template <int PREC>
__device__ __forceinline__ void mma_issue(uint32_t tmem, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
  if (PREC == TG_PREC_BF16 || PREC == TG_PREC_F16X3) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
        "l"(da), "l"(db), "r"(idesc), "r"(acc));
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem),
        "l"(da), "l"(db), "r"(idesc), "r"(acc));
  }
}

// A operand in tensor memory (M = 128 lanes = rows; kind::tf32: one element per 32-bit column,
// kind::f16: two per column): the MMA reads only B from shared memory
template <int PREC>
__device__ __forceinline__ void mma_issue_ts(uint32_t tmem, uint32_t atmem, uint64_t db, uint32_t idesc, uint32_t acc) {
  if (PREC == TG_PREC_F16X3) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(tmem),
        "r"(atmem), "l"(db), "r"(idesc), "r"(acc));
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(tmem),
        "r"(atmem), "l"(db), "r"(idesc), "r"(acc));
  }
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};\n" ::"r"(
          taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
      "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&v)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};\n" ::"r"(taddr), "r"(v[0]),
               "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.b32 %0, 1, 0, P1;\n\t}\n"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  }
}
// cluster-scope variants for the LayerNorm statistics exchange (DSMEM)
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.b32 %0, 1, 0, P1;\n\t}\n"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  }
}
__device__ __forceinline__ uint32_t mapa_u32(uint32_t local, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;\n" : "=r"(r) : "r"(local), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_cluster_v4(uint32_t addr, float4 v) {
  asm volatile("st.shared::cluster.v4.f32 [%0], {%1, %2, %3, %4};\n" ::"r"(addr), "f"(v.x), "f"(v.y), "f"(v.z),
               "f"(v.w)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];\n" ::"r"(addr) : "memory");
}
// Chan et al. pairwise merge of (count, mean, M2) running statistics; fixed
// merge order keeps every row's result independent of the batch (row-invariant)
__device__ __forceinline__ void chan_merge(float& n, float& m, float& M2, float nb, float mb, float Mb) {
  if (nb == 0.f) return;
  if (n == 0.f) {
    n = nb;
    m = mb;
    M2 = Mb;
    return;
  }
  const float nn = n + nb, d = mb - m;
  m = m + d * (nb / nn);
  M2 = M2 + Mb + d * d * (n * nb / nn);
  n = nn;
}
__device__ __forceinline__ bool ln_valid(const GemmArgs& g, int c) {
  return c < g.N && (c < g.ln_dn || (c >= g.ln_s1 && c < g.ln_s1 + g.ln_de) || (c >= g.ln_s2 && c < g.ln_s2 + g.ln_dt));
}
// accumulator chunk (16 columns from local column cl) + bias (staged in shared memory)
__device__ __forceinline__ void ln_chunk(const uint32_t (&v)[16], const float* s_bias, int cl, float (&x)[16]) {
#pragma unroll
  for (int j = 0; j < 16; ++j) x[j] = __uint_as_float(v[j]) + s_bias[cl + j];
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ float rna_tf32(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;\n" : "=r"(r) : "f"(x));
  return __uint_as_float(r);
}
// The same rounding (nearest, ties away from zero, on the 13 dropped mantissa bits) with two
// full-rate integer ops instead of the conversion pipe -- the A producers' hot loop
// (bit-identical to cvt.rna.tf32.f32 for finite x; a NaN may come out as Inf)
__device__ __forceinline__ float rna_tf32_fast(float x) {
  return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xffffe000u);
}

__device__ __forceinline__ float4 tc_load4(const GemmArgs& g, const float* r0, const float* r1, int col) {
  if (col >= g.K) return make_float4(0.f, 0.f, 0.f, 0.f);
  const float* p = col < g.K0 ? r0 + col : r1 + (col - g.K0);
  return *reinterpret_cast<const float4*>(p);
}
__device__ __forceinline__ float4 tc_ldg4(const GemmArgs& g, const float* r0, const float* r1, int col) {
  if (col >= g.K) return make_float4(0.f, 0.f, 0.f, 0.f);
  const float* p = col < g.K0 ? r0 + col : r1 + (col - g.K0);
  return __ldg(reinterpret_cast<const float4*>(p));  // A is read-only for the whole launch
}

#ifdef TG_TC_TRACE
// Debug build only (build.py TG_TRACE=1 -> libtg_trace.so): clock64 stamps of the
// first tile of each CTA for launches whose (N, K) matches the armed shape.
constexpr int TCT_N = 64;
__device__ long long tg_tct[148][TCT_N];
__device__ int tg_tct_nk[3];  // N, K, (unused)
#define TCT(i, v)                                                                              \
  do {                                                                                         \
    if (tct_on && blockIdx.x < 148 && (i) < TCT_N) tg_tct[blockIdx.x][(i)] = (long long)(v); \
  } while (0)
#else
#define TCT(i, v) \
  do {            \
  } while (0)
#endif

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
}

// staging ring of the generic A producers: after stages, barriers, epilogue buffers [, LN], at a
// 1024-byte boundary (TMA's 128-byte swizzle is a function of the address); then the row-pointer
// table [2][128] and the staging mbarriers [landed 4 | read 4]
__device__ __forceinline__ unsigned char* tc_stage_ring(unsigned char* smem, uint32_t stage_total, int ln) {
  return smem + ((stage_total + TC_BAR_BYTES + TC_EPI_BYTES + (ln ? TC_LN_BYTES : 0) + 1023u) & ~1023u);
}
__device__ __forceinline__ uint64_t* tc_stage_bars(unsigned char* smem, uint32_t stage_total, int ln, int stg) {
  return reinterpret_cast<uint64_t*>(tc_stage_ring(smem, stage_total, ln) + (size_t)(stg > 0 ? stg : 0) * TC_STG_UNIT +
                                     2 * TC_BM * sizeof(float*));
}

template <int PREC>
__global__ void __launch_bounds__(TC_THREADS, 1)
    k_gemm_tc(GemmArgs g, TcWeights w, int stages, int stg, const __grid_constant__ CUtensorMap tmA, int a_tma,
              const __grid_constant__ CUtensorMap tmA2, int a2_kb0, int a2_x0) {
  constexpr int EPC = (PREC == TG_PREC_BF16 || PREC == TG_PREC_F16X3) ? 64 : 32;
  constexpr int PLANES = (PREC == TG_PREC_TF32X3 || PREC == TG_PREC_F16X3) ? 2 : 1;
  // fp32-level modes: the converted A operand goes to tensor memory (32 columns per plane and
  // k-block: tf32 one element, f16 two per column), shared-memory stages hold only B
  constexpr bool ATMEM = PLANES == 2;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // 1024-byte alignment (128B swizzle atoms) by an integer offset from smem_raw, so
  // the compiler keeps the shared address space (LDS/STS, not generic LD/ST)
  unsigned char* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const int BN = w.BN;
  // TMEM accumulators (512 columns allocated). tf32x3: each buffer holds [big | small]
  // (BNc = round32(BN) columns each): ah.bh accumulates into `big`, the correction terms
  // ah.bl + al.bh into `small`, summed in fp32 by the epilogue -- the tensor core's fp32
  // accumulation truncates at every MMA (error ~ steps x ulp(|acc|)), so keeping the
  // 2K/8 correction MMAs out of the large accumulator cuts that error 3x. Double-buffered
  // when 4 BNc <= 512, else one buffer. Other modes: two 256-column buffers.
  const int BNc = (BN + 31) & ~31;
  const uint32_t buf_cols = PLANES == 2 ? 2u * BNc : (uint32_t)tc_acc_cols(PREC);
  const uint32_t small_off = PLANES == 2 ? (uint32_t)BNc : 0u;
  const uint32_t nbuf = ATMEM ? (uint32_t)tc_tmem_nbuf(BN) : (4 * BNc > 512 ? 1u : 2u);
  const uint32_t a_plane = TC_BM * 128;
  const uint32_t b_plane = (uint32_t)BN * (ATMEM ? 64 : 128);
  const uint32_t a_bytes = ATMEM ? 0u : PLANES * a_plane;  // A bytes at the head of a smem stage
  const uint32_t stage_bytes = a_bytes + PLANES * b_plane;
  // ATMEM: A stage s at TMEM columns a_tcol0 + 32 s: [hi 16 | lo 16] per 64-byte k-block
  const uint32_t a_tcol0 = nbuf * buf_cols;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * stage_bytes);
  uint64_t* empty = full + TC_MAXSTAGES;
  uint64_t* tfull = empty + TC_MAXSTAGES;   // [2]
  uint64_t* tempty = tfull + 2;             // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint64_t* lnbar = tempty + 3;             // [2] LayerNorm statistics exchange (g.ln)
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
#ifdef TG_TC_TRACE
  const long long t_entry = clock64();
#endif
#ifdef TG_TC_TRACE
  // only full-grid launches are traced (a later partial launch would leave stale stamps)
  const int Mtr = *g.m_dev;  // debug build only: read before the PDL wait
  const bool tct_on = tg_tct_nk[0] == g.N && tg_tct_nk[1] == g.K && ((Mtr + TC_BM - 1) / TC_BM) * w.ntn >= (int)gridDim.x;
  if (tid == 0) {
    long long gt;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
    TCT(0, t_entry);
    TCT(1, gt);
    TCT(63, Mtr);
  }
#endif
  const int nkb = w.nkb;
  // the generic fp32 A producer (all TC_PROD_WARPS warps) unless A arrives by TMA, streams raw
  // (one-pass tf32) or as a dense bf16 activation (128 threads, warps 0-3)
  // a_tma == 2 (fp32-level modes, dense fp32 A): the producers' staging ring is filled by TMA
  // 2D tile loads (box 32 fp32 x 128 rows, 128B swizzle = the ring's layout) instead of
  // per-thread cp.async copies
  const bool stage_tma = ATMEM && a_tma == 2;
  const bool generic = (!a_tma || stage_tma) && PREC != TG_PREC_TF32 && !(PREC == TG_PREC_BF16 && g.a_h);
  if (tid == 0) {
    for (int s = 0; s < stages; ++s) {
      // arrivals: the A producer threads (256 generic, 128 streamed) + the TMA warp's expect_tx
      // (ATMEM tf32x3: each 64-byte k-block is produced by one half of the producers)
      mbar_init(&full[s], (a_tma && !stage_tma) ? 1 : ((generic && !(ATMEM && PREC == TG_PREC_TF32X3)) ? TC_PROD_WARPS * 32 : TC_BM) + 1);
      mbar_init(&empty[s], 1);         // MMA commit
    }
    if (stage_tma) {  // staging ring (ATMEM, dense A by TMA): landed (tx) / read by the 8 producer warps
      uint64_t* sb = tc_stage_bars(smem, stages * stage_bytes, g.ln, stg);
      for (int i = 0; i < stg; ++i) {
        mbar_init(&sb[i], 1);
        mbar_init(&sb[4 + i], TC_PROD_WARPS);
      }
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tfull[a], 1);     // MMA commit after the tile's last k-block
      mbar_init(&tempty[a], TC_EPI_WARPS * 32);  // epilogue threads drained the accumulator
      if (g.ln) mbar_init(&lnbar[a], w.ntn * TC_BM);  // one arrival per row from each CTA of the cluster
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                 "r"(2 * tc_acc_cols(PREC)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n");
  if (g.ln) {  // peers arrive on this CTA's lnbar: initialised cluster-wide first
    asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
    asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
  }
  const uint32_t tmem = *tmem_slot;
  // Everything above touches only shared memory / TMEM / parameters: with programmatic
  // dependent launch it overlaps the previous kernel's tail. The row count is its output.
  pdl_enter();
  const int M = *g.m_dev;
  const int tiles_m = (M + TC_BM - 1) / TC_BM;
  const int ntiles = tiles_m * w.ntn;  // CTAs past ntiles run no tile and fall through to the end
  if (tid == 0) TCT(2, clock64());

  if (warp < TC_PROD_WARPS && ((a_tma && !stage_tma) || (!generic && warp >= 4))) {
    // A arrives by TMA (issued by warp 4 with B): nothing to produce here
  } else if (warp < TC_PROD_WARPS && PREC == TG_PREC_TF32) {
    // ===================== A producers, streamed: raw fp32 rows go straight into
    // the swizzled operand with 16-byte cp.async (zero-fill past K / M); the
    // tensor core reads them as tf32. Completion is tracked by the full barrier
    // (cp.async.mbarrier.arrive.noinc), so `stages` k-blocks are in flight.
    uint32_t gk = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const int tm = t / w.ntn;
      const int row = tm * TC_BM + tid;
      const bool rv = row < M;
      const float* r0 = g.a_base0;  // any valid address for zero-fill copies
      const float* r1 = g.a_base0;
      if (rv) {
        r0 = g.a_rows0 ? g.a_rows0[row] : g.a_base0 + (size_t)row * g.lda0;
        if (g.K0 < g.K) r1 = g.a_rows1 ? g.a_rows1[row] : g.a_base1 + (size_t)row * g.lda1;
      } else if (g.a_rows0) {
        r0 = r1 = g.a_rows0[0];
      }
      for (int kb = 0; kb < nkb; ++kb, ++gk) {
        const int s = gk % stages;
        mbar_wait(&empty[s], ((gk / stages) & 1) ^ 1);
        const uint32_t sA = smem_u32(smem + s * stage_bytes);
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const int col = kb * EPC + c * 4;
          const bool ok = rv && col < g.K;
          const float* src = !ok ? r0 : (col < g.K0 ? r0 + col : r1 + (col - g.K0));
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sA + sw128(tid, c)), "l"(src),
                       "r"(ok ? 16 : 0)
                       : "memory");
        }
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(&full[s])) : "memory");
      }
    }
  } else if (warp < TC_PROD_WARPS && PREC == TG_PREC_BF16 && g.a_h) {
    // ===================== A producers, streamed bf16: the activation was
    // written in bf16 by the producing kernel (attention, LayerNorm, FFN1), so
    // its rows go straight into the swizzled operand (64 elements = 128 B per
    // k-block row) with cp.async; `stages` k-blocks are in flight.
    uint32_t gk = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const int tm = t / w.ntn;
      const int row = tm * TC_BM + tid;
      const bool rv = row < M;
      const unsigned short* ar = g.a_h + (size_t)(rv ? row : 0) * g.lda_h;
      for (int kb = 0; kb < nkb; ++kb, ++gk) {
        const int s = gk % stages;
        mbar_wait(&empty[s], ((gk / stages) & 1) ^ 1);
        const uint32_t sA = smem_u32(smem + s * stage_bytes);
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const int col = kb * EPC + c * 8;
          const bool ok = rv && col < g.lda_h;  // [K, lda_h) is zero padding
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sA + sw128(tid, c)),
                       "l"(ok ? ar + col : ar), "r"(ok ? 16 : 0)
                       : "memory");
        }
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(&full[s])) : "memory");
      }
    }
  } else if (warp < TC_PROD_WARPS) {
    // ===================== A producers (fp32 rows: gathered through row pointers or dense),
    // converted on the fly by the 256 threads of warps 0-7: thread p converts half the
    // columns (fp32 chunks 4 (p / 128) .. + 3 of each 32-float unit) of row p % 128. Loads
    // run ahead through a cp.async staging ring of `stg` units (a unit = 32 fp32 = 128 B of
    // each of the tile's 128 rows, 16 KB; UPK units per k-block), up to 64 KB per CTA in
    // flight without holding registers; the copies are coalesced (each warp instruction
    // moves 8 rows x 64 contiguous bytes). Named barrier 2 (the 256 producer threads) orders
    // the copies and the reads of a slot. The producers are instruction-latency bound (one
    // converting warp per scheduler measured ~1.2 us per 16 KB unit), hence 8 warps.
    constexpr int UPK = EPC / 32;
    constexpr int NPT = TC_PROD_WARPS * 32;
    const int prow = tid & (TC_BM - 1), ph = tid >> 7;  // row, column half
    // staging ring at a 1024-byte boundary: TMA's 128-byte swizzle is a function of the address
    unsigned char* sring = tc_stage_ring(smem, stages * stage_bytes, g.ln);
    const float** sptr = reinterpret_cast<const float**>(sring + (size_t)(stg > 0 ? stg : 0) * TC_STG_UNIT);  // [2][128]
    uint64_t* sbar = reinterpret_cast<uint64_t*>(sptr + 2 * TC_BM);  // [4] staging slots landed (stage_tma)
    uint64_t* sempty = sbar + 4;  // [4] staging slots read by every producer warp (stage_tma)
    // stg < 0: no staging ring -- each thread prefetches its own row half two units ahead
    // in registers (no shared-memory round trip, no producer barriers)
    const bool regpf = stg < 0;
    const int D = regpf ? 0 : stg;
    // units (32 fp32 of each row) per tile; ATMEM k-blocks are 64 B (tf32 16, f16 32 elements)
    constexpr int EPK = PREC == TG_PREC_F16X3 ? 32 : 16;
    const int upt = ATMEM ? (nkb * EPK + 31) / 32 : nkb * UPK;
    auto pbar = [] { asm volatile("bar.sync 2, %0;\n" ::"n"(NPT) : "memory"); };
    float4 pf0[4], pf1[4];
    int pt = blockIdx.x, pu = 0;
    const float* pr0 = nullptr;
    const float* pr1 = nullptr;
    bool prv = false;
    auto prow_of = [&](int tt) {
      const int row = (tt / w.ntn) * TC_BM + prow;
      prv = tt < ntiles && row < M;
      pr0 = pr1 = nullptr;
      if (prv) {
        pr0 = g.a_rows0 ? g.a_rows0[row] : g.a_base0 + (size_t)row * g.lda0;
        if (g.K0 < g.K) pr1 = g.a_rows1 ? g.a_rows1[row] : g.a_base1 + (size_t)row * g.lda1;
      }
    };
    auto fetch = [&](float4 (&d)[4]) {
      if (pt < ntiles) {
#pragma unroll
        for (int i = 0; i < 4; ++i)
          d[i] = prv ? tc_ldg4(g, pr0, pr1, pu * 32 + 4 * (4 * ph + i)) : make_float4(0.f, 0.f, 0.f, 0.f);
        if (++pu == upt) {
          pu = 0;
          pt += gridDim.x;
          prow_of(pt);
        }
      }
    };
    if (regpf) {
      prow_of(pt);
      fetch(pf0);
      fetch(pf1);
    }
    // issue cursor: tile it_t (this CTA's sequence), unit it_u within the tile
    int it_t = blockIdx.x, it_u = 0;
    const float* ir0 = nullptr;
    const float* ir1 = nullptr;
    bool irv = false;
    auto rows_of = [&](int tt) {
      const int row = (tt / w.ntn) * TC_BM + prow;
      irv = tt < ntiles && row < M;
      ir0 = ir1 = nullptr;
      if (irv) {
        ir0 = g.a_rows0 ? g.a_rows0[row] : g.a_base0 + (size_t)row * g.lda0;
        if (g.K0 < g.K) ir1 = g.a_rows1 ? g.a_rows1[row] : g.a_base1 + (size_t)row * g.lda1;
      }
    };
    auto publish = [&](int tt) {  // the tile's row pointers -> shared table (threads 0..127)
      if (ph == 0) rows_of(tt);
      pbar();                     // every thread is done issuing from the previous table
      if (ph == 0) {
        sptr[prow] = irv ? ir0 : nullptr;
        sptr[TC_BM + prow] = ir1;
      }
      pbar();
    };
    const void* dummy = w.hi;  // valid global address for zero-byte (zero-fill) copies
    auto issue = [&](int slot) {
      if (stage_tma) {  // one thread: TMA tile (32 fp32 x 128 rows) of dense A into the slot
        if (it_t < ntiles) {
          if (tid == 0) {
            // the producers' generic reads of this slot (ordered by named barrier 2) before the
            // async-proxy (TMA) write that refills it
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            const uint32_t bar = smem_u32(&sbar[slot]);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(TC_STG_UNIT)
                         : "memory");
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
                "[%4];\n" ::"r"(smem_u32(sring + (size_t)slot * TC_STG_UNIT)),
                "l"(reinterpret_cast<uint64_t>(&tmA)), "r"(it_u * 32), "r"((it_t / w.ntn) * TC_BM), "r"(bar)
                : "memory");
          }
          if (++it_u == upt) {
            it_u = 0;
            it_t += gridDim.x;
          }
        }
        return;
      }
      if (it_t < ntiles) {
        unsigned char* base = sring + (size_t)slot * TC_STG_UNIT;
        const int q = lane & 3;
#pragma unroll
        for (int it = 0; it < TC_BM / (TC_PROD_WARPS * 8); ++it) {
          const int r = warp * (TC_BM / TC_PROD_WARPS) + it * 8 + (lane >> 2);
          const float* p0 = sptr[r];
          const float* p1 = sptr[TC_BM + r];
#pragma unroll
          for (int hh = 0; hh < 2; ++hh) {
            const int c = q + 4 * hh;
            const int col = it_u * 32 + 4 * c;
            const bool ok = p0 && col < g.K;
            const void* src = !ok ? dummy : (const void*)(col < g.K0 ? p0 + col : p1 + (col - g.K0));
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(
                             smem_u32(base + r * 128 + ((c ^ (r & 7)) << 4))),
                         "l"(src), "r"(ok ? 16 : 0)
                         : "memory");
          }
        }
        if (++it_u == upt) {
          it_u = 0;
          it_t += gridDim.x;
          if (it_t < ntiles) publish(it_t);
        }
      }
      asm volatile("cp.async.commit_group;\n" ::: "memory");  // (empty past the last tile)
    };
    if (stage_tma) {
      // the staging warp (TC_STG_WARP) fills the ring; its barriers were initialised with the others
    } else if (D > 0) {  // (regpf: D = 0)
      if (it_t < ntiles) publish(it_t);
      for (int i = 0; i < D; ++i) issue(i);
    }
    uint32_t gk = 0, gu = 0;
    if (ATMEM) {
      // unit u of a tile feeds k-blocks 2u (thread half 0) and 2u + 1 (half 1) in tf32x3 --
      // the two halves fill different stages concurrently -- or k-block u (both halves,
      // 8 TMEM columns each) in f16x3
      const uint32_t lanes = (uint32_t)((warp & 3) * 32) << 16;
      int tseq = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++tseq) {
        if (D == 0) rows_of(t);
        for (int u = 0; u < upt; ++u, ++gu) {
#ifdef TG_TC_TRACE
          const bool tr5 = tg_tct_nk[2] == 5 && tseq == 0 && tid == 0 && u < 8;
#define TR5(i) do { if (tr5) TCT(8 + 6 * u + (i), clock64()); } while (0)
#else
#define TR5(i) do { } while (0)
#endif
          TR5(0);
          float4 x[4];  // fp32 chunks 4 ph .. 4 ph + 3 of unit u of row prow
          const int slot = D > 0 ? (int)(gu % (uint32_t)D) : 0;
          if (D <= 0) {
#pragma unroll
            for (int i = 0; i < 4; ++i)
              x[i] = irv ? tc_load4(g, ir0, ir1, u * 32 + 4 * (4 * ph + i)) : make_float4(0.f, 0.f, 0.f, 0.f);
          } else {
            if (stage_tma) {
              mbar_wait(&sbar[slot], (gu / (uint32_t)D) & 1);  // the unit's TMA tile has landed
              TR5(1);
              const unsigned char* src = sring + (size_t)slot * TC_STG_UNIT + prow * 128;
#pragma unroll
              for (int i = 0; i < 4; ++i)
                x[i] = *reinterpret_cast<const float4*>(src + (((4 * ph + i) ^ (prow & 7)) << 4));
              __syncwarp();
              if (lane == 0) mbar_arrive(&sempty[slot]);  // this warp is done with the slot
              TR5(2);
            } else {
              if (D == 1) asm volatile("cp.async.wait_group 0;\n" ::: "memory");
              else if (D == 2) asm volatile("cp.async.wait_group 1;\n" ::: "memory");
              else if (D == 3) asm volatile("cp.async.wait_group 2;\n" ::: "memory");
              else asm volatile("cp.async.wait_group 3;\n" ::: "memory");
              pbar();  // every producer's copies of this unit have landed
              TR5(1);
              const unsigned char* src = sring + (size_t)slot * TC_STG_UNIT + prow * 128;
#pragma unroll
              for (int i = 0; i < 4; ++i)
                x[i] = *reinterpret_cast<const float4*>(src + (((4 * ph + i) ^ (prow & 7)) << 4));
              pbar();  // every producer has read the slot: it may be refilled
              TR5(2);
              issue(slot);  // unit gu + D
            }
          }
          const int kbq = EPK == 16 ? 2 * u + ph : u;
          if (kbq >= nkb) continue;
          const uint32_t g2 = (uint32_t)tseq * (uint32_t)nkb + (uint32_t)kbq;
          const int s = (int)(g2 % (uint32_t)stages);
          TR5(3);
          mbar_wait(&empty[s], ((g2 / (uint32_t)stages) & 1) ^ 1);
          asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
          TR5(4);
          const uint32_t tq = tmem + lanes + a_tcol0 + 32u * (uint32_t)s;
          if (PREC == TG_PREC_F16X3) {
            uint32_t hv[8], lv[8];
            bool big = false;
#pragma unroll
            for (int e = 0; e < 8; ++e) {
              const float x0 = (&x[e >> 1].x)[2 * (e & 1)], x1 = (&x[e >> 1].x)[2 * (e & 1) + 1];
              const __half2 hh = __floats2half2_rn(x0, x1);
              const float2 hf = __half22float2(hh);
              const __half2 ll = __floats2half2_rn(x0 - hf.x, x1 - hf.y);
              big |= !(fabsf(x0) < 65504.f) | !(fabsf(x1) < 65504.f);
              hv[e] = *reinterpret_cast<const uint32_t*>(&hh);
              lv[e] = *reinterpret_cast<const uint32_t*>(&ll);
            }
            if (big && g.err) atomicOr(g.err, kErrF16Range);
            tmem_st8(tq + 8u * (uint32_t)ph, hv);
            tmem_st8(tq + 16u + 8u * (uint32_t)ph, lv);
          } else {
            uint32_t hv[16], lv[16];
#pragma unroll
            for (int e = 0; e < 16; ++e) {
              const float xv = (&x[e >> 2].x)[e & 3];
              const float hi = rna_tf32_fast(xv);
              hv[e] = __float_as_uint(hi);
              lv[e] = __float_as_uint(rna_tf32_fast(xv - hi));
            }
            tmem_st16(tq, hv);
            tmem_st16(tq + 16u, lv);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
          asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
          TR5(5);
          mbar_arrive(&full[s]);
        }
#undef TR5
      }
    }
    for (int t = blockIdx.x; t < (ATMEM ? 0 : ntiles); t += gridDim.x) {
      if (D == 0 && !regpf) rows_of(t);  // no room for staging (widest N tiles): blocking loads
      for (int kb = 0; kb < nkb; ++kb, ++gk) {
        const int s = gk % stages;
        mbar_wait(&empty[s], ((gk / stages) & 1) ^ 1);
#ifdef TG_TC_TRACE
        if (t == (int)blockIdx.x && tid == 0 && tg_tct_nk[2] == 1) TCT(8 + kb, clock64());
        if (t == (int)blockIdx.x && tid == 0 && tg_tct_nk[2] == 3 && kb < 16) TCT(24 + kb, clock64());
#endif
        unsigned char* sA = smem + s * stage_bytes;
        bool big = false;
#ifdef TG_TC_TRACE
        if (tg_tct_nk[2] == 4) {  // debug: MMA/TMA-bound cadence (producer does no work; results invalid)
          mbar_arrive(&full[s]);
          continue;
        }
#endif
#pragma unroll
        for (int h = 0; h < UPK; ++h, ++gu) {
          float4 x[4];  // fp32 chunks 4 ph .. 4 ph + 3 of this unit of row prow
          const int slot = D > 0 ? (int)(gu % (uint32_t)D) : 0;
          if (regpf) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              x[i] = pf0[i];
              pf0[i] = pf1[i];
            }
            fetch(pf1);  // unit gu + 2
          } else if (D == 0) {
#pragma unroll
            for (int i = 0; i < 4; ++i)
              x[i] = irv ? tc_load4(g, ir0, ir1, (kb * UPK + h) * 32 + 4 * (4 * ph + i))
                         : make_float4(0.f, 0.f, 0.f, 0.f);
          } else {
            if (D == 1) asm volatile("cp.async.wait_group 0;\n" ::: "memory");
            else if (D == 2) asm volatile("cp.async.wait_group 1;\n" ::: "memory");
            else if (D == 3) asm volatile("cp.async.wait_group 2;\n" ::: "memory");
            else asm volatile("cp.async.wait_group 3;\n" ::: "memory");
            pbar();  // every producer's copies of this unit have landed
            const unsigned char* src = sring + (size_t)slot * TC_STG_UNIT + prow * 128;
#pragma unroll
            for (int i = 0; i < 4; ++i)
              x[i] = *reinterpret_cast<const float4*>(src + (((4 * ph + i) ^ (prow & 7)) << 4));
            pbar();  // every producer has read the slot: it may be refilled
            issue(slot);  // unit gu + D
          }
          if (PREC == TG_PREC_F16X3) {
#pragma unroll
            for (int jj = 0; jj < 2; ++jj) {  // fp16 chunk j = 2 ph + jj <- fp32 chunks 2j, 2j + 1
              const float xs[8] = {x[2 * jj].x, x[2 * jj].y, x[2 * jj].z, x[2 * jj].w,
                                   x[2 * jj + 1].x, x[2 * jj + 1].y, x[2 * jj + 1].z, x[2 * jj + 1].w};
              uint32_t hv[4], lv[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const __half2 hh = __floats2half2_rn(xs[2 * e], xs[2 * e + 1]);
                const float2 hf = __half22float2(hh);
                const __half2 ll = __floats2half2_rn(xs[2 * e] - hf.x, xs[2 * e + 1] - hf.y);
                big |= !(fabsf(xs[2 * e]) < 65504.f) | !(fabsf(xs[2 * e + 1]) < 65504.f);
                hv[e] = *reinterpret_cast<const uint32_t*>(&hh);
                lv[e] = *reinterpret_cast<const uint32_t*>(&ll);
              }
              const int c = h * 4 + 2 * ph + jj;
              *reinterpret_cast<uint4*>(sA + sw128(prow, c)) = make_uint4(hv[0], hv[1], hv[2], hv[3]);
              *reinterpret_cast<uint4*>(sA + a_plane + sw128(prow, c)) = make_uint4(lv[0], lv[1], lv[2], lv[3]);
            }
          } else if (PREC == TG_PREC_BF16) {
#pragma unroll
            for (int jj = 0; jj < 2; ++jj) {
              const float4 x0 = x[2 * jj], x1 = x[2 * jj + 1];
              __nv_bfloat162 p0 = __floats2bfloat162_rn(x0.x, x0.y), p1 = __floats2bfloat162_rn(x0.z, x0.w);
              __nv_bfloat162 p2 = __floats2bfloat162_rn(x1.x, x1.y), p3 = __floats2bfloat162_rn(x1.z, x1.w);
              uint4 u;
              u.x = *reinterpret_cast<uint32_t*>(&p0);
              u.y = *reinterpret_cast<uint32_t*>(&p1);
              u.z = *reinterpret_cast<uint32_t*>(&p2);
              u.w = *reinterpret_cast<uint32_t*>(&p3);
              *reinterpret_cast<uint4*>(sA + sw128(prow, h * 4 + 2 * ph + jj)) = u;
            }
          } else {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const int c = 4 * ph + i;
              const float4 xv = x[i];
              float4 hi, lo;
              hi.x = rna_tf32_fast(xv.x);
              hi.y = rna_tf32_fast(xv.y);
              hi.z = rna_tf32_fast(xv.z);
              hi.w = rna_tf32_fast(xv.w);
              *reinterpret_cast<float4*>(sA + sw128(prow, c)) = hi;
              if (PLANES == 2) {
                lo.x = rna_tf32_fast(xv.x - hi.x);
                lo.y = rna_tf32_fast(xv.y - hi.y);
                lo.z = rna_tf32_fast(xv.z - hi.z);
                lo.w = rna_tf32_fast(xv.w - hi.w);
                *reinterpret_cast<float4*>(sA + a_plane + sw128(prow, c)) = lo;
              }
            }
          }
        }
        if (PREC == TG_PREC_F16X3 && big && g.err) atomicOr(g.err, kErrF16Range);
        asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");  // generic -> async proxy
#ifdef TG_TC_TRACE
        if (t == (int)blockIdx.x && tid == 0 && tg_tct_nk[2] == 2) TCT(8 + kb, clock64());
        if (t == (int)blockIdx.x && tid == 0 && tg_tct_nk[2] == 3 && kb < 16) TCT(40 + kb, clock64());
#endif
        mbar_arrive(&full[s]);
      }
    }
    asm volatile("cp.async.wait_group 0;\n" ::: "memory");
  } else if (warp == TC_TMA_WARP) {
    // ===================== B producer (TMA bulk copies of weight tile images)
    if (lane == 0) {
      uint32_t gk = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int tn = t % w.ntn;
        for (int kb = 0; kb < nkb; ++kb, ++gk) {
          const int s = gk % stages;
          mbar_wait(&empty[s], ((gk / stages) & 1) ^ 1);
          unsigned char* sB = smem + s * stage_bytes + a_bytes;
          const unsigned char* src =
              reinterpret_cast<const unsigned char*>(w.hi) + ((size_t)tn * nkb + kb) * PLANES * b_plane;
          if (gk == 0) TCT(4, clock64());
          mbar_expect_tx(&full[s], PLANES * b_plane + ((a_tma && !stage_tma) ? a_plane : 0u));
          if (a_tma && !stage_tma) {  // A tile [128 rows x 128 B] of the dense activation, 128B-swizzled by TMA
            // k-blocks >= a2_kb0 come from a second activation (columns a2_x0 + ...)
            const bool second = kb >= a2_kb0;
            const int x = second ? a2_x0 + (kb - a2_kb0) * EPC : kb * EPC, y = (t / w.ntn) * TC_BM;
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
                "[%4];\n" ::"r"(smem_u32(smem + s * stage_bytes)),
                "l"(reinterpret_cast<uint64_t>(second ? &tmA2 : &tmA)), "r"(x), "r"(y), "r"(smem_u32(&full[s]))
                : "memory");
          }
          bulk_g2s(sB, src, PLANES * b_plane, &full[s]);
        }
      }
    }
  } else if (warp == TC_MMA_WARP) {
    // ===================== MMA issuer
    if (lane == 0) {
      const uint32_t idesc = umma_idesc(PREC, BN);
      uint32_t gk = 0, tc = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++tc) {
        const uint32_t acc = tc % nbuf;
        mbar_wait(&tempty[acc], ((tc / nbuf) & 1) ^ 1);  // epilogue drained this accumulator
        asm volatile("tcgen05.fence::after_thread_sync;\n");
        const uint32_t dtm = tmem + acc * buf_cols;
        for (int kb = 0; kb < nkb; ++kb, ++gk) {
          const int s = gk % stages;
          mbar_wait(&full[s], (gk / stages) & 1);
#ifdef TG_TC_TRACE
          if (tc == 0 && (tg_tct_nk[2] == 0 || tg_tct_nk[2] == 4)) TCT(8 + kb, clock64());
          if (tc == 0 && tg_tct_nk[2] == 3 && kb < 16) TCT(8 + kb, clock64());
#endif
          asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");  // cp.async A -> tensor core
          asm volatile("tcgen05.fence::after_thread_sync;\n");
          const uint32_t aH = smem_u32(smem + s * stage_bytes);
          const uint32_t bH = aH + a_bytes;
          const uint32_t aT = tmem + a_tcol0 + 32u * (uint32_t)s;  // ATMEM: A planes at aT, aT + 16
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {  // 4 MMAs of 32 bytes of K per 128B k-block
            const uint32_t acc0 = (kb > 0 || kk > 0) ? 1u : 0u;
            if (ATMEM) {  // 64-byte k-block: 2 MMAs of 32 bytes of K, 8 TMEM columns of A each;
              // B 64B-swizzled; correction products into `small`
              if (kk < 2) {
                mma_issue_ts<PREC>(dtm, aT + kk * 8, umma_desc64(bH + kk * 32), idesc, acc0);
                mma_issue_ts<PREC>(dtm + small_off, aT + kk * 8, umma_desc64(bH + b_plane + kk * 32), idesc, acc0);
                mma_issue_ts<PREC>(dtm + small_off, aT + 16 + kk * 8, umma_desc64(bH + kk * 32), idesc, 1u);
              }
              continue;
            }
            mma_issue<PREC>(dtm, umma_desc(aH + kk * 32), umma_desc(bH + kk * 32), idesc, acc0);
            if (PLANES == 2) {
              mma_issue<PREC>(dtm + small_off, umma_desc(aH + kk * 32), umma_desc(bH + b_plane + kk * 32), idesc,
                              acc0);
              mma_issue<PREC>(dtm + small_off, umma_desc(aH + a_plane + kk * 32), umma_desc(bH + kk * 32), idesc,
                              1u);
            }
          }
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                           smem_u32(&empty[s]))
                       : "memory");
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                         smem_u32(&tfull[acc]))
                     : "memory");
        if (tc == 0) TCT(3, clock64());
      }
    }
  } else if (warp == TC_STG_WARP) {
    // ===================== staging warp (stage_tma): TMA 2D tiles (32 fp32 x 128 rows) of the
    // dense fp32 A into the producers' ring, `stg` units ahead; a slot is refilled once all 8
    // producer warps have read it (sempty), so no producer waits on the refill
    if (stage_tma && lane == 0) {
      unsigned char* sring = tc_stage_ring(smem, stages * stage_bytes, g.ln);
      uint64_t* sbar = tc_stage_bars(smem, stages * stage_bytes, g.ln, stg);
      uint64_t* sempty = sbar + 4;
      constexpr int EPK = PREC == TG_PREC_F16X3 ? 32 : 16;
      const int upt = (nkb * EPK + 31) / 32;
      uint32_t q = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int y = (t / w.ntn) * TC_BM;
        for (int u = 0; u < upt; ++u, ++q) {
          const uint32_t slot = q % (uint32_t)stg;
          if (q >= (uint32_t)stg) mbar_wait(&sempty[slot], ((q / (uint32_t)stg) - 1u) & 1u);
          // the producers' generic reads of the slot before the async-proxy write that refills it
          asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
          const uint32_t bar = smem_u32(&sbar[slot]);
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(TC_STG_UNIT)
                       : "memory");
          asm volatile(
              "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
              "[%4];\n" ::"r"(smem_u32(sring + (size_t)slot * TC_STG_UNIT)),
              "l"(reinterpret_cast<uint64_t>(&tmA)), "r"(u * 32), "r"(y), "r"(bar)
              : "memory");
        }
      }
    }
  } else if (g.ln) {
    // ===================== epilogue with the fused LayerNorm (G2, Eq. 6: r = LN(W_fc o +
    // b_fc + q), R1; the residual q = [h | 0 | Phi(0)] is already in the accumulator: h
    // through the identity block of the augmented K, Phi(0) folded into the bias). The ntn
    // CTAs of a cluster hold the ntn column tiles of the same 128 rows. Pass 1 reads the
    // accumulator and reduces each row's (count, mean, M2) over its valid columns; the
    // CTA's row statistics go to every CTA of the cluster through DSMEM (remote mbarrier
    // arrive); pass 2 re-reads the accumulator, normalises with the merged statistics
    // (fixed tile order) and stores the bf16 LN(y) block of the merge-FFN input (Eq. 7).
    const int quad = warp & 3;
    const int ew = warp - TC_EPI_WARP0;
    const int half = ew >> 2;
    float* stg = reinterpret_cast<float*>(smem + stages * stage_bytes + TC_BAR_BYTES) + ew * (32 * TC_STG_LD);
    float4* lnh = reinterpret_cast<float4*>(smem + stages * stage_bytes + TC_BAR_BYTES + TC_EPI_BYTES);  // [2][128]
    float4* lnx = lnh + 2 * TC_BM;  // [2][TC_LN_MAXTN][128]
    float* s_bias = reinterpret_cast<float*>(lnx + 2 * TC_LN_MAXTN * TC_BM);  // [BN] x 3
    float* s_g = s_bias + 256;
    float* s_b = s_g + 256;
    float* s_w = s_b + 256;  // 1 for the valid LayerNorm columns of the tile, else 0 (gamma = beta = 0 there)
    const int rq = lane >> 2, cq = lane & 3;
    const int rloc = quad * 32 + lane;
    const int ntn = w.ntn;
    {  // this CTA's column tile is fixed (grid is a multiple of ntn)
      const int nb0 = (int)(blockIdx.x % ntn) * BN;
      for (int i = tid - TC_EPI_WARP0 * 32; i < BN; i += TC_EPI_WARPS * 32) {
        const int c = nb0 + i;
        const bool in = c < g.N;
        s_bias[i] = in ? g.bias[c] : 0.f;
        s_g[i] = in ? g.ln_g[c] : 0.f;
        s_b[i] = in ? g.ln_b[c] : 0.f;
        s_w[i] = ln_valid(g, c) ? 1.f : 0.f;
      }
      asm volatile("bar.sync 1, %0;\n" ::"n"(TC_EPI_WARPS * 32) : "memory");
    }
    uint32_t tc = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++tc) {
      const int tm = t / ntn, tn = t - tm * ntn;
      const int m0 = tm * TC_BM, n0 = tn * BN;
      const uint32_t acc = tc % nbuf, par = tc & 1;
      const int er = m0 + rloc;
      unsigned short* hrow = er < M ? g.c_h + (size_t)er * g.ldc_h : nullptr;
      mbar_wait(&tfull[acc], (tc / nbuf) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;\n");
      const uint32_t tacc = tmem + acc * buf_cols + ((uint32_t)(quad * 32) << 16);
      // ---- pass 1: row statistics of this thread's column chunks
      float sn = 0.f, sm = 0.f, sM = 0.f;
      for (int c0 = 16 * half; c0 < BN; c0 += 16 * TC_EPI_HALVES) {
        uint32_t v[16];
        tmem_ld16(tacc + (uint32_t)c0, v);
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        float x[16];
        ln_chunk(v, s_bias, c0, x);
        float cs = 0.f, cn = 0.f;  // branch-free: weights s_w select the valid columns
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          cs = fmaf(s_w[c0 + j], x[j], cs);
          cn += s_w[c0 + j];
        }
        if (cn > 0.f) {
          const float cm = cs / cn;
          float cM = 0.f;
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            const float d = x[j] - cm;
            cM = fmaf(s_w[c0 + j] * d, d, cM);
          }
          chan_merge(sn, sm, sM, cn, cm, cM);
        }
      }
      lnh[half * TC_BM + rloc] = make_float4(sn, sm, sM, 0.f);
      asm volatile("bar.sync 1, %0;\n" ::"n"(TC_EPI_WARPS * 32) : "memory");
      if (half == 0) {
        if (TC_EPI_HALVES == 2) {
          const float4 o = lnh[TC_BM + rloc];
          chan_merge(sn, sm, sM, o.x, o.y, o.z);
        }
        const float4 st4 = make_float4(sn, sm, sM, 0.f);
        const uint32_t slot = smem_u32(lnx + (par * TC_LN_MAXTN + tn) * TC_BM + rloc);
        for (int r = 0; r < ntn; ++r) st_cluster_v4(mapa_u32(slot, (uint32_t)r), st4);
        const uint32_t bar = smem_u32(&lnbar[par]);
        for (int r = 0; r < ntn; ++r) mbar_arrive_remote(mapa_u32(bar, (uint32_t)r));
      }
      mbar_wait_cluster(&lnbar[par], (tc >> 1) & 1);
      float n = 0.f, mu = 0.f, M2 = 0.f;
      for (int r = 0; r < ntn; ++r) {
        const float4 o = lnx[(par * TC_LN_MAXTN + r) * TC_BM + rloc];
        chan_merge(n, mu, M2, o.x, o.y, o.z);
      }
      const float rstd = rsqrtf(M2 / fmaxf(n, 1.f) + 1e-5f);
      // ---- pass 2: normalise, transpose through shared memory, coalesced bf16 stores
      bool released = false;
      for (int c0 = 16 * half; c0 < BN; c0 += 16 * TC_EPI_HALVES) {
        uint32_t v[16];
        tmem_ld16(tacc + (uint32_t)c0, v);
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        if (c0 + 16 * TC_EPI_HALVES >= BN) {  // this warp's last chunk: hand the accumulator back
          asm volatile("tcgen05.fence::before_thread_sync;\n");
          mbar_arrive(&tempty[acc]);
          released = true;
        }
        float x[16];
        ln_chunk(v, s_bias, c0, x);
#pragma unroll
        for (int j = 0; j < 16; ++j)
          x[j] = fmaf((x[j] - mu) * rstd, s_g[c0 + j], s_b[c0 + j]);  // 0 where gamma = beta = 0
#pragma unroll
        for (int j = 0; j < 4; ++j)
          *reinterpret_cast<float4*>(stg + lane * TC_STG_LD + 4 * j) =
              make_float4(x[4 * j], x[4 * j + 1], x[4 * j + 2], x[4 * j + 3]);
        __syncwarp();
        const int c = n0 + c0 + 4 * cq;
        const bool cin = c0 + 4 * cq < BN && c < g.N;  // N % 4 == 0: all 4 or none
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int r = rq + 8 * i;
          const float4 y = *reinterpret_cast<const float4*>(stg + r * TC_STG_LD + 4 * cq);
          unsigned short* hr =
              reinterpret_cast<unsigned short*>(__shfl_sync(0xffffffffu, reinterpret_cast<long long>(hrow), r));
          if (hr && cin) {
            __nv_bfloat162 lo = __floats2bfloat162_rn(y.x, y.y), hi = __floats2bfloat162_rn(y.z, y.w);
            uint2 pk;
            pk.x = *reinterpret_cast<uint32_t*>(&lo);
            pk.y = *reinterpret_cast<uint32_t*>(&hi);
            *reinterpret_cast<uint2*>(hr + c) = pk;
          }
        }
        __syncwarp();
      }
      if (!released) {
        asm volatile("tcgen05.fence::before_thread_sync;\n");
        mbar_arrive(&tempty[acc]);
      }
    }
  } else {
    // ===================== epilogue: warps 6-13; warp w reads TMEM lane quadrant
    // w % 4 (rows 32*(w%4) ..), the two warps of a quadrant take alternate
    // 16-column chunks. tcgen05.ld leaves one row per thread, so each chunk is
    // transposed through a per-warp shared buffer (row stride 20 floats: 16B
    // aligned, conflict-free STS.128) and written back with lanes = 4 columns x
    // 8 rows: float4 bias/ReLU and 64-byte coalesced row segments.
    const int quad = warp & 3;
    const int ew = warp - TC_EPI_WARP0;    // 0 .. TC_EPI_WARPS - 1
    const int half = ew >> 2;              // which alternate chunk (with 8 epilogue warps)
    float* stg = reinterpret_cast<float*>(smem + stages * stage_bytes + TC_BAR_BYTES) + ew * (32 * TC_STG_LD);
    const int rq = lane >> 2, cq = lane & 3;  // read-back: row rq + 8i, float4 column cq
    // the tile's bias (and F16X3 column scales) staged in shared memory before its accumulator
    // is ready -- no global-load latency inside the chunk loop
    float* s_eb = reinterpret_cast<float*>(smem + stages * stage_bytes + TC_BAR_BYTES + TC_EPI_XPOSE_BYTES);
    const int etid = tid - TC_EPI_WARP0 * 32;
    uint32_t tc = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++tc) {
      const int tm = t / w.ntn, tn = t - tm * w.ntn;
      const int m0 = tm * TC_BM, n0 = tn * BN;
      const uint32_t acc = tc % nbuf;
      float* sb = s_eb + (tc & 1) * 512;  // [bias 256 | scale 256]; buffer tc & 1 was last read by tile tc - 2
      for (int i = etid; i < BN; i += TC_EPI_WARPS * 32) {
        const int c = n0 + i;
        sb[i] = (g.bias && c < g.N) ? g.bias[c] : 0.f;
        if (PREC == TG_PREC_F16X3) sb[256 + i] = w.colscale[c];
      }
      asm volatile("bar.sync 1, %0;\n" ::"n"(TC_EPI_WARPS * 32) : "memory");
      const int er = m0 + quad * 32 + lane;
      float* orow = nullptr;
      unsigned short* hrow = nullptr;
      if (er < M) {
        if (g.c_rows) orow = g.c_rows[er];
        else if (g.C) orow = g.C + (size_t)er * g.ldc;
        if (g.c_h) hrow = g.c_h + (size_t)er * g.ldc_h;
      }
      mbar_wait(&tfull[acc], (tc / nbuf) & 1);
      if (tc == 0 && warp == TC_EPI_WARP0 && lane == 0) TCT(5, clock64());
      asm volatile("tcgen05.fence::after_thread_sync;\n");
      bool released = false;
      for (int c0 = 16 * half; c0 < BN; c0 += 16 * TC_EPI_HALVES) {
        uint32_t v[16];
        const uint32_t tq = tmem + acc * buf_cols + ((uint32_t)(quad * 32) << 16) + (uint32_t)c0;
        tmem_ld16(tq, v);
        if (PLANES == 2) {  // + the correction accumulator (fp32 RN add)
          uint32_t vs[16];
          tmem_ld16(tq + small_off, vs);
          asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = __float_as_uint(__uint_as_float(v[j]) + __uint_as_float(vs[j]));
        } else {
          asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        }
        if (c0 + 16 * TC_EPI_HALVES >= BN) {  // this warp's last chunk: hand the accumulator back
          asm volatile("tcgen05.fence::before_thread_sync;\n");
          mbar_arrive(&tempty[acc]);
          released = true;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j)
          *reinterpret_cast<float4*>(stg + lane * TC_STG_LD + 4 * j) =
              make_float4(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]), __uint_as_float(v[4 * j + 2]),
                          __uint_as_float(v[4 * j + 3]));
        __syncwarp();
        const int cl = c0 + 4 * cq;  // first of this lane's 4 columns inside the tile
        const int c = n0 + cl;
        const bool cin = cl < BN && c < g.N;                    // N % 4 == 0: all 4 or none
        const bool cpad = cl < BN && c >= g.N && c < g.ldc_h;  // bf16 zero padding [N, ldc_h)
        float4 b4 = make_float4(0.f, 0.f, 0.f, 0.f);
        if (cl < BN) b4 = *reinterpret_cast<const float4*>(sb + cl);  // 0 past N
        float4 s4 = make_float4(1.f, 1.f, 1.f, 1.f);  // F16X3: undo the weight-row scale (exact)
        if (PREC == TG_PREC_F16X3 && cl < BN) s4 = *reinterpret_cast<const float4*>(sb + 256 + cl);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int r = rq + 8 * i;
          float4 x = *reinterpret_cast<const float4*>(stg + r * TC_STG_LD + 4 * cq);
          if (PREC == TG_PREC_F16X3) {
            x.x *= s4.x;
            x.y *= s4.y;
            x.z *= s4.z;
            x.w *= s4.w;
          }
          x.x += b4.x;
          x.y += b4.y;
          x.z += b4.z;
          x.w += b4.w;
          if (g.relu) {
            x.x = fmaxf(x.x, 0.f);
            x.y = fmaxf(x.y, 0.f);
            x.z = fmaxf(x.z, 0.f);
            x.w = fmaxf(x.w, 0.f);
          }
          float* orr = reinterpret_cast<float*>(__shfl_sync(0xffffffffu, reinterpret_cast<long long>(orow), r));
          if (orr && cin) *reinterpret_cast<float4*>(orr + c) = x;
          if (g.c_h) {
            unsigned short* hr =
                reinterpret_cast<unsigned short*>(__shfl_sync(0xffffffffu, reinterpret_cast<long long>(hrow), r));
            if (hr && (cin || cpad)) {
              if (!cin) x = make_float4(0.f, 0.f, 0.f, 0.f);
              __nv_bfloat162 lo = __floats2bfloat162_rn(x.x, x.y), hi = __floats2bfloat162_rn(x.z, x.w);
              uint2 pk;
              pk.x = *reinterpret_cast<uint32_t*>(&lo);
              pk.y = *reinterpret_cast<uint32_t*>(&hi);
              *reinterpret_cast<uint2*>(hr + c) = pk;
            }
          }
        }
        __syncwarp();
      }
      if (!released) {  // no chunk for this warp (BN <= 16)
        asm volatile("tcgen05.fence::before_thread_sync;\n");
        mbar_arrive(&tempty[acc]);
      }
      if (tc == 0 && warp == TC_EPI_WARP0 && lane == 0) TCT(6, clock64());
    }
  }
  if (lane == 0 && warp >= TC_TMA_WARP && warp <= TC_EPI_WARP0) TCT(60 + warp - TC_TMA_WARP, clock64());  // role done (before the barrier)
  asm volatile("tcgen05.fence::before_thread_sync;\n");
  __syncthreads();
  if (tid == 0) TCT(7, clock64());
  if (tid == TC_EPI_WARP0 * 32) TCT(55, clock64());
  asm volatile("tcgen05.fence::after_thread_sync;\n");
  if (g.ln) {  // no CTA leaves while a peer may still address its shared memory
    asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
    asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
  }
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(2 * tc_acc_cols(PREC)));
}

static size_t tc_smem(int prec, int BN, int stages, int stg, int ln = 0) {
  const size_t planes = tc_planes(prec);
  size_t s = 1024 + (size_t)stages * planes * ((tc_atmem(prec) ? 0 : (size_t)TC_BM * 128) + (size_t)BN * tc_kb_bytes(prec)) +
             TC_BAR_BYTES + TC_EPI_BYTES +
             (ln ? TC_LN_BYTES : 0) + (size_t)(stg > 0 ? stg : 0) * TC_STG_UNIT + (stg > 0 ? TC_PTR_BYTES + 1024 : 0);
  // tf32x3: one CTA per SM (it allocates all 512 TMEM columns; a second
  // co-resident CTA would block in tcgen05.alloc until the first one exits).
  const size_t one_per_sm = 120 * 1024;
  if (tc_ctas_per_sm(prec) == 1 && s < one_per_sm) return one_per_sm;
  return s;
}

tg_status tc_make_tensor_a(const void* base, int elem_bytes, int ld, int rows, TcTensorA* out) {
  out->valid = 0;
  if (!base || ld < 1 || rows < 1 || ((size_t)ld * elem_bytes) % 16) return TG_EINVAL;
  cuuint64_t dims[2] = {(cuuint64_t)ld, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * elem_bytes};
  cuuint32_t box[2] = {(cuuint32_t)(128 / elem_bytes), (cuuint32_t)TC_BM};
  cuuint32_t estr[2] = {1, 1};
  const CUtensorMapDataType dt = elem_bytes == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  // Resolved through the runtime so libtg.so does not link libcuda (absent on GPU-less build hosts).
  typedef CUresult (*encode_fn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  static encode_fn encode = nullptr;
  if (!encode) {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !fp)
      return TG_ECUDA;
    encode = (encode_fn)fp;
  }
  CUresult r = encode(&out->map, dt, 2, const_cast<void*>(base), dims, strides, box, estr,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return TG_ECUDA;
  out->valid = 1;
  return TG_OK;
}

void launch_gemm_tc(const GemmArgs& g, const TcWeights& w, int precision, cudaStream_t st, const TcTensorA* ta,
                    const TcTensorA* ta2, int a2_kb0, int a2_x0) {
  static const CUtensorMap zero_map{};
  const CUtensorMap& tm = (ta && ta->valid) ? ta->map : zero_map;
  int a_tma = (ta && ta->valid) ? 1 : 0;
  if (a_tma && tc_atmem(precision)) a_tma = 2;  // fp32-level modes: the map feeds the producers' staging ring
  const bool two = a_tma && ta2 && ta2->valid;
  const CUtensorMap& tm2 = two ? ta2->map : zero_map;
  if (!two) a2_kb0 = 1 << 30;
  const int ln = g.ln ? 1 : 0;
  // the generic fp32 A producer (cp.async staging) runs unless A comes by TMA, as raw fp32
  // (one-pass tf32) or as a dense bf16 activation
  const bool generic = (!a_tma || a_tma == 2) && precision != TG_PREC_TF32 && !(precision == TG_PREC_BF16 && g.a_h);
  int stages = 2, stg = 0;
  tc_plan(precision, w.BN, ln, generic, &stages, &stg);
  if (a_tma == 2 && stg <= 0) a_tma = 0;  // no staging ring: per-thread loads
  const size_t smem = tc_smem(precision, w.BN, stages, stg, ln);
  const int tiles = ((g.m_max + TC_BM - 1) / TC_BM) * w.ntn;
  static const int grid_cap = [] {  // TG_GEMM_GRID: cap on persistent CTAs (experiments)
    const char* e = getenv("TG_GEMM_GRID");
    return e ? atoi(e) : 148;
  }();
  int slots = grid_cap * tc_ctas_per_sm(precision);
  if (ln) slots = slots / w.ntn * w.ntn;  // whole clusters; a cluster walks the M tiles in lockstep
  int grid = tiles < slots ? tiles : slots;
  if (grid < 1) grid = 1;
  if (precision == TG_PREC_BF16) {
    static size_t set = 0;
    if (smem > set) {
      cudaFuncSetAttribute(k_gemm_tc<TG_PREC_BF16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      set = smem;
    }
    if (ln) {  // as many clusters as can be co-resident (GPC sizes), each walks M tiles
      static int max_cl = -1;
      static int max_cl_smem = -1;
      if (max_cl_smem != (int)smem) {
        cudaLaunchConfig_t oc = {};
        oc.gridDim = dim3(grid);
        oc.blockDim = dim3(TC_THREADS);
        oc.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = w.ntn;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        oc.attrs = at;
        oc.numAttrs = 1;
        int n = 0;
        if (cudaOccupancyMaxActiveClusters(&n, k_gemm_tc<TG_PREC_BF16>, &oc) != cudaSuccess) n = 0;
        cudaGetLastError();
        max_cl = n;
        max_cl_smem = (int)smem;
        if (getenv("TG_VERBOSE")) fprintf(stderr, "libtg: LN GEMM max active clusters of %d: %d (smem %zu)\n", w.ntn, n, smem);
      }
      if (max_cl > 0 && grid > max_cl * w.ntn) grid = max_cl * w.ntn;
    }
    if (ln)
      launch_k_cluster(k_gemm_tc<TG_PREC_BF16>, dim3(grid), dim3(TC_THREADS), smem, st, w.ntn, g, w, stages, stg, tm,
                       a_tma, tm2, a2_kb0, a2_x0);
    else
      launch_k(k_gemm_tc<TG_PREC_BF16>, dim3(grid), dim3(TC_THREADS), smem, st, g, w, stages, stg, tm, a_tma, tm2,
               a2_kb0, a2_x0);
  } else if (precision == TG_PREC_TF32) {
    static size_t set = 0;
    if (smem > set) {
      cudaFuncSetAttribute(k_gemm_tc<TG_PREC_TF32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      set = smem;
    }
    launch_k(k_gemm_tc<TG_PREC_TF32>, dim3(grid), dim3(TC_THREADS), smem, st, g, w, stages, stg, tm, a_tma, tm2,
             a2_kb0, a2_x0);
  } else if (precision == TG_PREC_F16X3) {
    static size_t set = 0;
    if (smem > set) {
      cudaFuncSetAttribute(k_gemm_tc<TG_PREC_F16X3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      set = smem;
    }
    launch_k(k_gemm_tc<TG_PREC_F16X3>, dim3(grid), dim3(TC_THREADS), smem, st, g, w, stages, stg, tm, a_tma, tm2,
             1 << 30, 0);
  } else {
    static size_t set = 0;
    if (smem > set) {
      cudaFuncSetAttribute(k_gemm_tc<TG_PREC_TF32X3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      set = smem;
    }
    launch_k(k_gemm_tc<TG_PREC_TF32X3>, dim3(grid), dim3(TC_THREADS), smem, st, g, w, stages, stg, tm, a_tma, tm2,
             1 << 30, 0);
  }
}

#ifdef TG_TC_TRACE
extern "C" int tg_debug_tc_trace(int arm_n, int arm_k, int mode, long long* host) {
  if (host) return (int)cudaMemcpyFromSymbol(host, tg_tct, sizeof(tg_tct));
  int nk[3] = {arm_n, arm_k, mode};
  static long long zero[148][TCT_N] = {};
  cudaMemcpyToSymbol(tg_tct, zero, sizeof(zero));
  return (int)cudaMemcpyToSymbol(tg_tct_nk, nk, sizeof(nk));
}
#endif

}  // namespace tg
