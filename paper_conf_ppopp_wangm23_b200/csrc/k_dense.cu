// Dense per-target stages of M and the merge FFN (Eqs. 6-7) on CUDA cores
// (TG_PREC_FP32), LayerNorm (R1), the link-prediction score (R10) and the
// DedupInvert row copy (Alg. 1 l.20).
#include <cuda_bf16.h>

#include "tg_internal.cuh"

namespace tg {

// ----------------------------------------------------------- SIMT fp32 GEMM
// C[M x N] = epi(A[M x K] . B[N x K]^T); 64x64 tiles, BK = 16, 256 threads,
// 4x4 outputs per thread, fixed K order (batch-invariant rows).
constexpr int GBM = 64, GBN = 64, GBK = 16;

__device__ __forceinline__ float4 gemm_load_a(const GemmArgs& g, int row, int M, int c) {
  if (row >= M || c >= g.K) return make_float4(0.f, 0.f, 0.f, 0.f);
  const float* p;
  if (c < g.K0) {
    p = g.a_rows0 ? g.a_rows0[row] + c : g.a_base0 + (size_t)row * g.lda0 + c;
  } else {
    const int cc = c - g.K0;
    p = g.a_rows1 ? g.a_rows1[row] + cc : g.a_base1 + (size_t)row * g.lda1 + cc;
  }
  return *reinterpret_cast<const float4*>(p);
}

__global__ void __launch_bounds__(256) k_gemm_simt(GemmArgs g) { pdl_enter();
  __shared__ __align__(16) float As[GBK][GBM + 4];
  __shared__ __align__(16) float Bs[GBK][GBN + 4];
  const int M = *g.m_dev;
  const int tiles_m = (M + GBM - 1) / GBM, tiles_n = (g.N + GBN - 1) / GBN;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int lr = tid >> 2, lc4 = tid & 3;  // loader: row, float4 column
  for (int t = blockIdx.x; t < tiles_m * tiles_n; t += gridDim.x) {
    const int tm = t / tiles_n, tn = t - tm * tiles_n;
    const int m0 = tm * GBM, n0 = tn * GBN;
    float acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
    for (int k0 = 0; k0 < g.K; k0 += GBK) {
      const float4 av = gemm_load_a(g, m0 + lr, M, k0 + 4 * lc4);
      float4 bv = make_float4(0.f, 0.f, 0.f, 0.f);
      if (n0 + lr < g.N && k0 + 4 * lc4 < g.K)
        bv = *reinterpret_cast<const float4*>(g.B + (size_t)(n0 + lr) * g.K + k0 + 4 * lc4);
      As[4 * lc4 + 0][lr] = av.x;
      As[4 * lc4 + 1][lr] = av.y;
      As[4 * lc4 + 2][lr] = av.z;
      As[4 * lc4 + 3][lr] = av.w;
      Bs[4 * lc4 + 0][lr] = bv.x;
      Bs[4 * lc4 + 1][lr] = bv.y;
      Bs[4 * lc4 + 2][lr] = bv.z;
      Bs[4 * lc4 + 3][lr] = bv.w;
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < GBK; ++kk) {
        const float4 a4 = *reinterpret_cast<const float4*>(&As[kk][ty * 4]);
        const float4 b4 = *reinterpret_cast<const float4*>(&Bs[kk][tx * 4]);
        const float a[4] = {a4.x, a4.y, a4.z, a4.w};
        const float b[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
      }
      __syncthreads();
    }
    // epilogue: bias, residual q = [hs || 0 || Phi(0)] (Eq. 4), ReLU, store
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = m0 + ty * 4 + i;
      const int c = n0 + tx * 4;
      if (r >= M || c >= g.N) continue;
      float v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        float x = acc[i][j];
        if (g.bias) x += g.bias[c + j];
        if (g.relu) x = fmaxf(x, 0.f);
        v[j] = x;
      }
      float* out = g.c_rows ? g.c_rows[r] + c : g.C + (size_t)r * g.ldc + c;
      *reinterpret_cast<float4*>(out) = make_float4(v[0], v[1], v[2], v[3]);
    }
  }
}

void launch_gemm_simt(const GemmArgs& g, cudaStream_t st) {
  const int tiles = ((g.m_max + GBM - 1) / GBM) * ((g.N + GBN - 1) / GBN);
  int blocks = tiles < 148 * 4 ? tiles : 148 * 4;
  if (blocks < 1) blocks = 1;
  launch_k(k_gemm_simt, dim3(blocks), dim3(256), 0, st, g);
}

// ---------------------------------------------------------------- LayerNorm
// r = LN(y + q; gamma, beta) with q = [h^(l-1) | 0 | Phi(0)] (Eq. 4/6, R1, R3),
// mean and biased variance over the D valid columns, eps 1e-5. Warp per row;
// per-column parameters (gamma, beta, valid weight, Phi(0) block of q) are
// staged in shared memory once per CTA; the grid is one resident wave that
// strides over the rows. Outputs: fp32 r [M x (Dp + dnp)] = [LN(y) | h^(l-1)] (the
// dense A operand of the merge FFN, Eq. 7) and/or the bf16 merge-FFN
// input row rh = [LN(y) (Dp) | 0 | h^(l-1) at rh_off (16-byte aligned) | 0] (Eq. 7).
constexpr int kLnMaxD4 = 256;  // Dp <= 1024 (checked at model load)
// NJ = ceil(Dp / 128) float4 per lane and row. Two rows per warp iteration (r2): their loads
// (y rows, the h row pointers, then the h rows) are all issued before either row is reduced,
// so each warp keeps two rows of memory in flight (the single-row loop exposed the pointer ->
// h-row dependent latency once per row: 107 us per launch at 50k rows, 2.6 TB/s).
template <int NJ>
__global__ void __launch_bounds__(256, 3)
    k_layernorm(const float* __restrict__ y, float* __restrict__ r, int Dp, int dn, int dnp, int de, int dep, int dt,
                const float* __restrict__ gamma, const float* __restrict__ beta, const int* __restrict__ m_dev,
                const float* const* __restrict__ hs_rows, const float* __restrict__ phi0,
                unsigned short* __restrict__ rh, int ldrh, int rh_off) {
  const int ldr = Dp + dnp;
  __shared__ float4 s_g[kLnMaxD4], s_b[kLnMaxD4], s_w[kLnMaxD4], s_q[kLnMaxD4];
  const int D4 = Dp >> 2;
  const int s1 = dnp, s2 = dnp + dep;
  for (int q = threadIdx.x; q < D4; q += blockDim.x) {  // parameters only: before the PDL wait
    s_g[q] = reinterpret_cast<const float4*>(gamma)[q];
    s_b[q] = reinterpret_cast<const float4*>(beta)[q];
    float w[4];
    for (int i = 0; i < 4; ++i) {
      const int c = 4 * q + i;
      w[i] = (c < dn || (c >= s1 && c < s1 + de) || (c >= s2 && c < s2 + dt)) ? 1.f : 0.f;
    }
    s_w[q] = make_float4(w[0], w[1], w[2], w[3]);
    s_q[q] = 4 * q >= s2 ? reinterpret_cast<const float4*>(phi0)[q - (s2 >> 2)] : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  pdl_enter();
  __syncthreads();
  const int M = *m_dev;
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  const float D = (float)(dn + de + dt);
  const int nh4 = dnp >> 2;
  for (int row0 = warp; row0 < M; row0 += 2 * nw) {
    const int rows[2] = {row0, row0 + nw};
    const bool live1 = rows[1] < M;
    float4 v[2][NJ];
    const float4* hr[2];
#pragma unroll
    for (int u = 0; u < 2; ++u) hr[u] = (u == 0 || live1) ? reinterpret_cast<const float4*>(hs_rows[rows[u]]) : nullptr;
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const float4* yr = reinterpret_cast<const float4*>(y + (size_t)rows[u] * Dp);
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int q = lane + 32 * j;
        v[u][j] = (q < D4 && (u == 0 || live1)) ? yr[q] : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
    float4 hv[2][2];  // the first 64 float4 of each h row (d_n <= 256), issued with the y loads
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int q = lane + 32 * j;
        hv[u][j] = (q < nh4 && (u == 0 || live1)) ? hr[u][q] : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      if (u == 1 && !live1) break;
      const int row = rows[u];
      float sum = 0.f;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int q = lane + 32 * j;
        if (q < D4) {
          const float4 b = q < nh4 ? (j < 2 ? hv[u][j < 2 ? j : 0] : hr[u][q]) : s_q[q];  // + q = [h || 0 || Phi(0)]
          v[u][j] = make_float4(v[u][j].x + b.x, v[u][j].y + b.y, v[u][j].z + b.z, v[u][j].w + b.w);
          sum += (v[u][j].x + v[u][j].y) + (v[u][j].z + v[u][j].w);  // padded columns are exact zeros
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
      const float mu = sum / D;
      float var = 0.f;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int q = lane + 32 * j;
        if (q < D4) {
          const float4 w = s_w[q];
          const float dx = v[u][j].x - mu, dy = v[u][j].y - mu, dz = v[u][j].z - mu, dw = v[u][j].w - mu;
          var = fmaf(w.x * dx, dx, var);
          var = fmaf(w.y * dy, dy, var);
          var = fmaf(w.z * dz, dz, var);
          var = fmaf(w.w * dw, dw, var);
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) var += __shfl_xor_sync(0xffffffffu, var, o);
      const float rstd = rsqrtf(var / D + 1e-5f);
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int q = lane + 32 * j;
        if (q < D4) {
          const float4 g = s_g[q], b = s_b[q];  // zero on padded columns -> output 0 there
          const float4 o4 = make_float4(fmaf((v[u][j].x - mu) * rstd, g.x, b.x), fmaf((v[u][j].y - mu) * rstd, g.y, b.y),
                                        fmaf((v[u][j].z - mu) * rstd, g.z, b.z), fmaf((v[u][j].w - mu) * rstd, g.w, b.w));
          if (r) reinterpret_cast<float4*>(r + (size_t)row * ldr)[q] = o4;
          if (rh) {
            __nv_bfloat162 lo = __floats2bfloat162_rn(o4.x, o4.y), hi = __floats2bfloat162_rn(o4.z, o4.w);
            uint2 pk;
            pk.x = *reinterpret_cast<uint32_t*>(&lo);
            pk.y = *reinterpret_cast<uint32_t*>(&hi);
            *reinterpret_cast<uint2*>(rh + (size_t)row * ldrh + 4 * q) = pk;
          }
        }
      }
      if (r)  // h^(l-1) after LN(y): the merge FFN's [LN(y) | h] row is dense
        for (int q = lane, j = 0; q < nh4; q += 32, ++j)
          reinterpret_cast<float4*>(r + (size_t)row * ldr + Dp)[q] = j < 2 ? hv[u][j & 1] : hr[u][q];
      if (rh) {  // [Dp, ldrh): zeros, h^(l-1) at rh_off, zeros
        const int q0 = (rh_off - Dp) >> 2;
        for (int q = lane; 4 * q < ldrh - Dp; q += 32) {
          float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
          if (q >= q0 && q - q0 < nh4) x = hr[u][q - q0];
          __nv_bfloat162 lo = __floats2bfloat162_rn(x.x, x.y), hi = __floats2bfloat162_rn(x.z, x.w);
          uint2 pk;
          pk.x = *reinterpret_cast<uint32_t*>(&lo);
          pk.y = *reinterpret_cast<uint32_t*>(&hi);
          *reinterpret_cast<uint2*>(rh + (size_t)row * ldrh + Dp + 4 * q) = pk;
        }
      }
    }
  }
}

void launch_layernorm(const float* y, float* r, int Dp, int dn, int dnp, int de, int dep, int dt,
                      const float* gamma, const float* beta, const int* m_dev, int m_max,
                      const float* const* hs_rows, const float* phi0, unsigned short* rh, int ldrh, int rh_off,
                      cudaStream_t st) {
  int blocks = (m_max + 15) / 16;  // 8 warps per CTA, two rows per warp iteration
  if (blocks > 148 * 3) blocks = 148 * 3;  // one resident wave (3 CTAs / SM at <= 85 registers)
  if (blocks < 1) blocks = 1;
  const int nj = ((Dp >> 2) + 31) / 32;
#define TG_LN(NJ)                                                                                              \
  case NJ:                                                                                                     \
    launch_k(k_layernorm<NJ>, dim3(blocks), dim3(256), 0, st, y, r, Dp, dn, dnp, de, dep, dt, gamma, beta, m_dev, \
             hs_rows, phi0, rh, ldrh, rh_off);                                                                 \
    break;
  switch (nj) {
    TG_LN(1) TG_LN(2) TG_LN(3) TG_LN(4) TG_LN(5) TG_LN(6) TG_LN(7) default: TG_LN(8)
  }
#undef TG_LN
}

// -------------------------------------------------------------------- score
// p_e = sigmoid(W_a2 ReLU(W_a1 [h_src || h_dst] + b_a1) + b_a2) (R10) as
// (1) row resolution through each batch's inverse index (DedupInvert),
// (2) the hidden layer as a projection GEMM over the S*B edges, (3) a warp
// per edge for the W_a2 dot product and the sigmoid. With negatives (es.neg,
// NEXT-3) rows S*B.. score (src_e, neg_e) into scores[n_edges + e].
__global__ void k_score_rows(const float* __restrict__ HL, int ldh, LevelDev top, int S, EdgeSrc es,
                             const float** __restrict__ rs, const float** __restrict__ rd,
                             long long* __restrict__ oidx, int* __restrict__ m_dev) { pdl_enter();
  const int half = S * es.B;
  const int tot = es.neg ? 2 * half : half;
  if (blockIdx.x == 0 && threadIdx.x == 0) *m_dev = tot;
  for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < tot; w += gridDim.x * blockDim.x) {
    const int ng = w >= half;
    const int wp = w - ng * half;
    const int b = wp / es.B, e = wp - b * es.B;
    const int64_t lo = es.e0 + (int64_t)b * es.B;
    const int64_t rem = es.n_edges - lo;
    const int Bb = (int)(rem < es.B ? (rem < 0 ? 0 : rem) : es.B);
    if (e < Bb) {
      const size_t seg = (size_t)b * top.cap;
      rs[w] = HL + (size_t)(top.c_base[b] + top.inv[seg + e]) * ldh;
      rd[w] = HL + (size_t)(top.c_base[b] + top.inv[seg + (ng ? 2 : 1) * Bb + e]) * ldh;
      oidx[w] = (ng ? es.n_edges : 0) + lo + e;
    } else {  // past the stream end: any valid row, result discarded
      rs[w] = HL;
      rd[w] = HL;
      oidx[w] = -1;
    }
  }
}

void launch_score_rows(const float* HL, int ldh, LevelDev top, int S, EdgeSrc es, const float** rs,
                       const float** rd, long long* oidx, int* m_dev, cudaStream_t st) {
  int blocks = ((es.neg ? 2 : 1) * S * es.B + 255) / 256;
  if (blocks < 1) blocks = 1;
  launch_k(k_score_rows, dim3(blocks), dim3(256), 0, st, HL, ldh, top, S, es, rs, rd, oidx, m_dev);
}

__global__ void k_score_head(const float* __restrict__ z, int ldz, const long long* __restrict__ oidx, int M,
                             const float* __restrict__ Wa2, float ba2, int dn, float* __restrict__ scores) { pdl_enter();
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  for (int w = warp; w < M; w += nw) {
    const long long o = oidx[w];
    if (o < 0) continue;
    const float* zr = z + (size_t)w * ldz;
    float s = 0.f;
    for (int j = lane; j < dn; j += 32) s = fmaf(Wa2[j], zr[j], s);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if (lane == 0) scores[o] = 1.f / (1.f + expf(-(s + ba2)));
  }
}

void launch_score_head(const float* z, int ldz, const long long* oidx, int M, const float* Wa2, float ba2, int dn,
                       float* scores, cudaStream_t st) {
  int blocks = (M * 32 + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  launch_k(k_score_head, dim3(blocks), dim3(256), 0, st, z, ldz, oidx, M, Wa2, ba2, dn, scores);
}

// Pair rows for tg_score_pairs (NEXT-3 link prediction with negatives): pair p scores
// target pa[p] against target pb[p] of a single-batch target list, both resolved through
// the batch's inverse index (DedupInvert, Alg. 1 l.20); an out-of-range index is an error.
__global__ void k_pair_rows(const float* __restrict__ HL, int ldh, LevelDev top, int n_targets,
                            const int32_t* __restrict__ pa, const int32_t* __restrict__ pb, int n_pairs,
                            const float** __restrict__ rs, const float** __restrict__ rd,
                            long long* __restrict__ oidx, int* __restrict__ m_dev, int* __restrict__ err) { pdl_enter();
  if (blockIdx.x == 0 && threadIdx.x == 0) *m_dev = n_pairs;
  for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < n_pairs; w += gridDim.x * blockDim.x) {
    const int a = pa[w], b = pb[w];
    if (a < 0 || a >= n_targets || b < 0 || b >= n_targets) {
      atomicOr(err, kErrPairIndex);
      rs[w] = HL;
      rd[w] = HL;
      oidx[w] = -1;
      continue;
    }
    rs[w] = HL + (size_t)(top.c_base[0] + top.inv[a]) * ldh;
    rd[w] = HL + (size_t)(top.c_base[0] + top.inv[b]) * ldh;
    oidx[w] = w;
  }
}

void launch_pair_rows(const float* HL, int ldh, LevelDev top, int n_targets, const int32_t* pa, const int32_t* pb,
                      int n_pairs, const float** rs, const float** rd, long long* oidx, int* m_dev, int* err,
                      cudaStream_t st) {
  int blocks = (n_pairs + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  launch_k(k_pair_rows, dim3(blocks), dim3(256), 0, st, HL, ldh, top, n_targets, pa, pb, n_pairs, rs, rd, oidx,
           m_dev, err);
}

__global__ void k_invert(const float* __restrict__ HL, int ldh, LevelDev top, int n, int dn,
                         float* __restrict__ out) { pdl_enter();
  const long long tot = (long long)n * dn;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < tot; i += (long long)gridDim.x * blockDim.x) {
    const long long r = i / dn;
    const int c = (int)(i - r * dn);
    out[i] = HL[(size_t)(top.c_base[0] + top.inv[r]) * ldh + c];
  }
}

void launch_invert(const float* HL, int ldh, LevelDev top, int n, int dn, float* out, cudaStream_t st) {
  if (n <= 0) return;
  long long tot = (long long)n * dn;
  int blocks = (int)((tot + 255) / 256);
  if (blocks > 1184) blocks = 1184;
  launch_k(k_invert, dim3(blocks), dim3(256), 0, st, HL, ldh, top, n, dn, out);
}

__global__ void k_set_int(int* p, int v) { pdl_enter(); *p = v; }
void launch_set_int(int* p, int v, cudaStream_t st) { launch_k(k_set_int, dim3(1), dim3(1), 0, st, p, v); }

}  // namespace tg
