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
__global__ void k_layernorm(const float* __restrict__ y, float* __restrict__ r, int Dp, int dn, int dnp, int de,
                            int dep, int dt, const float* __restrict__ gamma, const float* __restrict__ beta,
                            const int* __restrict__ m_dev, const float* const* __restrict__ hs_rows,
                            const float* __restrict__ phi0, unsigned short* __restrict__ rh, int ldrh) { pdl_enter();
  const int M = *m_dev;
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  const int D = dn + de + dt;
  const int s1 = dnp, s2 = dnp + dep;
  const int D4 = Dp >> 2;
  // warp per row; the row (<= 1024 floats) is read once into registers
  for (int row = warp; row < M; row += nw) {
    const float4* yr = reinterpret_cast<const float4*>(y + (size_t)row * Dp);
    const float4* hr = reinterpret_cast<const float4*>(hs_rows[row]);
    const float4* p0 = reinterpret_cast<const float4*>(phi0);
    float4* rr = r ? reinterpret_cast<float4*>(r + (size_t)row * Dp) : nullptr;
    float4 v[8];
    float sum = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int q = lane + 32 * j;
      v[j] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (q < D4) {
        v[j] = yr[q];
        // + q = [h^(l-1) || 0 || Phi(0)] (padded columns of each part are zero)
        float4 a = make_float4(0.f, 0.f, 0.f, 0.f);
        if (4 * q < dnp) a = hr[q];
        else if (4 * q >= s2) a = p0[q - (s2 >> 2)];
        v[j].x += a.x;
        v[j].y += a.y;
        v[j].z += a.z;
        v[j].w += a.w;
        // padded columns are exact zeros (zero weight rows / bias), so they do not bias the sum
        sum += (v[j].x + v[j].y) + (v[j].z + v[j].w);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    const float mu = sum / (float)D;
    float var = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int q = lane + 32 * j;
      if (q < D4) {
        const float e[4] = {v[j].x, v[j].y, v[j].z, v[j].w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int c = 4 * q + i;
          const bool valid = c < dn || (c >= s1 && c < s1 + de) || (c >= s2 && c < s2 + dt);
          const float d = e[i] - mu;
          if (valid) var = fmaf(d, d, var);
        }
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) var += __shfl_xor_sync(0xffffffffu, var, o);
    const float rstd = rsqrtf(var / (float)D + 1e-5f);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int q = lane + 32 * j;
      if (q < D4) {
        const float e[4] = {v[j].x, v[j].y, v[j].z, v[j].w};
        float o4[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int c = 4 * q + i;
          const bool valid = c < dn || (c >= s1 && c < s1 + de) || (c >= s2 && c < s2 + dt);
          o4[i] = valid ? (e[i] - mu) * rstd * gamma[c] + beta[c] : 0.f;
        }
        if (rr) rr[q] = make_float4(o4[0], o4[1], o4[2], o4[3]);
        if (rh) {
          __nv_bfloat162 lo = __floats2bfloat162_rn(o4[0], o4[1]), hi = __floats2bfloat162_rn(o4[2], o4[3]);
          uint2 pk;
          pk.x = *reinterpret_cast<uint32_t*>(&lo);
          pk.y = *reinterpret_cast<uint32_t*>(&hi);
          *reinterpret_cast<uint2*>(rh + (size_t)row * ldrh + 4 * q) = pk;
        }
      }
    }
    if (rh) {  // [LN(y) | h^(l-1) | 0]: the merge-FFN input (Eq. 7) as one bf16 row
      for (int q = lane; 4 * q < ldrh - Dp; q += 32) {
        float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
        if (4 * q < dnp) x = hr[q];
        __nv_bfloat162 lo = __floats2bfloat162_rn(x.x, x.y), hi = __floats2bfloat162_rn(x.z, x.w);
        uint2 pk;
        pk.x = *reinterpret_cast<uint32_t*>(&lo);
        pk.y = *reinterpret_cast<uint32_t*>(&hi);
        *reinterpret_cast<uint2*>(rh + (size_t)row * ldrh + Dp + 4 * q) = pk;
      }
    }
  }
}

void launch_layernorm(const float* y, float* r, int Dp, int dn, int dnp, int de, int dep, int dt,
                      const float* gamma, const float* beta, const int* m_dev, int m_max,
                      const float* const* hs_rows, const float* phi0, unsigned short* rh, int ldrh,
                      cudaStream_t st) {
  int blocks = (m_max * 32 + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  launch_k(k_layernorm, dim3(blocks), dim3(256), 0, st, y, r, Dp, dn, dnp, de, dep, dt, gamma, beta, m_dev, hs_rows, phi0, rh,
                                      ldrh);
}

// -------------------------------------------------------------------- score
// p_e = sigmoid(W_a2 ReLU(W_a1 [h_src || h_dst] + b_a1) + b_a2) (R10) as
// (1) row resolution through each batch's inverse index (DedupInvert),
// (2) the hidden layer as a projection GEMM over the S*B edges, (3) a warp
// per edge for the W_a2 dot product and the sigmoid.
__global__ void k_score_rows(const float* __restrict__ HL, int ldh, LevelDev top, int S, EdgeSrc es,
                             const float** __restrict__ rs, const float** __restrict__ rd,
                             long long* __restrict__ oidx, int* __restrict__ m_dev) { pdl_enter();
  const int tot = S * es.B;
  if (blockIdx.x == 0 && threadIdx.x == 0) *m_dev = tot;
  for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < tot; w += gridDim.x * blockDim.x) {
    const int b = w / es.B, e = w - b * es.B;
    const int64_t lo = es.e0 + (int64_t)b * es.B;
    const int64_t rem = es.n_edges - lo;
    const int Bb = (int)(rem < es.B ? (rem < 0 ? 0 : rem) : es.B);
    if (e < Bb) {
      const size_t seg = (size_t)b * top.cap;
      rs[w] = HL + (size_t)(top.c_base[b] + top.inv[seg + e]) * ldh;
      rd[w] = HL + (size_t)(top.c_base[b] + top.inv[seg + Bb + e]) * ldh;
      oidx[w] = lo + e;
    } else {  // past the stream end: any valid row, result discarded
      rs[w] = HL;
      rd[w] = HL;
      oidx[w] = -1;
    }
  }
}

void launch_score_rows(const float* HL, int ldh, LevelDev top, int S, EdgeSrc es, const float** rs,
                       const float** rd, long long* oidx, int* m_dev, cudaStream_t st) {
  int blocks = (S * es.B + 255) / 256;
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
