// tcgen05 tensor-core GEMM for the dense per-target projections (sm_100a).
#pragma once
#include <vector>

#include "tg_internal.cuh"

namespace tg {

// Weight operand B[N x K] re-laid out for UMMA (K-major, 128B-swizzled
// 8-row core-matrix groups), as tf32 hi/lo planes (TG_PREC_TF32X3) or bf16.
struct TcWeights {
  void* hi = nullptr;      // images [ntn][nkb][planes][BN x 128 B]
  void* lo = nullptr;      // unused (lo plane interleaved after hi)
  int N = 0, K = 0, Np = 0, Kp = 0;
  int BN = 0;              // N tile (multiple of 16, <= 256)
  int ntn = 0;             // N tiles
  int nkb = 0;             // K blocks of 128 bytes
};

tg_status tc_prepare_weights(const float* W, int N, int K, int precision, TcWeights* out,
                             std::vector<void*>& owned);
void launch_gemm_tc(const GemmArgs& g, const TcWeights& w, int precision, cudaStream_t st);

}  // namespace tg
