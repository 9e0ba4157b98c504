// tcgen05 tensor-core GEMM for the dense per-target projections (sm_100a).
#pragma once
#include <vector>

#include "tg_internal.cuh"

namespace tg {

// Weight operand B[N x K] re-laid out for UMMA (K-major, 128B-swizzled
// 8-row core-matrix groups), as tf32 hi/lo planes (TG_PREC_TF32X3) or bf16.
struct TcWeights {
  void* hi = nullptr;
  void* lo = nullptr;
  int N = 0, K = 0, Np = 0, Kp = 0;
};

tg_status tc_prepare_weights(const float* W, int N, int K, int precision, TcWeights* out,
                             std::vector<void*>& owned);
void launch_gemm_tc(const GemmArgs& g, const TcWeights& w, int precision, cudaStream_t st);

}  // namespace tg
