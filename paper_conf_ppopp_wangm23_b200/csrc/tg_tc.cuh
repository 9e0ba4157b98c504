// tcgen05 tensor-core GEMM for the dense per-target projections (sm_100a).
#pragma once
#include <cuda.h>

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
  float* colscale = nullptr;  // F16X3: per output column 2^-e undoing the weight-row scale [ntn * BN]
};

// Dense A operand loaded by TMA tensor copies (cp.async.bulk.tensor.2d, 128B
// swizzle, box = 128 rows x 128 bytes) instead of per-thread loads.
struct TcTensorA {
  CUtensorMap map;
  int valid = 0;
};
// base: dense row-major [rows x ld] of 2-byte (bf16) or 4-byte (fp32) elements; ld*elem % 16 == 0.
tg_status tc_make_tensor_a(const void* base, int elem_bytes, int ld, int rows, TcTensorA* out);

tg_status tc_prepare_weights(const float* W, int N, int K, int precision, TcWeights* out,
                             std::vector<void*>& owned);
// ta (optional): the A operand as a tensor map (must match the element type of
// the precision: bf16 for TG_PREC_BF16, fp32 for TG_PREC_TF32).
// ta2 (optional): k-blocks >= a2_kb0 of A come from this second map at columns a2_x0 + 64 (kb - a2_kb0)
void launch_gemm_tc(const GemmArgs& g, const TcWeights& w, int precision, cudaStream_t st,
                    const TcTensorA* ta = nullptr, const TcTensorA* ta2 = nullptr, int a2_kb0 = 0, int a2_x0 = 0);

}  // namespace tg
