// tcgen05 GEMM (placeholder until the UMMA kernel lands: falls back to nothing).
#include "tg_tc.cuh"

namespace tg {

tg_status tc_prepare_weights(const float* W, int N, int K, int precision, TcWeights* out,
                             std::vector<void*>& owned) {
  (void)W; (void)N; (void)K; (void)precision; (void)out; (void)owned;
  return TG_EINVAL;
}

void launch_gemm_tc(const GemmArgs& g, const TcWeights& w, int precision, cudaStream_t st) {
  (void)g; (void)w; (void)precision; (void)st;
}

}  // namespace tg
