// Loop body: dense GEMM C = A.B, bf16 inputs, fp32 accumulation (config C3), rows [m0, m1) of one
// partition. tcgen05 implementation pending; the body reports "unsupported" until then.
#include "kernels.h"

namespace accmg {
namespace k {

cudaError_t gemm_bf16(const uint16_t* A, const uint16_t* B, float* C, int64_t M, int64_t N, int64_t K, int64_t m0,
                      int64_t m1, cudaStream_t s, int64_t* launches) {
    (void)A; (void)B; (void)C; (void)M; (void)N; (void)K; (void)m0; (void)m1; (void)s; (void)launches;
    return cudaErrorNotSupported;
}

}  // namespace k
}  // namespace accmg
