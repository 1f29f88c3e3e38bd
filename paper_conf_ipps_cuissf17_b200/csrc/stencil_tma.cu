// stencil_tma.cu — TMA-staged stencil path (placeholder until the TMA kernel lands; the generic
// path serves every shape meanwhile).
#include "kernels.cuh"

namespace pp {
bool stencil7_tma_supported(int, const DView &, const DView &, int64_t, int64_t) { return false; }
cudaError_t launch_stencil7_tma(int, const DView &, int64_t, const DView &, int64_t, int64_t, int64_t,
                                int64_t, int64_t, double, double, bool, cudaStream_t) {
    return cudaErrorNotSupported;
}
bool tma_available() { return false; }
}  // namespace pp
