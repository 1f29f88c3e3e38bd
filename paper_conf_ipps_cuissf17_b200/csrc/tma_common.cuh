// tma_common.cuh — shared pieces of the TMA-staged kernels (stencil_tma.cu, stencil_fused.cu):
// PTX wrappers for mbarriers and cp.async.bulk.tensor, and the host-side tensor-map cache and
// per-device launch helpers. Product side only (sm_100a).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <utility>

#include "kernels.cuh"

namespace pp {

// ---------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, int x, int y, int z, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
            smem_u32(dst)),
        "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

// packed fp32 pair (lo = a, hi = b) and the lane-wise round-to-nearest packed add (sm_100 FADD2)
__device__ __forceinline__ uint64_t pack2(float a, float b) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ uint64_t pack2(double, double) { return 0; }   // unused (fp64 is never paired)
__device__ __forceinline__ uint64_t add2_rn(uint64_t x, uint64_t y) {
    uint64_t r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(x), "l"(y));
    return r;
}
// lane-wise d = a*b + c with ONE rounding (sm_100 FFMA2). Used only where a*b is exact (a power-of-two
// coefficient), so the result equals RN(RN(a*b) + c), the unfused product-then-add
__device__ __forceinline__ uint64_t fma2_rn(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ void unpack2(uint64_t x, float &a, float &b) {
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(x));
}
__device__ __forceinline__ void unpack2(uint64_t, double &, double &) {}

// ---------------------------------------------------------------- host helpers (stencil_tma.cu)
// 3-D tensor map over a device ring [R][ny][nx] of `esize`-byte floats with a (boxw, boxh, 1) box,
// cached per thread; nullptr if the driver cannot encode it.
const CUtensorMap *tma_map_3d(const DView &in, int64_t ny, int64_t nx, int esize, int boxw, int boxh);
int sm_count();                                   // SMs of the current device
int env_int(const char *name, int dflt, int lo, int hi);

// ---------------------------------------------------------------- programmatic dependent launch
// Back-to-back kernels on one stream (the level kernels of a multi-sweep chain, PP_OPT_SWEEPS) are
// launched with cudaLaunchAttributeProgrammaticStreamSerialization: the next grid may be scheduled
// while this one drains. Every kernel that is launched this way calls pdl_release_and_wait() before
// its first global-memory access: it lets its own successor start, then waits (griddepcontrol.wait)
// until its predecessor has completed and flushed — the same ordering as plain stream order, minus
// the launch gap. For a kernel launched without the attribute both instructions are no-ops.
__device__ __forceinline__ void pdl_release_and_wait() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
}
bool pdl_enabled();                               // PP_PDL (default 1); stencil_tma.cu

template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kernel)(KArgs...), unsigned grid, unsigned block, size_t smem, cudaStream_t st,
                       Args &&...args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = tls_pdl && pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

}  // namespace pp
