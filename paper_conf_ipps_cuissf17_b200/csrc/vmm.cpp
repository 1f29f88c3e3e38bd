// vmm.cpp — mirrored ring buffers (PP_OPT_MIRROR): one physical allocation of R plane
// slots mapped at two adjacent virtual ranges, [slots 0..R-1][slots 0..R-1 again]. A chunk's planes
// that run past the ring end (the index handler's wrap) are then contiguous in the
// device address space, so the H2D/D2H of a chunk is ONE cudaMemcpyAsync instead of two (each copy
// costs ~12-17 us of setup on the B200 host link: profiles/r1_cupti_overlap.jsonl; configs[1]
// 25.55 -> 23.43 ms, profiles/r1_mirror_ab.jsonl). Built on the
// CUDA virtual memory management driver calls, fetched with cudaGetDriverEntryPoint (no libcuda link).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <mutex>
#include <string>

#include "region.hpp"

namespace pprt {
namespace {

struct Vmm {
    CUresult (*granularity)(size_t *, const CUmemAllocationProp *, CUmemAllocationGranularity_flags) = nullptr;
    CUresult (*create)(CUmemGenericAllocationHandle *, size_t, const CUmemAllocationProp *, unsigned long long) = nullptr;
    CUresult (*release)(CUmemGenericAllocationHandle) = nullptr;
    CUresult (*reserve)(CUdeviceptr *, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
    CUresult (*free_va)(CUdeviceptr, size_t) = nullptr;
    CUresult (*map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
    CUresult (*unmap)(CUdeviceptr, size_t) = nullptr;
    CUresult (*access)(CUdeviceptr, size_t, const CUmemAccessDesc *, size_t) = nullptr;
    bool ok = false;
};

template <typename F> bool entry(const char *name, F *fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess || !p) {
        cudaGetLastError();
        return false;
    }
    *fn = reinterpret_cast<F>(p);
    return true;
}

const Vmm &vmm() {
    static Vmm v;
    static std::once_flag once;
    std::call_once(once, [] {
        v.ok = entry("cuMemGetAllocationGranularity", &v.granularity) && entry("cuMemCreate", &v.create) &&
               entry("cuMemRelease", &v.release) && entry("cuMemAddressReserve", &v.reserve) &&
               entry("cuMemAddressFree", &v.free_va) && entry("cuMemMap", &v.map) &&
               entry("cuMemUnmap", &v.unmap) && entry("cuMemSetAccess", &v.access);
    });
    return v;
}

CUmemAllocationProp prop_for(int device) {
    CUmemAllocationProp p = {};
    p.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    p.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    p.location.id = device;
    return p;
}

}  // namespace

uint64_t vmm_granularity(int device) {
    static std::mutex mu;
    static uint64_t cache[64] = {};
    if (device < 0 || device >= 64) return 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!cache[device]) {
        const Vmm &v = vmm();
        size_t g = 0;
        CUmemAllocationProp p = prop_for(device);
        if (!v.ok || v.granularity(&g, &p, CU_MEM_ALLOC_GRANULARITY_MINIMUM) != CUDA_SUCCESS || !g)
            g = ~uint64_t(0);                        // unsupported: never mirror
        cache[device] = g;
    }
    return cache[device] == ~uint64_t(0) ? 0 : cache[device];
}

void mirror_free(MirrorBuf *m) {
    if (!m->va) return;
    const Vmm &v = vmm();
    const CUdeviceptr va = (CUdeviceptr)(uintptr_t)m->va;
    v.unmap(va, m->bytes);                       // each mapping separately
    v.unmap(va + m->bytes, m->bytes);
    v.free_va(va, 2 * m->bytes);
    v.release((CUmemGenericAllocationHandle)m->handle);
    *m = MirrorBuf{};
}

pp_status mirror_alloc(int device, uint64_t bytes, MirrorBuf *out) {
    const Vmm &v = vmm();
    const uint64_t g = vmm_granularity(device);
    if (!g || bytes % g) return fail(PP_EINVAL, "mirrored ring size is not a multiple of the VMM granularity");
    static const bool refuse = getenv("PP_TEST_REFUSE_VMM") != nullptr;   // tests of the fallback only
    if (refuse) return fail(PP_ECUDA, "cuMemCreate refused (PP_TEST_REFUSE_VMM)");
    CUmemAllocationProp p = prop_for(device);
    CUmemGenericAllocationHandle h = 0;
    CUresult e = v.create(&h, bytes, &p, 0);
    if (e != CUDA_SUCCESS) return fail(PP_ENOMEM, "cuMemCreate of a mirrored ring failed (" + std::to_string((int)e) + ")");
    CUdeviceptr va = 0;
    e = v.reserve(&va, 2 * bytes, g, 0, 0);
    if (e != CUDA_SUCCESS) {
        v.release(h);
        return fail(PP_ENOMEM, "cuMemAddressReserve failed (" + std::to_string((int)e) + ")");
    }
    e = v.map(va, bytes, 0, h, 0);
    if (e == CUDA_SUCCESS) {
        e = v.map(va + bytes, bytes, 0, h, 0);
        if (e != CUDA_SUCCESS) v.unmap(va, bytes);
    }
    if (e == CUDA_SUCCESS) {
        CUmemAccessDesc d = {};
        d.location = p.location;
        d.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        e = v.access(va, 2 * bytes, &d, 1);
        if (e != CUDA_SUCCESS) {
            v.unmap(va, bytes);
            v.unmap(va + bytes, bytes);
        }
    }
    if (e != CUDA_SUCCESS) {
        v.free_va(va, 2 * bytes);
        v.release(h);
        return fail(PP_ECUDA, "mapping a mirrored ring failed (" + std::to_string((int)e) + ")");
    }
    out->va = (void *)(uintptr_t)va;
    out->bytes = bytes;
    out->handle = (unsigned long long)h;
    return PP_OK;
}

}  // namespace pprt
