// persist.cpp — the persistent pipeline executor (PP_OPT_PERSISTENT). The planner's ops are kept, but
// the chunk kernels become ONE resident kernel (stencil7_pipe_kernel, stencil_tma.cu) and the event
// edges between the copy streams and the kernel become flag words in device memory: the copy streams
// write and wait on them with stream memory operations (cuStreamWriteValue32 / cuStreamWaitValue32),
// the kernel polls them. That removes the per-chunk kernel launch and the two cross-engine event hops
// per chunk that sit on the critical path of a one-chunk-in-flight schedule.
//
// The gating is coarser than the planner's exact dependencies (whole chunks instead of planes), so a
// plan is accepted only if every exact dependency is implied by it: an H2D of chunk j may depend only on
// kernels of chunks <= j - S, a kernel of chunk j only on H2D of chunks <= j and D2H of chunks <= j - S,
// a D2H of chunk j only on kernels of chunks <= j (checked on the full dependency lists).
#include <cuda.h>

#include <cstring>

#include "region.hpp"

namespace pprt {
using namespace pp;

namespace {
typedef CUresult (*PFN_streamValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
struct MemOps {
    PFN_streamValue32 wait = nullptr, write = nullptr;
    bool ok = false;
};
const MemOps &memops() {
    static MemOps m;
    static bool init = false;
    if (!init) {
        init = true;
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.wait = (PFN_streamValue32)p;
        p = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.write = (PFN_streamValue32)p;
        cudaGetLastError();
        m.ok = m.wait && m.write;
    }
    return m;
}

cudaError_t wait_value(cudaStream_t st, uint32_t *addr, uint32_t v) {
    return memops().wait((CUstream)st, (CUdeviceptr)addr, v, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS
               ? cudaSuccess : cudaErrorUnknown;
}
cudaError_t write_value(cudaStream_t st, uint32_t *addr, uint32_t v) {
    return memops().write((CUstream)st, (CUdeviceptr)addr, v, CU_STREAM_WRITE_VALUE_DEFAULT) == CUDA_SUCCESS
               ? cudaSuccess : cudaErrorUnknown;
}
}  // namespace

// Is this launch one the persistent executor can run? (why = the reason if not)
bool persistent_eligible(const pp_region *r, const Body &body, std::string *why) {
    const auto *b = dynamic_cast<const BuiltinBody *>(&body);
    const auto &A = r->arrs;
    auto no = [&](const char *m) { *why = m; return false; };
    if (!b || b->k != PP_K_STENCIL7) return no("PP_OPT_PERSISTENT runs the built-in PP_K_STENCIL7 body only");
    if (r->sweeps > 1) return no("PP_OPT_PERSISTENT runs single sweeps (PP_OPT_SWEEPS = 1)");
    if (A.size() != 2 || A[0].resident || A[1].resident || !A[0].pinned || !A[1].pinned)
        return no("PP_OPT_PERSISTENT needs two pinned host arrays");
    if (A[0].outer != 1 || A[1].outer != 1) return no("PP_OPT_PERSISTENT needs arrays split on dim 0");
    if (r->halo_in.arr >= 0 || r->halo_out.arr >= 0 || r->debug_tags || r->d2h_interior || r->sm_copy || r->trace)
        return no("PP_OPT_PERSISTENT does not combine with peer halos, tag checks, interior copy-back, SM copies "
                  "or traces");
    if (r->kernel_path == KPATH_GENERIC) return no("PP_OPT_PERSISTENT uses the TMA kernel");
    if (!memops().ok) return no("stream memory operations (cuStreamWaitValue32) are unavailable");
    // the chunk-granular gates must imply every exact dependency of the plan
    const Plan &P = r->plan;
    for (size_t i = 0; i < P.ops.size(); ++i) {
        const Op &op = P.ops[i];
        for (int32_t d = 0; d < op.full_dep_count; ++d) {
            const Op &dep = P.ops[(size_t)P.full_deps[(size_t)(op.full_dep_begin + d)]];
            bool ok = true;
            if (op.kind == OpKind::H2D)
                ok = dep.kind == OpKind::H2D || (dep.kind == OpKind::KER && dep.chunk <= op.chunk - P.S);
            else if (op.kind == OpKind::KER)
                ok = (dep.kind == OpKind::H2D && dep.chunk <= op.chunk) ||
                     (dep.kind == OpKind::D2H && dep.chunk <= op.chunk - P.S);
            else
                ok = (dep.kind == OpKind::KER && dep.chunk <= op.chunk) || dep.kind == OpKind::D2H;
            if (!ok) return no("PP_OPT_PERSISTENT needs full-overlap rings (PP_OPT_RING_EXTRA = -1)");
        }
    }
    return true;
}

pp_status enqueue_persistent(pp_region *r, Body &body, int64_t lo, int64_t hi) {
    const Plan &P = r->plan;
    const auto &b = dynamic_cast<const BuiltinBody &>(body);
    const auto &A = r->arrs;
    cudaError_t e;
    if (!r->pipe_flags) {
        if ((e = cudaMalloc(&r->pipe_flags, sizeof(PipeFlags))) != cudaSuccess) {
            cudaGetLastError();
            r->pipe_flags = nullptr;
            return fail(PP_ENOMEM, "PP_OPT_PERSISTENT flags");
        }
    }
    PipeFlags *fl = (PipeFlags *)r->pipe_flags;
    cudaStream_t sh = r->streams[0], sk = r->streams[1], sd = r->streams[2];
    if ((e = cudaMemsetAsync(fl, 0, sizeof(PipeFlags), sh)) != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync");
    if ((e = cudaEventRecord(r->join[0], sh)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
    for (cudaStream_t s : {sk, sd})
        if ((e = cudaStreamWaitEvent(s, r->join[0], 0)) != cudaSuccess) return cuda_fail(e, "cudaStreamWaitEvent");
    // the kernel first: if it cannot launch, nothing waits on it
    std::vector<DView> v = views_for(r);
    e = launch_stencil7_pipe(A[0].dtype, v[0], A[0].off + 1, v[1], A[1].off, A[0].ext[1], A[0].ext[2], lo, hi, P.c, P.S,
                             b.p0, b.p1, r->fmad != 0, fl, sk);
    if (e == cudaErrorNotSupported) return fail(PP_EUNSUPPORTED, "PP_OPT_PERSISTENT: shape not supported by the kernel");
    if (e != cudaSuccess) return cuda_fail(e, "persistent kernel launch");
    r->last_path = KPATH_TMA;
    std::vector<std::vector<int32_t>> h2d((size_t)P.nchunks), d2h((size_t)P.nchunks);
    for (size_t i = 0; i < P.ops.size(); ++i) {
        const Op &op = P.ops[i];
        if (op.kind == OpKind::H2D) h2d[(size_t)op.chunk].push_back((int32_t)i);
        if (op.kind == OpKind::D2H) d2h[(size_t)op.chunk].push_back((int32_t)i);
    }
    auto copy = [&](const Op &op, cudaStream_t st) {
        const auto &a = A[(size_t)op.arr];
        const size_t pb = (size_t)a.plane_bytes, bytes = (size_t)(op.p1 - op.p0) * pb;
        char *dev = (op.arr == 0 ? (char *)v[0].ring : (char *)v[1].ring) + (size_t)op.s0 * pb;
        char *host = (char *)a.host + (size_t)op.p0 * pb;
        return op.kind == OpKind::H2D ? cudaMemcpyAsync(dev, host, bytes, cudaMemcpyHostToDevice, st)
                                      : cudaMemcpyAsync(host, dev, bytes, cudaMemcpyDeviceToHost, st);
    };
    for (int64_t j = 0; j < P.nchunks; ++j) {
        // H2D of chunk j: its slots held planes of chunk j - S's window
        if (j >= P.S && (e = wait_value(sh, &fl->computed, (uint32_t)(j - P.S + 1))) != cudaSuccess)
            return cuda_fail(e, "cuStreamWaitValue32");
        for (int32_t i : h2d[(size_t)j])
            if ((e = copy(P.ops[(size_t)i], sh)) != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync");
        if ((e = write_value(sh, &fl->loaded, (uint32_t)(j + 1))) != cudaSuccess) return cuda_fail(e, "cuStreamWriteValue32");
        // D2H of chunk j once the kernel is done with it
        if ((e = wait_value(sd, &fl->computed, (uint32_t)(j + 1))) != cudaSuccess) return cuda_fail(e, "cuStreamWaitValue32");
        for (int32_t i : d2h[(size_t)j])
            if ((e = copy(P.ops[(size_t)i], sd)) != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync");
        if ((e = write_value(sd, &fl->drained, (uint32_t)(j + 1))) != cudaSuccess) return cuda_fail(e, "cuStreamWriteValue32");
    }
    for (int s = 1; s <= 2; ++s) {
        if ((e = cudaEventRecord(r->join[s], r->streams[s])) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
        if ((e = cudaStreamWaitEvent(sh, r->join[s], 0)) != cudaSuccess) return cuda_fail(e, "cudaStreamWaitEvent");
    }
    r->pipe_used = true;
    return PP_OK;
}

// after the launch: did a gate time out?
pp_status persistent_report(pp_region *r) {
    uint32_t err = 0;
    cudaError_t e = cudaMemcpy(&err, &((PipeFlags *)r->pipe_flags)->err, sizeof err, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) {
        r->poisoned = true;
        return cuda_fail(e, "persistent pipeline status");
    }
    if (err) return fail(PP_ECUDA, "PP_OPT_PERSISTENT: a chunk gate timed out; output planes are undefined");
    return PP_OK;
}

}  // namespace pprt
