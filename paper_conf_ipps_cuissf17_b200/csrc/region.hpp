// region.hpp — internal (not exported) definitions shared by the C-ABI translation units:
// the region object, the executor entry points and the built-in loop bodies.
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdint>
#include <string>
#include <vector>

#include "kernels.cuh"
#include "plan.hpp"
#include "ppipe.h"

namespace pprt {

pp_status fail(pp_status s, const std::string &msg);
pp_status cuda_fail(cudaError_t e, const char *what);
void set_last_error(const std::string &msg);
inline int64_t dtype_size(int dt) { return dt == PP_F32 ? 4 : 8; }

// Saves/restores the caller's current device around a region call.
struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev) {
        if (dev < 0) return;
        cudaGetDevice(&prev);
        if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard() {
        int cur;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

// The loop body of one chunk: enqueue the kernel for iterations [k0,k1) on `st`.
struct Body {
    virtual ~Body() = default;
    // level: the op's stage (1 for single sweeps; 1..T in a multi-sweep chain)
    virtual cudaError_t run(int64_t j, int64_t k0, int64_t k1, int level, const std::vector<pp::DView> &v,
                            cudaStream_t st, std::string *err) = 0;
    virtual bool graphable() const { return true; }
};

// A mirrored ring (vmm.cpp): `bytes` of device memory mapped at [va, va+bytes) and again at
// [va+bytes, va+2*bytes).
struct MirrorBuf {
    void *va = nullptr;
    uint64_t bytes = 0;
    unsigned long long handle = 0;
};
uint64_t vmm_granularity(int device);          // 0 if the device cannot mirror
pp_status mirror_alloc(int device, uint64_t bytes, MirrorBuf *out);
void mirror_free(MirrorBuf *m);

// Pinned bounce ring of a pageable host array (PP_OPT_BOUNCE; bounce.cpp): `nslots` pinned staging
// buffers between the pageable array and its device ring. Host memcpy worker threads fill / drain a
// slot inside a host function on a staging stream; the DMA waits for `ready`, the next reuse of the
// slot waits for `free`.
struct HostPool;
struct BounceRing {
    void *buf = nullptr;
    size_t slot_bytes = 0;
    int nslots = 0, next = 0;
    std::vector<cudaEvent_t> free_ev, ready_ev;
};
struct HostCopyJob {
    void *dst;
    const void *src;
    size_t bytes;
    HostPool *pool;
};

}  // namespace pprt

// One side of a peer halo exchange (pp_halo_export / pp_halo_import).
struct PeerHalo {
    int arr = -1;                               // -1: not set
    int64_t plane = 0;
    void *side = nullptr;
    int side_device = -1;
    uint32_t *flag = nullptr;
    uint32_t epoch = 0;
};

struct pp_region {
    int device = -1;
    PeerHalo halo_out, halo_in;                 // export (side slot) / import (peer copy)
    uint32_t *halo_err = nullptr;               // device word the import's wait sets on a timeout
    bool halo_used = false;                     // the pending launch imported a plane: check halo_err
    std::vector<pp::ArraySpec> arrs;
    int64_t chunk = 0;
    int S = 1;
    uint64_t mem_limit = 0;
    int policy = 1, graph = 0, fmad = 0, auto_pin = 1, kernel_path = pp::KPATH_AUTO, fault = 0, trace = 0, inplace = 0;
    int64_t sweeps = 1;                         // PP_OPT_SWEEPS (stencil launches)
    int64_t fuse = 1;                           // PP_OPT_FUSE: sweeps per kernel pass of a chain
    int64_t ring_extra = -1;
    int64_t mirror = 1;                         // PP_OPT_MIRROR: 0 off, 1 auto, > 1 forced granule bytes
    int d2h_interior = 0;                       // PP_OPT_D2H_INTERIOR: copy back output-plane interiors only
    int debug_tags = 0;                         // PP_OPT_DEBUG_TAGS: device-side schedule check
    int bounce = 1;                             // PP_OPT_BOUNCE: 0 off, 1 auto workers, n > 1 workers
    int64_t sm_copy = 0;                        // PP_OPT_SM_COPY: max bytes of an SM-driven copy (0 off)
    int persistent = 0;                         // PP_OPT_PERSISTENT: one resident kernel + flag gates
    int merge_copies = 1;                       // PP_OPT_MERGE_COPIES: one 2-D copy per run of array copies
    int64_t max_pitch = -1;                     // cudaDevAttrMaxPitch (queried on first use)
    int64_t merged = 0;                         // copies folded into another's 2-D copy by the last enqueue
    struct HostAlloc { const void *host = nullptr; intptr_t start = 0, size = 0; };
    std::vector<HostAlloc> host_alloc;          // per array: the host allocation holding it (merge check)
    void *pipe_flags = nullptr;                 // its PipeFlags (device memory)
    bool pipe_used = false;                     // the pending launch ran persistent: check its flags
    std::vector<pprt::BounceRing> bounce_rings; // per array (empty buffers for arrays that do not bounce)
    cudaStream_t stage_stream[2] = {nullptr, nullptr};   // host copies in (H2D) / out (D2H)
    cudaEvent_t stage_join[2] = {nullptr, nullptr};
    pprt::HostPool *pool = nullptr;
    std::vector<pprt::HostCopyJob> *jobs = nullptr;      // the launch's host copies (alive until it ends)
    bool bounce_used = false;
    // per launch in debug mode: tag arrays per ring, the error record, drains per output plane
    std::vector<int64_t *> dbg_tags;
    int64_t *dbg_err = nullptr;
    int32_t *dbg_visits = nullptr;
    std::vector<int64_t> dbg_voff;              // per ring: offset of its planes in dbg_visits (-1: none)
    int64_t dbg_nvisits = 0;
    bool dbg_pending = false;
    std::string dbg_first;                      // detail of the first violation of the last check
    bool mirror_failed = false;                 // auto mode fell back to plain rings after a VMM failure
    bool poisoned = false;

    std::vector<cudaStream_t> streams;
    bool borrowed_streams = false;
    std::vector<cudaEvent_t> events;            // op events (no timing)
    std::vector<cudaEvent_t> join;              // fork/join helpers
    std::vector<cudaEvent_t> tev;               // timing events (PP_OPT_TRACE): 2 per op
    std::vector<pp_trace_rec> trace_recs;
    bool trace_pending = false;
    cudaEvent_t t0 = nullptr, t1 = nullptr, th = nullptr, tk = nullptr;
    void *dbuf = nullptr;
    uint64_t dbuf_bytes = 0;
    bool borrowed_buf = false;
    std::vector<pprt::MirrorBuf> mirrors;       // per ring (plan.rings index); va null = not mirrored

    // plan cache
    bool plan_valid = false;
    pp::PlanParams plan_key;
    pp::Plan plan;

    // graph cache
    cudaGraphExec_t gexec = nullptr;
    std::vector<uint8_t> graph_key;

    // naive baseline
    std::vector<void *> naive;
    uint64_t naive_bytes = 0;

    pp_info info{};
    int last_path = 0, graph_path = 0;
    bool pending = false;                       // an async launch has not been waited for

    void invalidate() {
        plan_valid = false;
        drop_graph();
    }
    void drop_graph() {
        if (gexec) cudaGraphExecDestroy(gexec);
        gexec = nullptr;
        graph_key.clear();
    }
};


namespace pprt {

pp_status check_region(pp_region *r, bool need_device);
uint64_t resolve_budget(pp_region *r);
pp_status get_plan(pp_region *r, int64_t lo, int64_t hi, uint64_t budget);
pp_status finish_pending(pp_region *r);
pp_status run_launch(pp_region *r, int64_t lo, int64_t hi, Body &body, const void *key, size_t key_len,
                     bool wait);
// PP_OPT_D2H_INTERIOR: is array a's copy-back restricted to its planes' interiors, and are all
// outputs eligible (3-D, split on dim 0, on the host, at least 3 x 3 per plane)?
bool interior_d2h(const pp_region *r, const pp::ArraySpec &a);
pp_status check_interior_d2h(const pp_region *r);
// PP_OPT_BOUNCE (bounce.cpp): does array a's traffic go through a bounce ring; size the rings for the
// current plan; enqueue one staged copy; join the staging streams into s0; release everything.
bool bounced(const pp_region *r, const pp::ArraySpec &a);
pp_status bounce_prepare(pp_region *r);
cudaError_t bounce_h2d(pp_region *r, int arr, void *dev, const void *host, size_t bytes, cudaStream_t st);
cudaError_t bounce_d2h(pp_region *r, int arr, void *host, const void *dev, size_t bytes, cudaStream_t st);
cudaError_t bounce_join(pp_region *r, cudaStream_t s0);
void bounce_free(pp_region *r);
// PP_OPT_PERSISTENT (persist.cpp)
bool persistent_eligible(const pp_region *r, const Body &body, std::string *why);
pp_status enqueue_persistent(pp_region *r, Body &body, int64_t lo, int64_t hi);
pp_status persistent_report(pp_region *r);
std::vector<pp::DView> views_for(pp_region *r);
// D2H of planes [p0, p0+n) of 3-D array a, interior rows/columns only: device planes start at `dev`
cudaError_t copy_interior_d2h(const pp::ArraySpec &a, const void *dev, int64_t p0, int64_t n, cudaStream_t st);

struct BuiltinBody : Body {
    pp_region *r;
    pp_kernel k;
    double p0 = 0, p1 = 0;
    int64_t lo = 0, hi = 0;                     // the launch's loop range (chain boundary planes)
    BuiltinBody(pp_region *r_, pp_kernel k_) : r(r_), k(k_) {}
    cudaError_t run(int64_t, int64_t k0, int64_t k1, int level, const std::vector<pp::DView> &v,
                    cudaStream_t st, std::string *) override {
        const auto &A = r->arrs;
        switch (k) {
        case PP_K_TRIAD:
            return pp::launch_triad(A[0].dtype, v[0], A[0].off, v[1], A[1].off, v[2], A[2].off, k0, k1, p0,
                                r->fmad != 0, st);
        case PP_K_STENCIL7: {
            int used = 0;
            cudaError_t e;
            if (r->sweeps > 1) {
                // chain stage ending at level `level`: ring of the previous stage end -> ring of this
                // one (0 = A0 ring, 1 = output ring, device-only stage rings after the mapped arrays);
                // planes outside [lo,hi) are copies. A stage of h > 1 levels is one fused pass.
                const int64_t T = r->sweeps, L = std::min(r->fuse, T), G = (T + L - 1) / L;
                const int64_t s = (level + L - 1) / L, h = level - (s - 1) * L;
                const int in = s == 1 ? 0 : (int)s;
                const int out = s == G ? 1 : (int)(1 + s);
                if (h > 1) {
                    e = pp::launch_stencil7_fused(A[0].dtype, (int)h, v[in], v[out], A[0].ext[1], A[0].ext[2], k0, k1,
                                                  lo - 1, hi + 1, lo, hi, p0, p1, r->fmad != 0, st);
                    used = pp::KPATH_TMA;
                } else {
                    e = pp::launch_stencil7(A[0].dtype, v[in], 0, v[out], 0, A[0].ext[1], A[0].ext[2], k0, k1, lo, hi,
                                            p0, p1, r->fmad != 0, r->kernel_path, &used, st);
                }
            } else {
                e = pp::launch_stencil7(A[0].dtype, v[0], A[0].off + 1, v[1], A[1].off, A[0].ext[1], A[0].ext[2],
                                        k0, k1, INT64_MIN, INT64_MAX, p0, p1, r->fmad != 0, r->kernel_path,
                                        &used, st);
            }
            r->last_path = std::max(r->last_path, used);
            return e;
        }
        case PP_K_PROBE:
            return pp::launch_probe(v[0], A[0].off + 1, v[1], A[1].off, k0, k1, st);
        case PP_K_CONV3D: {
            int used = 0;
            cudaError_t e = pp::launch_conv3d(A[0].dtype, v[0], A[0].off + 1, v[1], A[1].off, A[0].ext[1],
                                              A[0].ext[2], k0, k1, r->kernel_path, &used, st);
            r->last_path = std::max(r->last_path, used);
            return e;
        }
        }
        return cudaErrorInvalidValue;
    }
};

pp_status bind_builtin(pp_region *r, pp_kernel k, const void *args, size_t args_size, BuiltinBody *b);

}  // namespace pprt
