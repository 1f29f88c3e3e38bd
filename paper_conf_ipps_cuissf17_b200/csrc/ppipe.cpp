// ppipe.cpp — the C ABI (include/ppipe.h): regions, the CUDA executor (multi-stream scheduler with
// event-gated ring-slot reuse), optional CUDA-graph replay, the naive
// synchronous baseline, the host-link probe, and error handling.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "region.hpp"

using namespace pp;

namespace pprt {

thread_local std::string g_last_error;

pp_status fail(pp_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

pp_status cuda_fail(cudaError_t e, const char *what) {
    std::string m = std::string(what) + ": " + cudaGetErrorString(e);
    g_last_error = m;
    return PP_ECUDA;
}

void set_last_error(const std::string &msg) { g_last_error = msg; }

}  // namespace pprt

using namespace pprt;

namespace pprt {

pp_status check_region(pp_region *r, bool need_device) {
    if (!r) return fail(PP_EINVAL, "null region");
    if (r->poisoned) return fail(PP_ESTATE, "region poisoned by an earlier failure; destroy it");
    if (need_device && r->device < 0) return fail(PP_ESTATE, "host-only region (device = -1)");
    return PP_OK;
}

PlanParams params_for(pp_region *r, int64_t lo, int64_t hi, uint64_t budget) {
    PlanParams p;
    p.lo = lo;
    p.hi = hi;
    p.chunk = r->chunk;
    p.streams = r->S;
    p.budget = budget;
    p.policy = r->policy;
    p.ring_extra = r->ring_extra;
    p.fault = r->fault;
    p.sweeps = r->sweeps;
    p.fuse = r->fuse;
    // mirrored rings need memory the region allocates itself (not a borrowed buffer)
    if (r->mirror > 1) p.mirror_gran = (uint64_t)r->mirror;
    else if (r->mirror == 1 && !r->borrowed_buf && !r->mirror_failed && r->device >= 0)
        p.mirror_gran = vmm_granularity(r->device);
    return p;
}

bool same_params(const PlanParams &a, const PlanParams &b) {
    return a.lo == b.lo && a.hi == b.hi && a.chunk == b.chunk && a.streams == b.streams &&
           a.budget == b.budget && a.policy == b.policy && a.ring_extra == b.ring_extra &&
           a.fault == b.fault && a.sweeps == b.sweeps &&
           a.fuse == b.fuse && a.mirror_gran == b.mirror_gran;
}

pp_status get_plan(pp_region *r, int64_t lo, int64_t hi, uint64_t budget) {
    PlanParams p = params_for(r, lo, hi, budget);
    if (r->plan_valid) {
        // The budget may drift between launches (it defaults to free device memory); the cached
        // plan stays valid as long as the budget resolves to the same chunk size and stream count.
        PlanParams q = r->plan_key;
        q.budget = p.budget;
        if (same_params(p, q)) {
            int64_t c = 0;
            int S = 0;
            std::string m;
            if (resolve(r->arrs, p, &c, &S, &m) == OK && c == r->plan.c && S == r->plan.S) return PP_OK;
        }
    }
    std::string msg;
    Plan P;
    int rc = build_plan(r->arrs, p, &P, &msg);
    if (rc != OK) return fail((pp_status)rc, msg);
    r->plan = std::move(P);
    r->plan_key = p;
    r->plan_valid = true;
    r->drop_graph();
    return PP_OK;
}

uint64_t resolve_budget(pp_region *r) {
    if (r->mem_limit) return r->mem_limit;
    // cudaMemGetInfo costs 0.3-10 ms on the target VM: the default budget (free HBM) is resolved once
    // per configuration and reused while the cached plan stays valid
    if (r->plan_valid) return r->plan_key.budget;
    if (r->device < 0) return ~uint64_t(0) >> 1;
    size_t fr = 0, tot = 0;
    cudaMemGetInfo(&fr, &tot);
    uint64_t avail = (uint64_t)fr + (r->borrowed_buf ? 0 : r->dbuf_bytes);
    for (const auto &m : r->mirrors) avail += m.bytes;
    const uint64_t margin = 512ull << 20;
    return avail > margin ? avail - margin : avail / 2;
}

pp_status ensure_streams(pp_region *r, int n) {
    if (r->borrowed_streams) {
        if ((int)r->streams.size() < n)
            return fail(PP_EINVAL, "the schedule needs " + std::to_string(n) + " streams but only " +
                                       std::to_string(r->streams.size()) + " were borrowed");
        return PP_OK;
    }
    while ((int)r->streams.size() < n) {
        cudaStream_t s;
        cudaError_t e = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamCreate");
        r->streams.push_back(s);
    }
    return PP_OK;
}

pp_status ensure_events(pp_region *r, size_t nev, size_t njoin) {
    auto grow = [&](std::vector<cudaEvent_t> &v, size_t n) -> cudaError_t {
        while (v.size() < n) {
            cudaEvent_t e;
            cudaError_t x = cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
            if (x != cudaSuccess) return x;
            v.push_back(e);
        }
        return cudaSuccess;
    };
    cudaError_t e = grow(r->events, nev);
    if (e == cudaSuccess) e = grow(r->join, njoin);
    if (e == cudaSuccess && !r->t0) {
        e = cudaEventCreate(&r->t0);
        if (e == cudaSuccess) e = cudaEventCreate(&r->t1);
        if (e == cudaSuccess) e = cudaEventCreate(&r->th);
        if (e == cudaSuccess) e = cudaEventCreate(&r->tk);
    }
    return e == cudaSuccess ? PP_OK : cuda_fail(e, "cudaEventCreate");
}

pp_status ensure_dbuf(pp_region *r, uint64_t bytes) {
    if (bytes == 0) return PP_OK;
    if (r->borrowed_buf) {
        if (r->dbuf_bytes < bytes) return fail(PP_EBUDGET, "borrowed device buffer smaller than the rings");
        return PP_OK;
    }
    if (r->dbuf_bytes >= bytes) return PP_OK;
    if (r->dbuf) cudaFree(r->dbuf);
    r->dbuf = nullptr;
    r->dbuf_bytes = 0;
    r->drop_graph();
    cudaError_t e = cudaMalloc(&r->dbuf, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(PP_ENOMEM, std::string("cudaMalloc of ring buffer: ") + cudaGetErrorString(e));
    }
    r->dbuf_bytes = bytes;
    return PP_OK;
}

// The plan's rings: non-mirrored ones inside the one plain buffer, each mirrored one in its own VMM
// range (allocated, or re-allocated when its size changed, here).
pp_status ensure_rings(pp_region *r) {
    const Plan &P = r->plan;
    if (r->mirrors.size() < P.rings.size()) r->mirrors.resize(P.rings.size());
    auto keep = [&](size_t i) {
        return i < P.rings.size() && P.rings[i].mirror && r->mirrors[i].va && r->mirrors[i].bytes == P.rings[i].bytes;
    };
    // release the mirrors this plan does not reuse first, so their memory is free for what follows
    bool synced = false;
    for (size_t i = 0; i < r->mirrors.size(); ++i) {
        if (!r->mirrors[i].va || keep(i)) continue;
        if (!synced) { cudaDeviceSynchronize(); synced = true; }   // earlier launches may still use it
        mirror_free(&r->mirrors[i]);
        r->drop_graph();
    }
    pp_status s = ensure_dbuf(r, P.plain_bytes);
    if (s) return s;
    for (size_t i = 0; i < P.rings.size(); ++i) {
        if (!P.rings[i].mirror || r->mirrors[i].va) continue;
        r->drop_graph();
        if ((s = mirror_alloc(r->device, P.rings[i].bytes, &r->mirrors[i]))) return s;
    }
    return PP_OK;
}

// device address of ring i's slot 0
static inline char *ring_ptr(pp_region *r, size_t i) {
    const Ring &rg = r->plan.rings[i];
    return rg.mirror ? (char *)r->mirrors[i].va : (char *)r->dbuf + rg.offset;
}

std::vector<DView> views_for(pp_region *r) {
    // one view per ring: the mapped arrays first, then any device-only level rings of a chain
    std::vector<DView> v(r->plan.rings.size());
    for (size_t i = 0; i < r->plan.rings.size(); ++i) {
        const Ring &rg = r->plan.rings[i];
        if (i < r->arrs.size() && r->arrs[i].resident) {
            const auto &a = r->arrs[i];
            v[i] = DView{a.host, a.nsplit, 0, a.plane_elems, a.outer, a.nsplit * a.inner};
        } else if (i < r->arrs.size()) {
            const auto &a = r->arrs[i];   // ring layout [outer][R][inner]
            v[i] = DView{ring_ptr(r, i), rg.R, rg.base, rg.plane_elems, a.outer, rg.R * a.inner};
        } else {
            v[i] = DView{ring_ptr(r, i), rg.R, rg.base, rg.plane_elems, 1, 0};
        }
    }
    return v;
}

static pp_status dbg_report(pp_region *r);

// Wait for an outstanding (async) launch; fills info.last_ms. Poisons the region on failure.
pp_status finish_pending(pp_region *r) {
    if (!r->pending) return PP_OK;
    r->pending = false;
    cudaError_t e = cudaEventSynchronize(r->t1);
    if (e != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "launch execution"); }
    float ms = 0;
    cudaEventElapsedTime(&ms, r->t0, r->t1);
    r->info.last_ms = ms;
    if (r->pipe_used) {                              // PP_OPT_PERSISTENT: did every chunk gate open?
        r->pipe_used = false;
        pp_status ps = persistent_report(r);
        if (ps) return ps;
    }
    if (r->dbg_pending) {                            // PP_OPT_DEBUG_TAGS: what the device saw
        r->dbg_pending = false;
        pp_status ds = dbg_report(r);
        if (ds) return ds;
    }
    if (r->halo_used) {                              // did the peer's side slot arrive in time?
        r->halo_used = false;
        uint32_t err = 0;
        if ((e = cudaMemcpy(&err, r->halo_err, sizeof err, cudaMemcpyDeviceToHost)) != cudaSuccess) {
            r->poisoned = true;
            return cuda_fail(e, "peer halo status");
        }
        if (err) {
            cudaMemset(r->halo_err, 0, sizeof err);
            return fail(PP_ECUDA, "peer halo: the side slot's flag did not reach the epoch within 10 s "
                                  "(exporter not running?); output planes are undefined");
        }
    }
    if (r->trace_pending) {
        r->trace_pending = false;
        const Plan &P = r->plan;
        r->trace_recs.assign(P.ops.size(), pp_trace_rec{});
        for (size_t i = 0; i < P.ops.size(); ++i) {
            const Op &op = P.ops[i];
            pp_trace_rec &t = r->trace_recs[i];
            t.kind = (int32_t)op.kind;
            t.stream = op.stream;
            t.chunk = op.chunk;
            t.array = op.arr;
            t.p0 = op.p0;
            t.p1 = op.p1;
            const auto &arr = r->arrs[op.arr];
            t.bytes = op.kind == OpKind::KER ? 0
                      : (uint64_t)(op.p1 - op.p0) * (uint64_t)(op.kind == OpKind::D2H && interior_d2h(r, arr)
                                                                   ? (arr.ext[1] - 2) * (arr.ext[2] - 2) * arr.esize
                                                                   : arr.plane_bytes);
            float a = 0, b = 0;
            cudaEventElapsedTime(&a, r->t0, r->tev[2 * i]);
            cudaEventElapsedTime(&b, r->t0, r->tev[2 * i + 1]);
            t.start_ms = a;
            t.end_ms = b;
        }
    }
    return PP_OK;
}

// ---- PP_OPT_DEBUG_TAGS: per-launch device buffers, the check/stamp kernels around each op, the report
static void dbg_free(pp_region *r) {
    for (int64_t *t : r->dbg_tags)
        if (t) cudaFree(t);
    r->dbg_tags.clear();
    if (r->dbg_err) cudaFree(r->dbg_err);
    if (r->dbg_visits) cudaFree(r->dbg_visits);
    r->dbg_err = nullptr;
    r->dbg_visits = nullptr;
    r->dbg_nvisits = 0;
}

static pp_status dbg_alloc(pp_region *r) {
    const Plan &P = r->plan;
    dbg_free(r);
    cudaError_t e = cudaSuccess;
    r->dbg_tags.assign(P.rings.size(), nullptr);
    r->dbg_voff.assign(P.rings.size(), -1);
    for (size_t i = 0; i < P.rings.size() && e == cudaSuccess; ++i) {
        if (P.rings[i].R <= 0) continue;
        e = cudaMalloc(&r->dbg_tags[i], (size_t)P.rings[i].R * sizeof(int64_t));
        if (e == cudaSuccess) e = cudaMemset(r->dbg_tags[i], 0xff, (size_t)P.rings[i].R * sizeof(int64_t));
    }
    for (size_t i = 0; i < P.out_lo.size() && i < P.rings.size(); ++i)
        if (P.out_hi[i] > P.out_lo[i]) {
            r->dbg_voff[i] = r->dbg_nvisits;
            r->dbg_nvisits += P.out_hi[i] - P.out_lo[i];
        }
    if (e == cudaSuccess) e = cudaMalloc(&r->dbg_err, 5 * sizeof(int64_t));
    if (e == cudaSuccess) e = cudaMemset(r->dbg_err, 0, 5 * sizeof(int64_t));
    if (e == cudaSuccess && r->dbg_nvisits) e = cudaMalloc(&r->dbg_visits, (size_t)r->dbg_nvisits * sizeof(int32_t));
    if (e == cudaSuccess && r->dbg_nvisits) e = cudaMemset(r->dbg_visits, 0, (size_t)r->dbg_nvisits * sizeof(int32_t));
    if (e != cudaSuccess) {
        cudaGetLastError();
        dbg_free(r);
        return fail(PP_ENOMEM, "PP_OPT_DEBUG_TAGS buffers");
    }
    return PP_OK;
}

// phase 0: check the slots op i reads (before it); phase 1: stamp the slots it wrote (after it)
static cudaError_t dbg_op(pp_region *r, size_t i, int phase, cudaStream_t st) {
    const Plan &P = r->plan;
    const Op &op = P.ops[i];
    TagOp t{};
    t.op = (int32_t)i;
    for (int32_t k = 0; k < op.acc_count && t.n < kTagAccMax; ++k) {
        const Acc &ac = P.accs[(size_t)(op.acc_begin + k)];
        if ((phase == 1) != ac.write) continue;
        const Ring &rg = P.rings[(size_t)ac.arr];
        if (rg.R <= 0 || !r->dbg_tags[(size_t)ac.arr]) continue;
        TagAcc &a = t.a[t.n++];
        a.tags = r->dbg_tags[(size_t)ac.arr];
        a.R = rg.R;
        // copies use the slot the executor copies from/to (op.s0); kernels the ring's slot map
        a.s0 = op.kind == OpKind::KER ? pmod(ac.p0 - rg.base, rg.R) : op.s0;
        a.p0 = ac.p0;
        a.p1 = ac.p1;
        a.level = ac.level;
        a.write = ac.write;
        if (op.kind == OpKind::D2H && r->dbg_voff[(size_t)ac.arr] >= 0) {
            a.visits = r->dbg_visits + r->dbg_voff[(size_t)ac.arr];
            a.vbase = P.out_lo[(size_t)ac.arr];
        }
    }
    if (!t.n) return cudaSuccess;
    return launch_tags(t, phase, r->dbg_err, st);
}

// after the launch: tag mismatches + output planes not drained exactly once
static pp_status dbg_report(pp_region *r) {
    int64_t err[5] = {0, 0, 0, 0, 0};
    cudaError_t e = cudaMemcpy(err, r->dbg_err, sizeof err, cudaMemcpyDeviceToHost);
    std::vector<int32_t> v((size_t)r->dbg_nvisits);
    if (e == cudaSuccess && r->dbg_nvisits)
        e = cudaMemcpy(v.data(), r->dbg_visits, v.size() * sizeof(int32_t), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) {
        dbg_free(r);
        r->poisoned = true;
        return cuda_fail(e, "PP_OPT_DEBUG_TAGS report");
    }
    int64_t bad = err[0];
    int64_t first_visit = -1;
    for (size_t k = 0; k < v.size(); ++k)
        if (v[k] != 1) {
            ++bad;
            if (first_visit < 0) first_visit = (int64_t)k;
        }
    r->info.debug_violations = bad;
    r->dbg_first.clear();
    if (err[0])
        r->dbg_first = "op " + std::to_string(err[1]) + " access " + std::to_string(err[2]) + " plane " +
                       std::to_string(err[3]) + ": slot tag " + std::to_string(err[4]) + " (plane " +
                       std::to_string(err[4] >> 8) + ", level " + std::to_string(err[4] & 255) + ")";
    else if (first_visit >= 0)
        r->dbg_first = "output plane index " + std::to_string(first_visit) + " drained " +
                       std::to_string(v[(size_t)first_visit]) + " times";
    if (bad) set_last_error("PP_OPT_DEBUG_TAGS: " + std::to_string(bad) + " violations; first: " + r->dbg_first);
    dbg_free(r);
    return PP_OK;
}

bool interior_d2h(const pp_region *r, const pp::ArraySpec &a) {
    return r->d2h_interior && a.is_output() && a.ndim == 3 && a.split_dim == 0 && !a.resident && a.ext[1] >= 3 &&
           a.ext[2] >= 3;
}

pp_status check_interior_d2h(const pp_region *r) {
    if (!r->d2h_interior) return PP_OK;
    for (const auto &a : r->arrs)
        if (a.is_output() && !interior_d2h(r, a))
            return fail(PP_EUNSUPPORTED, "PP_OPT_D2H_INTERIOR needs host outputs that are 3-D [nz][ny][nx] arrays "
                                         "split on dim 0 with ny, nx >= 3");
    return PP_OK;
}

// One 3-D copy: x = bytes of columns 1..nx-2, y = rows 1..ny-2, z = planes; both sides have the
// array's row pitch and plane height, so the slot run on the device (contiguous, also across a
// mirrored ring's wrap) and the host planes are addressed alike.
cudaError_t copy_interior_d2h(const pp::ArraySpec &a, const void *dev, int64_t p0, int64_t n, cudaStream_t st) {
    const size_t ny = (size_t)a.ext[1], nx = (size_t)a.ext[2], e = (size_t)a.esize;
    cudaMemcpy3DParms m = {};
    m.srcPtr = make_cudaPitchedPtr(const_cast<void *>(dev), nx * e, nx, ny);
    m.srcPos = make_cudaPos(e, 1, 0);
    m.dstPtr = make_cudaPitchedPtr(a.host, nx * e, nx, ny);
    m.dstPos = make_cudaPos(e, 1, (size_t)p0);
    m.extent = make_cudaExtent((nx - 2) * e, ny - 2, (size_t)n);
    m.kind = cudaMemcpyDeviceToHost;
    return cudaMemcpy3DAsync(&m, st);
}

// The host allocation (pinned or registered) holding array i, via the driver's pointer range
// attributes; {0, 0} if unknown. A 2-D copy must stay inside one allocation on each side.
static pp_region::HostAlloc host_alloc_of(pp_region *r, size_t i) {
    typedef CUresult (*PFN_ptrattr)(void *, CUpointer_attribute, CUdeviceptr);
    static PFN_ptrattr fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        PFN_ptrattr f = nullptr;
        if (cudaGetDriverEntryPoint("cuPointerGetAttribute", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            f = (PFN_ptrattr)p;
        cudaGetLastError();
        return f;
    }();
    if (r->host_alloc.size() < r->arrs.size()) r->host_alloc.resize(r->arrs.size());
    pp_region::HostAlloc &h = r->host_alloc[i];
    const void *host = r->arrs[i].host;
    if (h.host != host) {
        h = pp_region::HostAlloc{host, 0, 0};
        CUdeviceptr start = 0;
        size_t size = 0;
        if (fn && fn(&start, CU_POINTER_ATTRIBUTE_RANGE_START_ADDR, (CUdeviceptr)host) == CUDA_SUCCESS &&
            fn(&size, CU_POINTER_ATTRIBUTE_RANGE_SIZE, (CUdeviceptr)host) == CUDA_SUCCESS) {
            h.start = (intptr_t)start;
            h.size = (intptr_t)size;
        }
    }
    return h;
}

// PP_OPT_MERGE_COPIES: the run of copies starting at op i that can go out as one 2-D copy — the next
// ops on the same stream move the same planes [p0,p1) of arrays with the same plane bytes in the same
// direction for the same chunk, with constant positive host and device distances between
// consecutive arrays' pieces. Returns the run length (1 = no merge) and the two pitches.
static int merge_run(pp_region *r, const Plan &P, size_t i, size_t *hpitch, size_t *dpitch) {
    const Op &op = P.ops[i];
    if (!r->merge_copies || r->trace || r->dbg_pending || op.kind == OpKind::KER) return 1;
    auto plain = [&](const Op &o) {
        const auto &a = r->arrs[(size_t)o.arr];
        // device side: both rings in the one plain ring buffer (a mirrored ring is its own mapping)
        if (P.rings[(size_t)o.arr].mirror) return false;
        const int64_t bytes = (o.p1 - o.p0) * a.plane_bytes;
        const bool halo = (r->halo_in.arr == o.arr && r->halo_in.plane >= o.p0 && r->halo_in.plane < o.p1) ||
                          (r->halo_out.arr == o.arr && r->halo_out.plane >= o.p0 && r->halo_out.plane < o.p1);
        return a.outer == 1 && a.pinned && !halo && !interior_d2h(r, a) && !(r->bounce_used && bounced(r, a)) &&
               bytes > r->sm_copy;
    };
    if (!plain(op)) return 1;
    if (r->max_pitch < 0) {
        int mp = 0;
        r->max_pitch = cudaDeviceGetAttribute(&mp, cudaDevAttrMaxPitch, r->device) == cudaSuccess ? mp : 0;
    }
    const auto &a0 = r->arrs[(size_t)op.arr];
    auto dev_of = [&](const Op &o) {
        return (intptr_t)(ring_ptr(r, (size_t)o.arr) + (size_t)o.s0 * (size_t)r->arrs[(size_t)o.arr].plane_bytes);
    };
    auto host_of = [&](const Op &o) {
        const auto &a = r->arrs[(size_t)o.arr];
        return (intptr_t)((const char *)a.host + (size_t)o.p0 * (size_t)a.plane_bytes);
    };
    const intptr_t width = (intptr_t)((op.p1 - op.p0) * a0.plane_bytes);
    int k = 1;
    intptr_t hp = 0, dp = 0;
    for (size_t j = i + 1; j < P.ops.size(); ++j, ++k) {
        const Op &o = P.ops[j], &prev = P.ops[j - 1];
        if (o.kind != op.kind || o.stream != op.stream || o.chunk != op.chunk || o.p0 != op.p0 || o.p1 != op.p1 ||
            r->arrs[(size_t)o.arr].plane_bytes != a0.plane_bytes || !plain(o))
            break;
        const intptr_t h = host_of(o) - host_of(prev), d = dev_of(o) - dev_of(prev);
        if (k == 1) {
            if (h < width || d < width || h > r->max_pitch || d > r->max_pitch) break;
            hp = h;
            dp = d;
        } else if (h != hp || d != dp) {
            break;
        }
        // host side: every row inside the first array's allocation
        const pp_region::HostAlloc ha = host_alloc_of(r, (size_t)op.arr);
        if (!ha.size || host_of(op) < ha.start || host_of(o) + width > ha.start + ha.size) break;
    }
    *hpitch = (size_t)hp;
    *dpitch = (size_t)dp;
    return k;
}

// Enqueue the whole plan on the region's streams (fork from streams[0], join back to it).
pp_status enqueue_plan(pp_region *r, Body &body) {
    const Plan &P = r->plan;
    const PdlScope pdl(r->sweeps > 1);                  // chains: level kernels back to back (PDL)
    const int ns = P.nstreams;
    cudaStream_t s0 = r->streams[0];
    std::vector<DView> v = views_for(r);
    std::vector<int32_t> ev_of(P.ops.size(), -1);
    int32_t nev = 0;
    r->merged = 0;
    for (size_t i = 0; i < P.ops.size(); ++i)
        if (P.ops[i].need_event) ev_of[i] = nev++;
    cudaError_t e;
    // fork
    if (ns > 1) {
        if ((e = cudaEventRecord(r->join[0], s0)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
        for (int s = 1; s < ns; ++s)
            if ((e = cudaStreamWaitEvent(r->streams[s], r->join[0], 0)) != cudaSuccess)
                return cuda_fail(e, "cudaStreamWaitEvent");
    }
    std::string err;
    for (size_t i = 0; i < P.ops.size(); ++i) {
        const Op &op = P.ops[i];
        cudaStream_t st = r->streams[op.stream];
        size_t hpitch = 0, dpitch = 0;
        if (const int k = merge_run(r, P, i, &hpitch, &dpitch); k > 1) {
            // one 2-D copy for ops i .. i+k-1: every op's waits first, every op's event after
            for (int m = 0; m < k; ++m)
                for (int32_t d = 0; d < P.ops[i + m].dep_count; ++d)
                    if ((e = cudaStreamWaitEvent(st, r->events[ev_of[P.deps[P.ops[i + m].dep_begin + d]]], 0)) !=
                        cudaSuccess)
                        return cuda_fail(e, "cudaStreamWaitEvent");
            const auto &a = r->arrs[op.arr];
            const size_t width = (size_t)(op.p1 - op.p0) * (size_t)a.plane_bytes;
            char *dev = ring_ptr(r, (size_t)op.arr) + (size_t)op.s0 * (size_t)a.plane_bytes;
            char *host = (char *)a.host + (size_t)op.p0 * (size_t)a.plane_bytes;
            e = op.kind == OpKind::H2D
                    ? cudaMemcpy2DAsync(dev, dpitch, host, hpitch, width, (size_t)k, cudaMemcpyHostToDevice, st)
                    : cudaMemcpy2DAsync(host, hpitch, dev, dpitch, width, (size_t)k, cudaMemcpyDeviceToHost, st);
            if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy2DAsync (merged copies)");
            for (int m = 0; m < k; ++m)
                if (P.ops[i + m].need_event && (e = cudaEventRecord(r->events[ev_of[i + m]], st)) != cudaSuccess)
                    return cuda_fail(e, "cudaEventRecord");
            r->merged += k - 1;
            i += (size_t)k - 1;
            continue;
        }
        for (int32_t d = 0; d < op.dep_count; ++d) {
            int32_t dep = P.deps[op.dep_begin + d];
            if ((e = cudaStreamWaitEvent(st, r->events[ev_of[dep]], 0)) != cudaSuccess)
                return cuda_fail(e, "cudaStreamWaitEvent");
        }
        const bool tr = r->trace && r->tev.size() >= 2 * P.ops.size();
        if (r->dbg_pending && (e = dbg_op(r, i, 0, st)) != cudaSuccess) return cuda_fail(e, "debug tag check");
        if (tr && (e = cudaEventRecord(r->tev[2 * i], st)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
        if (op.kind == OpKind::KER) {
            e = body.run(op.chunk, op.p0, op.p1, op.level, v, st, &err);
            if (e != cudaSuccess) {
                if (e == cudaErrorUnknown && !err.empty()) return fail(PP_EINVAL, err);
                if (e == cudaErrorNotSupported)
                    return fail(PP_EUNSUPPORTED, "requested kernel path does not support this shape/alignment");
                return cuda_fail(e, "kernel launch");
            }
        } else {
            const auto &a = r->arrs[op.arr];
            const Ring &rg = P.rings[op.arr];
            if (a.outer == 1) {
                size_t bytes = (size_t)(op.p1 - op.p0) * (size_t)a.plane_bytes;
                // (a mirrored ring continues past slot R - 1 into its second mapping)
                char *dev = ring_ptr(r, (size_t)op.arr) + (size_t)op.s0 * (size_t)a.plane_bytes;
                char *host = (char *)a.host + (size_t)op.p0 * (size_t)a.plane_bytes;
                const size_t pb = (size_t)a.plane_bytes;
                const PeerHalo &hin = r->halo_in, &hout = r->halo_out;
                if (op.kind == OpKind::H2D && hin.arr == op.arr && hin.plane >= op.p0 && hin.plane < op.p1) {
                    // the imported plane comes from the peer's side slot once its flag shows the epoch
                    const size_t q = (size_t)(hin.plane - op.p0), rest = (size_t)(op.p1 - hin.plane - 1);
                    e = q ? cudaMemcpyAsync(dev, host, q * pb, cudaMemcpyHostToDevice, st) : cudaSuccess;
                    if (e == cudaSuccess) e = launch_flag_wait(hin.flag, hin.epoch, 10000000000ull, r->halo_err, st);
                    if (e == cudaSuccess)
                        e = cudaMemcpyPeerAsync(dev + q * pb, r->device, hin.side, hin.side_device, pb, st);
                    if (e == cudaSuccess && rest)
                        e = cudaMemcpyAsync(dev + (q + 1) * pb, host + (q + 1) * pb, rest * pb, cudaMemcpyHostToDevice, st);
                } else if (a.pinned && (int64_t)bytes <= r->sm_copy && !interior_d2h(r, a) &&
                           ((uintptr_t)dev | (uintptr_t)host) % 16 == 0) {
                    e = op.kind == OpKind::H2D ? launch_sm_copy(dev, host, bytes, st) : launch_sm_copy(host, dev, bytes, st);
                } else if (op.kind == OpKind::H2D) {
                    e = r->bounce_used && bounced(r, a) ? bounce_h2d(r, op.arr, dev, host, bytes, st)
                                                        : cudaMemcpyAsync(dev, host, bytes, cudaMemcpyHostToDevice, st);
                } else if (interior_d2h(r, a)) {
                    e = copy_interior_d2h(a, dev, op.p0, op.p1 - op.p0, st);
                } else {
                    e = r->bounce_used && bounced(r, a) ? bounce_d2h(r, op.arr, host, dev, bytes, st)
                                                        : cudaMemcpyAsync(host, dev, bytes, cudaMemcpyDeviceToHost, st);
                }
                if (e == cudaSuccess && op.kind == OpKind::H2D && hout.arr == op.arr && hout.plane >= op.p0 &&
                    hout.plane < op.p1) {
                    // exported plane: keep a copy in the side slot, then publish the epoch
                    e = cudaMemcpyAsync(hout.side, dev + (size_t)(hout.plane - op.p0) * pb, pb,
                                        cudaMemcpyDeviceToDevice, st);
                    if (e == cudaSuccess) e = launch_flag_set(hout.flag, hout.epoch, st);
                }
            } else {
                // 2-D block region: `outer` rows of (p1-p0)*inner elements, pitched on both
                // sides (the paper's cudaMallocPitch + cudaMemcpy2DAsync data regions)
                const size_t row = (size_t)a.inner * (size_t)a.esize;
                const size_t width = (size_t)(op.p1 - op.p0) * row;
                char *dev = ring_ptr(r, (size_t)op.arr) + (size_t)op.s0 * row;
                char *host = (char *)a.host + (size_t)op.p0 * row;
                const size_t dpitch = (size_t)rg.R * row, hpitch = (size_t)a.nsplit * row;
                if (op.kind == OpKind::H2D)
                    e = cudaMemcpy2DAsync(dev, dpitch, host, hpitch, width, (size_t)a.outer, cudaMemcpyHostToDevice, st);
                else
                    e = cudaMemcpy2DAsync(host, hpitch, dev, dpitch, width, (size_t)a.outer, cudaMemcpyDeviceToHost, st);
            }
            if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync");
        }
        if (tr && (e = cudaEventRecord(r->tev[2 * i + 1], st)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
        if (r->dbg_pending && (e = dbg_op(r, i, 1, st)) != cudaSuccess) return cuda_fail(e, "debug tag stamp");
        if (op.need_event)
            if ((e = cudaEventRecord(r->events[ev_of[i]], st)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
    }
    // join (the bounce ring's staging streams too: the last host copies end the launch)
    if ((e = bounce_join(r, s0)) != cudaSuccess) return cuda_fail(e, "bounce join");
    for (int s = 1; s < ns; ++s) {
        if ((e = cudaEventRecord(r->join[s], r->streams[s])) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
        if ((e = cudaStreamWaitEvent(s0, r->join[s], 0)) != cudaSuccess) return cuda_fail(e, "cudaStreamWaitEvent");
    }
    return PP_OK;
}

pp_status run_launch(pp_region *r, int64_t lo, int64_t hi, Body &body, const void *key, size_t key_len,
                     bool wait) {
    pp_status s = check_region(r, true);
    if (s) return s;
    DeviceGuard g(r->device);
    if (!g.ok) return fail(PP_ECUDA, "cudaSetDevice failed");
    if (hi < lo) return fail(PP_EINVAL, "hi < lo");
    if ((s = check_interior_d2h(r))) return s;
    // A previous async launch needs no host wait: it ended by joining every stream into streams[0],
    // and this launch forks all its streams from streams[0], so the device orders them. Its
    // last_ms is dropped (t0/t1 are re-recorded).
    r->pending = false;
    static const bool dbg = getenv("PP_DEBUG_TIMING") != nullptr;
    auto now = [] { return std::chrono::steady_clock::now(); };
    auto us = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
        return std::chrono::duration<double, std::micro>(b - a).count();
    };
    auto t_a = now();
    uint64_t budget = resolve_budget(r);
    auto t_b = now();
    if ((s = get_plan(r, lo, hi, budget))) return s;
    auto t_c = now();
    if (dbg) fprintf(stderr, "[pp] budget %.1f us, plan %.1f us\n", us(t_a, t_b), us(t_b, t_c));
    const Plan &P = r->plan;
    if (hi == lo) {                                  // empty loop: nothing to move or compute
        r->info = pp_info{};
        r->info.chunk_size = P.c;
        r->info.num_streams = P.S;
        r->info.narrays = (int32_t)r->arrs.size();
        return PP_OK;
    }
    if ((s = ensure_rings(r))) {
        // a device or driver that refuses the VMM mapping falls back to plain (split-copy) rings
        bool mirrored = false;
        for (const auto &rg : r->plan.rings) mirrored = mirrored || rg.mirror;
        if (!mirrored || r->mirror > 1) return s;
        r->mirror_failed = true;
        r->invalidate();
        if ((s = get_plan(r, lo, hi, budget))) return s;
        if ((s = ensure_rings(r))) return s;
    }
    if ((s = ensure_streams(r, P.nstreams))) return s;
    if ((s = ensure_events(r, (size_t)P.n_events, (size_t)P.nstreams + 1))) return s;
    if ((s = bounce_prepare(r))) return s;

    bool pinned_all = true;
    for (const auto &a : r->arrs) pinned_all = pinned_all && (a.resident || a.pinned);
    cudaError_t e;
    const bool halos = r->halo_in.arr >= 0 || r->halo_out.arr >= 0;
    if (r->halo_in.arr >= 0 && !r->halo_err) {
        if ((e = cudaMalloc(&r->halo_err, sizeof(uint32_t))) != cudaSuccess ||
            (e = cudaMemset(r->halo_err, 0, sizeof(uint32_t))) != cudaSuccess) {
            cudaGetLastError();
            r->halo_err = nullptr;
            return fail(PP_ENOMEM, "peer halo status word");
        }
    }
    bool persist = false;
    if (r->persistent && hi > lo) {
        std::string why;
        if (!persistent_eligible(r, body, &why)) return fail(PP_EUNSUPPORTED, why);
        persist = true;
        if ((s = ensure_streams(r, std::max(3, P.nstreams)))) return s;
        if ((s = ensure_events(r, (size_t)P.n_events, (size_t)std::max(3, P.nstreams) + 1))) return s;
    }
    const bool use_graph = r->graph && !r->trace && body.graphable() && pinned_all && hi > lo && !halos &&
                           !r->debug_tags && !persist;
    r->dbg_pending = false;
    if (r->debug_tags && hi > lo) {
        if ((s = dbg_alloc(r))) return s;
        r->dbg_pending = true;
    }
    for (const PeerHalo *h : {&r->halo_in, &r->halo_out}) {
        if (h->arr < 0 || hi == lo) continue;
        const auto &a = r->arrs[(size_t)h->arr];
        if (h->plane < lo + a.off || h->plane >= hi + a.off + a.size - 1)
            return fail(PP_ERANGE, "peer halo plane is not loaded by this launch");
    }
    r->halo_used = r->halo_in.arr >= 0 && hi > lo;
    if (r->trace) {
        while (r->tev.size() < 2 * P.ops.size()) {
            cudaEvent_t ev;
            if ((e = cudaEventCreate(&ev)) != cudaSuccess) return cuda_fail(e, "cudaEventCreate");
            r->tev.push_back(ev);
        }
    }
    cudaStream_t s0 = r->streams[0];
    r->last_path = 0;
    bool replayed = false;
    if (use_graph) {
        std::vector<uint8_t> k((const uint8_t *)key, (const uint8_t *)key + key_len);
        auto put = [&](const void *p, size_t n) { k.insert(k.end(), (const uint8_t *)p, (const uint8_t *)p + n); };
        put(&lo, sizeof lo);
        put(&hi, sizeof hi);
        put(&r->dbuf, sizeof r->dbuf);
        for (const auto &m : r->mirrors) put(&m.va, sizeof m.va);
        for (const auto &a : r->arrs) put(&a.host, sizeof a.host);
        if (!r->gexec || k != r->graph_key) {
            r->drop_graph();
            if ((e = cudaStreamBeginCapture(s0, cudaStreamCaptureModeThreadLocal)) != cudaSuccess)
                return cuda_fail(e, "cudaStreamBeginCapture");
            pp_status es = enqueue_plan(r, body);
            cudaGraph_t graph = nullptr;
            e = cudaStreamEndCapture(s0, &graph);
            if (es) { if (graph) cudaGraphDestroy(graph); r->poisoned = true; return es; }
            if (e != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "cudaStreamEndCapture"); }
            e = cudaGraphInstantiate(&r->gexec, graph, 0);
            cudaGraphDestroy(graph);
            if (e != cudaSuccess) { r->gexec = nullptr; r->poisoned = true; return cuda_fail(e, "cudaGraphInstantiate"); }
            r->graph_key = k;
            r->graph_path = r->last_path;
        } else {
            replayed = true;
            r->last_path = r->graph_path;
        }
        if ((e = cudaEventRecord(r->t0, s0)) != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "cudaEventRecord"); }
        if ((e = cudaGraphLaunch(r->gexec, s0)) != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "cudaGraphLaunch"); }
    } else {
        if ((e = cudaEventRecord(r->t0, s0)) != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "cudaEventRecord"); }
        auto t_d = now();
        pp_status es = persist ? enqueue_persistent(r, body, lo, hi) : enqueue_plan(r, body);
        if (dbg) fprintf(stderr, "[pp] setup %.1f us, enqueue %.1f us (%zu ops)\n", us(t_c, t_d), us(t_d, now()), r->plan.ops.size());
        if (es) {
            cudaDeviceSynchronize();
            r->poisoned = true;
            return es;
        }
    }
    if ((e = cudaEventRecord(r->t1, s0)) != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "cudaEventRecord"); }
    pp_info &I = r->info;
    I.last_ms = 0;
    I.chunk_size = P.c;
    I.num_streams = P.S;
    I.narrays = (int32_t)r->arrs.size();
    I.nchunks = P.nchunks;
    for (size_t i = 0; i < r->arrs.size() && i < PP_MAX_ARRAYS; ++i) {
        I.ring_planes[i] = r->arrs[i].resident ? 0 : P.rings[i].R;
        I.resident[i] = r->arrs[i].resident;
        I.pinned[i] = r->arrs[i].pinned;
    }
    I.ring_bytes = P.ring_bytes;
    I.h2d_bytes = P.h2d_bytes;
    I.d2h_bytes = P.d2h_bytes;
    if (r->d2h_interior) {                           // interior-only copy-back moves fewer bytes
        I.d2h_bytes = 0;
        for (const Op &op : P.ops)
            if (op.kind == OpKind::D2H) {
                const auto &a = r->arrs[op.arr];
                I.d2h_bytes += (uint64_t)(op.p1 - op.p0) * (uint64_t)((a.ext[1] - 2) * (a.ext[2] - 2) * a.esize);
            }
    }
    I.peer_bytes = 0;
    I.debug_violations = -1;
    I.merged_copies = persist ? 0 : r->merged;
    if (r->halo_in.arr >= 0) {                       // one plane came over NVLink instead of the host link
        I.peer_bytes = (uint64_t)r->arrs[(size_t)r->halo_in.arr].plane_bytes;
        I.h2d_bytes -= I.peer_bytes;
    }
    I.n_h2d = P.n_h2d;
    I.n_d2h = P.n_d2h;
    I.n_kernels = persist ? 1 : P.n_ker;           // (the persistent kernel: one launch per sweep)
    I.n_waits = P.n_waits;
    I.graph_replayed = replayed;
    I.kernel_path = r->last_path;
    r->pending = true;
    r->trace_pending = r->trace && !use_graph;
    return wait ? finish_pending(r) : PP_OK;
}

// ------------------------------------------------------------------------------------------------
// Built-in bodies and their binding checks
// ------------------------------------------------------------------------------------------------
pp_status bind_builtin(pp_region *r, pp_kernel k, const void *args, size_t args_size, BuiltinBody *b) {
    const auto &A = r->arrs;
    auto same_plane = [&](size_t i, size_t j) {
        if (A[i].ndim != A[j].ndim || A[i].split_dim != A[j].split_dim) return false;
        for (int d = 0; d < A[i].ndim; ++d)
            if (d != A[i].split_dim && A[i].ext[d] != A[j].ext[d]) return false;
        return true;
    };
    if (k != PP_K_TRIAD)
        for (const auto &a : A)
            if (a.split_dim != 0)
                return fail(PP_EUNSUPPORTED, "this kernel needs arrays split on dim 0 (2-D block regions: "
                                             "PP_K_TRIAD or pp_launch_fn)");
    switch (k) {
    case PP_K_TRIAD: {
        if (r->sweeps > 1) return fail(PP_EUNSUPPORTED, "PP_OPT_SWEEPS applies to PP_K_STENCIL7 only");
        if (A.size() != 3) return fail(PP_EINVAL, "PP_K_TRIAD binds 3 arrays: a (to), b (to), c (from)");
        if (A[0].type != Map::To || A[1].type != Map::To || A[2].type != Map::From)
            return fail(PP_EINVAL, "PP_K_TRIAD map types must be to, to, from");
        if (A[0].dtype != A[1].dtype || A[0].dtype != A[2].dtype || A[0].dtype == PP_I64)
            return fail(PP_EINVAL, "PP_K_TRIAD needs three f32 or three f64 arrays");
        if (!same_plane(0, 1) || !same_plane(0, 2)) return fail(PP_EINVAL, "PP_K_TRIAD plane shapes differ");
        for (int i = 0; i < 3; ++i)
            if (A[i].size != 1) return fail(PP_EINVAL, "PP_K_TRIAD windows must have size 1");
        if (!args || args_size != sizeof(pp_triad_args)) return fail(PP_EINVAL, "PP_K_TRIAD needs pp_triad_args");
        b->p0 = ((const pp_triad_args *)args)->s;
        return PP_OK;
    }
    case PP_K_STENCIL7: {
        if (A.size() != 2) return fail(PP_EINVAL, "PP_K_STENCIL7 binds 2 arrays: A0 (to), Anext (from)");
        if (A[0].type != Map::To || A[1].type != Map::From)
            return fail(PP_EINVAL, "PP_K_STENCIL7 map types must be to, from");
        if (A[0].ndim != 3 || A[1].ndim != 3 || !same_plane(0, 1))
            return fail(PP_EINVAL, "PP_K_STENCIL7 needs two 3-D arrays with equal [ny][nx]");
        if (A[0].dtype != A[1].dtype) return fail(PP_EINVAL, "PP_K_STENCIL7 dtypes differ");
        if (A[0].size != 3 || A[1].size != 1)
            return fail(PP_EINVAL, "PP_K_STENCIL7 needs windows A0[k+o:3], Anext[k+o:1]");
        if (!args || args_size != sizeof(pp_stencil_args)) return fail(PP_EINVAL, "PP_K_STENCIL7 needs pp_stencil_args");
        if (r->sweeps > 1 && (A[0].off != -1 || A[1].off != 0 || A[0].resident || A[1].resident))
            return fail(PP_EUNSUPPORTED, "multi-sweep chains need host arrays mapped A0[k-1:3], Anext[k:1]");
        if (r->sweeps > 1 && r->fuse > 1 && (A[0].dtype == PP_I64 || (A[0].ext[2] * A[0].esize) % 16))
            return fail(PP_EUNSUPPORTED, "PP_OPT_FUSE > 1 needs f32/f64 planes with a 16-byte row pitch");
        b->p0 = ((const pp_stencil_args *)args)->c0;
        b->p1 = ((const pp_stencil_args *)args)->c1;
        return PP_OK;
    }
    case PP_K_CONV3D: {
        if (r->sweeps > 1) return fail(PP_EUNSUPPORTED, "PP_OPT_SWEEPS applies to PP_K_STENCIL7 only");
        if (A.size() != 2) return fail(PP_EINVAL, "PP_K_CONV3D binds 2 arrays: A (to), B (from)");
        if (A[0].type != Map::To || A[1].type != Map::From)
            return fail(PP_EINVAL, "PP_K_CONV3D map types must be to, from");
        if (A[0].ndim != 3 || A[1].ndim != 3 || !same_plane(0, 1))
            return fail(PP_EINVAL, "PP_K_CONV3D needs two 3-D arrays with equal [ny][nx]");
        if (A[0].dtype != A[1].dtype || A[0].dtype == PP_I64) return fail(PP_EINVAL, "PP_K_CONV3D needs f32 or f64");
        if (A[0].size != 3 || A[1].size != 1) return fail(PP_EINVAL, "PP_K_CONV3D needs windows A[k+o:3], B[k+o:1]");
        return PP_OK;
    }
    case PP_K_PROBE: {
        if (r->sweeps > 1) return fail(PP_EUNSUPPORTED, "PP_OPT_SWEEPS applies to PP_K_STENCIL7 only");
        if (A.size() != 2) return fail(PP_EINVAL, "PP_K_PROBE binds 2 arrays: in (to), out (from)");
        if (A[0].type != Map::To || A[1].type != Map::From)
            return fail(PP_EINVAL, "PP_K_PROBE map types must be to, from");
        if (A[0].dtype != PP_I64 || A[1].dtype != PP_I64) return fail(PP_EINVAL, "PP_K_PROBE needs int64 arrays");
        if (A[0].plane_elems != A[1].plane_elems) return fail(PP_EINVAL, "PP_K_PROBE plane sizes differ");
        if (A[0].size != 3 || A[1].size != 1) return fail(PP_EINVAL, "PP_K_PROBE needs windows in[k+o:3], out[k+o:1]");
        return PP_OK;
    }
    }
    return fail(PP_EINVAL, "unknown kernel");
}

struct FnBody : Body {
    pp_region *r;
    pp_chunk_fn fn;
    void *user;
    FnBody(pp_region *r_, pp_chunk_fn f, void *u) : r(r_), fn(f), user(u) {}
    bool graphable() const override { return false; }
    cudaError_t run(int64_t j, int64_t k0, int64_t k1, int, const std::vector<DView> &v, cudaStream_t st,
                    std::string *err) override {
        pp_chunk c{};
        c.index = j;
        c.k0 = k0;
        c.k1 = k1;
        c.narrays = (int)r->arrs.size();
        for (size_t i = 0; i < r->arrs.size(); ++i)
            c.view[i] = pp_view{v[i].ring, v[i].R, v[i].base, v[i].plane_elems, r->arrs[i].plane_bytes, v[i].outer,
                                v[i].ostride};
        if (fn(&c, (void *)st, user) != 0) {
            *err = "pp_launch_fn: chunk callback returned non-zero";
            return cudaErrorUnknown;
        }
        return cudaGetLastError();
    }
};

}  // namespace pprt

// ================================================================================================
// C ABI
// ================================================================================================
extern "C" {

const char *pp_strerror(pp_status s) {
    switch (s) {
    case PP_OK: return "ok";
    case PP_EINVAL: return "invalid argument";
    case PP_ERANGE: return "window out of range";
    case PP_EBUDGET: return "ring does not fit pipeline_mem_limit";
    case PP_ENOMEM: return "out of memory";
    case PP_ECUDA: return "CUDA error";
    case PP_ESTATE: return "invalid region state";
    case PP_EUNSUPPORTED: return "unsupported";
    }
    return "unknown status";
}

const char *pp_last_error(void) { return g_last_error.c_str(); }

int pp_version(void) { return (PP_VERSION_MAJOR << 16) | PP_VERSION_MINOR; }

int pp_build_flags(void) {
#if defined(PP_TUNING_VARIANTS) && PP_TUNING_VARIANTS
    return PP_BUILD_TUNING;
#else
    return 0;
#endif
}

pp_status pp_view_plane(const pp_view *v, int64_t plane, int64_t nplanes, void **addr, int64_t *run) {
    if (!v || !addr || !run || nplanes < 1 || v->R < 1 || v->outer < 1) return fail(PP_EINVAL, "bad view arguments");
    int64_t slot = (plane - v->base) % v->R;             // the index handler's slot map
    if (slot < 0) slot += v->R;
    const int64_t slot_bytes = v->plane_bytes / v->outer;   // one plane's run within a row (1 row: the plane)
    *addr = (char *)v->ring + slot * slot_bytes;
    *run = std::min<int64_t>(nplanes, v->R - slot);
    return PP_OK;
}

pp_status pp_region_create(pp_region **out, int device) {
    if (!out) return fail(PP_EINVAL, "null out");
    *out = nullptr;
    if (device >= 0) {
        int n = 0;
        cudaError_t e = cudaGetDeviceCount(&n);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
        if (device >= n) return fail(PP_EINVAL, "device ordinal out of range");
    } else if (device != -1) {
        return fail(PP_EINVAL, "device must be >= 0 or -1 (host-only)");
    }
    pp_region *r = new (std::nothrow) pp_region();
    if (!r) return fail(PP_ENOMEM, "new pp_region");
    r->device = device;
    *out = r;
    return PP_OK;
}

void pp_region_destroy(pp_region *r) {
    if (!r) return;
    {
        DeviceGuard g(r->device);
        if (r->device >= 0) {
            r->pending = false;
            for (auto s : r->streams) cudaStreamSynchronize(s);
            r->drop_graph();
            if (!r->borrowed_streams)
                for (auto s : r->streams) cudaStreamDestroy(s);
            for (auto e : r->events) cudaEventDestroy(e);
            for (auto e : r->join) cudaEventDestroy(e);
            for (auto e : r->tev) cudaEventDestroy(e);
            for (auto e : {r->t0, r->t1, r->th, r->tk})
                if (e) cudaEventDestroy(e);
            if (r->dbuf && !r->borrowed_buf) cudaFree(r->dbuf);
            if (r->halo_err) cudaFree(r->halo_err);
            if (r->pipe_flags) cudaFree(r->pipe_flags);
            dbg_free(r);
            for (auto s : r->stage_stream)
                if (s) cudaStreamSynchronize(s);
            bounce_free(r);
            for (auto &m : r->mirrors) mirror_free(&m);
            for (void *p : r->naive)
                if (p) cudaFree(p);
            for (auto &a : r->arrs)
                if (a.registered) cudaHostUnregister(a.host);
            cudaGetLastError();
        }
    }
    delete r;
}

pp_status pp_map(pp_region *r, pp_map_type type, void *host, pp_dtype dt, int ndim,
                 const int64_t *extents, int64_t split_offset, int64_t split_size, int *array_id) {
    return pp_map_ex(r, type, host, dt, ndim, extents, 0, split_offset, split_size, array_id);
}

pp_status pp_map_ex(pp_region *r, pp_map_type type, void *host, pp_dtype dt, int ndim, const int64_t *extents,
                    int split_dim, int64_t split_offset, int64_t split_size, int *array_id) {
    pp_status s = check_region(r, false);
    if (s) return s;
    if (!host || !extents) return fail(PP_EINVAL, "null host pointer or extents");
    if (type != PP_TO && type != PP_FROM && type != PP_TOFROM) return fail(PP_EINVAL, "bad map type");
    if (dt != PP_F32 && dt != PP_F64 && dt != PP_I64) return fail(PP_EINVAL, "bad dtype");
    if (ndim < 1 || ndim > PP_MAX_DIMS) return fail(PP_EINVAL, "ndim must be in [1, 8]");
    if (r->arrs.size() >= PP_MAX_ARRAYS) return fail(PP_EINVAL, "too many arrays (max 8)");
    if (split_size < 1) return fail(PP_EINVAL, "split_size must be >= 1");
    if (type != PP_TO && split_size != 1)
        return fail(PP_EUNSUPPORTED, "from/tofrom arrays need split_size == 1 (reading S12)");
    if (split_dim < 0 || split_dim >= ndim) return fail(PP_EINVAL, "split_dim must be in [0, ndim)");
    ArraySpec a;
    a.type = (Map)type;
    a.dtype = dt;
    a.ndim = ndim;
    a.split_dim = split_dim;
    a.plane_elems = 1;
    for (int d = 0; d < ndim; ++d) {
        if (extents[d] < 1) return fail(PP_EINVAL, "extents must be >= 1");
        a.ext[d] = extents[d];
        if (d < split_dim) a.outer *= extents[d];
        if (d > split_dim) a.inner *= extents[d];
    }
    a.nsplit = extents[split_dim];
    a.plane_elems = a.outer * a.inner;
    a.esize = dtype_size(dt);
    a.plane_bytes = a.plane_elems * a.esize;
    a.off = split_offset;
    a.size = split_size;
    a.host = host;
    const uint64_t total = (uint64_t)a.nsplit * (uint64_t)a.plane_bytes;
    if (r->device >= 0) {
        DeviceGuard g(r->device);
        cudaPointerAttributes at{};
        cudaError_t e = cudaPointerGetAttributes(&at, host);
        if (e != cudaSuccess) { cudaGetLastError(); at.type = cudaMemoryTypeUnregistered; }
        if (at.type == cudaMemoryTypeDevice) {
            if (at.device != r->device) return fail(PP_EINVAL, "device array lives on another GPU");
            a.resident = true;
        } else if (at.type == cudaMemoryTypeManaged) {
            return fail(PP_EUNSUPPORTED, "managed memory is not supported");
        } else if (at.type == cudaMemoryTypeHost) {
            a.pinned = true;
        } else if (r->auto_pin) {
            e = cudaHostRegister(host, total, cudaHostRegisterPortable);
            if (e == cudaSuccess) { a.pinned = true; a.registered = true; }
            else cudaGetLastError();   // stays pageable (slower, still correct)
        }
    }
    // host aliasing between an input and an output is rejected (reading S24), except the exact
    // in-place alias PP_OPT_INPLACE allows (input PP_TO, output PP_FROM, same pointer and geometry)
    for (size_t bi = 0; bi < r->arrs.size(); ++bi) {
        const auto &b = r->arrs[bi];
        if (a.resident != b.resident) continue;
        if (!(a.is_output() || b.is_output())) continue;
        const char *x0 = (const char *)a.host, *x1 = x0 + total;
        const char *y0 = (const char *)b.host, *y1 = y0 + (uint64_t)b.nsplit * (uint64_t)b.plane_bytes;
        if (!(x0 < y1 && y0 < x1)) continue;
        bool same_geom = a.host == b.host && a.dtype == b.dtype && a.ndim == b.ndim && a.split_dim == b.split_dim;
        for (int d = 0; same_geom && d < a.ndim; ++d) same_geom = a.ext[d] == b.ext[d];
        if (r->inplace && same_geom && !a.resident && a.type == Map::From && b.type == Map::To && a.alias < 0) {
            a.alias = (int)bi;
            continue;
        }
        if (a.registered) cudaHostUnregister(a.host);
        return fail(PP_EINVAL, r->inplace ? "in-place alias must be an exact to/from pair (same pointer, dtype, extents)"
                                          : "mapped arrays overlap in memory and one of them is an output");
    }
    r->arrs.push_back(a);
    r->invalidate();
    if (array_id) *array_id = (int)r->arrs.size() - 1;
    return PP_OK;
}

pp_status pp_pipeline(pp_region *r, pp_sched kind, int64_t chunk_size, int num_streams) {
    pp_status s = check_region(r, false);
    if (s) return s;
    if (kind == PP_ADAPTIVE) return fail(PP_EUNSUPPORTED, "adaptive schedule is not defined (P:L218-219)");
    if (kind != PP_STATIC) return fail(PP_EINVAL, "bad schedule kind");
    if (chunk_size < 0) return fail(PP_EINVAL, "chunk_size < 0");
    if (num_streams < 1) return fail(PP_EINVAL, "num_streams < 1");
    r->chunk = chunk_size;
    r->S = num_streams;
    r->invalidate();
    return PP_OK;
}

pp_status pp_mem_limit(pp_region *r, size_t bytes) {
    pp_status s = check_region(r, false);
    if (s) return s;
    r->mem_limit = bytes;
    r->invalidate();
    return PP_OK;
}

pp_status pp_set_option(pp_region *r, pp_option opt, int64_t value) {
    pp_status s = check_region(r, false);
    if (s) return s;
    switch (opt) {
    case PP_OPT_STREAM_POLICY:
        if (value < 0 || value > 5) return fail(PP_EINVAL, "stream policy must be in [0, 5]");
        r->policy = (int)value;
        break;
    case PP_OPT_GRAPH: r->graph = value != 0; break;
    case PP_OPT_FMAD: r->fmad = value != 0; break;
    case PP_OPT_RING_EXTRA:
        if (value < -1) return fail(PP_EINVAL, "ring extra must be >= -1");
        r->ring_extra = value;
        break;
    case PP_OPT_AUTO_PIN: r->auto_pin = value != 0; break;
    case PP_OPT_KERNEL_PATH:
        if (value < 0 || value > 2) return fail(PP_EINVAL, "kernel path must be 0, 1 or 2");
        r->kernel_path = (int)value;
        break;
    case PP_OPT_TRACE: r->trace = value != 0; break;
    case PP_OPT_INPLACE: r->inplace = value != 0; break;
    case PP_OPT_SWEEPS:
        if (value < 1 || value > 4096) return fail(PP_EINVAL, "sweeps must be in [1, 4096]");
        r->sweeps = value;
        break;
    case PP_OPT_FUSE:
        if (value < 1 || value > pp::kMaxFuse) return fail(PP_EINVAL, "fuse must be in [1, 4]");
        r->fuse = value;
        break;
    case PP_OPT_MIRROR:
        if (value < 0) return fail(PP_EINVAL, "mirror must be 0, 1 or a granule size in bytes");
        r->mirror = value;
        r->mirror_failed = false;
        break;
    case PP_OPT_D2H_INTERIOR: r->d2h_interior = value != 0; break;
    case PP_OPT_DEBUG_TAGS: r->debug_tags = value != 0; break;
    case PP_OPT_PERSISTENT: r->persistent = value != 0; break;
    case PP_OPT_MERGE_COPIES: r->merge_copies = value != 0; break;
    case PP_OPT_SM_COPY: {
        if (value < 0) return fail(PP_EINVAL, "SM copy threshold must be >= 0");
        if (value > 0 && r->device >= 0) {
            // the copy kernel dereferences the host pointer itself (registered pages included)
            int ok = 0;
            cudaDeviceGetAttribute(&ok, cudaDevAttrCanUseHostPointerForRegisteredMem, r->device);
            if (!ok) return fail(PP_EUNSUPPORTED, "device cannot use host pointers of registered memory");
        }
        r->sm_copy = value;
        break;
    }
    case PP_OPT_BOUNCE:
        if (value < 0 || value > 64) return fail(PP_EINVAL, "bounce workers must be in [0, 64]");
        r->bounce = (int)value;
        break;
    case PP_OPT_FAULT_INJECT:
        if (value < 0 || value > 4) return fail(PP_EINVAL, "fault mode must be in [0,4]");
        r->fault = (int)value;
        break;
    default: return fail(PP_EINVAL, "unknown option");
    }
    r->invalidate();
    return PP_OK;
}

static pp_status halo_check(pp_region *r, int array_id, const void *side, const void *flag) {
    pp_status s = check_region(r, true);
    if (s) return s;
    if (array_id < 0 || array_id >= (int)r->arrs.size()) return fail(PP_EINVAL, "bad array id");
    const auto &a = r->arrs[(size_t)array_id];
    if (!a.is_input() || a.resident) return fail(PP_EINVAL, "peer halos apply to host input arrays");
    if (a.outer != 1) return fail(PP_EUNSUPPORTED, "peer halos need arrays split on dim 0");
    if (!side || !flag) return fail(PP_EINVAL, "null side slot or flag");
    return PP_OK;
}

pp_status pp_halo_export(pp_region *r, int array_id, int64_t plane, void *side, uint32_t *flag, uint32_t epoch) {
    pp_status s = halo_check(r, array_id, side, flag);
    if (s) return s;
    r->halo_out = PeerHalo{array_id, plane, side, r->device, flag, epoch};
    r->drop_graph();
    return PP_OK;
}

pp_status pp_halo_import(pp_region *r, int array_id, int64_t plane, const void *side, int side_device,
                         const uint32_t *flag, uint32_t epoch) {
    pp_status s = halo_check(r, array_id, side, flag);
    if (s) return s;
    if (side_device < 0) return fail(PP_EINVAL, "bad side device");
    r->halo_in = PeerHalo{array_id, plane, const_cast<void *>(side), side_device, const_cast<uint32_t *>(flag), epoch};
    r->drop_graph();
    return PP_OK;
}

pp_status pp_halo_clear(pp_region *r) {
    pp_status s = check_region(r, false);
    if (s) return s;
    r->halo_in = PeerHalo{};
    r->halo_out = PeerHalo{};
    r->drop_graph();
    return PP_OK;
}

pp_status pp_launch(pp_region *r, int64_t lo, int64_t hi, pp_kernel k, const void *args, size_t args_size) {
    pp_status s = check_region(r, true);
    if (s) return s;
    BuiltinBody b(r, k);
    if ((s = bind_builtin(r, k, args, args_size, &b))) return s;
    b.lo = lo;
    b.hi = hi;
    std::vector<uint8_t> key(sizeof k + sizeof b.p0 + sizeof b.p1);
    memcpy(key.data(), &k, sizeof k);
    memcpy(key.data() + sizeof k, &b.p0, sizeof b.p0);
    memcpy(key.data() + sizeof k + sizeof b.p0, &b.p1, sizeof b.p1);
    return run_launch(r, lo, hi, b, key.data(), key.size(), true);
}

pp_status pp_launch_async(pp_region *r, int64_t lo, int64_t hi, pp_kernel k, const void *args,
                          size_t args_size) {
    pp_status s = check_region(r, true);
    if (s) return s;
    BuiltinBody b(r, k);
    if ((s = bind_builtin(r, k, args, args_size, &b))) return s;
    b.lo = lo;
    b.hi = hi;
    std::vector<uint8_t> key(sizeof k + sizeof b.p0 + sizeof b.p1);
    memcpy(key.data(), &k, sizeof k);
    memcpy(key.data() + sizeof k, &b.p0, sizeof b.p0);
    memcpy(key.data() + sizeof k + sizeof b.p0, &b.p1, sizeof b.p1);
    return run_launch(r, lo, hi, b, key.data(), key.size(), false);
}

pp_status pp_wait(pp_region *r) {
    pp_status s = check_region(r, true);
    if (s) return s;
    DeviceGuard g(r->device);
    return finish_pending(r);
}

pp_status pp_launch_fn(pp_region *r, int64_t lo, int64_t hi, pp_chunk_fn fn, void *user) {
    pp_status s = check_region(r, true);
    if (s) return s;
    if (!fn) return fail(PP_EINVAL, "null chunk function");
    if (r->sweeps > 1) return fail(PP_EUNSUPPORTED, "PP_OPT_SWEEPS applies to PP_K_STENCIL7 only");
    FnBody b(r, fn, user);
    return run_launch(r, lo, hi, b, nullptr, 0, true);
}

// ------------------------------------------------------------------------------------------------
// Naive offload (independent of the planner): full device arrays, synchronous phases.
// ------------------------------------------------------------------------------------------------
namespace {
// planes [p0,p1) of array a between its host copy and a full device copy of the same layout
cudaError_t naive_copy(const pp::ArraySpec &a, void *dev, int64_t p0, int64_t p1, cudaMemcpyKind kind, cudaStream_t st) {
    const size_t row = (size_t)a.inner * (size_t)a.esize, pitch = (size_t)a.nsplit * row;
    char *d = (char *)dev + (size_t)p0 * row, *h = (char *)a.host + (size_t)p0 * row;
    const size_t width = (size_t)(p1 - p0) * row;
    if (a.outer == 1)
        return kind == cudaMemcpyHostToDevice ? cudaMemcpyAsync(d, h, width, kind, st) : cudaMemcpyAsync(h, d, width, kind, st);
    return kind == cudaMemcpyHostToDevice ? cudaMemcpy2DAsync(d, pitch, h, pitch, width, (size_t)a.outer, kind, st)
                                          : cudaMemcpy2DAsync(h, pitch, d, pitch, width, (size_t)a.outer, kind, st);
}
}  // namespace

// ------------------------------------------------------------------------------------------------
// ------------------------------------------------------------------------------------------------
pp_status pp_naive(pp_region *r, int64_t lo, int64_t hi, pp_kernel k, const void *args, size_t args_size) {
    pp_status s = check_region(r, true);
    if (s) return s;
    DeviceGuard g(r->device);
    BuiltinBody b(r, k);
    if ((s = bind_builtin(r, k, args, args_size, &b))) return s;
    if (hi < lo) return fail(PP_EINVAL, "hi < lo");
    if ((s = check_interior_d2h(r))) return s;
    for (size_t i = 0; i < r->arrs.size(); ++i) {
        const auto &a = r->arrs[i];
        if (hi > lo && (lo + a.off < 0 || hi - 1 + a.off + a.size > a.nsplit))
            return fail(PP_ERANGE, "naive: window out of range for array " + std::to_string(i));
    }
    if ((s = finish_pending(r))) return s;
    if ((s = ensure_streams(r, 1))) return s;
    if ((s = ensure_events(r, 0, 1))) return s;
    cudaError_t e;
    if (r->naive.size() != r->arrs.size()) {
        for (void *p : r->naive)
            if (p) cudaFree(p);
        r->naive.assign(r->arrs.size(), nullptr);
        r->naive_bytes = 0;
        for (size_t i = 0; i < r->arrs.size(); ++i) {
            const auto &a = r->arrs[i];
            if (a.resident) continue;
            uint64_t bytes = (uint64_t)a.nsplit * (uint64_t)a.plane_bytes;
            if ((e = cudaMalloc(&r->naive[i], bytes)) != cudaSuccess) {
                cudaGetLastError();
                return fail(PP_ENOMEM, std::string("naive cudaMalloc: ") + cudaGetErrorString(e));
            }
            r->naive_bytes += bytes;
        }
    }
    cudaStream_t st = r->streams[0];
    std::vector<DView> v(r->arrs.size());
    for (size_t i = 0; i < r->arrs.size(); ++i) {
        const auto &a = r->arrs[i];
        v[i] = DView{a.resident ? a.host : r->naive[i], a.nsplit, 0, a.plane_elems, a.outer, a.nsplit * a.inner};
    }
    uint64_t h2d = 0, d2h = 0;
    if ((e = cudaEventRecord(r->t0, st)) != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
    if (hi > lo) {
        for (size_t i = 0; i < r->arrs.size(); ++i) {
            const auto &a = r->arrs[i];
            if (a.resident || !a.is_input()) continue;
            int64_t p0 = lo + a.off, p1 = hi + a.off + a.size - 1;
            if ((e = naive_copy(a, r->naive[i], p0, p1, cudaMemcpyHostToDevice, st)))
                { r->poisoned = true; return cuda_fail(e, "naive H2D"); }
            h2d += (size_t)(p1 - p0) * a.plane_bytes;
        }
    }
    cudaEventRecord(r->th, st);
    std::string err;
    int result_buf = -1;                            // multi-sweep: which device array holds A^T
    if (hi > lo && k == PP_K_STENCIL7 && r->sweeps > 1) {
        // T sweeps ping-ponging the two full device arrays; both carry the fixed planes lo-1, hi
        const auto &A = r->arrs[0];
        const size_t pb = (size_t)A.plane_bytes;
        for (int64_t q : {lo - 1, hi})
            if ((e = cudaMemcpyAsync((char *)r->naive[1] + q * pb, (char *)r->naive[0] + q * pb, pb,
                                     cudaMemcpyDeviceToDevice, st))) { r->poisoned = true; return cuda_fail(e, "naive D2D"); }
        int used = 0;
        int src = 0;
        for (int64_t t = 0; t < r->sweeps;) {
            // groups of up to PP_OPT_FUSE sweeps per launch (one fused pass), ping-ponging the arrays
            const int64_t h = std::min<int64_t>(r->fuse, r->sweeps - t);
            const int dst = 1 - src;
            if (h > 1) {
                e = launch_stencil7_fused(A.dtype, (int)h, v[src], v[dst], A.ext[1], A.ext[2], lo, hi, lo - 1, hi + 1, lo,
                                          hi, b.p0, b.p1, r->fmad != 0, st);
                if (e == cudaErrorNotSupported) {
                    r->poisoned = true;
                    return fail(PP_EUNSUPPORTED, "PP_OPT_FUSE needs f32/f64 planes with a 16-byte row pitch");
                }
                used = std::max(used, (int)KPATH_TMA);
            } else {
                e = launch_stencil7(A.dtype, v[src], 0, v[dst], 0, A.ext[1], A.ext[2], lo, hi, INT64_MIN, INT64_MAX,
                                    b.p0, b.p1, r->fmad != 0, r->kernel_path, &used, st);
            }
            if (e != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "naive kernel"); }
            result_buf = dst;
            src = dst;
            t += h;
        }
        r->last_path = std::max(r->last_path, used);
    } else if (hi > lo && (e = b.run(0, lo, hi, 1, v, st, &err)) != cudaSuccess) {
        r->poisoned = true;
        return cuda_fail(e, "naive kernel");
    }
    cudaEventRecord(r->tk, st);
    if (hi > lo) {
        for (size_t i = 0; i < r->arrs.size(); ++i) {
            const auto &a = r->arrs[i];
            if (a.resident || !a.is_output()) continue;
            int64_t p0 = lo + a.off, p1 = hi + a.off;
            const int srcbuf = result_buf >= 0 ? result_buf : (int)i;
            if (interior_d2h(r, a)) {
                e = copy_interior_d2h(a, (const char *)r->naive[srcbuf] + (size_t)p0 * a.plane_bytes, p0, p1 - p0, st);
                d2h += (size_t)(p1 - p0) * (size_t)((a.ext[1] - 2) * (a.ext[2] - 2) * a.esize);
            } else {
                e = naive_copy(a, r->naive[srcbuf], p0, p1, cudaMemcpyDeviceToHost, st);
                d2h += (size_t)(p1 - p0) * a.plane_bytes;
            }
            if (e) { r->poisoned = true; return cuda_fail(e, "naive D2H"); }
        }
    }
    cudaEventRecord(r->t1, st);
    if ((e = cudaEventSynchronize(r->t1)) != cudaSuccess) { r->poisoned = true; return cuda_fail(e, "naive execution"); }
    float a_ms = 0, b_ms = 0, c_ms = 0;
    cudaEventElapsedTime(&a_ms, r->t0, r->th);
    cudaEventElapsedTime(&b_ms, r->th, r->tk);
    cudaEventElapsedTime(&c_ms, r->tk, r->t1);
    pp_info &I = r->info;
    I.naive_h2d_ms = a_ms;
    I.naive_kernel_ms = b_ms;
    I.naive_d2h_ms = c_ms;
    I.last_ms = a_ms + b_ms + c_ms;
    I.naive_bytes = r->naive_bytes;
    I.h2d_bytes = h2d;
    I.d2h_bytes = d2h;
    I.n_h2d = I.n_d2h = 0;
    I.n_kernels = hi > lo ? (k == PP_K_STENCIL7 ? (r->sweeps + r->fuse - 1) / r->fuse : 1) : 0;
    I.kernel_path = r->last_path;
    return PP_OK;
}

pp_status pp_naive_release(pp_region *r) {
    if (!r) return fail(PP_EINVAL, "null region");
    DeviceGuard g(r->device);
    for (void *p : r->naive)
        if (p) cudaFree(p);
    r->naive.clear();
    r->naive_bytes = 0;
    r->info.naive_bytes = 0;
    return PP_OK;
}

pp_status pp_use_streams(pp_region *r, void *const *streams, int n) {
    pp_status s = check_region(r, true);
    if (s) return s;
    if (!streams || n < 1) return fail(PP_EINVAL, "need >= 1 stream");
    DeviceGuard g(r->device);
    for (auto st : r->streams) cudaStreamSynchronize(st);
    if (!r->borrowed_streams)
        for (auto st : r->streams) cudaStreamDestroy(st);
    r->streams.assign((cudaStream_t const *)streams, (cudaStream_t const *)streams + n);
    r->borrowed_streams = true;
    r->drop_graph();
    return PP_OK;
}

pp_status pp_use_device_buffer(pp_region *r, void *dptr, size_t bytes) {
    pp_status s = check_region(r, true);
    if (s) return s;
    if (!dptr || bytes == 0) return fail(PP_EINVAL, "null buffer");
    if ((uintptr_t)dptr % 256) return fail(PP_EINVAL, "device buffer must be 256-byte aligned");
    DeviceGuard g(r->device);
    for (auto st : r->streams) cudaStreamSynchronize(st);
    if (r->dbuf && !r->borrowed_buf) cudaFree(r->dbuf);
    r->dbuf = dptr;
    r->dbuf_bytes = bytes;
    r->borrowed_buf = true;
    if (!r->mem_limit || r->mem_limit > bytes) r->mem_limit = bytes;
    r->invalidate();
    return PP_OK;
}

pp_status pp_query(const pp_region *r, pp_info *out) {
    if (!r || !out) return fail(PP_EINVAL, "null argument");
    *out = r->info;
    return PP_OK;
}

pp_status pp_trace(const pp_region *r, pp_trace_rec *out, int64_t cap, int64_t *n) {
    if (!r || !n || cap < 0) return fail(PP_EINVAL, "bad argument");
    *n = (int64_t)r->trace_recs.size();
    if (out)
        for (int64_t i = 0; i < cap && i < *n; ++i) out[i] = r->trace_recs[(size_t)i];
    return PP_OK;
}

pp_status pp_plan_dump(pp_region *r, int64_t lo, int64_t hi, char *buf, size_t cap, size_t *needed) {
    pp_status s = check_region(r, false);
    if (s) return s;
    if ((s = get_plan(r, lo, hi, resolve_budget(r)))) return s;
    std::string d = dump_plan(r->plan);
    if (needed) *needed = d.size() + 1;
    if (buf && cap) {
        size_t n = std::min(cap - 1, d.size());
        memcpy(buf, d.data(), n);
        buf[n] = 0;
    }
    return PP_OK;
}

pp_status pp_plan_check(pp_region *r, int64_t lo, int64_t hi, int64_t orders, uint64_t seed, int64_t *violations) {
    pp_status s = check_region(r, false);
    if (s) return s;
    if (!violations || orders < 0) return fail(PP_EINVAL, "bad argument");
    if ((s = get_plan(r, lo, hi, resolve_budget(r)))) return s;
    std::string first;
    *violations = check_plan(r->arrs, r->plan, orders, seed, &first);
    if (*violations) g_last_error = first;
    return PP_OK;
}

pp_status pp_partition(int64_t lo, int64_t hi, int G, int g, int64_t *lo_g, int64_t *hi_g) {
    if (G < 1 || g < 0 || g >= G || hi < lo || !lo_g || !hi_g) return fail(PP_EINVAL, "bad partition arguments");
    partition(lo, hi, G, g, lo_g, hi_g);
    return PP_OK;
}

pp_status pp_probe_link(int device, size_t bytes, int reps, double out[4]) {
    if (!out || bytes == 0 || reps < 1) return fail(PP_EINVAL, "bad probe arguments");
    DeviceGuard g(device);
    if (!g.ok) return fail(PP_ECUDA, "cudaSetDevice failed");
    void *h1 = nullptr, *h2 = nullptr, *d1 = nullptr, *d2 = nullptr;
    cudaStream_t s1 = nullptr, s2 = nullptr;
    cudaEvent_t e[4] = {}, gate = nullptr;
    cudaError_t e0 = cudaHostAlloc(&h1, bytes, cudaHostAllocPortable);
    if (!e0) e0 = cudaHostAlloc(&h2, bytes, cudaHostAllocPortable);
    if (!e0) e0 = cudaMalloc(&d1, bytes);
    if (!e0) e0 = cudaMalloc(&d2, bytes);
    if (!e0) e0 = cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    if (!e0) e0 = cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    for (int i = 0; i < 4 && !e0; ++i) e0 = cudaEventCreate(&e[i]);
    if (!e0) e0 = cudaEventCreateWithFlags(&gate, cudaEventDisableTiming);
    if (!e0) {
        memset(h1, 1, bytes);
        memset(h2, 2, bytes);
        double best[4] = {0, 0, 0, 0};
        for (int mode = 0; mode < 3 && !e0; ++mode) {
            for (int t = 0; t < reps + 1 && !e0; ++t) {   // first rep is a warm-up
                if (mode == 2) {
                    // start both directions together: both streams are held behind one event that
                    // fires after a short device-side delay, by when both copies are queued
                    launch_delay(200000, s1);
                    cudaEventRecord(gate, s1);
                    cudaStreamWaitEvent(s2, gate, 0);
                }
                if (mode != 1) { cudaEventRecord(e[0], s1); cudaMemcpyAsync(d1, h1, bytes, cudaMemcpyHostToDevice, s1); cudaEventRecord(e[1], s1); }
                if (mode != 0) { cudaEventRecord(e[2], s2); cudaMemcpyAsync(h2, d2, bytes, cudaMemcpyDeviceToHost, s2); cudaEventRecord(e[3], s2); }
                e0 = cudaDeviceSynchronize();
                if (t == 0) continue;
                float a = 0, b = 0;
                if (mode != 1) cudaEventElapsedTime(&a, e[0], e[1]);
                if (mode != 0) cudaEventElapsedTime(&b, e[2], e[3]);
                if (mode == 2) {
                    // both directions over their COMMON window (first start to last end), so a
                    // direction that ran alone after the other finished is not credited with it
                    float d2h_start = 0, d2h_end = 0;
                    cudaEventElapsedTime(&d2h_start, e[0], e[2]);
                    cudaEventElapsedTime(&d2h_end, e[0], e[3]);
                    a = b = std::max(a, d2h_end) - std::min(0.0f, d2h_start);
                }
                double ga = a > 0 ? bytes / (a * 1e-3) / 1e9 : 0, gb = b > 0 ? bytes / (b * 1e-3) / 1e9 : 0;
                if (mode == 0) best[0] = std::max(best[0], ga);
                if (mode == 1) best[1] = std::max(best[1], gb);
                if (mode == 2 && ga + gb > best[2] + best[3]) { best[2] = ga; best[3] = gb; }
            }
        }
        for (int i = 0; i < 4; ++i) out[i] = best[i];
    }
    for (int i = 0; i < 4; ++i)
        if (e[i]) cudaEventDestroy(e[i]);
    if (gate) cudaEventDestroy(gate);
    if (s1) cudaStreamDestroy(s1);
    if (s2) cudaStreamDestroy(s2);
    if (d1) cudaFree(d1);
    if (d2) cudaFree(d2);
    if (h1) cudaFreeHost(h1);
    if (h2) cudaFreeHost(h2);
    if (e0) return cuda_fail(e0, "pp_probe_link");
    return PP_OK;
}

}  // extern "C"
