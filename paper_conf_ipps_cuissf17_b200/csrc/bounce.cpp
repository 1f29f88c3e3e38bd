// bounce.cpp — the pageable-host path of §8(a) row a4 (PP_OPT_BOUNCE). The paper allocates its host
// arrays pinned with cudaHostAlloc "which avoids the data movement time from virtual to pinned
// buffer memory"; a caller's PAGEABLE array either gets page-locked in place
// (PP_OPT_AUTO_PIN, cudaHostRegister) or, when that is off or refused, goes through a small ring of
// pinned staging slots here: host memcpy worker threads move each copy's planes between the pageable
// array and a staging slot (in a host function on a staging stream, so the order is the device's),
// and the copy engine moves the slot to / from the device ring. With nslots >= 2 the host memcpy of
// the next copy overlaps the DMA of this one.
#include <condition_variable>
#include <cstring>
#include <mutex>
#include <thread>

#include "region.hpp"

namespace pprt {

// Fixed pool of worker threads; copy() splits one memcpy into equal parts, runs them on the workers
// (and the calling thread) and returns when all are done. One copy at a time.
struct HostPool {
    explicit HostPool(int n) {
        for (int i = 0; i < n; ++i) workers.emplace_back([this, i] { loop(i); });
    }
    ~HostPool() {
        {
            std::lock_guard<std::mutex> lk(mu);
            stop = true;
        }
        cv.notify_all();
        for (auto &t : workers) t.join();
    }
    void copy(void *dst, const void *src, size_t bytes) {
        std::lock_guard<std::mutex> one(busy);
        const size_t parts = workers.size() + 1;
        const size_t step = (bytes / parts + 4095) & ~size_t(4095);   // page-aligned slices
        {
            std::lock_guard<std::mutex> lk(mu);
            d = (char *)dst;
            s = (const char *)src;
            n = bytes;
            chunk = step ? step : bytes;
            remaining = (int)workers.size();
            ++gen;
        }
        cv.notify_all();
        part(0);                                                 // the caller takes slice 0
        std::unique_lock<std::mutex> lk(mu);
        done_cv.wait(lk, [this] { return remaining == 0; });
    }

  private:
    void part(size_t i) {
        const size_t a = i * chunk;
        if (a >= n) return;
        memcpy(d + a, s + a, std::min(chunk, n - a));
    }
    void loop(int i) {
        uint64_t seen = 0;
        for (;;) {
            {
                std::unique_lock<std::mutex> lk(mu);
                cv.wait(lk, [&] { return stop || gen != seen; });
                if (stop) return;
                seen = gen;
            }
            part((size_t)i + 1);
            std::lock_guard<std::mutex> lk(mu);
            if (--remaining == 0) done_cv.notify_one();
        }
    }
    std::vector<std::thread> workers;
    std::mutex mu, busy;
    std::condition_variable cv, done_cv;
    bool stop = false;
    uint64_t gen = 0;
    char *d = nullptr;
    const char *s = nullptr;
    size_t n = 0, chunk = 0;
    int remaining = 0;
};

static void CUDART_CB host_copy_fn(void *p) {
    HostCopyJob *j = (HostCopyJob *)p;
    j->pool->copy(j->dst, j->src, j->bytes);
}

bool bounced(const pp_region *r, const pp::ArraySpec &a) {
    return r->bounce && !a.pinned && !a.resident && a.outer == 1;
}

void bounce_free(pp_region *r) {
    for (auto &b : r->bounce_rings) {
        if (b.buf) cudaFreeHost(b.buf);
        for (auto e : b.free_ev) cudaEventDestroy(e);
        for (auto e : b.ready_ev) cudaEventDestroy(e);
    }
    r->bounce_rings.clear();
    for (int i = 0; i < 2; ++i) {
        if (r->stage_stream[i]) cudaStreamDestroy(r->stage_stream[i]);
        if (r->stage_join[i]) cudaEventDestroy(r->stage_join[i]);
        r->stage_stream[i] = nullptr;
        r->stage_join[i] = nullptr;
    }
    delete r->pool;
    r->pool = nullptr;
    delete r->jobs;
    r->jobs = nullptr;
}

pp_status bounce_prepare(pp_region *r) {
    r->bounce_used = false;
    const pp::Plan &P = r->plan;
    std::vector<size_t> need(r->arrs.size(), 0);
    for (const pp::Op &op : P.ops)
        if (op.kind != pp::OpKind::KER && bounced(r, r->arrs[(size_t)op.arr]))
            need[(size_t)op.arr] = std::max(need[(size_t)op.arr], (size_t)(op.p1 - op.p0) * (size_t)r->arrs[(size_t)op.arr].plane_bytes);
    bool any = false;
    for (size_t n : need) any = any || n;
    if (!any) return PP_OK;
    cudaError_t e = cudaSuccess;
    if (!r->pool) {
        const unsigned hw = std::thread::hardware_concurrency();
        const int n = r->bounce > 1 ? r->bounce : (int)std::max(1u, std::min(8u, hw / 2));
        r->pool = new HostPool(n - 1);                      // + the calling thread
    }
    if (!r->jobs) r->jobs = new std::vector<HostCopyJob>();
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
        if (!r->stage_stream[i]) e = cudaStreamCreateWithFlags(&r->stage_stream[i], cudaStreamNonBlocking);
        if (e == cudaSuccess && !r->stage_join[i]) e = cudaEventCreateWithFlags(&r->stage_join[i], cudaEventDisableTiming);
    }
    if (r->bounce_rings.size() < r->arrs.size()) r->bounce_rings.resize(r->arrs.size());
    for (size_t i = 0; i < need.size() && e == cudaSuccess; ++i) {
        BounceRing &b = r->bounce_rings[i];
        if (!need[i] || b.slot_bytes >= need[i]) continue;
        if (b.buf) {
            // an earlier asynchronous launch may still be copying from / to the old slots: its host
            // copies run on the staging streams, its DMAs on the region's streams
            for (cudaStream_t hs : r->stage_stream) cudaStreamSynchronize(hs);
            for (cudaStream_t os : r->streams) cudaStreamSynchronize(os);
            cudaFreeHost(b.buf);
            b.buf = nullptr;
        }
        b.nslots = 3;
        b.slot_bytes = (need[i] + 4095) & ~size_t(4095);
        e = cudaHostAlloc(&b.buf, b.slot_bytes * (size_t)b.nslots, cudaHostAllocPortable);
        while (e == cudaSuccess && (int)b.free_ev.size() < b.nslots) {
            cudaEvent_t x, y;
            e = cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&y, cudaEventDisableTiming);
            if (e == cudaSuccess) {
                b.free_ev.push_back(x);
                b.ready_ev.push_back(y);
            }
        }
        b.next = 0;
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(PP_ENOMEM, std::string("PP_OPT_BOUNCE staging ring: ") + cudaGetErrorString(e));
    }
    // an earlier asynchronous launch may still have host copies queued: let them finish before their
    // job records are reused
    for (cudaStream_t hs : r->stage_stream) cudaStreamSynchronize(hs);
    r->jobs->clear();
    r->jobs->reserve(P.ops.size());                          // job addresses must stay stable
    r->bounce_used = true;
    return PP_OK;
}

cudaError_t bounce_h2d(pp_region *r, int arr, void *dev, const void *host, size_t bytes, cudaStream_t st) {
    BounceRing &b = r->bounce_rings[(size_t)arr];
    const int k = b.next;
    b.next = (k + 1) % b.nslots;
    char *stg = (char *)b.buf + (size_t)k * b.slot_bytes;
    cudaStream_t hs = r->stage_stream[0];
    r->jobs->push_back(HostCopyJob{stg, host, bytes, r->pool});
    cudaError_t e = cudaStreamWaitEvent(hs, b.free_ev[(size_t)k], 0);   // slot's previous DMA done
    if (e == cudaSuccess) e = cudaLaunchHostFunc(hs, host_copy_fn, &r->jobs->back());
    if (e == cudaSuccess) e = cudaEventRecord(b.ready_ev[(size_t)k], hs);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(st, b.ready_ev[(size_t)k], 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dev, stg, bytes, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaEventRecord(b.free_ev[(size_t)k], st);
    return e;
}

cudaError_t bounce_d2h(pp_region *r, int arr, void *host, const void *dev, size_t bytes, cudaStream_t st) {
    BounceRing &b = r->bounce_rings[(size_t)arr];
    const int k = b.next;
    b.next = (k + 1) % b.nslots;
    char *stg = (char *)b.buf + (size_t)k * b.slot_bytes;
    cudaStream_t hs = r->stage_stream[1];
    r->jobs->push_back(HostCopyJob{host, stg, bytes, r->pool});
    cudaError_t e = cudaStreamWaitEvent(st, b.free_ev[(size_t)k], 0);    // slot drained to the host
    if (e == cudaSuccess) e = cudaMemcpyAsync(stg, dev, bytes, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaEventRecord(b.ready_ev[(size_t)k], st);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(hs, b.ready_ev[(size_t)k], 0);
    if (e == cudaSuccess) e = cudaLaunchHostFunc(hs, host_copy_fn, &r->jobs->back());
    if (e == cudaSuccess) e = cudaEventRecord(b.free_ev[(size_t)k], hs);
    return e;
}

cudaError_t bounce_join(pp_region *r, cudaStream_t s0) {
    if (!r->bounce_used) return cudaSuccess;
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
        e = cudaEventRecord(r->stage_join[i], r->stage_stream[i]);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(s0, r->stage_join[i], 0);
    }
    return e;
}

}  // namespace pprt
