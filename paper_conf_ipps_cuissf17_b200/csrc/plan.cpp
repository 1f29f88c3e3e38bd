// plan.cpp — planner, index handler and schedule checker (pure host). See plan.hpp for citations.
#include "plan.hpp"

#include <algorithm>
#include <cstdio>
#include <map>
#include <random>
#include <tuple>
#include <sstream>

namespace pp {

static int64_t iters_of(const PlanParams &pp) { return pp.hi - pp.lo; }

// A ring is mirrored (one copy per chunk, never split at the wrap) when its array is copied plane-
// contiguously (outer == 1) and its bytes fill whole VMM granules, so it can be mapped twice.
static bool mirrorable(const PlanParams &pp, const ArraySpec &a, const Ring &rg) {
    return pp.mirror_gran > 0 && !a.resident && a.outer == 1 && rg.R > 1 && rg.bytes > 0 &&
           rg.bytes % pp.mirror_gran == 0;
}

int64_t ring_planes(const ArraySpec &a, const PlanParams &pp, int64_t c, int S) {
    if (a.resident) return 0;
    const int64_t n = iters_of(pp);
    if (n <= 0) return 0;
    const int64_t total = n + a.size - 1;          // planes of `a` the whole launch references
    // a multi-sweep chain's first chunk pulls T more input planes ahead (the light cone of T sweeps);
    // a fused first stage of h levels reads 2h planes beyond the c it advances in steady state
    const int64_t lead = (pp.sweeps > 1 && a.is_input()) ? std::max(pp.sweeps - 1, 2 * stage_end(pp, 1) - 2) : 0;
    int64_t R;
    if (pp.ring_extra < 0)                         // full overlap: S chunks in flight (reading S10)
        R = (int64_t)S * c + a.size - 1 + lead;
    else                                           // correctness minimum + extra
        R = c + a.size - 1 + lead + pp.ring_extra;
    R = std::min(R, total);
    if (pp.fault == 2 && a.is_input() && a.size > 1) R = c + a.size - 2;
    return std::max<int64_t>(1, R);
}

// Capacity of the device-only ring of chain stage end s (level e = stage_end(s), 1 <= s < G): its
// first chunk produces planes [lo-1, k1 + T - e); in steady state the next stage (halo h') still
// needs the 2h' planes below the c new ones. Single-level stages: S*c + T - e + 1 as before.
int64_t level_ring_planes(const PlanParams &pp, int64_t c, int S, int64_t s) {
    const int64_t n = iters_of(pp);
    const int64_t e = stage_end(pp, s), h2 = stage_end(pp, s + 1) - e;
    const int64_t need = std::max(pp.sweeps - e + 1, 2 * h2);
    int64_t R = pp.ring_extra < 0 ? (int64_t)S * c + need : c + need + pp.ring_extra;
    return std::max<int64_t>(1, std::min(R, n + 2));
}

uint64_t ring_bytes_for(const std::vector<ArraySpec> &arrs, const PlanParams &pp, int64_t c, int S) {
    uint64_t b = 0;
    for (const auto &a : arrs) {
        // each ring starts 256-byte aligned
        uint64_t rb = (uint64_t)ring_planes(a, pp, c, S) * (uint64_t)a.plane_bytes;
        b += (rb + 255) & ~uint64_t(255);
    }
    if (pp.sweeps > 1 && !arrs.empty() && iters_of(pp) > 0)
        for (int64_t st = 1; st < chain_stages(pp); ++st) {
            uint64_t rb = (uint64_t)level_ring_planes(pp, c, S, st) * (uint64_t)arrs[0].plane_bytes;
            b += (rb + 255) & ~uint64_t(255);
        }
    return b;
}

// Automatic chunk size ("we control the chunk size in the runtime system automatically"):
// aim for >= 16 MiB of input per chunk (the measured host-link size curve saturates there, see
// DESIGN.md §5) — >= 256 MiB for a multi-sweep chain, whose every chunk also pays ceil(T/L) level
// kernels (configs[2]'s 64 MiB planes, T = 8: c = 1 4.24 s, c = 4 4.13 s per pass,
// profiles/r2s2_ooc_temporal_chunk.jsonl) — but keep >= 8*S chunks so fill/drain stays small;
// resident-only launches are one chunk (nothing to overlap).
static int64_t auto_chunk(const std::vector<ArraySpec> &arrs, const PlanParams &pp, int S) {
    const int64_t n = iters_of(pp);
    int64_t in_bytes = 0, any_bytes = 0;
    for (const auto &a : arrs) {
        if (a.resident) continue;
        any_bytes += a.plane_bytes;
        if (a.is_input()) in_bytes += a.plane_bytes;
    }
    if (any_bytes == 0) return std::max<int64_t>(1, n);
    if (in_bytes == 0) in_bytes = any_bytes;
    const int64_t target = pp.sweeps > 1 ? 256ll << 20 : 16ll << 20;
    int64_t c = std::max<int64_t>(1, target / in_bytes);
    int64_t cap = std::max<int64_t>(1, (n + 8 * S - 1) / (8 * S));
    return std::max<int64_t>(1, std::min(c, cap));
}

int resolve(const std::vector<ArraySpec> &arrs, const PlanParams &pp, int64_t *c_out, int *S_out,
            std::string *msg) {
    if (pp.hi < pp.lo) { *msg = "hi < lo"; return EINVAL_; }
    if (pp.streams < 1) { *msg = "num_streams < 1"; return EINVAL_; }
    if (pp.chunk < 0) { *msg = "chunk_size < 0"; return EINVAL_; }
    const int64_t n = iters_of(pp);
    for (size_t i = 0; i < arrs.size(); ++i) {
        const auto &a = arrs[i];
        if (n == 0) break;
        if (pp.lo + a.off < 0 || pp.hi - 1 + a.off + a.size > a.nsplit) {
            char b[256];
            snprintf(b, sizeof b, "array %zu window [%lld,%lld) outside [0,%lld)", i,
                     (long long)(pp.lo + a.off), (long long)(pp.hi - 1 + a.off + a.size),
                     (long long)a.nsplit);
            *msg = b;
            return ERANGE_;
        }
    }
    int S = pp.streams;
    if (n == 0) { *c_out = std::max<int64_t>(1, pp.chunk); *S_out = S; return OK; }
    int64_t creq = pp.chunk > 0 ? pp.chunk : auto_chunk(arrs, pp, S);
    creq = std::min(creq, n);
    // budget fit: shrink c first (keeps S chunks of overlap), then S (reading S11)
    for (; S >= 1; --S) {
        if (ring_bytes_for(arrs, pp, 1, S) > pp.budget) continue;
        int64_t lo = 1, hi = creq;                 // largest c in [1,creq] that fits (monotone)
        while (lo < hi) {
            int64_t mid = lo + (hi - lo + 1) / 2;
            if (ring_bytes_for(arrs, pp, mid, S) <= pp.budget) lo = mid; else hi = mid - 1;
        }
        *c_out = lo;
        *S_out = S;
        return OK;
    }
    char b[256];
    snprintf(b, sizeof b, "ring of %llu bytes at chunk_size=1, num_streams=1 exceeds budget %llu",
             (unsigned long long)ring_bytes_for(arrs, pp, 1, 1), (unsigned long long)pp.budget);
    *msg = b;
    return EBUDGET_;
}

namespace {

struct Builder {
    const std::vector<ArraySpec> &arrs;
    const PlanParams &pp;
    Plan &P;
    std::vector<std::vector<int32_t>> load_op;    // per array: op that loaded plane (p - base)
    std::vector<std::vector<int32_t>> drain_op;   // per array: D2H op that drained plane (p - base)
    std::vector<int32_t> ker_op;                  // per chunk
    std::vector<int32_t> tmp;

    Builder(const std::vector<ArraySpec> &a, const PlanParams &p, Plan &pl) : arrs(a), pp(p), P(pl) {}

    int64_t chunk_of_iter(int64_t k) const { return (k - P.lo) / P.c; }

    bool no_copies = false;                       // every array resident: one stream suffices

    int stream_for(OpKind k, int64_t j, int arr = 0) const {
        const int S = P.S;
        if (no_copies) return 0;
        const int na = (int)arrs.size();
        switch (pp.policy) {
        case 5:                                                 // per-array copy streams: the H2D of
            if (k == OpKind::H2D) return arr;                   // each input on its own stream (copy
            if (k == OpKind::KER) return na;                    // engine), kernels on one, the D2H
            return na + 1 + arr;                                // of each output on its own
        case 1: return (int)k;                                  // per-stage: H2D 0, KER 1, D2H 2
        case 2: return k == OpKind::H2D ? 0 : 1;                // H2D 0; KER then D2H FIFO on 1
        case 3:                                                 // copies round robin over S streams
            if (k == OpKind::H2D) return (int)(j % S);          // per direction, kernels on stream S
            if (k == OpKind::KER) return S;
            return S + 1 + (int)(j % S);
        case 4:                                                 // H2D+KER per-chunk streams, D2H on
            return k == OpKind::D2H ? S + (int)(j % S) : (int)(j % S);   // its own S streams
        default: return (int)(j % S);                           // per-chunk round robin (reading S8)
        }
    }
    static int streams_of(int policy, int S, int na) {
        switch (policy) {
        case 5: return 2 * na + 1;
        case 1: return 3;
        case 2: return 2;
        case 3: return 2 * S + 1;
        case 4: return 2 * S;
        default: return S;
        }
    }

    int32_t emit(Op op, std::vector<int32_t> &deps, const std::vector<Acc> &acc = {}) {
        op.acc_begin = (int32_t)P.accs.size();
        op.acc_count = (int32_t)acc.size();
        P.accs.insert(P.accs.end(), acc.begin(), acc.end());
        std::sort(deps.begin(), deps.end());
        deps.erase(std::unique(deps.begin(), deps.end()), deps.end());
        op.full_dep_begin = (int32_t)P.full_deps.size();
        op.full_dep_count = (int32_t)deps.size();
        P.full_deps.insert(P.full_deps.end(), deps.begin(), deps.end());
        // prune: same-stream deps are implied by FIFO; per other stream only the latest matters
        op.dep_begin = (int32_t)P.deps.size();
        std::vector<int32_t> latest(P.nstreams, -1);
        for (int32_t d : deps) {
            int st = P.ops[d].stream;
            if (st == op.stream) continue;
            latest[st] = std::max(latest[st], d);
        }
        for (int st = 0; st < P.nstreams; ++st)
            if (latest[st] >= 0 && pp.fault != 1) {
                P.deps.push_back(latest[st]);
                P.ops[latest[st]].need_event = true;
            }
        op.dep_count = (int32_t)(P.deps.size() - op.dep_begin);
        P.n_waits += op.dep_count;
        P.ops.push_back(op);
        deps.clear();
        return (int32_t)P.ops.size() - 1;
    }

    // kernels of every chunk that reads any plane in [o0,o1) of array a
    void readers(int ai, int64_t o0, int64_t o1, std::vector<int32_t> &deps) {
        const auto &a = arrs[ai];
        int64_t kmin = std::max(P.lo, o0 - a.off - a.size + 1);
        int64_t kmax = std::min(P.hi - 1, o1 - 1 - a.off);
        if (kmin > kmax) return;
        // (a reader that is the current or a later chunk only happens with a ring smaller than one
        // chunk's window — fault mode 2 — and is left for the checker to report)
        for (int64_t j = chunk_of_iter(kmin); j <= chunk_of_iter(kmax); ++j)
            if (ker_op[j] >= 0) deps.push_back(ker_op[j]);
    }

    void drains(int ai, int64_t o0, int64_t o1, std::vector<int32_t> &deps) {
        const Ring &rg = P.rings[ai];
        for (int64_t q = std::max(o0, rg.base); q < o1; ++q) {
            int32_t d = drain_op[ai][q - rg.base];
            if (d >= 0) deps.push_back(d);
        }
    }

    void copy_ops(OpKind kind, int ai, int64_t j, int64_t p0, int64_t p1, const std::vector<int32_t> &deps_in) {
        const Ring &rg = P.rings[ai];
        const auto &a = arrs[ai];
        int64_t p = p0;
        while (p < p1) {
            int64_t s0 = pmod(p - rg.base, rg.R);
            if (pp.fault == 4 && kind == OpKind::D2H) s0 = pmod(s0 + 1, rg.R);
            // split at the ring wrap (<= 2 segments), unless the ring is mirrored: then one copy
            int64_t n = std::min(p1 - p, rg.mirror ? rg.R : rg.R - s0);
            std::vector<int32_t> deps = deps_in;
            if (kind == OpKind::H2D) {
                // previous occupants of the target slots must no longer be needed
                int64_t o0 = p - rg.R, o1 = p + n - rg.R;
                if (o1 > rg.base) {
                    readers(ai, std::max(o0, rg.base), o1, deps);
                    if (a.type == Map::ToFrom) drains(ai, o0, o1, deps);
                }
            }
            Op op{kind};
            op.arr = ai;
            op.chunk = j;
            op.p0 = p;
            op.p1 = p + n;
            op.s0 = s0;
            op.stream = stream_for(kind, j, ai);
            // H2D writes the host input (level 0); D2H reads the kernel's output (level 1)
            int32_t id = emit(op, deps, {Acc{ai, kind == OpKind::H2D ? 0 : 1, p, p + n, kind == OpKind::H2D}});
            for (int64_t q = p; q < p + n; ++q) {
                if (kind == OpKind::H2D) load_op[ai][q - rg.base] = id;
                else drain_op[ai][q - rg.base] = id;
            }
            uint64_t bytes = (uint64_t)n * (uint64_t)a.plane_bytes;
            if (kind == OpKind::H2D) { P.h2d_bytes += bytes; P.n_h2d++; }
            else { P.d2h_bytes += bytes; P.n_d2h++; }
            p += n;
        }
    }

    // Would any copy of array i cross the end of its (unmirrored) ring? The same plane ranges as the
    // copies run() emits below; a ring none of whose copies wraps gains nothing from a mirror (and
    // stays in the one plain buffer, where PP_OPT_MERGE_COPIES can use it).
    bool wraps(int i) const {
        const Ring &rg = P.rings[i];
        const auto &a = arrs[i];
        auto crosses = [&](int64_t p, int64_t n, bool d2h) {
            int64_t s0 = pmod(p - rg.base, rg.R);
            if (pp.fault == 4 && d2h) s0 = pmod(s0 + 1, rg.R);
            return s0 + n > rg.R;
        };
        int64_t loaded = rg.base;
        for (int64_t j = 0; j < P.nchunks; ++j) {
            const int64_t k0 = P.chunk_lo(j), k1 = P.chunk_hi(j);
            if (a.is_input()) {
                const int64_t wlo = k0 + a.off, whi = k1 + a.off + a.size - 1;
                const int64_t p0 = pp.fault == 3 ? wlo : std::max(loaded, wlo);
                if (p0 < whi && crosses(p0, whi - p0, false)) return true;
                loaded = std::max(loaded, whi);
            }
            if (a.is_output() && crosses(k0 + a.off, k1 - k0, true)) return true;
        }
        return false;
    }

    void run() {
        const int na = (int)arrs.size();
        P.rings.assign(na, Ring{});
        P.nchunks = (P.hi - P.lo + P.c - 1) / P.c;
        uint64_t off = 0, mirrored = 0;
        for (int i = 0; i < na; ++i) {
            Ring &rg = P.rings[i];
            rg.R = ring_planes(arrs[i], pp, P.c, P.S);
            rg.base = P.lo + arrs[i].off;
            rg.bytes = (uint64_t)rg.R * (uint64_t)arrs[i].plane_bytes;
            rg.plane_elems = arrs[i].plane_elems;
            rg.mirror = mirrorable(pp, arrs[i], rg) && wraps(i);
            if (rg.mirror) {
                mirrored += rg.bytes;
            } else {
                rg.offset = off;
                off += (rg.bytes + 255) & ~uint64_t(255);
            }
            if (arrs[i].resident) { rg.R = arrs[i].nsplit; rg.base = 0; rg.bytes = 0; }
        }
        P.plain_bytes = off;
        P.ring_bytes = off + mirrored;
        no_copies = std::all_of(arrs.begin(), arrs.end(), [](const ArraySpec &a) { return a.resident; });
        P.nstreams = no_copies ? 1 : streams_of(pp.policy, P.S, na);
        load_op.assign(na, {});
        drain_op.assign(na, {});
        for (int i = 0; i < na; ++i) {
            if (arrs[i].resident) continue;
            int64_t span = (P.hi - P.lo) + arrs[i].size - 1;
            load_op[i].assign(span, -1);
            drain_op[i].assign(span, -1);
        }
        ker_op.assign(P.nchunks, -1);
        P.in_lo.assign(na, 0);
        P.in_hi.assign(na, 0);
        P.out_lo.assign(na, 0);
        P.out_hi.assign(na, 0);
        P.final_level.assign(na, 1);
        for (int i = 0; i < na; ++i) {
            const auto &a = arrs[i];
            if (a.resident) continue;
            if (a.is_input()) { P.in_lo[i] = P.lo + a.off; P.in_hi[i] = P.hi + a.off + a.size - 1; }
            if (a.is_output()) { P.out_lo[i] = P.lo + a.off; P.out_hi[i] = P.hi + a.off; }
        }
        std::vector<int64_t> loaded_hi(na);
        for (int i = 0; i < na; ++i) loaded_hi[i] = P.rings[i].base;
        std::vector<int32_t> deps;
        for (int64_t j = 0; j < P.nchunks; ++j) {
            const int64_t k0 = P.chunk_lo(j), k1 = P.chunk_hi(j);
            // H2D of the planes this chunk needs that are not yet in the ring (halo reuse, S13)
            for (int i = 0; i < na; ++i) {
                const auto &a = arrs[i];
                if (a.resident || !a.is_input()) continue;
                int64_t wlo = k0 + a.off, whi = k1 + a.off + a.size - 1;
                int64_t p0 = pp.fault == 3 ? wlo : std::max(loaded_hi[i], wlo);
                if (p0 < whi) copy_ops(OpKind::H2D, i, j, p0, whi, {});
                loaded_hi[i] = std::max(loaded_hi[i], whi);
            }
            // kernel: waits for the loads of its whole window and for the drains of its out-slots
            for (int i = 0; i < na; ++i) {
                const auto &a = arrs[i];
                if (a.resident) continue;
                const Ring &rg = P.rings[i];
                if (a.is_input())
                    for (int64_t q = k0 + a.off; q < k1 + a.off + a.size - 1; ++q)
                        deps.push_back(load_op[i][q - rg.base]);
                if (a.is_output()) drains(i, k0 + a.off - rg.R, k1 + a.off - rg.R, deps);
            }
            Op ko{OpKind::KER};
            ko.chunk = j;
            ko.p0 = k0;
            ko.p1 = k1;
            ko.stream = stream_for(OpKind::KER, j);
            std::vector<Acc> acc;
            for (int i = 0; i < na; ++i) {
                const auto &a = arrs[i];
                if (a.resident) continue;
                if (a.is_input()) acc.push_back(Acc{i, 0, k0 + a.off, k1 + a.off + a.size - 1, false});
                if (a.is_output()) acc.push_back(Acc{i, 1, k0 + a.off, k1 + a.off, true});
            }
            ker_op[j] = emit(ko, deps, acc);
            P.n_ker++;
            // D2H of the chunk's output planes
            for (int i = 0; i < na; ++i) {
                const auto &a = arrs[i];
                if (a.resident || !a.is_output()) continue;
                copy_ops(OpKind::D2H, i, j, k0 + a.off, k1 + a.off, {ker_op[j]});
            }
        }
        for (auto &op : P.ops)
            if (op.need_event) P.n_events++;
    }
};


// -----------------------------------------------------------------------------------------------
// Multi-sweep chain (temporal blocking): T Jacobi sweeps of the Fig. 2 body
// (the Parboil stencil is iterative) streamed through the link ONCE. Level 0 is the input
// ring (A0 planes [lo-1, hi+1)); level t (1 <= t < T) is a device-only ring of A^t planes over the
// same domain, whose two boundary planes lo-1 and hi are copies (they never change); level T is the
// output ring (A^T planes [lo, hi)). Output chunk j = [k0,k1) needs level t up to plane
// k1 + T - t (the light cone), so each chunk loads its new input planes, advances every level by
// the planes that became computable (one kernel op per level, in order), then drains [k0,k1).
// Dependencies come from per-plane producer/reader tracking: a read waits for the plane's producer;
// overwriting a ring slot waits for every reader (and the producer) of its previous occupant.
// -----------------------------------------------------------------------------------------------
struct ChainBuilder {
    const std::vector<ArraySpec> &arrs;
    const PlanParams &pp;
    Plan &P;
    Builder base;                                  // reuses emit() and the stream mapping
    struct Track {
        std::vector<int32_t> producer;
        std::vector<std::vector<int32_t>> readers;
        int64_t dom_lo = 0;
    };
    std::vector<Track> tr;                         // per ring

    ChainBuilder(const std::vector<ArraySpec> &a, const PlanParams &p, Plan &pl) : arrs(a), pp(p), P(pl), base(a, p, pl) {}

    int64_t G = 1;                                 // stages
    int ring_of_stage(int64_t s) const { return s == 0 ? 0 : (s == G ? 1 : (int)(1 + s)); }

    void slot_reuse_deps(int ring, int64_t p0, int64_t p1, std::vector<int32_t> &deps) {
        const Ring &rg = P.rings[ring];
        Track &t = tr[ring];
        for (int64_t p = p0; p < p1; ++p) {
            const int64_t q = p - rg.R;
            if (q < t.dom_lo) continue;
            const int64_t i = q - t.dom_lo;
            for (int32_t r : t.readers[i]) deps.push_back(r);
            if (t.producer[i] >= 0) deps.push_back(t.producer[i]);
        }
    }
    void read_deps(int ring, int64_t p0, int64_t p1, std::vector<int32_t> &deps) {
        Track &t = tr[ring];
        for (int64_t p = p0; p < p1; ++p)
            if (t.producer[p - t.dom_lo] >= 0) deps.push_back(t.producer[p - t.dom_lo]);
    }
    void mark(int ring, int64_t p0, int64_t p1, int32_t op, bool write) {
        Track &t = tr[ring];
        for (int64_t p = p0; p < p1; ++p) {
            if (write) { t.producer[p - t.dom_lo] = op; t.readers[p - t.dom_lo].clear(); }
            else t.readers[p - t.dom_lo].push_back(op);
        }
    }

    void copy(OpKind kind, int ring, int64_t j, int64_t p0, int64_t p1) {
        const Ring &rg = P.rings[ring];
        const int64_t pb = (int64_t)rg.plane_elems * arrs[0].esize;
        const int level = kind == OpKind::H2D ? 0 : (int)pp.sweeps;
        int64_t p = p0;
        while (p < p1) {
            const int64_t s0 = pmod(p - rg.base, rg.R);
            const int64_t n = std::min(p1 - p, rg.mirror ? rg.R : rg.R - s0);
            std::vector<int32_t> deps;
            if (kind == OpKind::H2D) slot_reuse_deps(ring, p, p + n, deps);
            else read_deps(ring, p, p + n, deps);
            Op op{kind};
            op.arr = ring;
            op.chunk = j;
            op.p0 = p;
            op.p1 = p + n;
            op.s0 = s0;
            op.stream = base.stream_for(kind, j, ring);
            const int32_t id = base.emit(op, deps, {Acc{ring, level, p, p + n, kind == OpKind::H2D}});
            mark(ring, p, p + n, id, kind == OpKind::H2D);
            const uint64_t bytes = (uint64_t)n * (uint64_t)pb;
            if (kind == OpKind::H2D) { P.h2d_bytes += bytes; P.n_h2d++; }
            else { P.d2h_bytes += bytes; P.n_d2h++; }
            p += n;
        }
    }

    void run() {
        const int64_t T = pp.sweeps, lo = P.lo, hi = P.hi;
        G = chain_stages(pp);
        const int nr = (int)(G + 1);               // ring 0 = A0, 1 = output, 2.. = stage ends 1..G-1
        const ArraySpec &A = arrs[0], &Y = arrs[1];
        P.rings.assign(nr, Ring{});
        uint64_t off = 0, mirrored = 0;
        auto place = [&](int i, int64_t R, int64_t b, int64_t elems, int64_t esize, const ArraySpec *copied) {
            Ring &rg = P.rings[i];
            rg.R = R;
            rg.base = b;
            rg.plane_elems = elems;
            rg.bytes = (uint64_t)R * (uint64_t)(elems * esize);
            rg.mirror = copied && mirrorable(pp, *copied, rg);   // level rings have no copies
            if (rg.mirror) {
                mirrored += rg.bytes;
            } else {
                rg.offset = off;
                off += (rg.bytes + 255) & ~uint64_t(255);
            }
        };
        place(0, ring_planes(A, pp, P.c, P.S), lo - 1, A.plane_elems, A.esize, &A);
        place(1, ring_planes(Y, pp, P.c, P.S), lo + Y.off, Y.plane_elems, Y.esize, &Y);
        for (int64_t st = 1; st < G; ++st) place((int)(1 + st), level_ring_planes(pp, P.c, P.S, st), lo - 1, A.plane_elems, A.esize, nullptr);
        P.plain_bytes = off;
        P.ring_bytes = off + mirrored;
        P.nchunks = (hi - lo + P.c - 1) / P.c;
        P.nstreams = Builder::streams_of(pp.policy, P.S, (int)arrs.size());
        base.no_copies = false;
        P.in_lo.assign(nr, 0);
        P.in_hi.assign(nr, 0);
        P.out_lo.assign(nr, 0);
        P.out_hi.assign(nr, 0);
        P.final_level.assign(nr, 0);
        P.in_lo[0] = lo - 1;
        P.in_hi[0] = hi + 1;
        P.out_lo[1] = lo;
        P.out_hi[1] = hi;
        P.final_level[1] = (int32_t)T;
        tr.assign(nr, Track{});
        for (int i = 0; i < nr; ++i) {
            tr[i].dom_lo = i == 1 ? lo : lo - 1;
            const int64_t span = i == 1 ? hi - lo : hi - lo + 2;
            tr[i].producer.assign(span, -1);
            tr[i].readers.assign(span, {});
        }
        std::vector<int64_t> produced(G + 1, lo - 1);   // per stage end: planes [lo-1, produced)
        produced[G] = lo;
        for (int64_t j = 0; j < P.nchunks; ++j) {
            const int64_t k0 = P.chunk_lo(j), k1 = P.chunk_hi(j);
            const int64_t in_hi = std::min(hi + 1, k1 + T);
            if (produced[0] < in_hi) copy(OpKind::H2D, 0, j, produced[0], in_hi);
            produced[0] = std::max(produced[0], in_hi);
            for (int64_t st = 1; st <= G; ++st) {
                const int64_t e = stage_end(pp, st), h = e - stage_end(pp, st - 1);
                const int64_t p0 = produced[st];
                const int64_t p1 = st < G ? std::min(hi + 1, k1 + T - e) : k1;
                if (p0 >= p1) continue;
                // the stage reads h planes of halo each side; the fixed planes lo-1, hi only their own
                const int64_t r0 = std::max(lo - 1, p0 - h);
                const int64_t r1 = std::min(hi + 1, p1 + h);
                const int rin = ring_of_stage(st - 1), rout = ring_of_stage(st);
                std::vector<int32_t> deps;
                read_deps(rin, r0, r1, deps);
                slot_reuse_deps(rout, p0, p1, deps);
                Op ko{OpKind::KER};
                ko.chunk = j;
                ko.level = (int)e;
                ko.p0 = p0;
                ko.p1 = p1;
                ko.stream = base.stream_for(OpKind::KER, j);
                const int32_t id = base.emit(ko, deps, {Acc{rin, (int32_t)(e - h), r0, r1, false},
                                                        Acc{rout, (int32_t)e, p0, p1, true}});
                mark(rin, r0, r1, id, false);
                mark(rout, p0, p1, id, true);
                P.n_ker++;
                produced[st] = p1;
            }
            copy(OpKind::D2H, 1, j, k0, k1);
        }
        for (auto &op : P.ops)
            if (op.need_event) P.n_events++;
    }
};

}  // namespace

int build_plan(const std::vector<ArraySpec> &arrs, const PlanParams &pp, Plan *out, std::string *msg) {
    int64_t c;
    int S;
    int rc = resolve(arrs, pp, &c, &S, msg);
    if (rc != OK) return rc;
    Plan P;
    P.lo = pp.lo;
    P.hi = pp.hi;
    P.c = c;
    P.S = S;
    if (pp.hi > pp.lo && pp.sweeps > 1) {
        ChainBuilder b(arrs, pp, P);
        b.run();
    } else if (pp.hi > pp.lo) {
        Builder b(arrs, pp, P);
        b.run();
    } else {
        P.nstreams = Builder::streams_of(pp.policy, S, (int)arrs.size());
    }
    *out = std::move(P);
    return OK;
}

std::string dump_plan(const Plan &p) {
    std::ostringstream os;
    os << "PLAN c=" << p.c << " S=" << p.S << " N=" << p.nchunks << " streams=" << p.nstreams
       << " ring_bytes=" << p.ring_bytes << " R=";
    for (size_t i = 0; i < p.rings.size(); ++i) os << (i ? "," : "") << p.rings[i].R;
    os << " mirror=";
    for (size_t i = 0; i < p.rings.size(); ++i) os << (i ? "," : "") << (int)p.rings[i].mirror;
    os << "\n";
    static const char *names[] = {"H2D", "KER", "D2H"};
    for (const auto &op : p.ops) {
        os << names[(int)op.kind] << " j=" << op.chunk << " a=" << (op.kind == OpKind::KER ? op.level : op.arr)
           << " p=" << op.p0 << ":" << op.p1
           << " s=" << op.s0 << " st=" << op.stream << " deps=";
        for (int32_t d = 0; d < op.dep_count; ++d) os << (d ? "," : "") << p.deps[op.dep_begin + d];
        os << "\n";
    }
    return os.str();
}

// ---------------------------------------------------------------------------------------------
// Schedule checker. Two independent checks of the SAME constraint set the GPU enforces (pruned
// event deps + same-stream FIFO):
//  (1) race freedom: every pair of ops touching the same ring slot, at least one writing, is ordered
//      by happens-before (so overlapping copies/kernels can never corrupt a slot);
//  (2) semantics under random topological orders: slot tags prove each kernel sees exactly the
//      planes its window needs; every iteration runs once; each input plane is copied in once;
//      every output plane is drained once with its computed content; <= 2 segments per chunk.
// ---------------------------------------------------------------------------------------------
int64_t check_plan(const std::vector<ArraySpec> &arrs, const Plan &P, int64_t orders, uint64_t seed,
                   std::string *first) {
    int64_t bad = 0;
    auto viol = [&](const std::string &s) {
        if (bad == 0 && first) *first = s;
        ++bad;
    };
    const int64_t N = (int64_t)P.ops.size();
    const int na = (int)P.rings.size();
    if (N == 0) return 0;
    auto slot_of = [&](int ai, int64_t p) { return pmod(p - P.rings[ai].base, P.rings[ai].R); };
    // predecessor lists: pruned deps + FIFO predecessor on the same stream
    std::vector<std::vector<int32_t>> preds(N);
    std::vector<int32_t> last_on(P.nstreams, -1);
    for (int64_t i = 0; i < N; ++i) {
        const Op &op = P.ops[i];
        for (int32_t d = 0; d < op.dep_count; ++d) preds[i].push_back(P.deps[op.dep_begin + d]);
        if (last_on[op.stream] >= 0) preds[i].push_back(last_on[op.stream]);
        last_on[op.stream] = (int32_t)i;
        for (int32_t d : preds[i])
            if (d >= i) viol("dependency on a later op");
    }
    // (1) happens-before closure (issue order is topological)
    const int64_t W = (N + 63) / 64;
    std::vector<uint64_t> reach((size_t)(N * W), 0);
    for (int64_t i = 0; i < N; ++i) {
        uint64_t *ri = &reach[(size_t)(i * W)];
        for (int32_t d : preds[i]) {
            const uint64_t *rd = &reach[(size_t)((int64_t)d * W)];
            for (int64_t w = 0; w < W; ++w) ri[w] |= rd[w];
            ri[d / 64] |= 1ull << (d % 64);
        }
    }
    auto hb = [&](int64_t a, int64_t b) { return (reach[(size_t)(b * W + a / 64)] >> (a % 64)) & 1; };
    // (1a) race freedom on ring slots, from the ops' explicit access lists
    struct SAcc { int64_t op, s0, s1; bool w; };
    std::vector<std::vector<SAcc>> sacc(na);
    for (int64_t i = 0; i < N; ++i) {
        const Op &op = P.ops[i];
        for (int32_t x = 0; x < op.acc_count; ++x) {
            const Acc &A = P.accs[op.acc_begin + x];
            const Ring &rg = P.rings[A.arr];
            int64_t n = A.p1 - A.p0;
            if (n <= 0) continue;
            if (n > rg.R) viol("slot index out of ring");
            // copies address the ring exactly as the executor does (op.s0); kernels via base/R
            int64_t s0 = op.kind == OpKind::KER ? slot_of(A.arr, A.p0) : op.s0 + (A.p0 - op.p0);
            if (op.kind != OpKind::KER && s0 + n > rg.R && !rg.mirror) viol("copy segment crosses ring end");
            while (n > 0) {                                          // split at the wrap
                int64_t m = std::min(n, rg.R - s0);
                sacc[A.arr].push_back({i, s0, s0 + m, A.write});
                n -= m;
                s0 = 0;
            }
        }
    }
    for (int ai = 0; ai < na; ++ai) {
        const auto &acc = sacc[ai];
        for (size_t x = 0; x < acc.size(); ++x)
            for (size_t y = x + 1; y < acc.size(); ++y) {
                const SAcc &A = acc[x], &B = acc[y];
                if (A.op == B.op || !(A.w || B.w)) continue;
                if (A.s1 <= B.s0 || B.s1 <= A.s0) continue;
                if (!hb(A.op, B.op)) {
                    char b[200];
                    snprintf(b, sizeof b, "race: array %d ops %lld and %lld share slots unordered", ai,
                             (long long)A.op, (long long)B.op);
                    viol(b);
                }
            }
    }
    // (1b) in-place host aliases: the D2H that overwrites host plane p of an aliased output must be
    //      ordered after the H2D that copied host plane p of the input it aliases
    for (int yi = 0; yi < (int)arrs.size(); ++yi) {
        const int xi = arrs[yi].alias;
        if (xi < 0) continue;
        std::vector<int64_t> h2d_of(std::max<int64_t>(0, P.in_hi[xi] - P.in_lo[xi]), -1);
        for (int64_t i = 0; i < N; ++i) {
            const Op &op = P.ops[i];
            if (op.kind == OpKind::H2D && op.arr == xi)
                for (int64_t q = op.p0; q < op.p1; ++q) h2d_of[q - P.in_lo[xi]] = i;
        }
        for (int64_t i = 0; i < N; ++i) {
            const Op &op = P.ops[i];
            if (op.kind != OpKind::D2H || op.arr != yi) continue;
            for (int64_t q = op.p0; q < op.p1; ++q) {
                const int64_t src = q - P.in_lo[xi];
                if (src < 0 || src >= (int64_t)h2d_of.size()) continue;   // plane never copied in
                const int64_t h = h2d_of[src];
                if (h >= 0 && !(h < i && hb(h, i))) viol("in-place: host plane overwritten before it was copied in");
            }
        }
    }
    // (2) semantics under random topological orders: slots hold (level, plane) tags
    std::mt19937_64 rng(seed);
    const int64_t TAG_BAD = -1;
    auto tag = [](int64_t level, int64_t p) { return level * (int64_t(1) << 40) + p; };
    for (int64_t o = 0; o < orders; ++o) {
        std::vector<std::vector<int64_t>> slots(na);
        std::vector<std::vector<int32_t>> nload(na), ndrain(na);
        std::vector<std::vector<int64_t>> host(na);
        std::vector<std::map<int64_t, int32_t>> nwrite(na);      // (level, plane) -> kernel writes
        for (int ai = 0; ai < na; ++ai) {
            slots[ai].assign((size_t)std::max<int64_t>(0, P.rings[ai].R), TAG_BAD);
            nload[ai].assign((size_t)std::max<int64_t>(0, P.in_hi[ai] - P.in_lo[ai]), 0);
            ndrain[ai].assign((size_t)std::max<int64_t>(0, P.out_hi[ai] - P.out_lo[ai]), 0);
            host[ai].assign((size_t)std::max<int64_t>(0, P.out_hi[ai] - P.out_lo[ai]), TAG_BAD);
        }
        std::vector<int32_t> indeg(N, 0);
        std::vector<std::vector<int32_t>> succ(N);
        for (int64_t i = 0; i < N; ++i)
            for (int32_t d : preds[i]) { indeg[i]++; succ[d].push_back((int32_t)i); }
        std::vector<int32_t> ready;
        for (int64_t i = 0; i < N; ++i)
            if (!indeg[i]) ready.push_back((int32_t)i);
        int64_t done = 0;
        while (!ready.empty()) {
            size_t pick = (size_t)(rng() % ready.size());
            int32_t i = ready[pick];
            ready[pick] = ready.back();
            ready.pop_back();
            ++done;
            const Op &op = P.ops[i];
            if (op.kind == OpKind::H2D) {
                for (int64_t p = op.p0; p < op.p1; ++p) {
                    slots[op.arr][pmod(op.s0 + (p - op.p0), P.rings[op.arr].R)] = tag(0, p);
                    const int64_t q = p - P.in_lo[op.arr];
                    if (q >= 0 && q < (int64_t)nload[op.arr].size()) nload[op.arr][q]++;
                    else viol("H2D of a plane outside the input domain");
                }
            } else if (op.kind == OpKind::D2H) {
                for (int64_t p = op.p0; p < op.p1; ++p) {
                    const int64_t q = p - P.out_lo[op.arr];
                    if (q < 0 || q >= (int64_t)host[op.arr].size()) { viol("D2H of a plane outside the output domain"); continue; }
                    host[op.arr][q] = slots[op.arr][pmod(op.s0 + (p - op.p0), P.rings[op.arr].R)];
                    ndrain[op.arr][q]++;
                }
            } else {
                bool ok = true;
                for (int32_t x = 0; x < op.acc_count; ++x) {
                    const Acc &A = P.accs[op.acc_begin + x];
                    if (A.write) continue;
                    for (int64_t q = A.p0; q < A.p1; ++q)
                        if (slots[A.arr][slot_of(A.arr, q)] != tag(A.level, q)) ok = false;
                }
                if (!ok) viol("kernel window slot holds the wrong plane");
                for (int32_t x = 0; x < op.acc_count; ++x) {
                    const Acc &A = P.accs[op.acc_begin + x];
                    if (!A.write) continue;
                    for (int64_t p = A.p0; p < A.p1; ++p) {
                        slots[A.arr][slot_of(A.arr, p)] = ok ? tag(A.level, p) : TAG_BAD;
                        nwrite[A.arr][tag(A.level, p)]++;
                    }
                }
            }
            for (int32_t s : succ[i])
                if (--indeg[s] == 0) ready.push_back(s);
        }
        if (done != N) viol("deadlock: dependency cycle");
        for (int ai = 0; ai < na; ++ai) {
            for (int32_t n : nload[ai])
                if (n != 1) viol("input plane not copied in exactly once");
            for (size_t q = 0; q < ndrain[ai].size(); ++q) {
                if (ndrain[ai][q] != 1) viol("output plane not drained exactly once");
                if (host[ai][q] != tag(P.final_level[ai], P.out_lo[ai] + (int64_t)q))
                    viol("output plane drained with wrong content");
            }
            for (const auto &kv : nwrite[ai])
                if (kv.second != 1) viol("iteration not executed exactly once");
        }
    }
    // <= 2 copy segments per array per chunk; exactly one on a mirrored ring
    std::map<std::tuple<int64_t, int, int>, int> segs;
    for (int64_t i = 0; i < N; ++i) {
        const Op &op = P.ops[i];
        if (op.kind == OpKind::KER) continue;
        const int n = ++segs[std::make_tuple(op.chunk, op.arr, (int)op.kind)];
        if (n > 2) viol("more than 2 copy segments for one array in one chunk");
        else if (n > 1 && P.rings[op.arr].mirror) viol("a mirrored ring's copy was split");
    }
    return bad;
}

void partition(int64_t lo, int64_t hi, int G, int g, int64_t *lo_g, int64_t *hi_g) {
    int64_t n = hi - lo, q = n / G, r = n % G;
    int64_t a = lo + g * q + std::min<int64_t>(g, r);
    *lo_g = a;
    *hi_g = a + q + (g < r ? 1 : 0);
}

}  // namespace pp
