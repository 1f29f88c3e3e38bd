// plan.hpp — the planner: chunk partitioner, ring sizing under a budget, index handler (global plane
// -> ring slot, halo reuse) and the op DAG with its event dependencies. Pure host C++17, no CUDA.
//
//   chunking        P:L220-222 (chunk_size indices, last chunk shorter)
//   ring sizing     P:L316-321 ("array dimensions, chunk_size and num_stream determine the size"),
//                   budget fit P:L336-340 ("tune before we allocate")
//   index handler   P:L300-308 (copy chunk i to position i % slots, replace stale data)
//                   (keep data later chunks still need: halo reuse), P:L400-402 (kernels get a new
//                   base pointer + offsets, body unchanged)
// Readings S7-S11, S13 of DESIGN.md fix what the paper leaves open (plane-granular slots, ring
// capacity R_in = S*c + size - 1 / R_out = S*c, shrink c then S).
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>

namespace pp {

enum class Map : int { To = 1, From = 2, ToFrom = 3 };
enum class OpKind : uint8_t { H2D = 0, KER = 1, D2H = 2 };

struct ArraySpec {
    Map type = Map::To;
    int dtype = 0;                 // pp_dtype
    int ndim = 1;
    int64_t ext[8] = {0};
    int64_t plane_elems = 1;
    int64_t esize = 4;
    int64_t plane_bytes = 4;
    // split geometry (2-D block regions): the array viewed as [outer][nsplit][inner]; a
    // plane is `outer` runs of `inner` contiguous elements, nsplit*inner apart (outer = 1 for dim 0)
    int split_dim = 0;
    int64_t nsplit = 0, outer = 1, inner = 1;
    int64_t off = 0, size = 1;     // window of iteration k: planes [k+off, k+off+size)
    void *host = nullptr;          // host (or device, if resident) base pointer
    bool resident = false;         // device memory: no ring, no copies
    bool pinned = false;
    bool registered = false;       // we cudaHostRegister'ed it (unregister at destroy)
    int alias = -1;                // PP_OPT_INPLACE: index of the input array this output aliases
    bool is_input() const { return type == Map::To || type == Map::ToFrom; }
    bool is_output() const { return type == Map::From || type == Map::ToFrom; }
};

struct PlanParams {
    int64_t lo = 0, hi = 0;
    int64_t chunk = 0;             // requested chunk size (0 = auto)
    int streams = 1;               // requested num_streams
    uint64_t budget = 0;           // ring byte budget (already resolved: 0 never reaches here)
    int policy = 1;                // stream policy (PP_OPT_STREAM_POLICY), default 1
    int64_t ring_extra = -1;       // PP_OPT_RING_EXTRA
    int64_t sweeps = 1;            // > 1: multi-sweep stencil chain (arrs[0] = A0, arrs[1] = output)
    int64_t fuse = 1;              // levels per kernel op of a chain (PP_OPT_FUSE): stages of <= fuse
    uint64_t mirror_gran = 0;      // PP_OPT_MIRROR: > 0 = the ring of a copied array whose bytes are a
                                   // multiple of this (the VMM allocation granularity) is mapped twice
                                   // back to back, so a copy that runs past the ring end is ONE copy
    int fault = 0;                 // PP_OPT_FAULT_INJECT (tests of the checker only):
                                   // 1 drop cross-stream deps, 2 input ring one plane too small,
                                   // 3 no halo reuse (re-copy whole windows), 4 D2H from slot+1
};

struct Ring {
    int64_t R = 0;                 // capacity in planes (0 for resident arrays)
    int64_t base = 0;              // global plane held by slot 0 at the first wrap
    int64_t plane_elems = 0;       // (rings beyond the mapped arrays are device-only level rings)
    uint64_t offset = 0;           // byte offset inside the region's device buffer (plain rings)
    uint64_t bytes = 0;
    bool mirror = false;           // own VMM range [R slots][the same R slots again] (PP_OPT_MIRROR)
};

// One op's access to one array's planes (ring slots) and the value level those planes hold: an H2D
// writes level 0 (the host input), a kernel of stage L reads level L-1 and writes level L, a D2H reads
// the final level. The checker works only from these lists, so every plan builder is checked the same.
struct Acc {
    int32_t arr, level;
    int64_t p0, p1;
    bool write;
};

struct Op {
    OpKind kind;
    int arr = -1;                  // array id (-1 for kernels)
    int level = 1;                 // level a kernel writes (1 for single sweeps; a stage end in 1..T for chains)
    int32_t acc_begin = 0, acc_count = 0;   // into Plan::accs
    int64_t chunk = 0;
    int64_t p0 = 0, p1 = 0;        // planes [p0,p1) (copies); iterations [k0,k1) for kernels
    int64_t s0 = 0;                // ring slot of p0 (copies)
    int stream = 0;
    int32_t dep_begin = 0, dep_count = 0;  // into Plan::deps, pruned (cross-stream, latest only)
    int32_t full_dep_begin = 0, full_dep_count = 0; // unpruned (for the checker)
    bool need_event = false;
};

struct Plan {
    int64_t lo = 0, hi = 0;
    int64_t c = 1;                 // resolved chunk size
    int S = 1;                     // resolved num_streams
    int nstreams = 1;              // CUDA streams used (S, or 3 for per-stage)
    int64_t nchunks = 0;
    std::vector<Ring> rings;       // per array
    uint64_t ring_bytes = 0;       // device bytes of all rings (the budget's measure)
    uint64_t plain_bytes = 0;      // the part in the one plain device buffer (non-mirrored rings)
    std::vector<Op> ops;
    std::vector<Acc> accs;
    // per array: host planes copied in [in_lo, in_hi), drained [out_lo, out_hi) with value level
    // final_level (empty ranges for device-only or resident arrays)
    std::vector<int64_t> in_lo, in_hi, out_lo, out_hi;
    std::vector<int32_t> final_level;
    std::vector<int32_t> deps;
    std::vector<int32_t> full_deps;
    int64_t n_events = 0;
    uint64_t h2d_bytes = 0, d2h_bytes = 0;
    int64_t n_h2d = 0, n_d2h = 0, n_ker = 0, n_waits = 0;
    int64_t chunk_lo(int64_t j) const { return lo + j * c; }
    int64_t chunk_hi(int64_t j) const { int64_t e = lo + (j + 1) * c; return e < hi ? e : hi; }
};

// Status codes mirror pp_status.
enum Err { OK = 0, EINVAL_ = 1, ERANGE_ = 2, EBUDGET_ = 3, EUNSUP_ = 7 };

// Ring capacity (planes) of array a for chunk size c and S streams (0 for resident arrays).
int64_t ring_planes(const ArraySpec &a, const PlanParams &pp, int64_t c, int S);
uint64_t ring_bytes_for(const std::vector<ArraySpec> &arrs, const PlanParams &pp, int64_t c, int S);

// Validate windows and resolve (c, S) under the budget. Returns Err; msg on error.
int resolve(const std::vector<ArraySpec> &arrs, const PlanParams &pp, int64_t *c_out, int *S_out,
            std::string *msg);

// Build the full plan (rings, ops, deps). Returns Err.
int build_plan(const std::vector<ArraySpec> &arrs, const PlanParams &pp, Plan *out, std::string *msg);

// Text dump (pp_plan_dump format).
std::string dump_plan(const Plan &p);

// Simulated execution in random topological orders; returns number of invariant violations.
int64_t check_plan(const std::vector<ArraySpec> &arrs, const Plan &p, int64_t orders, uint64_t seed,
                   std::string *first_violation);

// Balanced slab partition.
void partition(int64_t lo, int64_t hi, int G, int g, int64_t *lo_g, int64_t *hi_g);

// Multi-sweep chains run in stages of up to `fuse` levels: stage s (1..G) turns level
// stage_end(s-1) into level stage_end(s) in one kernel op (halo stage_end(s) - stage_end(s-1)).
inline int64_t chain_fuse(const PlanParams &pp) { return pp.fuse < 1 ? 1 : (pp.fuse > pp.sweeps ? pp.sweeps : pp.fuse); }
inline int64_t chain_stages(const PlanParams &pp) { const int64_t L = chain_fuse(pp); return (pp.sweeps + L - 1) / L; }
inline int64_t stage_end(const PlanParams &pp, int64_t s) { const int64_t e = s * chain_fuse(pp); return e < pp.sweeps ? e : pp.sweeps; }

inline int64_t pmod(int64_t a, int64_t m) { int64_t r = a % m; return r < 0 ? r + m : r; }

}  // namespace pp
