// kernels.cuh — launcher interface of the per-chunk loop bodies (sm_100a). Host-callable.
//
// Every kernel addresses array planes through a DView: the index handler's "new base pointer and
// offsets". Global plane p of an array lives at
//     ring + ((p - base) mod R) * plane_elems            (element units)
// (chunk i goes to position i % slots; here plane-granular, reading S9). A resident
// array is the degenerate view ring = array, R = extent, base = 0. Kernels step slots with an
// incremental wrap, never a per-element modulo.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace pp {

struct DView {
    void *ring;
    int64_t R;
    int64_t base;
    int64_t plane_elems;
    // 2-D block regions: a plane is `outer` runs of plane_elems/outer elements; consecutive runs are
    // `ostride` elements apart in the ring ([outer][R][inner] layout). outer = 1 for dim-0 splits.
    int64_t outer = 1, ostride = 0;
};

// Stencil kernel paths (PP_OPT_KERNEL_PATH).
enum { KPATH_AUTO = 0, KPATH_GENERIC = 1, KPATH_TMA = 2 };

// PAPER.md Fig. 2 body for output planes k in [k0,k1):
//   out(k + out_shift) = stencil of in planes (k-1, k, k+1) shifted by in_shift, where the caller
//   passes in/out views and shifts so that "plane k" of the loop maps to the right global planes.
// Iterations k outside the interior range [ilo, ihi) are whole-plane copies out = in(k) (the fixed
// boundary planes of a multi-sweep chain); pass INT64_MIN/INT64_MAX for none.
// dtype: 0 f32, 1 f64, 2 i64. Edge points of each plane: out = in (reading S5).
// path: KPATH_* request; *path_used receives what ran. Returns cudaErrorNotSupported if TMA was
// forced and the shape/alignment does not allow it.
cudaError_t launch_stencil7(int dtype, const DView &in, int64_t in_shift, const DView &out,
                            int64_t out_shift, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                            int64_t ilo, int64_t ihi, double c0, double c1, bool fmad, int path,
                            int *path_used, cudaStream_t st);

// h in [2, kMaxFuse] Jacobi sweeps of the Fig. 2 body in one pass (temporal blocking on chip):
// level-h planes [k0,k1) into `out` from level-0 planes of `in`, which must hold planes
// [max(k0-h, dlo), min(k1+h, dhi)); [dlo,dhi) is the plane domain and planes outside [ilo,ihi) are
// copies at every level (needs dlo < ilo, ihi < dhi). Edge points copy. Bit-identical to h
// single-level launches. f32/f64 with 16-byte row pitch only: cudaErrorNotSupported otherwise.
constexpr int kMaxFuse = 4;
bool stencil7_fused_supported(int dtype, int h, const DView &in, const DView &out, int64_t ny, int64_t nx);
cudaError_t launch_stencil7_fused(int dtype, int h, const DView &in, const DView &out, int64_t ny, int64_t nx,
                                  int64_t k0, int64_t k1, int64_t dlo, int64_t dhi, int64_t ilo, int64_t ihi,
                                  double c0, double c1, bool fmad, cudaStream_t st);

// Polybench 3DCONV body (reading C1): out(k + out_shift) from in planes (k-1, k, k+1) +
// in_shift, fixed coefficients, Polybench's summation order; edge points copy in. dtype 0 f32, 1 f64.
cudaError_t launch_conv3d(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                          int64_t ny, int64_t nx, int64_t k0, int64_t k1, int path, int *path_used,
                          cudaStream_t st);

// c(k + sc) = a(k + sa) + s * b(k + sb), elementwise over each plane, k in [k0,k1).
cudaError_t launch_triad(int dtype, const DView &a, int64_t sa, const DView &b, int64_t sb,
                         const DView &c, int64_t sc, int64_t k0, int64_t k1, double s, bool fmad,
                         cudaStream_t st);

// out(k + so) = in(k - 1 + si) + 3 in(k + si) + 9 in(k + 1 + si), int64 wrap, k in [k0,k1).
// Device-side schedule check (PP_OPT_DEBUG_TAGS): every ring slot carries a tag (plane << 8 | value
// level). Before an op, a check kernel on the op's stream compares the tags of every slot the op
// reads with what the plan says it reads (and counts drains per output plane); after it, a write
// kernel stamps the slots the op wrote. Violations are counted in err[0]; err[1..4] = first one
// (op index, ring, plane, tag found).
constexpr int kTagAccMax = 6;
struct TagAcc {
    int64_t *tags;             // the ring's tag array (R entries)
    int64_t R, s0, p0, p1;     // planes [p0, p1) in slots (s0 + (p - p0)) mod R
    int32_t level, write;
    int32_t *visits;           // drains per output plane (D2H reads), or null
    int64_t vbase;             // plane of visits[0]
};
struct TagOp {
    int32_t n, op;
    TagAcc a[kTagAccMax];
};
cudaError_t launch_tags(const TagOp &t, int phase /*0 check reads, 1 stamp writes*/, int64_t *err, cudaStream_t st);

// PP_OPT_SM_COPY: a host<->ring copy done by the SMs (16-byte loads/stores through the host-mapped
// pinned pages over PCIe) instead of the copy engine: no DMA descriptor setup, for small copies
cudaError_t launch_sm_copy(void *dst, const void *src, size_t bytes, cudaStream_t st);

// PP_OPT_PERSISTENT: flag words shared by the copy streams (stream memory operations) and the
// persistent pipeline kernel (stencil_tma.cu). Zeroed at the start of every launch.
struct PipeFlags {
    uint32_t loaded;                    // chunks whose H2D copies are complete
    uint32_t drained;                   // chunks whose D2H copies are complete
    uint32_t computed;                  // chunks every CTA has finished (monotonic: atomicMax)
    uint32_t err;                       // a gate timed out: the launch fails
    unsigned long long arrivals;        // CTA-chunk completions so far
};
// Launch the persistent pipeline stencil over iterations [lo, hi) in chunks of c, S chunks in flight;
// returns cudaErrorNotSupported if the shape cannot use it (TMA rules, or the grid would not be fully
// resident). *grid gets the CTA count.
cudaError_t launch_stencil7_pipe(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                                 int64_t ny, int64_t nx, int64_t lo, int64_t hi, int64_t c, int S, double c0, double c1,
                                 bool fmad, PipeFlags *flags, cudaStream_t st);

// a device-side delay of about `ns` (the link probe holds two streams behind it so both copies start together)
cudaError_t launch_delay(unsigned long long ns, cudaStream_t st);

// peer halo signalling (pp_halo_*): store `epoch` to *flag after everything before it on the stream
// (system-scope release); spin (with nanosleep) until *flag - epoch >= 0, or give up after ~timeout_ns
// and set *err = 1 (the host then fails the launch)
cudaError_t launch_flag_set(uint32_t *flag, uint32_t epoch, cudaStream_t st);
cudaError_t launch_flag_wait(const uint32_t *flag, uint32_t epoch, unsigned long long timeout_ns, uint32_t *err,
                             cudaStream_t st);
cudaError_t launch_probe(const DView &in, int64_t si, const DView &out, int64_t so, int64_t k0,
                         int64_t k1, cudaStream_t st);

// Driver entry point used to encode TMA descriptors (resolved once via cudaGetDriverEntryPoint).
bool tma_available();

// Programmatic dependent launch of the stencil kernels (tma_common.cuh launch_pdl). The executor
// turns PDL on only while it enqueues a multi-sweep chain, where a chunk's level kernels follow each
// other directly on the kernel stream (T = 32 at 512^3: 32.2 -> 26.2 ms per pass). Long
// back-to-back single sweeps gain nothing (their successor's CTAs would sit resident, waiting).
extern thread_local bool tls_pdl;
struct PdlScope {
    bool prev;
    explicit PdlScope(bool on) : prev(tls_pdl) { tls_pdl = on; }
    ~PdlScope() { tls_pdl = prev; }
};

}  // namespace pp
