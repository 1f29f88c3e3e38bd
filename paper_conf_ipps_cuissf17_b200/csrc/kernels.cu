// kernels.cu — per-chunk loop bodies for sm_100a: 1-D triad, Fig. 2 7-point stencil
// (generic z-march path), int64 index-handler probe. The TMA-staged stencil is in stencil_tma.cu.
//
// Exactness: the default bodies use __fadd_rn/__fmul_rn/__fsub_rn (and the f64 twins), which nvcc
// never contracts into FMA, in Fig. 2's printed order (reading S4), so results are bit-identical to
// the oracle regardless of -fmad. PP_OPT_FMAD selects fma(sum, c1, -(ctr*c0)) instead.
#include <algorithm>
#include <cstdint>

#include "kernels.cuh"
#include "kernels_common.cuh"

namespace pp {

// ------------------------------------------------------------------------------------------------
// Stencil, generic path: any shape/alignment/dtype. Block = 32 x 8 threads over (i, j); each thread
// marches k through a z-segment keeping planes k-1, k, k+1 of its column in registers (2.5-D
// blocking); x/y neighbours come from the centre plane through L1.
// ------------------------------------------------------------------------------------------------
template <typename T, bool FMAD>
__global__ void __launch_bounds__(256) stencil7_generic(DView in, int64_t in_shift, DView out,
                                                        int64_t out_shift, int64_t ny, int64_t nx,
                                                        int64_t k0, int64_t k1, int64_t ilo, int64_t ihi,
                                                        int64_t zseg, T c0, T c1) {
    const int64_t i = (int64_t)blockIdx.x * 32 + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * 8 + threadIdx.y;
    const int64_t kb = k0 + (int64_t)blockIdx.z * zseg;
    const int64_t ke = kb + zseg < k1 ? kb + zseg : k1;
    if (i >= nx || j >= ny || kb >= ke) return;
    const int64_t e = j * nx + i;
    const T *inb = static_cast<const T *>(in.ring);
    T *outb = static_cast<T *>(out.ring);
    const int64_t P = in.plane_elems, Q = out.plane_elems;
    // slot of input plane (kb + in_shift - 1) and of output plane (kb + out_shift)
    int64_t sm = pmod64(kb + in_shift - 1 - in.base, in.R);
    int64_t sc = sm + 1 == in.R ? 0 : sm + 1;
    int64_t so = pmod64(kb + out_shift - out.base, out.R);
    const bool edge = (i == 0 || i == nx - 1 || j == 0 || j == ny - 1);
    T zm = ldg(inb + sm * P + e);
    T ctr = ldg(inb + sc * P + e);
    for (int64_t k = kb; k < ke; ++k) {
        const int64_t sp = sc + 1 == in.R ? 0 : sc + 1;
        const T *pc = inb + sc * P;
        T zp = ldg(inb + sp * P + e);
        T r;
        if (edge || k < ilo || k >= ihi) {                   // edge point, or a boundary-copy plane
            r = ctr;
        } else {
            T yp = ldg(pc + e + nx), ym = ldg(pc + e - nx), xp = ldg(pc + e + 1), xm = ldg(pc + e - 1);
            r = Arith<T, FMAD>::stencil(zp, zm, yp, ym, xp, xm, ctr, c0, c1);
        }
        outb[so * Q + e] = r;
        zm = ctr;
        ctr = zp;
        sc = sp;
        so = so + 1 == out.R ? 0 : so + 1;
    }
}

template <typename T, bool FMAD>
static cudaError_t stencil_generic_launch(const DView &in, int64_t in_shift, const DView &out,
                                          int64_t out_shift, int64_t ny, int64_t nx, int64_t k0,
                                          int64_t k1, int64_t ilo, int64_t ihi, T c0, T c1,
                                          cudaStream_t st) {
    const int64_t nplanes = k1 - k0;
    const int64_t bx = (nx + 31) / 32, by = (ny + 7) / 8;
    // enough CTAs to fill 148 SMs several times; z-segments of >= 8 planes amortise the two
    // extra halo-plane loads of each segment
    const int64_t target = 148 * 16;
    int64_t segs = (target + bx * by - 1) / (bx * by);
    int64_t zseg = (nplanes + segs - 1) / segs;
    if (zseg < 8) zseg = 8;
    if (zseg > nplanes) zseg = nplanes;
    segs = (nplanes + zseg - 1) / zseg;
    if (segs > 65535 || by > 65535) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)bx, (unsigned)by, (unsigned)segs), block(32, 8);
    stencil7_generic<T, FMAD><<<grid, block, 0, st>>>(in, in_shift, out, out_shift, ny, nx, k0, k1,
                                                      ilo, ihi, zseg, c0, c1);
    return cudaGetLastError();
}

cudaError_t launch_stencil7_tma(int dtype, const DView &in, int64_t in_shift, const DView &out,
                                int64_t out_shift, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                                int64_t ilo, int64_t ihi, double c0, double c1, bool fmad, cudaStream_t st);
bool stencil7_tma_supported(int dtype, const DView &in, const DView &out, int64_t ny, int64_t nx);

cudaError_t launch_stencil7(int dtype, const DView &in, int64_t in_shift, const DView &out,
                            int64_t out_shift, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                            int64_t ilo, int64_t ihi, double c0, double c1, bool fmad, int path,
                            int *path_used, cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    const bool tma_ok = stencil7_tma_supported(dtype, in, out, ny, nx);
    if (path == KPATH_TMA && !tma_ok) return cudaErrorNotSupported;
    if (path != KPATH_GENERIC && tma_ok) {
        if (path_used) *path_used = KPATH_TMA;
        return launch_stencil7_tma(dtype, in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, fmad, st);
    }
    if (path_used) *path_used = KPATH_GENERIC;
    switch (dtype) {
    case 0:
        return fmad ? stencil_generic_launch<float, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, (float)c0, (float)c1, st)
                    : stencil_generic_launch<float, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, (float)c0, (float)c1, st);
    case 1:
        return fmad ? stencil_generic_launch<double, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st)
                    : stencil_generic_launch<double, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 2:
        return stencil_generic_launch<uint64_t, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi,
                                                       (uint64_t)(int64_t)c0, (uint64_t)(int64_t)c1, st);
    }
    return cudaErrorInvalidValue;
}

// ------------------------------------------------------------------------------------------------
// 3-D convolution (§V.B, Polybench 3DCONV; reading C1): 15 fixed-coefficient terms
// over planes k-1, k, k+1, summed in Polybench's order with RN intrinsics (bit-exact vs the oracle).
// One thread per (i, j) column, z-march through the chunk's planes; neighbours through L1.
// ------------------------------------------------------------------------------------------------
template <typename T> __device__ __forceinline__ T rn_mul(T a, T b);
template <> __device__ __forceinline__ float rn_mul(float a, float b) { return __fmul_rn(a, b); }
template <> __device__ __forceinline__ double rn_mul(double a, double b) { return __dmul_rn(a, b); }
template <typename T> __device__ __forceinline__ T rn_add(T a, T b);
template <> __device__ __forceinline__ float rn_add(float a, float b) { return __fadd_rn(a, b); }
template <> __device__ __forceinline__ double rn_add(double a, double b) { return __dadd_rn(a, b); }

template <typename T>
__global__ void __launch_bounds__(256) conv3d_generic(DView in, int64_t in_shift, DView out, int64_t out_shift,
                                                      int64_t ny, int64_t nx, int64_t k0, int64_t k1, int64_t zseg) {
    const int64_t i = (int64_t)blockIdx.x * 32 + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * 8 + threadIdx.y;
    const int64_t kb = k0 + (int64_t)blockIdx.z * zseg;
    const int64_t ke = kb + zseg < k1 ? kb + zseg : k1;
    if (i >= nx || j >= ny || kb >= ke) return;
    const T *inb = static_cast<const T *>(in.ring);
    T *outb = static_cast<T *>(out.ring);
    const int64_t P = in.plane_elems, Q = out.plane_elems, e = j * nx + i;
    const bool edge = (i == 0 || i == nx - 1 || j == 0 || j == ny - 1);
    int64_t sm = pmod64(kb + in_shift - 1 - in.base, in.R);
    int64_t so = pmod64(kb + out_shift - out.base, out.R);
    const T c11 = 2, c21 = 5, c31 = -8, c12 = -3, c22 = 6, c32 = -9, c13 = 4, c23 = 7, c33 = 10;
    for (int64_t k = kb; k < ke; ++k) {
        const int64_t sc = sm + 1 == in.R ? 0 : sm + 1, sp = sc + 1 == in.R ? 0 : sc + 1;
        const T *m = inb + sm * P + e, *c = inb + sc * P + e, *p = inb + sp * P + e;
        T r;
        if (edge) {
            r = ldg(c);
        } else {
            // Polybench order: (dk, dj, di) offsets relative to (k, j, i)
            const T mmm = ldg(m - nx - 1), pmm = ldg(p - nx - 1);
            r = rn_mul(c11, mmm);
            r = rn_add(r, rn_mul(c13, pmm));
            r = rn_add(r, rn_mul(c21, mmm));
            r = rn_add(r, rn_mul(c23, pmm));
            r = rn_add(r, rn_mul(c31, mmm));
            r = rn_add(r, rn_mul(c33, pmm));
            r = rn_add(r, rn_mul(c12, ldg(c - nx)));
            r = rn_add(r, rn_mul(c22, ldg(c)));
            r = rn_add(r, rn_mul(c32, ldg(c + nx)));
            r = rn_add(r, rn_mul(c11, ldg(m - nx + 1)));
            r = rn_add(r, rn_mul(c13, ldg(p - nx + 1)));
            r = rn_add(r, rn_mul(c21, ldg(m + 1)));
            r = rn_add(r, rn_mul(c23, ldg(p + 1)));
            r = rn_add(r, rn_mul(c31, ldg(m + nx + 1)));
            r = rn_add(r, rn_mul(c33, ldg(p + nx + 1)));
        }
        outb[so * Q + e] = r;
        sm = sc;
        so = so + 1 == out.R ? 0 : so + 1;
    }
}

cudaError_t launch_conv3d_tma(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                              int64_t ny, int64_t nx, int64_t k0, int64_t k1, cudaStream_t st);
bool stencil7_tma_supported(int dtype, const DView &in, const DView &out, int64_t ny, int64_t nx);

cudaError_t launch_conv3d(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                          int64_t ny, int64_t nx, int64_t k0, int64_t k1, int path, int *path_used,
                          cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    // same staging rules as the stencil; the conv kernel's stores add 32-bit row offsets of up to 4 rows
    const bool tma_ok = stencil7_tma_supported(dtype, in, out, ny, nx) && nx < (1ll << 28);
    if (path == KPATH_TMA && !tma_ok) return cudaErrorNotSupported;
    // auto: the staged path whenever its staging rules hold; measured on B200 (resident 512^3) it
    // beats the generic path for both types (fp64 5294 vs 3313 GB/s, fp32 3982 vs 2211)
    if (path == KPATH_TMA || (path == KPATH_AUTO && tma_ok)) {
        if (path_used) *path_used = KPATH_TMA;
        return launch_conv3d_tma(dtype, in, in_shift, out, out_shift, ny, nx, k0, k1, st);
    }
    if (path_used) *path_used = KPATH_GENERIC;
    const int64_t nplanes = k1 - k0, bx = (nx + 31) / 32, by = (ny + 7) / 8;
    int64_t segs = (148 * 16 + bx * by - 1) / (bx * by);
    int64_t zseg = std::max<int64_t>(8, (nplanes + segs - 1) / segs);
    zseg = std::min(zseg, nplanes);
    segs = (nplanes + zseg - 1) / zseg;
    if (segs > 65535 || by > 65535) return cudaErrorInvalidConfiguration;
    dim3 grid((unsigned)bx, (unsigned)by, (unsigned)segs), block(32, 8);
    if (dtype == 0) conv3d_generic<float><<<grid, block, 0, st>>>(in, in_shift, out, out_shift, ny, nx, k0, k1, zseg);
    else if (dtype == 1) conv3d_generic<double><<<grid, block, 0, st>>>(in, in_shift, out, out_shift, ny, nx, k0, k1, zseg);
    else return cudaErrorInvalidValue;
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// Triad: c = a + s*b elementwise over the chunk's planes. Each array's chunk is one run of
// consecutive slots that may wrap once. Vector path (16-byte LDG/STG) when every array's start slot,
// ring length and base address allow it; otherwise a scalar grid-stride loop.
// ------------------------------------------------------------------------------------------------
template <typename T, bool FMAD>
__global__ void triad_scalar(DView a, int64_t sa0, DView b, int64_t sb0, DView c, int64_t sc0,
                             int64_t n, T s) {
    const T *A = static_cast<const T *>(a.ring);
    const T *B = static_cast<const T *>(b.ring);
    T *C = static_cast<T *>(c.ring);
    const int64_t RA = a.R * a.plane_elems, RB = b.R * b.plane_elems, RC = c.R * c.plane_elems;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n;
         t += (int64_t)gridDim.x * blockDim.x) {
        int64_t ia = sa0 + t; if (ia >= RA) ia -= RA;
        int64_t ib = sb0 + t; if (ib >= RB) ib -= RB;
        int64_t ic = sc0 + t; if (ic >= RC) ic -= RC;
        C[ic] = Arith<T, FMAD>::triad(ldg(A + ia), ldg(B + ib), s);
    }
}

template <typename T, bool FMAD>
__global__ void triad_vec(DView a, int64_t sa0, DView b, int64_t sb0, DView c, int64_t sc0,
                          int64_t nv, T s) {
    using V = typename Vec16<T>::type;
    constexpr int W = Vec16<T>::width;
    const V *A = static_cast<const V *>(a.ring);
    const V *B = static_cast<const V *>(b.ring);
    V *C = static_cast<V *>(c.ring);
    const int64_t RA = a.R * a.plane_elems / W, RB = b.R * b.plane_elems / W, RC = c.R * c.plane_elems / W;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nv;
         t += (int64_t)gridDim.x * blockDim.x) {
        int64_t ia = sa0 + t; if (ia >= RA) ia -= RA;
        int64_t ib = sb0 + t; if (ib >= RB) ib -= RB;
        int64_t ic = sc0 + t; if (ic >= RC) ic -= RC;
        V x = ldg_nc(A + ia), y = ldg_nc(B + ib), z;
        T *xs = reinterpret_cast<T *>(&x), *ys = reinterpret_cast<T *>(&y), *zs = reinterpret_cast<T *>(&z);
#pragma unroll
        for (int q = 0; q < W; ++q) zs[q] = Arith<T, FMAD>::triad(xs[q], ys[q], s);
        stg_na(C + ic, z);
    }
}

template <typename T, bool FMAD>
static cudaError_t triad_launch(const DView &a, int64_t sa, const DView &b, int64_t sb, const DView &c,
                                int64_t sc, int64_t k0, int64_t k1, T s, cudaStream_t st) {
    const int64_t n = (k1 - k0) * c.plane_elems;
    const int64_t sa0 = pmod64(k0 + sa - a.base, a.R) * a.plane_elems;
    const int64_t sb0 = pmod64(k0 + sb - b.base, b.R) * b.plane_elems;
    const int64_t sc0 = pmod64(k0 + sc - c.base, c.R) * c.plane_elems;
    constexpr int W = Vec16<T>::width;
    auto al = [](const DView &v, int64_t s0) {
        return ((uintptr_t)v.ring % 16 == 0) && (s0 % W == 0) && ((v.R * v.plane_elems) % W == 0);
    };
    const int threads = 256;
    if (al(a, sa0) && al(b, sb0) && al(c, sc0) && n % W == 0) {
        int64_t nv = n / W;
        int64_t blocks = (nv + threads - 1) / threads;
        if (blocks > 148 * 32) blocks = 148 * 32;
        triad_vec<T, FMAD><<<(unsigned)blocks, threads, 0, st>>>(a, sa0 / W, b, sb0 / W, c, sc0 / W, nv, s);
    } else {
        int64_t blocks = (n + threads - 1) / threads;
        if (blocks > 148 * 32) blocks = 148 * 32;
        if (blocks < 1) blocks = 1;
        triad_scalar<T, FMAD><<<(unsigned)blocks, threads, 0, st>>>(a, sa0, b, sb0, c, sc0, n, s);
    }
    return cudaGetLastError();
}

// Triad over a 2-D block region (split on a non-outermost dimension): each of the `outer` rows holds a
// run of (k1-k0)*inner elements starting at slot (k0+shift-base) mod R, wrapping at R*inner.
template <typename T, bool FMAD>
__global__ void triad_rows(DView a, int64_t sa0, DView b, int64_t sb0, DView c, int64_t sc0, int64_t nrun,
                           int64_t outer, T s) {
    const T *A = static_cast<const T *>(a.ring);
    const T *B = static_cast<const T *>(b.ring);
    T *C = static_cast<T *>(c.ring);
    const int64_t ia_n = a.plane_elems / a.outer, ib_n = b.plane_elems / b.outer, ic_n = c.plane_elems / c.outer;
    const int64_t WA = a.R * ia_n, WB = b.R * ib_n, WC = c.R * ic_n;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nrun * outer;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t o = t / nrun, r = t - o * nrun;
        int64_t ia = sa0 + r; if (ia >= WA) ia -= WA;
        int64_t ib = sb0 + r; if (ib >= WB) ib -= WB;
        int64_t ic = sc0 + r; if (ic >= WC) ic -= WC;
        C[o * c.ostride + ic] = Arith<T, FMAD>::triad(ldg(A + o * a.ostride + ia), ldg(B + o * b.ostride + ib), s);
    }
}

template <typename T, bool FMAD>
static cudaError_t triad_rows_launch(const DView &a, int64_t sa, const DView &b, int64_t sb, const DView &c,
                                     int64_t sc, int64_t k0, int64_t k1, T s, cudaStream_t st) {
    const int64_t inner = c.plane_elems / c.outer, nrun = (k1 - k0) * inner;
    const int64_t sa0 = pmod64(k0 + sa - a.base, a.R) * (a.plane_elems / a.outer);
    const int64_t sb0 = pmod64(k0 + sb - b.base, b.R) * (b.plane_elems / b.outer);
    const int64_t sc0 = pmod64(k0 + sc - c.base, c.R) * inner;
    int64_t blocks = (nrun * c.outer + 255) / 256;
    blocks = std::max<int64_t>(1, std::min<int64_t>(blocks, 148 * 32));
    triad_rows<T, FMAD><<<(unsigned)blocks, 256, 0, st>>>(a, sa0, b, sb0, c, sc0, nrun, c.outer, s);
    return cudaGetLastError();
}

cudaError_t launch_triad(int dtype, const DView &a, int64_t sa, const DView &b, int64_t sb,
                         const DView &c, int64_t sc, int64_t k0, int64_t k1, double s, bool fmad,
                         cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    if (a.outer > 1 || b.outer > 1 || c.outer > 1) {
        if (dtype == 0)
            return fmad ? triad_rows_launch<float, true>(a, sa, b, sb, c, sc, k0, k1, (float)s, st)
                        : triad_rows_launch<float, false>(a, sa, b, sb, c, sc, k0, k1, (float)s, st);
        if (dtype == 1)
            return fmad ? triad_rows_launch<double, true>(a, sa, b, sb, c, sc, k0, k1, s, st)
                        : triad_rows_launch<double, false>(a, sa, b, sb, c, sc, k0, k1, s, st);
        return cudaErrorInvalidValue;
    }
    if (dtype == 0)
        return fmad ? triad_launch<float, true>(a, sa, b, sb, c, sc, k0, k1, (float)s, st)
                    : triad_launch<float, false>(a, sa, b, sb, c, sc, k0, k1, (float)s, st);
    if (dtype == 1)
        return fmad ? triad_launch<double, true>(a, sa, b, sb, c, sc, k0, k1, s, st)
                    : triad_launch<double, false>(a, sa, b, sb, c, sc, k0, k1, s, st);
    return cudaErrorInvalidValue;
}

// ---------------------------------------------------------------- SM-driven host <-> ring copies
__global__ void __launch_bounds__(256) sm_copy_kernel(int4 *__restrict__ dst, const int4 *__restrict__ src, size_t n16,
                                                      char *__restrict__ dtail, const char *__restrict__ stail, int ntail) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    // four independent 16-byte requests in flight per thread (PCIe latency is microseconds)
    for (; i + 3 * stride < n16; i += 4 * stride) {
        int4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
        dst[i] = a;
        dst[i + stride] = b;
        dst[i + 2 * stride] = c;
        dst[i + 3 * stride] = d;
    }
    for (; i < n16; i += stride) dst[i] = src[i];
    if (blockIdx.x == 0 && (int)threadIdx.x < ntail) dtail[threadIdx.x] = stail[threadIdx.x];
}

cudaError_t launch_sm_copy(void *dst, const void *src, size_t bytes, cudaStream_t st) {
    if (((uintptr_t)dst | (uintptr_t)src) % 16) return cudaErrorInvalidValue;
    const size_t n16 = bytes / 16;
    const int ntail = (int)(bytes % 16);
    // spread over as many SMs as possible: host reads are latency-bound per SM (each SM keeps only so
    // many requests to the host link in flight), so a 1 MiB copy uses 256 blocks of one 16-byte
    // request per thread rather than 64 blocks of four
    const size_t want = (n16 + 256 - 1) / 256;
    const unsigned grid = (unsigned)std::max<size_t>(1, std::min<size_t>(want, 148 * 8));
    sm_copy_kernel<<<grid, 256, 0, st>>>((int4 *)dst, (const int4 *)src, n16, (char *)dst + n16 * 16,
                                         (const char *)src + n16 * 16, ntail);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- device-side schedule check
__global__ void tags_kernel(TagOp t, int phase, int64_t *err) {
    for (int i = 0; i < t.n; ++i) {
        const TagAcc &a = t.a[i];
        if ((phase == 1) != (a.write != 0)) continue;
        for (int64_t p = a.p0 + threadIdx.x; p < a.p1; p += blockDim.x) {
            int64_t slot = (a.s0 + (p - a.p0)) % a.R;
            if (slot < 0) slot += a.R;
            const int64_t want = (p << 8) | (int64_t)a.level;
            if (phase == 1) {
                a.tags[slot] = want;
                continue;
            }
            const int64_t got = a.tags[slot];
            if (got != want) {
                if (atomicAdd((unsigned long long *)&err[0], 1ull) == 0) {
                    err[1] = t.op;
                    err[2] = i;
                    err[3] = p;
                    err[4] = got;
                }
            }
            if (a.visits) atomicAdd(&a.visits[p - a.vbase], 1);
        }
    }
    __threadfence();
}

cudaError_t launch_tags(const TagOp &t, int phase, int64_t *err, cudaStream_t st) {
    tags_kernel<<<1, 256, 0, st>>>(t, phase, err);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- delay (link probe)
__global__ void delay_kernel(unsigned long long ns) {
    unsigned long long t0, t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    do {
        __nanosleep(1000);
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    } while (t - t0 < ns);
}

cudaError_t launch_delay(unsigned long long ns, cudaStream_t st) {
    delay_kernel<<<1, 1, 0, st>>>(ns);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- peer halo flags (pp_halo_*)
__global__ void flag_set_kernel(uint32_t *flag, uint32_t epoch) {
    __threadfence_system();                     // the side-slot copy before us on the stream is complete
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(epoch) : "memory");
}

__global__ void flag_wait_kernel(const uint32_t *flag, uint32_t epoch, unsigned long long timeout_ns, uint32_t *err) {
    unsigned long long t0, t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (;;) {
        uint32_t v;
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
        if ((int32_t)(v - epoch) >= 0) break;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (t - t0 > timeout_ns) {              // never hang the GPU on a peer that does not come:
            *err = 1;                           // give up, and let the host fail the launch
            break;
        }
        __nanosleep(2000);
    }
}

cudaError_t launch_flag_set(uint32_t *flag, uint32_t epoch, cudaStream_t st) {
    flag_set_kernel<<<1, 1, 0, st>>>(flag, epoch);
    return cudaGetLastError();
}

cudaError_t launch_flag_wait(const uint32_t *flag, uint32_t epoch, unsigned long long timeout_ns, uint32_t *err,
                             cudaStream_t st) {
    flag_wait_kernel<<<1, 1, 0, st>>>(flag, epoch, timeout_ns, err);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// Probe (int64, wrap arithmetic): out(k) = in(k-1) + 3 in(k) + 9 in(k+1), elementwise per plane.
// ------------------------------------------------------------------------------------------------
__global__ void probe_kernel(DView in, int64_t si, DView out, int64_t so, int64_t k0, int64_t k1) {
    const uint64_t *I = static_cast<const uint64_t *>(in.ring);
    uint64_t *O = static_cast<uint64_t *>(out.ring);
    const int64_t P = in.plane_elems;
    const int64_t k = k0 + blockIdx.y;
    if (k >= k1) return;
    const int64_t s1 = pmod64(k + si - in.base, in.R);
    const int64_t s0 = s1 == 0 ? in.R - 1 : s1 - 1;
    const int64_t s2 = s1 + 1 == in.R ? 0 : s1 + 1;
    const int64_t d = pmod64(k + so - out.base, out.R);
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < P;
         e += (int64_t)gridDim.x * blockDim.x)
        O[d * P + e] = I[s0 * P + e] + 3u * I[s1 * P + e] + 9u * I[s2 * P + e];
}

cudaError_t launch_probe(const DView &in, int64_t si, const DView &out, int64_t so, int64_t k0,
                         int64_t k1, cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    int64_t bx = (in.plane_elems + 255) / 256;
    if (bx > 1024) bx = 1024;
    // grid.y is limited to 65535 planes per launch; loop over slices
    for (int64_t kb = k0; kb < k1; kb += 65535) {
        int64_t ke = kb + 65535 < k1 ? kb + 65535 : k1;
        probe_kernel<<<dim3((unsigned)bx, (unsigned)(ke - kb)), 256, 0, st>>>(in, si, out, so, kb, ke);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

}  // namespace pp
