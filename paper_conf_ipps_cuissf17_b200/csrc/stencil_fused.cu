// stencil_fused.cu — H Jacobi sweeps of the PAPER.md Fig. 2 body in ONE pass over the
// device ring: temporal blocking on chip for multi-sweep chains (PP_OPT_FUSE; the
// Parboil stencil is iterative).
//
// A single-level launch reads one level ring from HBM and writes the next, so T sweeps cost T ring
// round trips (2e bytes per point each). This kernel reads level t planes once and writes level t+H:
// the H-1 intermediate levels live only in shared memory and registers.
//   * Overlapped tiles: a CTA stages a (W x HH) tile of input planes with an H-point halo in y and
//     HX >= H (16-byte aligned) in x (TMA box, one elected thread, NS-stage mbarrier ring) and
//     computes level j on the staged region shrunk by j per side; the output tile is
//     (W-2HX) x (HH-2H). Halo points are recomputed by the
//     neighbouring CTAs (the price of having no inter-CTA exchange).
//   * z-march: step z receives input plane z, then computes level 1 at plane z-1, level 2 at z-2, ...,
//     level H at z-H (the wavefront). Each thread owns fixed points (lane-strided columns, rows
//     warp + NW*r), so the z-neighbours of its points at every level are values it computed itself:
//     they stay in registers (prev / cur per level). Only the x/y neighbours of the centre plane come
//     from shared memory: the TMA stage for level 0, a double-buffered plane per intermediate level.
//   * Planes outside [ilo, ihi) and the grid's edge points are copies at every level (readings S5, T1),
//     so every level is the exact composition of single sweeps: same RN operation order as the
//     single-level kernels (Arith::stencil), bit-identical to H separate launches.
// One named barrier per z-step separates a level's writes of plane q from the next level's reads.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <type_traits>

#include "kernels.cuh"
#include "kernels_common.cuh"
#include "tma_common.cuh"

namespace pp {

template <typename T, int H_, int U_, int NW_, int RPT_, int NS_, int MINB_> struct FusedCfg {
    static constexpr int H = H_;                     // levels per pass
    static constexpr int V = 16 / (int)sizeof(T);    // points per 16-byte vector
    static constexpr int U = U_;                     // 16-byte vectors per lane and row
    static constexpr int W = 32 * V * U;             // staged columns (TMA box width)
    static constexpr int NW = NW_;                   // warps
    static constexpr int RPT = RPT_;                 // rows per thread
    static constexpr int HH = NW * RPT;              // staged rows
    // x halo rounded up to a 16-byte multiple: a TMA box must start on a 16-byte boundary in global
    // memory (a misaligned start raises an illegal-instruction fault), so tiles are V-aligned
    static constexpr int HX = (H + V - 1) / V * V;
    static constexpr int TX = W - 2 * HX;            // output tile
    static constexpr int TY = HH - 2 * H;
    static constexpr int NS = NS_;                   // TMA stages (input planes)
    static constexpr int MINB = MINB_;               // CTAs per SM the launch bounds ask for
    static constexpr int THREADS = 32 * NW;
    static constexpr int PLANE_BYTES = W * HH * (int)sizeof(T);
    // border rows of the staged region read one row beyond it (garbage that never reaches a valid
    // point): every buffer is separated from the next by a pad row nobody writes, so those reads
    // stay inside shared memory and never touch a live buffer (racecheck-clean)
    static constexpr int PAD = (W * (int)sizeof(T) + 127) / 128 * 128;
    static constexpr int STAGE_STRIDE = (PLANE_BYTES + PAD + 127) / 128 * 128;
    static constexpr int LBUF_STRIDE = (PLANE_BYTES + PAD + 127) / 128 * 128;
    static constexpr int STAGE_OFF = PAD;
    static constexpr int LBUF_OFF = STAGE_OFF + NS * STAGE_STRIDE;
    static constexpr int BAR_OFF = LBUF_OFF + 2 * (H - 1) * LBUF_STRIDE + PAD;
    static constexpr int SMEM = BAR_OFF + NS * 8;
    static_assert(TX > 0 && TY > 0, "tile too small for H levels");
    static_assert(RPT * U * V <= 32, "point masks are 32-bit");
    static_assert(U == 1, "x neighbours come from adjacent lanes of one 32-vector row");
    static_assert((W * (int)sizeof(T)) % 16 == 0, "TMA box row must be a 16-byte multiple");
};

struct FusedParams {
    int64_t in_base, in_R;     // input (level t) ring: slot of plane p = (p - in_base) mod in_R
    int64_t k0, k1;            // output (level t+H) planes [k0, k1)
    int64_t dlo, dhi;          // plane domain: planes outside [dlo, dhi) never exist
    int64_t ilo, ihi;          // planes outside [ilo, ihi) are copies at every level
    int64_t zlen;              // output planes per z-segment
    int tiles, tiles_x, ny, nx;
};

__device__ __forceinline__ void cta_sync() { __syncthreads(); }

template <typename T, bool FMAD, typename C>
__global__ void __launch_bounds__(C::THREADS, C::MINB)
    stencil7_fused_kernel(const __grid_constant__ CUtensorMap tin, const FusedParams p, DView out, T c0, T c1) {
    constexpr int H = C::H, HX = C::HX, U = C::U, W = C::W, RPT = C::RPT, NS = C::NS, HH = C::HH;
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T *stage = reinterpret_cast<T *>(smem_raw + C::STAGE_OFF);
    T *lbuf = reinterpret_cast<T *>(smem_raw + C::LBUF_OFF);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + C::BAR_OFF);
    constexpr int SE = C::STAGE_STRIDE / (int)sizeof(T);    // element strides
    constexpr int LE = C::LBUF_STRIDE / (int)sizeof(T);

    const int tile = (int)(blockIdx.x % p.tiles);
    const int64_t zs = blockIdx.x / p.tiles;
    const int64_t K0 = p.k0 + zs * p.zlen;
    if (K0 >= p.k1) return;                                      // uniform per CTA
    pdl_release_and_wait();                                      // no global access above this line
    const int64_t K1 = min(p.k1, K0 + p.zlen);
    const int64_t a0 = max(K0 - H, p.dlo), b0 = min(K1 + H, p.dhi);   // input planes of this segment
    const int nin = (int)(b0 - a0);
    const int x0 = (tile % p.tiles_x) * C::TX, y0 = (tile / p.tiles_x) * C::TY;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    // TMA: thread 0 keeps NS input planes in flight; the stage of plane s-1 (step index s = z - a0)
    // is refilled right after the barrier that ends step s, when no thread reads it any more
    auto issue = [&](int x) {
        const int st = x % NS;
        const int slot = (int)pmod64(a0 + x - p.in_base, p.in_R);
        mbar_expect_tx(&full[st], C::PLANE_BYTES);
        tma_load_3d(stage + st * SE, &tin, x0 - HX, y0 - H, slot, &full[st]);
    };
    if (threadIdx.x == 0) {
        prefetch_tmap(&tin);
        for (int s = 0; s < NS; ++s) mbar_init(&full[s], 1);
        fence_barrier_init();
        for (int x = 0; x < NS && x < nin; ++x) issue(x);
    }
    cta_sync();

    // This thread's points: a strip of staged rows warp*RPT + r, columns V*lane + v (one 16-byte
    // vector per row, as the single-level kernel). Level j < H values of these points live in
    // registers B[j][slot]: the value computed at step s sits in slot s % 3, so level j at step s
    // reads level j-1 planes q-1, q, q+1 from slots (s+1)%3, (s+2)%3, s%3. The step loop is unrolled
    // by 3, making every slot index a compile-time constant (no register moves). Grid-edge points
    // (copies, reading S5) and output vectors are fixed per CTA: bit masks.
    constexpr int V = C::V;
    using VT = typename Vec16<T>::type;
    uint32_t emask = 0, smask = 0;
#pragma unroll
    for (int r = 0; r < RPT; ++r)
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const int row = warp * RPT + r, col = V * lane + 32 * V * u + v;
                const int yg = y0 - H + row, xg = x0 - HX + col;
                const int bit = (r * U + u) * V + v;
                if (xg <= 0 || xg >= p.nx - 1 || yg <= 0 || yg >= p.ny - 1) emask |= 1u << bit;
                // whole vectors are in or out of the output tile (HX, TX, nx are multiples of V)
                if (v == 0 && row >= H && row < HH - H && col >= HX && col < W - HX && yg < p.ny && xg < p.nx)
                    smask |= 1u << bit;
            }
    // step-index ranges (relative to a0): level j is computed at steps [sj_lo[j], sj_hi[j]); planes
    // outside [ilo, ihi) are copies; steps in [steady_lo, steady_hi) need no range checks at all
    int sj_lo[H + 1], sj_hi[H + 1];
#pragma unroll
    for (int j = 1; j <= H; ++j) {
        sj_lo[j] = (int)(max(K0 - (H - j), p.dlo) + j - a0);
        sj_hi[j] = (int)(min(K1 + (H - j), p.dhi) + j - a0);
    }
    const int cp_lo = (int)(max(p.ilo, p.dlo) - a0), cp_hi = (int)(min(p.ihi, p.dhi) - a0);   // plane index range
    int steady_lo = 0, steady_hi = 1 << 30;
#pragma unroll
    for (int j = 1; j <= H; ++j) {
        steady_lo = max(steady_lo, max(sj_lo[j], cp_lo + j));
        steady_hi = min(steady_hi, min(sj_hi[j], cp_hi + j));
    }
    const int slast = (int)(K1 - 1 + H - a0);

    T B[H][3][RPT][U][V];
    T *outb = static_cast<T *>(out.ring) + (y0 - H + warp * RPT) * (int64_t)p.nx + (x0 - HX + V * lane);
    int64_t so = pmod64(K0 - out.base, out.R);                  // output slot of the next final plane
    const int soff = warp * RPT * W + V * lane;                  // smem offset of point (0, 0, 0)

    auto step = [&](const int s, auto phc, auto steadyc) {
        constexpr int PH = decltype(phc)::value;
        constexpr bool STEADY = decltype(steadyc)::value;
        constexpr int SM = (PH + 1) % 3, SC = (PH + 2) % 3, SP = PH;   // planes q-1, q, q+1
        // ---- level 0: this thread's points of input plane s
        if (STEADY || s < nin) {
            const T *sz = stage + (s % NS) * SE + soff;
            mbar_wait(&full[s % NS], (uint32_t)((s / NS) & 1));
#pragma unroll
            for (int r = 0; r < RPT; ++r)
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const VT x = *reinterpret_cast<const VT *>(sz + r * W + 32 * V * u);
                    memcpy(B[0][PH][r][u], &x, 16);
                }
        }
        // ---- levels 1..H: level j at plane q = s - j (relative to a0)
#pragma unroll
        for (int j = 1; j <= H; ++j) {
            const int q = s - j;
            if (!STEADY && (s < sj_lo[j] || s >= sj_hi[j])) continue;   // uniform per CTA
            const bool cplane = !STEADY && (q < cp_lo || q >= cp_hi);
            // x/y neighbours: level j-1 plane q (TMA stage of plane s-1, or the level buffer of parity q)
            const T *sc = ((j == 1) ? stage + ((s + NS - 1) % NS) * SE : lbuf + (2 * (j - 2) + (q & 1)) * LE) + soff;
            T *d = lbuf + (2 * (j - 1) + (q & 1)) * LE + soff;
            T *og = outb + so * out.plane_elems;
#pragma unroll
            for (int r = 0; r < RPT; ++r)
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    T res[V];
                    const T *c = sc + r * W + 32 * V * u;
                    if (!cplane) {
                        // y neighbours: the thread's own rows (registers) inside its strip, smem at its ends;
                        // x neighbours: the adjacent lanes' vectors (shuffles; lanes 0 / 31 border on the
                        // staged region's edge columns, whose values never reach a valid point)
                        T ym[V], yp[V];
                        if (r > 0) {
#pragma unroll
                            for (int v = 0; v < V; ++v) ym[v] = B[j - 1][SC][r - 1][u][v];
                        } else {
                            const VT t = *reinterpret_cast<const VT *>(c - W);
                            memcpy(ym, &t, 16);
                        }
                        if (r < RPT - 1) {
#pragma unroll
                            for (int v = 0; v < V; ++v) yp[v] = B[j - 1][SC][r + 1][u][v];
                        } else {
                            const VT t = *reinterpret_cast<const VT *>(c + W);
                            memcpy(yp, &t, 16);
                        }
                        const T xm = __shfl_up_sync(0xffffffffu, B[j - 1][SC][r][u][V - 1], 1);
                        const T xp = __shfl_down_sync(0xffffffffu, B[j - 1][SC][r][u][0], 1);
                        T xl[V], xr[V];
#pragma unroll
                        for (int v = 0; v < V; ++v) {
                            xl[v] = v == 0 ? xm : B[j - 1][SC][r][u][v - 1];
                            xr[v] = v == V - 1 ? xp : B[j - 1][SC][r][u][v + 1];
                        }
                        if constexpr (sizeof(T) == 4) {
                            // fp32: the neighbour sum of two adjacent points at once with the lane-wise RN
                            // packed add (FADD2, bit-identical to two scalar adds); the products and the final
                            // subtraction stay scalar so nothing can be contracted (reading S4)
#pragma unroll
                            for (int v = 0; v < V; v += 2) {
                                const T *zp = B[j - 1][SP][r][u], *zm = B[j - 1][SM][r][u];
                                uint64_t acc = add2_rn(pack2(zp[v], zp[v + 1]), pack2(zm[v], zm[v + 1]));
                                acc = add2_rn(acc, pack2(yp[v], yp[v + 1]));
                                acc = add2_rn(acc, pack2(ym[v], ym[v + 1]));
                                acc = add2_rn(acc, pack2(xr[v], xr[v + 1]));
                                acc = add2_rn(acc, pack2(xl[v], xl[v + 1]));
                                T sum[2];
                                unpack2(acc, sum[0], sum[1]);
#pragma unroll
                                for (int w = 0; w < 2; ++w) {
                                    const T ctr = B[j - 1][SC][r][u][v + w];
                                    const T st = FMAD ? __fmaf_rn(sum[w], c1, -__fmul_rn(ctr, c0))
                                                      : __fsub_rn(__fmul_rn(sum[w], c1), __fmul_rn(ctr, c0));
                                    res[v + w] = (emask >> ((r * U + u) * V + v + w)) & 1 ? ctr : st;
                                }
                            }
                        } else {
#pragma unroll
                            for (int v = 0; v < V; ++v) {
                                const T ctr = B[j - 1][SC][r][u][v];
                                const T st = Arith<T, FMAD>::stencil(B[j - 1][SP][r][u][v], B[j - 1][SM][r][u][v], yp[v],
                                                                     ym[v], xr[v], xl[v], ctr, c0, c1);
                                res[v] = (emask >> ((r * U + u) * V + v)) & 1 ? ctr : st;
                            }
                        }
                    } else {
#pragma unroll
                        for (int v = 0; v < V; ++v) res[v] = B[j - 1][SC][r][u][v];
                    }
                    VT o;
                    memcpy(&o, res, 16);
                    if (j < H) {
#pragma unroll
                        for (int v = 0; v < V; ++v) B[j][PH][r][u][v] = res[v];
                        *reinterpret_cast<VT *>(d + r * W + 32 * V * u) = o;   // read by level j+1 next step
                    } else if ((smask >> ((r * U + u) * V)) & 1) {
                        stg_na(reinterpret_cast<VT *>(og + (int64_t)r * p.nx + 32 * V * u), o);
                    }
                }
            if (j == H) so = so + 1 == out.R ? 0 : so + 1;
        }
        cta_sync();
        // input plane s-1 is no longer read: refill its stage with plane s-1+NS
        if (threadIdx.x == 0 && s >= 1 && s - 1 + NS < nin) issue(s - 1 + NS);
    };
    using I0 = std::integral_constant<int, 0>;
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    using F = std::false_type;
    using Tr = std::true_type;
    int s = 0;
    // warm-up and drain steps check ranges; the steady run (all levels active, no copy planes)
    // is straight-line code. Phases stay aligned with s % 3 across the three loops.
    for (; s <= slast && (s < steady_lo || s % 3 != 0); ++s) {
        if (s % 3 == 0) step(s, I0{}, F{});
        else if (s % 3 == 1) step(s, I1{}, F{});
        else step(s, I2{}, F{});
    }
    for (; s + 2 < steady_hi; s += 3) {
        step(s, I0{}, Tr{});
        step(s + 1, I1{}, Tr{});
        step(s + 2, I2{}, Tr{});
    }
    for (; s <= slast; ++s) {
        if (s % 3 == 0) step(s, I0{}, F{});
        else if (s % 3 == 1) step(s, I1{}, F{});
        else step(s, I2{}, F{});
    }
}

// ---------------------------------------------------------------- host side
namespace {
constexpr int kMaxDev = 64;

template <typename T, bool FMAD, typename C> int fused_occupancy() {
    static std::mutex mu;
    static int occ[kMaxDev] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= kMaxDev) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!occ[dev]) {
        auto *kfn = stencil7_fused_kernel<T, FMAD, C>;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        int n = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kfn, C::THREADS, C::SMEM) != cudaSuccess) n = 0;
        cudaGetLastError();
        occ[dev] = n > 0 ? n : -1;
    }
    return occ[dev];
}

template <typename T, bool FMAD, typename C>
cudaError_t fused_launch(const DView &in, const DView &out, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                         int64_t dlo, int64_t dhi, int64_t ilo, int64_t ihi, T c0, T c1, cudaStream_t st) {
    const CUtensorMap *m = tma_map_3d(in, ny, nx, (int)sizeof(T), C::W, C::HH);
    if (!m) return cudaErrorNotSupported;
    const int occ = fused_occupancy<T, FMAD, C>();
    if (occ <= 0) return cudaErrorNotSupported;
    FusedParams p{};
    p.in_base = in.base;
    p.in_R = in.R;
    p.k0 = k0;
    p.k1 = k1;
    p.dlo = dlo;
    p.dhi = dhi;
    p.ilo = ilo;
    p.ihi = ihi;
    p.ny = (int)ny;
    p.nx = (int)nx;
    p.tiles_x = (int)((nx + C::TX - 1) / C::TX);
    p.tiles = p.tiles_x * (int)((ny + C::TY - 1) / C::TY);
    // z-segments: more segments fill the SMs but each re-reads (and recomputes) 2H halo planes. Pick
    // the count that minimises waves x (planes per segment + 2H), segments >= PP_FUSE_MINSEG*H planes.
    const int64_t n = k1 - k0;
    const int64_t slots = (int64_t)sm_count() * occ;
    static const int minseg = env_int("PP_FUSE_MINSEG", 4, 1, 64);
    const int64_t zmax = std::max<int64_t>(1, std::min<int64_t>(n / ((int64_t)minseg * C::H), 4 * slots));
    int64_t zsegs = 1;
    double best = 1e300;
    for (int64_t zz = 1; zz <= zmax; ++zz) {
        const int64_t len = (n + zz - 1) / zz;
        const int64_t waves = ((int64_t)p.tiles * ((n + len - 1) / len) + slots - 1) / slots;
        const double cost = (double)waves * (double)(len + 2 * C::H);
        if (cost < best * 0.999) { best = cost; zsegs = zz; }
    }
    p.zlen = (n + zsegs - 1) / zsegs;
    zsegs = (n + p.zlen - 1) / p.zlen;
    const int64_t grid = (int64_t)p.tiles * zsegs;
    if (grid >= (1ll << 31)) return cudaErrorInvalidConfiguration;
    cudaError_t e = launch_pdl(stencil7_fused_kernel<T, FMAD, C>, (unsigned)grid, C::THREADS, C::SMEM, st, *m, p, out,
                               c0, c1);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

// Variants per H: staged rows of one 16-byte vector per lane (64 f64 / 128 f32 columns). The live
// state is 3H values per point, so the point count per thread, not the smem, bounds occupancy.
// PP_FUSE_VARIANT (tuning build only, `make TUNING=1`) picks an alternative row split: 1 = 10 warps x 2 rows, 2 CTAs/SM;
// 2 = 12 x 3, 1 CTA; 3 = 12 x 2, 2 CTAs; 4 = 20 x 2, 1 CTA; 0 = the measured default below.
template <typename T, bool FMAD, int H>
cudaError_t fused_dispatch(const DView &in, const DView &out, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                           int64_t dlo, int64_t dhi, int64_t ilo, int64_t ihi, T c0, T c1, cudaStream_t st) {
#if PP_TUNING_VARIANTS
    static const int v = env_int("PP_FUSE_VARIANT", 0, 0, 4);
#else
    constexpr int v = 0;
#endif
    switch (v) {
#if PP_TUNING_VARIANTS
    case 1: return fused_launch<T, FMAD, FusedCfg<T, H, 1, 10, 2, 4, 2>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    case 2: return fused_launch<T, FMAD, FusedCfg<T, H, 1, 12, 3, 4, 1>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    case 3: return fused_launch<T, FMAD, FusedCfg<T, H, 1, 12, 2, 4, 2>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    case 4: return fused_launch<T, FMAD, FusedCfg<T, H, 1, 20, 2, 4, 1>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
#endif
    default:
        // measured best on a resident 512^3 sweep (profiles/r1_fused_variants.txt): two CTAs of 12 warps
        // for fp64 pairs of levels (latency-bound: more resident warps), one CTA of 16 warps otherwise
        if constexpr (sizeof(T) == 8 && H == 2)
            return fused_launch<T, FMAD, FusedCfg<T, H, 1, 12, 2, 4, 2>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
        else
            return fused_launch<T, FMAD, FusedCfg<T, H, 1, 16, 2, 4, 1>>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    }
}

template <typename T, bool FMAD>
cudaError_t fused_h(int h, const DView &in, const DView &out, int64_t ny, int64_t nx, int64_t k0, int64_t k1,
                    int64_t dlo, int64_t dhi, int64_t ilo, int64_t ihi, T c0, T c1, cudaStream_t st) {
    switch (h) {
    case 2: return fused_dispatch<T, FMAD, 2>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    case 3: return fused_dispatch<T, FMAD, 3>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    case 4: return fused_dispatch<T, FMAD, 4>(in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
    }
    return cudaErrorNotSupported;
}
}  // namespace

bool stencil7_fused_supported(int dtype, int h, const DView &in, const DView &out, int64_t ny, int64_t nx) {
    if (dtype != 0 && dtype != 1) return false;
    if (h < 2 || h > kMaxFuse) return false;
    const int es = dtype == 0 ? 4 : 8;
    if ((nx * es) % 16 || nx < 3 || ny < 3) return false;         // TMA: 16-byte row pitch
    if (nx >= (1ll << 31) || ny >= (1ll << 31) || in.R >= (1ll << 31)) return false;
    if ((uintptr_t)in.ring % 16 || (uintptr_t)out.ring % 16) return false;
    if (in.plane_elems != nx * ny || out.plane_elems != nx * ny || in.outer != 1 || out.outer != 1) return false;
    return tma_available();
}

cudaError_t launch_stencil7_fused(int dtype, int h, const DView &in, const DView &out, int64_t ny, int64_t nx,
                                  int64_t k0, int64_t k1, int64_t dlo, int64_t dhi, int64_t ilo, int64_t ihi,
                                  double c0, double c1, bool fmad, cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    // the domain's end planes must be copies (they have no outer neighbours)
    if (k0 < dlo || k1 > dhi || ilo < dlo + 1 || ihi > dhi - 1) return cudaErrorInvalidValue;
    if (!stencil7_fused_supported(dtype, h, in, out, ny, nx)) return cudaErrorNotSupported;
    if (dtype == 0)
        return fmad ? fused_h<float, true>(h, in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, (float)c0, (float)c1, st)
                    : fused_h<float, false>(h, in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, (float)c0, (float)c1, st);
    return fmad ? fused_h<double, true>(h, in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st)
                : fused_h<double, false>(h, in, out, ny, nx, k0, k1, dlo, dhi, ilo, ihi, c0, c1, st);
}

}  // namespace pp
