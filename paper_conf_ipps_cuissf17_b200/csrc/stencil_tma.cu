// stencil_tma.cu — TMA-staged 7-point stencil (Fig. 2 body) for sm_100a.
//
// Design: the work of one launch is (x,y) tiles x planes. A persistent grid of exactly
// the resident CTA slots (148 SMs x CTAs/SM) splits the tile-major list of (tile, plane) items into
// equal contiguous ranges, so every CTA streams the same number of plane-tiles; a range is one or
// a few "segments" (one tile, consecutive planes) marched in z (2.5-D blocking). For each segment
// the CTA consumes the input planes z-1 .. z_end (a halo of one plane each side). All those planes
// form ONE continuous sequence per CTA, fetched by the Tensor Memory Accelerator
// (cp.async.bulk.tensor.3d, one elected thread) into an NS-stage shared-memory ring with one mbarrier
// (expect_tx / complete_tx) per stage; the producer runs NS entries ahead and crosses segment
// boundaries, so the pipeline never drains. The TMA box reads the device ring [R][ny][nx] directly at
// (x0-V, y0-1, slot): the index handler's slot map costs one modulo per plane per CTA,
// halo cells outside the grid are zero-filled by the TMA unit and never used (edge points are passed
// through, reading S5). z-neighbours live in registers; x/y neighbours come from the staged centre
// plane (16-byte LDS); results leave as 16-byte streaming stores. Arithmetic is the RN-intrinsic
// sequence of the generic path (bit-exact, reading S4).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "kernels.cuh"
#include "kernels_common.cuh"
#include "tma_common.cuh"

namespace pp {

template <typename T, int WARPS_, int RPW_, int NS_, bool WS_ = false, int CPL_ = 16 / (int)sizeof(T)> struct TmaCfg {
    static constexpr int V = 16 / (int)sizeof(T);   // points per thread per row (one 16-B vector); x halo
    static constexpr int CPL = CPL_;                 // columns per lane (the stencil: V, one vector)
    static constexpr int TX = 32 * CPL;              // tile width: one warp spans a tile row
    static constexpr int W = TX + 2 * V;             // staged row width (16-B multiple, centres aligned)
    static constexpr int WARPS = WARPS_;             // consumer (compute) warps
    static constexpr bool WS = WS_;                  // + one producer warp, per-stage empty barriers
    static constexpr int THREADS = 32 * (WARPS + (WS ? 1 : 0));
    static constexpr int RPW = RPW_;                 // rows per warp
    static constexpr int TY = WARPS * RPW;           // tile height
    static constexpr int H = TY + 2;                 // staged rows (one halo row each side)
    static constexpr int NS = NS_;                   // smem pipeline stages (planes)
    static constexpr int STAGE_ELEMS = W * H;
    static constexpr int STAGE_BYTES = STAGE_ELEMS * (int)sizeof(T);      // bytes the TMA box writes
    static constexpr int STAGE_STRIDE = (STAGE_BYTES + 127) / 128 * 128;  // TMA smem dst: 128-B aligned
    static constexpr int STAGE_STRIDE_ELEMS = STAGE_STRIDE / (int)sizeof(T);
    static constexpr int SMEM = NS * STAGE_STRIDE + 128;
};

template <typename T> __device__ __forceinline__ typename Vec16<T>::type lds16(const T *p) {
    return *reinterpret_cast<const typename Vec16<T>::type *>(p);
}

struct TmaParams {
    int64_t in_base, in_R, in_shift;   // input ring view (slot of plane p = (p - base) mod R)
    int64_t out_shift;                  // output plane of iteration k = k + out_shift
    int64_t k0, nplanes;                // iterations [k0, k0 + nplanes)
    int64_t ilo, ihi;                   // iterations outside [ilo, ihi) copy their centre plane
    int64_t work, per_cta;              // tiles * nplanes items; contiguous items per CTA
    int64_t tiles, zlen;                // lockstep mode: CTA b = tile (b % tiles), z-segment (b / tiles)
    int ny, nx, tiles_x;
    int lockstep;
    int64_t fill_q, fill_r;             // > 0: conv3d slot-filling map (tiles < r get q + 1 z-segments)
};

// Persistent pipeline mode (PP_OPT_PERSISTENT): the flag words (PipeFlags, kernels.cuh) and the sweep.
struct PipeParams {
    int64_t lo, hi, c, nchunks;        // the launch's iterations, chunk size, chunk count
    int64_t zsegs;                      // z-segments per tile per chunk (grid = tiles * zsegs)
    int S;                              // chunks in flight (ring depth)
    PipeFlags *flags;
    unsigned long long timeout_ns;      // a gate that waits longer records an error and goes on
};

// Producer cursor over the CTA's sequence of input planes (leader thread only).
struct ProdCursor {
    int64_t segL;     // linear item index (tile * nplanes + z) where the current segment starts
    int64_t pe;       // entry within the segment, 0 .. m+1
    bool done;
};

// One output plane of this thread's points (rows y0 + warp*RPW + rr, columns xg .. xg+V-1): the Fig. 2
// body from the staged centre plane `sc` and z+1 plane `sp`, with z-1 / centre values carried in
// registers (zm, ctr; rotated on return). Shared by the per-launch and the persistent pipeline kernel.
template <typename T, bool FMAD, typename C>
__device__ __forceinline__ void stencil_plane(const T *sc, const T *sp, T (&zm)[C::RPW][C::V], T (&ctr)[C::RPW][C::V],
                                              T *op, int y0, int xl, int xg, bool xin, int warp, bool cplane, int nx,
                                              int ny, T c0, T c1) {
    using VT = typename Vec16<T>::type;
    constexpr int V = C::V, RPW = C::RPW;
#pragma unroll
    for (int rr = 0; rr < RPW; ++rr) {
        const int row = warp * RPW + rr + 1;
        const int yg = y0 + row - 1;
        const T *cr = sc + row * C::W + xl + V;          // centre row, 16-B aligned
        VT vzp = lds16(sp + row * C::W + xl + V);
        VT vyp = lds16(cr + C::W);
        VT vym = lds16(cr - C::W);
        T xm = cr[-1], xp = cr[V];
        T zp[V], yp[V], ym[V], res[V];
        memcpy(zp, &vzp, 16);
        memcpy(yp, &vyp, 16);
        memcpy(ym, &vym, 16);
        const bool yedge = (yg == 0 || yg == ny - 1) || cplane;
        if constexpr (sizeof(T) == 4 && !FMAD) {
            // fp32: the six neighbour adds of two adjacent points at once (packed RN FADD2,
            // bit-identical to the scalar Fig. 2 order); products and difference scalar
            T sum[V];
#pragma unroll
            for (int v = 0; v < V; v += 2) {
                const T l0 = v == 0 ? xm : ctr[rr][v - 1], l1 = ctr[rr][v];
                const T r0 = ctr[rr][v + 1], r1 = v + 1 == V - 1 ? xp : ctr[rr][v + 2];
                uint64_t acc = add2_rn(pack2(zp[v], zp[v + 1]), pack2(zm[rr][v], zm[rr][v + 1]));
                acc = add2_rn(acc, pack2(yp[v], yp[v + 1]));
                acc = add2_rn(acc, pack2(ym[v], ym[v + 1]));
                acc = add2_rn(acc, pack2(r0, r1));
                acc = add2_rn(acc, pack2(l0, l1));
                unpack2(acc, sum[v], sum[v + 1]);
            }
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const int xi = xg + v;
                const bool edge = yedge || xi == 0 || xi == nx - 1;
                res[v] = edge ? ctr[rr][v] : __fsub_rn(__fmul_rn(sum[v], c1), __fmul_rn(ctr[rr][v], c0));
            }
        } else {
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const T l = v == 0 ? xm : ctr[rr][v - 1];
                const T r = v == V - 1 ? xp : ctr[rr][v + 1];
                const int xi = xg + v;
                const bool edge = yedge || xi == 0 || xi == nx - 1;
                res[v] = edge ? ctr[rr][v]
                              : Arith<T, FMAD>::stencil(zp[v], zm[rr][v], yp[v], ym[v], r, l, ctr[rr][v], c0, c1);
            }
        }
        if (xin && yg < ny) {
            VT o;
            memcpy(&o, res, 16);
            stg_na(reinterpret_cast<VT *>(op + (int64_t)yg * nx + xg), o);
        }
#pragma unroll
        for (int v = 0; v < V; ++v) {
            zm[rr][v] = ctr[rr][v];
            ctr[rr][v] = zp[v];
        }
    }
}

// ---------------------------------------------------------------- the kernel
template <typename T, bool FMAD, int WARPS, int RPW, int NS, bool WS>
__global__ void __launch_bounds__((WARPS + (WS ? 1 : 0)) * 32, WARPS >= 16 || WS ? 2 : 1)
    stencil7_tma_kernel(const __grid_constant__ CUtensorMap tin, const TmaParams p, DView out, T c0, T c1) {
    using C = TmaCfg<T, WARPS, RPW, NS, WS>;
    using VT = typename Vec16<T>::type;
    constexpr int V = C::V;
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T *stage = reinterpret_cast<T *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * C::STAGE_STRIDE);
    uint64_t *empty = full + NS;                                 // WS: consumers release stages here

    // lockstep: CTA b owns z-segment (b / tiles) of tile (b % tiles); all CTAs of one z-segment start
    // together and march at the same rate, so x/y halo cells a CTA stages were just fetched into L2
    // by the neighbouring tile's CTA. balanced: equal contiguous ranges of the tile-major item list.
    int64_t L0, L1;
    if (p.lockstep) {
        const int64_t tile = blockIdx.x % p.tiles, zs = blockIdx.x / p.tiles;
        L0 = tile * p.nplanes + zs * p.zlen;
        L1 = std::min<int64_t>(tile * p.nplanes + p.nplanes, L0 + p.zlen);
        if (zs * p.zlen >= p.nplanes) L1 = L0;
    } else {
        L0 = (int64_t)blockIdx.x * p.per_cta;
        L1 = L0 + p.per_cta < p.work ? L0 + p.per_cta : p.work;
    }
    if (L0 >= L1) return;                                        // uniform per CTA
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool leader = threadIdx.x == 0;
    const int nx = p.nx, ny = p.ny;

    if (leader) {
        prefetch_tmap(&tin);
        for (int s = 0; s < NS; ++s) mbar_init(&full[s], 1);
        if (WS)
            for (int s = 0; s < NS; ++s) mbar_init(&empty[s], WARPS);
        fence_barrier_init();
    }
    __syncthreads();
    pdl_release_and_wait();                                      // no global access above this line

    // ---- producer (leader): issue entries [issued, min(total, released + NS))
    ProdCursor pc{L0, 0, false};
    int64_t issued = 0;
    auto issue_upto = [&](int64_t limit) {
        while (!pc.done && issued < limit) {
            const int64_t tile = pc.segL / p.nplanes, z0 = pc.segL % p.nplanes;
            const int64_t m = std::min<int64_t>(p.nplanes - z0, L1 - pc.segL);
            const int x0 = (int)(tile % p.tiles_x) * C::TX, y0 = (int)(tile / p.tiles_x) * C::TY;
            const int64_t plane = p.k0 + z0 + p.in_shift - 1 + pc.pe;
            const int slot = (int)pmod64(plane - p.in_base, p.in_R);
            const int s = (int)(issued % NS);
            mbar_expect_tx(&full[s], C::STAGE_BYTES);
            tma_load_3d(stage + s * C::STAGE_STRIDE_ELEMS, &tin, x0 - V, y0 - 1, slot, &full[s]);
            ++issued;
            if (++pc.pe == m + 2) {
                pc.segL += m;
                pc.pe = 0;
                pc.done = pc.segL >= L1;
            }
        }
    };
    if (WS) {
        // warp-specialised: the producer warp streams every entry as soon as its stage is released by
        // all consumer warps (empty barrier); consumers never meet at a block-wide barrier
        if (warp == WARPS) {
            if (lane == 0)
                for (int64_t x = 0; !pc.done; ++x) {
                    if (x >= NS) mbar_wait(&empty[x % NS], (uint32_t)(((x / NS) + 1) & 1));
                    fence_proxy_async();
                    issue_upto(x + 1);
                }
            return;
        }
    } else if (leader) {
        issue_upto(NS);
    }
    // release of a consumed entry: WS = one arrive per consumer warp; else the block barrier + leader
    auto release = [&](int64_t upto_excl, int64_t entry) {
        if (WS) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[entry % NS]);
        } else {
            __syncthreads();
            if (leader) {
                fence_proxy_async();
                issue_upto(upto_excl);
            }
        }
    };

    // ---- consumers: this thread's points are rows y0 + warp*RPW + rr, columns x0 + lane*V + v
    const int xl = lane * V;
    T *outb = static_cast<T *>(out.ring);
    int64_t e = 0;                                               // first entry of the current segment
    for (int64_t cL = L0; cL < L1;) {
        const int64_t tile = cL / p.nplanes, z0 = cL % p.nplanes;
        const int64_t m = std::min<int64_t>(p.nplanes - z0, L1 - cL);
        const int x0 = (int)(tile % p.tiles_x) * C::TX, y0 = (int)(tile / p.tiles_x) * C::TY;
        const int xg = x0 + xl;
        const bool xin = xg < nx;                                // whole vector in or out (nx % V == 0)
        T zm[RPW][V], ctr[RPW][V];
        mbar_wait(&full[e % NS], (uint32_t)((e / NS) & 1));
        mbar_wait(&full[(e + 1) % NS], (uint32_t)(((e + 1) / NS) & 1));
        {
            const T *s0 = stage + (e % NS) * C::STAGE_STRIDE_ELEMS;
            const T *s1 = stage + ((e + 1) % NS) * C::STAGE_STRIDE_ELEMS;
#pragma unroll
            for (int rr = 0; rr < RPW; ++rr) {
                const int row = warp * RPW + rr + 1;             // staged row (halo row 0)
                VT a = lds16(s0 + row * C::W + xl + V);
                VT b = lds16(s1 + row * C::W + xl + V);
                memcpy(zm[rr], &a, 16);
                memcpy(ctr[rr], &b, 16);
            }
        }
        release(e + 1 + NS, e);                                  // entry e consumed
        int64_t so = pmod64(p.k0 + z0 + p.out_shift - out.base, out.R);
        for (int64_t q = 0; q < m; ++q) {
            const int64_t ec = e + q + 1, ep = e + q + 2;        // centre / z+1 entries
            mbar_wait(&full[ep % NS], (uint32_t)((ep / NS) & 1));
            const T *sc = stage + (ec % NS) * C::STAGE_STRIDE_ELEMS;
            const T *sp = stage + (ep % NS) * C::STAGE_STRIDE_ELEMS;
            T *op = outb + so * out.plane_elems;
            const int64_t kk = p.k0 + z0 + q;
            const bool cplane = kk < p.ilo || kk >= p.ihi;     // boundary-copy plane of a chain
            stencil_plane<T, FMAD, C>(sc, sp, zm, ctr, op, y0, xl, xg, xin, warp, cplane, nx, ny, c0, c1);
            so = so + 1 == out.R ? 0 : so + 1;
            // entries <= ec consumed; after the segment's last plane its final z+1 entry too
            if (WS) {
                release(0, ec);
                if (q + 1 == m) release(0, ep);
            } else {
                release((q + 1 == m ? ep + 1 : ec + 1) + NS, ec);
            }
        }
        e += m + 2;
        cL += m;
    }
}

// ---------------------------------------------------------------- persistent pipeline kernel
// PP_OPT_PERSISTENT: ONE launch computes every chunk of a pipelined single sweep. The copy streams and
// the kernel hand chunks to each other through flag words in device memory instead of stream events
// and per-chunk launches (no launch latency, no event hop): the H2D stream writes `loaded` = j+1 after
// chunk j's copies (cuStreamWriteValue32), the kernel's producer waits for it before staging chunk j's
// planes, every CTA counts itself done with chunk j in `arrivals` and the last one raises `computed`
// to j+1, on which the D2H stream (cuStreamWaitValue32) and the H2D of chunk j+S (whose planes reuse
// chunk j's ring slots) wait; the D2H stream writes `drained` = j+1, on which the kernel waits before
// writing chunk j+S into the same output slots. Each CTA keeps one (x, y) tile for the whole sweep and
// takes z-segment blockIdx / tiles of every chunk.
template <typename T, bool FMAD, int WARPS, int RPW, int NS>
__global__ void __launch_bounds__((WARPS + 1) * 32, 2)
    stencil7_pipe_kernel(const __grid_constant__ CUtensorMap tin, const TmaParams p, const PipeParams q, DView out,
                         T c0, T c1) {
    using C = TmaCfg<T, WARPS, RPW, NS, true>;
    using VT = typename Vec16<T>::type;
    constexpr int V = C::V;
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T *stage = reinterpret_cast<T *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * C::STAGE_STRIDE);
    uint64_t *empty = full + NS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nx = p.nx, ny = p.ny;
    const int64_t tile = blockIdx.x % p.tiles, zs = blockIdx.x / p.tiles;
    const int x0 = (int)(tile % p.tiles_x) * C::TX, y0 = (int)(tile / p.tiles_x) * C::TY;
    PipeFlags *fl = q.flags;
    if (threadIdx.x == 0) {
        prefetch_tmap(&tin);
        for (int s = 0; s < NS; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], WARPS);
        }
        fence_barrier_init();
    }
    __syncthreads();
    // this CTA's planes of chunk j: [z0, z0 + m) of the chunk's planes [k0, k0 + np)
    auto seg = [&](int64_t j, int64_t *k0, int64_t *z0, int64_t *m) {
        *k0 = q.lo + j * q.c;
        const int64_t np = std::min<int64_t>(q.c, q.hi - *k0);
        const int64_t zlen = (np + q.zsegs - 1) / q.zsegs;
        *z0 = zs * zlen;
        *m = std::min<int64_t>(zlen, np - *z0);
    };
    auto gate = [&](const uint32_t *flag, uint32_t target) {  // wait until *flag >= target (or time out)
        if (*(volatile uint32_t *)&fl->err) return;             // after one timeout nothing waits again
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        for (;;) {
            uint32_t v;
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
            if ((int32_t)(v - target) >= 0) return;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > q.timeout_ns) {                         // never hang: record it and go on
                atomicExch(&fl->err, 1u);
                return;
            }
            __nanosleep(32);
        }
    };
    if (warp == WARPS) {                                         // producer warp
        if (lane == 0) {
            int64_t x = 0;
            for (int64_t j = 0; j < q.nchunks; ++j) {
                int64_t k0, z0, m;
                seg(j, &k0, &z0, &m);
                if (m <= 0) continue;
                gate(&fl->loaded, (uint32_t)(j + 1));            // chunk j's planes are in the ring
                asm volatile("fence.proxy.async.global;" ::: "memory");
                for (int64_t pe = 0; pe < m + 2; ++pe, ++x) {
                    if (x >= NS) mbar_wait(&empty[x % NS], (uint32_t)(((x / NS) + 1) & 1));
                    fence_proxy_async();
                    const int64_t plane = k0 + z0 + p.in_shift - 1 + pe;
                    const int slot = (int)pmod64(plane - p.in_base, p.in_R);
                    const int s = (int)(x % NS);
                    mbar_expect_tx(&full[s], C::STAGE_BYTES);
                    tma_load_3d(stage + s * C::STAGE_STRIDE_ELEMS, &tin, x0 - V, y0 - 1, slot, &full[s]);
                }
            }
        }
        return;
    }
    auto release = [&](int64_t entry) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[entry % NS]);
    };
    const int xl = lane * V, xg = x0 + xl;
    const bool xin = xg < nx;
    T *outb = static_cast<T *>(out.ring);
    int64_t e = 0;
    for (int64_t j = 0; j < q.nchunks; ++j) {
        int64_t k0, z0, m;
        seg(j, &k0, &z0, &m);
        if (m > 0) {
            if (j >= q.S) {                                      // chunk j-S's outputs left these slots
                if (lane == 0) gate(&fl->drained, (uint32_t)(j + 1 - q.S));
                __syncwarp();
            }
            T zm[RPW][V], ctr[RPW][V];
            mbar_wait(&full[e % NS], (uint32_t)((e / NS) & 1));
            mbar_wait(&full[(e + 1) % NS], (uint32_t)(((e + 1) / NS) & 1));
            {
                const T *s0 = stage + (e % NS) * C::STAGE_STRIDE_ELEMS;
                const T *s1 = stage + ((e + 1) % NS) * C::STAGE_STRIDE_ELEMS;
#pragma unroll
                for (int rr = 0; rr < RPW; ++rr) {
                    const int row = warp * RPW + rr + 1;
                    VT a = lds16(s0 + row * C::W + xl + V);
                    VT b = lds16(s1 + row * C::W + xl + V);
                    memcpy(zm[rr], &a, 16);
                    memcpy(ctr[rr], &b, 16);
                }
            }
            release(e);
            int64_t so = pmod64(k0 + z0 + p.out_shift - out.base, out.R);
            for (int64_t qq = 0; qq < m; ++qq) {
                const int64_t ec = e + qq + 1, ep = e + qq + 2;
                mbar_wait(&full[ep % NS], (uint32_t)((ep / NS) & 1));
                const T *sc = stage + (ec % NS) * C::STAGE_STRIDE_ELEMS;
                const T *sp = stage + (ep % NS) * C::STAGE_STRIDE_ELEMS;
                stencil_plane<T, FMAD, C>(sc, sp, zm, ctr, outb + so * out.plane_elems, y0, xl, xg, xin, warp, false,
                                          nx, ny, c0, c1);
                so = so + 1 == out.R ? 0 : so + 1;
                release(ec);
                if (qq + 1 == m) release(ep);
            }
            e += m + 2;
        }
        // this CTA is done with chunk j once every consumer warp's stores are out
        asm volatile("bar.sync 1, %0;" ::"r"(WARPS * 32) : "memory");
        if (threadIdx.x == 0) {
            __threadfence();
            const unsigned long long prev = atomicAdd(&fl->arrivals, 1ull);
            if (prev + 1 == (unsigned long long)gridDim.x * (unsigned long long)(j + 1)) {
                __threadfence();
                atomicMax(&fl->computed, (uint32_t)(j + 1));
            }
        }
    }
}

// ---------------------------------------------------------------- 3-D convolution (TMA, WS)
// Polybench 3DCONV body (reading C1) on the same warp-specialised TMA pipeline. Unlike the
// 7-point stencil it reads x/y neighbours on planes k-1 and k+1 as well, so three consecutive staged
// planes are live per output plane: entry z-1 is released one iteration later than the stencil's.
// Operand traffic, not HBM, bounds this body (ncu: shared-memory pipe at 96% with the 16-byte-vector
// mapping, half of it bank conflicts from the x+-1 scalars), so the thread mapping differs from the
// stencil's: lane l owns columns x0 + l + 32v (v < V), which makes every shared load — centre, x-1 or
// x+1 — one contiguous, conflict-free warp access, and each warp walks its RPW rows keeping a sliding
// window of the rows it already loaded (5 new loads per row and column instead of 15).
template <typename T, int WARPS, int RPW, int NS, int MINB, int CPL, bool LR>
__global__ void __launch_bounds__((WARPS + (LR ? 0 : 1)) * 32, MINB)
    conv3d_tma_kernel(const __grid_constant__ CUtensorMap tin, const TmaParams p, DView out) {
    using C = TmaCfg<T, WARPS, RPW, NS, !LR, CPL>;
    static_assert(2 * NS * sizeof(uint64_t) + NS * sizeof(uint32_t) <= 128, "barriers + counters fit the tail");
    constexpr int V = C::V;
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T *stage = reinterpret_cast<T *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * C::STAGE_STRIDE);
    uint64_t *empty = full + NS;
    // lockstep z-segments (as the stencil): CTA b owns z-segment b / tiles of tile b % tiles; or the
    // slot-filling map: one CTA per resident slot, tiles [0, r) cut into q + 1 z-segments, the others
    // into q, so every SM holds the same number of CTAs
    int64_t tile0, L0, L1;
    if (p.fill_q > 0) {
        const int64_t b = blockIdx.x, big = p.fill_r * (p.fill_q + 1);
        const int64_t n = b < big ? p.fill_q + 1 : p.fill_q;
        tile0 = b < big ? b / n : p.fill_r + (b - big) / n;
        const int64_t zs = b < big ? b % n : (b - big) % n;
        L0 = tile0 * p.nplanes + zs * p.nplanes / n;
        L1 = tile0 * p.nplanes + (zs + 1) * p.nplanes / n;
    } else {
        tile0 = blockIdx.x % p.tiles;
        const int64_t zs = blockIdx.x / p.tiles;
        L0 = tile0 * p.nplanes + zs * p.zlen;
        L1 = std::min<int64_t>(tile0 * p.nplanes + p.nplanes, L0 + p.zlen);
        if (zs * p.zlen >= p.nplanes) return;
    }
    if (L0 >= L1) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nx = p.nx, ny = p.ny;
    // Refill protocol. LR (fp32): no producer loop — thread 0 fills the NS stages, then the LAST
    // consumer warp to release an entry (a shared-memory counter per stage) issues the load of the entry
    // NS further on into that stage, so a refill starts the moment its stage is free. !LR (fp64): one
    // producer warp waits on per-stage empty barriers (measured: fp32 222 -> 212 us with LR, fp64
    // 370 -> 373 us, profiles/r2_conv3d.md). A CTA owns one segment (lockstep), so entry x is plane
    // k0 + z0 - 1 + x of its tile, x < m + 2.
    uint32_t *relcnt = reinterpret_cast<uint32_t *>(empty + NS);
    const int64_t segz0 = L0 % p.nplanes, segm = L1 - L0;
    const int tx0 = (int)(tile0 % p.tiles_x) * C::TX, ty0 = (int)(tile0 / p.tiles_x) * C::TY;
    auto issue = [&](int64_t x) {
        const int s = (int)(x % NS);
        const int slot = (int)pmod64(p.k0 + segz0 + p.in_shift - 1 + x - p.in_base, p.in_R);
        mbar_expect_tx(&full[s], C::STAGE_BYTES);
        tma_load_3d(stage + s * C::STAGE_STRIDE_ELEMS, &tin, tx0 - V, ty0 - 1, slot, &full[s]);
    };
    if (threadIdx.x == 0) {
        prefetch_tmap(&tin);
        for (int s = 0; s < NS; ++s) {
            mbar_init(&full[s], 1);
            if (LR) relcnt[s] = 0;
            else mbar_init(&empty[s], WARPS);
        }
        fence_barrier_init();
        if (LR)
            for (int64_t x = 0; x < NS && x < segm + 2; ++x) issue(x);
    }
    __syncthreads();
    if (!LR && warp == WARPS) {                                  // producer warp
        if (lane == 0)
            for (int64_t x = 0; x < segm + 2; ++x) {
                if (x >= NS) mbar_wait(&empty[x % NS], (uint32_t)(((x / NS) + 1) & 1));
                fence_proxy_async();
                issue(x);
            }
        return;
    }
    auto release = [&](int64_t entry) {
        __syncwarp();
        if (lane != 0) return;
        if (!LR) {
            mbar_arrive(&empty[entry % NS]);
            return;
        }
        // one acquire-release shared atomic: releases this warp's reads of the stage (ordered before lane
        // 0 by __syncwarp) and, for the last arrival, acquires every other warp's (same time as two
        // __threadfence_block around a relaxed atomicAdd, r2s2r)
        const int s = (int)(entry % NS);
        uint32_t old;
        asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], 1;" : "=r"(old) : "r"(smem_u32(&relcnt[s])) : "memory");
        if (old == (uint32_t)(WARPS - 1)) {
            relcnt[s] = 0;
            if (entry + NS < segm + 2) {
                fence_proxy_async();
                issue(entry + NS);
            }
        }
    };
    const T c11 = 2, c21 = 5, c31 = -8, c12 = -3, c22 = 6, c32 = -9, c13 = 4, c23 = 7, c33 = 10;
    T *outb = static_cast<T *>(out.ring);
    const int r0 = warp * RPW;                                   // staged row of this warp's first y-1
    int64_t e = 0;
    for (int64_t cL = L0; cL < L1;) {
        const int64_t tile = cL / p.nplanes, z0 = cL % p.nplanes;
        const int64_t m = std::min<int64_t>(p.nplanes - z0, L1 - cL);
        const int x0 = (int)(tile % p.tiles_x) * C::TX, y0 = (int)(tile / p.tiles_x) * C::TY;
        mbar_wait(&full[e % NS], (uint32_t)((e / NS) & 1));
        mbar_wait(&full[(e + 1) % NS], (uint32_t)(((e + 1) / NS) & 1));
        int64_t so = pmod64(p.k0 + z0 + p.out_shift - out.base, out.R);
        for (int64_t q = 0; q < m; ++q) {
            const int64_t em = e + q, ec = e + q + 1, ep = e + q + 2;
            mbar_wait(&full[ep % NS], (uint32_t)((ep / NS) & 1));
            // column (V + lane) of staged row 0 of planes z-1, z, z+1
            const T *sm = stage + (em % NS) * C::STAGE_STRIDE_ELEMS + V + lane;
            const T *sc = stage + (ec % NS) * C::STAGE_STRIDE_ELEMS + V + lane;
            const T *sp = stage + (ep % NS) * C::STAGE_STRIDE_ELEMS + V + lane;
            // this thread's first output point of the plane: row y0 + r0, column x0 + lane
            T *orow = outb + so * out.plane_elems + ((int64_t)(y0 + r0) * nx + x0 + lane);
            // tile-uniform: no point of an interior tile lies on the grid's edge ring or outside it
            const bool interior = x0 > 0 && x0 + C::TX < nx && y0 > 0 && y0 + C::TY < ny - 1;
            // NP columns per step: fp32 pairs two columns (v, v + 1) so the 14 dependent adds run as packed
            // add.rn.f32x2 (FADD2, lane-wise round-to-nearest: bit-identical to two scalar adds); products
            // stay scalar (ptxas fuses a packed mul into a following packed add as FFMA2, which would not be)
            constexpr int NP = sizeof(T) == 4 ? 2 : 1;
            static_assert(RPW % 2 == 0, "rows are processed in pairs");
#pragma unroll
            for (int v0 = 0; v0 < CPL; v0 += NP) {
                // Sliding windows over the staged rows of this column group: x+1 operands of planes z-1
                // (mx) and z+1 (px) and centre operands of plane z (cc) for rows R-1, R of the next pair.
                T mx0[NP], mx1[NP], px0[NP], px1[NP], cc0[NP], cc1[NP];
#pragma unroll
                for (int u = 0; u < NP; ++u) {
                    const int xo = 32 * (v0 + u);
                    mx0[u] = sm[r0 * C::W + xo + 1];
                    mx1[u] = sm[(r0 + 1) * C::W + xo + 1];
                    px0[u] = sp[r0 * C::W + xo + 1];
                    px1[u] = sp[(r0 + 1) * C::W + xo + 1];
                    cc0[u] = sc[r0 * C::W + xo];
                    cc1[u] = sc[(r0 + 1) * C::W + xo];
                }
#pragma unroll
                for (int rr = 0; rr < RPW; rr += 2) {
                    // two output rows at once (A = staged row R, B = R + 1): their 15-term chains are
                    // independent, so their dependent adds interleave instead of waiting on each other
                    const int R = r0 + rr + 1;
                    T mx2[NP], mx3[NP], px2[NP], px3[NP], cc2[NP], cc3[NP], mmA[NP], pmA[NP], mmB[NP], pmB[NP];
#pragma unroll
                    for (int u = 0; u < NP; ++u) {
                        const int xo = 32 * (v0 + u);
                        mx2[u] = sm[(R + 1) * C::W + xo + 1];
                        mx3[u] = sm[(R + 2) * C::W + xo + 1];
                        px2[u] = sp[(R + 1) * C::W + xo + 1];
                        px3[u] = sp[(R + 2) * C::W + xo + 1];
                        cc2[u] = sc[(R + 1) * C::W + xo];
                        cc3[u] = sc[(R + 2) * C::W + xo];
                        mmA[u] = sm[(R - 1) * C::W + xo - 1];
                        pmA[u] = sp[(R - 1) * C::W + xo - 1];
                        mmB[u] = sm[R * C::W + xo - 1];
                        pmB[u] = sp[R * C::W + xo - 1];
                    }
                    // the 15 operands of a row in Polybench's order (reading C1): row A uses window rows
                    // (R-1, R, R+1) = (0, 1, 2), row B (R, R+1, R+2) = (1, 2, 3)
                    auto opnd = [&](int i, int u, bool b) -> T {
                        switch (i) {
                        case 0: case 2: case 4: return b ? mmB[u] : mmA[u];
                        case 1: case 3: case 5: return b ? pmB[u] : pmA[u];
                        case 6: return b ? cc1[u] : cc0[u];
                        case 7: return b ? cc2[u] : cc1[u];
                        case 8: return b ? cc3[u] : cc2[u];
                        case 9: return b ? mx1[u] : mx0[u];
                        case 10: return b ? px1[u] : px0[u];
                        case 11: return b ? mx2[u] : mx1[u];
                        case 12: return b ? px2[u] : px1[u];
                        case 13: return b ? mx3[u] : mx2[u];
                        default: return b ? px3[u] : px2[u];
                        }
                    };
                    // Polybench's coefficients per term: c11 c13 c21 c23 c31 c33 c12 c22 c32 c11 c13 c21 c23 c31 c33
                    auto coef = [](int i) -> T {
                        constexpr int c[15] = {2, 4, 5, 7, -8, 10, -3, 6, -9, 2, 4, 5, 7, -8, 10};
                        return T(c[i]);
                    };
                    // Terms whose coefficient is a power of two (2, 4, -8: terms 1, 4, 9, 10, 13 after the
                    // first) have EXACT products, so RN(acc + RN(c*a)) = RN(acc + c*a): one fused
                    // multiply-add gives the unfused result bit for bit (the summation order is unchanged;
                    // only an overflowing product, |c*a| beyond the largest finite value, would differ —
                    // DESIGN.md §6). The other nine stay product-then-add.
                    auto exact_product = [](int i) { return i == 1 || i == 4 || i == 9 || i == 10 || i == 13; };
                    T resA[NP], resB[NP];
                    if constexpr (NP == 2) {
                        uint64_t a = pack2(__fmul_rn(coef(0), opnd(0, 0, false)), __fmul_rn(coef(0), opnd(0, 1, false)));
                        uint64_t b = pack2(__fmul_rn(coef(0), opnd(0, 0, true)), __fmul_rn(coef(0), opnd(0, 1, true)));
#pragma unroll
                        for (int i = 1; i < 15; ++i) {
                            const uint64_t cc = pack2(coef(i), coef(i));
                            if (exact_product(i)) {
                                a = fma2_rn(cc, pack2(opnd(i, 0, false), opnd(i, 1, false)), a);
                                b = fma2_rn(cc, pack2(opnd(i, 0, true), opnd(i, 1, true)), b);
                            } else {
                                a = add2_rn(a, pack2(__fmul_rn(coef(i), opnd(i, 0, false)), __fmul_rn(coef(i), opnd(i, 1, false))));
                                b = add2_rn(b, pack2(__fmul_rn(coef(i), opnd(i, 0, true)), __fmul_rn(coef(i), opnd(i, 1, true))));
                            }
                        }
                        unpack2(a, resA[0], resA[1]);
                        unpack2(b, resB[0], resB[1]);
                    } else {
                        T a = Arith<T, false>::mul(coef(0), opnd(0, 0, false));
                        T b = Arith<T, false>::mul(coef(0), opnd(0, 0, true));
#pragma unroll
                        for (int i = 1; i < 15; ++i) {
                            if (exact_product(i)) {
                                a = fma(coef(i), opnd(i, 0, false), a);
                                b = fma(coef(i), opnd(i, 0, true), b);
                            } else {
                                a = Arith<T, false>::add(a, Arith<T, false>::mul(coef(i), opnd(i, 0, false)));
                                b = Arith<T, false>::add(b, Arith<T, false>::mul(coef(i), opnd(i, 0, true)));
                            }
                        }
                        resA[0] = a;
                        resB[0] = b;
                    }
                    // one tile-uniform branch per row pair; addresses are the plane's row pointer plus
                    // 32-bit offsets (rows rr, rr + 1 of this warp, columns 32 (v0 + u) of this lane)
                    if (interior) {
#pragma unroll
                        for (int h = 0; h < 2; ++h)
#pragma unroll
                            for (int u = 0; u < NP; ++u)
                                __stcs(orow + ((rr + h) * nx + 32 * (v0 + u)), h ? resB[u] : resA[u]);
                    } else {
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            const int yg = y0 + R - 1 + h;
#pragma unroll
                            for (int u = 0; u < NP; ++u) {
                                const int xi = x0 + lane + 32 * (v0 + u);
                                const bool edge = xi == 0 || xi == nx - 1 || yg == 0 || yg == ny - 1;
                                if (xi < nx && yg < ny)
                                    __stcs(orow + ((rr + h) * nx + 32 * (v0 + u)),
                                           edge ? (h ? cc2[u] : cc1[u]) : (h ? resB[u] : resA[u]));
                            }
                        }
                    }
#pragma unroll
                    for (int u = 0; u < NP; ++u) {
                        mx0[u] = mx2[u]; mx1[u] = mx3[u];
                        px0[u] = px2[u]; px1[u] = px3[u];
                        cc0[u] = cc2[u]; cc1[u] = cc3[u];
                    }
                }
            }
            so = so + 1 == out.R ? 0 : so + 1;
            release(em);                                         // plane z-1 of this output is done
        }
        release(e + m);                                          // the segment's last two entries
        release(e + m + 1);
        e += m + 2;
        cL += m;
    }
}

// ---------------------------------------------------------------- host side
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
        cudaGetLastError();
    });
    return fn;
}

bool tma_available() { return encode_fn() != nullptr; }

bool stencil7_tma_supported(int dtype, const DView &in, const DView &out, int64_t ny, int64_t nx) {
    if (dtype != 0 && dtype != 1) return false;
    const int V = dtype == 0 ? 4 : 2;
    if (nx % V || nx < 3 || ny < 3) return false;                // 16-B row pitch (TMA stride rule)
    if (nx >= (1ll << 31) || ny >= (1ll << 31) || in.R >= (1ll << 31)) return false;
    if ((uintptr_t)in.ring % 16 || (uintptr_t)out.ring % 16) return false;
    if (in.plane_elems != nx * ny || out.plane_elems != nx * ny) return false;
    return tma_available();
}

namespace {
struct MapKey {
    const void *ptr;
    int64_t R, ny, nx;
    int esize, boxw, boxh;
    bool operator==(const MapKey &o) const {
        return ptr == o.ptr && R == o.R && ny == o.ny && nx == o.nx && esize == o.esize && boxw == o.boxw &&
               boxh == o.boxh;
    }
};
struct MapCache {
    static constexpr int N = 16;
    MapKey key[N];
    CUtensorMap map[N];
    int used = 0, next = 0;
};
thread_local MapCache g_maps;

bool encode(CUtensorMap *m, const DView &in, int64_t ny, int64_t nx, int esize, int boxw, int boxh) {
    const cuuint64_t dims[3] = {(cuuint64_t)nx, (cuuint64_t)ny, (cuuint64_t)in.R};
    const cuuint64_t strides[2] = {(cuuint64_t)(nx * esize), (cuuint64_t)(nx * ny * esize)};
    const cuuint32_t box[3] = {(cuuint32_t)boxw, (cuuint32_t)boxh, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = encode_fn()(m, esize == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                             3, in.ring, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}
}  // namespace

const CUtensorMap *tma_map_3d(const DView &in, int64_t ny, int64_t nx, int esize, int boxw, int boxh) {
    MapCache &c = g_maps;
    MapKey k{in.ring, in.R, ny, nx, esize, boxw, boxh};
    for (int i = 0; i < c.used; ++i)
        if (c.key[i] == k) return &c.map[i];
    int slot = c.used < MapCache::N ? c.used++ : (c.next++ % MapCache::N);
    if (!encode(&c.map[slot], in, ny, nx, esize, boxw, boxh)) {
        c.key[slot] = MapKey{nullptr, 0, 0, 0, 0, 0, 0};
        return nullptr;
    }
    c.key[slot] = k;
    return &c.map[slot];
}

namespace {
template <typename C, typename T> const CUtensorMap *get_map(const DView &in, int64_t ny, int64_t nx) {
    return tma_map_3d(in, ny, nx, (int)sizeof(T), C::W, C::H);
}

}  // namespace

constexpr int kMaxDevices = 64;

int sm_count() {
    static std::mutex mu;
    static int n[kMaxDevices] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= kMaxDevices) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!n[dev] && (cudaDeviceGetAttribute(&n[dev], cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n[dev] <= 0))
        n[dev] = 148;
    return n[dev];
}

thread_local bool tls_pdl = false;

bool pdl_enabled() {
    static const bool on = env_int("PP_PDL", 1, 0, 1) != 0;
    return on;
}

int env_int(const char *name, int dflt, int lo, int hi) {
    const char *s = getenv(name);
    int v = s ? atoi(s) : dflt;
    return v < lo || v > hi ? dflt : v;
}

namespace {
// Per-device setup of one kernel variant: the dynamic shared-memory opt-in (> 48 KB) is a per-device
// function attribute, so it is applied on every device the process launches on; the occupancy and SM
// count are per device too.

template <typename T, bool FMAD, int WARPS, int RPW, int NS, bool WS> int occupancy() {
    static std::mutex mu;
    static int occ[kMaxDevices] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= kMaxDevices) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!occ[dev]) {
        using C = TmaCfg<T, WARPS, RPW, NS, WS>;
        auto *kfn = stencil7_tma_kernel<T, FMAD, WARPS, RPW, NS, WS>;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        int n = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kfn, C::THREADS, C::SMEM) != cudaSuccess) n = 1;
        cudaGetLastError();
        occ[dev] = n > 0 ? n : 1;
    }
    return occ[dev];
}

template <typename T, bool FMAD, int WARPS, int RPW, int NS, bool WS = false>
cudaError_t launch_v(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny,
                     int64_t nx, int64_t k0, int64_t k1, int64_t ilo, int64_t ihi, T c0, T c1, cudaStream_t st) {
    using C = TmaCfg<T, WARPS, RPW, NS, WS>;
    const CUtensorMap *m = get_map<C, T>(in, ny, nx);
    if (!m) return cudaErrorNotSupported;
    TmaParams p{};
    p.in_base = in.base;
    p.in_R = in.R;
    p.in_shift = in_shift;
    p.out_shift = out_shift;
    p.k0 = k0;
    p.nplanes = k1 - k0;
    p.ilo = ilo;
    p.ihi = ihi;
    p.ny = (int)ny;
    p.nx = (int)nx;
    p.tiles_x = (int)((nx + C::TX - 1) / C::TX);
    p.tiles = (int64_t)p.tiles_x * ((ny + C::TY - 1) / C::TY);
    p.work = p.tiles * p.nplanes;
    const int64_t slots = (int64_t)sm_count() * occupancy<T, FMAD, WARPS, RPW, NS, WS>();
    static const int sched = env_int("PP_TMA_SCHED", 0, 0, 1);
    int64_t grid;
    if (sched == 0) {
        // lockstep z-segments: as many segments per tile as fit in one wave of resident CTAs
        p.lockstep = 1;
        int64_t zsegs = std::max<int64_t>(1, slots / p.tiles);
        // planes per segment >= PP_TMA_MINSEG (default 2): fewer halo re-reads vs more CTAs in flight
        // (2 measured best for small per-chunk launches: c = 6 chunk 12.3 -> 10.3 us; resident launches
        // are limited by the slot count, not by this)
        static const int minseg = env_int("PP_TMA_MINSEG", 2, 1, 64);
        zsegs = std::min<int64_t>(zsegs, std::max<int64_t>(1, p.nplanes / minseg));
        p.zlen = (p.nplanes + zsegs - 1) / zsegs;
        zsegs = (p.nplanes + p.zlen - 1) / p.zlen;
        grid = p.tiles * zsegs;
    } else {
        // balanced persistent grid: one CTA per resident slot, >= ~4 plane-tiles per CTA
        p.lockstep = 0;
        grid = std::min<int64_t>(slots, std::max<int64_t>(1, p.work / 4));
        p.per_cta = (p.work + grid - 1) / grid;
        grid = (p.work + p.per_cta - 1) / p.per_cta;
    }
    if (grid >= (1ll << 31)) return cudaErrorInvalidConfiguration;
    cudaError_t e = launch_pdl(stencil7_tma_kernel<T, FMAD, WARPS, RPW, NS, WS>, (unsigned)grid, C::THREADS, C::SMEM,
                               st, *m, p, out, c0, c1);
    return e != cudaSuccess ? e : cudaGetLastError();
}

// Tile/stage variant (PP_TMA_VARIANT overrides the default in a tuning build, `make TUNING=1`; the
// default build compiles variant 7 only). Default 7, measured best on
// B200 on a resident 512^3 sweep: 6226 GB/s fp64 / 5950 GB/s fp32 vs 5886 / 4905 for variant 2 on the
// same box (profiles/r1_tma_variants.txt):
//   0: 8 warps x 2 rows (TY 16), 4 stages    1: 8 warps x 4 rows (TY 32), 4 stages
//   2: 16 warps x 2 rows (TY 32), 4 stages   3: 16 warps x 2 rows (TY 32), 6 stages
//   4: 8 warps x 2 rows (TY 16), 6 stages
//   5-7: warp-specialised (one producer warp, per-stage empty mbarriers, no block barrier per plane):
//   5: 16 x 2 rows, 4 stages   6: 16 x 2 rows, 5 stages   7: 8 x 4 rows, 4 stages
template <typename T, bool FMAD>
cudaError_t launch_t(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny,
                     int64_t nx, int64_t k0, int64_t k1, int64_t ilo, int64_t ihi, T c0, T c1, cudaStream_t st) {
#if PP_TUNING_VARIANTS
    static const int v = env_int("PP_TMA_VARIANT", 7, 0, 7);
    switch (v) {
    case 5: return launch_v<T, FMAD, 16, 2, 4, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 6: return launch_v<T, FMAD, 16, 2, 5, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 1: return launch_v<T, FMAD, 8, 4, 4>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 2: return launch_v<T, FMAD, 16, 2, 4>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 3: return launch_v<T, FMAD, 16, 2, 6>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 4: return launch_v<T, FMAD, 8, 2, 6>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    case 0: return launch_v<T, FMAD, 8, 2, 4>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    default: break;
    }
#endif
    // (3 CTAs/SM: 432 us fp64, 3 stages x 3 CTAs: 366 us, 5 stages: 380-388 us — all slower than this
    // 340 us; profiles/r2_kernel_ab.md)
    return launch_v<T, FMAD, 8, 4, 4, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
}
}  // namespace

cudaError_t launch_stencil7_tma(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                                int64_t ny, int64_t nx, int64_t k0, int64_t k1, int64_t ilo, int64_t ihi, double c0,
                                double c1, bool fmad, cudaStream_t st) {
    if (dtype == 0)
        return fmad ? launch_t<float, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, (float)c0, (float)c1, st)
                    : launch_t<float, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, (float)c0, (float)c1, st);
    if (dtype == 1)
        return fmad ? launch_t<double, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st)
                    : launch_t<double, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, ilo, ihi, c0, c1, st);
    return cudaErrorNotSupported;
}

namespace {
template <typename T, bool FMAD, int WARPS, int RPW, int NS>
cudaError_t pipe_launch(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny, int64_t nx,
                        int64_t lo, int64_t hi, int64_t c, int S, T c0, T c1, PipeFlags *flags, cudaStream_t st) {
    using C = TmaCfg<T, WARPS, RPW, NS, true>;
    const CUtensorMap *m = get_map<C, T>(in, ny, nx);
    if (!m) return cudaErrorNotSupported;
    auto *kfn = stencil7_pipe_kernel<T, FMAD, WARPS, RPW, NS>;
    static std::mutex mu;
    static int occ[kMaxDevices] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= kMaxDevices) dev = 0;
    {
        std::lock_guard<std::mutex> lk(mu);
        if (!occ[dev]) {
            cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
            int n = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kfn, C::THREADS, C::SMEM) != cudaSuccess) n = 1;
            cudaGetLastError();
            occ[dev] = n > 0 ? n : 1;
        }
    }
    TmaParams p{};
    p.in_base = in.base;
    p.in_R = in.R;
    p.in_shift = in_shift;
    p.out_shift = out_shift;
    p.ny = (int)ny;
    p.nx = (int)nx;
    p.tiles_x = (int)((nx + C::TX - 1) / C::TX);
    p.tiles = (int64_t)p.tiles_x * ((ny + C::TY - 1) / C::TY);
    PipeParams q{};
    q.lo = lo;
    q.hi = hi;
    q.c = c;
    q.nchunks = (hi - lo + c - 1) / c;
    q.S = S;
    q.flags = flags;
    q.timeout_ns = 5000000000ull;
    const int64_t slots = (int64_t)sm_count() * occ[dev];
    // every CTA must be resident at once (they wait on each other's chunks through the flags)
    if (p.tiles > slots) return cudaErrorNotSupported;
    q.zsegs = std::max<int64_t>(1, std::min<int64_t>(slots / p.tiles, std::max<int64_t>(1, c / 2)));
    const int64_t grid = p.tiles * q.zsegs;
    kfn<<<(unsigned)grid, C::THREADS, C::SMEM, st>>>(*m, p, q, out, c0, c1);
    return cudaGetLastError();
}
}  // namespace

cudaError_t launch_stencil7_pipe(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                                 int64_t ny, int64_t nx, int64_t lo, int64_t hi, int64_t c, int S, double c0, double c1,
                                 bool fmad, PipeFlags *flags, cudaStream_t st) {
    if (hi <= lo || c < 1) return cudaErrorInvalidValue;
    if (!stencil7_tma_supported(dtype, in, out, ny, nx)) return cudaErrorNotSupported;
    if (dtype == 0)
        return fmad ? pipe_launch<float, true, 8, 4, 4>(in, in_shift, out, out_shift, ny, nx, lo, hi, c, S, (float)c0,
                                                        (float)c1, flags, st)
                    : pipe_launch<float, false, 8, 4, 4>(in, in_shift, out, out_shift, ny, nx, lo, hi, c, S, (float)c0,
                                                         (float)c1, flags, st);
    if (dtype == 1)
        return fmad ? pipe_launch<double, true, 8, 4, 4>(in, in_shift, out, out_shift, ny, nx, lo, hi, c, S, c0, c1,
                                                         flags, st)
                    : pipe_launch<double, false, 8, 4, 4>(in, in_shift, out, out_shift, ny, nx, lo, hi, c, S, c0, c1,
                                                          flags, st);
    return cudaErrorNotSupported;
}

namespace {
// LR: the last-releaser refill (no producer warp); chosen per dtype in conv_launch
template <typename T, int WARPS, int RPW, int NS, int MINB, int CPL, bool LR> int conv_occupancy() {
    using C = TmaCfg<T, WARPS, RPW, NS, !LR, CPL>;
    static std::mutex mu;
    static int occ[kMaxDevices] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= kMaxDevices) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!occ[dev]) {
        auto *kfn = conv3d_tma_kernel<T, WARPS, RPW, NS, MINB, CPL, LR>;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        int n = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kfn, C::THREADS, C::SMEM) != cudaSuccess) n = 1;
        cudaGetLastError();
        occ[dev] = n > 0 ? n : 1;
    }
    return occ[dev];
}

template <typename T, int WARPS, int RPW, int NS, int MINB, int CPL>
cudaError_t conv_launch(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny, int64_t nx,
                        int64_t k0, int64_t k1, cudaStream_t st) {
    constexpr bool LR = sizeof(T) == 4;
    using C = TmaCfg<T, WARPS, RPW, NS, !LR, CPL>;
    const CUtensorMap *m = get_map<C, T>(in, ny, nx);
    if (!m) return cudaErrorNotSupported;
    TmaParams p{};
    p.in_base = in.base;
    p.in_R = in.R;
    p.in_shift = in_shift;
    p.out_shift = out_shift;
    p.k0 = k0;
    p.nplanes = k1 - k0;
    p.ny = (int)ny;
    p.nx = (int)nx;
    p.tiles_x = (int)((nx + C::TX - 1) / C::TX);
    p.tiles = (int64_t)p.tiles_x * ((ny + C::TY - 1) / C::TY);
    const int64_t slots = (int64_t)sm_count() * conv_occupancy<T, WARPS, RPW, NS, MINB, CPL, LR>();
    // (a balanced split of the tile-major item list over all slots was measured slower, fp64 525 vs
    // 379 us: neighbouring tiles drift apart in z and their halos miss L2)
    int64_t zsegs = std::max<int64_t>(1, slots / p.tiles);
    zsegs = std::min<int64_t>(zsegs, std::max<int64_t>(1, p.nplanes / 4));
    p.zlen = (p.nplanes + zsegs - 1) / zsegs;
    zsegs = (p.nplanes + p.zlen - 1) / p.zlen;
    int64_t grid = p.tiles * zsegs;
    // fp32 (issue-bound, every warp counts): fill every resident slot — tiles [0, r) get one more
    // z-segment than the rest (512^3: 444 CTAs instead of 384, 219 -> 209 us). fp64 (closer to the
    // HBM bound) loses with it (370 -> 407 us: the two groups' z-fronts drift apart and their shared
    // halos miss L2), so it keeps the uniform map. profiles/r2_conv3d.md
    if (LR && slots > grid && slots % p.tiles && p.nplanes / (slots / p.tiles + 1) >= 4) {
        p.fill_q = slots / p.tiles;
        p.fill_r = slots % p.tiles;
        grid = slots;
    }
    if (grid >= (1ll << 31)) return cudaErrorInvalidConfiguration;
    conv3d_tma_kernel<T, WARPS, RPW, NS, MINB, CPL, LR><<<(unsigned)grid, C::THREADS, C::SMEM, st>>>(*m, p, out);
    return cudaGetLastError();
}

// PP_CONV_VARIANT (tuning build only, `make TUNING=1`): 0 = 8 warps x 4 rows, 5 stages, 2 CTAs/SM; 1 (default) = 8 x 4, 4 stages,
// 3 CTAs/SM (the body's serial 15-term chain needs the third resident CTA to hide its latency);
// 2 = 4 warps x 8 rows, 5 stages. Measurements: DESIGN.md §6 and profiles/r1_summary.md.
template <typename T>
cudaError_t conv_dispatch(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny,
                          int64_t nx, int64_t k0, int64_t k1, cudaStream_t st) {
#if PP_TUNING_VARIANTS
    static const int v = env_int("PP_CONV_VARIANT", 1, 0, 2);
    switch (v) {
    case 0: return conv_launch<T, 8, 4, 5, 2, TmaCfg<T, 1, 1, 1>::V>(in, in_shift, out, out_shift, ny, nx, k0, k1, st);
    case 2: return conv_launch<T, 4, 8, 5, 3, TmaCfg<T, 1, 1, 1>::V>(in, in_shift, out, out_shift, ny, nx, k0, k1, st);
    default: break;
    }
#endif
    // (fp32 alternatives measured slower on the resident 512^3 launch, profiles/r2_conv3d.md: two
    // columns per lane with 5 stages x 4 CTAs/SM 323 us, 6 stages x 3 CTAs 308 us; four columns with
    // 6 stages x 2 CTAs 263 us; 8 warps x 2 rows, 6 stages x 4 CTAs 403 us; 6 warps (88 tiles x 5
    // segments = 440 CTAs, every SM 3) 243 us; 5 warps x 4 CTAs 275 us; 4 warps x 6 rows 238 us;
    // this one 236 us)
    return conv_launch<T, 8, 4, 4, 3, TmaCfg<T, 1, 1, 1>::V>(in, in_shift, out, out_shift, ny, nx, k0, k1, st);
}
}  // namespace

cudaError_t launch_conv3d_tma(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                              int64_t ny, int64_t nx, int64_t k0, int64_t k1, cudaStream_t st) {
    if (k1 <= k0) return cudaSuccess;
    if (dtype == 0) return conv_dispatch<float>(in, in_shift, out, out_shift, ny, nx, k0, k1, st);
    if (dtype == 1) return conv_dispatch<double>(in, in_shift, out, out_shift, ny, nx, k0, k1, st);
    return cudaErrorNotSupported;
}

}  // namespace pp
