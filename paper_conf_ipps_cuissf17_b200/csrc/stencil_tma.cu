// stencil_tma.cu — TMA-staged 7-point stencil (Fig. 2 body) for sm_100a.
//
// Design: each CTA owns an (x,y) tile of TX x TY output points and marches through
// a contiguous range of planes (2.5-D blocking). Plane tiles of the input ring — with a one-point
// halo in y and a V-point halo in x, so the tile centres stay 16-byte aligned — are fetched by the
// Tensor Memory Accelerator (cp.async.bulk.tensor.3d, one elected thread) into an NS-stage shared
// memory ring; completion is signalled on one mbarrier per stage (complete_tx). The TMA box reads
// the device ring [R][ny][nx] directly at (x0-V, y0-1, slot), so the index handler's slot map
// costs one modulo per plane per CTA; out-of-range halo cells are zero-filled by the
// TMA unit and never used (edge points are passed through, reading S5). z-neighbours live in
// registers; x/y neighbours come from the staged centre plane; results go out as 16-byte stores.
// Arithmetic is the same RN-intrinsic sequence as the generic path (bit-exact, reading S4).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
#include <mutex>

#include "kernels.cuh"
#include "kernels_common.cuh"

namespace pp {

template <typename T> struct TmaCfg {
    static constexpr int V = 16 / (int)sizeof(T);   // points per thread per row (one 16-B vector)
    static constexpr int TX = 32 * V;                // tile width: one warp spans a tile row
    static constexpr int W = TX + 2 * V;             // staged row width (16-B multiple, centres aligned)
    static constexpr int WARPS = 8;
    static constexpr int RPW = 2;                    // rows per warp
    static constexpr int TY = WARPS * RPW;           // tile height
    static constexpr int H = TY + 2;                 // staged rows (one halo row each side)
    static constexpr int NS = 4;                     // smem pipeline stages (planes)
    static constexpr int STAGE_ELEMS = W * H;
    static constexpr int STAGE_BYTES = STAGE_ELEMS * (int)sizeof(T);      // bytes the TMA box writes
    static constexpr int STAGE_STRIDE = (STAGE_BYTES + 127) / 128 * 128;  // TMA smem dst: 128-B aligned
    static constexpr int STAGE_STRIDE_ELEMS = STAGE_STRIDE / (int)sizeof(T);
    static constexpr int SMEM = NS * STAGE_STRIDE + 128;
};

// ---------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, int x, int y, int z, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
            smem_u32(dst)),
        "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

template <typename T> __device__ __forceinline__ typename Vec16<T>::type lds16(const T *p) {
    return *reinterpret_cast<const typename Vec16<T>::type *>(p);
}

// ---------------------------------------------------------------- the kernel
template <typename T, bool FMAD>
__global__ void __launch_bounds__(256) stencil7_tma_kernel(const __grid_constant__ CUtensorMap tin,
                                                           int64_t in_base, int64_t in_R, int64_t in_shift,
                                                           DView out, int64_t out_shift, int ny, int nx,
                                                           int64_t k0, int64_t k1, int tiles_x, int tiles,
                                                           int64_t zlen, T c0, T c1) {
    using C = TmaCfg<T>;
    using VT = typename Vec16<T>::type;
    constexpr int V = C::V, NS = C::NS;
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T *stage = reinterpret_cast<T *>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem_raw + NS * C::STAGE_STRIDE);

    const int tile = blockIdx.x % tiles;
    const int64_t zs = blockIdx.x / tiles;
    const int x0 = (tile % tiles_x) * C::TX;
    const int y0 = (tile / tiles_x) * C::TY;
    const int64_t kb = k0 + zs * zlen;
    const int64_t ke = kb + zlen < k1 ? kb + zlen : k1;
    if (kb >= ke) return;                                        // uniform per CTA
    const int n_in = (int)(ke - kb) + 2;                         // input planes this CTA stages
    const int64_t g_first = kb + in_shift - 1;                   // global plane of input index 0
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool leader = threadIdx.x == 0;

    if (leader) {
        prefetch_tmap(&tin);
        for (int s = 0; s < NS; ++s) mbar_init(&full[s], 1);
        fence_barrier_init();
    }
    __syncthreads();
    int64_t slot_next = pmod64(g_first - in_base, in_R);         // slot of the next input index to issue
    auto issue = [&](int q) {                                    // leader only, q = input index
        const int s = q % NS;
        mbar_expect_tx(&full[s], C::STAGE_BYTES);
        tma_load_3d(stage + s * C::STAGE_STRIDE_ELEMS, &tin, x0 - V, y0 - 1, (int)slot_next, &full[s]);
        slot_next = slot_next + 1 == in_R ? 0 : slot_next + 1;
    };
    if (leader)
        for (int q = 0; q < NS && q < n_in; ++q) issue(q);

    // this thread's points: rows y0 + warp*RPW + rr, columns x0 + lane*V + v
    const int xl = lane * V;                                     // column in the tile
    const int xg = x0 + xl;
    const bool xin = xg < nx;                                    // whole vector in or out (nx % V == 0)
    T zm[C::RPW][V], ctr[C::RPW][V];

    mbar_wait(&full[0], 0);
    mbar_wait(&full[1 % NS], (1 / NS) & 1);
#pragma unroll
    for (int rr = 0; rr < C::RPW; ++rr) {
        const int row = warp * C::RPW + rr + 1;                  // staged row (halo row 0)
        VT a = lds16(stage + 0 * C::STAGE_STRIDE_ELEMS + row * C::W + xl + V);
        VT b = lds16(stage + (1 % NS) * C::STAGE_STRIDE_ELEMS + row * C::W + xl + V);
        memcpy(zm[rr], &a, 16);
        memcpy(ctr[rr], &b, 16);
    }
    __syncthreads();                                             // input index 0 consumed
    if (leader && NS < n_in) {
        fence_proxy_async();
        issue(NS);
    }

    T *outb = static_cast<T *>(out.ring);
    int64_t so = pmod64(kb + out_shift - out.base, out.R);
    for (int q = 0; q < n_in - 2; ++q) {                         // output plane kb + q
        const int qc = q + 1, qp = q + 2;                        // centre / z+1 input indices
        mbar_wait(&full[qp % NS], (qp / NS) & 1);
        const T *sc = stage + (qc % NS) * C::STAGE_STRIDE_ELEMS;
        const T *sp = stage + (qp % NS) * C::STAGE_STRIDE_ELEMS;
        T *op = outb + so * out.plane_elems;
#pragma unroll
        for (int rr = 0; rr < C::RPW; ++rr) {
            const int row = warp * C::RPW + rr + 1;
            const int yg = y0 + row - 1;
            const T *cr = sc + row * C::W + xl + V;              // centre row, aligned
            VT vzp = lds16(sp + row * C::W + xl + V);
            VT vyp = lds16(cr + C::W);
            VT vym = lds16(cr - C::W);
            T xm = cr[-1], xp = cr[V];
            T zp[V], yp[V], ym[V], res[V];
            memcpy(zp, &vzp, 16);
            memcpy(yp, &vyp, 16);
            memcpy(ym, &vym, 16);
            const bool yedge = (yg == 0 || yg == ny - 1);
#pragma unroll
            for (int v = 0; v < V; ++v) {
                const T l = v == 0 ? xm : ctr[rr][v - 1];
                const T r = v == V - 1 ? xp : ctr[rr][v + 1];
                const int xi = xg + v;
                const bool edge = yedge || xi == 0 || xi == nx - 1;
                res[v] = edge ? ctr[rr][v]
                              : Arith<T, FMAD>::stencil(zp[v], zm[rr][v], yp[v], ym[v], r, l, ctr[rr][v], c0, c1);
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
        so = so + 1 == out.R ? 0 : so + 1;
        __syncthreads();                                         // centre index qc consumed by all
        if (leader && qc + NS < n_in) {
            fence_proxy_async();
            issue(qc + NS);
        }
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
    const int64_t es = dtype == 0 ? 4 : 8;
    if (nx % V || nx < 3 || ny < 3) return false;                // 16-B row pitch (TMA stride rule)
    if (nx >= (1ll << 31) || ny >= (1ll << 31) || in.R >= (1ll << 31)) return false;
    if ((uintptr_t)in.ring % 16 || (uintptr_t)out.ring % 16) return false;
    if (in.plane_elems != nx * ny || out.plane_elems != nx * ny) return false;
    (void)es;
    return tma_available();
}

namespace {
struct MapKey {
    const void *ptr;
    int64_t R, ny, nx;
    int dtype;
    bool operator==(const MapKey &o) const {
        return ptr == o.ptr && R == o.R && ny == o.ny && nx == o.nx && dtype == o.dtype;
    }
};
struct MapCache {
    static constexpr int N = 16;
    MapKey key[N];
    CUtensorMap map[N];
    int used = 0, next = 0;
};
thread_local MapCache g_maps;

template <typename T> bool encode(CUtensorMap *m, const DView &in, int64_t ny, int64_t nx) {
    using C = TmaCfg<T>;
    const cuuint64_t dims[3] = {(cuuint64_t)nx, (cuuint64_t)ny, (cuuint64_t)in.R};
    const cuuint64_t strides[2] = {(cuuint64_t)(nx * sizeof(T)), (cuuint64_t)(nx * ny * sizeof(T))};
    const cuuint32_t box[3] = {(cuuint32_t)C::W, (cuuint32_t)C::H, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = encode_fn()(m, sizeof(T) == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                             3, in.ring, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

template <typename T> const CUtensorMap *get_map(const DView &in, int64_t ny, int64_t nx) {
    MapCache &c = g_maps;
    MapKey k{in.ring, in.R, ny, nx, (int)sizeof(T)};
    for (int i = 0; i < c.used; ++i)
        if (c.key[i] == k) return &c.map[i];
    int slot = c.used < MapCache::N ? c.used++ : (c.next++ % MapCache::N);
    if (!encode<T>(&c.map[slot], in, ny, nx)) {
        c.key[slot] = MapKey{nullptr, 0, 0, 0, 0};
        return nullptr;
    }
    c.key[slot] = k;
    return &c.map[slot];
}

template <typename T, bool FMAD> int occupancy() {
    static int occ = -1;
    static std::once_flag once;
    std::call_once(once, [] {
        using C = TmaCfg<T>;
        cudaFuncSetAttribute(stencil7_tma_kernel<T, FMAD>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        int n = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, stencil7_tma_kernel<T, FMAD>, 256, C::SMEM) != cudaSuccess)
            n = 1;
        cudaGetLastError();
        occ = n > 0 ? n : 1;
    });
    return occ;
}

int sm_count() {
    static int n = 0;
    static std::once_flag once;
    std::call_once(once, [] {
        int d = 0;
        cudaGetDevice(&d);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, d) != cudaSuccess || n <= 0) n = 148;
    });
    return n;
}

template <typename T, bool FMAD>
cudaError_t launch_t(const DView &in, int64_t in_shift, const DView &out, int64_t out_shift, int64_t ny,
                     int64_t nx, int64_t k0, int64_t k1, T c0, T c1, cudaStream_t st) {
    using C = TmaCfg<T>;
    const CUtensorMap *m = get_map<T>(in, ny, nx);
    if (!m) return cudaErrorNotSupported;
    const int64_t nplanes = k1 - k0;
    const int tiles_x = (int)((nx + C::TX - 1) / C::TX);
    const int64_t tiles = (int64_t)tiles_x * ((ny + C::TY - 1) / C::TY);
    // one wave: split the z range so tiles * zsegs fills the resident CTA slots (HBM-bound CTAs
    // progress at equal rates, so equal-length segments finish together)
    const int64_t slots = (int64_t)sm_count() * occupancy<T, FMAD>();
    int64_t zsegs = std::max<int64_t>(1, slots / tiles);
    zsegs = std::min<int64_t>(zsegs, std::max<int64_t>(1, nplanes / 4));
    const int64_t zlen = (nplanes + zsegs - 1) / zsegs;
    zsegs = (nplanes + zlen - 1) / zlen;
    const int64_t grid = tiles * zsegs;
    if (grid >= (1ll << 31) || tiles >= (1ll << 31)) return cudaErrorInvalidConfiguration;
    stencil7_tma_kernel<T, FMAD><<<(unsigned)grid, 256, C::SMEM, st>>>(
        *m, in.base, in.R, in_shift, out, out_shift, (int)ny, (int)nx, k0, k1, tiles_x, (int)tiles, zlen, c0, c1);
    return cudaGetLastError();
}
}  // namespace

cudaError_t launch_stencil7_tma(int dtype, const DView &in, int64_t in_shift, const DView &out, int64_t out_shift,
                                int64_t ny, int64_t nx, int64_t k0, int64_t k1, double c0, double c1, bool fmad,
                                cudaStream_t st) {
    if (dtype == 0)
        return fmad ? launch_t<float, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, (float)c0, (float)c1, st)
                    : launch_t<float, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, (float)c0, (float)c1, st);
    if (dtype == 1)
        return fmad ? launch_t<double, true>(in, in_shift, out, out_shift, ny, nx, k0, k1, c0, c1, st)
                    : launch_t<double, false>(in, in_shift, out, out_shift, ny, nx, k0, k1, c0, c1, st);
    return cudaErrorNotSupported;
}

}  // namespace pp
