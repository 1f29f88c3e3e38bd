// kernels_common.cuh — device helpers shared by the CUDA kernels (product side only).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace pp {

__host__ __device__ __forceinline__ int64_t pmod64(int64_t a, int64_t m) {
    int64_t r = a % m;
    return r < 0 ? r + m : r;
}

template <typename T> __device__ __forceinline__ T ldg(const T *p) { return __ldg(p); }
template <> __device__ __forceinline__ uint64_t ldg<uint64_t>(const uint64_t *p) {
    return (uint64_t)__ldg((const unsigned long long *)p);
}

template <typename T> struct Vec16;
template <> struct Vec16<float> { using type = float4; static constexpr int width = 4; };
template <> struct Vec16<double> { using type = double2; static constexpr int width = 2; };

// streaming 128-bit load (read once: do not allocate in L1) and store
__device__ __forceinline__ float4 ldg_nc(const float4 *p) {
    float4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ double2 ldg_nc(const double2 *p) {
    double2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(r.x), "=d"(r.y) : "l"(p));
    return r;
}
__device__ __forceinline__ void stg_na(float4 *p, const float4 &v) {
    asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y),
                 "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ void stg_na(double2 *p, const double2 &v) {
    asm volatile("st.global.L1::no_allocate.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(v.x), "d"(v.y) : "memory");
}

// Arithmetic in the loop bodies' exact order. Non-FMAD: every op individually rounded (RN intrinsics
// are never contracted). FMAD: one fused multiply-add for the final combination.
template <typename T, bool FMAD> struct Arith;

template <bool FMAD> struct Arith<float, FMAD> {
    static __device__ __forceinline__ float mul(float a, float b) { return __fmul_rn(a, b); }
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float stencil(float zp, float zm, float yp, float ym, float xp,
                                                    float xm, float ctr, float c0, float c1) {
        float s = __fadd_rn(zp, zm);
        s = __fadd_rn(s, yp);
        s = __fadd_rn(s, ym);
        s = __fadd_rn(s, xp);
        s = __fadd_rn(s, xm);
        if (FMAD) return __fmaf_rn(s, c1, -__fmul_rn(ctr, c0));
        return __fsub_rn(__fmul_rn(s, c1), __fmul_rn(ctr, c0));
    }
    static __device__ __forceinline__ float triad(float a, float b, float s) {
        if (FMAD) return __fmaf_rn(s, b, a);
        return __fadd_rn(a, __fmul_rn(s, b));
    }
};

template <bool FMAD> struct Arith<double, FMAD> {
    static __device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
    static __device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ double stencil(double zp, double zm, double yp, double ym, double xp,
                                                     double xm, double ctr, double c0, double c1) {
        double s = __dadd_rn(zp, zm);
        s = __dadd_rn(s, yp);
        s = __dadd_rn(s, ym);
        s = __dadd_rn(s, xp);
        s = __dadd_rn(s, xm);
        if (FMAD) return __fma_rn(s, c1, -__dmul_rn(ctr, c0));
        return __dsub_rn(__dmul_rn(s, c1), __dmul_rn(ctr, c0));
    }
    static __device__ __forceinline__ double triad(double a, double b, double s) {
        if (FMAD) return __fma_rn(s, b, a);
        return __dadd_rn(a, __dmul_rn(s, b));
    }
};

template <bool FMAD> struct Arith<uint64_t, FMAD> {
    static __device__ __forceinline__ uint64_t stencil(uint64_t zp, uint64_t zm, uint64_t yp, uint64_t ym,
                                                       uint64_t xp, uint64_t xm, uint64_t ctr, uint64_t c0,
                                                       uint64_t c1) {
        uint64_t s = zp + zm;
        s = s + yp;
        s = s + ym;
        s = s + xp;
        s = s + xm;
        return s * c1 - ctr * c0;
    }
};

}  // namespace pp
