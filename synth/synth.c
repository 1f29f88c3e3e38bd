/* synth.c — seeded, counter-based synthetic input generator (SURVEY.md §8(d) "Inputs, exactly").
 *
 * Shared by BOTH sides (the CUDA path's tests/bench and the oracle's tests). It holds none of the
 * method's arithmetic: it only produces input values as a pure function of (seed, global linear
 * index g), so any thread, GPU or rank can regenerate element g independently.
 *
 *   h = splitmix64(seed ^ (g * 0x9E3779B97F4A7C15))
 *   fp64 value = (h >> 11) * 2^-53      in U[0,1)
 *   fp32 value = (h >> 40) * 2^-24      in U[0,1)
 *
 * Closed-form fields (for the oracle pins) are functions of the coordinates
 * (i, j, k) of g in a row-major [nz][ny][nx] grid, i fastest (reading S1).
 */
#include <stdint.h>
#include <string.h>

enum { SY_RANDOM = 0, SY_CONST = 1, SY_LINEAR = 2, SY_QUAD = 3, SY_CHECKER = 4, SY_PLANE = 5,
       SY_INDEX = 6, SY_CUBIC = 7, SY_RANDINT = 8 };

static inline uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

static inline uint64_t sy_hash(uint64_t seed, uint64_t g) {
    return splitmix64(seed ^ (g * 0x9E3779B97F4A7C15ull));
}

/* Value of field `kind` at global index g, as an exact double (all closed forms are integers). */
static inline double sy_field(int kind, uint64_t seed, int64_t g, int64_t nx, int64_t ny) {
    int64_t i = g % nx, j = (g / nx) % ny, k = g / (nx * ny);
    switch (kind) {
    case SY_CONST: return (double)seed;
    case SY_LINEAR: return (double)(i + 2 * j + 3 * k);
    case SY_QUAD: return (double)(i * i + j * j + k * k);
    case SY_CHECKER: return (double)((i + j + k) & 1);
    case SY_PLANE: return (double)k;
    case SY_INDEX: return (double)g;
    case SY_CUBIC: return (double)(1 + i + 2 * j * j + 3 * k * k * k);
    case SY_RANDINT: return (double)(int64_t)(sy_hash(seed, (uint64_t)g) % 2001) - 1000.0;
    default: return 0.0;
    }
}

void sy_fill_f64(double *dst, int64_t g0, int64_t n, int kind, uint64_t seed, int64_t nx, int64_t ny) {
    #pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < n; ++t) {
        int64_t g = g0 + t;
        if (kind == SY_RANDOM)
            dst[t] = (double)(sy_hash(seed, (uint64_t)g) >> 11) * 0x1.0p-53;
        else
            dst[t] = sy_field(kind, seed, g, nx, ny);
    }
}

void sy_fill_f32(float *dst, int64_t g0, int64_t n, int kind, uint64_t seed, int64_t nx, int64_t ny) {
    #pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < n; ++t) {
        int64_t g = g0 + t;
        if (kind == SY_RANDOM)
            dst[t] = (float)(sy_hash(seed, (uint64_t)g) >> 40) * 0x1.0p-24f;
        else
            dst[t] = (float)sy_field(kind, seed, g, nx, ny);
    }
}

void sy_fill_i64(int64_t *dst, int64_t g0, int64_t n, int kind, uint64_t seed, int64_t nx, int64_t ny) {
    #pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < n; ++t) {
        int64_t g = g0 + t;
        if (kind == SY_RANDOM)
            dst[t] = (int64_t)sy_hash(seed, (uint64_t)g);
        else
            dst[t] = (int64_t)sy_field(kind, seed, g, nx, ny);
    }
}

/* Fill n elements of `elem` bytes each with the same bit pattern (the "untouched" sentinel:
 * fp64 0x7ff8dead0000beef, fp32 0x7fc0beef — quiet-NaN payloads). */
void sy_fill_pattern(void *dst, int64_t n, int elem, uint64_t pattern) {
    if (elem == 8) {
        uint64_t *d = (uint64_t *)dst;
        #pragma omp parallel for schedule(static)
        for (int64_t t = 0; t < n; ++t) d[t] = pattern;
    } else {
        uint32_t *d = (uint32_t *)dst;
        uint32_t p = (uint32_t)pattern;
        #pragma omp parallel for schedule(static)
        for (int64_t t = 0; t < n; ++t) d[t] = p;
    }
}

/* Count elements of `a` whose bits differ from `pattern` (sentinel survival checks). */
int64_t sy_count_pattern(const void *src, int64_t n, int elem, uint64_t pattern) {
    int64_t cnt = 0;
    if (elem == 8) {
        const uint64_t *d = (const uint64_t *)src;
        #pragma omp parallel for reduction(+:cnt) schedule(static)
        for (int64_t t = 0; t < n; ++t) cnt += (d[t] == pattern);
    } else {
        const uint32_t *d = (const uint32_t *)src;
        uint32_t p = (uint32_t)pattern;
        #pragma omp parallel for reduction(+:cnt) schedule(static)
        for (int64_t t = 0; t < n; ++t) cnt += (d[t] == p);
    }
    return cnt;
}

/* Worker threads of the fills (OpenMP). torchrun exports OMP_NUM_THREADS=1 to every rank; a rank that
 * owns a share of the host's cores sets its own count here. */
#include <omp.h>
void sy_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
int sy_threads(void) { return omp_get_max_threads(); }
