// hostlink_probe.cu — can SM-issued stores/loads over PCIe replace the copy engines?
// Measures (1 GiB each, CUDA events):
//   ce_d2h / ce_h2d        copy-engine cudaMemcpyAsync alone
//   sm_store               kernel streaming device -> pinned host (16-B stores), alone
//   sm_load                kernel streaming pinned host -> device (16-B loads), alone
//   ce_h2d + sm_store      concurrently (the fused-D2H pipeline's steady state)
//   ce_h2d + ce_d2h        concurrently (the copy-engine pipeline's steady state)
//   sm_load + sm_store     both directions by SMs
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/hostlink_probe tools/hostlink_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t e_ = (x);                                                                  \
        if (e_ != cudaSuccess) {                                                               \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_));         \
            exit(1);                                                                           \
        }                                                                                      \
    } while (0)

__global__ void stream_copy(const int4 *__restrict__ src, int4 *__restrict__ dst, size_t n16) {
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    size_t stride = (size_t)gridDim.x * blockDim.x;
#pragma unroll 4
    for (; i < n16; i += stride) dst[i] = src[i];
}

int main(int argc, char **argv) {
    const size_t GB = 1ull << 30;
    const int blocks = argc > 1 ? atoi(argv[1]) : 148 * 8;
    char *h_in, *h_out, *d_a, *d_b, *d_c, *d_d;
    CK(cudaHostAlloc(&h_in, GB, cudaHostAllocMapped | cudaHostAllocPortable));
    CK(cudaHostAlloc(&h_out, GB, cudaHostAllocMapped | cudaHostAllocPortable));
    CK(cudaMalloc(&d_a, GB));
    CK(cudaMalloc(&d_b, GB));
    CK(cudaMalloc(&d_c, GB));
    CK(cudaMalloc(&d_d, GB));
    for (size_t i = 0; i < GB; i += 4096) h_in[i] = 1, h_out[i] = 2;
    cudaStream_t s1, s2;
    CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
    cudaEvent_t a0, a1, b0, b1;
    CK(cudaEventCreate(&a0));
    CK(cudaEventCreate(&a1));
    CK(cudaEventCreate(&b0));
    CK(cudaEventCreate(&b1));
    const size_t n16 = GB / 16;
    auto sm_store = [&](cudaStream_t s) { stream_copy<<<blocks, 256, 0, s>>>((int4 *)d_a, (int4 *)h_out, n16); };
    auto sm_load = [&](cudaStream_t s) { stream_copy<<<blocks, 256, 0, s>>>((int4 *)h_in, (int4 *)d_b, n16); };
    auto ce_h2d = [&](cudaStream_t s) { CK(cudaMemcpyAsync(d_c, h_in, GB, cudaMemcpyHostToDevice, s)); };
    auto ce_d2h = [&](cudaStream_t s) { CK(cudaMemcpyAsync(h_out, d_d, GB, cudaMemcpyDeviceToHost, s)); };
    struct Case { const char *name; int mode; } cases[] = {
        {"ce_h2d", 0}, {"ce_d2h", 1}, {"sm_store", 2}, {"sm_load", 3},
        {"ce_h2d+sm_store", 4}, {"ce_h2d+ce_d2h", 5}, {"sm_load+sm_store", 6}, {"sm_load+ce_d2h", 7}};
    for (auto &c : cases) {
        float best1 = 1e30f, best2 = 1e30f;
        for (int rep = 0; rep < 4; ++rep) {
            CK(cudaDeviceSynchronize());
            CK(cudaEventRecord(a0, s1));
            CK(cudaEventRecord(b0, s2));
            switch (c.mode) {
            case 0: ce_h2d(s1); break;
            case 1: ce_d2h(s1); break;
            case 2: sm_store(s1); break;
            case 3: sm_load(s1); break;
            case 4: ce_h2d(s1); sm_store(s2); break;
            case 5: ce_h2d(s1); ce_d2h(s2); break;
            case 6: sm_load(s1); sm_store(s2); break;
            case 7: sm_load(s1); ce_d2h(s2); break;
            }
            CK(cudaEventRecord(a1, s1));
            CK(cudaEventRecord(b1, s2));
            CK(cudaDeviceSynchronize());
            float t1, t2;
            CK(cudaEventElapsedTime(&t1, a0, a1));
            CK(cudaEventElapsedTime(&t2, b0, b1));
            if (rep) { if (t1 < best1) best1 = t1; if (t2 < best2) best2 = t2; }
        }
        const bool two = c.mode >= 4;
        printf("{\"case\": \"%s\", \"blocks\": %d, \"gbs_1\": %.2f, \"gbs_2\": %s%.2f}\n", c.name, blocks,
               GB / (best1 * 1e-3) / 1e9, "", two ? GB / (best2 * 1e-3) / 1e9 : 0.0);
        fflush(stdout);
    }
    return 0;
}
