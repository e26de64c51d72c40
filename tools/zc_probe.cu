// zc_probe.cu -- host-link microbenchmark: random-row zero-copy gather (H2D) and
// scatter (D2H) of d=32 fp32 rows over an 8 GB pinned host table, for several host
// allocation methods.  Prints GB/s.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 zc_probe.cu -o zc_probe
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

template <int GS>
__global__ void gather(const int32_t* idx, int n, const float4* h, float4* out, int d4) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t gid = t / GS, gs = ((int64_t)gridDim.x * blockDim.x) / GS;
    int l = threadIdx.x & (GS - 1);
    for (int64_t u = gid; u < n; u += gs) {
        const float4* src = h + (int64_t)idx[u] * d4;
        for (int v = l; v < d4; v += GS) out[u * d4 + v] = src[v];
    }
}
template <int GS>
__global__ void scatter(const int32_t* idx, int n, float4* h, const float4* in, int d4) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t gid = t / GS, gs = ((int64_t)gridDim.x * blockDim.x) / GS;
    int l = threadIdx.x & (GS - 1);
    for (int64_t u = gid; u < n; u += gs) {
        float4* dst = h + (int64_t)idx[u] * d4;
        for (int v = l; v < d4; v += GS) dst[v] = in[u * d4 + v];
    }
    __threadfence_system();
}

int main(int argc, char** argv) {
    const int64_t N = 33762577;  // Criteo-Kaggle rows
    const int d = 32, d4 = 8;
    const size_t bytes = (size_t)N * d * 4;
    const int n = argc > 1 ? atoi(argv[1]) : 41000;
    int32_t* hidx = (int32_t*)malloc(n * 4);
    srand(1);
    for (int i = 0; i < n; i++) hidx[i] = (int32_t)(((int64_t)rand() * RAND_MAX + rand()) % N);
    int32_t* didx; float4* dout;
    CK(cudaMalloc(&didx, n * 4)); CK(cudaMalloc(&dout, (size_t)n * d * 4));
    CK(cudaMemcpy(didx, hidx, n * 4, cudaMemcpyHostToDevice));
    const char* names[] = {"mmap_shared_anon", "mmap_private_anon_thp", "cudaHostAlloc"};
    for (int m = 0; m < 3; m++) {
        void* h = nullptr;
        if (m == 0) { h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); }
        if (m == 1) { h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0); madvise(h, bytes, MADV_HUGEPAGE); }
        if (m == 0 || m == 1) { memset(h, 0, bytes); CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable)); }
        if (m == 2) { CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable)); memset(h, 0, bytes); }
        float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        for (int blocks : {32, 148, 296, 1184}) {
            float best_g = 1e9, best_s = 1e9;
            for (int it = 0; it < 5; it++) {
                cudaEventRecord(a); gather<8><<<blocks, 256>>>(didx, n, dh, dout, d4); cudaEventRecord(b); cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best_g) best_g = ms;
                cudaEventRecord(a); scatter<8><<<blocks, 256>>>(didx, n, dh, dout, d4); cudaEventRecord(b); cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms, a, b); if (ms < best_s) best_s = ms;
            }
            printf("%-24s blocks=%5d rows=%d gather %.3f ms %.1f GB/s | scatter %.3f ms %.1f GB/s\n", names[m], blocks, n,
                   best_g, n * 128.0 / best_g / 1e6, best_s, n * 128.0 / best_s / 1e6);
        }
        if (m == 2) cudaFreeHost(h); else { cudaHostUnregister(h); munmap(h, bytes); }
    }
    // sequential memcpy reference
    return 0;
}
