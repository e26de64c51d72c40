// zc_probe3.cu -- random-row zero-copy gather/scatter with FRESH random rows every
// iteration (cold GPU translation caches), per host allocation method.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return; } } while (0)
__global__ void gather(const int32_t* idx, int n, const float4* h, float4* out) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) out[u * 8 + l] = h[(int64_t)idx[u] * 8 + l];
}
__global__ void scatter(const int32_t* idx, int n, float4* h, const float4* in) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) h[(int64_t)idx[u] * 8 + l] = in[u * 8 + l];
}
static const int64_t N = 33762577;
static const int n = 41000, ITERS = 8;
static int32_t* didx;
static float4* obuf;
void run(const char* name, void* h, size_t bytes) {
    float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float tg = 0, ts = 0;
    for (int it = 0; it < ITERS; it++) {
        const int32_t* ig = didx + (size_t)(2 * it) * n;
        const int32_t* is = didx + (size_t)(2 * it + 1) * n;
        cudaEventRecord(a); gather<<<592, 256>>>(ig, n, dh, obuf); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); if (it) tg += ms;
        cudaEventRecord(a); scatter<<<592, 256>>>(is, n, dh, obuf); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b); if (it) ts += ms;
    }
    printf("%-28s cold gather %.3f ms (%.1f GB/s)  cold scatter %.3f ms (%.1f GB/s)\n", name, tg / (ITERS - 1),
           n * 128.0 / (tg / (ITERS - 1)) / 1e6, ts / (ITERS - 1), n * 128.0 / (ts / (ITERS - 1)) / 1e6);
}
int main() {
    const size_t bytes = (size_t)N * 128;
    int32_t* hidx = (int32_t*)malloc((size_t)2 * ITERS * n * 4);
    srand(7);
    for (size_t i = 0; i < (size_t)2 * ITERS * n; i++) hidx[i] = (int32_t)(((int64_t)rand() * RAND_MAX + rand()) % N);
    cudaMalloc(&didx, (size_t)2 * ITERS * n * 4); cudaMalloc(&obuf, (size_t)n * 128);
    cudaMemcpy(didx, hidx, (size_t)2 * ITERS * n * 4, cudaMemcpyHostToDevice);
    {
        void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); memset(h, 0, bytes);
        cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable); run("shm 4K", h, bytes);
        cudaHostUnregister(h); munmap(h, bytes);
    }
    {
        size_t al = 2 << 20; void* raw = mmap(0, bytes + al, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
        void* h = (void*)(((uintptr_t)raw + al - 1) & ~(al - 1));
        int r = madvise(h, bytes, MADV_HUGEPAGE); memset(h, 0, bytes);
        cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable); run(r ? "private THP(madvise failed)" : "private THP", h, bytes);
        cudaHostUnregister(h); munmap(raw, bytes + al);
    }
    {
        void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS | MAP_HUGETLB, -1, 0);
        if (h == MAP_FAILED) printf("hugetlbfs 2M: mmap failed\n");
        else { memset(h, 0, bytes); cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable); run("hugetlbfs 2M", h, bytes); cudaHostUnregister(h); munmap(h, bytes); }
    }
    {
        void* h; if (cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable) == cudaSuccess) { memset(h, 0, bytes); run("cudaHostAlloc", h, bytes); cudaFreeHost(h); }
    }
    return 0;
}
