// zc_probe5.cu -- is the random-row host-link ceiling a function of the FOOTPRINT (pages
// touched: IOMMU / GPU TLB reach) or of host DRAM latency?  Random 128-B rows drawn fresh
// every iteration from a window of F bytes at the start of a 4.3 GB host table, for F from
// 8 MB to the whole table; 4K pages vs THP (madvise) backing.  Gather (loads) and scatter
// (stores).  Output: one line per (backing, F, op).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__global__ void g_gather(const int32_t* idx, int n, const float4* h, float4* out) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) out[u * 8 + l] = h[(int64_t)idx[u] * 8 + l];
}
__global__ void g_scatter(const int32_t* idx, int n, float4* h, const float4* in) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) h[(int64_t)idx[u] * 8 + l] = in[u * 8 + l];
}

static uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull; x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull; return x ^ (x >> 31);
}

int main(int argc, char** argv) {
    const int64_t N = 33762577; const size_t bytes = (size_t)N * 128; const int n = 41000, IT = 8;
    int32_t* hidx = (int32_t*)malloc((size_t)IT * n * 4);
    int32_t* didx; float4* out; CK(cudaMalloc(&didx, (size_t)IT * n * 4)); CK(cudaMalloc(&out, (size_t)n * 128));
    CK(cudaMemset(out, 0, (size_t)n * 128));
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int thp = 0; thp < 2; thp++) {
        void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
        if (thp) madvise(h, bytes, MADV_HUGEPAGE); else madvise(h, bytes, MADV_NOHUGEPAGE);
        memset(h, 1, bytes);
        CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
        float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
        for (int64_t foot : {(int64_t)8 << 20, (int64_t)32 << 20, (int64_t)128 << 20, (int64_t)512 << 20, (int64_t)2048 << 20, (int64_t)bytes}) {
            int64_t rows = foot / 128; if (rows > N) rows = N;
            for (int op = 0; op < 2; op++) {
                uint64_t seed = 1234 + foot + op;
                for (size_t i = 0; i < (size_t)IT * n; i++) hidx[i] = (int32_t)(sm64(seed + i) % (uint64_t)rows);
                CK(cudaMemcpy(didx, hidx, (size_t)IT * n * 4, cudaMemcpyHostToDevice));
                float tot = 0;
                for (int it = 0; it < IT; it++) {
                    const int32_t* ix = didx + (size_t)it * n;
                    cudaEventRecord(a);
                    if (op == 0) g_gather<<<148, 256>>>(ix, n, dh, out); else g_scatter<<<148, 256>>>(ix, n, dh, out);
                    cudaEventRecord(b); CK(cudaEventSynchronize(b));
                    float ms; cudaEventElapsedTime(&ms, a, b); if (it) tot += ms;
                }
                float ms = tot / (IT - 1);
                printf("%-4s footprint %7.0f MB %-7s %.3f ms %5.1f GB/s\n", thp ? "THP" : "4K", foot / 1048576.0,
                       op ? "scatter" : "gather", ms, n * 128.0 / ms / 1e6);
                fflush(stdout);
            }
        }
        CK(cudaHostUnregister(h)); munmap(h, bytes);
    }
    return 0;
}
