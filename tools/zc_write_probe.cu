// zc_write_probe.cu -- sequential zero-copy write bandwidth to pinned host memory (the drain's pack
// into the flushing threads' staging queue): plain coalesced float4 stores vs TMA bulk stores
// (cp.async.bulk.global.shared::cta, 4 KB per instruction), by grid size; and the latency of a
// single host-flag read issued while the writes are in flight (PCIe reads are ordered behind
// posted writes).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o zc_write_probe zc_write_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__global__ void k_plain(const float4* __restrict__ src, float4* dst, long n4) {
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) dst[i] = src[i];
}
constexpr int CH = 4096;  // bytes per bulk store
__global__ void k_tma(const float4* __restrict__ src, char* dst, long nbytes) {
    __shared__ __align__(128) float4 sm[2][CH / 16];
    int stage = 0;
    for (long c = blockIdx.x; c * CH < nbytes; c += gridDim.x) {
        if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        __syncthreads();
        for (int i = threadIdx.x; i < CH / 16; i += blockDim.x) sm[stage][i] = src[c * (CH / 16) + i];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[stage][0]);
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + c * CH), "r"(sa), "r"(CH) : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
        stage ^= 1;
    }
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
__global__ void k_poll(const unsigned* f, unsigned long long* out) {
    unsigned long long t0, t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    unsigned x;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(x) : "l"(f) : "memory");
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    out[0] = t1 - t0 + (x == 12345u);
}
int main() {
    const long bytes = 6l << 20;
    float4* dsrc; char* h; char* dh; unsigned* hf; unsigned* df; unsigned long long* dlat;
    CK(cudaMalloc(&dsrc, bytes));
    CK(cudaMemset(dsrc, 1, bytes));
    CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
    CK(cudaHostAlloc(&hf, 64, cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer((void**)&df, hf, 0));
    CK(cudaMalloc(&dlat, 8));
    cudaStream_t s1, s2;
    cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    int grids[] = {8, 20, 40, 80, 148};
    for (int kind = 0; kind < 2; kind++)
        for (int g : grids) {
            float best = 1e9;
            for (int rep = 0; rep < 5; rep++) {
                cudaEventRecord(a, s1);
                if (kind == 0) k_plain<<<g, 256, 0, s1>>>(dsrc, (float4*)dh, bytes / 16);
                else k_tma<<<g, 128, 0, s1>>>(dsrc, dh, bytes);
                cudaEventRecord(b, s1);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (ms < best) best = ms;
            }
            // flag-read latency while this writer runs (poll issued ~5 us after the writer starts)
            if (kind == 0) k_plain<<<g, 256, 0, s1>>>(dsrc, (float4*)dh, bytes / 16);
            else k_tma<<<g, 128, 0, s1>>>(dsrc, dh, bytes);
            k_poll<<<1, 1, 0, s2>>>(df, dlat);
            cudaDeviceSynchronize();
            unsigned long long lat; cudaMemcpy(&lat, dlat, 8, cudaMemcpyDeviceToHost);
            k_poll<<<1, 1, 0, s2>>>(df, dlat);
            cudaDeviceSynchronize();
            unsigned long long lat0; cudaMemcpy(&lat0, dlat, 8, cudaMemcpyDeviceToHost);
            printf("%-6s grid %4d: %6.1f us for %ld MB = %5.1f GB/s   host-flag read during it %6.1f us (idle %4.1f us)\n",
                   kind ? "tma" : "plain", g, best * 1e3, bytes >> 20, bytes / (best * 1e-3) / 1e9, lat / 1e3, lat0 / 1e3);
        }
    return 0;
}
