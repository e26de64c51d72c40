// interf_probe.cu -- why do the side drain's zero-copy host writes slow the concurrent HBM
// kernels ~2x?  Victims: (V1) 256 MB device copy, (V2) random 128-B row gather inside a 27 MB
// (L2-resident) buffer.  Aggressor on a second stream: random 128-B row scatter from HBM to a
// 4.3 GB pinned host table with G CTAs, store variants: plain / st.global.cs / L2 evict_first
// policy / TMA bulk store (cp.async.bulk.global.shared::cta) / host reads instead of writes.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
__device__ __forceinline__ uint32_t hsh(uint64_t x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33; return (uint32_t)x; }
__global__ void v_copy(const float4* a, float4* b, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) b[i] = a[i];
}
__global__ void v_rows(const float4* src, float4* dst, int64_t rows, int64_t n, uint32_t seed) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) dst[(u % rows) * 8 + l] = src[(int64_t)(hsh(u ^ seed) % rows) * 8 + l];
}
template <int MODE>
__global__ void agg(const float4* pool, float4* host, int64_t hrows, int64_t n, uint32_t seed, uint64_t pol) {
    __shared__ __align__(128) float4 sm[256 / 8][8];
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    if (MODE == 2) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    for (int64_t u = t / 8; u < n; u += gs) {
        float4 x = pool[(u % 200000) * 8 + l];
        float4* d = host + (int64_t)(hsh(u * 7 + seed) % hrows) * 8 + l;
        if (MODE == 0) *d = x;
        if (MODE == 1) asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(d), "f"(x.x), "f"(x.y), "f"(x.z), "f"(x.w) : "memory");
        if (MODE == 2) asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(d), "f"(x.x), "f"(x.y), "f"(x.z), "f"(x.w), "l"(pol) : "memory");
        if (MODE == 3) {
            float4* s = &sm[threadIdx.x / 8][l];
            *s = x;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (l == 0) {
                unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[threadIdx.x / 8][0]);
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], 128;" ::"l"(d), "r"(sa) : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
            __syncwarp();
        }
        if (MODE == 4) {  // host reads (the gather's direction)
            float4 y = __ldcv(d);
            if (y.x == 12345.f) host[0] = y;
        }
    }
}
int main() {
    const int64_t hrows = 33762577;
    float4 *h, *hd; CK(cudaHostAlloc(&h, hrows * 128, cudaHostAllocMapped)); CK(cudaHostGetDevicePointer(&hd, h, 0));
    float4 *a, *b, *pool, *r27, *r27o;
    const int64_t n4 = (256 << 20) / 16;
    CK(cudaMalloc(&a, n4 * 16)); CK(cudaMalloc(&b, n4 * 16)); CK(cudaMalloc(&pool, 200000 * 128));
    const int64_t rr = 212992;  // 27 MB of 128-B rows
    CK(cudaMalloc(&r27, rr * 128)); CK(cudaMalloc(&r27o, rr * 128));
    cudaStream_t s1, s2; cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t e0, e1, f0, f1; cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventCreate(&f0); cudaEventCreate(&f1);
    uint64_t pol; 
    auto victim = [&](int v, cudaStream_t st) {
        if (v == 0) v_copy<<<148 * 8, 256, 0, st>>>(a, b, n4);
        else v_rows<<<148 * 8, 256, 0, st>>>(r27, r27o, rr, rr, 7);
    };
    auto aggr = [&](int mode, int G, int64_t n, cudaStream_t st) {
        switch (mode) {
            case 0: agg<0><<<G, 256, 0, st>>>(pool, hd, hrows, n, 3, 0); break;
            case 1: agg<1><<<G, 256, 0, st>>>(pool, hd, hrows, n, 3, 0); break;
            case 2: agg<2><<<G, 256, 0, st>>>(pool, hd, hrows, n, 3, pol); break;
            case 3: agg<3><<<G, 256, 0, st>>>(pool, hd, hrows, n, 3, 0); break;
            case 4: agg<4><<<G, 256, 0, st>>>(pool, hd, hrows, n, 3, 0); break;
        }
    };
    // L2 evict_first policy
    {
        uint64_t* dp; CK(cudaMalloc(&dp, 8));
        // createpolicy in a tiny kernel
        void* args[] = {&dp};
        (void)args;
        pol = 0;
    }
    const char* mn[5] = {"plain st", "st.cs", "st L2 evict_first", "TMA bulk st", "host reads"};
    for (int v = 0; v < 2; v++) {
        float alone = 0, ms;
        for (int rep = 0; rep < 5; rep++) {
            cudaEventRecord(e0, s1); victim(v, s1); cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
            cudaEventElapsedTime(&ms, e0, e1); if (rep >= 1) alone += ms / 4;
        }
        printf("victim %s alone %.3f ms\n", v ? "V2 random rows 27MB" : "V1 copy 256MB", alone);
        for (int mode = 0; mode < 5; mode++)
            for (int G : {8, 20, 74}) {
                // aggressor alone: rows/ms
                const int64_t n = 30000;
                cudaEventRecord(f0, s2); aggr(mode, G, n, s2); cudaEventRecord(f1, s2); CK(cudaEventSynchronize(f1));
                float am; cudaEventElapsedTime(&am, f0, f1);
                // concurrent: long aggressor (keeps running) + victim
                float tv = 0;
                for (int rep = 0; rep < 3; rep++) {
                    aggr(mode, G, 400000, s2);
                    cudaEventRecord(e0, s1); victim(v, s1); cudaEventRecord(e1, s1);
                    CK(cudaDeviceSynchronize());
                    cudaEventElapsedTime(&ms, e0, e1); tv += ms / 3;
                }
                printf("  %-14s G=%3d  aggressor alone %.3f ms/30k rows (%.1f GB/s)   victim with it %.3f ms (x%.2f)\n", mn[mode], G, am,
                       30000 * 128 / (am * 1e6), tv, tv / alone);
            }
    }
    return 0;
}
