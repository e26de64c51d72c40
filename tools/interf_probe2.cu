// interf_probe2.cu -- is the slowdown of HBM kernels under concurrent zero-copy host traffic
// (tools/interf_probe.cu: up to 34x) an address-translation effect?  Same victim (256 MB device
// copy) and aggressor (random 128-B host-row writes / reads, 20 and 74 CTAs), with the host
// table (a) cudaHostAlloc, (b) CUDA VMM cuMemCreate HOST_NUMA (2 MB granularity), (c) hugetlbfs
// 2 MB + cudaHostRegister, (d) THP-advised shm + cudaHostRegister; and footprints 64 MB .. 4.3 GB.
#include <cuda.h>
#include <cuda_runtime.h>
#include <fcntl.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <unistd.h>
#include <linux/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
__device__ __forceinline__ uint32_t hsh(uint64_t x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33; return (uint32_t)x; }
__global__ void v_copy(const float4* a, float4* b, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) b[i] = a[i];
}
template <int MODE>
__global__ void agg(const float4* pool, float4* host, int64_t hrows, int64_t n, uint32_t seed) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) {
        float4* d = host + (int64_t)(hsh(u * 7 + seed) % hrows) * 8 + l;
        if (MODE == 0) *d = pool[(u % 200000) * 8 + l];
        else { float4 y = __ldcv(d); if (y.x == 12345.f) host[0] = y; }
    }
}
int main() {
    const int64_t hrows = 33762577; const size_t bytes = hrows * 128;
    float4 *a, *b, *pool; const int64_t n4 = (256 << 20) / 16;
    CK(cudaMalloc(&a, n4 * 16)); CK(cudaMalloc(&b, n4 * 16)); CK(cudaMalloc(&pool, 200000 * 128));
    cudaStream_t s1, s2; cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t e0, e1, f0, f1; cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventCreate(&f0); cudaEventCreate(&f1);
    float alone = 0, ms;
    for (int rep = 0; rep < 5; rep++) {
        cudaEventRecord(e0, s1); v_copy<<<1184, 256, 0, s1>>>(a, b, n4); cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
        cudaEventElapsedTime(&ms, e0, e1); if (rep >= 1) alone += ms / 4;
    }
    printf("victim V1 copy 256MB alone %.3f ms\n", alone);
    for (int var = 0; var < 4; var++) {
        void* h = nullptr; float4* hd = nullptr; const char* nm = "?";
        if (var == 0) { nm = "cudaHostAlloc"; CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped)); memset(h, 0, bytes); CK(cudaHostGetDevicePointer((void**)&hd, h, 0)); }
        if (var == 1) {
            nm = "VMM HOST_NUMA 2MB";
            CUmemAllocationProp prop = {}; prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
            prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; prop.location.id = 0;
            size_t gran = 0; cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
            size_t tot = (bytes + gran - 1) / gran * gran; CUmemGenericAllocationHandle hd_;
            if (cuMemCreate(&hd_, tot, &prop, 0) != CUDA_SUCCESS) { printf("%s: cuMemCreate failed\n", nm); continue; }
            CUdeviceptr va; cuMemAddressReserve(&va, tot, 1ull << 30, 0, 0); cuMemMap(va, tot, 0, hd_, 0);
            CUmemAccessDesc acc[2] = {};
            acc[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; acc[0].location.id = 0; acc[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
            acc[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; acc[1].location.id = 0; acc[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
            if (cuMemSetAccess(va, tot, acc, 2) != CUDA_SUCCESS) { printf("%s: setaccess failed\n", nm); continue; }
            hd = (float4*)va; CK(cudaMemset(hd, 0, bytes)); printf("%s granularity %zu\n", nm, gran);
        }
        if (var == 2) {
            nm = "hugetlbfs 2MB+register";
            size_t tot = (bytes + (2 << 20) - 1) / (2 << 20) * (2 << 20);
            h = mmap(0, tot, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS | MAP_HUGETLB | MAP_HUGE_2MB, -1, 0);
            if (h == MAP_FAILED) { printf("%s: mmap failed (no hugepages reserved?)\n", nm); continue; }
            memset(h, 0, bytes);
            CK(cudaHostRegister(h, tot, cudaHostRegisterMapped)); CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
        }
        if (var == 3) {
            nm = "shm THP+register";
            shm_unlink("/ifp2"); int fd = shm_open("/ifp2", O_CREAT | O_RDWR, 0600);
            size_t tot = (bytes + (2 << 20) - 1) / (2 << 20) * (2 << 20);
            if (fd < 0 || ftruncate(fd, tot)) { printf("shm failed\n"); continue; }
            h = mmap(0, tot, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0); madvise(h, tot, MADV_HUGEPAGE); memset(h, 0, bytes);
            CK(cudaHostRegister(h, tot, cudaHostRegisterMapped)); CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
        }
        for (int64_t fp_rows : {hrows, (int64_t)(1 << 23), (int64_t)(1 << 21), (int64_t)(1 << 19)})
        for (int mode = 0; mode < 2; mode++)
            for (int G : {20, 74}) {
                auto aggr = [&](int64_t n) {
                    if (mode == 0) agg<0><<<G, 256, 0, s2>>>(pool, hd, fp_rows, n, 3);
                    else agg<1><<<G, 256, 0, s2>>>(pool, hd, fp_rows, n, 3);
                };
                cudaEventRecord(f0, s2); aggr(30000); cudaEventRecord(f1, s2); CK(cudaEventSynchronize(f1));
                float am; cudaEventElapsedTime(&am, f0, f1);
                float tv = 0;
                for (int rep = 0; rep < 3; rep++) {
                    aggr(400000);
                    cudaEventRecord(e0, s1); v_copy<<<1184, 256, 0, s1>>>(a, b, n4); cudaEventRecord(e1, s1);
                    CK(cudaDeviceSynchronize()); cudaEventElapsedTime(&ms, e0, e1); tv += ms / 3;
                }
                printf("%-24s footprint %6lld MB %-6s G=%3d  aggressor alone %5.1f GB/s   victim %.3f ms (x%.2f)\n", nm,
                       (long long)(fp_rows * 128 >> 20), mode ? "reads" : "writes", G, 30000 * 128 / (am * 1e6), tv, tv / alone);
            }
        fflush(stdout);
    }
    return 0;
}
