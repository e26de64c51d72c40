// zc_probe6.cu -- does the host-link random-row cliff (zc_probe5: 40-47 GB/s up to 512 MB
// footprint, 11 GB/s over 4 GB) move when the host table is a CUDA VMM host allocation
// (cuMemCreate, location HOST / HOST_NUMA, 2 MB+ granularity) instead of cudaHostRegister'd
// mmap?  If the limit is the GPU-side translation reach, VMM mappings with large pages lift
// it; if it is the IOMMU / hypervisor, nothing changes.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
#define CU(x) do { CUresult e = (x); if (e != CUDA_SUCCESS) { const char* s; cuGetErrorString(e, &s); printf("%s: %s\n", #x, s); return false; } } while (0)

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
__global__ void g_fill(float4* h, int64_t n4) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        h[i] = make_float4(1.f, 2.f, 3.f, (float)(i & 1023));
}
static uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull; x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull; return x ^ (x >> 31);
}
static const int64_t N = 33762577;
static const int n = 41000, IT = 8;

static void sweep(const char* name, float4* dh, int32_t* hidx, int32_t* didx, float4* out) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int64_t foot : {(int64_t)32 << 20, (int64_t)512 << 20, (int64_t)1024 << 20, (int64_t)2048 << 20, N * 128}) {
        int64_t rows = foot / 128; if (rows > N) rows = N;
        for (int op = 0; op < 2; op++) {
            uint64_t seed = 77 + foot + op;
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
            printf("%-22s footprint %7.0f MB %-7s %.3f ms %5.1f GB/s\n", name, foot / 1048576.0, op ? "scatter" : "gather",
                   ms, n * 128.0 / ms / 1e6);
            fflush(stdout);
        }
    }
}

static bool vmm(int loc_type, const char* name, int32_t* hidx, int32_t* didx, float4* out) {
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = (CUmemLocationType)loc_type;
    prop.location.id = 0;
    prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t gran = 0;
    CU(cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
    size_t bytes = ((size_t)N * 128 + gran - 1) / gran * gran;
    printf("%s: granularity %zu\n", name, gran);
    CUmemGenericAllocationHandle hd;
    CU(cuMemCreate(&hd, bytes, &prop, 0));
    CUdeviceptr va;
    CU(cuMemAddressReserve(&va, bytes, 0, 0, 0));
    CU(cuMemMap(va, bytes, 0, hd, 0));
    CUmemAccessDesc acc[2] = {};
    acc[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; acc[0].location.id = 0; acc[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    acc[1].location.type = (CUmemLocationType)loc_type; acc[1].location.id = 0; acc[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CU(cuMemSetAccess(va, bytes, acc, 2));
    // host access through the same VA?
    float* hp = (float*)va;
    hp[0] = 1.f; hp[bytes / 4 - 1] = 2.f;  // segfaults if not host-accessible
    printf("%s: host access ok (%f)\n", name, hp[0]);
    g_fill<<<1184, 256>>>((float4*)va, (int64_t)N * 8);
    CK(cudaDeviceSynchronize());
    printf("%s: host reads device fill: %f %f\n", name, hp[3], hp[7]);
    int fd = -1;
    CUresult r = cuMemExportToShareableHandle(&fd, hd, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0);
    printf("%s: export fd -> %d (%d)\n", name, fd, (int)r);
    sweep(name, (float4*)va, hidx, didx, out);
    cuMemUnmap(va, bytes); cuMemAddressFree(va, bytes); cuMemRelease(hd);
    return true;
}

int main() {
    CK(cudaSetDevice(0)); CK(cudaFree(0));
    int32_t* hidx = (int32_t*)malloc((size_t)IT * n * 4);
    int32_t* didx; float4* out; CK(cudaMalloc(&didx, (size_t)IT * n * 4)); CK(cudaMalloc(&out, (size_t)n * 128));
    CK(cudaMemset(out, 0, (size_t)n * 128));
    CUdevice dev; cuDeviceGet(&dev, 0);
    int s1 = 0, s2 = 0;
    cuDeviceGetAttribute(&s1, CU_DEVICE_ATTRIBUTE_HOST_NUMA_VIRTUAL_MEMORY_MANAGEMENT_SUPPORTED, dev);
    cuDeviceGetAttribute(&s2, CU_DEVICE_ATTRIBUTE_VIRTUAL_MEMORY_MANAGEMENT_SUPPORTED, dev);
    printf("VMM %d HOST_NUMA VMM %d\n", s2, s1);
    if (!vmm(CU_MEM_LOCATION_TYPE_HOST_NUMA, "vmm HOST_NUMA", hidx, didx, out)) printf("HOST_NUMA failed\n");
    if (!vmm(CU_MEM_LOCATION_TYPE_HOST, "vmm HOST", hidx, didx, out)) printf("HOST failed\n");
    {   // baseline: registered mmap
        size_t bytes = (size_t)N * 128;
        void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); memset(h, 1, bytes);
        CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
        float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
        sweep("registered mmap", dh, hidx, didx, out);
    }
    {   // cudaMallocHost
        void* h; CK(cudaMallocHost(&h, (size_t)N * 128)); memset(h, 1, (size_t)N * 128);
        sweep("cudaMallocHost", (float4*)h, hidx, didx, out);
    }
    return 0;
}
