// zc_probe7.cu -- replay of a Criteo-Kaggle step's host traffic (n=1): per step, the
// urgent+deferred flush set (all cold rows updated, zero-copy scatter) then the gather's
// host-read set (cold rows not in the pool window), for 40 consecutive steps, with the
// host table in id order vs in frequency order (tools/lay/*.i32 written by a numpy sim).
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <vector>
#include <fcntl.h>
#include <unistd.h>
#include <linux/mman.h>
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
static std::vector<std::vector<int32_t>> load(const char* p) {
    FILE* f = fopen(p, "rb"); if (!f) { printf("no %s\n", p); exit(1); }
    std::vector<int32_t> a; int32_t v; while (fread(&v, 4, 1, f) == 1) a.push_back(v); fclose(f);
    std::vector<std::vector<int32_t>> r; size_t i = 0;
    while (i < a.size()) { int n = a[i++]; r.emplace_back(a.begin() + i, a.begin() + i + n); i += n; }
    return r;
}
// HBM noise like the optimizer/segred between two steps: n random row RMWs over a big
// device array (Adagrad G is 4.3 GB at Criteo-Kaggle)
__global__ void g_noise(float4* big, int64_t rows, int n, uint64_t seed) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) {
        uint64_t x = (u + 1) * 0x9E3779B97F4A7C15ull ^ seed; x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29;
        int64_t r = (int64_t)(x % (uint64_t)rows);
        float4 v = big[r * 8 + l]; v.x += 1.f; big[r * 8 + l] = v;
    }
}
__global__ void g_init(float4* h, int64_t n4) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        h[i] = make_float4(1.f, 2.f, 3.f, 4.f);
}
int main(int argc, char** argv) {
    const int64_t N = 33762577; const size_t bytes = (size_t)N * 128;
    const int variant = argc > 1 ? atoi(argv[1]) : 0;
    size_t total = variant == 5 ? 2 * bytes + (4 << 20) : bytes;
    if (variant == 4) total = (total + (1ull << 30) - 1) >> 30 << 30;
    if (variant == 3) total = (total + (2 << 20) - 1) / (2 << 20) * (2 << 20);
    void* h = nullptr;
    const char* vname = "?";
    if (variant == 0) { vname = "anon+memset"; h = mmap(0, total, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); memset(h, 1, total); }
    if (variant == 1 || variant == 2 || variant == 5) {
        vname = variant == 1 ? "shm+THP, GPU init" : variant == 2 ? "shm+THP+memset" : "shm+THP w+G (8.6GB), GPU init";
        shm_unlink("/zcp7"); int fd = shm_open("/zcp7", O_CREAT | O_RDWR, 0600);
        if (fd < 0 || ftruncate(fd, total)) { printf("shm failed\n"); return 1; }
        h = mmap(0, total, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0); madvise(h, total, MADV_HUGEPAGE);
        if (variant == 2) memset(h, 1, total);
    }
    size_t off_w = 0;
    if (variant == 6) {  // as libfrugal: shm w+G with a header, THP advice, interleave, GPU init
        vname = "libfrugal-like shm (hdr + w + G)";
        off_w = 2 << 20;
        total = off_w + ((bytes + (2 << 20) - 1) / (2 << 20) * (2 << 20)) + bytes;
        shm_unlink("/zcp7"); int fd = shm_open("/zcp7", O_CREAT | O_EXCL | O_RDWR, 0600);
        if (fd < 0 || ftruncate(fd, total)) { printf("shm failed\n"); return 1; }
        h = mmap(0, total, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0); madvise(h, total, MADV_HUGEPAGE);
    }
    if (variant == 7) {  // CUDA VMM host allocation: 2 MB GPU mappings of host memory
        vname = "VMM cuMemCreate HOST_NUMA 2MB";
        CK(cudaFree(0));
        CUmemAllocationProp prop = {};
        prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
        prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
        prop.location.id = 0;
        size_t gran = 0;
        cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
        total = (bytes + gran - 1) / gran * gran;
        CUmemGenericAllocationHandle hd;
        if (cuMemCreate(&hd, total, &prop, 0) != CUDA_SUCCESS) { printf("cuMemCreate failed\n"); return 1; }
        CUdeviceptr va;
        cuMemAddressReserve(&va, total, 0, 0, 0);
        cuMemMap(va, total, 0, hd, 0);
        CUmemAccessDesc acc[2] = {};
        acc[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; acc[0].location.id = 0; acc[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        acc[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; acc[1].location.id = 0; acc[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        cuMemSetAccess(va, total, acc, 2);
        h = (void*)va;
    }
    if (variant == 3) { vname = "hugetlb 2M"; h = mmap(0, total, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS | MAP_HUGETLB | MAP_HUGE_2MB, -1, 0); }
    if (variant == 4) { vname = "hugetlb 1G"; h = mmap(0, total, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS | MAP_HUGETLB | MAP_HUGE_1GB, -1, 0); }
    if (h == MAP_FAILED || !h) { printf("variant %d (%s): mmap failed\n", variant, vname); return 0; }
    float4* dh = (float4*)h;
    if (variant != 7) {
        CK(cudaHostRegister(h, total, cudaHostRegisterMapped | cudaHostRegisterPortable));
        CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
    }
    if (variant != 0 && variant != 2) { g_init<<<1184, 256>>>(dh, (int64_t)(total / 16)); CK(cudaDeviceSynchronize()); }
    dh = (float4*)((char*)dh + off_w);
    float4* big = nullptr;
    const int noise = getenv("PROBE_HBM_NOISE") ? atoi(getenv("PROBE_HBM_NOISE")) : 0;
    if (noise) { CK(cudaMalloc(&big, bytes)); CK(cudaMemset(big, 0, bytes)); }
    printf("variant %d: %s\n", variant, vname);
    float4* buf; CK(cudaMalloc(&buf, 64 << 20)); CK(cudaMemset(buf, 0, 64 << 20));
    int32_t* didx; CK(cudaMalloc(&didx, 64 << 20));
    cudaEvent_t ev[3]; for (auto& x : ev) cudaEventCreate(&x);
    auto ur = load("tools/lay/urgent.i32"), rd = load("tools/lay/reads.i32"), dr = load("tools/lay/drain.i32");
    const int G = argc > 2 ? atoi(argv[2]) : 148;
    double t[3] = {0, 0, 0}, nr[3] = {0, 0, 0}; int cnt = 0;
    for (size_t s = 0; s < rd.size() && s < ur.size() && s < dr.size(); s++) {
        std::vector<int32_t>* L3[3] = {&ur[s], &rd[s], &dr[s]};
        for (int k = 0; k < 3; k++) CK(cudaMemcpy(didx + (size_t)k * (4 << 20), L3[k]->data(), L3[k]->size() * 4, cudaMemcpyHostToDevice));
        cudaEvent_t ev[4]; for (auto& x : ev) cudaEventCreate(&x);
        if (noise) g_noise<<<1184, 256>>>(big, N, noise, s * 7919);
        cudaEventRecord(ev[0]);
        g_scatter<<<G, 256>>>(didx, (int)ur[s].size(), dh, buf);
        cudaEventRecord(ev[1]);
        g_gather<<<G, 256>>>(didx + (4 << 20), (int)rd[s].size(), dh, buf);
        cudaEventRecord(ev[2]);
        g_scatter<<<G, 256>>>(didx + (8 << 20), (int)dr[s].size(), dh, buf);
        cudaEventRecord(ev[3]); CK(cudaEventSynchronize(ev[3]));
        if (s >= 60) {
            for (int k = 0; k < 3; k++) { float ms; cudaEventElapsedTime(&ms, ev[k], ev[k + 1]); t[k] += ms; nr[k] += L3[k]->size(); }
            cnt++;
        }
        for (auto& x : ev) cudaEventDestroy(x);
    }
    const char* nm[3] = {"urgent", "reads", "drain"};
    for (int k = 0; k < 3; k++)
        printf("grid %d  %-7s %7.0f rows/step %.3f ms %5.1f GB/s\n", G, nm[k], nr[k] / cnt, t[k] / cnt, nr[k] * 128 / (t[k] * 1e6));
    return 0;
}
