// layout_probe2.cu -- why do the library's exact host-row lists (tools/dump_lists.py) replay
// slower than simulated ones?  Same kernels as zc_probe7; factors: allocation (cudaHostAlloc vs
// mmap+memset+cudaHostRegister), per-step order (urgent -> reads -> drain vs flush -> reads),
// list source (exact tools/lay vs simulated tools/lay2).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <vector>
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
// HBM state touched like one step of the library: n random 128-B row RMWs over a big device
// array (Adagrad G / cache / pool) -- does it slow the next zero-copy host gather?
__global__ void g_noise(float4* big, int64_t rows, int n, uint64_t seed) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) {
        uint64_t x = (u + 1) * 0x9E3779B97F4A7C15ull ^ seed; x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29;
        float4* p = big + (int64_t)(x % rows) * 8 + l;
        float4 v = *p; v.x += 1.f; *p = v;
    }
}
typedef std::vector<std::vector<int32_t>> Lists;
static Lists load(const char* p) {
    FILE* f = fopen(p, "rb"); if (!f) { printf("no %s\n", p); exit(1); }
    Lists r; int32_t n;
    while (fread(&n, 4, 1, f) == 1) { std::vector<int32_t> a(n); if (fread(a.data(), 4, n, f) != (size_t)n) exit(2); r.push_back(a); }
    fclose(f); return r;
}
int main() {
    const int64_t N = 33762577; const size_t bytes = (size_t)N * 128;
    float4 *hA, *hB, *dA, *dB;
    CK(cudaHostAlloc(&hA, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(hA, 1, bytes);
    CK(cudaHostGetDevicePointer(&dA, hA, 0));
    hB = (float4*)mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0);
    memset(hB, 1, bytes);
    CK(cudaHostRegister(hB, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
    CK(cudaHostGetDevicePointer(&dB, hB, 0));
    float4* buf; CK(cudaMalloc(&buf, 64 << 20));
    int32_t* didx; CK(cudaMalloc(&didx, 3 * (4 << 20) * 4));
    Lists ex_u = load("tools/lay/urgent.i32"), ex_r = load("tools/lay/reads.i32"), ex_d = load("tools/lay/drain.i32");
    Lists fx_u = load("tools/lay/urgent_freq.i32"), fx_r = load("tools/lay/reads_freq.i32"), fx_d = load("tools/lay/drain_freq.i32");
    Lists empty(ex_r.size());
    Lists ex_f(ex_r.size());
    for (size_t s = 0; s < ex_r.size(); s++) { ex_f[s] = ex_u[s]; ex_f[s].insert(ex_f[s].end(), ex_d[s].begin(), ex_d[s].end()); }
    struct Case { const char* nm; Lists *a, *b, *c; };
    Case cases[] = {{"exact urgent>reads>drain", &ex_u, &ex_r, &ex_d}, {"exact flushall>reads", &ex_f, &ex_r, &empty},
                    {"exact reads only", &empty, &ex_r, &empty}, {"freq urgent>reads>drain", &fx_u, &fx_r, &fx_d},
                    {"freq reads only", &empty, &fx_r, &empty}};
    cudaEvent_t ev[4]; for (auto& x : ev) cudaEventCreate(&x);
    const int64_t big_rows = (5ll << 30) / 128;
    float4* big; CK(cudaMalloc(&big, big_rows * 128)); CK(cudaMemset(big, 0, big_rows * 128));
    for (int noise : {0, 65000, 200000})
    for (int alloc = 0; alloc < 1; alloc++)
    for (auto& cs : cases) {
        float4* dh = alloc ? dB : dA;
        double t[3] = {0, 0, 0}, nr[3] = {0, 0, 0}; int cnt = 0;
        size_t S = std::min(cs.b->size(), (size_t)100);
        for (size_t s = 0; s < S; s++) {
            Lists* L3[3] = {cs.a, cs.b, cs.c};
            for (int k = 0; k < 3; k++) if ((*L3[k])[s].size()) CK(cudaMemcpy(didx + (size_t)k * (4 << 20), (*L3[k])[s].data(), (*L3[k])[s].size() * 4, cudaMemcpyHostToDevice));
            if (noise) g_noise<<<1184, 256>>>(big, big_rows, noise, s * 7919);
            cudaEventRecord(ev[0]);
            if ((*L3[0])[s].size()) g_scatter<<<74, 256>>>(didx, (int)(*L3[0])[s].size(), dh, buf);
            cudaEventRecord(ev[1]);
            g_gather<<<74, 256>>>(didx + (4 << 20), (int)(*L3[1])[s].size(), dh, buf);
            cudaEventRecord(ev[2]);
            if ((*L3[2])[s].size()) g_scatter<<<74, 256>>>(didx + (8 << 20), (int)(*L3[2])[s].size(), dh, buf);
            cudaEventRecord(ev[3]); CK(cudaEventSynchronize(ev[3]));
            if (s >= 60) {
                for (int k = 0; k < 3; k++) { float ms; cudaEventElapsedTime(&ms, ev[k], ev[k + 1]); t[k] += ms; nr[k] += (*L3[k])[s].size(); }
                cnt++;
            }
        }
        printf("noise %6d %-14s %-26s", noise, alloc ? "mmap+register" : "cudaHostAlloc", cs.nm);
        const char* nm[3] = {"first", "reads", "last"};
        for (int k = 0; k < 3; k++) printf("  %s %6.0f rows %.3f ms %5.1f GB/s", nm[k], nr[k] / cnt, t[k] / cnt, t[k] > 0 ? nr[k] * 128 / (t[k] * 1e6) : 0.0);
        printf("\n");
    }
    return 0;
}
