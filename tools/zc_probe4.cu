// zc_probe4.cu -- random 128-B row gather from host-mapped memory with (a) plain loads,
// (b) cp.async 16 B (LDGSTS) staged in shared memory, (c) cp.async.bulk 1-D TMA copies
// (128 B per row) completing on an mbarrier.  Small grids: how many SMs does it take to
// fill the link?  Fresh random rows every iteration (cold).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__global__ void g_plain(const int32_t* idx, int n, const float4* h, float4* out) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    int l = threadIdx.x & 7;
    for (int64_t u = t / 8; u < n; u += gs) out[u * 8 + l] = h[(int64_t)idx[u] * 8 + l];
}
// cp.async: each group of 8 lanes owns ROWS rows in flight (smem ring), then copies out
template <int ROWS>
__global__ void g_cpasync(const int32_t* idx, int n, const float4* h, float4* out) {
    extern __shared__ float4 sm[];  // [ROWS][blockDim]
    const int t = threadIdx.x, l = t & 7;
    const int64_t gid = (blockIdx.x * (int64_t)blockDim.x + t) / 8, gs = ((int64_t)gridDim.x * blockDim.x) / 8;
    for (int64_t base = gid; base < n; base += gs * ROWS) {
#pragma unroll
        for (int r = 0; r < ROWS; r++) {
            int64_t u = base + r * gs;
            if (u < n) {
                unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[r * blockDim.x + t]);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(h + (int64_t)idx[u] * 8 + l) : "memory");
            }
        }
        asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
#pragma unroll
        for (int r = 0; r < ROWS; r++) {
            int64_t u = base + r * gs;
            if (u < n) out[u * 8 + l] = sm[r * blockDim.x + t];
        }
    }
}
// TMA 1-D bulk copies: one thread per row issues a 128-B bulk copy into smem, all
// complete on one mbarrier per batch; then the block writes the rows out
template <int BATCH>
__global__ void g_bulk(const int32_t* idx, int n, const float4* h, float4* out) {
    extern __shared__ float4 sm[];  // [BATCH][8]
    __shared__ __align__(8) uint64_t bar;
    const int t = threadIdx.x;
    unsigned bar_a = (unsigned)__cvta_generic_to_shared(&bar);
    if (t == 0) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bar_a));
    __syncthreads();
    unsigned phase = 0;
    for (int64_t b0 = (int64_t)blockIdx.x * BATCH; b0 < n; b0 += (int64_t)gridDim.x * BATCH) {
        const int cnt = (int)min((int64_t)BATCH, n - b0);
        if (t == 0) asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar_a), "r"(cnt * 128) : "memory");
        __syncthreads();
        for (int r = t; r < cnt; r += blockDim.x) {
            unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[r * 8]);
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 128, [%2];"
                         ::"r"(sa), "l"(h + (int64_t)idx[b0 + r] * 8), "r"(bar_a) : "memory");
        }
        // wait for the phase
        asm volatile("{\n.reg .pred p;\nWAIT_%=:\nmbarrier.try_wait.parity.shared.b64 p, [%0], %1;\n@!p bra WAIT_%=;\n}"
                     ::"r"(bar_a), "r"(phase) : "memory");
        phase ^= 1;
        for (int e = t; e < cnt * 8; e += blockDim.x) out[(b0 + e / 8) * 8 + (e & 7)] = sm[e];
        __syncthreads();
    }
}

int main() {
    const int64_t N = 33762577; const size_t bytes = (size_t)N * 128; const int n = 41000, IT = 6;
    int32_t* hidx = (int32_t*)malloc((size_t)IT * n * 4);
    srand(11);
    for (size_t i = 0; i < (size_t)IT * n; i++) hidx[i] = (int32_t)(((int64_t)rand() * RAND_MAX + rand()) % N);
    int32_t* didx; float4* out; CK(cudaMalloc(&didx, (size_t)IT * n * 4)); CK(cudaMalloc(&out, (size_t)n * 128));
    cudaMemcpy(didx, hidx, (size_t)IT * n * 4, cudaMemcpyHostToDevice);
    void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); memset(h, 1, bytes);
    CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
    float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
    CK(cudaFuncSetAttribute(g_cpasync<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 256 * 16));
    CK(cudaFuncSetAttribute(g_bulk<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, 1024 * 128));
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](const char* name, auto launch, bool warm) {
        float tot = 0;
        for (int it = 0; it < IT; it++) {
            const int32_t* ix = didx + (size_t)(warm ? 0 : it) * n;
            cudaEventRecord(a); launch(ix); cudaEventRecord(b); CK(cudaEventSynchronize(b));
            float ms; cudaEventElapsedTime(&ms, a, b); if (it) tot += ms;
        }
        float ms = tot / (IT - 1);
        printf("%-34s %s %.3f ms %5.1f GB/s\n", name, warm ? "warm" : "cold", ms, n * 128.0 / ms / 1e6);
    };
    for (int warm = 0; warm < 2; warm++) {
        for (int g : {16, 32, 74, 148, 296}) {
            char nm[64];
            snprintf(nm, 64, "plain  grid=%d", g); run(nm, [&](const int32_t* ix) { g_plain<<<g, 256>>>(ix, n, dh, out); }, warm);
            snprintf(nm, 64, "cp.async16x16 grid=%d", g); run(nm, [&](const int32_t* ix) { g_cpasync<16><<<g, 256, 16 * 256 * 16>>>(ix, n, dh, out); }, warm);
            snprintf(nm, 64, "bulk(TMA) 1024/batch grid=%d", g); run(nm, [&](const int32_t* ix) { g_bulk<1024><<<g, 256, 1024 * 128>>>(ix, n, dh, out); }, warm);
        }
    }
    // correctness of the bulk path
    g_bulk<1024><<<32, 256, 1024 * 128>>>(didx, n, dh, out); CK(cudaDeviceSynchronize());
    float4* ho = (float4*)malloc((size_t)n * 128); cudaMemcpy(ho, out, (size_t)n * 128, cudaMemcpyDeviceToHost);
    int bad = 0; for (int i = 0; i < n * 8; i++) { float4 v = ho[i]; const float4 r = ((float4*)h)[(int64_t)hidx[i / 8] * 8 + (i & 7)]; if (memcmp(&v, &r, 16)) bad++; }
    printf("bulk correctness: %d mismatches\n", bad);
    return 0;
}
