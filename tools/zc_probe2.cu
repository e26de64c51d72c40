// zc_probe2.cu -- does a zero-copy random-row gather (H2D) slow a concurrent zero-copy
// random-row scatter (D2H) on another stream?  Also the copy-engine sequential rates.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
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
int main() {
    const int64_t N = 33762577; const size_t bytes = (size_t)N * 128;
    const int n = 41000;
    int32_t *hi = (int32_t*)malloc(n * 4), *hj = (int32_t*)malloc(n * 4);
    srand(1);
    for (int i = 0; i < n; i++) { hi[i] = (int32_t)(((int64_t)rand() * RAND_MAX + rand()) % N); hj[i] = (int32_t)(((int64_t)rand() * RAND_MAX + rand()) % N); }
    int32_t *di, *dj; float4 *o1, *o2;
    CK(cudaMalloc(&di, n * 4)); CK(cudaMalloc(&dj, n * 4)); CK(cudaMalloc(&o1, n * 128)); CK(cudaMalloc(&o2, n * 128));
    cudaMemcpy(di, hi, n * 4, cudaMemcpyHostToDevice); cudaMemcpy(dj, hj, n * 4, cudaMemcpyHostToDevice);
    void* h = mmap(0, bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0); memset(h, 0, bytes);
    CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
    float4* dh; CK(cudaHostGetDevicePointer((void**)&dh, h, 0));
    cudaStream_t s1, s2; cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto timeit = [&](const char* name, auto fn) {
        float best = 1e9;
        for (int it = 0; it < 7; it++) { cudaDeviceSynchronize(); cudaEventRecord(a, s1); fn(); cudaEventRecord(b, s1); cudaStreamWaitEvent(s1, b, 0); cudaDeviceSynchronize(); float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms; }
        printf("%-40s %.3f ms\n", name, best);
    };
    cudaEvent_t j; cudaEventCreateWithFlags(&j, cudaEventDisableTiming);
    timeit("gather alone (592 blk)", [&] { gather<<<592, 256, 0, s1>>>(di, n, dh, o1); });
    timeit("scatter alone (592 blk)", [&] { scatter<<<592, 256, 0, s1>>>(dj, n, dh, o2); });
    timeit("scatter alone (32 blk)", [&] { scatter<<<32, 256, 0, s1>>>(dj, n, dh, o2); });
    timeit("gather||scatter(592/592)", [&] { cudaEventRecord(j, s1); cudaStreamWaitEvent(s2, j, 0); gather<<<592, 256, 0, s1>>>(di, n, dh, o1); scatter<<<592, 256, 0, s2>>>(dj, n, dh, o2); cudaEventRecord(j, s2); cudaStreamWaitEvent(s1, j, 0); });
    timeit("gather||scatter(592/32)", [&] { cudaEventRecord(j, s1); cudaStreamWaitEvent(s2, j, 0); gather<<<592, 256, 0, s1>>>(di, n, dh, o1); scatter<<<32, 256, 0, s2>>>(dj, n, dh, o2); cudaEventRecord(j, s2); cudaStreamWaitEvent(s1, j, 0); });
    timeit("gather then scatter (serial)", [&] { gather<<<592, 256, 0, s1>>>(di, n, dh, o1); scatter<<<592, 256, 0, s1>>>(dj, n, dh, o2); });
    // copy engines: sequential 5.25 MB each way
    char *dbuf; CK(cudaMalloc(&dbuf, 16 << 20)); char* pin; CK(cudaHostAlloc(&pin, 16 << 20, 0));
    timeit("CE H2D 5.25MB", [&] { cudaMemcpyAsync(dbuf, pin, n * 128, cudaMemcpyHostToDevice, s1); });
    timeit("CE D2H 5.25MB", [&] { cudaMemcpyAsync(pin, dbuf, n * 128, cudaMemcpyDeviceToHost, s1); });
    timeit("gather || CE D2H 5.25MB", [&] { cudaEventRecord(j, s1); cudaStreamWaitEvent(s2, j, 0); gather<<<592, 256, 0, s1>>>(di, n, dh, o1); cudaMemcpyAsync(pin, dbuf, n * 128, cudaMemcpyDeviceToHost, s2); cudaEventRecord(j, s2); cudaStreamWaitEvent(s1, j, 0); });
    return 0;
}
