// kernels_kg.cu -- KG glue: TransE-L2 with chunked shared negatives (R26; PAPER.md
// §4.1).  Not the library proper: it turns looked-up rows into
// gradients so the KG workload (BASELINE.json configs[3]) runs through the hot path.
// All arithmetic in fp64 with explicitly rounded ops in the order the definition is
// written (sums over k, j, b ascending), gradients rounded to fp32 once.
#include <cuda_runtime.h>
#include <stdint.h>

#include "frugal_internal.cuh"
#include "kutil.cuh"

namespace frugal {

__device__ __forceinline__ double sigm(double x) { return 1.0 / (1.0 + exp(-x)); }
__device__ __forceinline__ double softplus(double x) { return x > 0 ? x + log1p(exp(-x)) : log1p(exp(x)); }

// pass 1: one thread per (b, j) pair of a chunk (j == -1 encodes the positive (h, r, t)):
// distance, weight W[b][j] = sigma(score)/dist/nC  (positive: a_b = (1 - sigma)/dist), loss
__global__ void k_transe_pairs(const float* __restrict__ emb, int count, int C, int d, double gamma,
                               double* __restrict__ Wm, double* __restrict__ A, double* loss, double nb) {
    const int nchunks = (count + C - 1) / C;
    const int64_t total = (int64_t)nchunks * C * (C + 1);
    double lsum = 0.0;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int c = (int)(e / ((int64_t)C * (C + 1)));
        const int rem = (int)(e - (int64_t)c * C * (C + 1));
        const int bl = rem / (C + 1), jl = rem - bl * (C + 1) - 1;
        const int b0 = c * C, nC = min(C, count - b0);
        if (bl >= nC || jl >= nC) continue;
        const int b = b0 + bl;
        const float* h = emb + ((int64_t)b * 4 + 0) * d;
        const float* r = emb + ((int64_t)b * 4 + 1) * d;
        const float* x = jl < 0 ? emb + ((int64_t)b * 4 + 2) * d : emb + ((int64_t)(b0 + jl) * 4 + 3) * d;
        double acc = 0.0;
        for (int k = 0; k < d; k++) {
            const double P = __dadd_rn((double)h[k], (double)r[k]);
            const double u = __dsub_rn(P, (double)x[k]);
            acc = __dadd_rn(acc, __dmul_rn(u, u));
        }
        const double dist = __dsqrt_rn(acc);
        const double sc = __dsub_rn(gamma, dist);
        if (jl < 0) {
            lsum += softplus(-sc);
            A[b] = dist > 0.0 ? __ddiv_rn(__dsub_rn(1.0, sigm(sc)), dist) : 0.0;
        } else {
            lsum += __ddiv_rn(softplus(sc), (double)nC);
            Wm[(int64_t)b * C + jl] = dist > 0.0 ? __ddiv_rn(__ddiv_rn(sigm(sc), dist), (double)nC) : 0.0;
        }
    }
    // block-reduce the loss, one atomic per block
    __shared__ double sl[32];
    for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(FULL, lsum, o);
    if ((threadIdx.x & 31) == 0) sl[threadIdx.x >> 5] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int i = 0; i < (int)(blockDim.x >> 5); i++) t += sl[i];
        if (t != 0.0) atomicAdd(loss, t / nb);
    }
}

// pass 2: one thread per (b, k): gh = a_b v - sum_j W[b][j] (P_b - n_j) (j ascending) for h and
// r, gt = -a_b v; and one thread per (j, k): gn = sum_b W[b][j] (P_b - n_j) (b ascending)
__global__ void k_transe_grads(const float* __restrict__ emb, int count, int C, int d, const double* __restrict__ Wm,
                               const double* __restrict__ A, float* __restrict__ grad, double nb) {
    const int64_t total = (int64_t)count * d;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < 2 * total; e += (int64_t)gridDim.x * blockDim.x) {
        const bool neg = e >= total;
        const int64_t e2 = neg ? e - total : e;
        const int b = (int)(e2 / d), k = (int)(e2 - (int64_t)b * d);
        const int b0 = (b / C) * C, nC = min(C, count - b0);
        if (!neg) {
            const double P = __dadd_rn((double)emb[((int64_t)b * 4 + 0) * d + k], (double)emb[((int64_t)b * 4 + 1) * d + k]);
            const double v = __dsub_rn(P, (double)emb[((int64_t)b * 4 + 2) * d + k]);
            const double a = A[b];
            double gh = __dmul_rn(a, v);
            for (int jl = 0; jl < nC; jl++) {
                const double u = __dsub_rn(P, (double)emb[((int64_t)(b0 + jl) * 4 + 3) * d + k]);
                gh = __dsub_rn(gh, __dmul_rn(Wm[(int64_t)b * C + jl], u));
            }
            const float g = (float)__ddiv_rn(gh, nb);
            grad[((int64_t)b * 4 + 0) * d + k] = g;
            grad[((int64_t)b * 4 + 1) * d + k] = g;
            grad[((int64_t)b * 4 + 2) * d + k] = (float)__ddiv_rn(-__dmul_rn(a, v), nb);
        } else {
            const int j = b;  // this thread owns negative j of its chunk
            const double nk = (double)emb[((int64_t)j * 4 + 3) * d + k];
            double gn = 0.0;
            for (int bl = 0; bl < nC; bl++) {
                const int bb = b0 + bl;
                const double P = __dadd_rn((double)emb[((int64_t)bb * 4 + 0) * d + k],
                                           (double)emb[((int64_t)bb * 4 + 1) * d + k]);
                gn = __dadd_rn(gn, __dmul_rn(Wm[(int64_t)bb * C + (j - b0)], __dsub_rn(P, nk)));
            }
            grad[((int64_t)j * 4 + 3) * d + k] = (float)__ddiv_rn(gn, nb);
        }
    }
}

void launch_transe_model(frugal_ctx* c, QueueSlot& q, const float* emb, int C, double gamma, float* grad,
                         double* loss, int64_t nb, double* Wm, double* A, cudaStream_t st) {
    const int count = q.h_counts[c->g];
    if (count <= 0) return;
    const int nchunks = (count + C - 1) / C;
    k_transe_pairs<<<grid_for((int64_t)nchunks * C * (C + 1), 256, 8), 256, 0, st>>>(emb, count, C, c->d, gamma, Wm, A,
                                                                                   loss, (double)nb);
    k_transe_grads<<<grid_for(2 * (int64_t)count * c->d, 256, 8), 256, 0, st>>>(emb, count, C, c->d, Wm, A, grad,
                                                                              (double)nb);
    c->launches += 2;
}

}  // namespace frugal
