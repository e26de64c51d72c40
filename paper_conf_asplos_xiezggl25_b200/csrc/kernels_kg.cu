// kernels_kg.cu -- KG glue: TransE-L2 with chunked shared negatives (R26; PAPER.md
// §4.1).  Not the library proper: it turns looked-up rows into
// gradients so the KG workload (BASELINE.json configs[3]) runs through the hot path.
// All arithmetic in fp64 with explicitly rounded ops in the order the definition is
// written (sums over k, j, b ascending), gradients rounded to fp32 once.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

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

// ---- tiled versions (default): 32x32 output tiles per CTA; each thread RI x CQ outputs,
// rows ty + TY*i and columns tx + TX*q (interleaved: with a row stride of 33 doubles the
// shared-memory reads of a warp hit distinct bank pairs); operand tiles of 32 (k, j or b)
// staged in shared memory as fp64.  Every output still accumulates in the written order
// (k / j / b ascending), so the results equal the loops above bit for bit.
constexpr int TT = 32;

// distances of all (b, j) pairs of a chunk: W[b][j] = sigma(gamma - dist)/dist/nC, loss
template <int RI, int CQ>
__global__ void __launch_bounds__((TT / RI) * (TT / CQ)) k_transe_pairs_tiled(const float* __restrict__ emb, int count,
                                                                             int C, int d, double gamma,
                                                                             double* __restrict__ Wm, double* loss,
                                                                             double nb) {
    constexpr int TX = TT / CQ, TY = TT / RI, NT = TX * TY;
    __shared__ double Ps[TT][TT + 1];
    __shared__ double Ns[TT][TT + 1];
    const int tiles = (C + TT - 1) / TT;
    const int c = blockIdx.x / (tiles * tiles), tb = (blockIdx.x / tiles) % tiles, tj = blockIdx.x % tiles;
    const int b0 = c * C, nC = min(C, count - b0);
    if (tb * TT >= nC || tj * TT >= nC) return;
    const int tx = threadIdx.x % TX, ty = threadIdx.x / TX;  // thread owns b = ty + TY*i, j = tx + TX*q
    double acc[RI][CQ];
#pragma unroll
    for (int i = 0; i < RI; i++)
#pragma unroll
        for (int q = 0; q < CQ; q++) acc[i][q] = 0.0;
    for (int k0 = 0; k0 < d; k0 += TT) {
        for (int e = threadIdx.x; e < TT * TT; e += NT) {
            const int r = e / TT, kk = e % TT, k = k0 + kk;
            const int bl = tb * TT + r, jl = tj * TT + r;
            double pv = 0.0, nv = 0.0;
            if (k < d && bl < nC) {
                const int64_t b = b0 + bl;
                pv = __dadd_rn((double)emb[(b * 4 + 0) * d + k], (double)emb[(b * 4 + 1) * d + k]);
            }
            if (k < d && jl < nC) nv = (double)emb[((int64_t)(b0 + jl) * 4 + 3) * d + k];
            Ps[r][kk] = pv;
            Ns[r][kk] = nv;
        }
        __syncthreads();
        const int kend = min(TT, d - k0);
        for (int kk = 0; kk < kend; kk++) {
            double pv[RI], nv[CQ];
#pragma unroll
            for (int i = 0; i < RI; i++) pv[i] = Ps[ty + TY * i][kk];
#pragma unroll
            for (int q = 0; q < CQ; q++) nv[q] = Ns[tx + TX * q][kk];
#pragma unroll
            for (int i = 0; i < RI; i++)
#pragma unroll
                for (int q = 0; q < CQ; q++) {
                    const double u = __dsub_rn(pv[i], nv[q]);
                    acc[i][q] = __dadd_rn(acc[i][q], __dmul_rn(u, u));
                }
        }
        __syncthreads();
    }
    double lsum = 0.0;
#pragma unroll
    for (int i = 0; i < RI; i++)
#pragma unroll
        for (int q = 0; q < CQ; q++) {
            const int bl = tb * TT + ty + TY * i, jl = tj * TT + tx + TX * q;
            if (bl < nC && jl < nC) {
                const double dist = __dsqrt_rn(acc[i][q]);
                const double sc = __dsub_rn(gamma, dist);
                lsum += __ddiv_rn(softplus(sc), (double)nC);
                Wm[(int64_t)(b0 + bl) * C + jl] = dist > 0.0 ? __ddiv_rn(__ddiv_rn(sigm(sc), dist), (double)nC) : 0.0;
            }
        }
    __shared__ double sl[NT / 32];
    for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(FULL, lsum, o);
    if ((threadIdx.x & 31) == 0) sl[threadIdx.x >> 5] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int i = 0; i < NT / 32; i++) t += sl[i];
        if (t != 0.0) atomicAdd(loss, t / nb);
    }
}

// positive triples: a_b = (1 - sigma(gamma - |v|))/|v|, loss.  One warp per b: the lanes
// form the squared terms v_k^2 of the row in parallel (each exactly as written), lane 0 then
// adds them in k-ascending order (the canonical sum, R26) from shared memory.  (A thread per
// b walking its rows was L1-bound on the uncoalesced row reads: 174 us per step at FB15k.)
// smem: (blockDim / 32) * d doubles.
__global__ void k_transe_pos(const float* __restrict__ emb, int count, int d, double gamma, double* __restrict__ A,
                             double* loss, double nb) {
    extern __shared__ double sq[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    double* my = sq + (size_t)w * d;
    double lsum = 0.0;
    const int nw = (int)(gridDim.x * (blockDim.x >> 5));
    for (int b = blockIdx.x * (int)(blockDim.x >> 5) + w; b < count; b += nw) {
        const float* h = emb + ((int64_t)b * 4 + 0) * d;
        const float* r = emb + ((int64_t)b * 4 + 1) * d;
        const float* t = emb + ((int64_t)b * 4 + 2) * d;
        for (int k = lane; k < d; k += 32) {
            const double v = __dsub_rn(__dadd_rn((double)h[k], (double)r[k]), (double)t[k]);
            my[k] = __dmul_rn(v, v);
        }
        __syncwarp();
        if (lane == 0) {
            double acc = 0.0;
            for (int k = 0; k < d; k++) acc = __dadd_rn(acc, my[k]);
            const double dist = __dsqrt_rn(acc);
            const double sc = __dsub_rn(gamma, dist);
            lsum += softplus(-sc);
            A[b] = dist > 0.0 ? __ddiv_rn(__dsub_rn(1.0, sigm(sc)), dist) : 0.0;
        }
        __syncwarp();
    }
    if (lane == 0 && lsum != 0.0) atomicAdd(loss, lsum / nb);
}

// gradients: MODE 0: (h, r, t) rows, output tile (b, k), reduction over j ascending;
//            MODE 1: negative rows,  output tile (j, k), reduction over b ascending.
template <int MODE, int RI, int CQ>
__global__ void __launch_bounds__((TT / RI) * (TT / CQ)) k_transe_grads_tiled(const float* __restrict__ emb, int count,
                                                                             int C, int d,
                                                                             const double* __restrict__ Wm,
                                                                             const double* __restrict__ A,
                                                                             float* __restrict__ grad, double nb) {
    constexpr int TX = TT / CQ, TY = TT / RI, NT = TX * TY;
    __shared__ double Ws[TT][TT + 1];  // [out row][red]
    __shared__ double Xs[TT][TT + 1];  // [red][k]: N (mode 0) or P (mode 1)
    const int rtiles = (C + TT - 1) / TT, ktiles = (d + TT - 1) / TT;
    const int c = blockIdx.x / (rtiles * ktiles), tr = (blockIdx.x / ktiles) % rtiles, tk = blockIdx.x % ktiles;
    const int b0 = c * C, nC = min(C, count - b0);
    if (tr * TT >= nC) return;
    const int tx = threadIdx.x % TX, ty = threadIdx.x / TX;  // outputs rows ty + TY*i, k = tx + TX*q
    double own[RI][CQ], accv[RI][CQ];
#pragma unroll
    for (int i = 0; i < RI; i++)
#pragma unroll
        for (int q = 0; q < CQ; q++) {
            const int rl = tr * TT + ty + TY * i, k = tk * TT + tx + TX * q;
            own[i][q] = 0.0;
            accv[i][q] = 0.0;
            if (rl < nC && k < d) {
                const int64_t b = b0 + rl;
                if (MODE == 0) {
                    const double P = __dadd_rn((double)emb[(b * 4 + 0) * d + k], (double)emb[(b * 4 + 1) * d + k]);
                    own[i][q] = P;
                    accv[i][q] = __dmul_rn(A[b], __dsub_rn(P, (double)emb[(b * 4 + 2) * d + k]));  // a_b v
                } else {
                    own[i][q] = (double)emb[(b * 4 + 3) * d + k];  // n_j
                }
            }
        }
    double keep[RI][CQ];  // a_b v (mode 0)
#pragma unroll
    for (int i = 0; i < RI; i++)
#pragma unroll
        for (int q = 0; q < CQ; q++) keep[i][q] = accv[i][q];
    for (int r0 = 0; r0 < nC; r0 += TT) {
        for (int e = threadIdx.x; e < TT * TT; e += NT) {
            const int x = e / TT, y = e % TT;
            // Ws[x][y] = W[out row x][red y]   (mode 0: W[b][j]; mode 1: W[b=red][j=out])
            const int ol = tr * TT + x, rl = r0 + y;
            double wv = 0.0;
            if (ol < nC && rl < nC) wv = MODE == 0 ? Wm[(int64_t)(b0 + ol) * C + rl] : Wm[(int64_t)(b0 + rl) * C + ol];
            Ws[x][y] = wv;
            // Xs[x][y] = operand of reduction row x at k = tk*TT + y
            const int rl2 = r0 + x, k = tk * TT + y;
            double xv = 0.0;
            if (rl2 < nC && k < d) {
                const int64_t rr = b0 + rl2;
                xv = MODE == 0 ? (double)emb[(rr * 4 + 3) * d + k]
                               : __dadd_rn((double)emb[(rr * 4 + 0) * d + k], (double)emb[(rr * 4 + 1) * d + k]);
            }
            Xs[x][y] = xv;
        }
        __syncthreads();
        const int rend = min(TT, nC - r0);
        for (int y = 0; y < rend; y++) {
            double wv[RI], xv[CQ];
#pragma unroll
            for (int i = 0; i < RI; i++) wv[i] = Ws[ty + TY * i][y];
#pragma unroll
            for (int q = 0; q < CQ; q++) xv[q] = Xs[y][tx + TX * q];
#pragma unroll
            for (int i = 0; i < RI; i++)
#pragma unroll
                for (int q = 0; q < CQ; q++) {
                    if (MODE == 0) {  // gh -= W_bj (P_b - n_j)
                        accv[i][q] = __dsub_rn(accv[i][q], __dmul_rn(wv[i], __dsub_rn(own[i][q], xv[q])));
                    } else {          // gn += W_bj (P_b - n_j)
                        accv[i][q] = __dadd_rn(accv[i][q], __dmul_rn(wv[i], __dsub_rn(xv[q], own[i][q])));
                    }
                }
        }
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < RI; i++)
#pragma unroll
        for (int q = 0; q < CQ; q++) {
            const int rl = tr * TT + ty + TY * i, k = tk * TT + tx + TX * q;
            if (rl < nC && k < d) {
                const int64_t b = b0 + rl;
                if (MODE == 0) {
                    const float g = (float)__ddiv_rn(accv[i][q], nb);
                    grad[(b * 4 + 0) * d + k] = g;
                    grad[(b * 4 + 1) * d + k] = g;
                    grad[(b * 4 + 2) * d + k] = (float)__ddiv_rn(-keep[i][q], nb);
                } else {
                    grad[(b * 4 + 3) * d + k] = (float)__ddiv_rn(accv[i][q], nb);
                }
            }
        }
}

void launch_transe_model(frugal_ctx* c, QueueSlot& q, const float* emb, int C, double gamma, float* grad,
                         double* loss, int64_t nb, double* Wm, double* A, cudaStream_t st) {
    const int count = q.h_counts[c->g];
    if (count <= 0) return;
    const int nchunks = (count + C - 1) / C;
    static const bool naive = getenv("FRUGAL_TRANSE_NAIVE") != nullptr;  // reference loops (tests)
    if (naive) {
        k_transe_pairs<<<grid_for((int64_t)nchunks * C * (C + 1), 256, 8), 256, 0, st>>>(emb, count, C, c->d, gamma,
                                                                                       Wm, A, loss, (double)nb);
        k_transe_grads<<<grid_for(2 * (int64_t)count * c->d, 256, 8), 256, 0, st>>>(emb, count, C, c->d, Wm, A,
                                                                                  grad, (double)nb);
        c->launches += 2;
        return;
    }
    const int tiles = (C + TT - 1) / TT, ktiles = (c->d + TT - 1) / TT;
    k_transe_pos<<<grid_for((int64_t)count * 32, 128, 4), 128, (size_t)4 * c->d * sizeof(double), st>>>(
        emb, count, c->d, gamma, A, loss, (double)nb);
    // 2x2 outputs per thread, 256 threads per 32x32 tile: 4x4 / 2x4 / 1x2 / 2x1 measured slower at
    // C = 200 (profiles/r1_sweep23_kg_tile.txt, r1_sweep24_kg_tile.txt)
    constexpr int RI = 2, CQ = 2, nt = (TT / RI) * (TT / CQ);
    k_transe_pairs_tiled<RI, CQ><<<nchunks * tiles * tiles, nt, 0, st>>>(emb, count, C, c->d, gamma, Wm, loss,
                                                                         (double)nb);
    k_transe_grads_tiled<0, RI, CQ><<<nchunks * tiles * ktiles, nt, 0, st>>>(emb, count, C, c->d, Wm, A, grad,
                                                                             (double)nb);
    k_transe_grads_tiled<1, RI, CQ><<<nchunks * tiles * ktiles, nt, 0, st>>>(emb, count, C, c->d, Wm, A, grad,
                                                                             (double)nb);
    c->launches += 4;
}

// fp64 instruction-rate probe (frugal_probe_fp64): per thread 8 independent chains of
// dependent DADD/DMUL pairs (the KG glue's instruction mix, no FMA contraction), all SMs,
// 32 warps per SM; 2 ops per chain step
constexpr int kProbeChains = 8, kProbeInner = 256;
__global__ void __launch_bounds__(256) k_probe_fp64(double* out, int iters) {
    double x[kProbeChains];
#pragma unroll
    for (int c = 0; c < kProbeChains; c++) x[c] = 1.0 + 1e-3 * (threadIdx.x + c);
    const double a = 1.0000001, m = 0.9999999;
    for (int it = 0; it < iters; it++) {
#pragma unroll 4
        for (int i = 0; i < kProbeInner; i++) {
#pragma unroll
            for (int c = 0; c < kProbeChains; c++) x[c] = __dmul_rn(__dadd_rn(x[c], a), m);
        }
    }
    double acc = 0.0;
#pragma unroll
    for (int c = 0; c < kProbeChains; c++) acc += x[c];
    if (acc == 12345.678) out[threadIdx.x] = acc;  // keeps the chains live
}
void launch_probe_fp64(double* out, int iters, int64_t* ops, cudaStream_t st) {
    const int grid = kSMs * 8, block = 256;
    k_probe_fp64<<<grid, block, 0, st>>>(out, iters);
    *ops = (int64_t)grid * block * iters * kProbeInner * kProbeChains * 2;
}

}  // namespace frugal
