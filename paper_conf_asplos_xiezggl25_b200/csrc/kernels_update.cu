// kernels_update.cu -- backward (segment-reduce, mailbox, fused optimizer), final flush,
// table/metadata initialisation, cross-rank flags and introspection kernels (sm_100a).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "frugal_internal.cuh"
#include "kutil.cuh"

namespace frugal {

__device__ __forceinline__ float4 add4(float4 a, float4 b) {
    return make_float4(__fadd_rn(a.x, b.x), __fadd_rn(a.y, b.y), __fadd_rn(a.z, b.z), __fadd_rn(a.w, b.w));
}

// a8 elementwise optimizer on one float4 (reading R13; every op rounded separately, R22):
// Adagrad G += g*g; w -= (lr*g) / (sqrt(G) + eps), or SGD w -= lr*g
__device__ __forceinline__ void opt4(float4& w, float4& G, const float4& acc, int adagrad, float lr, float eps) {
    float* wp = &w.x;
    float* Gp = &G.x;
    const float* gp = &acc.x;
#pragma unroll
    for (int c = 0; c < 4; c++) {
        if (adagrad) {
            Gp[c] = __fadd_rn(Gp[c], __fmul_rn(gp[c], gp[c]));
            float num = __fmul_rn(lr, gp[c]);
            float den = __fadd_rn(__fsqrt_rn(Gp[c]), eps);
            wp[c] = __fsub_rn(wp[c], __fdiv_rn(num, den));
        } else {
            wp[c] = __fsub_rn(wp[c], __fmul_rn(lr, gp[c]));
        }
    }
}

// World 1: the owner's optimizer fused into the segment-reduce (T(s) == uniq(s), every
// partial is this rank's own) -- the reduced gradient of unique row j goes straight from
// registers into the update instead of through a partials buffer and a second kernel.
struct FusedOpt {
    int on;  // 0: write partials (world > 1, comparison path)
    int32_t s;
    int adagrad;
    float lr, eps;
    const int32_t* uniq;
    const float4* rows_w;  // this step's gathered rows (w of the cold rows)
    const int32_t* slot;
    int32_t* state;
    int32_t* last_upd;
    int32_t* pool_idx;
    uint64_t* rbits;
    float4* cw;
    float4* Gd;
    float4* pw;  // pool segment s % P
    int32_t gmask;  // diagnostic only (FRUGAL_DIAG_G_MASK): G row index & gmask (-1: all rows)
    int32_t* pkey;
    int32_t* pcount;
};

// row j of the fused update: lane l's columns from sum(v), then the row's metadata
template <int GS, typename SumF>
__device__ __forceinline__ void fused_update_row(const FusedOpt& fo, int j, int d4, int l, SumF sum, unsigned& nhot,
                                                 unsigned& ncold) {
    const int32_t lk = fo.uniq[j];
    const int sl = fo.slot[lk];
    for (int v = l; v < d4; v += GS) {
        const float4 acc = sum(v);
        float4 w = sl >= 0 ? fo.cw[(int64_t)sl * d4 + v] : fo.rows_w[(int64_t)j * d4 + v];
        float4 G = make_float4(0.f, 0.f, 0.f, 0.f);
        if (fo.adagrad) G = fo.Gd[(int64_t)lk * d4 + v];
        opt4(w, G, acc, fo.adagrad, fo.lr, fo.eps);
        if (sl >= 0) fo.cw[(int64_t)sl * d4 + v] = w;
        else fo.pw[(int64_t)j * d4 + v] = w;
        if (fo.adagrad) fo.Gd[(int64_t)lk * d4 + v] = G;
    }
    if (l == 0) {
        if (sl >= 0) nhot++;
        else ncold++;
        fo.state[lk] = ST_UPDATED;
        fo.last_upd[lk] = fo.s;
        const uint64_t clear = ~((1ull << (fo.s & 31)) | (1ull << (32 + (fo.s & 31))));
        atomicAnd((unsigned long long*)&fo.rbits[lk], (unsigned long long)clear);  // races with k_ingest_bits
        if (sl < 0) fo.pool_idx[lk] = j;
        fo.pkey[j] = sl < 0 ? lk : -1;
    }
}

// ============================================================================ a6 segment-reduce
// P[q] = sum over the occurrences of unique row u in the canonical fixed order
// (reading R23): positions ascending, cut into chunks of kChunk; each chunk summed
// sequentially, chunk sums added sequentially.  world == 1: q = u.  world > 1: q walks
// the owner-grouped order (gl); rows owned by this rank stay in HBM (Pp[q]), the others
// go to this rank's host mailbox (zero-copy stores; §3.2 "update
// staging queue").  Segments longer than one chunk (the Zipf head) are deferred to
// k_segreduce_long, which computes their chunks in parallel.
constexpr int kChunk = 64;

template <int GS, bool SHORT8 = true>
__device__ __forceinline__ float4 chunk_sum(const float4* __restrict__ grad, const int32_t* __restrict__ pos, int b,
                                            int e, int d4, int v) {
    if (SHORT8 && e - b <= 4) {  // short rows (most of them): all positions, then all gradient rows in flight
        const int n = e - b;
        int pq[4];
#pragma unroll
        for (int q = 0; q < 4; q++) pq[q] = q < n ? pos[b + q] : 0;
        float4 x[4];
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (q < n) x[q] = grad[(int64_t)pq[q] * d4 + v];
        float4 acc = x[0];
#pragma unroll
        for (int q = 1; q < 4; q++)
            if (q < n) acc = add4(acc, x[q]);
        return acc;
    }
    float4 acc = grad[(int64_t)pos[b] * d4 + v];
    int j = b + 1;
    for (; j + 16 <= e; j += 16) {  // 16 loads in flight, adds in position order
        int pq[16];
#pragma unroll
        for (int q = 0; q < 16; q++) pq[q] = pos[j + q];
        float4 x[16];
#pragma unroll
        for (int q = 0; q < 16; q++) x[q] = grad[(int64_t)pq[q] * d4 + v];
        asm volatile("" ::: "memory");  // keep all 16 loads issued before the first add
#pragma unroll
        for (int q = 0; q < 16; q++) acc = add4(acc, x[q]);
    }
    for (; j + 4 <= e; j += 4) {
        float4 x[4];
#pragma unroll
        for (int q = 0; q < 4; q++) x[q] = grad[(int64_t)pos[j + q] * d4 + v];
#pragma unroll
        for (int q = 0; q < 4; q++) acc = add4(acc, x[q]);
    }
    for (; j < e; j++) acc = add4(acc, grad[(int64_t)pos[j] * d4 + v]);
    return acc;
}

template <int GS>
__global__ void __launch_bounds__(256) k_segreduce(const int32_t* __restrict__ off, const int32_t* __restrict__ pos,
                            const int32_t* d_nu, const int32_t* __restrict__ gl, const int32_t* __restrict__ goff,
                            int g, int d4, const float4* __restrict__ grad, float4* __restrict__ Pp, float4* mail,
                            int32_t* long_q, int32_t* long_cnt, int2* tasks, int32_t* task_cnt,
                            unsigned long long* stats, const FusedOpt fo) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n = *d_nu;
    unsigned nhot = 0, ncold = 0;
    int own_lo = 0, own_hi = n;
    if (gl) {
        own_lo = goff[g];
        own_hi = goff[g + 1];
    }
    unsigned nlong = 0, nout = 0;
    for (int64_t q = gid; q < n; q += gs) {
        const int u = gl ? gl[q] : (int)q;
        const int b = off[u], e = off[u + 1];
        if (l == 0 && (q < own_lo || q >= own_hi)) nout++;
        if (e - b > kChunk) {  // Zipf head: chunk tasks for k_segred_chunks
            if (l == 0) {
                long_q[atomicAdd(long_cnt, 1)] = (int32_t)q;
                const int nch = (e - b + kChunk - 1) / kChunk;
                const int t0 = atomicAdd(task_cnt, nch);
                for (int cc = 0; cc < nch; cc++) tasks[t0 + cc] = make_int2(b + cc * kChunk, min(e, b + (cc + 1) * kChunk));
                nlong++;
            }
            continue;
        }
        if (fo.on) {
            fused_update_row<GS>(fo, u, d4, l, [&](int v) { return chunk_sum<GS>(grad, pos, b, e, d4, v); }, nhot, ncold);
            continue;
        }
        float4* dst = (q >= own_lo && q < own_hi) ? (Pp + q * d4) : (mail + q * d4);
        for (int v = l; v < d4; v += GS) dst[v] = chunk_sum<GS>(grad, pos, b, e, d4, v);
    }
    if (gl) block_fence_system();
    block_count(stats + FRUGAL_C_LONG_SEGMENTS, nlong);
    block_count(stats + FRUGAL_C_MAIL_OUT, nout);
    if (fo.on) {
        if (blockIdx.x == 0 && threadIdx.x == 0) *fo.pcount = n;
        block_count(stats + FRUGAL_C_OPT_HOT, nhot);
        block_count(stats + FRUGAL_C_OPT_COLD, ncold);
    }
}

// Ordered sum of n rows (row(0) first, then row(1), ...) of src, column v, with the row
// loads staged through shared memory by cp.async in double-buffered batches of 16, so
// 16-32 row loads are in flight per lane while the adds stay strictly in order.
// smem: [2][16][blockDim] float4, each thread touching only its own column.
constexpr int kBatch = 16;

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <typename RowF>
__device__ __forceinline__ float4 ordered_sum(RowF row, int n, const float4* __restrict__ src, int d4, int v,
                                              float4* smem) {
    const int nt = blockDim.x, t = threadIdx.x;
    auto issue = [&](int k) {
        const int q0 = k * kBatch, q1 = min(n, q0 + kBatch);
        float4* bb = smem + (size_t)(k & 1) * kBatch * nt;
        for (int q = q0; q < q1; q++) cp_async16(bb + (size_t)(q - q0) * nt + t, src + (int64_t)row(q) * d4 + v);
        cp_async_commit();
    };
    const int nb = (n + kBatch - 1) / kBatch;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    issue(0);
    for (int k = 0; k < nb; k++) {
        if (k + 1 < nb) {
            issue(k + 1);
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        const float4* bb = smem + (size_t)(k & 1) * kBatch * nt;
        const int q0 = k * kBatch, q1 = min(n, q0 + kBatch);
        for (int q = q0; q < q1; q++) {
            float4 x = bb[(size_t)(q - q0) * nt + t];
            acc = (q == 0) ? x : add4(acc, x);
        }
    }
    return acc;
}
constexpr size_t kOrderedSmem = 2 * kBatch * 256 * sizeof(float4);  // 128 KB for 256 threads

// Long segments, phase 1: every chunk [j0, j1) of every long segment in parallel (task
// list built by k_segreduce), summed in order into scratch[j0].
template <int GS>
__global__ void __launch_bounds__(256) k_segred_chunks(const int32_t* __restrict__ pos, int d4,
                                                       const float4* __restrict__ grad, float4* __restrict__ scratch,
                                                       const int2* __restrict__ tasks, const int32_t* task_cnt) {
    extern __shared__ float4 smem[];
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int nt = *task_cnt;
    const int64_t nloop = (nt + gs - 1) / gs * gs;  // uniform trip count: ordered_sum is per-thread
    for (int64_t t = gid; t < nloop; t += gs) {
        if (t >= nt) continue;
        const int2 tk = tasks[t];
        const int32_t* pj = pos + tk.x;
        for (int v = l; v < d4; v += GS)
            scratch[(int64_t)tk.x * d4 + v] = ordered_sum([&](int q) { return pj[q]; }, tk.y - tk.x, grad, d4, v, smem);
    }
}

// Long segments, phase 2: per long segment, add its chunk sums in order
template <int GS>
__global__ void __launch_bounds__(256) k_segred_combine(const int32_t* __restrict__ off,
                                                        const int32_t* __restrict__ gl,
                                                        const int32_t* __restrict__ goff, int g, int d4,
                                                        float4* __restrict__ Pp, float4* mail,
                                                        const int32_t* __restrict__ long_q, const int32_t* long_cnt,
                                                        const float4* __restrict__ scratch, unsigned long long* stats,
                                                        const FusedOpt fo) {
    extern __shared__ float4 smem[];
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int nl = *long_cnt;
    unsigned nhot = 0, ncold = 0;
    int own_lo = 0, own_hi = 0x7fffffff;
    if (gl) {
        own_lo = goff[g];
        own_hi = goff[g + 1];
    }
    const int64_t nloop = (nl + gs - 1) / gs * gs;
    for (int64_t t = gid; t < nloop; t += gs) {
        if (t >= nl) continue;
        const int q = long_q[t];
        const int u = gl ? gl[q] : q;
        const int b = off[u], e = off[u + 1];
        const int nch = (e - b + kChunk - 1) / kChunk;
        if (fo.on) {  // ordered_sum is per-thread with a uniform trip count: every lane calls it
            fused_update_row<GS>(fo, u, d4, l, [&](int v) {
                return ordered_sum([&](int c) { return b + c * kChunk; }, nch, scratch, d4, v, smem); }, nhot, ncold);
            continue;
        }
        float4* dst = (q >= own_lo && q < own_hi) ? (Pp + (int64_t)q * d4) : (mail + (int64_t)q * d4);
        for (int v = l; v < d4; v += GS)
            dst[v] = ordered_sum([&](int c) { return b + c * kChunk; }, nch, scratch, d4, v, smem);
    }
    if (gl) block_fence_system();
    if (fo.on) {
        block_count(stats + FRUGAL_C_OPT_HOT, nhot);
        block_count(stats + FRUGAL_C_OPT_COLD, ncold);
    }
}

void launch_segreduce(frugal_ctx* c, QueueSlot& q, const float* grad, int par, float* dest, cudaStream_t st,
                      int64_t fused_step) {
    const int d4 = c->d / 4, gs = group_size(d4);
    FusedOpt fo{};
    fo.gmask = -1;
    if (fused_step >= 0) {  // world 1: a6 + a8 in one pass (launch_optimizer is not called)
        const int seg = (int)(fused_step % c->P);
        fo.on = 1;
        fo.s = (int32_t)fused_step;
        fo.adagrad = c->cfg.opt == FRUGAL_ADAGRAD;
        fo.lr = c->cfg.lr;
        fo.eps = c->cfg.eps;
        fo.uniq = q.uniq;
        fo.rows_w = (const float4*)c->rows_buf[fused_step & 1];
        fo.slot = c->slot;
        fo.state = c->state;
        fo.last_upd = c->last_upd;
        fo.pool_idx = c->pool_idx;
        fo.rbits = c->rbits;
        fo.cw = (float4*)c->cw;
        fo.Gd = (float4*)c->Gd;
        fo.pw = (float4*)c->pw + (size_t)seg * c->capT * d4;
        fo.pkey = c->pkey + (size_t)seg * c->capT;
        fo.pcount = c->pcount + seg;
    }
    int grid = grid_for((int64_t)c->M * gs, 256, 8);
    const bool multi = c->n > 1;
    // dest (comparison path): every partial, own or not, to one device buffer in grouped order
    float4* mail = dest ? (float4*)dest
                        : multi ? (float4*)(c->dh_mail + ((size_t)par * c->n + c->g) * c->mail_stride + 256) : nullptr;
    float* Pp = dest ? dest : c->Pp;
    cudaMemsetAsync(c->long_cnt, 0, 8, st);  // long_cnt[0] = long segments, long_cnt[1] = chunk tasks
    DISPATCH_GS(gs, (k_segreduce<GS><<<grid, 256, 0, st>>>(q.off, q.pos, q.n_uniq, multi ? q.gl : nullptr, q.goff,
                                                           c->g, d4, (const float4*)grad, (float4*)Pp, mail,
                                                           c->long_q, c->long_cnt, c->long_tasks, c->long_cnt + 1,
                                                           c->dstats, fo)));
    DISPATCH_GS(gs, (k_segred_chunks<GS><<<kSMs, 256, kOrderedSmem, st>>>(q.pos, d4, (const float4*)grad,
                                                                          (float4*)c->chunk_scratch, c->long_tasks,
                                                                          c->long_cnt + 1)));
    DISPATCH_GS(gs, (k_segred_combine<GS><<<kSMs, 256, kOrderedSmem, st>>>(q.off, multi ? q.gl : nullptr, q.goff, c->g,
                                                                           d4, (float4*)Pp, mail, c->long_q,
                                                                           c->long_cnt,
                                                                           (const float4*)c->chunk_scratch, c->dstats,
                                                                           fo)));
    c->launches += 3;
}

// per-device kernel attributes (cudaFuncSetAttribute applies to the current device): called
// by frugal_init after cudaSetDevice, for every row-group width
cudaError_t setup_kernel_attrs() {
    cudaError_t e = cudaSuccess;
    for (int gs = 1; gs <= 32; gs <<= 1) {
        DISPATCH_GS(gs, (e = cudaFuncSetAttribute(k_segred_chunks<GS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                  (int)kOrderedSmem)));
        if (e != cudaSuccess) return e;
        DISPATCH_GS(gs, (e = cudaFuncSetAttribute(k_segred_combine<GS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                  (int)kOrderedSmem)));
        if (e != cudaSuccess) return e;
    }
    return e;
}

// ============================================================================ a6 + a8, world 1, one launch
// Long segments of a step (> kChunk occurrences), listed at ingest (one step ahead, off the
// critical path): per long row {u, first task, chunks}; per 64-chunk a task {b, e, row, c}.
// The order of the lists is irrelevant to the results: chunk c of a row always lands in
// scratch slot t0 + c and the chunk sums are added in c order.
__global__ void k_long_tasks(const int32_t* __restrict__ off, const int32_t* d_nu, int4* __restrict__ linfo,
                             int4* __restrict__ ltask, int32_t* __restrict__ lcnt, int32_t* lnum,
                             unsigned long long* stats) {
    const int n = *d_nu;
    unsigned nl = 0;
    for (int u = blockIdx.x * blockDim.x + threadIdx.x; u < n; u += gridDim.x * blockDim.x) {
        const int b = off[u], e = off[u + 1];
        if (e - b <= kChunk) continue;
        const int nch = (e - b + kChunk - 1) / kChunk;
        const int L = atomicAdd(&lnum[0], 1);
        const int t0 = atomicAdd(&lnum[1], nch);
        linfo[L] = make_int4(u, t0, nch, 0);
        lcnt[L] = 0;
        for (int c = 0; c < nch; c++) ltask[t0 + c] = make_int4(b + c * kChunk, min(e, b + (c + 1) * kChunk), L, c);
        nl++;
    }
    block_count(stats + FRUGAL_C_LONG_SEGMENTS, nl);
}
void launch_long_tasks(frugal_ctx* c, QueueSlot& q, cudaStream_t st) {
    cudaMemsetAsync(q.lnum, 0, 8, st);
    k_long_tasks<<<grid_for(c->M, 256, 2), 256, 0, st>>>(q.off, q.n_uniq, q.linfo, q.ltask, q.lcnt, q.lnum, c->dstats);
    c->launches++;
}

// ordered sum of n rows base[0], base[d4], ... (row 0 first), 16 loads in flight; L1 bypassed
// (the rows were written by other CTAs of this launch)
__device__ __forceinline__ float4 ordered_rows_cg(const float4* base, int d4, int n) {
    float4 acc = __ldcg(base);
    int c = 1;
    for (; c + 16 <= n; c += 16) {
        float4 x[16];
#pragma unroll
        for (int q = 0; q < 16; q++) x[q] = __ldcg(base + (int64_t)(c + q) * d4);
#pragma unroll
        for (int q = 0; q < 16; q++) acc = add4(acc, x[q]);
    }
    for (; c < n; c++) acc = add4(acc, __ldcg(base + (int64_t)c * d4));
    return acc;
}

// the fused update of unique row j with the row's w and G loaded BEFORE its gradient sum (they
// do not depend on it): lane l owns columns v = l + k*GS, k < VPL
template <int GS, int VPL, typename SumF>
__device__ __forceinline__ void update_row_pf(const FusedOpt& fo, int j, int d4, int l, SumF sum, unsigned& nhot,
                                              unsigned& ncold) {
    const int32_t lk = fo.uniq[j];
    const int sl = fo.slot[lk];
    const float4* wsrc = sl >= 0 ? fo.cw + (int64_t)sl * d4 : fo.rows_w + (int64_t)j * d4;
    float4 w[VPL], G[VPL];
#pragma unroll
    for (int k = 0; k < VPL; k++) {
        const int v = l + k * GS;
        G[k] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (v < d4) {
            w[k] = wsrc[v];
            if (fo.adagrad) G[k] = fo.Gd[(int64_t)(lk & fo.gmask) * d4 + v];
        }
    }
#pragma unroll
    for (int k = 0; k < VPL; k++) {
        const int v = l + k * GS;
        if (v < d4) {
            const float4 acc = sum(v);
            opt4(w[k], G[k], acc, fo.adagrad, fo.lr, fo.eps);
            if (sl >= 0) fo.cw[(int64_t)sl * d4 + v] = w[k];
            else fo.pw[(int64_t)j * d4 + v] = w[k];
            if (fo.adagrad) fo.Gd[(int64_t)(lk & fo.gmask) * d4 + v] = G[k];
        }
    }
    if (l == 0) {
        if (sl >= 0) nhot++;
        else ncold++;
        fo.state[lk] = ST_UPDATED;
        fo.last_upd[lk] = fo.s;
        const uint64_t clear = ~((1ull << (fo.s & 31)) | (1ull << (32 + (fo.s & 31))));
        atomicAnd((unsigned long long*)&fo.rbits[lk], (unsigned long long)clear);  // races with k_ingest_bits
        if (sl < 0) fo.pool_idx[lk] = j;
        fo.pkey[j] = sl < 0 ? lk : -1;
    }
}

// One launch for the whole world-1 backward (a6 + a8): work items [0, nt) are the 64-chunks
// of the long rows (summed in order into scratch[item]; the group that completes a row's last
// chunk adds the row's chunk sums in chunk order and applies the optimizer), items
// [nt, nt + nu) the unique rows, of which the short ones (<= 64 occurrences) are reduced
// and updated directly.  Same arithmetic, same order as k_segreduce + k_segred_chunks +
// k_segred_combine (reading R23), without their serialisation.
constexpr int kUpdBatch = 8;  // work items a warp takes per fetch (dynamic mode)

template <int GS, int VPL, bool SHORT8>
__global__ void __launch_bounds__(256) k_update1(const int32_t* __restrict__ off, const int32_t* __restrict__ pos,
                                                 const int32_t* d_nu, const int4* __restrict__ ltask,
                                                 const int4* __restrict__ linfo, int32_t* lcnt,
                                                 const int32_t* lnum, int d4, const float4* __restrict__ grad,
                                                 float4* scratch, unsigned long long* stats, const FusedOpt fo,
                                                 int32_t* ctr, int par) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const unsigned gmask = GS == 32 ? 0xffffffffu : (((1u << GS) - 1u) << ((threadIdx.x & 31) & ~(GS - 1)));
    const int leader = (threadIdx.x & 31) & ~(GS - 1);
    const int nt = lnum[1], nu = *d_nu;
    const int64_t total = (int64_t)nt + nu;
    unsigned nhot = 0, ncold = 0;
    auto item = [&](int64_t w) {
        if (w < nt) {
            const int4 tk = ltask[w];
            for (int v = l; v < d4; v += GS)
                __stcg(scratch + w * d4 + v, chunk_sum<GS, SHORT8>(grad, pos, tk.x, tk.y, d4, v));
            __threadfence();
            __syncwarp(gmask);
            const int4 li = linfo[tk.z];
            int last = 0;
            if (l == 0) last = atomicAdd(&lcnt[tk.z], 1) == li.z - 1;
            last = __shfl_sync(gmask, last, leader);
            if (!last) return;
            __threadfence();  // every chunk of the row is in scratch
            update_row_pf<GS, VPL>(fo, li.x, d4, l, [&](int v) {
                return ordered_rows_cg(scratch + (int64_t)li.y * d4 + v, d4, li.z); }, nhot, ncold);
        } else {
            const int u = (int)(w - nt);
            const int b = off[u], e = off[u + 1];
            if (e - b > kChunk) return;  // a long row: its last chunk task updates it
            update_row_pf<GS, VPL>(fo, u, d4, l, [&](int v) { return chunk_sum<GS, SHORT8>(grad, pos, b, e, d4, v); },
                                   nhot, ncold);
        }
    };
    if (!ctr) {
        for (int64_t w = gid; w < total; w += gs) item(w);
    } else {
        // dynamic: each warp takes the next kUpdBatch items (the long rows' chunks come first) --
        // no block waits for a slow neighbour's static share; the counter of the next step's
        // launch (other parity) is reset here, before that launch can start
        if (blockIdx.x == 0 && threadIdx.x == 0) ctr[par ^ 1] = 0;
        const int lane = threadIdx.x & 31, gpw = 32 / GS, grp = lane / GS;
        for (;;) {
            int base = 0;
            if (lane == 0) base = atomicAdd(&ctr[par], kUpdBatch);
            base = __shfl_sync(0xffffffffu, base, 0);
            if (base >= total) break;
            for (int k = grp; k < kUpdBatch; k += gpw)
                if (base + k < total) item((int64_t)base + k);
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *fo.pcount = nu;
    block_count(stats + FRUGAL_C_OPT_HOT, nhot);
    block_count(stats + FRUGAL_C_OPT_COLD, ncold);
}

void launch_update1(frugal_ctx* c, QueueSlot& q, const float* grad, int64_t s, cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    const int vpl = (d4 + gs - 1) / gs;
    const int seg = (int)(s % c->P);
    FusedOpt fo{};
    fo.on = 1;
    fo.s = (int32_t)s;
    fo.adagrad = c->cfg.opt == FRUGAL_ADAGRAD;
    // diagnostic only (wrong results): G footprint folded to gmask+1 rows -- is the update
    // bound by address translation of its random G accesses over the dense [N][d] array?
    static const int32_t diag_gmask = getenv("FRUGAL_DIAG_G_MASK") ? atoi(getenv("FRUGAL_DIAG_G_MASK")) : -1;
    fo.gmask = diag_gmask;
    fo.lr = c->cfg.lr;
    fo.eps = c->cfg.eps;
    fo.uniq = q.uniq;
    fo.rows_w = (const float4*)c->rows_buf[s & 1];
    fo.slot = c->slot;
    fo.state = c->state;
    fo.last_upd = c->last_upd;
    fo.pool_idx = c->pool_idx;
    fo.rbits = c->rbits;
    fo.cw = (float4*)c->cw;
    fo.Gd = (float4*)c->Gd;
    fo.pw = (float4*)c->pw + (size_t)seg * c->capT * d4;
    fo.pkey = c->pkey + (size_t)seg * c->capT;
    fo.pcount = c->pcount + seg;
    const int grid = grid_for((int64_t)c->M * gs, 256, 8);
    int32_t* ctr = c->update_dyn ? c->upd_ctr : nullptr;
    const int par = (int)(s & 1);
#define U1S(V, SH)                                                                                                \
    do {                                                                                                          \
        DISPATCH_GS(gs, (k_update1<GS, V, SH><<<grid, 256, 0, st>>>(q.off, q.pos, q.n_uniq, q.ltask, q.linfo,     \
                                                                     q.lcnt, q.lnum, d4, (const float4*)grad,      \
                                                                     (float4*)c->chunk_scratch, c->dstats, fo,     \
                                                                     ctr, par)));                                  \
    } while (0)
#define U1(V)                          \
    do {                               \
        if (c->update_short8) U1S(V, true); \
        else U1S(V, false);            \
    } while (0)
    if (vpl <= 1) U1(1);
    else if (vpl <= 2) U1(2);
    else if (vpl <= 4) U1(4);
    else U1(8);
#undef U1
#undef U1S
    c->launches++;
}

// mailbox header of (parity, this sender): goff[0..world]
__global__ void k_mail_header(const int32_t* __restrict__ goff, int world, int32_t* hdr) {
    if (threadIdx.x <= world) hdr[threadIdx.x] = goff[threadIdx.x];
    __threadfence_system();
}
void launch_mail_header(frugal_ctx* c, QueueSlot& q, int par, cudaStream_t st) {
    int32_t* hdr = (int32_t*)(c->dh_mail + ((size_t)par * c->n + c->g) * c->mail_stride);
    k_mail_header<<<1, 64, 0, st>>>(q.goff, c->n, hdr);
    c->launches++;
}

// ============================================================================ a8 merge + fused optimizer
// For each owned row touched at s (T, ascending): g = sum of partials over ranks in
// ascending order (own from HBM, others from their host mailboxes), then SGD/Adagrad
// (elementwise, each op rounded separately).  Hot rows update the HBM cache in place;
// cold rows read (w, G) fresh from the host table and go to pool segment s % P.
// Marks dirty (last update s) and consumes read bit s.
template <int GS>
__global__ void k_optimizer(const int32_t* __restrict__ T, const int32_t* d_nT, const uint32_t* __restrict__ Tmask,
                            const int32_t* __restrict__ Tidx, int64_t capT, int world, int g, int d4, int32_t s,
                            int adagrad, float lr, float eps, const float4* __restrict__ Pp,
                            const int32_t* __restrict__ goff_own, const char* mail_par, size_t mail_stride,
                            const float4* __restrict__ rows_w, const int32_t* __restrict__ slot,
                            int32_t* __restrict__ state, int32_t* __restrict__ last_upd, int32_t* __restrict__ pool_idx,
                            uint64_t* __restrict__ rbits, float4* __restrict__ cw, float4* __restrict__ Gd,
                            float4* __restrict__ pw, int32_t* __restrict__ pkey, int32_t* pcount, const float4* hw,
                            const float4* __restrict__ pw_all, int P, int32_t pool_min,
                            const float4* __restrict__ recv, const int32_t* __restrict__ roff,
                            const int32_t* __restrict__ hs, unsigned long long* stats) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n = *d_nT;
    unsigned nhot = 0, ncold = 0, nin = 0;
    const uint64_t clear = ~((1ull << (s & 31)) | (1ull << (32 + (s & 31))));
    for (int64_t j = gid; j < n; j += gs) {
        const int32_t lk = T[j];
        const int64_t k = (int64_t)lk * world + g;
        const int sl = slot[lk];
        // world > 1: the latest w of a recently updated cold row is still in this owner's pool
        // (segment last_upd % P, not this step's segment s % P); read before lane 0 rewrites it
        const int32_t lu = last_upd[lk];
        const int64_t prow = (sl < 0 && !rows_w && lu >= 0 && lu >= pool_min)
                                 ? ((int64_t)(lu % P) * capT + pool_idx[lk]) : -1;
        const int64_t hrow = (sl < 0 && !rows_w && prow < 0) ? host_row(hs, k) : 0;
        {  // the group's lanes all read `lu` before its lane 0 rewrites last_upd below
            const unsigned gmask = GS == 32 ? 0xffffffffu : (((1u << GS) - 1u) << ((threadIdx.x & 31) & ~(GS - 1)));
            __syncwarp(gmask);
        }
        uint32_t mask = 1u;
        if (world > 1) mask = Tmask[j];
        for (int v = l; v < d4; v += GS) {
            float4 acc;
            if (world == 1) {
                acc = Pp[j * d4 + v];
            } else {
                bool first = true;
                for (int r = 0; r < world; r++) {
                    if (!((mask >> r) & 1u)) continue;
                    const int idx = Tidx[(int64_t)r * capT + j];
                    float4 x;
                    if (recv) {  // comparison path: partials arrived by the caller's all-to-all
                        x = recv[(int64_t)(roff[r] + idx) * d4 + v];
                    } else if (r == g) {
                        x = Pp[(int64_t)(goff_own[g] + idx) * d4 + v];
                    } else {
                        const char* mb = mail_par + (size_t)r * mail_stride;
                        const int base = ((const int32_t*)mb)[g];
                        x = ((const float4*)(mb + 256))[(int64_t)(base + idx) * d4 + v];
                    }
                    acc = first ? x : add4(acc, x);
                    first = false;
                }
            }
            float4 w, G = make_float4(0.f, 0.f, 0.f, 0.f);
            if (sl >= 0) w = cw[(int64_t)sl * d4 + v];
            else if (rows_w) w = rows_w[j * d4 + v];  // world 1: staged by this step's gather
            else w = prow >= 0 ? pw_all[prow * d4 + v] : hw[hrow * d4 + v];
            if (adagrad) G = Gd[(int64_t)lk * d4 + v];
            opt4(w, G, acc, adagrad, lr, eps);
            if (sl >= 0) cw[(int64_t)sl * d4 + v] = w;
            else pw[j * d4 + v] = w;
            if (adagrad) Gd[(int64_t)lk * d4 + v] = G;
        }
        if (l == 0) {
            if (sl >= 0) nhot++;
            else ncold++;
            nin += __popc(mask & ~(1u << g));
            state[lk] = ST_UPDATED;
            last_upd[lk] = s;
            atomicAnd((unsigned long long*)&rbits[lk], (unsigned long long)clear);  // races with k_ingest_bits
            if (sl < 0) pool_idx[lk] = (int32_t)j;
            pkey[j] = sl < 0 ? lk : -1;
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *pcount = n;
    block_count(stats + FRUGAL_C_OPT_HOT, nhot);
    block_count(stats + FRUGAL_C_OPT_COLD, ncold);
    block_count(stats + FRUGAL_C_MAIL_IN, world > 1 ? nin : 0u);
}

void launch_optimizer(frugal_ctx* c, QueueSlot& q, int64_t s, int par, const float* recv, const int32_t* roff,
                      cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    int grid = grid_for(c->capT * gs, 256, 8);
    const int seg = (int)(s % c->P);
    const size_t pofs = (size_t)seg * c->capT * d4;
    const bool adag = c->cfg.opt == FRUGAL_ADAGRAD;
    (void)adag;
    const char* mail_par = c->n > 1 ? c->dh_mail + (size_t)par * c->n * c->mail_stride : nullptr;
    // world == 1: the owner gathered every touched row itself this step (T == uniq),
    // so the cold rows' w is taken from the staging rows instead of a second host read.
    const float4* rows_w = c->n == 1 ? (const float4*)c->rows_buf[s & 1] : nullptr;
    DISPATCH_GS(gs, (k_optimizer<GS><<<grid, 256, 0, st>>>(
                        q.T, q.nT, q.Tmask, q.Tidx, c->capT, c->n, c->g, d4, (int32_t)s, adag, c->cfg.lr, c->cfg.eps,
                        (const float4*)c->Pp, q.goff, mail_par, c->mail_stride, rows_w, c->slot, c->state,
                        c->last_upd, c->pool_idx, c->rbits, (float4*)c->cw, (float4*)c->Gd, (float4*)c->pw + pofs,
                        c->pkey + (size_t)seg * c->capT, c->pcount + seg, (const float4*)c->dh_w,
                        (const float4*)c->pw, c->P, (int32_t)std::max<int64_t>(0, s - c->P + 2),
                        (const float4*)recv, roff, c->hs, c->dstats)));
    c->launches++;
}

// ============================================================================ a12 final flush
__global__ void k_final_collect(int64_t No, int32_t* __restrict__ state, int32_t* rows, int32_t* cnt) {
    for (int64_t lk = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; lk < ((No + 31) / 32) * 32;
         lk += (int64_t)gridDim.x * blockDim.x) {
        bool dirty = lk < No && state[lk] != ST_CLEAN;
        if (dirty) state[lk] = ST_CLEAN;
        unsigned m = __ballot_sync(FULL, dirty);
        if (dirty) {
            int leader = __ffs(m) - 1, lane = threadIdx.x & 31, base = 0;
            if (lane == leader) base = atomicAdd(cnt, __popc(m));
            base = __shfl_sync(m, base, leader);
            rows[base + __popc(m & lanemask_lt())] = (int32_t)lk;
        }
    }
}
// G of every owned row (HBM) to the host table, once, at the end of training
template <int GS>
__global__ void k_g_push(int64_t No, int world, int g, int d4, const float4* __restrict__ Gd, float4* hG,
                         const int32_t* __restrict__ hs) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    for (int64_t lk = gid; lk < No; lk += gs) {
        const int64_t hk = host_row(hs, lk * world + g);
        for (int v = l; v < d4; v += GS) hG[hk * d4 + v] = Gd[lk * d4 + v];
    }
    block_fence_system();
}

void launch_final_flush(frugal_ctx* c, cudaStream_t st) {
    cudaMemsetAsync(c->ff_cnt, 0, sizeof(int32_t), st);
    k_final_collect<<<grid_for(c->No, 256, 8), 256, 0, st>>>(c->No, c->state, c->ff_rows, c->ff_cnt);
    c->launches++;
    launch_flush_rows(c, c->ff_rows, nullptr, c->ff_cnt, 1 << 30, FRUGAL_C_FINAL_HOT, st);
    if (c->cfg.opt == FRUGAL_ADAGRAD && c->No > 0 && c->dh_G) {
        const int d4 = c->d / 4, gs = group_size(d4);
        int grid = grid_for(c->No * gs, 256, 8);
        DISPATCH_GS(gs, (k_g_push<GS><<<grid, 256, 0, st>>>(c->No, c->n, c->g, d4, (const float4*)c->Gd,
                                                            (float4*)c->dh_G, c->hs)));
        c->launches++;
    }
}

// ============================================================================ initialisation
// w0[k][j] = init_scale * (2u - 1), u = top 24 bits of splitmix64(seed ^ (k*d + j)) / 2^24
__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
    z += 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
__device__ __forceinline__ float w0(uint64_t seed, int64_t k, int d, int j, float scale) {
    uint64_t h = splitmix64(seed ^ (uint64_t)(k * (int64_t)d + j));
    float u = (float)(h >> 40) * (1.0f / 16777216.0f);
    return __fmul_rn(scale, __fsub_rn(__fmul_rn(2.0f, u), 1.0f));
}

__global__ void k_init_table(float4* hw, float4* hG, int64_t N, int d, uint64_t seed, float scale, float accum,
                             const int32_t* __restrict__ hs) {
    const int d4 = d / 4;
    const int64_t total = N * d4;
    for (int64_t e0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e0 < total; e0 += (int64_t)gridDim.x * blockDim.x) {
        int64_t k = e0 / d4;
        int j = (int)(e0 - k * d4) * 4;
        const int64_t e = host_row(hs, k) * d4 + j / 4;  // row k lives in host slot hs[k]
        hw[e] = make_float4(w0(seed, k, d, j, scale), w0(seed, k, d, j + 1, scale), w0(seed, k, d, j + 2, scale),
                            w0(seed, k, d, j + 3, scale));
        if (hG) hG[e] = make_float4(accum, accum, accum, accum);
    }
}
void launch_init_table(frugal_ctx* c, cudaStream_t st) {
    k_init_table<<<kSMs * 8, 256, 0, st>>>((float4*)c->dh_w, (float4*)c->dh_G, c->N, c->d,
                                           c->cfg.init_seed, c->cfg.init_scale, c->cfg.init_accum, c->hs);
    c->launches++;
}

__global__ void k_fill(float* a, int64_t n, float v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}
__global__ void k_init_meta(int64_t No, int32_t* slot, int32_t* state, int32_t* last_upd, int32_t* pool_idx,
                            uint64_t* rbits) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < No; i += (int64_t)gridDim.x * blockDim.x) {
        slot[i] = -1;
        state[i] = ST_CLEAN;
        last_upd[i] = -1;
        pool_idx[i] = -1;
        rbits[i] = 0ull;
    }
}
// hot slots: d_hot_lk sorted owned local ids; cache rows start at w0 (same pure function)
__global__ void k_init_hot(const int32_t* __restrict__ hot_lk, int64_t cap_hot, int world, int g, int d,
                           uint64_t seed, float scale, int32_t* slot, float* cw) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < cap_hot * d;
         e += (int64_t)gridDim.x * blockDim.x) {
        int64_t sl = e / d;
        int j = (int)(e - sl * d);
        int64_t k = (int64_t)hot_lk[sl] * world + g;
        cw[e] = w0(seed, k, d, j, scale);
        if (j == 0) slot[hot_lk[sl]] = (int32_t)sl;
    }
}
void launch_init_meta(frugal_ctx* c, const int64_t* unused, int64_t n_hot, cudaStream_t st) {
    (void)unused;
    (void)n_hot;
    k_init_meta<<<grid_for(c->No, 256, 8), 256, 0, st>>>(c->No, c->slot, c->state, c->last_upd, c->pool_idx,
                                                          c->rbits);
    c->launches++;
    if (c->cap_hot > 0) {
        k_init_hot<<<grid_for(c->cap_hot * c->d, 256, 8), 256, 0, st>>>(
            c->hot_lk, c->cap_hot, c->n, c->g, c->d, c->cfg.init_seed, c->cfg.init_scale, c->slot, c->cw);
        c->launches++;
    }
    if (c->cfg.opt == FRUGAL_ADAGRAD) {
        k_fill<<<grid_for(c->No * c->d, 256, 8), 256, 0, st>>>(c->Gd, c->No * c->d, c->cfg.init_accum);
        c->launches++;
    }
}

// ============================================================================ cross-rank flags (host memory)
// flags layout: [which][rank] uint32, 16 words (64 B) apart
__global__ void k_set_flag(uint32_t* f, uint32_t v) {
    __threadfence_system();
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(f), "r"(v) : "memory");
}
__global__ void k_wait_flags(const uint32_t* f, int world, uint32_t v, int32_t* err) {
    int r = threadIdx.x;
    if (r < world) {
        const uint32_t* p = f + r * 16;
        uint64_t t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (true) {
            uint32_t x;
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(x) : "l"(p) : "memory");
            if ((int32_t)(x - v) >= 0) break;
            uint64_t t1;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            if (t1 - t0 > 120ull * 1000000000ull) {  // 120 s: a peer is gone
                atomicExch(err, 2);
                break;
            }
            __nanosleep(256);
        }
    }
    __syncwarp();
    // acquire only (each lane already loaded its flag with ld.acquire.sys): a fence.sc.sys here
    // would wait for every outstanding system-scope access of the GPU -- with the drain's
    // zero-copy stores in flight on the side stream that cost ~70 us per gate
    asm volatile("fence.acquire.sys;" ::: "memory");
}
// flag value from the ingest's parameter block (graph-replayed launches)
__global__ void k_set_flag_prm(uint32_t* f, const int32_t* __restrict__ prm) {
    __threadfence_system();
    const uint32_t v = (uint32_t)prm[IP_FLAGV];
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(f), "r"(v) : "memory");
}
__global__ void k_wait_flags_prm(const uint32_t* f, int world, const int32_t* __restrict__ prm, int32_t* err) {
    const uint32_t v = (uint32_t)prm[IP_FLAGV];
    int r = threadIdx.x;
    if (r < world) {
        const uint32_t* p = f + r * 16;
        uint64_t t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (true) {
            uint32_t x;
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(x) : "l"(p) : "memory");
            if ((int32_t)(x - v) >= 0) break;
            uint64_t t1;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            if (t1 - t0 > 120ull * 1000000000ull) {
                atomicExch(err, 2);
                break;
            }
            __nanosleep(256);
        }
    }
    __syncwarp();
    // acquire only (each lane already loaded its flag with ld.acquire.sys): a fence.sc.sys here
    // would wait for every outstanding system-scope access of the GPU -- with the drain's
    // zero-copy stores in flight on the side stream that cost ~70 us per gate
    asm volatile("fence.acquire.sys;" ::: "memory");
}
void launch_set_flag_prm(frugal_ctx* c, int which, const int32_t* prm, cudaStream_t st) {
    k_set_flag_prm<<<1, 1, 0, st>>>(c->dh_flags + (which * 32 + c->g) * 16, prm);
    c->launches++;
}
void launch_wait_flags_prm(frugal_ctx* c, int which, const int32_t* prm, cudaStream_t st) {
    k_wait_flags_prm<<<1, 32, 0, st>>>(c->dh_flags + which * 32 * 16, c->n, prm, c->err);
    c->launches++;
}

// wait (device side) until one host word reaches `value` (wrap-around compare)
void launch_wait_word(frugal_ctx* c, const uint32_t* dflag, uint32_t value, cudaStream_t st) {
    k_wait_flags<<<1, 32, 0, st>>>(dflag, 1, value, c->err);
    c->launches++;
}
void launch_set_flag(frugal_ctx* c, int which, uint32_t value, cudaStream_t st) {
    k_set_flag<<<1, 1, 0, st>>>(c->dh_flags + (which * 32 + c->g) * 16, value);
    c->launches++;
}
void launch_wait_flags(frugal_ctx* c, int which, uint32_t value, cudaStream_t st) {
    k_wait_flags<<<1, 32, 0, st>>>(c->dh_flags + which * 32 * 16, c->n, value, c->err);
    c->launches++;
}

// ============================================================================ comparison path (a2a)
__global__ void k_a2a_ids(const int32_t* __restrict__ uniq, const int32_t* __restrict__ gl, const int32_t* d_nu,
                          int32_t* __restrict__ ids) {
    const int n = *d_nu;
    for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < n; q += gridDim.x * blockDim.x) ids[q] = uniq[gl[q]];
}
// owner side: rows other ranks asked for (cache / pool / host, as k_gather_uniq)
template <int GS>
__global__ void k_serve_rows(const int32_t* __restrict__ ids, int64_t n, int world, int d4,
                             const int32_t* __restrict__ slot, const float4* __restrict__ cw, const float4* hw,
                             const int32_t* __restrict__ last_upd, const int32_t* __restrict__ pool_idx,
                             const float4* __restrict__ pw, int P, int64_t capT, int32_t pool_min,
                             const int32_t* __restrict__ hs, float4* __restrict__ out, unsigned long long* stats) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    unsigned nh = 0, nc = 0, np = 0;
    for (int64_t a = gid; a < n; a += gs) {
        const int32_t k = ids[a], lk = k / world;
        const float4* src = nullptr;
        const int sl = slot[lk];
        int kind = 0;
        if (sl >= 0) {
            src = cw + (int64_t)sl * d4;
            kind = 1;
        } else {
            const int32_t lu = last_upd[lk];
            if (lu >= 0 && lu >= pool_min) {
                src = pw + ((int64_t)(lu % P) * capT + pool_idx[lk]) * d4;
                kind = 2;
            }
        }
        if (kind == 0) src = hw + host_row(hs, k) * d4;
        if (l == 0) {
            nh += kind == 0;
            nc += kind == 1;
            np += kind == 2;
        }
        for (int v = l; v < d4; v += GS) out[a * d4 + v] = src[v];
    }
    block_count(stats + FRUGAL_C_GATHER_HOST, nh);
    block_count(stats + FRUGAL_C_GATHER_CACHE, nc);
    block_count(stats + FRUGAL_C_GATHER_POOL, np);
}
template <int GS>
__global__ void k_a2a_place(const int32_t* __restrict__ gl, const int32_t* d_nu, int d4,
                            const float4* __restrict__ in, float4* __restrict__ rows) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n = *d_nu;
    for (int64_t q = gid; q < n; q += gs)
        for (int v = l; v < d4; v += GS) rows[(int64_t)gl[q] * d4 + v] = in[q * d4 + v];
}

void launch_a2a_ids(frugal_ctx* c, QueueSlot& q, int32_t* ids, cudaStream_t st) {
    k_a2a_ids<<<grid_for(c->M, 256, 4), 256, 0, st>>>(q.uniq, q.gl, q.n_uniq, ids);
    c->launches++;
}
void launch_serve_rows(frugal_ctx* c, const int32_t* ids, int64_t n, int64_t s, float* out, cudaStream_t st) {
    if (n <= 0) return;
    const int d4 = c->d / 4, gs = group_size(d4);
    int grid = std::min(grid_for(n * gs, 256, 8), c->gather_blocks);
    const int32_t pool_min = (int32_t)std::max<int64_t>(0, s - c->P + 2);
    DISPATCH_GS(gs, (k_serve_rows<GS><<<grid, 256, 0, st>>>(ids, n, c->n, d4, c->slot, (const float4*)c->cw,
                                                            (const float4*)c->dh_w, c->last_upd, c->pool_idx,
                                                            (const float4*)c->pw, c->P, c->capT, pool_min, c->hs,
                                                            (float4*)out, c->dstats)));
    c->launches++;
}
void launch_a2a_place(frugal_ctx* c, QueueSlot& q, const float* in, float* rows, cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    DISPATCH_GS(gs, (k_a2a_place<GS><<<grid_for((int64_t)c->M * gs, 256, 8), 256, 0, st>>>(
                        q.gl, q.n_uniq, d4, (const float4*)in, (float4*)rows)));
    c->launches++;
}

// ============================================================================ introspection
// authoritative value of owned rows: hot -> cache; cold & dirty -> pool; else host
__global__ void k_read_rows(const int32_t* __restrict__ lks, int64_t n, int world, int g, int d, int P, int64_t capT,
                            const int32_t* slot, const int32_t* state, const int32_t* last_upd,
                            const int32_t* pool_idx, const float* cw, const float* Gd, const float* pw,
                            const float* hw, const int32_t* __restrict__ hs, float* ow, float* oG) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n * d; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = e / d;
        int j = (int)(e - a * d);
        int32_t lk = lks[a];
        int64_t k = (int64_t)lk * world + g;
        int sl = slot[lk];
        float w;
        if (sl >= 0) {
            w = cw[(int64_t)sl * d + j];
        } else if (state[lk] == ST_UPDATED || state[lk] == ST_INF) {
            int64_t pr = (int64_t)(last_upd[lk] % P) * capT + pool_idx[lk];
            w = pw[pr * d + j];
        } else {
            w = hw[host_row(hs, k) * d + j];
        }
        float G = Gd ? Gd[(int64_t)lk * d + j] : 0.f;
        ow[e] = w;
        oG[e] = G;
    }
}
void launch_read_rows(frugal_ctx* c, const int32_t* d_lk, int64_t n, float* d_w, float* d_G, cudaStream_t st) {
    const bool ad = c->cfg.opt == FRUGAL_ADAGRAD;
    k_read_rows<<<grid_for(n * c->d, 256, 8), 256, 0, st>>>(d_lk, n, c->n, c->g, c->d, c->P, c->capT, c->slot,
                                                             c->state, c->last_upd, c->pool_idx, c->cw,
                                                             ad ? c->Gd : nullptr, c->pw, c->dh_w, c->hs, d_w, d_G);
    c->launches++;
}
__global__ void k_read_host(const int64_t* __restrict__ ks, int64_t n, int d, const float* hw, const float* hG,
                            const int32_t* __restrict__ hs, float* ow, float* oG) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n * d; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = e / d;
        int j = (int)(e - a * d);
        const int64_t hk = host_row(hs, ks[a]);
        ow[e] = hw[hk * d + j];
        oG[e] = hG ? hG[hk * d + j] : 0.f;
    }
}
void launch_read_host(frugal_ctx* c, const int64_t* d_k, int64_t n, float* d_w, float* d_G, cudaStream_t st) {
    k_read_host<<<grid_for(n * c->d, 256, 8), 256, 0, st>>>(d_k, n, c->d, c->dh_w, c->dh_G, c->hs, d_w, d_G);
    c->launches++;
}

}  // namespace frugal
