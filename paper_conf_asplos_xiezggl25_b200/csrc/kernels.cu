// kernels.cu -- sm_100a kernels of the Frugal step (CUDA path; shares nothing with oracle/).
//
// Every kernel here is HBM- or host-link-bound integer / fp32 copy work; nothing is a
// dense contraction, so there are no tensor-core paths.  Rows are
// moved as float4 by "row groups" of GS lanes (GS = pow2 >= d/4, capped at 32) so a
// 128-byte d=32 row is one coalesced 8-lane access; host-table rows are read/written
// with zero-copy loads/stores through the mapped alias of the pinned shm table
// (§3.1: "fuses the local GPU cache access and host memory access
// into one GPU kernel ... zero-copy").
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "frugal_internal.cuh"
#include "kutil.cuh"

namespace frugal {

// ============================================================================ block scan helpers
// exclusive scan of one int per thread over a 256-thread block; returns total in *tot
__device__ __forceinline__ int block_excl_scan(int v, int* sm_w /*[8]*/, int* tot) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) sm_w[w] = x;
    __syncthreads();
    int base = 0, all = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        int c = sm_w[i];
        if (i < w) base += c;
        all += c;
    }
    __syncthreads();
    *tot = all;
    return base + x - v;
}

// single-block exclusive scan of a small int array in place; writes the total
__global__ void k_scan_small(int32_t* a, int len, int32_t* total) {
    __shared__ int sm[32];
    const int t = threadIdx.x, nt = blockDim.x;
    int per = (len + nt - 1) / nt, lo = min(len, t * per), hi = min(len, lo + per);
    int s = 0;
    for (int i = lo; i < hi; i++) s += a[i];
    // block exclusive scan (1024 threads)
    const int lane = t & 31, w = t >> 5;
    int x = s;
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) sm[w] = x;
    __syncthreads();
    if (w == 0) {
        int v = (lane < (nt >> 5)) ? sm[lane] : 0;
        int z = v;
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(FULL, z, o);
            if (lane >= o) z += y;
        }
        sm[lane] = z - v;
        if (lane == 31 && total) *total = z;
    }
    __syncthreads();
    int run = sm[w] + x - s;
    for (int i = lo; i < hi; i++) {
        int c = a[i];
        a[i] = run;
        run += c;
    }
}

// ============================================================================ radix sort
// Stable LSD radix sort, 9-bit digits (3 passes for the 26-bit ids of Criteo-Kaggle).
// Per pass: k_radix_hist (per-block digit counts, digit-major), k_radix_scan_rows (one
// block per digit: exclusive scan over blocks + digit total), k_radix_scatter (each block
// derives the digit bases from the totals, then ranks its tiles stably with
// __match_any_sync and scatters).  All counts are device-resident.
constexpr int kRadixBits = 9;
constexpr int kDigits = 1 << kRadixBits;

__global__ void k_radix_hist(const uint32_t* __restrict__ keys, const int32_t* d_n, int shift,
                             int32_t* hist, int nblk) {
    __shared__ int h[kDigits];
    for (int i = threadIdx.x; i < kDigits; i += blockDim.x) h[i] = 0;
    __syncthreads();
    int lo, hi;
    chunk_range(*d_n, nblk, blockIdx.x, lo, hi);
    for (int i = lo + threadIdx.x; i < hi; i += blockDim.x) atomicAdd(&h[(keys[i] >> shift) & (kDigits - 1)], 1);
    __syncthreads();
    for (int i = threadIdx.x; i < kDigits; i += blockDim.x) hist[(size_t)i * nblk + blockIdx.x] = h[i];
}

// block dg: exclusive scan of hist[dg][0..nblk) in place, total -> tot[dg]
__global__ void k_radix_scan_rows(int32_t* __restrict__ hist, int nblk, int32_t* __restrict__ tot) {
    __shared__ int smw[8];
    int32_t* row = hist + (size_t)blockIdx.x * nblk;
    int run = 0;
    for (int b0 = 0; b0 < nblk; b0 += blockDim.x) {
        int i = b0 + threadIdx.x;
        int v = i < nblk ? row[i] : 0;
        int t;
        int ex = block_excl_scan(v, smw, &t);
        if (i < nblk) row[i] = run + ex;
        run += t;
    }
    if (threadIdx.x == 0) tot[blockIdx.x] = run;
}

// Super-tiles of kSub * 256 keys: warp w ranks its kSub consecutive 32-key sub-tiles in
// order with __match_any_sync and a running per-warp digit count, then one block-wide
// prefix over the 8 warps per digit places all of them -- the digit-count zeroing and
// prefix (8 x 512 counters) are paid once per 1024 keys instead of once per 256.
constexpr int kSub = 4;
__global__ void __launch_bounds__(256) k_radix_scatter(const uint32_t* __restrict__ kin, const int32_t* __restrict__ vin,
                                uint32_t* __restrict__ kout, int32_t* __restrict__ vout, const int32_t* d_n,
                                int shift, const int32_t* __restrict__ hist, const int32_t* __restrict__ dtot,
                                int nblk) {
    __shared__ int run[kDigits];
    __shared__ int wcnt[8][kDigits];
    __shared__ int tot[kDigits];
    __shared__ int smw[8];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    {   // digit bases: exclusive scan of the digit totals (2 digits per thread)
        int a0 = dtot[2 * tid], a1 = dtot[2 * tid + 1], t;
        int ex = block_excl_scan(a0 + a1, smw, &t);
        run[2 * tid] = ex + hist[(size_t)(2 * tid) * nblk + blockIdx.x];
        run[2 * tid + 1] = ex + a0 + hist[(size_t)(2 * tid + 1) * nblk + blockIdx.x];
    }
    int lo, hi;
    chunk_range(*d_n, nblk, blockIdx.x, lo, hi);
    for (int base = lo; base < hi; base += kTile * kSub) {
#pragma unroll
        for (int i = 0; i < 8; i++) {
            wcnt[i][tid] = 0;
            wcnt[i][tid + 256] = 0;
        }
        __syncthreads();
        // warp w: keys [base + w*32*kSub, +32*kSub), sub-tile j = 32 consecutive keys
        uint32_t key[kSub];
        int32_t val[kSub];
        int dg[kSub], loc[kSub];
#pragma unroll
        for (int j = 0; j < kSub; j++) {
            const int i = base + (w * kSub + j) * 32 + lane;
            const bool valid = i < hi;
            key[j] = valid ? kin[i] : 0u;
            val[j] = valid ? vin[i] : 0;
            dg[j] = valid ? (int)((key[j] >> shift) & (kDigits - 1)) : -1;
        }
#pragma unroll
        for (int j = 0; j < kSub; j++) {
            const unsigned peers = __match_any_sync(FULL, dg[j]);
            const int rank = __popc(peers & lanemask_lt());
            loc[j] = dg[j] >= 0 ? wcnt[w][dg[j]] + rank : 0;  // keys of this digit in earlier sub-tiles
            __syncwarp();
            if (dg[j] >= 0 && rank == 0) wcnt[w][dg[j]] += __popc(peers);
            __syncwarp();
        }
        __syncthreads();
#pragma unroll
        for (int h = 0; h < 2; h++) {  // per digit: exclusive prefix over the warps
            const int d = tid + h * 256;
            int acc = 0;
#pragma unroll
            for (int q = 0; q < 8; q++) {
                int c = wcnt[q][d];
                wcnt[q][d] = acc;
                acc += c;
            }
            tot[d] = acc;
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kSub; j++) {
            if (dg[j] >= 0) {
                const int dst = run[dg[j]] + wcnt[w][dg[j]] + loc[j];
                kout[dst] = key[j];
                vout[dst] = val[j];
            }
        }
        __syncthreads();
        run[tid] += tot[tid];
        run[tid + 256] += tot[tid + 256];
    }
}

void sort_alloc(SortScratch& s, int64_t cap) {
    s.cap = cap < 1 ? 1 : cap;
    for (int i = 0; i < 2; i++) {
        cudaMalloc(&s.k[i], s.cap * sizeof(uint32_t));
        cudaMalloc(&s.v[i], s.cap * sizeof(int32_t));
    }
    s.nblk = grid_for(s.cap, kTile * 4, 2);
    cudaMalloc(&s.hist, ((size_t)kDigits * s.nblk + kDigits) * sizeof(int32_t));
}
void sort_free(SortScratch& s) {
    for (int i = 0; i < 2; i++) {
        cudaFree(s.k[i]);
        cudaFree(s.v[i]);
    }
    cudaFree(s.hist);
    s = SortScratch();
}

int sort_pairs(SortScratch& s, const int32_t* d_n, int bits, cudaStream_t st, int64_t* launches) {
    int cur = 0;
    int32_t* tot = s.hist + (size_t)kDigits * s.nblk;
    for (int shift = 0; shift < bits; shift += kRadixBits) {
        k_radix_hist<<<s.nblk, 256, 0, st>>>(s.k[cur], d_n, shift, s.hist, s.nblk);
        k_radix_scan_rows<<<kDigits, 256, 0, st>>>(s.hist, s.nblk, tot);
        k_radix_scatter<<<s.nblk, 256, 0, st>>>(s.k[cur], s.v[cur], s.k[cur ^ 1], s.v[cur ^ 1], d_n, shift,
                                                s.hist, tot, s.nblk);
        *launches += 3;
        cur ^= 1;
    }
    return cur;
}

void scan_alloc(ScanScratch& s, int64_t cap) {
    s.nblk = grid_for(cap < 1 ? 1 : cap, kTile * 4, 2);
    cudaMalloc(&s.part, ((size_t)s.nblk * 33 + 1) * sizeof(int32_t));
}
void scan_free(ScanScratch& s) {
    cudaFree(s.part);
    s = ScanScratch();
}

// ============================================================================ ingest: ids
// int64 ids of all ranks -> int32 ring copy (validated) + this rank's sort input
__global__ void k_convert_ids(const int64_t* __restrict__ ids64, int32_t* __restrict__ ids32,
                              const int32_t* __restrict__ counts, int world, int M, int F, int64_t N,
                              int g, uint32_t* __restrict__ sk, int32_t* __restrict__ sv,
                              int32_t* __restrict__ d_m, int32_t* err, int own_only) {
    // err lives in mapped pinned host memory: the host sees a bad id without a sync.
    // own_only (ingest v2): only rank g's row of ids64 / ids32 exists and is converted
    const int64_t total = own_only ? (int64_t)M : (int64_t)world * M;
    for (int64_t e0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e0 < total;
         e0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t e = own_only ? (int64_t)g * M + e0 : e0;
        int r = (int)(e / M), i = (int)(e - (int64_t)r * M);
        if (i >= counts[r] * F) continue;
        int64_t k = ids64[e];
        if (k < 0 || k >= N) {
            atomicExch(err, 1);
            k = 0;
        }
        ids32[e] = (int32_t)k;
        if (r == g) {
            sk[i] = (uint32_t)k;
            sv[i] = i;
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *d_m = counts[g] * F;
}

// ============================================================================ dedup emit
// sorted (key, pos) -> uniq ascending, CSR (off, pos), inv
__global__ void k_head_count(const uint32_t* __restrict__ ks, const int32_t* d_n, int32_t* part, int nblk) {
    __shared__ int sm[8];
    int lo, hi;
    chunk_range(*d_n, nblk, blockIdx.x, lo, hi);
    int c = 0;
    for (int i = lo + threadIdx.x; i < hi; i += blockDim.x) c += (i == 0 || ks[i] != ks[i - 1]);
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
    if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int i = 0; i < 8; i++) t += sm[i];
        part[blockIdx.x] = t;
    }
}

__global__ void k_dedup_emit(const uint32_t* __restrict__ ks, const int32_t* __restrict__ vs, const int32_t* d_n,
                             const int32_t* __restrict__ part, int nblk, int32_t* __restrict__ uniq,
                             int32_t* __restrict__ off, int32_t* __restrict__ inv, int32_t* __restrict__ pos,
                             int32_t* d_nuniq, unsigned long long* stats) {
    __shared__ int smw[8];
    const int n = *d_n;
    int lo, hi;
    chunk_range(n, nblk, blockIdx.x, lo, hi);
    int run = part[blockIdx.x];
    for (int base = lo; base < hi; base += kTile) {
        const int i = base + threadIdx.x;
        const bool valid = i < hi;
        uint32_t key = valid ? ks[i] : 0u;
        int head = valid && (i == 0 || ks[i - 1] != key);
        int tot;
        int ex = block_excl_scan(head, smw, &tot);
        if (valid) {
            int seg = run + ex + head - 1;
            if (head) {
                uniq[seg] = (int32_t)key;
                off[seg] = i;
            }
            int p = vs[i];
            pos[i] = p;
            inv[p] = seg;
            if (i == n - 1) {
                off[seg + 1] = n;
                *d_nuniq = seg + 1;
                atomicAdd(&stats[FRUGAL_C_POSITIONS], (unsigned long long)n);
                atomicAdd(&stats[FRUGAL_C_UNIQUE], (unsigned long long)(seg + 1));
            }
        }
        run += tot;
    }
    if (n == 0 && blockIdx.x == 0 && threadIdx.x == 0) {
        off[0] = 0;
        *d_nuniq = 0;
    }
}

void launch_convert_ids(frugal_ctx* c, QueueSlot& q, cudaStream_t st) {
    int64_t total = (int64_t)c->n * c->M;
    if (c->own_ids) total = c->M;
    k_convert_ids<<<grid_for(total, 256), 256, 0, st>>>(c->ids_stage, q.ids, q.counts, c->n, c->M, c->F, c->N,
                                                         c->g, c->sort.k[0], c->sort.v[0], q.m, c->err,
                                                         c->own_ids ? 1 : 0);
    c->launches++;
}

// own-rank dedup of the sample-queue slot: keys were staged by k_convert_ids, count in owned_cnt
void launch_dedup(frugal_ctx* c, QueueSlot& q, cudaStream_t st) {
    int r = sort_pairs(c->sort, q.m, c->key_bits, st, &c->launches);
    int nb = c->scan.nblk;
    k_head_count<<<nb, 256, 0, st>>>(c->sort.k[r], q.m, c->scan.part, nb);
    k_scan_small<<<1, 1024, 0, st>>>(c->scan.part, nb, nullptr);
    k_dedup_emit<<<nb, 256, 0, st>>>(c->sort.k[r], c->sort.v[r], q.m, c->scan.part, nb, q.uniq, q.off,
                                     q.inv, q.pos, q.n_uniq, c->dstats);
    c->launches += 3;
}

// ============================================================================ owner side (world > 1)
// owned entries of all ranks -> composite key (lk * world + r), stable compaction
__global__ void k_owned_count(const int32_t* __restrict__ ids32, const int32_t* __restrict__ counts, int world,
                              int M, int F, int g, int32_t* part, int nblk) {
    __shared__ int sm[8];
    int total = world * M, lo, hi;
    chunk_range(total, nblk, blockIdx.x, lo, hi);
    int cnt = 0;
    for (int e = lo + threadIdx.x; e < hi; e += blockDim.x) {
        int r = e / M, i = e - r * M;
        cnt += (i < counts[r] * F) && (ids32[e] % world == g);
    }
    for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(FULL, cnt, o);
    if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = cnt;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int i = 0; i < 8; i++) t += sm[i];
        part[blockIdx.x] = t;
    }
}

__global__ void k_owned_emit(const int32_t* __restrict__ ids32, const int32_t* __restrict__ counts, int world,
                             int M, int F, int g, const int32_t* __restrict__ part, int nblk,
                             uint32_t* __restrict__ sk, int32_t* __restrict__ sv, int32_t* d_cnt) {
    __shared__ int smw[8];
    int total = world * M, lo, hi;
    chunk_range(total, nblk, blockIdx.x, lo, hi);
    int run = part[blockIdx.x];
    for (int base = lo; base < hi; base += kTile) {
        int e = base + threadIdx.x;
        int own = 0, r = 0, k = 0;
        if (e < hi) {
            r = e / M;
            int i = e - r * M;
            if (i < counts[r] * F) {
                k = ids32[e];
                own = (k % world == g);
            }
        }
        int tot;
        int ex = block_excl_scan(own, smw, &tot);
        if (own) {
            sk[run + ex] = (uint32_t)(k / world) * (uint32_t)world + (uint32_t)r;
            sv[run + ex] = r;
        }
        run += tot;
    }
    if (blockIdx.x == nblk - 1 && threadIdx.x == 0) *d_cnt = run;
}

// unique (lk, r) pairs sorted by (lk, r) -> per-block counts of (lk heads, rank r pairs)
__global__ void k_pairs_count(const uint32_t* __restrict__ ks, const int32_t* d_n, int world, int32_t* part,
                              int nblk) {
    // part layout: [(world+1)][nblk], counter 0 = lk heads, 1+r = pairs of rank r
    __shared__ int sm[33];
    if (threadIdx.x < 33) sm[threadIdx.x] = 0;
    __syncthreads();
    int lo, hi;
    chunk_range(*d_n, nblk, blockIdx.x, lo, hi);
    for (int i = lo + threadIdx.x; i < hi; i += blockDim.x) {
        uint32_t key = ks[i];
        bool pair_head = (i == 0 || ks[i - 1] != key);
        if (!pair_head) continue;
        uint32_t lk = key / world;
        bool lk_head = (i == 0 || ks[i - 1] / world != lk);
        if (lk_head) atomicAdd(&sm[0], 1);
        atomicAdd(&sm[1 + key % world], 1);
    }
    __syncthreads();
    if (threadIdx.x <= world) part[threadIdx.x * nblk + blockIdx.x] = sm[threadIdx.x];
}

__global__ void k_pairs_emit(const uint32_t* __restrict__ ks, const int32_t* d_n, int world, const int32_t* part,
                             int nblk, int capT, int32_t* __restrict__ T, uint32_t* __restrict__ Tmask,
                             int32_t* __restrict__ Tidx, int32_t* d_nT) {
    __shared__ int smw[8];
    __shared__ int run[33];
    const int n = *d_n;
    if (threadIdx.x <= world) run[threadIdx.x] = part[threadIdx.x * nblk + blockIdx.x];
    __syncthreads();
    int lo, hi;
    chunk_range(n, nblk, blockIdx.x, lo, hi);
    for (int base = lo; base < hi; base += kTile) {
        int i = base + threadIdx.x;
        bool valid = i < hi;
        uint32_t key = valid ? ks[i] : 0u;
        bool ph = valid && (i == 0 || ks[i - 1] != key);
        uint32_t lk = key / world;
        int r = (int)(key % world);
        bool lh = ph && (i == 0 || ks[i - 1] / world != lk);
        int tot;
        int ex = block_excl_scan(lh ? 1 : 0, smw, &tot);
        int j = run[0] + ex + (lh ? 1 : 0) - 1;  // T index of this pair
        // rank-local index: exclusive count of earlier pairs of rank r
        int ridx = 0;
        for (int q = 0; q < world; q++) {
            int t2;
            int e2 = block_excl_scan((ph && r == q) ? 1 : 0, smw, &t2);
            if (q == r) ridx = run[1 + q] + e2;
            __syncthreads();
            if (threadIdx.x == 0) run[1 + q] += t2;
        }
        if (ph) {
            if (lh) T[j] = (int32_t)lk;
            atomicOr(&Tmask[j], 1u << r);
            Tidx[(int64_t)r * capT + j] = ridx;
        }
        __syncthreads();
        if (threadIdx.x == 0) run[0] += tot;
        __syncthreads();
    }
    if (blockIdx.x == nblk - 1 && threadIdx.x == 0) *d_nT = run[0];
}

// grouping of this rank's uniq by owner: owner keys for a 1-pass stable sort
__global__ void k_owner_keys(const int32_t* __restrict__ uniq, const int32_t* d_nu, int world,
                             uint32_t* __restrict__ sk, int32_t* __restrict__ sv) {
    int n = *d_nu;
    for (int u = blockIdx.x * blockDim.x + threadIdx.x; u < n; u += gridDim.x * blockDim.x) {
        sk[u] = (uint32_t)(uniq[u] % world);
        sv[u] = u;
    }
}
__global__ void k_goff(const uint32_t* __restrict__ sk, const int32_t* d_nu, int world, int32_t* goff) {
    int o = threadIdx.x;
    if (o > world) return;
    int n = *d_nu, lo = 0, hi = n;
    while (lo < hi) {  // lower_bound of o
        int mid = (lo + hi) >> 1;
        if ((int)sk[mid] < o) lo = mid + 1;
        else hi = mid;
    }
    goff[o] = lo;
}
__global__ void k_copy_i32(const int32_t* __restrict__ a, int32_t* __restrict__ b, const int32_t* d_n) {
    int n = *d_n;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) b[i] = a[i];
}

// ---------------------------------------------------------------------------- ingest v2 (FRUGAL_F_OWN_IDS)
// (1) this rank's distinct ids of step t, grouped by owner (gl, goff), to its id-mailbox slot:
// [goff[0..world]] in a 256-B header, then the ids (coalesced zero-copy stores, sequential)
__global__ void k_idbox_write(const int32_t* __restrict__ uniq, const int32_t* __restrict__ gl,
                              const int32_t* __restrict__ goff, const int32_t* d_nu, int world, char* boxes,
                              size_t stride, int g, const int32_t* __restrict__ prm) {
    char* box = boxes + ((size_t)prm[IP_IDSLOT] * world + g) * stride;
    const int n = *d_nu;
    int32_t* hdr = (int32_t*)box;
    int32_t* ids = (int32_t*)(box + 256);
    if (blockIdx.x == 0 && threadIdx.x <= world) hdr[threadIdx.x] = goff[threadIdx.x];
    for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < n; q += gridDim.x * blockDim.x) ids[q] = uniq[gl[q]];
    block_fence_system();
}
// (2) every rank r's segment of ids owned by this rank g (ascending), as composite sort keys
// (lk * world + r) -- the same key set k_owned_emit builds from all ranks' raw ids, minus the
// duplicates; one block per rank r (segment offsets from the world headers)
__global__ void k_idbox_gather(const char* boxes0, size_t stride, int world, int g, uint32_t* __restrict__ sk,
                               int32_t* __restrict__ sv, int32_t* d_cnt, const int32_t* __restrict__ prm) {
    const char* boxes = boxes0 + (size_t)prm[IP_IDSLOT] * world * stride;
    const int r = blockIdx.x;
    int base = 0, total = 0;
    for (int q = 0; q < world; q++) {
        const int32_t* h = (const int32_t*)(boxes + (size_t)q * stride);
        const int len = h[g + 1] - h[g];
        if (q < r) base += len;
        total += len;
    }
    const int32_t* h = (const int32_t*)(boxes + (size_t)r * stride);
    const int b = h[g], len = h[g + 1] - h[g];
    const int32_t* ids = (const int32_t*)(boxes + (size_t)r * stride + 256);
    for (int i = threadIdx.x; i < len; i += blockDim.x) {
        const uint32_t k = (uint32_t)ids[b + i];
        sk[base + i] = (k / (uint32_t)world) * (uint32_t)world + (uint32_t)r;
        sv[base + i] = r;
    }
    if (r == 0 && threadIdx.x == 0) *d_cnt = total;
}

static void owner_group(frugal_ctx* c, QueueSlot& q, cudaStream_t st) {
    // this rank's uniq grouped by owner (stable 1-pass partition): gl, goff
    const int n = c->n;
    k_owner_keys<<<grid_for(c->M, 256), 256, 0, st>>>(q.uniq, q.n_uniq, n, c->sort.k[0], c->sort.v[0]);
    int obits = 1;
    while ((1 << obits) < n) obits++;
    int r2 = sort_pairs(c->sort, q.n_uniq, obits, st, &c->launches);
    k_copy_i32<<<grid_for(c->M, 256), 256, 0, st>>>(c->sort.v[r2], q.gl, q.n_uniq);
    k_goff<<<1, 64, 0, st>>>(c->sort.k[r2], q.n_uniq, n, q.goff);
    c->launches += 3;
}
static void owner_pairs(frugal_ctx* c, QueueSlot& q, cudaStream_t st) {
    // composite keys (lk, r) in sort.k[0] (count owned_cnt) -> T, Tmask, Tidx
    const int n = c->n;
    const int nb = c->scan.nblk;
    int bits = 1;
    while ((((int64_t)1) << bits) < ((c->No + 1) * (int64_t)n)) bits++;
    int r = sort_pairs(c->sort, c->owned_cnt, bits, st, &c->launches);
    k_pairs_count<<<nb, 256, 0, st>>>(c->sort.k[r], c->owned_cnt, n, c->scan.part, nb);
    for (int qq = 0; qq <= n; qq++) {
        k_scan_small<<<1, 1024, 0, st>>>(c->scan.part + (size_t)qq * nb, nb, nullptr);
        c->launches++;
    }
    k_pairs_emit<<<nb, 256, 0, st>>>(c->sort.k[r], c->owned_cnt, n, c->scan.part, nb, (int)c->capT, q.T, q.Tmask,
                                     q.Tidx, q.nT);
    c->launches += 2;
}
void launch_owner_side_v2(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st) {
    const int n = c->n;
    cudaMemsetAsync(q.Tmask, 0, c->capT * sizeof(uint32_t), st);
    owner_group(c, q, st);
    k_idbox_write<<<grid_for(c->M, 256, 2), 256, 0, st>>>(q.uniq, q.gl, q.goff, q.n_uniq, n, c->dh_idbox,
                                                          c->idbox_stride, c->g, prm);
    c->launches++;
    launch_set_flag_prm(c, FLAG_IDS_KIND, prm, st);
    launch_wait_flags_prm(c, FLAG_IDS_KIND, prm, st);  // every rank's ids of step t are out
    k_idbox_gather<<<n, 256, 0, st>>>(c->dh_idbox, c->idbox_stride, n, c->g, c->sort.k[0], c->sort.v[0],
                                      c->owned_cnt, prm);
    c->launches++;
    owner_pairs(c, q, st);
}

void launch_owner_side(frugal_ctx* c, QueueSlot& q, int64_t t, cudaStream_t st) {
    (void)t;
    const int n = c->n;
    const int nb = c->scan.nblk;
    // (1) owned entries of all ranks, composite key (lk, r)
    cudaMemsetAsync(q.Tmask, 0, c->capT * sizeof(uint32_t), st);
    k_owned_count<<<nb, 256, 0, st>>>(q.ids, q.counts, n, c->M, c->F, c->g, c->scan.part, nb);
    k_scan_small<<<1, 1024, 0, st>>>(c->scan.part, nb, nullptr);
    k_owned_emit<<<nb, 256, 0, st>>>(q.ids, q.counts, n, c->M, c->F, c->g, c->scan.part, nb, c->sort.k[0],
                                     c->sort.v[0], c->owned_cnt);
    c->launches += 3;
    owner_pairs(c, q, st);
    owner_group(c, q, st);
}
// ============================================================================ scheduler (P2F)
// warp-aggregated append of (row, p) to the newly-bucketed list
__device__ __forceinline__ void nb_append(int32_t* rows, int32_t* ps, int32_t* cnt, bool pred, int32_t lk,
                                          int32_t p) {
    unsigned m = __ballot_sync(__activemask(), pred);
    if (!pred) return;
    int leader = __ffs(m) - 1, lane = threadIdx.x & 31;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(m));
    base = __shfl_sync(m, base, leader);
    int at = base + __popc(m & lanemask_lt());
    rows[at] = lk;
    ps[at] = p;
}

// zero the AdjustPriority list count the ingest of this step appends to (by parity, prm)
__global__ void k_ingest_prologue(const int32_t* __restrict__ prm, int32_t* cnt0, int32_t* cnt1) {
    *(prm[IP_APAR] ? cnt1 : cnt0) = 0;
}
void launch_ingest_prologue(frugal_ctx* c, const int32_t* prm, cudaStream_t st) {
    k_ingest_prologue<<<1, 1, 0, st>>>(prm, c->adj_cnt[0], c->adj_cnt[1]);
    c->launches++;
}

// a1: set read-ring bits of step t for the owned rows read at t; AdjustPriority inf -> t.
// t, the adjust switch, the list parity and the hot map of t's epoch come from prm
__global__ void k_ingest_bits(const int32_t* __restrict__ T, const uint32_t* __restrict__ Tmask,
                              const int32_t* d_nT, int world, int g, const int32_t* __restrict__ prm,
                              const int32_t* __restrict__ slot, const uint32_t* __restrict__ hmap0,
                              const uint32_t* __restrict__ hmap1, uint64_t* __restrict__ rbits,
                              int32_t* __restrict__ state, int32_t* rows0, int32_t* p0, int32_t* cnt0,
                              int32_t* rows1, int32_t* p1, int32_t* cnt1) {
    const int32_t t = prm[IP_T];
    const int bit = t & 31, adjust = prm[IP_ADJUST], par = prm[IP_APAR], hm = prm[IP_HMAP];
    const uint32_t* hmap = hm < 0 ? nullptr : (hm ? hmap1 : hmap0);
    int32_t* nb_rows = par ? rows1 : rows0;
    int32_t* nb_p = par ? p1 : p0;
    int32_t* nb_cnt = par ? cnt1 : cnt0;
    int n = *d_nT;
    int nloop = (n + blockDim.x * gridDim.x - 1) / (blockDim.x * gridDim.x) * (blockDim.x * gridDim.x);
    for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < nloop; j += gridDim.x * blockDim.x) {
        bool valid = j < n;
        bool app = false;
        int32_t lk = 0;
        if (valid) {
            lk = T[j];
            uint32_t mask = (world > 1) ? Tmask[j] : 1u;
            // host-reader (R7): any other rank, or the owner itself when the row is not
            // hot at step t (hmap: the hot set of t's epoch, N3; else the static cache)
            const bool hot = hmap ? ((hmap[lk >> 5] >> (lk & 31)) & 1u) != 0u : slot[lk] >= 0;
            bool host = (mask & ~(1u << g)) != 0u || !hot;
            uint64_t b = (1ull << bit) | (host ? (1ull << (32 + bit)) : 0ull);
            atomicOr((unsigned long long*)&rbits[lk], (unsigned long long)b);  // races with k_optimizer's clear
            if (adjust && state[lk] == ST_INF) {
                if (host) {
                    state[lk] = ST_CLEAN;
                    app = true;
                } else {
                    state[lk] = ST_EXEMPT;
                }
            }
        }
        nb_append(nb_rows, nb_p, nb_cnt, app, lk, t);
    }
}

// a9 + a11 scheduler of step s, one kernel.  Three inputs, one virtual index range:
//  [0, nA)        rows updated at s-1 (T(s-1)): priority = next access step within
//                 [s, s+L-1] (Eq. (1)) read off the read ring; host-read there
//                 -> flush class by deadline; owner-only hot read -> EXEMPT; none -> INF;
//  [nA, nA+nB)    rows AdjustPriority'd inf -> s+L-1 by the ingest of that step;
//  [nA+nB, ...)   age-out candidates: cold rows of pool segment s-1-D still INF.
// Level 1 of the two-level PQ (§3.4) is the deadline relative to s; the drain policy (R9)
// needs three of its classes: 0 urgent (p == s), 1 next (p == s+1), 2 later (p > s+1),
// plus 3 = age-out.  Rows are appended to the four lists with warp-aggregated atomics.
__global__ void k_schedule(const int32_t* __restrict__ T, const int32_t* d_nT, const int32_t* __restrict__ adj_rows,
                           const int32_t* __restrict__ adj_p, const int32_t* adj_cnt,
                           const int32_t* __restrict__ pkey, const int32_t* pcount_seg, int32_t u_age, int32_t s,
                           int write_through, const uint64_t* __restrict__ rbits, int32_t* __restrict__ state,
                           const int32_t* __restrict__ last_upd, int32_t* __restrict__ lists,
                           int32_t* __restrict__ plist, int32_t* cnt, int64_t cap, const int32_t* __restrict__ slot,
                           const int32_t* __restrict__ pool_idx, int P, int64_t capT, int32_t* __restrict__ srcl,
                           int age_seg) {
    const int nA = d_nT ? *d_nT : 0;
    const int nB = *adj_cnt;
    const int nC = pcount_seg ? *pcount_seg : 0;
    const int n = nA + nB + nC;
    const int nloop = (n + blockDim.x * gridDim.x - 1) / (blockDim.x * gridDim.x) * (blockDim.x * gridDim.x);
    const int rot = s & 31;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nloop; i += gridDim.x * blockDim.x) {
        int cls = -1;
        int32_t lk = 0, p = s;
        if (i < nA && state[T[i]] != ST_UPDATED) {
            // cleaned by this step's cache transition (N3) before the scheduler
        } else if (i < nA) {
            lk = T[i];
            if (write_through) {
                state[lk] = ST_CLEAN;
                cls = 0;
            } else {
                const uint64_t b = rbits[lk];
                const uint32_t any = (uint32_t)b, hst = (uint32_t)(b >> 32);
                const uint32_t r = (any >> rot) | (rot ? (any << (32 - rot)) : 0u);
                if (r == 0u) {
                    state[lk] = ST_INF;
                } else {
                    const int off = __ffs(r) - 1;
                    p = s + off;
                    if ((hst >> ((rot + off) & 31)) & 1u) {
                        state[lk] = ST_CLEAN;  // flushed before gate p
                        cls = off == 0 ? 0 : (off == 1 ? 1 : 2);
                    } else {
                        state[lk] = ST_EXEMPT;
                    }
                }
            }
        } else if (i < nA + nB) {
            lk = adj_rows[i - nA];
            p = adj_p[i - nA];
            cls = lk >= 0 ? (p == s + 1 ? 1 : 2) : -1;  // -1: taken over by a cache transition
        } else if (i < n) {
            lk = pkey[i - nA - nB];
            if (lk >= 0 && state[lk] == ST_INF && last_upd[lk] == u_age) {
                state[lk] = ST_CLEAN;
                cls = 3;
            }
        }
        const unsigned peers = __match_any_sync(FULL, cls);
        if (cls >= 0) {
            const int leader = __ffs(peers) - 1, lane = threadIdx.x & 31;
            int base = 0;
            if (lane == leader) base = atomicAdd(&cnt[cls], __popc(peers));
            base = __shfl_sync(peers, base, leader);
            const int64_t at = (int64_t)cls * cap + base + __popc(peers & lanemask_lt());
            lists[at] = lk;
            if (cls < 3) plist[at] = p;
            // the row's current source -- its cache slot (-1 - slot) or its dirty-pool row -- read
            // now: the flushes and the drain's pack then need one dependent load per row instead
            // of three, and an urgent row (read and updated at s, world 1 flushes it off the
            // critical path) is copied from exactly its post-(s-1) bytes.  Age-outs come from
            // pool segment age_seg, row i of it.
            int32_t code;
            if (cls == 3) {
                code = (int32_t)((int64_t)age_seg * capT + (i - nA - nB));
            } else {
                const int sl = slot[lk];
                code = sl >= 0 ? -1 - sl : (int32_t)((int64_t)(last_upd[lk] % P) * capT + pool_idx[lk]);
            }
            srcl[at] = code;
        }
    }
}

void launch_ingest_bits(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st) {
    k_ingest_bits<<<grid_for(c->capT, 256), 256, 0, st>>>(q.T, q.Tmask, q.nT, c->n, c->g, prm, c->slot, c->hot_map[0],
                                                           c->hot_map[1], c->rbits, c->state, c->adj_rows[0],
                                                           c->adj_p[0], c->adj_cnt[0], c->adj_rows[1], c->adj_p[1],
                                                           c->adj_cnt[1]);
    c->launches++;
}

void launch_schedule(frugal_ctx* c, QueueSlot* prev, int64_t s, int par, cudaStream_t st) {
    cudaMemsetAsync(c->sl_cnt[par], 0, 4 * sizeof(int32_t), st);
    const int64_t u = s - 1 - c->D;
    const int seg = u >= 0 ? (int)(u % c->P) : 0;
    k_schedule<<<grid_for(3 * c->capT, 256, 4), 256, 0, st>>>(
        prev ? prev->T : nullptr, prev ? prev->nT : nullptr, c->adj_rows[par], c->adj_p[par], c->adj_cnt[par],
        c->pkey + (size_t)seg * c->capT, u >= 0 ? c->pcount + seg : nullptr, (int32_t)u, (int32_t)s,
        c->cfg.mode == FRUGAL_MODE_WRITE_THROUGH, c->rbits, c->state, c->last_upd, c->sl_rows[par], c->sl_p[par],
        c->sl_cnt[par], c->sl_cap, c->slot, c->pool_idx, c->P, c->capT, c->sl_src[par], seg);
    c->launches++;
}

// ============================================================================ N3 cache transition
// Epoch boundary t0 of the dynamic cache (reading R27), before the scheduler of
// t0: every row whose hotness changes (old: holds a slot; new: in the pending hot set) and
// whose host copy is not current -- dirty, or AdjustPriority'd by the ingest of t0+L-1
// but not yet drained -- is flushed now (the transition set X(t0)) and marked clean; then
// evicted rows release their slots and admitted rows take free slots, loaded from the pool
// (recently updated) or the host table.  G never moves (HBM-resident for every owned row).
__device__ __forceinline__ bool hot_bit(const uint32_t* __restrict__ m, int32_t lk) {
    return ((m[lk >> 5] >> (lk & 31)) & 1u) != 0u;
}
__device__ __forceinline__ void tr_append(int32_t* xl, int32_t* xcnt, bool pred, int32_t lk) {
    const unsigned m = __ballot_sync(__activemask(), pred);
    if (!pred) return;
    const int leader = __ffs(m) - 1, lane = threadIdx.x & 31;
    int base = 0;
    if (lane == leader) base = atomicAdd(xcnt, __popc(m));
    base = __shfl_sync(m, base, leader);
    xl[base + __popc(m & lanemask_lt())] = lk;
}
// (1) pending AdjustPriority entries of t0 whose row changes hotness: into X, cancelled
__global__ void k_tr_adjust(int32_t* __restrict__ adj_rows, const int32_t* adj_cnt, const int32_t* __restrict__ slot,
                            const uint32_t* __restrict__ hnew, int32_t* xl, int32_t* xcnt) {
    const int n = *adj_cnt;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const int32_t lk = adj_rows[i];
        const bool x = lk >= 0 && ((slot[lk] >= 0) != hot_bit(hnew, lk));
        if (x) adj_rows[i] = -1;
        tr_append(xl, xcnt, x, lk);
    }
}
// (2) dirty rows among the evicted (old slots not in the new set) and the admitted
__global__ void k_tr_dirty(const int32_t* __restrict__ hot_lk, int64_t cap_slots, const int32_t* __restrict__ new_lk,
                           const int32_t* d_nnew, const int32_t* __restrict__ slot, const uint32_t* __restrict__ hnew,
                           int32_t* __restrict__ state, int32_t* xl, int32_t* xcnt) {
    const int64_t n = cap_slots + min((int64_t)*d_nnew, cap_slots);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t lk = -1;
        if (i < cap_slots) {
            lk = hot_lk[i];
            if (lk >= 0 && hot_bit(hnew, lk)) lk = -1;  // stays hot
        } else {
            lk = new_lk[i - cap_slots];
            if (slot[lk] >= 0) lk = -1;  // already hot
        }
        const bool x = lk >= 0 && state[lk] != ST_CLEAN;
        if (x) state[lk] = ST_CLEAN;
        tr_append(xl, xcnt, x, lk);
    }
}
// (3) evict: release the slot; no pool copy of the row is live any more (its value is on
// the host), so the gather and the flushes read it from the host table
__global__ void k_tr_evict(int32_t* __restrict__ hot_lk, int64_t cap_slots, const uint32_t* __restrict__ hnew,
                           int32_t* __restrict__ slot, int32_t* __restrict__ last_upd, int32_t* free_slots,
                           int32_t* nfree) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < cap_slots; j += (int64_t)gridDim.x * blockDim.x) {
        const int32_t lk = hot_lk[j];
        if (lk < 0 || hot_bit(hnew, lk)) continue;
        slot[lk] = -1;
        last_upd[lk] = -1;
        hot_lk[j] = -1;
        free_slots[atomicAdd(nfree, 1)] = (int32_t)j;
    }
}
// (4) admit: take a free slot, load the current value (pool when updated within the
// window, else the host table -- current: X flushed every dirty admitted row)
template <int GS>
__global__ void k_tr_admit(const int32_t* __restrict__ new_lk, const int32_t* d_nnew, int64_t cap, int world, int g, int d4,
                           int32_t* __restrict__ slot, int32_t* __restrict__ hot_lk, const int32_t* __restrict__ free_slots,
                           int32_t* nfree, const int32_t* __restrict__ last_upd, const int32_t* __restrict__ pool_idx,
                           const float4* __restrict__ pw, int P, int64_t capT, int32_t pool_min, const float4* hw,
                           const int32_t* __restrict__ hs, float4* __restrict__ cw, int32_t* err) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int64_t n_new = min((int64_t)*d_nnew, cap);
    for (int64_t i = gid; i < n_new; i += gs) {
        const int32_t lk = new_lk[i];
        if (slot[lk] >= 0) continue;
        int j = 0;
        if (l == 0) {
            const int at = atomicSub(nfree, 1) - 1;
            j = at >= 0 ? free_slots[at] : -1;
        }
        j = __shfl_sync(GS >= 32 ? 0xffffffffu : (((1u << GS) - 1u) << ((threadIdx.x & 31) & ~(GS - 1))), j,
                        (threadIdx.x & 31) & ~(GS - 1));
        if (j < 0) {  // more admitted rows than slots: frugal_set_hot checked the size
            if (l == 0) atomicExch(err, 3);
            continue;
        }
        const int32_t lu = last_upd[lk];
        const float4* src = (lu >= 0 && lu >= pool_min) ? pw + ((int64_t)(lu % P) * capT + pool_idx[lk]) * d4
                                                         : hw + host_row(hs, (int64_t)lk * world + g) * d4;
        for (int v = l; v < d4; v += GS) cw[(int64_t)j * d4 + v] = src[v];
        if (l == 0) {
            slot[lk] = j;
            hot_lk[j] = lk;
        }
    }
}
// hot bit array of an epoch from a hot set: global ids (ids64, validated, foreign ones
// skipped) or owned local ids (lks); the distinct owned rows are appended to new_lk
__global__ void k_hot_build(uint32_t* __restrict__ map, const int64_t* __restrict__ ids64,
                            const int32_t* __restrict__ lks, int64_t n, int64_t N, int world, int g,
                            int32_t* __restrict__ new_lk, int32_t* d_nnew, int64_t cap, int32_t* err) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t lk;
        if (ids64) {
            const int64_t k = ids64[i];
            if (k < 0 || k >= N) {
                atomicExch(err, 1);
                continue;
            }
            if (k % world != g) continue;
            lk = (int32_t)(k / world);
        } else {
            lk = lks[i];
        }
        const uint32_t bit = 1u << (lk & 31);
        if (atomicOr(&map[lk >> 5], bit) & bit) continue;  // duplicate
        if (!new_lk) continue;
        const int at = atomicAdd(d_nnew, 1);
        if (at < cap) new_lk[at] = lk;
        else atomicExch(err, 3);
    }
}
void launch_hot_map(frugal_ctx* c, int which, const int64_t* ids64, const int32_t* lks, int64_t n, bool list,
                    cudaStream_t st) {
    cudaMemsetAsync(c->hot_map[which], 0, (size_t)((c->No + 31) / 32) * 4, st);
    if (list) cudaMemsetAsync(c->tr_cnt + 2, 0, 4, st);
    if (n > 0)
        k_hot_build<<<grid_for(n, 256, 4), 256, 0, st>>>(c->hot_map[which], ids64, lks, n, c->N, c->n, c->g,
                                                          list ? c->new_lk : nullptr, c->tr_cnt + 2, c->cap_slots,
                                                          c->err);
    c->launches++;
}


void launch_cache_transition(frugal_ctx* c, int64_t s, int par, cudaStream_t st) {
    const uint32_t* hnew = c->hot_map[c->hot_cur ^ 1];
    int32_t* xcnt = c->tr_cnt + 1;
    cudaMemsetAsync(xcnt, 0, 4, st);
    k_tr_adjust<<<grid_for(c->capT, 256, 4), 256, 0, st>>>(c->adj_rows[par], c->adj_cnt[par], c->slot, hnew,
                                                            c->tr_rows, xcnt);
    k_tr_dirty<<<grid_for(2 * c->cap_slots, 256, 4), 256, 0, st>>>(c->hot_lk, c->cap_slots, c->new_lk, c->tr_cnt + 2,
                                                                   c->slot, hnew, c->state, c->tr_rows, xcnt);
    launch_flush_rows(c, c->tr_rows, nullptr, xcnt, 1 << 30, FRUGAL_C_TRANSITION_HOT, st);
    k_tr_evict<<<grid_for(c->cap_slots, 256, 4), 256, 0, st>>>(c->hot_lk, c->cap_slots, hnew, c->slot, c->last_upd,
                                                                c->free_slots, c->tr_cnt);
    const int d4 = c->d / 4, gs = group_size(d4);
    // no optimizer runs concurrently with the transition: segment u % P is intact for u >= s-P+1
    const int32_t pool_min = (int32_t)std::max<int64_t>(0, s - c->P + 1);
    DISPATCH_GS(gs, (k_tr_admit<GS><<<grid_for(c->cap_slots * gs, 256, 8), 256, 0, st>>>(
                        c->new_lk, c->tr_cnt + 2, c->cap_slots, c->n, c->g, d4, c->slot, c->hot_lk, c->free_slots, c->tr_cnt,
                        c->last_upd, c->pool_idx, (const float4*)c->pw, c->P, c->capT, pool_min,
                        (const float4*)c->dh_w, c->hs, (float4*)c->cw, c->err)));
    c->launches += 4;
}

// ============================================================================ row movers
// a10/a11/a12: flush rows (local ids) to the host table: w of hot rows from the HBM
// cache, w of cold rows from the dirty pool.  Zero-copy stores to host memory.  (The
// owner's Adagrad state G never leaves HBM during training -- no other rank reads it;
// frugal_flush writes it back once, reading R8.)
// TMA=true: each row is staged in shared memory and written to the host by one bulk
// async copy (cp.async.bulk.global.shared::cta) instead of the group's zero-copy stores --
// the same link rate, but the outstanding host writes sit in the TMA unit instead of the
// SM's store path, which slows the concurrent HBM kernels about half as much
// (profiles/r1_interference_probe.txt).  smem: (blockDim / GS) * d4 float4.
template <int GS, bool TMA>
__global__ void k_flush_rows(const int32_t* __restrict__ rows, const int32_t* d_begin, const int32_t* d_end,
                             int world, int g, int d4, const int32_t* __restrict__ slot,
                             const int32_t* __restrict__ last_upd, const int32_t* __restrict__ pool_idx, int P,
                             int64_t capT, const float4* __restrict__ cw, const float4* __restrict__ pw, float4* hw,
                             const int32_t* __restrict__ hs, unsigned long long* stats, int sysfence,
                             const int32_t* __restrict__ srcs) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int b = d_begin ? *d_begin : 0, e = *d_end;
    unsigned nh = 0, nc = 0;
    extern __shared__ __align__(128) float4 fsm[];
    float4* my = TMA ? fsm + (threadIdx.x / GS) * d4 : nullptr;
    const unsigned gmask = GS == 32 ? 0xffffffffu : (((1u << GS) - 1u) << ((threadIdx.x & 31) & ~(GS - 1)));
    for (int64_t a = b + gid; a < e; a += gs) {
        int32_t lk = rows[a];
        int64_t k = (int64_t)lk * world + g;
        // source: the location recorded by the scheduler (urgent bucket off the critical path),
        // else the row's live metadata
        const int32_t code = srcs ? srcs[a] : 0;
        int sl = srcs ? (code < 0 ? -1 - code : -1) : slot[lk];
        const float4* src;
        if (sl >= 0) {
            src = cw + (int64_t)sl * d4;
            nh += (l == 0);
        } else {
            src = pw + (srcs ? (int64_t)code : ((int64_t)(last_upd[lk] % P) * capT + pool_idx[lk])) * d4;
            nc += (l == 0);
        }
        float4* dst = hw + host_row(hs, k) * d4;
        if (TMA) {
            for (int v = l; v < d4; v += GS) my[v] = src[v];
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp(gmask);
            if (l == 0) {
                const unsigned sa = (unsigned)__cvta_generic_to_shared(my);
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(sa),
                             "r"(d4 * 16)
                             : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // smem reusable
            }
            __syncwarp(gmask);
        } else {
            for (int v = l; v < d4; v += GS) dst[v] = src[v];
        }
    }
    if (TMA && l == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // writes complete
    if (sysfence) block_fence_system();
    if (stats) {
        block_count(stats, nh);
        block_count(stats + 1, nc);
    }
}

void launch_flush_rows(frugal_ctx* c, const int32_t* rows, const int32_t* d_begin, const int32_t* d_end,
                       int max_blocks, int counter, cudaStream_t st, bool side, const int32_t* srcs) {
    const int d4 = c->d / 4, gs = group_size(d4);
    int grid = std::min(grid_for(c->capT * (int64_t)gs, 256, 4), max_blocks);
    const bool tma = c->flush_tma == 2 || (c->flush_tma == 1 && side);
#define FLUSH_ARGS                                                                                                \
    rows, d_begin, d_end, c->n, c->g, d4, c->slot, c->last_upd, c->pool_idx, c->P, c->capT, (const float4*)c->cw, \
        (const float4*)c->pw, (float4*)c->dh_w, c->hs, counter >= 0 ? c->dstats + counter : nullptr, c->n > 1, srcs
    if (tma) {
        const size_t smem = (size_t)(256 / gs) * d4 * 16;
        DISPATCH_GS(gs, (k_flush_rows<GS, true><<<grid, 256, smem, st>>>(FLUSH_ARGS)));
    } else {
        DISPATCH_GS(gs, (k_flush_rows<GS, false><<<grid, 256, 0, st>>>(FLUSH_ARGS)));
    }
#undef FLUSH_ARGS
    c->launches++;
}

// a11 with host flushing threads (default; FRUGAL_F_GPU_DRAIN: k_flush_rows instead; §3.2:
// "background flushing threads ... flush the parameter updates ... to host memory"): the
// drain's rows -- list 1 (deadline s+1) first, then list 2 (later deadlines) and list 3
// (age-outs) -- are packed into a host staging queue as ONE contiguous run (coalesced
// zero-copy stores over a few MB that are reused every other step, instead of scattered
// 128-B stores over the whole table), with the host-table slot of every row; the library's
// flushing threads then copy them into the table.  The rows are untouched until their
// deadline (> s), so packing them at any point of step s reads their post-(s-1) values.
// The publish kernel that follows tells the threads how many rows each part has.
template <int GS, int R>
__global__ void k_pack_drain(const int32_t* __restrict__ lists, const int32_t* __restrict__ srcl,
                             const int32_t* __restrict__ cnt, int64_t cap, int world, int g, int d4,
                             const float4* __restrict__ cw, const float4* __restrict__ pw,
                             const int32_t* __restrict__ hs, float4* hrows, int64_t* hkeys,
                             unsigned long long* stats, unsigned long long* ustats, int part, int with_urgent,
                             int to_host) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n1 = cnt[1], n2 = cnt[2], n3 = cnt[3], n0 = with_urgent ? cnt[0] : 0;
    // part 0: list 1 (deadline s+1) -> staging [0, n1); part 1: lists 2, 3 (and, world 1 with
    // the urgent bucket off the critical path, list 0) -> [n1, n1+n2+n3+n0)
    const int lo = part == 0 ? 0 : n1, n = part == 0 ? n1 : n1 + n2 + n3 + n0;
    unsigned nh = 0, nc = 0, uh = 0, uc = 0;
    // R rows in flight per lane group: list entry + source (coalesced), then the row
    for (int64_t a0 = lo + gid; a0 < n; a0 += gs * R) {
        int64_t at[R];
        int32_t code[R], lk[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            const int64_t a = a0 + (int64_t)r * gs;
            at[r] = a >= n ? -1
                  : a < n1 ? cap + a : a < n1 + n2 ? 2 * cap + (a - n1)
                  : a < n1 + n2 + n3 ? 3 * cap + (a - n1 - n2) : (a - n1 - n2 - n3);
            code[r] = at[r] >= 0 ? srcl[at[r]] : 0;
            lk[r] = at[r] >= 0 ? lists[at[r]] : 0;
        }
        for (int v0 = 0; v0 < d4; v0 += GS) {
            const int v = v0 + l;
            float4 x[R];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (at[r] >= 0 && v < d4)
                    x[r] = code[r] < 0 ? cw[(int64_t)(-1 - code[r]) * d4 + v] : pw[(int64_t)code[r] * d4 + v];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (at[r] >= 0 && v < d4) hrows[(a0 + (int64_t)r * gs) * d4 + v] = x[r];
        }
#pragma unroll
        for (int r = 0; r < R; r++) {
            if (at[r] < 0 || l != 0) continue;
            const int64_t a = a0 + (int64_t)r * gs;
            hkeys[a] = host_row(hs, (int64_t)lk[r] * world + g);
            const bool urg = a >= n1 + n2 + n3;
            if (code[r] < 0) { if (urg) uh++; else nh++; }
            else { if (urg) uc++; else nc++; }
        }
    }
    if (to_host) block_fence_system();  // rows and keys reach host memory before the publish kernel's flag
    block_count(stats, nh);
    block_count(stats + 1, nc);
    block_count(ustats, uh);
    block_count(ustats + 1, uc);
}

// TMA variant of the pack (default): each CTA stages a chunk of kPackChunk consecutive rows
// (and their keys) in shared memory and writes it to the pinned staging queue with two bulk
// async copies (cp.async.bulk.global.shared::cta) -- a few large writes per chunk instead of a
// 128-B store per row group, ~50 GB/s from 8 CTAs (profiles/r2_zc_write_probe.txt) with the same
// short queue of posted writes.  Two smem buffers: the next chunk is gathered while the bulk
// copy of this one drains.
template <int GS>
__global__ void __launch_bounds__(256) k_pack_drain_tma(const int32_t* __restrict__ lists,
                                                        const int32_t* __restrict__ srcl,
                                                        const int32_t* __restrict__ cnt, int64_t cap, int world,
                                                        int g, int d4, const float4* __restrict__ cw,
                                                        const float4* __restrict__ pw, const int32_t* __restrict__ hs,
                                                        char* hrows, int64_t* hkeys, unsigned long long* stats,
                                                        unsigned long long* ustats, int part, int with_urgent,
                                                        int kPackChunk) {
    extern __shared__ __align__(128) float4 psm[];  // [2][kPackChunk * d4] rows, then [2][kPackChunk] keys
    int64_t* ksm = (int64_t*)(psm + 2 * kPackChunk * d4);
    const int n1 = cnt[1], n2 = cnt[2], n3 = cnt[3], n0 = with_urgent ? cnt[0] : 0;
    const int lo = part == 0 ? 0 : n1, n = part == 0 ? n1 : n1 + n2 + n3 + n0;
    const int l = threadIdx.x & (GS - 1), grp = threadIdx.x / GS, ngrp = blockDim.x / GS;
    unsigned nh = 0, nc = 0, uh = 0, uc = 0;
    int stage = 0;
    for (int64_t c0 = lo + (int64_t)blockIdx.x * kPackChunk; c0 < n; c0 += (int64_t)gridDim.x * kPackChunk) {
        const int rows = (int)min((int64_t)kPackChunk, n - c0);
        float4* rb = psm + (size_t)stage * kPackChunk * d4;
        int64_t* kb = ksm + stage * kPackChunk;
        // this buffer's previous bulk copy has finished reading shared memory
        if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        __syncthreads();
        for (int r = grp; r < rows; r += ngrp) {
            const int64_t a = c0 + r;
            const int64_t at = a < n1 ? cap + a : a < n1 + n2 ? 2 * cap + (a - n1)
                             : a < n1 + n2 + n3 ? 3 * cap + (a - n1 - n2) : (a - n1 - n2 - n3);
            const int32_t code = srcl[at];
            const float4* src = code < 0 ? cw + (int64_t)(-1 - code) * d4 : pw + (int64_t)code * d4;
            for (int v = l; v < d4; v += GS) rb[r * d4 + v] = src[v];
            if (l == 0) {
                kb[r] = host_row(hs, (int64_t)lists[at] * world + g);
                const bool urg = a >= n1 + n2 + n3;
                if (code < 0) { if (urg) uh++; else nh++; }
                else { if (urg) uc++; else nc++; }
            }
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (threadIdx.x == 0) {
            const unsigned sr = (unsigned)__cvta_generic_to_shared(rb), sk = (unsigned)__cvta_generic_to_shared(kb);
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(hrows + c0 * d4 * 16),
                         "r"(sr), "r"(rows * d4 * 16) : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            (void)sk;
        }
        for (int r = threadIdx.x; r < rows; r += blockDim.x) hkeys[c0 + r] = kb[r];  // coalesced; 8-B aligned only
        stage ^= 1;
    }
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // writes complete
    block_fence_system();
    block_count(stats, nh);
    block_count(stats + 1, nc);
    block_count(ustats, uh);
    block_count(ustats + 1, uc);
}

// second stage of the two-stage pack: one part of the job, already contiguous in HBM, copied to
// the pinned staging queue by a FEW CTAs as one sequential run (8 CTAs reach ~50 GB/s of
// zero-copy writes, profiles/r2_zc_write_probe.txt) -- few CTAs keep the queue of posted PCIe
// writes short, and a PCIe read issued meanwhile (the gather's host rows, a gate's flag) waits
// behind that queue
__global__ void __launch_bounds__(256) k_copy_seq(const int32_t* __restrict__ cnt, int part, int with_urgent, int d4,
                                                  const float4* __restrict__ srows, const int64_t* __restrict__ skeys,
                                                  float4* hrows, int64_t* hkeys) {
    const int n1 = cnt[1], nall = cnt[1] + cnt[2] + cnt[3] + (with_urgent ? cnt[0] : 0);
    const int64_t lo = part == 0 ? 0 : n1, hi = part == 0 ? n1 : nall;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
    for (int64_t e = lo * d4 + t; e < hi * d4; e += nt) hrows[e] = srows[e];
    for (int64_t a = lo + t; a < hi; a += nt) hkeys[a] = skeys[a];
    block_fence_system();
}
// publish part `part` of job `seq` (= s+1) of staging buffer `par`: part sizes, then the part's
// ready word (release) -- the threads start on part 0 (deadline s+1, the next gate waits for
// it) while the kernel packs part 1
__global__ void k_publish_drain(const int32_t* __restrict__ cnt, uint32_t* ctl, int par, uint32_t seq, int part,
                                int with_urgent) {
    ctl[CTL_N1 + par] = (uint32_t)cnt[1];
    ctl[CTL_NTOT + par] = (uint32_t)(cnt[1] + cnt[2] + cnt[3] + (with_urgent ? cnt[0] : 0));
    __threadfence_system();
    uint32_t* w = ctl + (part == 0 ? CTL_READY1 : CTL_READY) + par;
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(w), "r"(seq) : "memory");
}
void launch_pack_drain(frugal_ctx* c, int par, uint32_t seq, int max_blocks, cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    const int nthr = c->pack_threads;
    const int wu = c->urgent_side ? 1 : 0;  // world 1: the urgent bucket goes with the drain
    // two stages (default): the rows are gathered into a contiguous HBM staging run by a full
    // grid (HBM-bound, a few us), then copied to the host by k_copy_seq with max_blocks CTAs;
    // FRUGAL_PACK_2STAGE=0: one kernel gathers straight to the host with max_blocks CTAs
    const bool ce = c->pack_ce;  // HBM run only: the flushing threads copy it with the copy engine
    const bool two = c->pack_2stage || ce;
    const int grid = two ? grid_for(3 * c->sl_cap * (int64_t)gs, 256, 2)
                         : std::min(grid_for(3 * c->sl_cap * (int64_t)gs, nthr, 4), max_blocks);
    float4* rows_dst = two ? (float4*)c->dst_rows[par] : (float4*)c->dfl_rows[par];
    int64_t* keys_dst = two ? c->dst_keys[par] : c->dfl_keys[par];
    for (int part = 0; part < 2; part++) {
#define PACK(RR)                                                                                              \
    DISPATCH_GS(gs, (k_pack_drain<GS, RR><<<grid, two ? 256 : nthr, 0, st>>>(                                \
                        c->sl_rows[par], c->sl_src[par], c->sl_cnt[par], c->sl_cap, c->n, c->g, d4,           \
                        (const float4*)c->cw, (const float4*)c->pw, c->hs, rows_dst, keys_dst,                \
                        c->dstats + FRUGAL_C_SIDE_HOT, c->dstats + FRUGAL_C_URGENT_HOT, part, wu, two ? 0 : 1)))
        if (c->pack_tma && !two) {
            // chunk rows: two buffers of chunk * d floats + keys within 48 KB of shared memory
            const int chunk = std::max(1, std::min(64, (int)(49152 / (2 * (c->d * 4 + 8)))));
            const size_t smem = 2 * (size_t)chunk * d4 * 16 + 2 * (size_t)chunk * 8;
            DISPATCH_GS(gs, (k_pack_drain_tma<GS><<<grid, 256, smem, st>>>(
                                c->sl_rows[par], c->sl_src[par], c->sl_cnt[par], c->sl_cap, c->n, c->g, d4,
                                (const float4*)c->cw, (const float4*)c->pw, c->hs, (char*)c->dfl_rows[par],
                                c->dfl_keys[par], c->dstats + FRUGAL_C_SIDE_HOT, c->dstats + FRUGAL_C_URGENT_HOT, part,
                                wu, chunk)));
        } else if (c->pack_rows >= 4) {
            PACK(4);
        } else {
            PACK(1);
        }
#undef PACK
        if (two && !ce) {
            k_copy_seq<<<max_blocks, 256, 0, st>>>(c->sl_cnt[par], part, wu, d4, (const float4*)c->dst_rows[par],
                                                    c->dst_keys[par], (float4*)c->dfl_rows[par], c->dfl_keys[par]);
            c->launches++;
        }
        k_publish_drain<<<1, 1, 0, st>>>(c->sl_cnt[par], c->dfl_ctl, par, seq, part, wu);
    }
    c->launches += 4;
}

// a4 gather: unique rows -> staging (owned hot: HBM cache; else host, zero-copy).
// list: the uniq indices to gather (early or late part), cnt: its device count.
// An owned cold row whose latest update is still in the dirty pool is read from the pool
// (HBM) instead of the host: the pool holds exactly the value the flush wrote (or will
// write), so the result is bit-identical and the flush schedule unchanged; only where the
// owner reads from moves (R7').  Segment last_upd % P is intact while
// last_upd >= pool_min (the optimizer of step u overwrites segment u % P; pool_min = u-P+2
// also covers a gather running concurrently with the optimizer of u-1).
template <int GS>
__global__ void k_gather_uniq(const int32_t* __restrict__ uniq, const int32_t* __restrict__ list, const int32_t* cnt,
                              int world, int g, int d4, const int32_t* __restrict__ slot,
                              const float4* __restrict__ cw, const float4* hw, float4* __restrict__ rows,
                              const int32_t* __restrict__ last_upd, const int32_t* __restrict__ pool_idx,
                              const float4* __restrict__ pw, int P, int64_t capT, int32_t pool_min,
                              const int32_t* __restrict__ gslot, const PeerTab* __restrict__ pt,
                              const int32_t* __restrict__ hs, unsigned long long* stats, int64_t hmask) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n = *cnt;
    unsigned nh = 0, nc = 0, np = 0, npeer = 0;
    for (int64_t a = gid; a < n; a += gs) {
        const int u = list ? list[a] : (int)a;
        int32_t k = uniq[u];
        const float4* src = nullptr;
        int kind = 0;  // 0 host, 1 cache, 2 pool
        if (k % world == g) {
            const int32_t lk = k / world;
            int sl = slot[lk];
            if (sl >= 0) {
                src = cw + (int64_t)sl * d4;
                kind = 1;
            } else if (pw) {
                const int32_t lu = last_upd[lk];
                if (lu >= 0 && lu >= pool_min) {
                    src = pw + ((int64_t)(lu % P) * capT + pool_idx[lk]) * d4;
                    kind = 2;
                }
            }
        } else if (pt) {
            // N4: the owner's HBM holds this row (cache, or pool within the window) -> peer
            // load over NVLink; its values are the post-(s-1) ones for as long as this gather
            // runs (the gate waited for the owner's urgent flush, which follows its optimizer
            // of s-1; its optimizer of s waits for this rank's mailbox flag of s)
            const int o = k % world;
            const int32_t lk = k / world;
            const int sl = gslot[k];
            if (sl >= 0) {
                src = pt->cw[o] + (int64_t)sl * d4;
                kind = 3;
            } else {
                const int32_t lu = pt->lu[o][lk];
                if (lu >= 0 && lu >= pool_min) {
                    src = pt->pw[o] + ((int64_t)(lu % P) * pt->capT[o] + pt->pi[o][lk]) * d4;
                    kind = 3;
                }
            }
        }
        if (kind == 0) src = hw + (host_row(hs, k) & hmask) * d4;  // hmask: -1 (diagnostic knob aside)
        if (l == 0) {
            nh += kind == 0;
            nc += kind == 1;
            np += kind == 2;
            npeer += kind == 3;
        }
        for (int v = l; v < d4; v += GS) rows[(int64_t)u * d4 + v] = src[v];
    }
    block_count(stats + FRUGAL_C_GATHER_HOST, nh);
    block_count(stats + FRUGAL_C_GATHER_CACHE, nc);
    block_count(stats + FRUGAL_C_GATHER_POOL, np);
    block_count(stats + FRUGAL_C_GATHER_PEER, npeer);
}
// a4 gather, R rows in flight per lane group (default R = 4, FRUGAL_GATHER_ROWS): the
// per-row chain uniq -> {slot, last update, pool index} -> row is latency-bound (one dependent
// HBM round trip per link, then a host read of ~2 us); here the R rows' uniq loads, then all
// their metadata loads (independent of each other: last update and pool index are read for
// every owned row, needed or not), then their row loads are issued together.  Same sources
// as k_gather_uniq (R7'), same bits.
template <int GS, int R>
__global__ void k_gather_uniq_r(const int32_t* __restrict__ uniq, const int32_t* __restrict__ list,
                                const int32_t* cnt, int world, int g, int d4, const int32_t* __restrict__ slot,
                                const float4* __restrict__ cw, const float4* hw, float4* __restrict__ rows,
                                const int32_t* __restrict__ last_upd, const int32_t* __restrict__ pool_idx,
                                const float4* __restrict__ pw, int P, int64_t capT, int32_t pool_min,
                                const int32_t* __restrict__ gslot, const PeerTab* __restrict__ pt,
                                const int32_t* __restrict__ hs, unsigned long long* stats) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int n = *cnt;
    unsigned nh = 0, nc = 0, np = 0, npeer = 0;
    for (int64_t a0 = gid; a0 < n; a0 += gs * R) {
        int u[R];
        int32_t k[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            const int64_t a = a0 + (int64_t)r * gs;
            u[r] = a < n ? (list ? list[a] : (int)a) : -1;
        }
#pragma unroll
        for (int r = 0; r < R; r++) k[r] = u[r] >= 0 ? uniq[u[r]] : -1;
        int32_t sl[R], lu[R], pi[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            sl[r] = -1;
            lu[r] = -1;
            pi[r] = 0;
            if (k[r] < 0) continue;
            const int32_t lk = k[r] / world;
            if (k[r] % world == g) {
                sl[r] = slot[lk];
                if (pw) {
                    lu[r] = last_upd[lk];
                    pi[r] = pool_idx[lk];
                }
            } else if (pt) {
                const int o = k[r] % world;
                sl[r] = gslot[k[r]];
                lu[r] = pt->lu[o][lk];
                pi[r] = pt->pi[o][lk];
            }
        }
        const float4* src[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            src[r] = nullptr;
            if (k[r] < 0) continue;
            int kind = 0;  // 0 host, 1 cache, 2 pool, 3 peer
            if (k[r] % world == g) {
                if (sl[r] >= 0) {
                    src[r] = cw + (int64_t)sl[r] * d4;
                    kind = 1;
                } else if (pw && lu[r] >= 0 && lu[r] >= pool_min) {
                    src[r] = pw + ((int64_t)(lu[r] % P) * capT + pi[r]) * d4;
                    kind = 2;
                }
            } else if (pt) {  // N4: see k_gather_uniq
                const int o = k[r] % world;
                if (sl[r] >= 0) {
                    src[r] = pt->cw[o] + (int64_t)sl[r] * d4;
                    kind = 3;
                } else if (lu[r] >= 0 && lu[r] >= pool_min) {
                    src[r] = pt->pw[o] + ((int64_t)(lu[r] % P) * pt->capT[o] + pi[r]) * d4;
                    kind = 3;
                }
            }
            if (kind == 0) src[r] = hw + host_row(hs, k[r]) * d4;
            if (l == 0) {
                nh += kind == 0;
                nc += kind == 1;
                np += kind == 2;
                npeer += kind == 3;
            }
        }
        for (int v0 = 0; v0 < d4; v0 += GS) {
            const int v = v0 + l;
            float4 x[R];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (src[r] && v < d4) x[r] = src[r][v];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (src[r] && v < d4) rows[(int64_t)u[r] * d4 + v] = x[r];
        }
    }
    block_count(stats + FRUGAL_C_GATHER_HOST, nh);
    block_count(stats + FRUGAL_C_GATHER_CACHE, nc);
    block_count(stats + FRUGAL_C_GATHER_POOL, np);
    block_count(stats + FRUGAL_C_GATHER_PEER, npeer);
}
// a4 expand: out[i] = rows[inv[i]]
template <int GS>
__global__ void k_expand(const int32_t* __restrict__ inv, const int32_t* d_m, int d4, const float4* __restrict__ rows,
                         float4* __restrict__ out) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    const int m = *d_m;
    // 4 positions per row group in flight: their inv loads, then their row loads, are
    // issued together (latency-bound dependent pairs otherwise)
    constexpr int R = 4;
    for (int64_t i0 = gid; i0 < m; i0 += gs * R) {
        int32_t iv[R];
#pragma unroll
        for (int r = 0; r < R; r++) iv[r] = i0 + (int64_t)r * gs < m ? inv[i0 + (int64_t)r * gs] : -1;
        for (int v0 = 0; v0 < d4; v0 += GS) {
            const int v = v0 + l;
            float4 x[R];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (iv[r] >= 0 && v < d4) x[r] = rows[(int64_t)iv[r] * d4 + v];
#pragma unroll
            for (int r = 0; r < R; r++)
                if (iv[r] >= 0 && v < d4) out[(i0 + (int64_t)r * gs) * d4 + v] = x[r];
        }
    }
}

void launch_gather(frugal_ctx* c, QueueSlot& q, const int32_t* list, const int32_t* cnt, float* rows, int64_t step,
                   cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    // zero-copy host loads are latency-bound: ~148x256 threads already keep the link's
    // read requests in flight (tools/zc_probe: 148 vs 1184 CTAs, same GB/s), and a
    // bigger grid only parks stalled warps on SMs other streams need
    int grid = std::min(grid_for((int64_t)c->M * gs, 256, 8), c->gather_blocks);
    const int32_t pool_min = (int32_t)std::max<int64_t>(0, step - c->P + 2);
#define GATHER_ARGS                                                                                          \
    q.uniq, list, cnt, c->n, c->g, d4, c->slot, (const float4*)c->cw, (const float4*)c->dh_w, (float4*)rows,   \
        c->last_upd, c->pool_idx, c->pool_hits ? (const float4*)c->pw : nullptr, c->P, c->capT, pool_min, c->gslot, \
        c->peer_tab, c->hs, c->dstats
    if (c->gather_rows >= 4) {
        DISPATCH_GS(gs, (k_gather_uniq_r<GS, 4><<<grid, 256, 0, st>>>(GATHER_ARGS)));
    } else if (c->gather_rows >= 2) {
        DISPATCH_GS(gs, (k_gather_uniq_r<GS, 2><<<grid, 256, 0, st>>>(GATHER_ARGS)));
    } else {
        // FRUGAL_DIAG_HOST_MASK (diagnostic only, wrong rows): host row index & mask -- is the
        // gather bound by the translation of its random host reads over the whole table?
        static const int64_t hmask = getenv("FRUGAL_DIAG_HOST_MASK") ? atoll(getenv("FRUGAL_DIAG_HOST_MASK")) : -1;
        DISPATCH_GS(gs, (k_gather_uniq<GS><<<grid, 256, 0, st>>>(GATHER_ARGS, hmask)));
    }
#undef GATHER_ARGS
    c->launches++;
}
// host-link calibration: n pseudo-random rows of the host table (hash of i and seed) read
// with the gather's access pattern (row groups, zero-copy, same grid cap) into scratch
template <int GS>
__global__ void k_probe_rows(int64_t n, int64_t N, uint64_t seed, int d4, const float4* hw, float4* __restrict__ out,
                             int64_t out_rows) {
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    for (int64_t i = gid; i < n; i += gs) {
        uint64_t z = seed + 0x9e3779b97f4a7c15ULL * (uint64_t)(i + 1);
        z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
        z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
        z ^= z >> 31;
        const int64_t k = (int64_t)(z % (uint64_t)N);
        for (int v = l; v < d4; v += GS) out[(i % out_rows) * d4 + v] = hw[k * d4 + v];
    }
}
void launch_probe_rows(frugal_ctx* c, int64_t n, uint64_t seed, float* out, int64_t out_rows, cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    int grid = std::min(grid_for(n * gs, 256, 8), c->gather_blocks);
    DISPATCH_GS(gs, (k_probe_rows<GS><<<grid, 256, 0, st>>>(n, c->N, seed, d4, (const float4*)c->dh_w, (float4*)out,
                                                            out_rows)));
    c->launches++;
}

void launch_expand(frugal_ctx* c, QueueSlot& q, const float* rows, float* out, cudaStream_t st) {
    const int d4 = c->d / 4, gs = group_size(d4);
    int grid = grid_for((int64_t)c->M * gs, 256, 8);
    DISPATCH_GS(gs, (k_expand<GS><<<grid, 256, 0, st>>>(q.inv, q.m, d4, (const float4*)rows, (float4*)out)));
    c->launches++;
}

// world 1: split uniq(t) into rows not read at t-1 (early) and rows read at t-1 (late;
// they are updated at t-1 and may be urgent at t).  Read-ring bit t-1 is still set: it is
// cleared by the optimizer of step t-1, which runs after this ingest (one step ahead).
__global__ void k_split_early(const int32_t* __restrict__ uniq, const int32_t* d_nu, const int32_t* __restrict__ prm,
                              const uint64_t* __restrict__ rbits, int32_t* eidx, int32_t* lidx, int32_t* elcnt) {
    const int64_t t = prm[IP_T];
    const int n = *d_nu;
    const int nloop = (n + blockDim.x * gridDim.x - 1) / (blockDim.x * gridDim.x) * (blockDim.x * gridDim.x);
    const uint64_t bit = t > 0 ? (1ull << ((t - 1) & 31)) : 0ull;
    for (int u = blockIdx.x * blockDim.x + threadIdx.x; u < nloop; u += gridDim.x * blockDim.x) {
        bool valid = u < n;
        bool late = valid && (rbits[uniq[valid ? u : 0]] & bit);
        bool early = valid && !late;
        unsigned me = __ballot_sync(FULL, early), ml = __ballot_sync(FULL, late);
        const int lane = threadIdx.x & 31;
        int be = 0, bl = 0;
        if (lane == 0) {
            if (me) be = atomicAdd(&elcnt[0], __popc(me));
            if (ml) bl = atomicAdd(&elcnt[1], __popc(ml));
        }
        be = __shfl_sync(FULL, be, 0);
        bl = __shfl_sync(FULL, bl, 0);
        if (early) eidx[be + __popc(me & lanemask_lt())] = u;
        if (late) lidx[bl + __popc(ml & lanemask_lt())] = u;
    }
}
void launch_split_early(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st) {
    cudaMemsetAsync(q.elcnt, 0, 8, st);
    k_split_early<<<grid_for(c->M, 256, 4), 256, 0, st>>>(q.uniq, q.n_uniq, prm, c->rbits, q.eidx, q.lidx, q.elcnt);
    c->launches++;
}

// ============================================================================ model glue
// row f of sample b: the expanded [count*F][d] array, or (fused lookup, inv != NULL) the
// gathered unique row inv[b*F + f] -- the expand folded into the glue's loads
template <bool FUSED>
__device__ __forceinline__ const float* glue_row(const float* emb, const int32_t* inv, int64_t b, int F, int f, int d) {
    return FUSED ? emb + (int64_t)__ldg(inv + b * F + f) * d : emb + (b * F + f) * d;
}
// warp per sample; lane j holds element j (+32q) of S and, when F <= FC, of every e_f
// in registers (one HBM read of the embeddings); the loss is block-reduced, one atomic
// per block.
template <int J, int FC, bool FUSED>
__global__ void __launch_bounds__(256) k_dot_model(const float* __restrict__ emb, const int32_t* __restrict__ inv,
                                                   const float* __restrict__ x,
                                                   const float* __restrict__ y, float* __restrict__ grad,
                                                   double* loss, int count, int F, int d, double nb) {
    __shared__ double sl[8];
    const int lane = threadIdx.x & 31;
    const int wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nw = (gridDim.x * blockDim.x) >> 5;
    double lsum = 0.0;
    for (int b = wid; b < count; b += nw) {
        float S[J];
        float ec[FC > 0 ? FC : 1][J];
#pragma unroll
        for (int q = 0; q < J; q++) S[q] = 0.0f;
        double ee = 0.0;
        if (FC > 0) {
            // fused lookup: one coalesced load of the sample's F (<= 32) row indices, then
            // broadcast by shuffle (instead of F same-address loads per warp)
            const int32_t myiv = (FUSED && lane < F) ? __ldg(inv + b * F + lane) : 0;
#pragma unroll
            for (int f = 0; f < FC; f++) {
                const int32_t rf = FUSED ? __shfl_sync(FULL, myiv, f) : 0;
                const float* ef = FUSED ? emb + (int64_t)rf * d : emb + (b * F + f) * d;
#pragma unroll
                for (int q = 0; q < J; q++) {
                    int j = lane + 32 * q;
                    ec[f][q] = (f < F && j < d) ? ef[j] : 0.0f;
                }
            }
#pragma unroll
            for (int f = 0; f < FC; f++) {
                if (f < F) {
#pragma unroll
                    for (int q = 0; q < J; q++) {
                        S[q] = __fadd_rn(S[q], ec[f][q]);
                        ee += (double)ec[f][q] * (double)ec[f][q];
                    }
                }
            }
        } else {
            for (int f = 0; f < F; f++) {
                const float* ef = glue_row<FUSED>(emb, inv, b, F, f, d);
#pragma unroll
                for (int q = 0; q < J; q++) {
                    int j = lane + 32 * q;
                    if (j < d) {
                        float v = ef[j];
                        S[q] = __fadd_rn(S[q], v);
                        ee += (double)v * (double)v;
                    }
                }
            }
        }
        double sq = 0.0, xs = 0.0;
        const float* xb = x + (int64_t)b * d;
        float xv[J];
#pragma unroll
        for (int q = 0; q < J; q++) {
            int j = lane + 32 * q;
            xv[q] = j < d ? xb[j] : 0.0f;
            sq += (double)S[q] * (double)S[q];
            xs += (double)xv[q] * (double)S[q];
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            sq += __shfl_xor_sync(FULL, sq, o);
            ee += __shfl_xor_sync(FULL, ee, o);
            xs += __shfl_xor_sync(FULL, xs, o);
        }
        double z = 0.5 * (sq - ee) + xs;
        double p = 1.0 / (1.0 + exp(-z));
        double yb = (double)y[b];
        if (lane == 0) lsum += (z > 0 ? z + log1p(exp(-z)) : log1p(exp(z))) - yb * z;
        float cc = (float)((p - yb) / nb);  // same rounding as the definition (R16)
        float* g0 = grad + (int64_t)b * F * d;
        if (FC > 0) {
#pragma unroll
            for (int f = 0; f < FC; f++) {
                if (f < F) {
#pragma unroll
                    for (int q = 0; q < J; q++) {
                        int j = lane + 32 * q;
                        if (j < d) g0[f * d + j] = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[q], ec[f][q]), xv[q]));
                    }
                }
            }
        } else {
            for (int f = 0; f < F; f++) {
                const float* ef = glue_row<FUSED>(emb, inv, b, F, f, d);
#pragma unroll
                for (int q = 0; q < J; q++) {
                    int j = lane + 32 * q;
                    if (j < d) g0[f * d + j] = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[q], ef[j]), xv[q]));
                }
            }
        }
    }
    if (lane == 0) sl[threadIdx.x >> 5] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int i = 0; i < 8; i++) t += sl[i];
        if (t != 0.0) atomicAdd(loss, t / nb);  // mean over the global batch (R17)
    }
}

// Row-group glue: GS lanes per sample (GS = pow2 >= d/4, <= 32), lane l holds columns
// v = l + k*GS (float4, k < VPL) of S and x; the sample's F rows are read twice from L2 (the
// fused lookup's distinct rows, or the expanded rows) -- once for S and |e|^2, once for the
// gradient -- instead of being kept in registers, so ~40 registers and full occupancy.
// Same arithmetic as k_dot_model: S in fp32, f ascending; z, p, loss in fp64; c rounded to
// fp32 once; grad = c*((S - e_f) + x) with each op rounded (R16).
template <int GS, int VPL, bool FUSED, int U>
__global__ void __launch_bounds__(256) k_dot_rg(const float4* __restrict__ emb, const int32_t* __restrict__ inv,
                                                const float4* __restrict__ x, const float* __restrict__ y,
                                                float4* __restrict__ grad, double* loss, int count, int F, int d4,
                                                double nb) {
    // U rows of the sample in flight (FRUGAL_GLUE_UNROLL): their inverse indices, then their
    // columns, are loaded together before the adds, which stay in f order (f outer, k inner:
    // the same order as U = 1) -- one L2 round trip per U rows instead of two per row
    __shared__ double sl[8];
    int64_t gid, gs;
    int l;
    RowGroup<GS>::ids(gid, gs, l);
    double lsum = 0.0;
    const unsigned gmask = GS == 32 ? FULL : (((1u << GS) - 1u) << ((threadIdx.x & 31) & ~(GS - 1)));
    auto row = [&](int64_t b, int f) -> const float4* {
        return FUSED ? emb + (int64_t)__ldg(inv + b * F + f) * d4 : emb + (b * F + f) * d4;
    };
    for (int64_t b = gid; b < count; b += gs) {
        float4 S[VPL], xv[VPL];
        double ee = 0.0, sq = 0.0, xs = 0.0;
#pragma unroll
        for (int k = 0; k < VPL; k++) {
            S[k] = make_float4(0.f, 0.f, 0.f, 0.f);
            const int v = l + k * GS;
            xv[k] = v < d4 ? x[b * d4 + v] : make_float4(0.f, 0.f, 0.f, 0.f);
        }
        for (int f0 = 0; f0 < F; f0 += U) {
            const float4* e[U];
#pragma unroll
            for (int u = 0; u < U; u++) e[u] = f0 + u < F ? row(b, f0 + u) : nullptr;
            float4 a[U][VPL];
#pragma unroll
            for (int u = 0; u < U; u++)
#pragma unroll
                for (int k = 0; k < VPL; k++) {
                    const int v = l + k * GS;
                    if (e[u] && v < d4) a[u][k] = e[u][v];
                }
#pragma unroll
            for (int u = 0; u < U; u++)
#pragma unroll
                for (int k = 0; k < VPL; k++) {
                    const int v = l + k * GS;
                    if (e[u] && v < d4) {
                        S[k].x = __fadd_rn(S[k].x, a[u][k].x);
                        S[k].y = __fadd_rn(S[k].y, a[u][k].y);
                        S[k].z = __fadd_rn(S[k].z, a[u][k].z);
                        S[k].w = __fadd_rn(S[k].w, a[u][k].w);
                        ee += (double)a[u][k].x * a[u][k].x + (double)a[u][k].y * a[u][k].y +
                              (double)a[u][k].z * a[u][k].z + (double)a[u][k].w * a[u][k].w;
                    }
                }
        }
#pragma unroll
        for (int k = 0; k < VPL; k++) {
            sq += (double)S[k].x * S[k].x + (double)S[k].y * S[k].y + (double)S[k].z * S[k].z + (double)S[k].w * S[k].w;
            xs += (double)xv[k].x * S[k].x + (double)xv[k].y * S[k].y + (double)xv[k].z * S[k].z +
                  (double)xv[k].w * S[k].w;
        }
#pragma unroll
        for (int o = GS / 2; o; o >>= 1) {  // within the sample's lane group only
            sq += __shfl_xor_sync(gmask, sq, o);
            ee += __shfl_xor_sync(gmask, ee, o);
            xs += __shfl_xor_sync(gmask, xs, o);
        }
        const double z = 0.5 * (sq - ee) + xs;
        const double p = 1.0 / (1.0 + exp(-z));
        const double yb = (double)y[b];
        if (l == 0) lsum += (z > 0 ? z + log1p(exp(-z)) : log1p(exp(z))) - yb * z;
        const float cc = (float)((p - yb) / nb);  // same rounding as the definition (R16)
        for (int f0 = 0; f0 < F; f0 += U) {
            const float4* e[U];
#pragma unroll
            for (int u = 0; u < U; u++) e[u] = f0 + u < F ? row(b, f0 + u) : nullptr;
            float4 a[U][VPL];
#pragma unroll
            for (int u = 0; u < U; u++)
#pragma unroll
                for (int k = 0; k < VPL; k++) {
                    const int v = l + k * GS;
                    if (e[u] && v < d4) a[u][k] = e[u][v];
                }
#pragma unroll
            for (int u = 0; u < U; u++) {
                float4* g0 = grad + (b * F + f0 + u) * d4;
#pragma unroll
                for (int k = 0; k < VPL; k++) {
                    const int v = l + k * GS;
                    if (e[u] && v < d4) {
                        float4 r;
                        r.x = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[k].x, a[u][k].x), xv[k].x));
                        r.y = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[k].y, a[u][k].y), xv[k].y));
                        r.z = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[k].z, a[u][k].z), xv[k].z));
                        r.w = __fmul_rn(cc, __fadd_rn(__fsub_rn(S[k].w, a[u][k].w), xv[k].w));
                        g0[v] = r;
                    }
                }
            }
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(FULL, lsum, o);  // whole warp, after the loop
    if ((threadIdx.x & 31) == 0) sl[threadIdx.x >> 5] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int i = 0; i < 8; i++) t += sl[i];
        if (t != 0.0) atomicAdd(loss, t / nb);  // mean over the global batch (R17)
    }
}

void launch_dot_model(frugal_ctx* c, QueueSlot& q, const float* emb, const int32_t* inv, const float* x,
                      const float* y, float* grad, double* loss, int64_t nb, cudaStream_t st) {
    int count = q.h_counts[c->g];
    if (count <= 0) return;
    if (c->glue_rg) {
        const int d4 = c->d / 4, gs = group_size(d4), vpl = (d4 + gs - 1) / gs;
        const double nbd = (double)nb;
        // rows in flight per sample: 8 / VPL (register budget), FRUGAL_GLUE_UNROLL=1: one at a time
        const int un = c->glue_unroll;
#define RGU(V, UU)                                                                                                    \
    do {                                                                                                              \
        if (inv) {                                                                                                    \
            DISPATCH_GS(gs, (k_dot_rg<GS, V, true, UU><<<grid_for((int64_t)count * GS, 256, 8), 256, 0, st>>>(       \
                                (const float4*)emb, inv, (const float4*)x, y, (float4*)grad, loss, count, c->F, d4, nbd))); \
        } else {                                                                                                      \
            DISPATCH_GS(gs, (k_dot_rg<GS, V, false, UU><<<grid_for((int64_t)count * GS, 256, 8), 256, 0, st>>>(      \
                                (const float4*)emb, inv, (const float4*)x, y, (float4*)grad, loss, count, c->F, d4, nbd))); \
        }                                                                                                             \
    } while (0)
        if (vpl <= 1) {
            if (un >= 8) RGU(1, 8);
            else if (un >= 4) RGU(1, 4);
            else RGU(1, 1);
        } else if (vpl <= 2) {
            if (un >= 4) RGU(2, 4);
            else RGU(2, 1);
        } else if (vpl <= 4) {
            if (un >= 2) RGU(4, 2);
            else RGU(4, 1);
        } else {
            RGU(8, 1);
        }
#undef RGU
        c->launches++;
        return;
    }
    int J = (c->d + 31) / 32;
    int grid = grid_for((int64_t)count * 32, 256, 4);
    const double nbd = (double)nb;
    // register-cached rows: one read per row, but 180-250 registers/thread (8 warps/SM); the
    // uncached variant re-reads each row for the gradient (48-54 registers).  With the fused
    // lookup the re-reads hit the L2-resident distinct rows: uncached wins from d > 32 on
    // (Avazu d 64: glue 134 -> 51 us, +23 % samples/s), cached stays at d <= 32
    // (Criteo: within noise; profiles/r1_sweep35_glue.txt)
    const bool cache = c->F <= 32 && (c->glue_cache < 0 ? (J <= 1 || inv == nullptr) : c->glue_cache != 0);
#define DM(JJ, FC)                                                                                     \
    do {                                                                                               \
        if (inv) k_dot_model<JJ, FC, true><<<grid, 256, 0, st>>>(emb, inv, x, y, grad, loss, count, c->F, c->d, nbd); \
        else k_dot_model<JJ, FC, false><<<grid, 256, 0, st>>>(emb, inv, x, y, grad, loss, count, c->F, c->d, nbd);    \
    } while (0)
    if (J <= 1) { if (cache) DM(1, 32); else DM(1, 0); }
    else if (J <= 2) { if (cache) DM(2, 32); else DM(2, 0); }
    else if (J <= 4) DM(4, 0);
    else if (J <= 8) DM(8, 0);
    else if (J <= 16) DM(16, 0);
    else DM(32, 0);
#undef DM
    c->launches++;
}

}  // namespace frugal
