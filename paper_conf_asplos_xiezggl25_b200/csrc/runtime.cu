// runtime.cu -- host runtime of libfrugal: the C ABI (include/frugal.h), context setup,
// the shared host table, the sample queue and the per-step orchestration of the kernels.
//
// Process model (§3.2 Fig. 5, re-designed): one process per GPU; the
// paper's controller process is replaced by device kernels on each rank plus host-memory
// flags.  The host parameter table w[N][d] (+ G[N][d]) lives in a POSIX shm segment
// registered mapped+portable in every rank (L772-774 "shared memory interface"), so every
// GPU reads it with zero-copy loads and the owners flush into it with zero-copy stores.
#include <cuda_runtime.h>
#include <fcntl.h>
#include <stdarg.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/syscall.h>
#include <time.h>
#include <unistd.h>
#include <stdlib.h>

#include <immintrin.h>

#include <algorithm>
#include <atomic>
#include <string>
#include <thread>
#include <vector>

#include "frugal_internal.cuh"

using namespace frugal;

static thread_local std::string g_err;
static void set_err(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
}

#define CK(call)                                                                  \
    do {                                                                          \
        cudaError_t e_ = (call);                                                  \
        if (e_ != cudaSuccess) {                                                  \
            set_err("%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
            return FRUGAL_ECUDA;                                                  \
        }                                                                         \
    } while (0)

#define CKL()                                                                     \
    do {                                                                          \
        cudaError_t e_ = cudaGetLastError();                                      \
        if (e_ != cudaSuccess) {                                                  \
            set_err("kernel launch failed: %s (%s:%d)", cudaGetErrorString(e_), __FILE__, __LINE__); \
            return FRUGAL_ECUDA;                                                  \
        }                                                                         \
    } while (0)

namespace {

constexpr uint64_t kMagic = 0x46525547414c3235ULL;  // "FRUGAL25"
constexpr size_t kHdr = 4096;
constexpr size_t kFlags = 16384;  // 8 kinds x 32 ranks x 64 B (FLAG_* below, FLAG_IDS_KIND)
constexpr size_t kIpc = 32 * 512;  // per rank: IPC handles of cache / pool / last_upd / pool_idx (PEER)

struct IpcRecord {
    volatile uint64_t ready;
    int64_t capT;
    cudaIpcMemHandle_t h[4];
};
static_assert(sizeof(IpcRecord) <= 512, "IPC record");
enum { FLAG_URGENT = 0, FLAG_SIDE = 1, FLAG_MAIL = 2, FLAG_SIDE_FIRST = 3 };
enum { PH_INGEST, PH_SCHED, PH_URGENT, PH_GATE, PH_GATHER, PH_EXPAND, PH_MODEL, PH_SEGRED, PH_EXCH, PH_OPT, PH_SIDE,
       PH_PREFETCH };

struct ShmHeader {
    uint64_t magic;
    volatile uint64_t ready;
    uint64_t total_bytes;
    int64_t n_rows;
    int32_t dim, world, opt, pad;
    volatile uint64_t nonce;  // frugal_config.run_nonce of the run that created the segment
};

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

double now_s() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec + 1e-9 * ts.tv_nsec;
}

int bits_for(int64_t maxval) {  // bits to represent values in [0, maxval]
    int b = 1;
    while (b < 62 && ((int64_t)1 << b) <= maxval) b++;
    return b;
}

struct Timer {
    frugal_ctx* c;
    int ph;
    cudaStream_t st;
    cudaEvent_t a = nullptr;
    Timer(frugal_ctx* c_, int ph_, cudaStream_t st_) : c(c_), ph(ph_), st(st_) {
        if (!(c->cfg.flags & FRUGAL_F_TIMERS)) return;
        if (c->timer_every > 1 && (c->tstep < 0 || c->tstep % c->timer_every != 0)) return;
        if (c->ev_used + 2 > c->ev_pool.size()) {
            for (int i = 0; i < 64; i++) {
                cudaEvent_t e;
                cudaEventCreate(&e);
                c->ev_pool.push_back(e);
            }
        }
        a = c->ev_pool[c->ev_used++];
        cudaEventRecord(a, st);
    }
    ~Timer() {
        if (!a) return;
        cudaEvent_t b = c->ev_pool[c->ev_used++];
        cudaEventRecord(b, st);
        c->evs.push_back({ph, a, b});
    }
};

}  // namespace

// ================================================================================ flushing threads
// PAPER.md §3.2 (L794-797) and §3.3 (L1055-1059): "background flushing threads ... flush the
// parameter updates ... to host memory".  By default (no FRUGAL_F_GPU_DRAIN) the side-stream drain of
// step s packs its rows into staging buffer s&1 and publishes job s (READY[s&1] = s+1); the
// threads copy part 1 (deadline s+1) into the table, publish APPLIED_FIRST = s+1 (and, with a
// shared table, this rank's FLAG_SIDE_FIRST), then part 2 (later deadlines, age-outs) and
// APPLIED_ALL = s+1 (FLAG_SIDE).  Jobs are applied strictly in order, so APPLIED_FIRST >= s+1
// also covers every earlier job.  Each thread copies a contiguous share of the part with
// non-temporal stores (the rows are not read back by the CPU).
struct frugal::Flushers {
    std::vector<std::thread> th;
    std::atomic<bool> stop{false};
    std::atomic<int> done[2][2];  // [parity][part]: threads finished
    std::atomic<uint32_t> copied[2][2];  // [parity][part]: job seq whose rows thread 0 copied D2H (FRUGAL_PACK_CE)
    std::atomic<int> ce_error{0};
    // instrumentation (thread 0): jobs, ns copying its share, ns waiting for the device's flags
    std::atomic<int64_t> jobs{0}, busy_ns{0}, wait_ns{0};
};
static inline int64_t mono_ns() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (int64_t)ts.tv_sec * 1000000000 + ts.tv_nsec;
}

static inline uint32_t ctl_load(const uint32_t* p) { return __atomic_load_n(p, __ATOMIC_ACQUIRE); }
static inline void ctl_store(uint32_t* p, uint32_t v) { __atomic_store_n(p, v, __ATOMIC_RELEASE); }
static inline bool seq_reached(uint32_t x, uint32_t v) { return (int32_t)(x - v) >= 0; }

static void copy_rows_nt(float* table, const float* rows, const int64_t* keys, int64_t lo, int64_t hi, int d) {
    const int n16 = d / 4;  // 16-byte chunks per row (d is a multiple of 4)
    for (int64_t i = lo; i < hi; i++) {
        __m128i* dst = (__m128i*)(table + keys[i] * d);
        const __m128i* src = (const __m128i*)(rows + i * d);
        for (int q = 0; q < n16; q++) _mm_stream_si128(dst + q, _mm_load_si128(src + q));
    }
    _mm_sfence();
}

static void flusher_main(frugal_ctx* c, int t) {
    frugal::Flushers* F = c->flushers;
    if (c->pack_ce && t == 0) cudaSetDevice(c->cfg.device);  // thread 0 issues the D2H copies
    const int T = c->n_flushers;
    uint32_t* ctl = c->hfl_ctl;
    double idle_since = 0.0;
    for (int64_t job = 0;; job++) {
        const int par = (int)(job & 1);
        const uint32_t seq = (uint32_t)(job + 1);
        const float* rows = c->hfl_rows[par];
        const int64_t* keys = c->hfl_keys[par];
        for (int part = 0; part < 2; part++) {
            const int64_t t_wait0 = t == 0 ? mono_ns() : 0;
            // wait for the device to publish the part: spin while jobs keep coming, then poll gently
            const uint32_t* ready = ctl + (part == 0 ? CTL_READY1 : CTL_READY) + par;
            while (!seq_reached(ctl_load(ready), seq)) {
                if (F->stop.load(std::memory_order_relaxed)) return;
                timespec ts;
                clock_gettime(CLOCK_MONOTONIC, &ts);
                const double now = ts.tv_sec + 1e-9 * ts.tv_nsec;
                if (idle_since == 0.0) idle_since = now;
                if (now - idle_since < 2e-3) {
                    for (int k = 0; k < 64; k++) _mm_pause();
                } else {
                    usleep(20);
                }
            }
            idle_since = 0.0;
            int64_t t_start = 0;
            if (t == 0) {
                t_start = mono_ns();
                F->wait_ns.fetch_add(t_start - t_wait0, std::memory_order_relaxed);
            }
            const int64_t n1 = ctl_load(ctl + CTL_N1 + par), nt = ctl_load(ctl + CTL_NTOT + par);
            const int64_t b = part == 0 ? 0 : n1, e = part == 0 ? n1 : nt;
            if (c->pack_ce) {
                // the part is packed in HBM: thread 0 moves it into the pinned staging buffer with
                // the copy engine (one sequential DMA per part), the others wait for it
                if (t == 0) {
                    if (e > b) {
                        const size_t rb = (size_t)c->d * 4;
                        bool ok = cudaMemcpyAsync((char*)c->hfl_rows[par] + b * rb, (char*)c->dst_rows[par] + b * rb,
                                                  (size_t)(e - b) * rb, cudaMemcpyDeviceToHost, c->ce_stream) == cudaSuccess;
                        ok = ok && cudaMemcpyAsync(c->hfl_keys[par] + b, c->dst_keys[par] + b, (size_t)(e - b) * 8,
                                                   cudaMemcpyDeviceToHost, c->ce_stream) == cudaSuccess;
                        ok = ok && cudaStreamSynchronize(c->ce_stream) == cudaSuccess;
                        if (!ok) F->ce_error.store(1);
                    }
                    F->copied[par][part].store(seq, std::memory_order_release);
                } else {
                    while (F->copied[par][part].load(std::memory_order_acquire) != seq) {
                        if (F->stop.load(std::memory_order_relaxed)) return;
                        _mm_pause();
                    }
                }
            }
            static const bool diag_no_apply = getenv("FRUGAL_DIAG_NO_APPLY") && atoi(getenv("FRUGAL_DIAG_NO_APPLY"));
            if (!diag_no_apply)  // (diagnostic only: without the copy the host table is stale)
                copy_rows_nt(c->h_w, rows, keys, b + (e - b) * t / T, b + (e - b) * (t + 1) / T, c->d);
            if (t == 0) F->busy_ns.fetch_add(mono_ns() - t_start, std::memory_order_relaxed);
            if (F->done[par][part].fetch_add(1, std::memory_order_acq_rel) + 1 == T) {
                F->done[par][part].store(0, std::memory_order_relaxed);
                ctl_store(ctl + (part == 0 ? CTL_APPLIED_FIRST : CTL_APPLIED_ALL), seq);
                if (c->xhost) {  // readers on other GPUs wait for this owner's flags
                    const int which = part == 0 ? 3 /* FLAG_SIDE_FIRST */ : 1 /* FLAG_SIDE */;
                    ctl_store((uint32_t*)(c->h_flags + (which * 32 + c->g) * 16), seq);
                }
            }
        }
        if (t == 0) F->jobs.fetch_add(1, std::memory_order_relaxed);
    }
}

// host side: every published drain job applied (frugal_flush, introspection); 120 s bound
static frugal_status wait_flushers(frugal_ctx* c) {
    if (!c->host_flush || c->drains_issued == 0) return FRUGAL_OK;
    const uint32_t want = (uint32_t)c->drains_issued;
    timespec t0, t1;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    while (!seq_reached(ctl_load(c->hfl_ctl + CTL_APPLIED_ALL), want)) {
        usleep(10);
        clock_gettime(CLOCK_MONOTONIC, &t1);
        if (t1.tv_sec - t0.tv_sec > 120) {
            set_err("flushing threads did not apply drain %u within 120 s", want);
            return FRUGAL_ETIMEOUT;
        }
    }
    return FRUGAL_OK;
}

// ================================================================================ helpers
// Spread the host table over every NUMA node (best effort, before the pages are first
// touched): on a two-socket host each GPU then finds half the rows behind its own root
// complex instead of all of them behind rank 0's.
static void interleave_numa(void* base, size_t bytes) {
    FILE* f = fopen("/sys/devices/system/node/online", "r");
    if (!f) return;
    int lo = 0, hi = 0;
    int got = fscanf(f, "%d-%d", &lo, &hi);
    fclose(f);
    if (got < 2 || hi <= lo || hi >= 64) return;
    unsigned long mask = 0;
    for (int n = lo; n <= hi; n++) mask |= 1ul << n;
    syscall(SYS_mbind, base, bytes, 3 /* MPOL_INTERLEAVE */, &mask, 65ul, 0u);
}
static frugal_status check_err_word(frugal_ctx* c) {
    if (c->flushers && c->flushers->ce_error.load()) {
        set_err("flushing threads: a device-to-host copy of the drain staging run failed");
        return FRUGAL_ECUDA;
    }
    if (c->herr && *(volatile int32_t*)c->herr) {
        int e = *(volatile int32_t*)c->herr;
        if (e == 2) {
            set_err("a peer rank did not publish its flag within 120 s");
            return FRUGAL_ETIMEOUT;
        }
        if (e == 3) {
            set_err("dynamic cache: more admitted rows than free slots");
            return FRUGAL_EINVAL;
        }
        set_err("a row id outside [0, n_rows) was passed in a sample batch");
        return FRUGAL_EINVAL;
    }
    return FRUGAL_OK;
}

static void free_ctx(frugal_ctx* c) {
    if (!c) return;
    cudaSetDevice(c->cfg.device);
    cudaDeviceSynchronize();
    if (c->flushers) {
        c->flushers->stop.store(true);
        for (auto& t : c->flushers->th) t.join();
        delete c->flushers;
        c->flushers = nullptr;
    }
    for (int i = 0; i < 2; i++) {
        if (c->dst_rows[i]) cudaFree(c->dst_rows[i]);
        if (c->dst_keys[i]) cudaFree(c->dst_keys[i]);
        if (c->hfl_rows[i]) cudaFreeHost(c->hfl_rows[i]);
        if (c->hfl_keys[i]) cudaFreeHost(c->hfl_keys[i]);
    }
    if (c->hfl_ctl) cudaFreeHost(c->hfl_ctl);
    for (auto e : c->ingest_exec)
        if (e) cudaGraphExecDestroy(e);
    if (c->gstream) cudaStreamDestroy(c->gstream);
    if (c->xstream) cudaStreamDestroy(c->xstream);
    if (c->ev_xy) cudaEventDestroy(c->ev_xy);
    for (int i = 0; i < 2; i++) {
        if (c->ev_glue[i]) cudaEventDestroy(c->ev_glue[i]);
        if (c->x_stage[i]) cudaFree(c->x_stage[i]);
        if (c->y_stage[i]) cudaFree(c->y_stage[i]);
    }
    if (c->d_iprm) cudaFree(c->d_iprm);
    if (c->h_iprm) cudaFreeHost(c->h_iprm);
    auto F = [](void* p) {
        if (p) cudaFree(p);
    };
    F(c->slot); F(c->state); F(c->last_upd); F(c->pool_idx); F(c->rbits);
    F(c->cw); F(c->Gd); F(c->hot_lk); F(c->pw); F(c->pkey); F(c->pcount);
    F(c->hot_map[0]); F(c->hot_map[1]); F(c->new_lk); F(c->free_slots); F(c->tr_cnt); F(c->tr_rows); F(c->hot_stage);
    for (auto& q : c->q) {
        F(q.eidx); F(q.lidx); F(q.elcnt);
        F(q.ids); F(q.counts); F(q.m); F(q.uniq); F(q.inv); F(q.off); F(q.pos); F(q.n_uniq);
        F(q.linfo); F(q.ltask); F(q.lcnt); F(q.lnum);
        if (c->n > 1) { F(q.T); F(q.Tmask); F(q.Tidx); F(q.nT); F(q.gl); F(q.goff); }
    }
    F(c->hs); F(c->rows_buf[0]); F(c->rows_buf[1]); F(c->Pp); F(c->chunk_scratch); F(c->long_q); F(c->long_cnt); F(c->upd_ctr); F(c->long_tasks); F(c->owned_cnt);
    for (int i = 0; i < 2; i++) { F(c->adj_rows[i]); F(c->adj_p[i]); F(c->adj_cnt[i]); }
    for (int i = 0; i < 2; i++) { F(c->sl_rows[i]); F(c->sl_p[i]); F(c->sl_src[i]); F(c->sl_cnt[i]); }
    F(c->dstats); F(c->kg_W); F(c->kg_A); F(c->a2a_roff); F(c->peer_tab); F(c->gslot);
    for (int r = 0; r < 32; r++)
        for (int i = 0; i < 4; i++)
            if (c->peer_open[r][i]) cudaIpcCloseMemHandle(c->peer_open[r][i]); F(c->ff_rows); F(c->ff_cnt); F(c->ids_stage);
    if (c->herr) cudaFreeHost(c->herr);
    if (c->counts_pin) cudaFreeHost(c->counts_pin);
    for (auto e : c->ev_counts) cudaEventDestroy(e);
    sort_free(c->sort);
    scan_free(c->scan);
    if (c->side) cudaStreamDestroy(c->side);
    if (c->istream) cudaStreamDestroy(c->istream);
    if (c->ev_call) cudaEventDestroy(c->ev_call);
    if (c->ev_copied) cudaEventDestroy(c->ev_copied);
    if (c->ev_gathered) cudaEventDestroy(c->ev_gathered);
    for (auto e : c->ev_ingest) cudaEventDestroy(e);
    if (c->ev_sched) cudaEventDestroy(c->ev_sched);
    for (int i = 0; i < 2; i++) {
        if (c->ev_side[i]) cudaEventDestroy(c->ev_side[i]);
        if (c->ev_side_first[i]) cudaEventDestroy(c->ev_side_first[i]);
        if (c->ev_early[i]) cudaEventDestroy(c->ev_early[i]);
        if (c->ev_opt[i]) cudaEventDestroy(c->ev_opt[i]);
    }
    if (c->pstream) cudaStreamDestroy(c->pstream);
    if (c->ce_stream) cudaStreamDestroy(c->ce_stream);
    for (auto e : c->ev_pool) cudaEventDestroy(e);
    if (c->ev_hot) cudaEventDestroy(c->ev_hot);
    if (c->shm_base) {
        cudaHostUnregister(c->shm_base);
        munmap(c->shm_base, c->shm_bytes);
    }
    if (c->shm_fd >= 0) close(c->shm_fd);
    if (c->shm_owner && c->cfg.shm_name) shm_unlink(c->cfg.shm_name);
    delete c;
}

#define DMALLOC(ptr, bytes)                                                                     \
    do {                                                                                         \
        size_t b_ = (bytes) < 16 ? 16 : (bytes);                                                 \
        if (cudaMalloc((void**)&(ptr), b_) != cudaSuccess) {                                     \
            cudaGetLastError();                                                                  \
            set_err("cudaMalloc of %zu bytes failed (%s)", b_, #ptr);                            \
            free_ctx(c);                                                                         \
            return FRUGAL_ENOMEM;                                                                \
        }                                                                                        \
    } while (0)

// ================================================================================ peers (N4)
// Publish this rank's cache / pool / metadata as CUDA IPC handles in the shared segment,
// wait for every rank, open the others' (lazy peer access), and build the dense map
// gslot[k] = slot of hot row k in its owner's cache (owners number their hot rows in
// ascending local id, as frugal_init does).
static frugal_status setup_peers(frugal_ctx* c, char* ipc_base, std::vector<int64_t>& hot_global) {
    IpcRecord* mine = (IpcRecord*)(ipc_base + (size_t)c->g * 512);
    CK(cudaIpcGetMemHandle(&mine->h[0], c->cw));
    CK(cudaIpcGetMemHandle(&mine->h[1], c->pw));
    CK(cudaIpcGetMemHandle(&mine->h[2], c->last_upd));
    CK(cudaIpcGetMemHandle(&mine->h[3], c->pool_idx));
    mine->capT = c->capT;
    __sync_synchronize();
    mine->ready = kMagic;
    PeerTab tab;
    memset(&tab, 0, sizeof tab);
    const double t0 = now_s();
    for (int r = 0; r < c->n; r++) {
        IpcRecord* rec = (IpcRecord*)(ipc_base + (size_t)r * 512);
        while (rec->ready != kMagic) {
            if (now_s() - t0 > 600) { set_err("timed out waiting for rank %d's IPC handles", r); return FRUGAL_ETIMEOUT; }
            usleep(5000);
        }
        __sync_synchronize();
        tab.capT[r] = rec->capT;
        if (r == c->g) {
            tab.cw[r] = (const float4*)c->cw;
            tab.pw[r] = (const float4*)c->pw;
            tab.lu[r] = c->last_upd;
            tab.pi[r] = c->pool_idx;
            continue;
        }
        for (int i = 0; i < 4; i++) {
            void* p = nullptr;
            CK(cudaIpcOpenMemHandle(&p, rec->h[i], cudaIpcMemLazyEnablePeerAccess));
            c->peer_open[r][i] = p;
        }
        tab.cw[r] = (const float4*)c->peer_open[r][0];
        tab.pw[r] = (const float4*)c->peer_open[r][1];
        tab.lu[r] = (const int32_t*)c->peer_open[r][2];
        tab.pi[r] = (const int32_t*)c->peer_open[r][3];
    }
    CK(cudaMalloc(&c->peer_tab, sizeof(PeerTab)));
    CK(cudaMemcpy(c->peer_tab, &tab, sizeof tab, cudaMemcpyHostToDevice));
    std::sort(hot_global.begin(), hot_global.end());
    hot_global.erase(std::unique(hot_global.begin(), hot_global.end()), hot_global.end());
    std::vector<int32_t> gslot((size_t)c->N, -1), next(c->n, 0);
    for (int64_t k : hot_global) gslot[k] = next[k % c->n]++;  // ascending k == ascending local id per owner
    CK(cudaMalloc(&c->gslot, (size_t)c->N * 4));
    CK(cudaMemcpy(c->gslot, gslot.data(), (size_t)c->N * 4, cudaMemcpyHostToDevice));
    return FRUGAL_OK;
}

// ================================================================================ init
extern "C" frugal_status frugal_init(const frugal_config* cfg, frugal_ctx** out) {
    if (!out) { set_err("out is NULL"); return FRUGAL_EINVAL; }
    *out = nullptr;
    if (!cfg) { set_err("cfg is NULL"); return FRUGAL_EINVAL; }
    const frugal_config& k = *cfg;
    if (k.world < 1 || k.world > 32 || k.rank < 0 || k.rank >= k.world) { set_err("bad world/rank"); return FRUGAL_EINVAL; }
    if (k.dim < 4 || k.dim > 1024 || k.dim % 4) { set_err("dim must be a multiple of 4 in [4, 1024]"); return FRUGAL_EINVAL; }
    if (k.n_rows < 1 || k.n_rows > 0x7fffffffLL) { set_err("n_rows must be in [1, 2^31-1]"); return FRUGAL_EINVAL; }
    if (k.slots < 1 || k.batch < 1 || (int64_t)k.slots * k.batch * k.world > 0x7fffffffLL) { set_err("bad slots/batch"); return FRUGAL_EINVAL; }
    if (k.lookahead < 2 || k.lookahead > 31) { set_err("lookahead must be in [2, 31]"); return FRUGAL_EINVAL; }
    if (k.age_out < 1) { set_err("age_out must be >= 1"); return FRUGAL_EINVAL; }
    if (k.opt != FRUGAL_SGD && k.opt != FRUGAL_ADAGRAD) { set_err("bad opt"); return FRUGAL_EINVAL; }
    if (k.mode != FRUGAL_MODE_P2F && k.mode != FRUGAL_MODE_WRITE_THROUGH) { set_err("bad mode"); return FRUGAL_EINVAL; }
    if (!k.shm_name && k.world != 1) { set_err("world > 1 needs shm_name"); return FRUGAL_EINVAL; }
    if (k.shm_name && k.world > 1 && k.run_nonce == 0) {
        set_err("world > 1 needs a run_nonce != 0 (the same on every rank)");
        return FRUGAL_EINVAL;
    }
    if ((k.flags & FRUGAL_F_A2A) && k.world < 2) { set_err("FRUGAL_F_A2A needs world > 1"); return FRUGAL_EINVAL; }
    if ((k.flags & FRUGAL_F_PEER) && (k.world < 2 || (k.flags & FRUGAL_F_A2A))) {
        set_err("FRUGAL_F_PEER needs world > 1 and the host-bounced exchange");
        return FRUGAL_EINVAL;
    }
    if ((k.flags & FRUGAL_F_DYNAMIC_CACHE) && (k.flags & FRUGAL_F_PEER)) {
        set_err("FRUGAL_F_DYNAMIC_CACHE does not combine with FRUGAL_F_PEER");
        return FRUGAL_EINVAL;
    }
    if (k.n_hot < 0 || (k.n_hot > 0 && !k.hot_ids)) { set_err("bad hot set"); return FRUGAL_EINVAL; }
    if (k.n_order < 0 || k.n_order > k.n_rows || (k.n_order > 0 && !k.host_order)) {
        set_err("bad host_order");
        return FRUGAL_EINVAL;
    }
    for (int64_t i = 0; i < k.n_hot; i++)
        if (k.hot_ids[i] < 0 || k.hot_ids[i] >= k.n_rows) { set_err("hot id out of range"); return FRUGAL_EINVAL; }
    if (cudaSetDevice(k.device) != cudaSuccess) { set_err("cudaSetDevice(%d) failed", k.device); return FRUGAL_ECUDA; }
    if (cudaError_t e = setup_kernel_attrs(); e != cudaSuccess) {
        set_err("kernel attributes on device %d: %s", k.device, cudaGetErrorString(e));
        return FRUGAL_ECUDA;
    }

    frugal_ctx* c = new frugal_ctx();
    c->cfg = k;
    c->cfg.hot_ids = nullptr;
    c->cfg.host_order = nullptr;
    if (k.n_order > 0) {  // host-table layout: slot of row host_order[i] = i, the rest in id order
        c->hs_host.assign((size_t)k.n_rows, -1);
        for (int64_t i = 0; i < k.n_order; i++) {
            const int64_t id = k.host_order[i];
            if (id < 0 || id >= k.n_rows || c->hs_host[id] >= 0) {
                set_err("host_order: id out of range or repeated at %lld", (long long)i);
                free_ctx(c);
                return FRUGAL_EINVAL;
            }
            c->hs_host[id] = (int32_t)i;
        }
        int32_t next = (int32_t)k.n_order;
        for (auto& v : c->hs_host)
            if (v < 0) v = next++;
    }
    c->n = k.world; c->g = k.rank; c->d = k.dim; c->F = k.slots; c->B = k.batch;
    c->L = k.lookahead; c->D = k.age_out; c->M = k.batch * k.slots; c->N = k.n_rows;
    c->No = c->g < c->N ? (c->N - c->g + c->n - 1) / c->n : 0;
    // pool segments: a row updated at u sits in segment u % P until the optimizer of u+P;
    // its last reader is the drain of step u+1+D (age-out), which step u+D+3 waits for
    c->P = c->D + 3;
    // N3: a cold dirty row may wait for a cache transition instead of its age-out (EXEMPT
    // for a read under the next hot set): its pool copy must live until that boundary,
    // at most D + L steps after its update
    if (k.flags & FRUGAL_F_DYNAMIC_CACHE) c->P = std::max(c->P, c->D + c->L + 1);
    // FRUGAL_POOL_STEPS=P' > D+3 keeps every segment for P' steps: owned cold rows updated
    // within the last P'-2 steps are then read from HBM (R7') -- more HBM, fewer host reads
    if (getenv("FRUGAL_POOL_STEPS")) c->P = std::max(c->P, atoi(getenv("FRUGAL_POOL_STEPS")));
    c->QN = c->L + 2;
    // pipelined early gather (world 1): off by default -- measured no gain on a PCIe-bound
    // box (the zero-copy loads of the next step only delay this step's); FRUGAL_EARLY=1
    c->early = c->n == 1 && getenv("FRUGAL_EARLY") && atoi(getenv("FRUGAL_EARLY"));
    c->pool_hits = !(getenv("FRUGAL_NO_POOL_HITS") && atoi(getenv("FRUGAL_NO_POOL_HITS")));
    c->early_blocks = getenv("FRUGAL_EARLY_BLOCKS") ? atoi(getenv("FRUGAL_EARLY_BLOCKS")) : 16;
    c->early_rows = getenv("FRUGAL_EARLY_ROWS") ? atoi(getenv("FRUGAL_EARLY_ROWS")) : 4;
    c->early_on_side = getenv("FRUGAL_EARLY_ON_SIDE") && atoi(getenv("FRUGAL_EARLY_ON_SIDE"));
    c->a2a = (k.flags & FRUGAL_F_A2A) != 0;
    c->peer = (k.flags & FRUGAL_F_PEER) != 0;
    c->dyn = (k.flags & FRUGAL_F_DYNAMIC_CACHE) != 0;
    if (c->dyn) c->early = false;
    // host flushing threads (default), or the GPU scatter drain (FRUGAL_F_GPU_DRAIN);
    // FRUGAL_HOST_FLUSH=0/1 (experiments) overrides the flag
    c->host_flush = (k.flags & FRUGAL_F_GPU_DRAIN) == 0;
    if (getenv("FRUGAL_HOST_FLUSH")) c->host_flush = atoi(getenv("FRUGAL_HOST_FLUSH")) != 0;
    c->xhost = c->n > 1 && !c->a2a;
    c->own_ids = (k.flags & FRUGAL_F_OWN_IDS) != 0 && c->n > 1;
    // side-drain flushes by TMA bulk stores (FRUGAL_FLUSH_TMA=0 none, 1 side, 2 all)
    if (getenv("FRUGAL_FLUSH_TMA")) c->flush_tma = atoi(getenv("FRUGAL_FLUSH_TMA"));
    // world 1: optimizer fused into the segment-reduce (FRUGAL_FUSE_OPT=0: two kernels)
    if (getenv("FRUGAL_GLUE_CACHE")) c->glue_cache = atoi(getenv("FRUGAL_GLUE_CACHE"));
    c->glue_rg = !(getenv("FRUGAL_GLUE_RG") && !atoi(getenv("FRUGAL_GLUE_RG")));
    if (getenv("FRUGAL_GLUE_CACHE")) c->glue_rg = false;  // the warp-per-sample variants were asked for
    c->fuse_opt = !(getenv("FRUGAL_FUSE_OPT") && !atoi(getenv("FRUGAL_FUSE_OPT")));
    c->update1 = !(getenv("FRUGAL_UPDATE1") && !atoi(getenv("FRUGAL_UPDATE1")));
    c->side_blocks = getenv("FRUGAL_SIDE_BLOCKS") ? atoi(getenv("FRUGAL_SIDE_BLOCKS")) : 20;
    // few CTAs for the zero-copy writes of the pack: 8 reach the link rate, and a short queue of
    // posted writes keeps concurrent PCIe reads fast (profiles/r2_zc_write_probe.txt, r2_sweep_pack*.txt)
    c->pack_blocks = getenv("FRUGAL_PACK_BLOCKS") ? atoi(getenv("FRUGAL_PACK_BLOCKS")) : 8;
    c->pack_ce = getenv("FRUGAL_PACK_CE") && atoi(getenv("FRUGAL_PACK_CE"));
    c->pack_2stage = getenv("FRUGAL_PACK_2STAGE") && atoi(getenv("FRUGAL_PACK_2STAGE"));  // measured slower (r2_sweep_pack_2stage.txt)
    c->pack_rows = getenv("FRUGAL_PACK_ROWS") ? atoi(getenv("FRUGAL_PACK_ROWS")) : 1;
    c->pack_tma = getenv("FRUGAL_PACK_TMA") && atoi(getenv("FRUGAL_PACK_TMA"));  // measured slower (r2_sweep_pack_tma.txt)
    c->pack_threads = getenv("FRUGAL_PACK_THREADS") ? atoi(getenv("FRUGAL_PACK_THREADS")) : 256;
    // the deadline-(s+1) part of the drain (the next gate waits for it) may run wider
    c->side_first_blocks = getenv("FRUGAL_SIDE_FIRST_BLOCKS") ? atoi(getenv("FRUGAL_SIDE_FIRST_BLOCKS"))
                                                               : c->side_blocks;
    c->gather_blocks = getenv("FRUGAL_GATHER_BLOCKS") ? atoi(getenv("FRUGAL_GATHER_BLOCKS")) : 120;
    c->side_inline = getenv("FRUGAL_SIDE_INLINE") && atoi(getenv("FRUGAL_SIDE_INLINE"));
    c->gather_rows = getenv("FRUGAL_GATHER_ROWS") ? atoi(getenv("FRUGAL_GATHER_ROWS")) : 1;
    c->timer_every = getenv("FRUGAL_TIMER_EVERY") ? std::max(1, atoi(getenv("FRUGAL_TIMER_EVERY"))) : 1;
    c->glue_unroll = getenv("FRUGAL_GLUE_UNROLL") ? atoi(getenv("FRUGAL_GLUE_UNROLL")) : 8;
    c->update_short8 = getenv("FRUGAL_UPDATE_SHORT") && atoi(getenv("FRUGAL_UPDATE_SHORT"));  // measured slower (r2_sweep_glue_update.txt)
    c->update_dyn = getenv("FRUGAL_UPDATE_DYN") && atoi(getenv("FRUGAL_UPDATE_DYN"));  // measured slower (r2_sweep_update_dyn.txt)
    c->pack_serial = getenv("FRUGAL_PACK_SERIAL") && atoi(getenv("FRUGAL_PACK_SERIAL"));
    c->drain_after_gather = !(getenv("FRUGAL_DRAIN_AT") && !strcmp(getenv("FRUGAL_DRAIN_AT"), "sched"));
    // world 1 with pool reads (R7'): the urgent bucket is not read from the host at its step
    // (FRUGAL_URGENT_SIDE=0: keep it on the critical path)
    c->urgent_side = c->n == 1 && c->pool_hits && !c->side_inline && (!c->early || c->L >= 3) &&
                     k.mode == FRUGAL_MODE_P2F &&
                     !(getenv("FRUGAL_URGENT_SIDE") && !atoi(getenv("FRUGAL_URGENT_SIDE")));
    // the early gather waits for the GPU drain's events -- or, world 1 under the lag rule
    // (urgent_side), for the flushing threads' progress word
    if (c->host_flush && !c->urgent_side) c->early = false;
    c->capT = std::max<int64_t>(1, std::min<int64_t>((int64_t)c->n * c->M, c->No));
    c->sl_cap = 2 * c->capT;
    c->key_bits = bits_for(c->N - 1);
    c->lk_bits = bits_for(std::max<int64_t>(c->No - 1, 0));
    const bool adag = k.opt == FRUGAL_ADAGRAD;
    const bool host_G = adag && !(k.flags & FRUGAL_F_NO_HOST_STATE);
    const size_t rowb = (size_t)c->d * sizeof(float);

    // ---------------------------------------------------------------- host table (shm)
    c->mail_stride = c->n > 1 ? align_up(256 + (size_t)c->M * rowb, 4096) : 0;
    const size_t mail_bytes = c->n > 1 ? 2 * (size_t)c->n * c->mail_stride : 0;
    c->idbox_stride = c->own_ids ? align_up(256 + (size_t)c->M * 4, 4096) : 0;
    const size_t idbox_bytes = c->own_ids ? (size_t)kIdSlots * c->n * c->idbox_stride : 0;
    const size_t off_ipc = kHdr + kFlags;
    const size_t off_mail = off_ipc + kIpc;
    const size_t off_idbox = off_mail + mail_bytes;
    const size_t off_w = align_up(off_idbox + idbox_bytes, 2 << 20);
    const size_t tab = (size_t)c->N * rowb;
    const size_t off_G = align_up(off_w + tab, 2 << 20);
    const size_t total = host_G ? off_G + tab : off_w + tab;
    c->shm_bytes = total;
    if (k.shm_name) {
        if (c->g == 0) {
            shm_unlink(k.shm_name);
            c->shm_fd = shm_open(k.shm_name, O_CREAT | O_EXCL | O_RDWR, 0600);
            if (c->shm_fd < 0 || ftruncate(c->shm_fd, (off_t)total) != 0) {
                set_err("shm_open/ftruncate(%s, %zu) failed", k.shm_name, total);
                free_ctx(c);
                return FRUGAL_ESHM;
            }
            c->shm_owner = true;
            c->shm_base = mmap(nullptr, total, PROT_READ | PROT_WRITE, MAP_SHARED, c->shm_fd, 0);
        } else {
            // attach only to the segment of THIS run: rank 0 stamps run_nonce into the header
            // once the table is initialised; a stale segment left under the same name by a
            // crashed run (other nonce) is closed and the name re-opened until rank 0's new
            // segment (created after it unlinked the old one) carries our nonce
            double t0 = now_s();
            while (true) {
                c->shm_fd = shm_open(k.shm_name, O_RDWR, 0600);
                struct stat sb;
                if (c->shm_fd >= 0 && fstat(c->shm_fd, &sb) == 0 && (size_t)sb.st_size == total) {
                    void* m = mmap(nullptr, total, PROT_READ | PROT_WRITE, MAP_SHARED, c->shm_fd, 0);
                    if (m != MAP_FAILED) {
                        const ShmHeader* h = (const ShmHeader*)m;
                        if (h->ready == kMagic && h->nonce == k.run_nonce) {
                            __sync_synchronize();
                            c->shm_base = m;
                            break;
                        }
                        munmap(m, total);
                    }
                }
                if (c->shm_fd >= 0) { close(c->shm_fd); c->shm_fd = -1; }
                if (now_s() - t0 > 600) {
                    set_err("timed out attaching shm %s (no segment of run %llx)", k.shm_name,
                            (unsigned long long)k.run_nonce);
                    delete c;
                    return FRUGAL_ESHM;
                }
                usleep(20000);
            }
        }
    } else {
        // private anonymous memory: transparent huge pages apply (shmem usually has them off),
        // so the flushing threads' scattered row stores miss the TLB far less often
        c->shm_base = mmap(nullptr, total, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    }
    if (c->shm_base == MAP_FAILED) {
        c->shm_base = nullptr;
        set_err("mmap of %zu bytes failed", total);
        free_ctx(c);
        return FRUGAL_ESHM;
    }
    madvise(c->shm_base, total, MADV_HUGEPAGE);
    if (c->g == 0 || !k.shm_name) interleave_numa(c->shm_base, total);
    if (cudaHostRegister(c->shm_base, total, cudaHostRegisterMapped | cudaHostRegisterPortable) != cudaSuccess) {
        cudaGetLastError();
        munmap(c->shm_base, total);
        c->shm_base = nullptr;
        set_err("cudaHostRegister of %zu bytes failed", total);
        free_ctx(c);
        return FRUGAL_ENOMEM;
    }
    char* dbase = nullptr;
    if (cudaHostGetDevicePointer((void**)&dbase, c->shm_base, 0) != cudaSuccess) {
        set_err("cudaHostGetDevicePointer failed");
        free_ctx(c);
        return FRUGAL_ECUDA;
    }
    char* hbase = (char*)c->shm_base;
    ShmHeader* hdr = (ShmHeader*)hbase;
    c->h_flags = (volatile uint32_t*)(hbase + kHdr);
    c->dh_flags = (uint32_t*)(dbase + kHdr);
    c->h_mail = hbase + off_mail;
    c->dh_mail = dbase + off_mail;
    if (c->own_ids) c->dh_idbox = dbase + off_idbox;
    c->h_w = (float*)(hbase + off_w);
    c->dh_w = (float*)(dbase + off_w);
    if (host_G) {
        c->h_G = (float*)(hbase + off_G);
        c->dh_G = (float*)(dbase + off_G);
    }
    if (cudaHostAlloc((void**)&c->herr, 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess ||
        cudaHostAlloc((void**)&c->counts_pin, (size_t)(c->L + 2) * c->n * 4, cudaHostAllocPortable) != cudaSuccess) {
        set_err("cudaHostAlloc(err/counts) failed");
        free_ctx(c);
        return FRUGAL_ENOMEM;
    }
    memset(c->herr, 0, 64);
    cudaHostGetDevicePointer((void**)&c->err, c->herr, 0);

    // ---------------------------------------------------------------- device state
    if (!c->hs_host.empty()) {
        DMALLOC(c->hs, (size_t)c->N * 4);
        if (cudaMemcpy(c->hs, c->hs_host.data(), (size_t)c->N * 4, cudaMemcpyHostToDevice) != cudaSuccess) {
            set_err("host_order upload failed");
            free_ctx(c);
            return FRUGAL_ECUDA;
        }
    }
    DMALLOC(c->slot, c->No * 4);
    DMALLOC(c->state, c->No * 4);
    DMALLOC(c->last_upd, c->No * 4);
    DMALLOC(c->pool_idx, c->No * 4);
    DMALLOC(c->rbits, c->No * 8);
    // the whole hot set (PEER: every owner's slot of every hot row) and this rank's share
    std::vector<int64_t> hot_global(k.hot_ids, k.hot_ids + k.n_hot);
    // owned share of the hot set, sorted, deduplicated
    std::vector<int32_t> hot;
    for (int64_t i = 0; i < k.n_hot; i++)
        if (k.hot_ids[i] % c->n == c->g) hot.push_back((int32_t)(k.hot_ids[i] / c->n));
    std::sort(hot.begin(), hot.end());
    hot.erase(std::unique(hot.begin(), hot.end()), hot.end());
    c->cap_hot = (int64_t)hot.size();
    c->cap_slots = c->dyn ? c->cap_hot + std::max<int64_t>(64, c->cap_hot / 4) : c->cap_hot;
    DMALLOC(c->hot_lk, c->cap_slots * 4);
    DMALLOC(c->cw, c->cap_slots * rowb);
    if (c->dyn) {
        DMALLOC(c->hot_map[0], (size_t)((c->No + 31) / 32) * 4);
        DMALLOC(c->hot_map[1], (size_t)((c->No + 31) / 32) * 4);
        DMALLOC(c->new_lk, c->cap_slots * 4);
        DMALLOC(c->free_slots, c->cap_slots * 4);
        DMALLOC(c->tr_cnt, 12);
        DMALLOC(c->tr_rows, ((size_t)c->capT + 2 * c->cap_slots) * 4);
    }
    if (adag) DMALLOC(c->Gd, (size_t)c->No * rowb);
    DMALLOC(c->pw, (size_t)c->P * c->capT * rowb);
    DMALLOC(c->pkey, (size_t)c->P * c->capT * 4);
    DMALLOC(c->pcount, (size_t)c->P * 4);
    c->q.resize(c->QN);
    for (auto& q : c->q) {
        DMALLOC(q.ids, (size_t)c->n * c->M * 4);
        DMALLOC(q.counts, (size_t)c->n * 4);
        DMALLOC(q.m, 4);
        DMALLOC(q.uniq, (size_t)c->M * 4);
        DMALLOC(q.inv, (size_t)c->M * 4);
        DMALLOC(q.off, ((size_t)c->M + 1) * 4);
        DMALLOC(q.pos, (size_t)c->M * 4);
        DMALLOC(q.n_uniq, 4);
        DMALLOC(q.eidx, (size_t)c->M * 4);
        DMALLOC(q.lidx, (size_t)c->M * 4);
        DMALLOC(q.elcnt, 8);
        if (c->n == 1) {
            DMALLOC(q.linfo, ((size_t)c->M / 65 + 1) * sizeof(int4));
            DMALLOC(q.ltask, ((size_t)c->M / 64 + c->M / 65 + 2) * sizeof(int4));
            DMALLOC(q.lcnt, ((size_t)c->M / 65 + 1) * 4);
            DMALLOC(q.lnum, 8);
        }
        if (c->n > 1) {
            DMALLOC(q.T, c->capT * 4);
            DMALLOC(q.Tmask, c->capT * 4);
            DMALLOC(q.Tidx, (size_t)c->n * c->capT * 4);
            DMALLOC(q.nT, 4);
            DMALLOC(q.gl, (size_t)c->M * 4);
            DMALLOC(q.goff, 64 * 4);
        } else {
            q.T = q.uniq;  // world 1: every row is owned, T(t) == uniq(t)
            q.nT = q.n_uniq;
        }
        q.h_counts.assign(c->n, 0);
    }
    DMALLOC(c->rows_buf[0], (size_t)c->M * rowb);
    DMALLOC(c->rows_buf[1], (size_t)c->M * rowb);
    DMALLOC(c->Pp, (size_t)c->M * rowb);
    DMALLOC(c->chunk_scratch, (size_t)c->M * rowb);
    DMALLOC(c->long_q, (size_t)c->M * 4);
    DMALLOC(c->long_cnt, 8);
    DMALLOC(c->upd_ctr, 8);
    CK(cudaMemset(c->upd_ctr, 0, 8));
    DMALLOC(c->long_tasks, ((size_t)c->M / 32 + 2) * sizeof(int2));
    DMALLOC(c->owned_cnt, 4);

    for (int i = 0; i < 2; i++) {
        DMALLOC(c->adj_rows[i], c->capT * 4);
        DMALLOC(c->adj_p[i], c->capT * 4);
        DMALLOC(c->adj_cnt[i], 4);
        cudaMemset(c->adj_cnt[i], 0, 4);
    }
    for (int i = 0; i < 2; i++) {
        DMALLOC(c->sl_rows[i], 4 * c->sl_cap * 4);
        DMALLOC(c->sl_p[i], 3 * c->sl_cap * 4);
        DMALLOC(c->sl_src[i], 4 * c->sl_cap * 4);
        DMALLOC(c->sl_cnt[i], 4 * 4);
        cudaMemset(c->sl_cnt[i], 0, 16);
    }

    DMALLOC(c->ff_rows, std::max<int64_t>(c->No, 1) * 4);
    DMALLOC(c->ff_cnt, 4);
    DMALLOC(c->ids_stage, (size_t)c->n * c->M * 8);
    DMALLOC(c->dstats, FRUGAL_N_COUNTERS * 8);
    DMALLOC(c->a2a_roff, 64 * 4);
    cudaMemset(c->dstats, 0, FRUGAL_N_COUNTERS * 8);
    sort_alloc(c->sort, (int64_t)c->n * c->M);
    scan_alloc(c->scan, (int64_t)c->n * c->M);
    if (!c->sort.hist || !c->scan.part) {
        set_err("scratch allocation failed");
        free_ctx(c);
        return FRUGAL_ENOMEM;
    }
    int lo_prio, hi_prio;
    cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio);
    // side-stream priority (FRUGAL_SIDE_PRIO=low|normal|high): low by default; measured
    // within noise of the others on a PCIe-bound step
    {
        const char* sp = getenv("FRUGAL_SIDE_PRIO");
        int prio = lo_prio;
        if (sp && !strcmp(sp, "high")) prio = hi_prio;
        if (sp && !strcmp(sp, "normal")) prio = 0;
        if (!sp && c->host_flush) prio = hi_prio;  // the flushing-thread pack: 8 small CTAs, scheduled promptly
        CK(cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, prio));
    }
    CK(cudaEventCreateWithFlags(&c->ev_sched, cudaEventDisableTiming));
    {   // ingest-stream priority (FRUGAL_INGEST_PRIO=low|normal|high, default normal)
        const char* ip = getenv("FRUGAL_INGEST_PRIO");
        int prio = 0;
        if (ip && !strcmp(ip, "high")) prio = hi_prio;
        if (ip && !strcmp(ip, "low")) prio = lo_prio;
        CK(cudaStreamCreateWithPriority(&c->istream, cudaStreamNonBlocking, prio));
    }
    CK(cudaEventCreateWithFlags(&c->ev_call, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&c->ev_copied, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&c->ev_gathered, cudaEventDisableTiming));
    for (int i = 0; i < 2; i++) {
        CK(cudaEventCreateWithFlags(&c->ev_side[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c->ev_side_first[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c->ev_early[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c->ev_opt[i], cudaEventDisableTiming));
    }
    CK(cudaStreamCreateWithPriority(&c->pstream, cudaStreamNonBlocking, hi_prio));
    c->ev_counts.resize(c->QN);
    for (auto& e : c->ev_counts) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    c->ev_ingest.resize(c->QN);
    for (auto& e : c->ev_ingest) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    CK(cudaStreamCreateWithFlags(&c->xstream, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&c->ev_xy, cudaEventDisableTiming));
    for (int i = 0; i < 2; i++) CK(cudaEventCreateWithFlags(&c->ev_glue[i], cudaEventDisableTiming));
    c->use_graphs = !(getenv("FRUGAL_GRAPHS") && !atoi(getenv("FRUGAL_GRAPHS")));
    c->ingest_exec.assign(c->QN, nullptr);
    c->ingest_nodes.assign(c->QN, 0);
    CK(cudaStreamCreateWithFlags(&c->gstream, cudaStreamNonBlocking));
    DMALLOC(c->d_iprm, (size_t)c->QN * IP_N * 4);
    if (cudaHostAlloc((void**)&c->h_iprm, (size_t)c->QN * IP_N * 4, cudaHostAllocPortable) != cudaSuccess) {
        set_err("cudaHostAlloc(ingest parameters) failed");
        free_ctx(c);
        return FRUGAL_ENOMEM;
    }

    cudaStream_t st = 0;
    cudaMemset(c->hot_lk, 0xff, c->cap_slots * 4);  // spare slots (N3) are free
    if (c->dyn) {
        std::vector<int32_t> fr;
        for (int64_t j = c->cap_slots - 1; j >= c->cap_hot; j--) fr.push_back((int32_t)j);
        const int32_t cnt3[3] = {(int32_t)fr.size(), 0, 0};
        cudaMemcpy(c->free_slots, fr.data(), fr.size() * 4, cudaMemcpyHostToDevice);
        cudaMemcpy(c->tr_cnt, cnt3, 12, cudaMemcpyHostToDevice);
        CK(cudaEventCreateWithFlags(&c->ev_hot, cudaEventDisableTiming));
    }
    if (cudaMemcpy(c->hot_lk, hot.data(), hot.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) {
        set_err("hot upload failed");
        free_ctx(c);
        return FRUGAL_ECUDA;
    }
    launch_init_meta(c, nullptr, 0, st);
    if (c->dyn) launch_hot_map(c, 0, nullptr, c->hot_lk, c->cap_hot, false, st);
    cudaMemset(c->pcount, 0, (size_t)c->P * 4);
    cudaMemset(c->pkey, 0xff, (size_t)c->P * c->capT * 4);
    if (c->g == 0 || !k.shm_name) {
        memset(hbase + kHdr, 0, kFlags + kIpc);
        launch_init_table(c, st);
        if (cudaDeviceSynchronize() != cudaSuccess) {
                set_err("table init failed: %s", cudaGetErrorString(cudaGetLastError()));
            free_ctx(c);
            return FRUGAL_ECUDA;
        }
        hdr->magic = kMagic;
        hdr->total_bytes = total;
        hdr->n_rows = c->N;
        hdr->dim = c->d;
        hdr->world = c->n;
        hdr->opt = k.opt;
        hdr->nonce = k.run_nonce;
        __sync_synchronize();
        hdr->ready = kMagic;
    } else {
        // attached above to a segment whose header is ready and carries this run's nonce
        if (hdr->n_rows != c->N || hdr->dim != c->d || hdr->world != c->n || hdr->opt != k.opt) {
                set_err("shm table config mismatch with rank 0");
            free_ctx(c);
            return FRUGAL_ESHM;
        }
    }
    if (cudaDeviceSynchronize() != cudaSuccess) {
        set_err("init failed: %s", cudaGetErrorString(cudaGetLastError()));
        free_ctx(c);
        return FRUGAL_ECUDA;
    }
    if (c->host_flush) {
        const int64_t cap = std::max<int64_t>(1, std::min<int64_t>(4 * c->sl_cap, c->No));
        bool ok = cudaHostAlloc((void**)&c->hfl_ctl, 4096, cudaHostAllocMapped | cudaHostAllocPortable) == cudaSuccess;
        for (int i = 0; ok && i < 2; i++) {
            ok = cudaHostAlloc((void**)&c->hfl_rows[i], (size_t)cap * rowb, cudaHostAllocMapped | cudaHostAllocPortable) ==
                     cudaSuccess &&
                 cudaHostAlloc((void**)&c->hfl_keys[i], (size_t)cap * 8, cudaHostAllocMapped | cudaHostAllocPortable) ==
                     cudaSuccess;
            if (ok) {
                cudaHostGetDevicePointer((void**)&c->dfl_rows[i], c->hfl_rows[i], 0);
                cudaHostGetDevicePointer((void**)&c->dfl_keys[i], c->hfl_keys[i], 0);
            }
        }
        if (!ok) {
            cudaGetLastError();
            set_err("cudaHostAlloc of the drain staging queue failed");
            free_ctx(c);
            return FRUGAL_ENOMEM;
        }
        memset(c->hfl_ctl, 0, 4096);
        if (c->pack_2stage || c->pack_ce)
            for (int i = 0; i < 2; i++) {
                DMALLOC(c->dst_rows[i], (size_t)cap * rowb);
                DMALLOC(c->dst_keys[i], (size_t)cap * 8);
            }
        cudaHostGetDevicePointer((void**)&c->dfl_ctl, c->hfl_ctl, 0);
        const long ncpu = sysconf(_SC_NPROCESSORS_ONLN);
        c->n_flushers = getenv("FRUGAL_FLUSH_THREADS") ? atoi(getenv("FRUGAL_FLUSH_THREADS"))
                                                       : (int)std::max(2L, std::min(8L, ncpu / 4));
        c->n_flushers = std::max(1, c->n_flushers);
        c->flushers = new frugal::Flushers();
        for (int i = 0; i < 2; i++)
            for (int j = 0; j < 2; j++) {
                c->flushers->done[i][j].store(0);
                c->flushers->copied[i][j].store(0);
            }
        if (c->pack_ce) CK(cudaStreamCreateWithFlags(&c->ce_stream, cudaStreamNonBlocking));
        for (int t = 0; t < c->n_flushers; t++) c->flushers->th.emplace_back(flusher_main, c, t);
    }
    if (c->peer) {
        frugal_status r = setup_peers(c, hbase + off_ipc, hot_global);
        if (r) {
            free_ctx(c);
            return r;
        }
    }
    *out = c;
    return FRUGAL_OK;
}

// ================================================================================ sample queue
// Ingest step t of all ranks into queue slot t % (L+2) on the ingest stream: copy + convert
// + validate ids, own dedup, owner-side T (world > 1), read-ring bits of step t and
// AdjustPriority inf -> t (into the adjust list consumed by frugal_step(t-L+1)).  The
// ingest of step s+L runs one step ahead, overlapping step s's gather.
// `after`: an event the ingest must follow (the scheduler of the current step).
// The ingest of step t in two parts.  Part A (id conversion, dedup, long-segment tasks,
// owner side) only needs the ids: it starts as soon as they are copied.  Part B (read-ring
// bits of t, AdjustPriority inf -> t) must follow the scheduler of t-L (which buckets the rows
// updated at t-L-1 over the window [t-L, t-1] and marks the inf ones) -- only this small part
// sits between two schedulers.  Every per-step value is read from the device parameter block
// prm, so part A's launch sequence is identical every step (graph-captured once per slot).
static void enqueue_ingest_a(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t is) {
    launch_convert_ids(c, q, is);
    launch_dedup(c, q, is);
    if (c->n == 1) launch_long_tasks(c, q, is);
    if (c->own_ids) launch_owner_side_v2(c, q, prm, is);
    else if (c->n > 1) launch_owner_side(c, q, 0, is);
}
static void enqueue_ingest_b(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t is) {
    launch_ingest_prologue(c, prm, is);
    launch_ingest_bits(c, q, prm, is);
    if (c->early) launch_split_early(c, q, prm, is);
}

static frugal_status ingest(frugal_ctx* c, int64_t t, const int64_t* ids_all, const int32_t* counts, int adjust,
                            cudaStream_t caller, cudaEvent_t after) {
    for (int r = 0; r < c->n; r++)
        if (counts[r] < 0 || counts[r] > c->B) {
            set_err("counts[%d] = %d outside [0, batch=%d]", r, counts[r], c->B);
            return FRUGAL_EINVAL;
        }
    const int qi = (int)(t % c->QN);
    QueueSlot& q = c->q[qi];
    q.step = t;
    q.h_counts.assign(counts, counts + c->n);
    // FRUGAL_INGEST_SERIAL=1 (diagnostic): ingest on the caller's stream, no overlap
    static const bool serial = getenv("FRUGAL_INGEST_SERIAL") && atoi(getenv("FRUGAL_INGEST_SERIAL"));
    cudaStream_t is = serial ? caller : c->istream;
    // the caller's buffer is read after the caller's prior work on `caller`; the copy of the
    // previous call has finished once this call returns (host wait, normally long done), so
    // the caller may reuse a buffer after the next frugal_step/frugal_prefetch returns
    static const bool no_copy_wait = getenv("FRUGAL_NO_COPY_WAIT") && atoi(getenv("FRUGAL_NO_COPY_WAIT"));  // diagnostic
    const int64_t hw0 = mono_ns();
    if (!no_copy_wait) CK(cudaEventSynchronize(c->ev_copied));
    CK(cudaEventRecord(c->ev_call, caller));
    CK(cudaStreamWaitEvent(is, c->ev_call, 0));
    CK(cudaEventSynchronize(c->ev_counts[qi]));  // pinned counts / parameter staging of this slot is free
    c->host_wait_ns += mono_ns() - hw0;
    int32_t* pin = c->counts_pin + (size_t)qi * c->n;
    memcpy(pin, counts, (size_t)c->n * 4);
    CK(cudaMemcpyAsync(q.counts, pin, (size_t)c->n * 4, cudaMemcpyHostToDevice, is));
    // the ingest's per-step parameters (its kernels read them: one graph per slot)
    int32_t* hp = c->h_iprm + (size_t)qi * IP_N;
    int32_t* dp = c->d_iprm + (size_t)qi * IP_N;
    hp[IP_T] = (int32_t)t;
    hp[IP_APAR] = (int)((t - c->L + 1) & 1);  // adjust list consumed by frugal_step(t - L + 1)
    hp[IP_ADJUST] = adjust;
    hp[IP_HMAP] = c->dyn ? ((c->hot_pending && t >= c->hot_t0) ? (c->hot_cur ^ 1) : c->hot_cur) : -1;
    hp[IP_IDSLOT] = (int)(t % kIdSlots);
    hp[IP_FLAGV] = (int32_t)(uint32_t)(t + 1);
    CK(cudaMemcpyAsync(dp, hp, IP_N * 4, cudaMemcpyHostToDevice, is));
    CK(cudaEventRecord(c->ev_counts[qi], is));
    if (c->own_ids)  // this rank's ids only (ingest v2): into its row of the staging array
        CK(cudaMemcpyAsync(c->ids_stage + (size_t)c->g * c->M, ids_all, (size_t)c->M * 8, cudaMemcpyDefault, is));
    else
        CK(cudaMemcpyAsync(c->ids_stage, ids_all, (size_t)c->n * c->M * 8, cudaMemcpyDefault, is));
    CK(cudaEventRecord(c->ev_copied, is));
    {
        Timer tm(c, PH_INGEST, is);
        if (c->use_graphs && !serial) {
            if (!c->ingest_exec[qi]) {  // first use of this slot: capture its launch sequence once
                cudaGraph_t g = nullptr;
                const int64_t l0 = c->launches;
                CK(cudaStreamBeginCapture(c->gstream, cudaStreamCaptureModeThreadLocal));
                enqueue_ingest_a(c, q, dp, c->gstream);
                CK(cudaStreamEndCapture(c->gstream, &g));
                CK(cudaGraphInstantiate(&c->ingest_exec[qi], g, 0));
                cudaGraphDestroy(g);
                c->ingest_nodes[qi] = c->launches - l0;
                c->launches = l0;
            }
            CK(cudaGraphLaunch(c->ingest_exec[qi], is));
            c->launches += c->ingest_nodes[qi];
        } else {
            enqueue_ingest_a(c, q, dp, is);
        }
    }
    if (after) CK(cudaStreamWaitEvent(is, after, 0));  // part B follows the current step's scheduler
    {
        Timer tm(c, PH_INGEST, is);
        enqueue_ingest_b(c, q, dp, is);
    }
    CK(cudaEventRecord(c->ev_ingest[qi], is));
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_prefetch(frugal_ctx* c, int64_t t, const int64_t* ids_all, const int32_t* counts,
                                         frugal_stream stream) {
    if (!c || !ids_all || !counts) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (c->cur_step != -1 || t != c->next_prefetch || t > c->L - 1) {
        set_err("prefetch(%lld): expected t = %lld (only steps 0..L-1 before step 0)", (long long)t,
                (long long)c->next_prefetch);
        return FRUGAL_ESTATE;
    }
    frugal_status r = ingest(c, t, ids_all, counts, 0, (cudaStream_t)stream, nullptr);
    if (r) return r;
    c->next_prefetch++;
    return check_err_word(c);
}

static void record_schedule(frugal_ctx* c, int par, cudaStream_t st) {
    cudaStreamSynchronize(st);
    int32_t cnt[4];
    cudaMemcpy(cnt, c->sl_cnt[par], sizeof cnt, cudaMemcpyDeviceToHost);
    auto get = [&](int which, std::vector<int32_t>& rows, std::vector<int32_t>* ps) {
        rows.resize(cnt[which]);
        if (cnt[which]) {
            cudaMemcpy(rows.data(), c->sl_rows[par] + (size_t)which * c->sl_cap, cnt[which] * 4, cudaMemcpyDeviceToHost);
            if (ps) {
                ps->resize(cnt[which]);
                cudaMemcpy(ps->data(), c->sl_p[par] + (size_t)which * c->sl_cap, cnt[which] * 4, cudaMemcpyDeviceToHost);
            }
        } else if (ps) {
            ps->clear();
        }
    };
    std::vector<int32_t> r1, p1, r2, p2;
    get(0, c->rec_urgent, nullptr);
    get(1, r1, &p1);
    get(2, r2, &p2);
    get(3, c->rec_ageout, nullptr);
    c->rec_deferred = r1;
    c->rec_deferred.insert(c->rec_deferred.end(), r2.begin(), r2.end());
    c->rec_deferred_p = p1;
    c->rec_deferred_p.insert(c->rec_deferred_p.end(), p2.begin(), p2.end());
    c->rec_gate_wait = cnt[0] > 0;
}

// a4 (pipelined, world 1): gather the rows of step u that were not read at u-1 into
// rows_buf[u&1] on the prefetch stream, once (i) the ingest of u is done, (ii) the side
// stream has drained every flush with deadline u, (iii) the optimizer of u-2 released
// rows_buf[u&1].  None of these rows is updated at u-1, so the host table / cache already
// hold their step-u values (invariant (2)); the rest is gathered after gate u.
static frugal_status launch_early_gather(frugal_ctx* c, int64_t u, cudaEvent_t side_first) {
    QueueSlot& q = c->q[u % c->QN];
    // with the drain placed after the gather, the early gather follows the drain on the
    // side stream: one FIFO of host-link work (late gather, drain, early gather of the
    // next step) that fills the link while the main stream runs the backward
    cudaStream_t ps = c->early_on_side ? c->side : c->pstream;
    CK(cudaStreamWaitEvent(ps, c->ev_ingest[u % c->QN], 0));
    if (c->opt_pending[u & 1]) CK(cudaStreamWaitEvent(ps, c->ev_opt[u & 1], 0));
    Timer tm(c, PH_PREFETCH, ps);
    if (c->urgent_side) {
        // world 1 reading its dirty pool (R7'): the early rows of u that come from the host were
        // last updated before u-D-1, so their host copies are final once the drains up to
        // u - lag are applied (the gate's rule, frugal_step) -- long before step u-1 runs
        const int64_t lag = std::min<int64_t>(c->L - 1, (int64_t)c->D + 1);
        if (u - lag >= 0) {
            if (c->host_flush) {
                const uint32_t need = (uint32_t)(u - lag + 1);
                if (!seq_reached(ctl_load(c->hfl_ctl + CTL_APPLIED_ALL), need))
                    launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, need, ps);
            } else if (u >= 2 && c->side_pending[(u - 2) & 1]) {
                CK(cudaStreamWaitEvent(ps, c->ev_side[(u - 2) & 1], 0));  // drain u-2 (FIFO: and earlier)
            }
        }
    } else if (side_first) {
        CK(cudaStreamWaitEvent(ps, side_first, 0));
    }
    {
        const int keep = c->gather_blocks, keep_rows = c->gather_rows;
        c->gather_blocks = c->early_blocks;  // few SMs: its loads must not crowd the backward
        c->gather_rows = c->early_rows;
        launch_gather(c, q, q.eidx, q.elcnt, c->rows_buf[u & 1], u, ps);
        c->gather_blocks = keep;
        c->gather_rows = keep_rows;
    }
    CK(cudaEventRecord(c->ev_early[u & 1], ps));
    c->early_issued = u;
    CKL();
    return FRUGAL_OK;
}

// a11: deferred buckets (priorities s+1 .. s+L-1, ascending) and age-outs of step s on the
// side stream, after `after` (the scheduler, or -- default -- the step's gather, so the
// zero-copy stores of the drain do not compete with the zero-copy loads of the gather:
// measured, a concurrent random gather and scatter over PCIe take longer than the two in
// sequence).  Deadline s+1 is drained first; the next step's early gather
// waits only for that part.
static frugal_status launch_drain(frugal_ctx* c, int64_t s, cudaStream_t st, cudaEvent_t after) {
    const int par = (int)(s & 1);
    cudaStream_t sd = c->side_inline ? st : c->side;
    if (!c->side_inline) CK(cudaStreamWaitEvent(c->side, after, 0));
    if (c->host_flush) {
        // host flushing threads: staging buffer `par` was last used by job s-2 (one timer over
        // the wait and the pack: an event recorded between them measurably slowed the step,
        // 25.3 vs 26.7 M samples/s, profiles/r2_ab_side_timer.txt)
        Timer tm(c, PH_SIDE, sd);
        if (s >= 2) launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, (uint32_t)(s - 1), sd);
        launch_pack_drain(c, par, (uint32_t)(s + 1), c->pack_blocks, sd);
        CK(cudaEventRecord(c->ev_side_first[par], sd));  // the lists of this parity were read
        CKL();
    } else {
        Timer tm(c, PH_SIDE, sd);
        launch_flush_rows(c, c->sl_rows[par] + c->sl_cap, nullptr, c->sl_cnt[par] + 1, c->side_first_blocks,
                          FRUGAL_C_SIDE_HOT, sd, true, c->sl_src[par] + c->sl_cap);
        CK(cudaEventRecord(c->ev_side_first[par], sd));
        if (c->xhost) launch_set_flag(c, FLAG_SIDE_FIRST, (uint32_t)(s + 1), sd);
        launch_flush_rows(c, c->sl_rows[par] + 2 * c->sl_cap, nullptr, c->sl_cnt[par] + 2, c->side_blocks,
                          FRUGAL_C_SIDE_HOT, sd, true, c->sl_src[par] + 2 * c->sl_cap);
        launch_flush_rows(c, c->sl_rows[par] + 3 * c->sl_cap, nullptr, c->sl_cnt[par] + 3, c->side_blocks,
                          FRUGAL_C_SIDE_HOT, sd, true, c->sl_src[par] + 3 * c->sl_cap);
        if (c->xhost) launch_set_flag(c, FLAG_SIDE, (uint32_t)(s + 1), sd);
        CKL();
    }
    CK(cudaEventRecord(c->ev_side[par], sd));
    c->side_pending[par] = true;
    c->drains_issued = s + 1;
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_step(frugal_ctx* c, int64_t s, const int64_t* ids_next_all, const int32_t* counts_next,
                                     frugal_stream stream) {
    if (!c) { set_err("NULL ctx"); return FRUGAL_EINVAL; }
    if (c->phase_in_step != 0 || s != c->cur_step + 1) {
        set_err("step(%lld) out of order (current step %lld, phase %d)", (long long)s, (long long)c->cur_step,
                c->phase_in_step);
        return FRUGAL_ESTATE;
    }
    const int64_t t = s + c->L;  // the step enqueued by this call (ingested during step s)
    if (ids_next_all) {
        if (c->ids_exhausted || c->next_prefetch != t || !counts_next) {
            set_err("step(%lld): steps 0..%lld must be enqueued first (and counts given)", (long long)s,
                    (long long)(t - 1));
            return FRUGAL_ESTATE;
        }
    } else {
        if (c->next_prefetch <= s) { set_err("step(%lld) was never enqueued", (long long)s); return FRUGAL_ESTATE; }
    }
    cudaStream_t st = (cudaStream_t)stream;
    const int par = (int)(s & 1);
    c->tstep = s;
    // the read bits of steps <= s+L-1 and the adjust list of this step are complete
    {
        const int64_t last = std::min<int64_t>(s + c->L - 1, c->next_prefetch - 1);
        CK(cudaStreamWaitEvent(st, c->ev_ingest[last % c->QN], 0));
    }
    // the bucket / age-out lists of this parity were last read by the whole drain of s-2
    if (c->side_pending[par]) CK(cudaStreamWaitEvent(st, c->ev_side[par], 0));
    if (s + c->L - 1 >= c->next_prefetch) CK(cudaMemsetAsync(c->adj_cnt[par], 0, 4, st));  // stream end: no adjust
    c->rec_transition.clear();
    if (c->dyn && c->hot_pending && s == c->hot_t0) {
        // N3 epoch boundary: the whole drain of s-1 (it reads cache slots) and the upload
        // of the new set precede the transition; it runs on the critical path
        Timer tm(c, PH_URGENT, st);
        if (s >= 1 && c->side_pending[par ^ 1]) CK(cudaStreamWaitEvent(st, c->ev_side[par ^ 1], 0));
        if (s >= 1 && c->host_flush && c->side_pending[par ^ 1])  // ... and applied by the flushing threads
            launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, (uint32_t)s, st);
        CK(cudaStreamWaitEvent(st, c->ev_hot, 0));
        launch_cache_transition(c, s, par, st);
        CK(cudaEventRecord(c->ev_hot, st));  // the next frugal_set_hot reuses new_lk after it
        CKL();
        c->hot_cur ^= 1;
        c->hot_pending = false;
        if (c->cfg.flags & FRUGAL_F_RECORD) {
            CK(cudaStreamSynchronize(st));
            int32_t nx = 0;
            CK(cudaMemcpy(&nx, c->tr_cnt + 1, 4, cudaMemcpyDeviceToHost));
            c->rec_transition.resize(nx);
            if (nx) CK(cudaMemcpy(c->rec_transition.data(), c->tr_rows, (size_t)nx * 4, cudaMemcpyDeviceToHost));
        }
    }
    {
        Timer tm(c, PH_SCHED, st);
        QueueSlot* prev = nullptr;
        if (s >= 1) {
            prev = &c->q[(s - 1) % c->QN];
            if (prev->step != s - 1) { set_err("internal: queue slot of step %lld lost", (long long)(s - 1)); return FRUGAL_ESTATE; }
        }
        launch_schedule(c, prev, s, par, st);
        CKL();
    }
    if (c->cfg.flags & FRUGAL_F_RECORD) record_schedule(c, par, st);
    if (c->urgent_side) {
        // a10 at world 1 (reading R7'): the only reader of step s is this owner, and it reads
        // every row updated within the pool window -- the whole urgent bucket (updated at s-1)
        // -- from its dirty pool in HBM, so no read of step s needs the bucket's host copies;
        // they are written off the critical path, long before any host read of those rows
        // (after the pool window, P = D+3 >= 4 steps): with the flushing threads as the last
        // part of this step's drain job, else on the side stream ahead of the drain.  Same set,
        // same bytes.
        if (!c->host_flush) {
            CK(cudaEventRecord(c->ev_sched, st));
            CK(cudaStreamWaitEvent(c->side, c->ev_sched, 0));
            Timer tm(c, PH_URGENT, c->side);
            launch_flush_rows(c, c->sl_rows[par], nullptr, c->sl_cnt[par], 1 << 30, FRUGAL_C_URGENT_HOT, c->side,
                              false, c->sl_src[par] /* sources recorded by the scheduler */);
            CKL();
        }
    } else {
        // a10: urgent bucket (priority == s) to the host table on the critical path
        Timer tm(c, PH_URGENT, st);
        launch_flush_rows(c, c->sl_rows[par], nullptr, c->sl_cnt[par], 1 << 30, FRUGAL_C_URGENT_HOT, st, false,
                          c->sl_src[par]);
        if (c->xhost) launch_set_flag(c, FLAG_URGENT, (uint32_t)(s + 1), st);
        CKL();
    }
    CK(cudaEventRecord(c->ev_sched, st));
    if (!c->drain_after_gather) {
        frugal_status r = launch_drain(c, s, st, c->ev_sched);
        if (r) return r;
    }
    // a1/a2: ingest step s+L on the ingest stream, after this step's scheduler, so it
    // overlaps the gate, the gather and the backward of step s
    if (ids_next_all) {
        frugal_status r = ingest(c, t, ids_next_all, counts_next, 1, st, c->ev_sched);
        if (r) return r;
        c->next_prefetch++;
    } else {
        c->ids_exhausted = true;
    }
    if (c->early && c->early_issued < s) {  // step 0: nothing precedes it
        frugal_status r = launch_early_gather(c, s, nullptr);
        if (r) return r;
    }
    if (c->early && !c->drain_after_gather && s + 1 < c->next_prefetch) {
        frugal_status r = launch_early_gather(c, s + 1, c->ev_side_first[par]);
        if (r) return r;
    }
    {
        // a3: gate of step s -- PQ front > s: every owner's urgent bucket s and every
        // deferred bucket drained by its side stream at steps <= s-1
        Timer tm(c, PH_GATE, st);
        // (deadline-s rows are the first part of drain s-1; the side stream is FIFO, so that
        // event also covers every earlier drain)
        static const bool strict_gate = getenv("FRUGAL_GATE_STRICT") && atoi(getenv("FRUGAL_GATE_STRICT"));
        if (!c->xhost && c->urgent_side && c->L >= 3 && !strict_gate) {
            // world 1 reading its dirty pool (R7'): step s reads from the host only rows outside
            // the pool window (last update < s-D-1, or never).  Such a row, if it was ever
            // updated, was flushed by (a) an AdjustPriority'd deferral made at s-L+1 (deadline s),
            // (b) a deferral with deadline s made at b <= s-D-1 (its update b-1 is outside the
            // window at s only if s-b > D), or (c) an age-out at a <= s-L (an aged row had no
            // read in sight, L steps).  So the gate of s needs the drains up to s - lag applied,
            // lag = min(L-1, D+1) >= 2 -- instead of the deadline-s part of drain s-1 (which
            // holds rows updated at s-2, inside the window).  The GPU drain waits for drain s-2.
            const int64_t lag = std::min<int64_t>(c->L - 1, (int64_t)c->D + 1);
            if (c->host_flush) {
                // the threads' progress word is host memory: when it already covers the job the
                // gate needs (nearly always, lag steps back) no device wait is enqueued -- a
                // device-side read of it would queue behind the pack's posted PCIe writes
                const uint32_t need = (uint32_t)(s - lag + 1);
                if (s - lag >= 0 && !seq_reached(ctl_load(c->hfl_ctl + CTL_APPLIED_ALL), need))
                    launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, need, st);
            } else if (s >= 2 && c->side_pending[par]) {
                CK(cudaStreamWaitEvent(st, c->ev_side[par], 0));
            }
        } else if (!c->xhost) {  // world 1, or the comparison path: only this rank reads its host rows
            if (s >= 1 && c->side_pending[par ^ 1]) {
                if (c->host_flush) launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_FIRST, (uint32_t)s, st);
                else CK(cudaStreamWaitEvent(st, c->ev_side_first[par ^ 1], 0));
            }
        } else {
            launch_wait_flags(c, FLAG_URGENT, (uint32_t)(s + 1), st);
            if (s >= 1) launch_wait_flags(c, FLAG_SIDE_FIRST, (uint32_t)s, st);
            CKL();
        }
    }
    c->cur_step = s;
    c->phase_in_step = 1;
    return check_err_word(c);
}

extern "C" frugal_status frugal_lookup(frugal_ctx* c, int64_t s, float* d_out, frugal_stream stream) {
    if (!c) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (c->a2a) { set_err("context uses FRUGAL_F_A2A: use frugal_a2a_requests/serve/lookup"); return FRUGAL_ESTATE; }
    if (c->phase_in_step != 1 || s != c->cur_step) {
        set_err("lookup(%lld) out of order", (long long)s);
        return FRUGAL_ESTATE;
    }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    float* rows = c->rows_buf[s & 1];
    {
        // the gather's PCIe reads would queue behind the pack's posted writes: with
        // FRUGAL_PACK_SERIAL the pack of s-1 (run beside the backward of s-1) is complete first
        if (c->pack_serial && s >= 1 && c->side_pending[(s - 1) & 1])
            CK(cudaStreamWaitEvent(st, c->ev_side[(s - 1) & 1], 0));
        Timer tm(c, PH_GATHER, st);
        if (c->early) {
            CK(cudaStreamWaitEvent(st, c->ev_early[s & 1], 0));
            launch_gather(c, q, q.lidx, q.elcnt + 1, rows, s, st);  // rows read at s-1 (updated then)
        } else {
            launch_gather(c, q, nullptr, q.n_uniq, rows, s, st);
        }
    }
    if (c->drain_after_gather) {
        CK(cudaEventRecord(c->ev_gathered, st));
        frugal_status r = launch_drain(c, s, st, c->ev_gathered);
        if (r) return r;
        if (c->early && s + 1 < c->next_prefetch) {
            r = launch_early_gather(c, s + 1, c->urgent_side ? nullptr : c->ev_side_first[s & 1]);
            if (r) return r;
        }
    }
    c->lookup_fused = d_out == nullptr;
    if (d_out) {
        Timer tm(c, PH_EXPAND, st);
        launch_expand(c, q, rows, d_out, st);
    }
    CKL();
    c->phase_in_step = 2;
    return check_err_word(c);
}

extern "C" frugal_status frugal_dot_model(frugal_ctx* c, int64_t s, const float* d_emb, const float* d_x,
                                          const float* d_y, float* d_grad, double* d_loss, frugal_stream stream) {
    if (!c || !d_x || !d_y || !d_grad || !d_loss) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (c->phase_in_step != 2 || s != c->cur_step) {
        set_err("dot_model(%lld) must follow lookup(%lld)", (long long)s, (long long)s);
        return FRUGAL_ESTATE;
    }
    if ((d_emb == nullptr) != c->lookup_fused) {
        set_err("dot_model: d_emb must be NULL exactly when lookup(%lld) ran with d_out == NULL", (long long)s);
        return FRUGAL_EINVAL;
    }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    int64_t nb = 0;
    for (int r = 0; r < c->n; r++) nb += q.h_counts[r];
    // host x / y (pinned or pageable): copied into a library staging pair (by step parity) on
    // the copy stream as soon as this call is made -- the host usually runs ahead of the GPU,
    // so the copy overlaps the step's gather
    cudaPointerAttributes ax{}, ay{};
    if (cudaPointerGetAttributes(&ax, d_x) != cudaSuccess) { cudaGetLastError(); ax.type = cudaMemoryTypeUnregistered; }
    if (cudaPointerGetAttributes(&ay, d_y) != cudaSuccess) { cudaGetLastError(); ay.type = cudaMemoryTypeUnregistered; }
    if (ax.type != cudaMemoryTypeDevice && ax.type != cudaMemoryTypeManaged) {
        const int par = (int)(s & 1);
        if (!c->x_stage[par]) {
            CK(cudaMalloc(&c->x_stage[par], (size_t)c->B * c->d * 4));
            CK(cudaMalloc(&c->y_stage[par], (size_t)c->B * 4));
        }
        const int cnt = q.h_counts[c->g];
        CK(cudaStreamWaitEvent(c->xstream, c->ev_glue[par], 0));  // the glue of s-2 read this pair
        CK(cudaMemcpyAsync(c->x_stage[par], d_x, (size_t)cnt * c->d * 4, cudaMemcpyDefault, c->xstream));
        CK(cudaMemcpyAsync(c->y_stage[par], d_y, (size_t)cnt * 4, cudaMemcpyDefault, c->xstream));
        CK(cudaEventRecord(c->ev_xy, c->xstream));
        CK(cudaStreamWaitEvent(st, c->ev_xy, 0));
        d_x = c->x_stage[par];
        d_y = c->y_stage[par];
    } else if (ay.type != cudaMemoryTypeDevice && ay.type != cudaMemoryTypeManaged) {
        set_err("dot_model: x and y must both be device or both host pointers");
        return FRUGAL_EINVAL;
    }
    Timer tm(c, PH_MODEL, st);
    if (d_emb) launch_dot_model(c, q, d_emb, nullptr, d_x, d_y, d_grad, d_loss, nb, st);
    else launch_dot_model(c, q, c->rows_buf[s & 1], q.inv, d_x, d_y, d_grad, d_loss, nb, st);
    CK(cudaEventRecord(c->ev_glue[s & 1], st));
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_transe_model(frugal_ctx* c, int64_t s, const float* d_emb, int32_t chunk, float gamma,
                                             float* d_grad, double* d_loss, frugal_stream stream) {
    if (!c || !d_emb || !d_grad || !d_loss) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (c->F != 4) { set_err("transe_model needs slots == 4 (h, r, t, neg)"); return FRUGAL_EINVAL; }
    if (chunk < 1 || chunk > 4096) { set_err("chunk must be in [1, 4096]"); return FRUGAL_EINVAL; }
    if (c->phase_in_step != 2 || s != c->cur_step) {
        set_err("transe_model(%lld) must follow lookup(%lld)", (long long)s, (long long)s);
        return FRUGAL_ESTATE;
    }
    if (c->lookup_fused) { set_err("transe_model needs the expanded rows: lookup with d_out != NULL"); return FRUGAL_EINVAL; }
    if (c->kg_C != chunk) {
        cudaFree(c->kg_W);
        cudaFree(c->kg_A);
        c->kg_W = c->kg_A = nullptr;
        CK(cudaMalloc(&c->kg_W, ((size_t)c->B + chunk) * chunk * sizeof(double)));
        CK(cudaMalloc(&c->kg_A, ((size_t)c->B + chunk) * sizeof(double)));
        c->kg_C = chunk;
    }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    int64_t nb = 0;
    for (int r = 0; r < c->n; r++) nb += q.h_counts[r];
    Timer tm(c, PH_MODEL, st);
    launch_transe_model(c, q, d_emb, chunk, (double)gamma, d_grad, d_loss, nb, c->kg_W, c->kg_A, st);
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_backward_update(frugal_ctx* c, int64_t s, const float* d_grad, frugal_stream stream) {
    if (!c || !d_grad) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (c->a2a) { set_err("context uses FRUGAL_F_A2A: use frugal_a2a_pack/update"); return FRUGAL_ESTATE; }
    if (c->phase_in_step != 2 || s != c->cur_step) {
        set_err("backward_update(%lld) out of order", (long long)s);
        return FRUGAL_ESTATE;
    }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    const int par = (int)(s & 1);
    if (c->n == 1 && c->fuse_opt && c->update1) {
        // world 1: every partial is this rank's own -- segment-reduce (short rows and the long
        // rows' chunks) and optimizer in one launch
        Timer tm(c, PH_SEGRED, st);
        launch_update1(c, q, d_grad, s, st);
    } else if (c->n == 1 && c->fuse_opt) {
        Timer tm(c, PH_SEGRED, st);
        launch_segreduce(c, q, d_grad, par, nullptr, st, s);
    } else {
        Timer tm(c, PH_SEGRED, st);
        launch_segreduce(c, q, d_grad, par, nullptr, st);
    }
    if (c->n > 1) {
        // a7: partials of rows owned by other ranks are in this rank's host mailbox;
        // publish and wait for every sender (the update staging queue, L785-789)
        Timer tm(c, PH_EXCH, st);
        launch_mail_header(c, q, par, st);
        launch_set_flag(c, FLAG_MAIL, (uint32_t)(s + 1), st);
        launch_wait_flags(c, FLAG_MAIL, (uint32_t)(s + 1), st);
    }
    if (!(c->n == 1 && c->fuse_opt)) {
        Timer tm(c, PH_OPT, st);
        launch_optimizer(c, q, s, par, nullptr, nullptr, st);
    }
    CK(cudaEventRecord(c->ev_opt[s & 1], st));
    c->opt_pending[s & 1] = true;
    CKL();
    c->phase_in_step = 0;
    c->timed_steps++;
    if ((c->cfg.flags & FRUGAL_F_TIMERS) && (c->timer_every <= 1 || (s >= 0 && s % c->timer_every == 0))) c->timer_steps++;
    return check_err_word(c);
}

// ================================================================================ comparison path
static frugal_status a2a_check(frugal_ctx* c, int64_t s, int phase, const char* what) {
    if (!c) { set_err("NULL ctx"); return FRUGAL_EINVAL; }
    if (!c->a2a) { set_err("%s needs a context created with FRUGAL_F_A2A", what); return FRUGAL_ESTATE; }
    if (c->phase_in_step != phase || s != c->cur_step) { set_err("%s(%lld) out of order", what, (long long)s); return FRUGAL_ESTATE; }
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_a2a_requests(frugal_ctx* c, int64_t s, int32_t* d_ids, int64_t* counts,
                                             frugal_stream stream) {
    if (frugal_status r = a2a_check(c, s, 1, "a2a_requests")) return r;
    if (!d_ids || !counts) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    Timer tm(c, PH_EXCH, st);
    launch_a2a_ids(c, q, d_ids, st);
    int32_t goff[33];
    CK(cudaMemcpyAsync(goff, q.goff, (size_t)(c->n + 1) * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    for (int r = 0; r < c->n; r++) counts[r] = goff[r + 1] - goff[r];
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_a2a_serve(frugal_ctx* c, int64_t s, const int32_t* d_ids_in, int64_t n_in, float* d_rows,
                                          frugal_stream stream) {
    if (frugal_status r = a2a_check(c, s, 1, "a2a_serve")) return r;
    if (n_in < 0 || (n_in && (!d_ids_in || !d_rows))) { set_err("bad arguments"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    Timer tm(c, PH_GATHER, st);
    launch_serve_rows(c, d_ids_in, n_in, s, d_rows, st);
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_a2a_lookup(frugal_ctx* c, int64_t s, const float* d_rows_in, float* d_out,
                                           frugal_stream stream) {
    if (frugal_status r = a2a_check(c, s, 1, "a2a_lookup")) return r;
    QueueSlot& q0 = c->q[s % c->QN];
    if ((!d_rows_in || !d_out) && q0.h_counts[c->g] > 0) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    float* rows = c->rows_buf[s & 1];
    {
        Timer tm(c, PH_EXPAND, st);
        launch_a2a_place(c, q, d_rows_in, rows, st);
        launch_expand(c, q, rows, d_out, st);
    }
    if (c->drain_after_gather) {
        CK(cudaEventRecord(c->ev_gathered, st));
        frugal_status r = launch_drain(c, s, st, c->ev_gathered);
        if (r) return r;
    }
    CKL();
    c->lookup_fused = false;
    c->phase_in_step = 2;
    return check_err_word(c);
}

extern "C" frugal_status frugal_a2a_pack(frugal_ctx* c, int64_t s, const float* d_grad, float* d_partials,
                                         frugal_stream stream) {
    if (frugal_status r = a2a_check(c, s, 2, "a2a_pack")) return r;
    if (!d_grad || !d_partials) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    Timer tm(c, PH_SEGRED, st);
    launch_segreduce(c, q, d_grad, (int)(s & 1), d_partials, st);
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_a2a_update(frugal_ctx* c, int64_t s, const float* d_partials_in,
                                           const int64_t* recv_counts, frugal_stream stream) {
    if (frugal_status r = a2a_check(c, s, 2, "a2a_update")) return r;
    if (!recv_counts) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    int64_t nrecv = 0;
    for (int r = 0; r < c->n; r++) nrecv += recv_counts[r];
    if (!d_partials_in && nrecv > 0) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    QueueSlot& q = c->q[s % c->QN];
    int32_t roff[33];  // pageable source: the copy is staged before cudaMemcpyAsync returns
    roff[0] = 0;
    for (int r = 0; r < c->n; r++) roff[r + 1] = roff[r] + (int32_t)recv_counts[r];
    CK(cudaMemcpyAsync(c->a2a_roff, roff, (size_t)c->n * 4, cudaMemcpyHostToDevice, st));
    {
        Timer tm(c, PH_OPT, st);
        launch_optimizer(c, q, s, (int)(s & 1), d_partials_in, c->a2a_roff, st);
    }
    CK(cudaEventRecord(c->ev_opt[s & 1], st));
    c->opt_pending[s & 1] = true;
    CKL();
    c->phase_in_step = 0;
    c->timed_steps++;
    if ((c->cfg.flags & FRUGAL_F_TIMERS) && (c->timer_every <= 1 || (s >= 0 && s % c->timer_every == 0))) c->timer_steps++;
    return check_err_word(c);
}

extern "C" frugal_status frugal_flush(frugal_ctx* c, int32_t what, frugal_stream stream) {
    if (!c) { set_err("NULL ctx"); return FRUGAL_EINVAL; }
    if (what != FRUGAL_FLUSH_ALL) { set_err("unknown flush kind %d", what); return FRUGAL_EINVAL; }
    if (c->phase_in_step != 0) { set_err("flush in the middle of a step"); return FRUGAL_ESTATE; }
    cudaStream_t st = (cudaStream_t)stream;
    for (int i = 0; i < 2; i++)
        if (c->side_pending[i]) CK(cudaStreamWaitEvent(st, c->ev_side[i], 0));
    if (c->host_flush) {  // every drain job applied by the flushing threads before the final flush
        CK(cudaStreamSynchronize(c->side));
        if (frugal_status r = wait_flushers(c)) return r;
    }
    launch_final_flush(c, st);
    CKL();
    CK(cudaStreamSynchronize(st));
    int32_t nff = 0;
    CK(cudaMemcpy(&nff, c->ff_cnt, 4, cudaMemcpyDeviceToHost));
    c->rec_final.resize(nff);
    if (nff) CK(cudaMemcpy(c->rec_final.data(), c->ff_rows, (size_t)nff * 4, cudaMemcpyDeviceToHost));
    return check_err_word(c);
}

extern "C" frugal_status frugal_destroy(frugal_ctx* c) {
    if (!c) return FRUGAL_OK;
    free_ctx(c);
    return FRUGAL_OK;
}

extern "C" const char* frugal_last_error(void) { return g_err.c_str(); }

// ================================================================================ introspection
extern "C" frugal_status frugal_get_dedup(frugal_ctx* c, int64_t t, int64_t* uniq, int32_t* inv, int64_t* n_uniq) {
    if (!c || !n_uniq) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    QueueSlot& q = c->q[t % c->QN];
    if (t < 0 || q.step != t) { set_err("step %lld is not in the sample queue", (long long)t); return FRUGAL_EINVAL; }
    CK(cudaDeviceSynchronize());
    int32_t nu = 0;
    CK(cudaMemcpy(&nu, q.n_uniq, 4, cudaMemcpyDeviceToHost));
    *n_uniq = nu;
    if (uniq && nu) {
        std::vector<int32_t> u(nu);
        CK(cudaMemcpy(u.data(), q.uniq, (size_t)nu * 4, cudaMemcpyDeviceToHost));
        for (int i = 0; i < nu; i++) uniq[i] = u[i];
    }
    const int m = q.h_counts[c->g] * c->F;
    if (inv && m) CK(cudaMemcpy(inv, q.inv, (size_t)m * 4, cudaMemcpyDeviceToHost));
    return check_err_word(c);
}

extern "C" frugal_status frugal_get_schedule(frugal_ctx* c, frugal_schedule_info* info, int64_t* urgent,
                                             int64_t* deferred, int32_t* deferred_p, int64_t* ageout) {
    if (!c || !info) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (!(c->cfg.flags & FRUGAL_F_RECORD)) { set_err("context was created without FRUGAL_F_RECORD"); return FRUGAL_ESTATE; }
    info->n_urgent = (int64_t)c->rec_urgent.size();
    info->n_deferred = (int64_t)c->rec_deferred.size();
    info->n_ageout = (int64_t)c->rec_ageout.size();
    info->gate_wait = c->rec_gate_wait;
    auto glob = [c](int32_t lk) { return (int64_t)lk * c->n + c->g; };
    if (urgent) for (size_t i = 0; i < c->rec_urgent.size(); i++) urgent[i] = glob(c->rec_urgent[i]);
    if (deferred) for (size_t i = 0; i < c->rec_deferred.size(); i++) deferred[i] = glob(c->rec_deferred[i]);
    if (deferred_p) for (size_t i = 0; i < c->rec_deferred_p.size(); i++) deferred_p[i] = c->rec_deferred_p[i];
    if (ageout) for (size_t i = 0; i < c->rec_ageout.size(); i++) ageout[i] = glob(c->rec_ageout[i]);
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_set_hot(frugal_ctx* c, int64_t t0, const int64_t* hot_ids, int64_t n_hot) {
    if (!c || n_hot < 0 || (n_hot > 0 && !hot_ids)) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (!c->dyn) { set_err("frugal_set_hot needs FRUGAL_F_DYNAMIC_CACHE"); return FRUGAL_ESTATE; }
    if (c->hot_pending) { set_err("set_hot(%lld): a change is already pending", (long long)t0); return FRUGAL_ESTATE; }
    if (t0 < 1 || t0 < c->next_prefetch) {
        set_err("set_hot(%lld): the ingest of that step was already enqueued (next: %lld)", (long long)t0,
                (long long)c->next_prefetch);
        return FRUGAL_ESTATE;
    }
    cudaStream_t is = c->istream;
    if (n_hot > c->hot_stage_cap) {  // rare: grow the device staging of the id list
        CK(cudaStreamSynchronize(is));
        if (c->hot_stage) cudaFree(c->hot_stage);
        c->hot_stage = nullptr;
        c->hot_stage_cap = 0;
        if (cudaMalloc(&c->hot_stage, (size_t)n_hot * 8) != cudaSuccess) {
            cudaGetLastError();
            set_err("set_hot: staging allocation failed");
            return FRUGAL_ENOMEM;
        }
        c->hot_stage_cap = n_hot;
    }
    // everything on the ingest stream, in order after every ingest that read the other map,
    // and after the previous transition (it read new_lk); ids are validated and filtered to
    // the owned share on the device (an id >= n_rows or a share beyond the slots fails the
    // next call)
    CK(cudaStreamWaitEvent(is, c->ev_hot, 0));
    if (n_hot) CK(cudaMemcpyAsync(c->hot_stage, hot_ids, (size_t)n_hot * 8, cudaMemcpyDefault, is));
    launch_hot_map(c, c->hot_cur ^ 1, c->hot_stage, nullptr, n_hot, true, is);
    CK(cudaEventRecord(c->ev_hot, is));
    CKL();
    c->hot_t0 = t0;
    c->hot_pending = true;
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_get_transition(frugal_ctx* c, int64_t* rows, int64_t* n) {
    if (!c || !n) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    *n = (int64_t)c->rec_transition.size();
    if (rows) for (size_t i = 0; i < c->rec_transition.size(); i++) rows[i] = (int64_t)c->rec_transition[i] * c->n + c->g;
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_get_final_flush(frugal_ctx* c, int64_t* rows, int64_t* n) {
    if (!c || !n) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    *n = (int64_t)c->rec_final.size();
    if (rows) for (size_t i = 0; i < c->rec_final.size(); i++) rows[i] = (int64_t)c->rec_final[i] * c->n + c->g;
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_read_rows(frugal_ctx* c, const int64_t* ids, int64_t n, float* w, float* G) {
    if (!c || (n && (!ids || !w))) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    if (n == 0) return FRUGAL_OK;
    std::vector<int32_t> lk(n);
    for (int64_t i = 0; i < n; i++) {
        if (ids[i] < 0 || ids[i] >= c->N || ids[i] % c->n != c->g) {
            set_err("read_rows: id %lld is not owned by rank %d", (long long)ids[i], c->g);
            return FRUGAL_EINVAL;
        }
        lk[i] = (int32_t)(ids[i] / c->n);
    }
    CK(cudaDeviceSynchronize());
    if (frugal_status r = wait_flushers(c)) return r;
    int32_t* d_lk;
    float *d_w, *d_G;
    CK(cudaMalloc(&d_lk, n * 4));
    CK(cudaMalloc(&d_w, n * c->d * 4));
    CK(cudaMalloc(&d_G, n * c->d * 4));
    cudaMemcpy(d_lk, lk.data(), n * 4, cudaMemcpyHostToDevice);
    launch_read_rows(c, d_lk, n, d_w, d_G, 0);
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) {
        cudaMemcpy(w, d_w, n * c->d * 4, cudaMemcpyDeviceToHost);
        if (G) cudaMemcpy(G, d_G, n * c->d * 4, cudaMemcpyDeviceToHost);
    }
    cudaFree(d_lk);
    cudaFree(d_w);
    cudaFree(d_G);
    if (e != cudaSuccess) { set_err("read_rows: %s", cudaGetErrorString(e)); return FRUGAL_ECUDA; }
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_read_host(frugal_ctx* c, const int64_t* ids, int64_t n, float* w, float* G) {
    if (!c || (n && (!ids || !w))) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    CK(cudaDeviceSynchronize());
    if (frugal_status r = wait_flushers(c)) return r;
    for (int64_t i = 0; i < n; i++) {
        if (ids[i] < 0 || ids[i] >= c->N) { set_err("read_host: id out of range"); return FRUGAL_EINVAL; }
        const int64_t hk = c->hs_host.empty() ? ids[i] : c->hs_host[ids[i]];  // host_order layout
        memcpy(w + i * c->d, c->h_w + hk * c->d, c->d * 4);
        if (G) {
            if (c->h_G) memcpy(G + i * c->d, c->h_G + hk * c->d, c->d * 4);
            else memset(G + i * c->d, 0, c->d * 4);
        }
    }
    return FRUGAL_OK;
}

// timeline of the recorded phases (FRUGAL_F_TIMERS): for each of the last `cap` recorded
// phase instances, (phase, start_ms, end_ms) relative to the first recorded event.  Call
// before frugal_get_stats (which consumes the events).
extern "C" frugal_status frugal_get_timeline(frugal_ctx* c, int32_t* phase, double* t0, double* t1, int64_t cap,
                                             int64_t* n) {
    if (!c || !n) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    CK(cudaDeviceSynchronize());
    *n = (int64_t)c->evs.size();
    if (!phase || c->evs.empty()) return FRUGAL_OK;
    const size_t first = c->evs.size() > (size_t)cap ? c->evs.size() - (size_t)cap : 0;
    cudaEvent_t ref = c->evs[first].a;
    for (size_t i = first; i < c->evs.size(); i++) {
        float a = 0.f, b = 0.f;
        cudaEventElapsedTime(&a, ref, c->evs[i].a);
        cudaEventElapsedTime(&b, ref, c->evs[i].b);
        phase[i - first] = c->evs[i].phase;
        t0[i - first] = a;
        t1[i - first] = b;
    }
    cudaGetLastError();
    *n = (int64_t)(c->evs.size() - first);
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_get_stats(frugal_ctx* c, frugal_stats* out) {
    if (!c || !out) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    CK(cudaDeviceSynchronize());
    for (auto& e : c->evs) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, e.a, e.b) == cudaSuccess) c->phase_ms[e.phase] += ms;
    }
    cudaGetLastError();
    c->evs.clear();
    c->ev_used = 0;
    for (int i = 0; i < FRUGAL_N_PHASES; i++) out->ms[i] = c->phase_ms[i];
    out->steps = c->timed_steps;
    out->timer_steps = c->timer_steps;
    out->host_wait_ms = c->host_wait_ns * 1e-6;
    c->host_wait_ns = 0;
    c->timer_steps = 0;
    out->kernel_launches = c->launches;
    unsigned long long cnt[FRUGAL_N_COUNTERS];
    CK(cudaMemcpy(cnt, c->dstats, sizeof cnt, cudaMemcpyDeviceToHost));
    for (int i = 0; i < FRUGAL_N_COUNTERS; i++) out->count[i] = (int64_t)cnt[i];
    for (int i = 0; i < FRUGAL_N_PHASES; i++) c->phase_ms[i] = 0;
    c->timed_steps = 0;
    out->flush_jobs = 0;
    out->flush_ms = out->flush_wait_ms = 0.0;
    if (c->flushers) {
        out->flush_jobs = c->flushers->jobs.exchange(0);
        out->flush_ms = c->flushers->busy_ns.exchange(0) * 1e-6;
        out->flush_wait_ms = c->flushers->wait_ns.exchange(0) * 1e-6;
    }
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_probe_host_reads(frugal_ctx* c, int64_t n, uint64_t seed, double* ms) {
    if (!c || !ms || n <= 0) { set_err("bad arguments"); return FRUGAL_EINVAL; }
    if (c->phase_in_step != 0) { set_err("probe in the middle of a step"); return FRUGAL_ESTATE; }
    CK(cudaDeviceSynchronize());
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    const int64_t out_rows = std::min<int64_t>(n, c->M);
    CK(cudaEventRecord(a, 0));
    launch_probe_rows(c, n, seed, c->chunk_scratch, out_rows, 0);
    CK(cudaEventRecord(b, 0));
    CK(cudaEventSynchronize(b));
    float f = 0.f;
    cudaEventElapsedTime(&f, a, b);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    *ms = f;
    CKL();
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_join(frugal_ctx* c, frugal_stream stream) {
    if (!c) { set_err("NULL ctx"); return FRUGAL_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    for (cudaStream_t s : {c->istream, c->side, c->pstream}) {
        if (!s) continue;
        cudaEvent_t e;
        CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        cudaError_t r1 = cudaEventRecord(e, s);
        cudaError_t r2 = r1 == cudaSuccess ? cudaStreamWaitEvent(st, e, 0) : r1;
        cudaEventDestroy(e);  // released once the wait resolves
        if (r2 != cudaSuccess) { set_err("join: %s", cudaGetErrorString(r2)); return FRUGAL_ECUDA; }
    }
    // host flushing threads: every drain job issued so far applied to the host table
    if (c->host_flush && c->drains_issued > 0) {
        launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, (uint32_t)c->drains_issued, st);
        CKL();
    }
    return FRUGAL_OK;
}

extern "C" frugal_status frugal_probe_fp64(int32_t device, double* ops_per_s) {
    if (!ops_per_s) { set_err("NULL argument"); return FRUGAL_EINVAL; }
    CK(cudaSetDevice(device));
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    double* out = nullptr;
    CK(cudaMalloc(&out, 1 << 20));
    int64_t ops = 0;
    launch_probe_fp64(out, 1, &ops, 0);  // warm-up
    CK(cudaEventRecord(a, 0));
    launch_probe_fp64(out, 64, &ops, 0);
    CK(cudaEventRecord(b, 0));
    CK(cudaEventSynchronize(b));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(out);
    CKL();
    *ops_per_s = ms > 0 ? (double)ops / (ms * 1e-3) : 0.0;
    return FRUGAL_OK;
}

extern "C" int64_t frugal_owned_rows(frugal_ctx* c) { return c ? c->No : -1; }
extern "C" int64_t frugal_hot_slots(frugal_ctx* c) { return c ? c->cap_hot : -1; }
