// frugal_internal.cuh -- shared device/host declarations of libfrugal (CUDA path only).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "frugal.h"

namespace frugal {

constexpr int kSMs = 148;              // B200
constexpr int kThreads = 256;          // default block size
constexpr int kTile = 256;             // radix/scan tile (elements per block iteration)
constexpr int32_t kInfP = 0x7fffffff;  // priority "infinity" (Eq. (1) second case)

// per-owned-row state (the g-entry, made dense)
enum RowState : int32_t {
    ST_CLEAN = 0,    // no pending update (W set empty) or flush already scheduled
    ST_UPDATED = 1,  // updated at last_upd, not yet prioritised
    ST_INF = 2,      // dirty, no read within the lookahead window (priority inf)
    ST_EXEMPT = 3    // dirty hot row whose next reader is only its owner (cache hit)
};

// ---------------------------------------------------------------- radix sort
// Stable LSD radix sort of (uint32 key, int32 val) pairs, device-resident count.
struct SortScratch {
    uint32_t* k[2] = {nullptr, nullptr};
    int32_t* v[2] = {nullptr, nullptr};
    int32_t* hist = nullptr;  // [256][nblk]
    int nblk = 0;
    int64_t cap = 0;
};
void sort_alloc(SortScratch& s, int64_t cap);
void sort_free(SortScratch& s);
// Sorts keys/vals of length *d_n (<= cap) held in s.k[0]/s.v[0]; returns index of
// the buffer holding the result (0 or 1).  Only bits [0, bits) of the keys matter.
int sort_pairs(SortScratch& s, const int32_t* d_n, int bits, cudaStream_t st, int64_t* launches);

// ---------------------------------------------------------------- scan
struct ScanScratch {
    int32_t* part = nullptr;
    int nblk = 0;
};
void scan_alloc(ScanScratch& s, int64_t cap);
void scan_free(ScanScratch& s);

// ---------------------------------------------------------------- sample-queue slot
struct QueueSlot {
    int64_t step = -1;      // which step this slot holds
    int32_t* ids = nullptr;     // [world][M] int32 (converted, validated)
    int32_t* counts = nullptr;  // [world] device
    int32_t* m = nullptr;       // device scalar: counts[g] * slots
    std::vector<int32_t> h_counts;
    // own dedup (rank g)
    int32_t* uniq = nullptr;  // [M] ascending
    int32_t* inv = nullptr;   // [M]
    int32_t* off = nullptr;   // [M+1] CSR offsets
    int32_t* pos = nullptr;   // [M] positions grouped by uniq, ascending within
    int32_t* n_uniq = nullptr;  // device scalar
    // owner side: T = owned rows read at this step by any rank, ascending
    int32_t* T = nullptr;      // [capT] local row index lk = k / world
    uint32_t* Tmask = nullptr; // [capT] rank mask
    int32_t* Tidx = nullptr;   // [world][capT] index of T[j] in rank r's owner segment
    int32_t* nT = nullptr;     // device scalar
    // gather split (world 1): uniq indices whose row was not read at t-1 ("early": can be
    // gathered during step t-1) and the rest ("late": after gate t)
    int32_t* eidx = nullptr;   // [M]
    int32_t* lidx = nullptr;   // [M]
    int32_t* elcnt = nullptr;  // [2] early, late counts
    // world 1, fused update: the long segments (> 64 occurrences, Zipf head) of this step,
    // found at ingest: per long row {u, first task, chunks}, one task per 64-chunk
    // {begin, end, long row, chunk}, arrival counters, counts {long rows, tasks}
    int4* linfo = nullptr;     // [M/65 + 1]
    int4* ltask = nullptr;     // [M/64 + M/65 + 2]
    int32_t* lcnt = nullptr;   // [M/65 + 1]
    int32_t* lnum = nullptr;   // [2]
    // sender side grouping (world > 1): uniq positions grouped by owner
    int32_t* gl = nullptr;     // [M] grouped position -> uniq index
    int32_t* goff = nullptr;   // [world+1]
};

struct PhaseEv {
    int phase;
    cudaEvent_t a, b;
};

struct HostShared;  // shm segment layout (runtime.cu)
struct Flushers;    // host flushing threads (runtime.cu)
// control words of the drain staging queue (uint32, host memory): the device writes READY
// (job seq of each parity buffer) and the part sizes; the flushing threads write APPLIED_*
enum { CTL_READY = 0, CTL_N1 = 2, CTL_NTOT = 4, CTL_READY1 = 8, CTL_APPLIED_FIRST = 16, CTL_APPLIED_ALL = 32 };

// NVLink-native variant (FRUGAL_F_PEER): every rank's HBM cache / pool / metadata, opened
// through CUDA IPC (device pointers valid in this process)
struct PeerTab {
    const float4* cw[32];
    const float4* pw[32];
    const int32_t* lu[32];
    const int32_t* pi[32];
    int64_t capT[32];
};

}  // namespace frugal

struct frugal_ctx {
    frugal_config cfg;
    int n, g, d, F, B, L, D, M;  // world, rank, dim, slots, batch, lookahead, age_out, B*F
    int64_t N, No;               // rows, owned rows
    int P;                       // pool segments = D + 3
    int QN;                      // sample-queue slots = L + 2 (steps s-1 .. s+L)
    int side_blocks = 20;        // grid cap of the side-stream drain: its zero-copy D2H stores slow the concurrent backward kernels, 16-24 CTAs balance the two (profiles/r1_sweep15.txt)
    int32_t* hs = nullptr;           // [N] host-table slot of every global row (host_order), or null
    std::vector<int32_t> hs_host;    // host copy (frugal_read_host)
    int side_first_blocks = 20;      // grid cap of the drain's deadline-(s+1) part
    int pack_blocks = 20;            // grid cap of the drain's pack kernel (flushing-thread drain)
    int pack_rows = 1;               // rows in flight per lane group in the pack kernel (FRUGAL_PACK_ROWS=4)
    int pack_threads = 256;          // threads per CTA of the pack kernel (FRUGAL_PACK_THREADS)
    bool pack_ce = false;            // pack into HBM, the flushing threads move it D2H with cudaMemcpyAsync (FRUGAL_PACK_CE=1)
    cudaStream_t ce_stream = nullptr; // their copy stream
    bool pack_2stage = false;        // pack via a contiguous HBM run + an 8-CTA sequential copy (FRUGAL_PACK_2STAGE=1)
    bool pack_tma = false;           // pack chunks staged in smem, written by TMA bulk copies (FRUGAL_PACK_TMA=1)
    float* dst_rows[2] = {nullptr, nullptr};    // HBM staging of the two-stage pack
    int64_t* dst_keys[2] = {nullptr, nullptr};
    int flush_tma = 0;               // flushes by TMA bulk stores: 0 none, 1 side drain, 2 all (FRUGAL_FLUSH_TMA; measured no gain: profiles/r1_sweep21_flush_tma.txt)
    int glue_cache = -1;         // REC glue keeps a sample's rows in registers (F <= 32): -1 auto, 0 never, 1 always
    bool update_short8 = false;
    bool update_dyn = false;     // k_update1: warps fetch batches of work items from a counter (FRUGAL_UPDATE_DYN=1; measured slower)   // k_update1: rows with <= 8 occurrences load all their gradient rows at once (FRUGAL_UPDATE_SHORT)
    int glue_unroll = 8;         // REC glue k_dot_rg: rows of a sample in flight (FRUGAL_GLUE_UNROLL; 1 = round-1 order of loads)
    bool glue_rg = true;         // REC glue: row-group kernel k_dot_rg (FRUGAL_GLUE_RG=0: the warp-per-sample k_dot_model)
    bool fuse_opt = true;        // world 1: a8 fused into a6 (k_segreduce / k_segred_combine)
    bool update1 = true;         // world 1 fused: one-launch k_update1 (FRUGAL_UPDATE1=0: the 3-kernel path)
    int gather_blocks = 120;     // grid cap of the zero-copy gathers (120 CTAs: +3% over 74 and 148 in the step, profiles/r1_sweep34_gather_grid.txt)
    bool side_inline = false;    // experiment: drain on the caller stream
    int gather_rows = 1;         // rows in flight per lane group in the gather (FRUGAL_GATHER_ROWS)
    bool pack_serial = false;    // the gather of s+1 waits for the pack of s (no posted writes beside it)
    bool drain_after_gather = true;  // side drain after the step's gather (FRUGAL_DRAIN_AT=sched: after the scheduler)
    bool urgent_side = false;        // world 1: urgent flush on the side stream (reading R7'), see frugal_step
    int64_t capT;                // max owned rows touched per step
    int key_bits, lk_bits;       // bits of global ids / local ids

    // host table (pinned/registered) and its device aliases
    void* shm_base = nullptr;
    size_t shm_bytes = 0;
    int shm_fd = -1;
    bool shm_owner = false;
    float* h_w = nullptr;  // host pointers
    float* h_G = nullptr;
    float* dh_w = nullptr;  // device-side aliases (mapped)
    float* dh_G = nullptr;
    // cross-rank flags and mailboxes (world > 1), host memory
    volatile uint32_t* h_flags = nullptr;
    uint32_t* dh_flags = nullptr;
    char* h_mail = nullptr;
    char* dh_mail = nullptr;
    size_t mail_stride = 0;  // bytes per (parity, sender) mailbox region

    // per-owned-row metadata (HBM)
    int32_t* slot = nullptr;      // [No] cache slot or -1
    int32_t* state = nullptr;     // [No]
    int32_t* last_upd = nullptr;  // [No]
    int32_t* pool_idx = nullptr;  // [No]
    uint64_t* rbits = nullptr;    // [No] low 32: any-reader ring, high 32: host-reader ring

    // HBM cache of owned hot rows
    int64_t cap_hot = 0;
    float* cw = nullptr;        // [cap_hot][d] w of the owned hot rows
    float* Gd = nullptr;        // [No][d] Adagrad state of every owned row (HBM-resident, R8)
    int32_t* hot_lk = nullptr;  // [cap_slots] local index held by each slot, -1 = free

    // N3 dynamic cache (FRUGAL_F_DYNAMIC_CACHE, frugal_set_hot): the hot set changes at epoch
    // boundaries t0; cap_slots >= cap_hot leaves room for the owned share to grow
    bool dyn = false;
    int64_t cap_slots = 0;
    uint32_t* hot_map[2] = {nullptr, nullptr}; // [(No+31)/32] hot bits used by the ingest of a step
    int hot_cur = 0;                           // map of the epoch in force
    bool hot_pending = false;                  // a frugal_set_hot waits for its t0
    int64_t hot_t0 = -1;                       // first step of the pending epoch
    int32_t* new_lk = nullptr;                 // [cap_slots] owned share of the pending hot set
    int64_t* hot_stage = nullptr;              // device copy of the ids passed to frugal_set_hot
    int64_t hot_stage_cap = 0;
    int32_t* free_slots = nullptr;             // [cap_slots] stack of free slots
    int32_t* tr_cnt = nullptr;                 // [3]: free-stack size, transition-list size, |new_lk|
    int32_t* tr_rows = nullptr;                // [capT + cap_slots] rows flushed by the transition
    cudaEvent_t ev_hot = nullptr;              // pending map / list uploaded
    std::vector<int32_t> rec_transition;

    // dirty-row pool for cold owned rows: P segments x capT rows
    float* pw = nullptr;        // [P][capT][d] w of updated cold rows until flushed
    int32_t* pkey = nullptr;   // [P][capT] local index
    int32_t* pcount = nullptr; // [P]

    // sample queue
    std::vector<frugal::QueueSlot> q;

    // per-step scratch
    float* rows_buf[2] = {nullptr, nullptr};  // [M][d] gathered unique rows, by step parity
    float* Pp = nullptr;    // [M][d] partials (grouped order for world > 1)
    float* chunk_scratch = nullptr;  // [M][d] chunk sums of long segments
    int32_t* long_q = nullptr;       // [M] long segments of the current step
    int32_t* long_cnt = nullptr;     // [2]: long segments, chunk tasks
    int32_t* upd_ctr = nullptr;      // [2]: k_update1 work counters by step parity (dynamic fetch)
    int2* long_tasks = nullptr;      // [M/32 + 2] chunk [begin, end) positions
    int32_t* owned_cnt = nullptr;  // scalar
    // schedule lists (double buffered by step parity): 4 lists of sl_cap rows each --
    // 0 urgent (deadline s), 1 next (deadline s+1), 2 later (> s+1), 3 age-out; deadlines
    // of lists 0..2 in sl_p; the 4 counts in sl_cnt
    int64_t sl_cap = 0;
    int32_t* sl_rows[2] = {nullptr, nullptr};
    int32_t* sl_p[2] = {nullptr, nullptr};
    int32_t* sl_src[2] = {nullptr, nullptr};  // [4][sl_cap]: each listed row's source at schedule time (-1-slot | pool row)
    int32_t* sl_cnt[2] = {nullptr, nullptr};
    int32_t* adj_rows[2] = {nullptr, nullptr};  // AdjustPriority inf -> t rows, by consuming step parity
    int32_t* adj_p[2] = {nullptr, nullptr};
    int32_t* adj_cnt[2] = {nullptr, nullptr};
    int32_t* err = nullptr;   // device alias of the error word (mapped pinned host memory)
    int32_t* herr = nullptr;  // host pointer of the same word
    int32_t* sched_info = nullptr;  // device [4]
    int32_t* ff_rows = nullptr;  // final flush list
    int32_t* ff_cnt = nullptr;
    int64_t* ids_stage = nullptr;  // device int64 staging for incoming ids [world][M]
    int32_t* counts_pin = nullptr;  // pinned [L+1][world] staging of per-step counts
    std::vector<cudaEvent_t> ev_counts;  // one per queue slot: staging reusable

    frugal::SortScratch sort;
    frugal::ScanScratch scan;

    cudaStream_t side = nullptr;
    cudaStream_t istream = nullptr;  // sample-queue ingest, one step ahead
    cudaEvent_t ev_call = nullptr, ev_copied = nullptr, ev_gathered = nullptr;
    std::vector<cudaEvent_t> ev_ingest;  // per queue slot: ingest complete
    cudaEvent_t ev_sched = nullptr;
    cudaEvent_t ev_side[2] = {nullptr, nullptr};
    cudaEvent_t ev_side_first[2] = {nullptr, nullptr};  // side drain of the next step's deadline done
    cudaStream_t pstream = nullptr;                     // early gather of the next step
    cudaEvent_t ev_early[2] = {nullptr, nullptr};
    cudaEvent_t ev_opt[2] = {nullptr, nullptr};         // optimizer of a step done (rows_buf free)
    bool opt_pending[2] = {false, false};
    int64_t early_issued = -1;                          // last step whose early gather was launched
    bool early = false;                                 // pipelined gather enabled (world 1)
    bool pool_hits = true;                              // owner reads its dirty-pool rows from HBM
    int early_blocks = 16;                              // grid of the early gather
    int early_rows = 4;                                 // rows in flight per lane group in the early gather
    bool early_on_side = false;                         // early gather queued behind the drain
    bool a2a = false;                                   // comparison path (FRUGAL_F_A2A)
    bool peer = false;                                  // NVLink-native variant (FRUGAL_F_PEER)
    frugal::PeerTab* peer_tab = nullptr;                // device copy
    void* peer_open[32][4] = {};                        // opened IPC mappings (to close)
    int32_t* gslot = nullptr;                           // [N] owner's cache slot of every hot row
    bool xhost = false;                                 // world > 1 and host-bounced exchange
    bool own_ids = false;                               // FRUGAL_F_OWN_IDS: ingest v2 (id mailbox)
    char* dh_idbox = nullptr;                           // device alias of the id mailbox [kIdSlots][world]
    size_t idbox_stride = 0;                            // bytes per (slot, rank): 256 B header + M int32
    int32_t* a2a_roff = nullptr;                        // [world] receive offsets (device)
    bool side_pending[2] = {false, false};

    // call-order state
    int64_t next_prefetch = 0;  // next t expected by prefetch/step
    int64_t cur_step = -1;
    int phase_in_step = 0;  // 0 = need step, 1 = need lookup, 2 = need backward
    bool lookup_fused = false;  // lookup(s) ran with d_out == NULL: the glue reads rows_buf through inv
    bool ids_exhausted = false;

    // KG glue scratch (allocated on first use): W [batch][C] and A [batch] (fp64)
    double* kg_W = nullptr;
    double* kg_A = nullptr;
    int kg_C = 0;

    // host flushing threads (default; FRUGAL_F_GPU_DRAIN: off): the side drain is packed into a pinned staging
    // queue (2 buffers, by step parity) and copied into the host table by these threads
    bool host_flush = false;
    int n_flushers = 0;
    frugal::Flushers* flushers = nullptr;
    float* hfl_rows[2] = {nullptr, nullptr};     // host pointers of the staging rows [cap][d]
    int64_t* hfl_keys[2] = {nullptr, nullptr};   // host-table row slot of each staged row
    float* dfl_rows[2] = {nullptr, nullptr};     // device aliases
    int64_t* dfl_keys[2] = {nullptr, nullptr};
    uint32_t* hfl_ctl = nullptr;                 // control words (host): ready[2], n1[2], ntot[2], ...
    uint32_t* dfl_ctl = nullptr;                 // device alias
    int64_t drains_issued = 0;                   // drain jobs published so far (job s = drain of step s)

    // ingest as CUDA graphs (one per queue slot; FRUGAL_GRAPHS=0: direct launches)
    bool use_graphs = true;
    cudaStream_t gstream = nullptr;              // capture stream
    std::vector<cudaGraphExec_t> ingest_exec;    // [QN]
    std::vector<int64_t> ingest_nodes;           // kernels per graph (launch counter)
    int32_t* d_iprm = nullptr;                   // [QN][IP_N] device
    int32_t* h_iprm = nullptr;                   // [QN][IP_N] pinned staging

    // host dense inputs of the REC glue (frugal_dot_model with host x / y): staging by step parity
    cudaStream_t xstream = nullptr;
    cudaEvent_t ev_xy = nullptr, ev_glue[2] = {nullptr, nullptr};
    float* x_stage[2] = {nullptr, nullptr};
    float* y_stage[2] = {nullptr, nullptr};

    // instrumentation
    int64_t launches = 0;
    std::vector<frugal::PhaseEv> evs;
    std::vector<cudaEvent_t> ev_pool;
    size_t ev_used = 0;
    double phase_ms[FRUGAL_N_PHASES] = {0};
    int64_t timed_steps = 0;
    int64_t tstep = -1;            // step of the current frugal_step call (phase-timer sampling)
    int timer_every = 1;           // FRUGAL_TIMER_EVERY: phase timers on steps s % k == 0 only
    int64_t timer_steps = 0;
    int64_t host_wait_ns = 0;      // host time blocked in the ingest's buffer-reuse waits since the last get_stats       // steps whose phases were timed since the last get_stats
    unsigned long long* dstats = nullptr;  // device counters [FRUGAL_N_COUNTERS]
    // recorded schedule artefacts (FRUGAL_F_RECORD)
    std::vector<int32_t> rec_urgent, rec_deferred, rec_deferred_p, rec_ageout, rec_final;
    int rec_gate_wait = 0;
};

namespace frugal {
// kernels' host launchers (kernels.cu)
void launch_convert_ids(frugal_ctx* c, QueueSlot& q, cudaStream_t st);
void launch_dedup(frugal_ctx* c, QueueSlot& q, cudaStream_t st);
void launch_owner_side(frugal_ctx* c, QueueSlot& q, int64_t t, cudaStream_t st);
void launch_owner_side_v2(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st);
void launch_set_flag_prm(frugal_ctx* c, int which, const int32_t* prm, cudaStream_t st);
void launch_wait_flags_prm(frugal_ctx* c, int which, const int32_t* prm, cudaStream_t st);
constexpr int kIdSlots = 4;  // id-mailbox slots (step t uses slot t % kIdSlots)
enum { FLAG_IDS_KIND = 4 };  // host flag kind: this rank's distinct ids of step t published (t+1)
void launch_cache_transition(frugal_ctx* c, int64_t s, int par, cudaStream_t st);
void launch_hot_map(frugal_ctx* c, int which, const int64_t* ids64, const int32_t* lks, int64_t n, bool list,
                    cudaStream_t st);
// per-step parameters of the ingest (device words, one block of IP_N per queue slot): the
// ingest's kernels read them, so its launch sequence is the same every step and is replayed
// as one CUDA graph per queue slot
enum { IP_T = 0, IP_APAR = 1, IP_ADJUST = 2, IP_HMAP = 3, IP_IDSLOT = 4, IP_FLAGV = 5, IP_N = 8 };
void launch_ingest_prologue(frugal_ctx* c, const int32_t* prm, cudaStream_t st);
void launch_ingest_bits(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st);
void launch_schedule(frugal_ctx* c, QueueSlot* prev, int64_t s, int par, cudaStream_t st);
void launch_flush_rows(frugal_ctx* c, const int32_t* rows, const int32_t* d_begin, const int32_t* d_end,
                       int max_blocks, int counter, cudaStream_t st, bool side = false,
                       const int32_t* srcs = nullptr);
void launch_pack_drain(frugal_ctx* c, int par, uint32_t seq, int max_blocks, cudaStream_t st);
void launch_wait_word(frugal_ctx* c, const uint32_t* dflag, uint32_t value, cudaStream_t st);
void launch_gather(frugal_ctx* c, QueueSlot& q, const int32_t* list, const int32_t* cnt, float* rows, int64_t step,
                   cudaStream_t st);
void launch_expand(frugal_ctx* c, QueueSlot& q, const float* rows, float* out, cudaStream_t st);
void launch_probe_rows(frugal_ctx* c, int64_t n, uint64_t seed, float* out, int64_t out_rows, cudaStream_t st);
void launch_split_early(frugal_ctx* c, QueueSlot& q, const int32_t* prm, cudaStream_t st);
void launch_mail_header(frugal_ctx* c, QueueSlot& q, int par, cudaStream_t st);
void launch_transe_model(frugal_ctx* c, QueueSlot& q, const float* emb, int C, double gamma, float* grad,
                         double* loss, int64_t nb, double* Wm, double* A, cudaStream_t st);
void launch_dot_model(frugal_ctx* c, QueueSlot& q, const float* emb, const int32_t* inv, const float* x,
                      const float* y, float* grad, double* loss, int64_t nb, cudaStream_t st);
void launch_segreduce(frugal_ctx* c, QueueSlot& q, const float* grad, int par, float* dest, cudaStream_t st, int64_t fused_step = -1);
void launch_long_tasks(frugal_ctx* c, QueueSlot& q, cudaStream_t st);
void launch_update1(frugal_ctx* c, QueueSlot& q, const float* grad, int64_t s, cudaStream_t st);
void launch_optimizer(frugal_ctx* c, QueueSlot& q, int64_t s, int par, const float* recv, const int32_t* roff,
                      cudaStream_t st);
void launch_a2a_ids(frugal_ctx* c, QueueSlot& q, int32_t* ids, cudaStream_t st);
void launch_serve_rows(frugal_ctx* c, const int32_t* ids, int64_t n, int64_t s, float* out, cudaStream_t st);
void launch_a2a_place(frugal_ctx* c, QueueSlot& q, const float* in, float* rows, cudaStream_t st);
void launch_final_flush(frugal_ctx* c, cudaStream_t st);
void launch_init_table(frugal_ctx* c, cudaStream_t st);
void launch_init_meta(frugal_ctx* c, const int64_t* d_hot_global, int64_t n_hot, cudaStream_t st);
void launch_wait_flags(frugal_ctx* c, int which, uint32_t value, cudaStream_t st);
void launch_set_flag(frugal_ctx* c, int which, uint32_t value, cudaStream_t st);
void launch_read_rows(frugal_ctx* c, const int32_t* d_lk, int64_t n, float* d_w, float* d_G, cudaStream_t st);
void launch_read_host(frugal_ctx* c, const int64_t* d_k, int64_t n, float* d_w, float* d_G, cudaStream_t st);
cudaError_t setup_kernel_attrs();
void launch_probe_fp64(double* out, int iters, int64_t* ops, cudaStream_t st);
}  // namespace frugal
