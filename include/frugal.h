/*
 * frugal.h -- C ABI of the B200-native Frugal training-step hot path.
 *
 * Frugal (Xie et al., ASPLOS '25; /root/reference/PAPER.md) trains embedding
 * models on several GPUs that share one parameter table in pinned host memory.
 * Each GPU keeps a private cache of hot rows; rows updated on one GPU are
 * *proactively flushed* to host memory before any GPU reads them again
 * (§3.1), scheduled by a priority = next access step (Eq. (1),
 * L902-911) held in a two-level priority queue (§3.4).
 *
 * One process per GPU, one context per process.  Every call returns a
 * frugal_status (0 = ok, < 0 = error; the text is in frugal_last_error()); no
 * call throws, aborts or exits.  Device work is enqueued asynchronously on the
 * caller's stream `stream` (plus one library-owned low-priority side stream);
 * calls on one context are not thread-safe.
 *
 * Row ids are GLOBAL ids in [0, n_rows) (table offset + local id; slot f of a
 * sample reads table f).  Position i of a rank's step is i = b*slots + f.
 * Rank g owns row k iff k mod world == g (reading R12 in DESIGN.md): the owner
 * caches it if hot and applies its optimizer update (R6).
 *
 * Per-step call order (after frugal_prefetch(t) for t = 0 .. L-1):
 *     frugal_step(s) [enqueues step s+L] -> frugal_lookup(s) -> [model] ->
 *     frugal_backward_update(s)
 * and frugal_flush(FRUGAL_FLUSH_ALL) at the end of training.  Any other order
 * returns FRUGAL_ESTATE.
 */
#ifndef FRUGAL_H
#define FRUGAL_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct frugal_ctx frugal_ctx;
typedef void* frugal_stream; /* a cudaStream_t (NULL = legacy default stream) */

typedef enum {
    FRUGAL_OK = 0,
    FRUGAL_EINVAL = -1,   /* bad argument / config, or an id >= n_rows seen by a kernel */
    FRUGAL_ENOMEM = -2,   /* device or pinned-host allocation failed */
    FRUGAL_ECUDA = -3,    /* a CUDA runtime/driver call failed */
    FRUGAL_ESTATE = -4,   /* out-of-order call (e.g. lookup(s) before step(s)) */
    FRUGAL_ETIMEOUT = -5, /* a peer rank never published a flag */
    FRUGAL_ESHM = -6      /* shared-memory host table could not be created/attached */
} frugal_status;

typedef enum { FRUGAL_SGD = 0, FRUGAL_ADAGRAD = 1 } frugal_opt;

typedef enum {
    FRUGAL_MODE_P2F = 0,          /* priority-based proactive flushing (§3.3) */
    FRUGAL_MODE_WRITE_THROUGH = 1 /* Frugal-Sync baseline: every update flushed on the
                                     critical path of the next step (§4.1) */
} frugal_mode;

enum {
    FRUGAL_F_RECORD = 1,        /* keep per-step schedule artefacts for frugal_get_schedule  */
    FRUGAL_F_TIMERS = 2,        /* record CUDA events around every phase (frugal_get_stats)  */
    FRUGAL_F_NO_HOST_STATE = 4, /* Adagrad: no host copy of G (it lives in HBM, R8); the final
                                   flush then writes w only -- for tables whose w and G do not
                                   both fit in host memory (e.g. configs[3], 2 x 138 GB)      */
    FRUGAL_F_PEER = 16,         /* NVLink-native variant: a non-owned row
                                   the owner holds in HBM (cache, or dirty pool) is loaded from
                                   the owner's GPU over peer memory (CUDA IPC) instead of the
                                   host table; flush schedule and results unchanged; world > 1 */
    FRUGAL_F_DYNAMIC_CACHE = 32,/* N3: the hot set may change at epoch
                                   boundaries (frugal_set_hot); the cache gets 25% spare
                                   slots; not with FRUGAL_F_PEER or the early gather      */
    FRUGAL_F_GPU_DRAIN = 64,    /* the side-stream drain (a11) scatters its rows into the host
                                   table with zero-copy stores from a kernel.  Default (flag
                                   clear): the drain kernel packs the rows into a pinned staging
                                   queue as one contiguous run and the library's background
                                   flushing threads (§3.2) copy them
                                   into the table; the gate of s+1 waits for the threads' progress
                                   word.  Random 128-B zero-copy stores over the whole table stall
                                   the concurrent HBM kernels; the staging run is
                                   sequential.  Threads: FRUGAL_FLUSH_THREADS (env, default
                                   nproc/4 in [2, 8]) */
    FRUGAL_F_OWN_IDS = 128,     /* world > 1: frugal_prefetch/frugal_step get only THIS rank's
                                   ids (int64 [batch*slots]) instead of all ranks' ([world][...]);
                                   every rank publishes its distinct ids, grouped by owner, in a
                                   host id mailbox and each owner merges the ids it owns from
                                   all ranks (its read sets) -- per-rank
                                   ingest bytes and work no longer grow with world.  counts is
                                   still [world] (the global batch size of the loss mean) */
    FRUGAL_F_A2A = 8            /* comparison path (the message pipeline of
                                   PAPER.md Fig. 2b): rows and gradients move between
                                   ranks by the caller's all-to-all (NCCL over NVLink) through
                                   the frugal_a2a_* calls instead of the host table/mailbox;
                                   world > 1 only                                           */
};

enum { FRUGAL_FLUSH_ALL = 0 };

typedef struct {
    int32_t world;      /* n ranks (GPUs), 1..32                                          */
    int32_t rank;       /* this rank, 0..world-1 (== torch.distributed rank)               */
    int32_t device;     /* CUDA ordinal this context runs on                               */
    int32_t dim;        /* d: embedding dimension, multiple of 4, 4..1024                 */
    int64_t n_rows;     /* N: rows over all tables, 1 .. 2^31-1                            */
    int32_t slots;      /* F: lookups per sample                                           */
    int32_t batch;      /* B: max samples per rank per step                               */
    int32_t lookahead;  /* L: sample-queue depth, 2..31 (paper default 10, L783-784)      */
    int32_t age_out;    /* D >= 1: cold dirty rows with no read in sight are flushed D
                           steps after their update (reading R9)                          */
    int32_t opt;        /* frugal_opt                                                      */
    float lr, eps;      /* SGD: w -= lr*g; Adagrad: G += g*g; w -= (lr*g)/(sqrt(G)+eps)    */
    float init_accum;   /* Adagrad G0                                                      */
    float init_scale;   /* w0[k][j] = init_scale*(2u-1), u = top24(splitmix64(seed ^ (k*d+j)))/2^24 */
    uint64_t init_seed;
    const int64_t* hot_ids; /* host array: the static hot (cached) set, global ids, any
                               order; each owner caches its share (reading R10/R11)       */
    int64_t n_hot;
    const char* shm_name;   /* POSIX shm name of the shared host table ("/frugal_x");
                               rank 0 creates + initialises, others attach.  NULL:
                               private pinned table (world must be 1)                     */
    int32_t mode;           /* frugal_mode                                                 */
    int32_t flags;          /* FRUGAL_F_*                                                  */
    const int64_t* host_order; /* optional host array of distinct global ids: the host-table
                               layout.  Row host_order[i] lives in host row slot i; the rows
                               not listed follow in ascending id.  NULL: slot = id.  Every
                               rank of a shared table must pass the same list.  A layout
                               only moves bytes: no result depends on it.  Meant for a
                               frequency order (random host writes and reads
                               over a compact footprint run faster on the host link)      */
    int64_t n_order;
    uint64_t run_nonce;     /* identifies this training run (world > 1 with shm_name: required,
                               != 0, the same on every rank, e.g. drawn by rank 0 and broadcast
                               through the process group).  Rank 0 stamps it into the segment
                               header; other ranks attach only to a segment carrying it, so a
                               stale segment of a crashed run under the same name is never
                               used (they re-open the name until rank 0's new one appears).  */
} frugal_config;

/* Create the context of this rank: validates cfg, maps (and for rank 0 creates and
   initialises) the host table w[N][d] (+ G[N][d] for Adagrad), registers it with
   CUDA (mapped, portable), allocates the HBM cache of the owned hot rows, per-row
   metadata, sample-queue ring, dirty-row pool and scratch.  Ranks > 0 wait (bounded,
   600 s) for rank 0's table stamped with cfg->run_nonce.  On error *out is NULL. */
frugal_status frugal_init(const frugal_config* cfg, frugal_ctx** out);

/* Sample queue (§3.2, §3.3): enqueue the ids of step t of ALL
   ranks (FRUGAL_F_OWN_IDS: of this rank only, int64 [batch*slots]; the ranks exchange
   their distinct ids through the host table's id mailbox).
   ids_all: int64 [world][batch*slots], host (pageable or pinned) or device
   pointer; it is read after the work already on `stream`, asynchronously on a library
   stream: the caller may overwrite it once the next frugal_prefetch/frugal_step call
   has returned (pageable host memory: as soon as this call returns).
   counts: host int32[world], samples of each rank (0..batch).  Only for t = 0..L-1
   before step 0.  The queue holds L+1 future steps: the ingest of step t (id
   conversion, dedup, read bits) runs on a library stream one step ahead, overlapping
   the previous step; priorities still only see the L steps [s, s+L-1] (R1). */
frugal_status frugal_prefetch(frugal_ctx* ctx, int64_t t, const int64_t* ids_all,
                              const int32_t* counts, frugal_stream stream);

/* Begin step s: run the P2F scheduler for the rows updated at s-1 (priority buckets over
   [s, s+L-1], AdjustPriority inf->s+L-1, age-out), flush the urgent bucket on `stream`,
   hand the deferred buckets to the side stream, enqueue step s+L (ids_next_all /
   counts_next as in prefetch; NULL past the end of the stream) and the gate (PQ front
   > s, §3.3) on `stream`.  Returns once enqueued. */
frugal_status frugal_step(frugal_ctx* ctx, int64_t s, const int64_t* ids_next_all,
                          const int32_t* counts_next, frugal_stream stream);

/* Forward query (§3.2): d_out[i] = current value of row ids[rank][i], for
   i < counts[rank]*slots, row-major fp32 [count*slots][dim] in device memory.  Owned
   hot rows come from the HBM cache, all others from the host table by zero-copy
   loads (CPU bypass, §3.1).  d_out == NULL (fused lookup, REC glue only):
   the expand is skipped and the gathered distinct rows stay in the library's step
   buffer; frugal_dot_model(s) must then be called with d_emb == NULL and reads row
   ids[rank][i] through the dedup's inverse index (same values, no [count*slots][dim]
   round trip through HBM).  frugal_transe_model returns FRUGAL_EINVAL after it. */
frugal_status frugal_lookup(frugal_ctx* ctx, int64_t s, float* d_out, frugal_stream stream);

/* Backward update (§3.2, §3.3): d_grad has d_out's shape.
   Segment-reduces the gradients per distinct row (positions ascending), routes
   partials of rows owned by other ranks through the host mailbox (the update
   staging queue), merges per owned row in ascending rank order and applies the
   fused optimizer; marks rows dirty and removes s from their read sets. */
frugal_status frugal_backward_update(frugal_ctx* ctx, int64_t s, const float* d_grad,
                                     frugal_stream stream);

/* N3 dynamic cache (needs FRUGAL_F_DYNAMIC_CACHE; reading R27).  From step t0
   on, the hot (cached) set is hot_ids (host array of global ids, any order; each owner
   keeps its share) instead of the previous one.  The reads of steps >= t0 are classified
   against it as soon as they are ingested, so this must be called before the ingest of t0
   is enqueued (before frugal_step(t0 - L), or frugal_prefetch(t0) for t0 < L) and at most
   one change may be pending.  At the start of frugal_step(t0) the owner flushes every row
   whose hotness changes and whose host copy is not current (the transition set, on the
   critical path, like the urgent bucket), then evicts and admits rows.  Results (tables,
   losses) do not depend on the hot sets.  hot_ids is copied to the device asynchronously
   (duplicates are ignored): a pageable buffer may be reused on return, a pinned one once
   frugal_step(t0) has returned.  Ids are validated on the device: an id >= n_rows, or an
   owned share beyond the slot capacity (1.25x the initial share + 64), fails the next call
   with FRUGAL_EINVAL.  FRUGAL_ESTATE: too late, or a change is already pending. */
frugal_status frugal_set_hot(frugal_ctx* ctx, int64_t t0, const int64_t* hot_ids, int64_t n_hot);

/* End of training (L1082-1083): every dirty owned row (w and G) and the G of every
   hot row to the host table; waits for the side stream.  Afterwards the host table
   is authoritative. */
frugal_status frugal_flush(frugal_ctx* ctx, int32_t what, frugal_stream stream);

frugal_status frugal_destroy(frugal_ctx* ctx);
const char* frugal_last_error(void);

/* ---- model glue (not the library proper) ----------------------
   Frozen-dense dot-interaction BCE for the synthetic REC workload (R15):
   per sample b: S = sum_f e_f (f ascending, fp32), z = 0.5(|S|^2 - sum_f |e_f|^2)
   + <x_b,S> (fp64), p = sigmoid(z); loss += softplus(z) - y z (fp64, into *d_loss);
   grad_f = c*((S - e_f) + x_b), c = (float)((p - y)/nb), nb = samples of step s over
   all ranks.  d_emb/d_grad: [count*slots][dim] (device); x: [count][dim]; y: [count]: both
   device pointers, or both host pointers (pinned or pageable: the library copies them to its
   own device staging on a copy stream as soon as the call is made; a host buffer may be
   reused once `stream` has passed this call).
   d_emb == NULL exactly when lookup(s) ran with d_out == NULL (fused lookup), else
   FRUGAL_EINVAL. */
frugal_status frugal_dot_model(frugal_ctx* ctx, int64_t s, const float* d_emb, const float* d_x,
                               const float* d_y, float* d_grad, double* d_loss,
                               frugal_stream stream);

/* KG glue (R26): TransE-L2, samples = triples with slots (h, r, t, neg), the
   negatives of each chunk of `chunk` consecutive samples of this rank shared by the chunk:
   score = gamma - |h + r - x|_2, loss_b = softplus(-score(h,r,t)) + mean_j softplus(
   score(h,r,n_j)); *d_loss += sum_b loss_b / nb.  fp64 internally, d_grad fp32 [count*4][dim].
   Requires slots == 4. */
frugal_status frugal_transe_model(frugal_ctx* ctx, int64_t s, const float* d_emb, int32_t chunk, float gamma,
                                  float* d_grad, double* d_loss, frugal_stream stream);

/* ---- comparison path (FRUGAL_F_A2A) -------------------------------------------------
   Per step: frugal_step(s) -> frugal_a2a_requests(s) -> [caller: all-to-all of the ids] ->
   frugal_a2a_serve(s) -> [all-to-all of the rows back] -> frugal_a2a_lookup(s) -> glue ->
   frugal_a2a_pack(s) -> [all-to-all of the partials] -> frugal_a2a_update(s).  Segment r of
   every buffer is the part to/from rank r, ids ascending within a segment.
   requests: d_ids [n_uniq] (device, int32 global ids, grouped by owner), counts[world] (host)
             = ids this rank asks each owner for.
   serve:    d_ids_in [n_in]: ids other ranks asked this owner for (segments by requester);
             d_rows [n_in][dim]: their current values (cache, pool or host).
   lookup:   d_rows_in [n_uniq][dim] in the order of requests (NULL if none); d_out as
             frugal_lookup.
   pack:     d_partials [n_uniq][dim]: per distinct row, the segment-reduced gradient, in the
             order of requests.
   update:   d_partials_in: the partials other ranks sent this owner, segments by sender;
             recv_counts[world] (host; d_partials_in may be NULL if they sum to 0).  Merge in
             rank order + optimizer, as backward_update. */
frugal_status frugal_a2a_requests(frugal_ctx* ctx, int64_t s, int32_t* d_ids, int64_t* counts, frugal_stream stream);
frugal_status frugal_a2a_serve(frugal_ctx* ctx, int64_t s, const int32_t* d_ids_in, int64_t n_in, float* d_rows,
                               frugal_stream stream);
frugal_status frugal_a2a_lookup(frugal_ctx* ctx, int64_t s, const float* d_rows_in, float* d_out,
                                frugal_stream stream);
frugal_status frugal_a2a_pack(frugal_ctx* ctx, int64_t s, const float* d_grad, float* d_partials,
                              frugal_stream stream);
frugal_status frugal_a2a_update(frugal_ctx* ctx, int64_t s, const float* d_partials_in, const int64_t* recv_counts,
                                frugal_stream stream);

/* ---- introspection (tests / bench only; synchronise and copy to caller-owned host
   buffers) ---------------------------------------------------------------------- */
/* dedup of this rank's ids at step t (t within the sample queue): uniq ascending
   (int64), inv[i] = index of ids[i] in uniq. *n_uniq receives the count; uniq/inv may
   be NULL to query sizes. */
frugal_status frugal_get_dedup(frugal_ctx* ctx, int64_t t, int64_t* uniq, int32_t* inv,
                               int64_t* n_uniq);

/* schedule artefacts of the last frugal_step (needs FRUGAL_F_RECORD): rows (global ids)
   flushed urgently, deferred rows and their deadlines, aged-out rows; gate_wait = 1 iff
   the urgent bucket was non-empty. Arrays may be NULL to query sizes (cap ignored). */
typedef struct {
    int64_t n_urgent, n_deferred, n_ageout;
    int32_t gate_wait;
} frugal_schedule_info;
frugal_status frugal_get_schedule(frugal_ctx* ctx, frugal_schedule_info* info, int64_t* urgent,
                                  int64_t* deferred, int32_t* deferred_p, int64_t* ageout);

/* rows flushed by the cache transition of the last frugal_step (global ids, any order;
   empty unless that step was an epoch boundary; needs FRUGAL_F_RECORD) */
frugal_status frugal_get_transition(frugal_ctx* ctx, int64_t* rows, int64_t* n);

/* rows flushed by the last frugal_flush(FRUGAL_FLUSH_ALL) (global ids, any order) */
frugal_status frugal_get_final_flush(frugal_ctx* ctx, int64_t* rows, int64_t* n);

/* authoritative current values of rows owned by this rank (cache, dirty pool or
   host).  ids: host int64[n]; w, G: host float[n][dim] (G may be NULL). */
frugal_status frugal_read_rows(frugal_ctx* ctx, const int64_t* ids, int64_t n, float* w, float* G);

/* raw host-table contents (any row). */
frugal_status frugal_read_host(frugal_ctx* ctx, const int64_t* ids, int64_t n, float* w, float* G);

/* per-phase device time (ms) summed over the steps since the last call (needs
   FRUGAL_F_TIMERS; CUDA events on the phase's stream).  Phases, in order: ingest (a1+a2),
   schedule (a9), urgent (a10), gate (a3), gather (a4, unique rows), expand (a4, per
   position), model (a5), segred (a6), exchange (a7), optimizer (a8), side (a11, side
   stream), prefetch (a4, the early part of the next step's gather, prefetch stream).
   Device counters are cumulative since init (always on; one atomic per block). */
#define FRUGAL_N_PHASES 12
enum {
    FRUGAL_C_POSITIONS = 0,     /* lookups (positions) of this rank                         */
    FRUGAL_C_UNIQUE = 1,        /* distinct rows of this rank (sum over steps)               */
    FRUGAL_C_GATHER_HOST = 2,   /* unique rows gathered from the host table (zero-copy)      */
    FRUGAL_C_GATHER_CACHE = 3,  /* unique rows gathered from the HBM cache                   */
    FRUGAL_C_OPT_HOT = 4,       /* owned rows updated in the cache                           */
    FRUGAL_C_OPT_COLD = 5,      /* owned rows updated via host (w,G) -> dirty pool           */
    FRUGAL_C_URGENT_HOT = 6,    /* rows flushed on the critical path (hot: w)                */
    FRUGAL_C_URGENT_COLD = 7,   /* (cold: w and G)                                           */
    FRUGAL_C_SIDE_HOT = 8,      /* rows flushed by the side stream (deferred + age-out)      */
    FRUGAL_C_SIDE_COLD = 9,
    FRUGAL_C_FINAL_HOT = 10,    /* rows flushed by frugal_flush                              */
    FRUGAL_C_FINAL_COLD = 11,
    FRUGAL_C_LONG_SEGMENTS = 12,/* unique rows with > 64 occurrences (chunked reduction)     */
    FRUGAL_C_MAIL_OUT = 13,     /* partial rows written to this rank's host mailbox          */
    FRUGAL_C_MAIL_IN = 14,      /* partial rows read from other ranks' mailboxes             */
    FRUGAL_C_GATHER_POOL = 15,  /* unique owned cold rows gathered from the dirty pool (HBM)  */
    FRUGAL_C_GATHER_PEER = 16,  /* unique non-owned rows loaded from the owner's HBM (PEER)  */
    FRUGAL_C_TRANSITION_HOT = 17,  /* rows flushed by cache transitions (N3), from the cache */
    FRUGAL_C_TRANSITION_COLD = 18, /* ... from the dirty pool                               */
    FRUGAL_N_COUNTERS = 20
};
typedef struct {
    double ms[FRUGAL_N_PHASES];
    int64_t steps;                 /* backward_update calls since the last get_stats       */
    int64_t kernel_launches;       /* library kernels launched since init                  */
    int64_t count[FRUGAL_N_COUNTERS];
    int64_t flush_jobs;            /* drain jobs applied by the flushing threads (since the last call) */
    double flush_ms;               /* time thread 0 spent copying its share of the rows, summed      */
    double flush_wait_ms;          /* time thread 0 waited for the device's part flags, summed       */
    int64_t timer_steps;           /* steps whose phases `ms` covers (FRUGAL_F_TIMERS; with the
                                      environment knob FRUGAL_TIMER_EVERY=k only steps s % k == 0
                                      are timed, so per-step phase time = ms / timer_steps)        */
    double host_wait_ms;           /* host time the calls spent blocked on the device (the ingest's
                                      staging-buffer reuse waits): the caller's enqueue cost per
                                      step is its call time minus this                           */
} frugal_stats;
frugal_status frugal_get_stats(frugal_ctx* ctx, frugal_stats* out);

/* timeline of the last `cap` recorded phase instances (FRUGAL_F_TIMERS): phase index,
   start and end (ms) relative to the first returned one, across all library streams.
   Arrays may be NULL to query *n.  Call before frugal_get_stats (which consumes them). */
frugal_status frugal_get_timeline(frugal_ctx* ctx, int32_t* phase, double* t0, double* t1, int64_t cap,
                                  int64_t* n);

/* host-link calibration (bench only): time (*ms) to read n pseudo-random rows of the host
   table with the gather's access pattern and grid (read-only; between steps) -- the
   random-row ceiling of this machine's host link, next to the sequential pinned-copy peak */
frugal_status frugal_probe_host_reads(frugal_ctx* ctx, int64_t n, uint64_t seed, double* ms);

/* make `stream` wait for every piece of work the library has enqueued on its own streams so
   far (the ingest of the sample queue, the side-stream drain, the early gather): a timing
   event recorded on `stream` after this call covers all of the steps' device work.  The
   bench joins before its closing event; training loops never need it (the library orders
   its streams itself). */
frugal_status frugal_join(frugal_ctx* ctx, frugal_stream stream);

/* fp64 calibration (bench only, no context): *ops_per_s = separately rounded fp64 add/mul
   instructions per second of a full-device kernel of independent DADD/DMUL chains (the
   peak of the KG glue, whose every op is such an instruction, reading R26) */
frugal_status frugal_probe_fp64(int32_t device, double* ops_per_s);

/* number of owned rows / hot slots of this rank */
int64_t frugal_owned_rows(frugal_ctx* ctx);
int64_t frugal_hot_slots(frugal_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* FRUGAL_H */
