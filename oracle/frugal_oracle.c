/*
 * frugal_oracle.c -- CPU ORACLE for the Frugal training step.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (libfrugal.so + the Python binding) never links, imports or calls it, and this
 * file shares no code, header, table or constant generator with the CUDA path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md):
 *
 *  VALUES -- plain single-process synchronous training (§3,
 *  footnote L269-270: Frugal is exactly equivalent to synchronous training, proof
 *  §3.3) of the embedding-only synthetic workload (§4.1)
 *  with a frozen-dense dot-interaction BCE glue (reading R15):
 *     e_f = W[id_f];  S = sum_f e_f;  z = sum_{f<f'} <e_f,e_f'> + sum_f <x,e_f>
 *     p = sigmoid(z); loss = BCE(p, y); dL/de_f = c (S - e_f + x), c = (p-y)/nb
 *  then per rank: partial P_g[k] = sum over positions i ascending of grad[i]
 *  (fp32, fixed order: sequential within chunks of 64 occurrences, chunk sums
 *  added sequentially -- reading R23), per row: g_k = sum over ranks ascending of P_g[k], then
 *  SGD  w -= lr*g   or   Adagrad  G += g*g; w -= (lr*g)/(sqrt(G)+eps)
 *  (elementwise fp32, each operation rounded separately; built with
 *  -ffp-contract=off, no fast-math).
 *
 *  SCHEDULE -- the P2F artefacts by brute-force definition:
 *   * priority = Eq. (1): min R set if W set != {} else INF;
 *   * next(k,u) = min{ t in [u+1, min(u+L, S-1)] : k read at t by any rank }
 *     else INF (sample queue of L steps, L781-784, L1042-1049; reading R1);
 *   * the gate of step s passes iff no dirty host-read row has priority <= s
 *     (L913-916, L1034: "strictly greater than s");
 *   * a host-reader of k at t is any reader except the owner (k mod n) reading
 *     its own hot (cached) row (reading R7);
 *   * bucketing at step s of the rows updated at s-1: p = next(k,s-1); p == s
 *     -> urgent U(s) (flushed on the critical path); p in [s+1,s+L-1] -> deferred
 *     D(s); owner-only hot read -> EXEMPT (stays dirty); no read -> INF;
 *   * AdjustPriority INF -> t for dirty INF rows read at t = s+L-1 (Fig. 6 step 4,
 *     L1074-1077) -> D(s) (or EXEMPT);
 *   * age-out A(s): cold INF rows whose last update <= s-1-D (reading R9);
 *   * final flush: every still-dirty row (L1082-1083); hot rows also push G.
 *   * dynamic cache (reading R27): the hot set H_t is a
 *     step function (epochs starting at t0); every "hot" above means "hot at the step in
 *     question".  At an epoch boundary t0, before anything else of step t0, every row
 *     whose hotness changes and that is dirty is flushed (w and G) -- the transition set
 *     X(t0) -- and an evicted row's G is pushed to the host (G follows w out of the cache).
 *  A simulated host table Hw/HG is written only by flushes; invariant (2)
 *  (L1104-1108) is checked on every host read: no host-read of a dirty row and
 *  Hw == W bit-for-bit.
 */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define OR_INF INT32_MAX
#define OR_CHUNK 64 /* R23: segment-reduce chunk length */
enum { OR_SGD = 0, OR_ADAGRAD = 1 };
enum { OR_MODEL_DOT = 0, OR_MODEL_CONST = 1, OR_MODEL_L2 = 2, OR_MODEL_TRANSE = 3 };
enum { OR_CLEAN = 0, OR_UPDATED = 1, OR_INFP = 2, OR_EXEMPT = 3 };
enum { OR_L_URGENT = 0, OR_L_DEFERRED = 1, OR_L_DEFERRED_P = 2, OR_L_AGEOUT = 3,
       OR_L_FINAL = 4, OR_L_UPDATED = 5, OR_L_INF = 6, OR_L_EXEMPT = 7, OR_L_TRANSITION = 8 };
#define OR_NLISTS 9
#define OR_MAX_EPOCHS 4096

typedef struct {
    int32_t world, dim, slots, batch, lookahead, age_out, opt, model;
    int64_t n_rows;
    float lr, eps, init_accum, init_scale;
    uint64_t init_seed;
    int32_t write_through;    /* 1: every update flushed at the next step (Frugal-Sync, L1399-1402) */
    int32_t skip_urgent_step; /* negative test: urgent (and transition) flushes of this step are lost (-1: never) */
    float gamma;              /* TransE margin */
    int32_t neg_chunk;        /* TransE: triples per negative-sharing chunk */
} oracle_config;

typedef struct { int64_t key; int32_t state, last_update; } rowmeta;
typedef struct { int64_t v; int64_t p; } pair64;

typedef struct {
    oracle_config c;
    /* hot sets by epoch: epoch e is in force for steps [ep_t0[e], ep_t0[e+1]) (N3) */
    int64_t n_ep; int64_t ep_t0[OR_MAX_EPOCHS]; int64_t* ep_hot[OR_MAX_EPOCHS]; int64_t ep_n[OR_MAX_EPOCHS];
    /* lazily materialised rows: open-addressing map key -> index */
    int64_t* hkeys; int64_t* hidx; int64_t hcap;
    int64_t n, cap; rowmeta* meta; float *W, *G, *Hw, *HG;
    /* stream (borrowed) */
    int64_t S; const int64_t* ids; const int32_t* counts; const float* x; const float* y;
    int64_t** uq; int64_t* uq_n; /* per (s,g) sorted distinct ids, lazily built */
    int64_t cur;                  /* next step to run */
    int64_t* upd; int64_t n_upd;  /* rows updated at cur-1 (sorted) */
    /* artefacts of the last step() */
    int64_t* lists[OR_NLISTS]; int64_t nl[OR_NLISTS], capl[OR_NLISTS];
    int gate_wait;
    double* loss;
    float* grad; /* last step grads [world][batch*slots][dim] */
    int64_t** pk; float** pv; int64_t* pn; /* last step partials per rank */
    int64_t violations;
} oracle;

/* ---------------------------------------------------------------- init (R18) */
static uint64_t splitmix64(uint64_t z) {
    z += 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
static float init_w(const oracle* o, int64_t k, int j) {
    uint64_t h = splitmix64(o->c.init_seed ^ (uint64_t)(k * (int64_t)o->c.dim + j));
    float u = (float)(h >> 40) / 16777216.0f;
    return o->c.init_scale * (2.0f * u - 1.0f);
}

/* ---------------------------------------------------------------- helpers */
static int cmp_i64(const void* a, const void* b) {
    int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    return (x > y) - (x < y);
}
static int cmp_pair(const void* a, const void* b) {
    const pair64 *x = a, *y = b;
    if (x->v != y->v) return (x->v > y->v) - (x->v < y->v);
    return (x->p > y->p) - (x->p < y->p);
}
static void push(oracle* o, int which, int64_t v) {
    if (o->nl[which] == o->capl[which]) {
        o->capl[which] = o->capl[which] ? 2 * o->capl[which] : 1024;
        o->lists[which] = realloc(o->lists[which], o->capl[which] * sizeof(int64_t));
    }
    o->lists[which][o->nl[which]++] = v;
}
/* k is hot (cached by its owner) at step t: the hot set of t's epoch */
static int is_hot(const oracle* o, int64_t k, int64_t t) {
    int64_t e = o->n_ep - 1;
    while (e > 0 && o->ep_t0[e] > t) e--;
    return o->ep_n[e] && bsearch(&k, o->ep_hot[e], o->ep_n[e], sizeof(int64_t), cmp_i64) != NULL;
}
static int epoch_starts_at(const oracle* o, int64_t t) {
    for (int64_t e = 1; e < o->n_ep; e++) if (o->ep_t0[e] == t) return 1;
    return 0;
}
static int owner(const oracle* o, int64_t k) { return (int)(k % o->c.world); }

static void grow_rows(oracle* o) {
    int64_t nc = o->cap ? 2 * o->cap : 4096, d = o->c.dim;
    o->meta = realloc(o->meta, nc * sizeof(rowmeta));
    o->W = realloc(o->W, nc * d * sizeof(float));
    o->G = realloc(o->G, nc * d * sizeof(float));
    o->Hw = realloc(o->Hw, nc * d * sizeof(float));
    o->HG = realloc(o->HG, nc * d * sizeof(float));
    o->cap = nc;
}
static void rehash(oracle* o) {
    int64_t nc = o->hcap ? 2 * o->hcap : 8192;
    int64_t* nk = malloc(nc * sizeof(int64_t));
    int64_t* ni = malloc(nc * sizeof(int64_t));
    for (int64_t i = 0; i < nc; i++) nk[i] = -1;
    for (int64_t i = 0; i < o->hcap; i++) {
        if (o->hkeys[i] < 0) continue;
        uint64_t h = splitmix64((uint64_t)o->hkeys[i]) & (uint64_t)(nc - 1);
        while (nk[h] >= 0) h = (h + 1) & (uint64_t)(nc - 1);
        nk[h] = o->hkeys[i]; ni[h] = o->hidx[i];
    }
    free(o->hkeys); free(o->hidx);
    o->hkeys = nk; o->hidx = ni; o->hcap = nc;
}
/* index of row k; materialise W0 = init(seed,k,j), G0 = init_accum, host = same */
static int64_t row(oracle* o, int64_t k) {
    if (2 * (o->n + 1) > o->hcap) rehash(o);
    uint64_t h = splitmix64((uint64_t)k) & (uint64_t)(o->hcap - 1);
    while (o->hkeys[h] >= 0) {
        if (o->hkeys[h] == k) return o->hidx[h];
        h = (h + 1) & (uint64_t)(o->hcap - 1);
    }
    if (o->n == o->cap) grow_rows(o);
    int64_t i = o->n++, d = o->c.dim;
    o->hkeys[h] = k; o->hidx[h] = i;
    o->meta[i].key = k; o->meta[i].state = OR_CLEAN; o->meta[i].last_update = -1;
    for (int j = 0; j < d; j++) {
        o->W[i * d + j] = init_w(o, k, j);
        o->G[i * d + j] = o->c.init_accum;
        o->Hw[i * d + j] = o->W[i * d + j];
        o->HG[i * d + j] = o->G[i * d + j];
    }
    return i;
}
static int64_t find_row(const oracle* o, int64_t k) {
    if (!o->hcap) return -1;
    uint64_t h = splitmix64((uint64_t)k) & (uint64_t)(o->hcap - 1);
    while (o->hkeys[h] >= 0) {
        if (o->hkeys[h] == k) return o->hidx[h];
        h = (h + 1) & (uint64_t)(o->hcap - 1);
    }
    return -1;
}

static const int64_t* step_ids(const oracle* o, int64_t s, int g) {
    return o->ids + (s * o->c.world + g) * (int64_t)o->c.batch * o->c.slots;
}
static int64_t step_len(const oracle* o, int64_t s, int g) {
    return (int64_t)o->counts[s * o->c.world + g] * o->c.slots;
}
/* distinct ids read by rank g at step s, ascending (dedup definition, reading R21) */
static const int64_t* uniq(oracle* o, int64_t s, int g, int64_t* n) {
    int64_t idx = s * o->c.world + g;
    if (!o->uq[idx]) {
        int64_t m = step_len(o, s, g);
        int64_t* a = malloc((m ? m : 1) * sizeof(int64_t));
        memcpy(a, step_ids(o, s, g), m * sizeof(int64_t));
        qsort(a, m, sizeof(int64_t), cmp_i64);
        int64_t u = 0;
        for (int64_t i = 0; i < m; i++)
            if (i == 0 || a[i] != a[i - 1]) a[u++] = a[i];
        o->uq[idx] = a; o->uq_n[idx] = u;
    }
    *n = o->uq_n[idx];
    return o->uq[idx];
}
static int read_by(oracle* o, int64_t k, int64_t t, int g) {
    int64_t n; const int64_t* u = uniq(o, t, g, &n);
    return n && bsearch(&k, u, n, sizeof(int64_t), cmp_i64) != NULL;
}
static int any_read(oracle* o, int64_t k, int64_t t) {
    for (int g = 0; g < o->c.world; g++) if (read_by(o, k, t, g)) return 1;
    return 0;
}
/* a host-reader at t: any reader except the owner reading its own hot row (R7) */
static int host_reader(const oracle* o, int64_t k, int g, int64_t t) {
    return !(g == owner(o, k) && is_hot(o, k, t));
}
static int needs_host(oracle* o, int64_t k, int64_t t) {
    for (int g = 0; g < o->c.world; g++)
        if (read_by(o, k, t, g) && host_reader(o, k, g, t)) return 1;
    return 0;
}
static int32_t next_access(oracle* o, int64_t k, int64_t u) {
    int64_t hi = u + o->c.lookahead;
    if (hi > o->S - 1) hi = o->S - 1;
    for (int64_t t = u + 1; t <= hi; t++) if (any_read(o, k, t)) return (int32_t)t;
    return OR_INF;
}
/* a flush copies the current values to the host table (hot rows: w only, R8) */
static void flush_row(oracle* o, int64_t i, int with_g) {
    int64_t d = o->c.dim;
    memcpy(o->Hw + i * d, o->W + i * d, d * sizeof(float));
    if (with_g) memcpy(o->HG + i * d, o->G + i * d, d * sizeof(float));
    o->meta[i].state = OR_CLEAN;
}
static int host_fresh_w(const oracle* o, int64_t i) {
    int64_t d = o->c.dim;
    return memcmp(o->Hw + i * d, o->W + i * d, d * sizeof(float)) == 0;
}
static int host_fresh_g(const oracle* o, int64_t i) {
    int64_t d = o->c.dim;
    return memcmp(o->HG + i * d, o->G + i * d, d * sizeof(float)) == 0;
}

/* ---------------------------------------------------------------- API */
void* oracle_new(const oracle_config* c, const int64_t* hot, int64_t n_hot) {
    oracle* o = calloc(1, sizeof(oracle));
    o->c = *c;
    o->n_ep = 1;
    o->ep_t0[0] = 0;
    o->ep_n[0] = n_hot;
    o->ep_hot[0] = malloc((n_hot ? n_hot : 1) * sizeof(int64_t));
    memcpy(o->ep_hot[0], hot, n_hot * sizeof(int64_t));
    qsort(o->ep_hot[0], n_hot, sizeof(int64_t), cmp_i64);
    rehash(o);
    return o;
}

void oracle_free(void* p) {
    oracle* o = p;
    if (!o) return;
    for (int64_t i = 0; i < o->S * o->c.world; i++) free(o->uq[i]);
    for (int i = 0; i < OR_NLISTS; i++) free(o->lists[i]);
    for (int64_t e = 0; e < o->n_ep; e++) free(o->ep_hot[e]);
    for (int g = 0; g < o->c.world && o->pk; g++) { free(o->pk[g]); free(o->pv[g]); }
    free(o->pk); free(o->pv); free(o->pn);
    free(o->uq); free(o->uq_n); free(o->upd); free(o->loss); free(o->grad);
    free(o->hkeys); free(o->hidx);
    free(o->meta); free(o->W); free(o->G); free(o->Hw); free(o->HG);
    free(o);
}

/* N3: from step t0 on the hot set is hot[0..n) (t0 after every earlier epoch start) */
int oracle_set_hot(void* p, int64_t t0, const int64_t* hot, int64_t n) {
    oracle* o = p;
    if (o->n_ep >= OR_MAX_EPOCHS || t0 <= o->ep_t0[o->n_ep - 1]) return -1;
    int64_t e = o->n_ep++;
    o->ep_t0[e] = t0;
    o->ep_n[e] = n;
    o->ep_hot[e] = malloc((n ? n : 1) * sizeof(int64_t));
    memcpy(o->ep_hot[e], hot, n * sizeof(int64_t));
    qsort(o->ep_hot[e], n, sizeof(int64_t), cmp_i64);
    return 0;
}

/* the whole stream is given up front: the lookahead reads future steps */
int oracle_set_stream(void* p, int64_t S, const int64_t* ids, const int32_t* counts,
                      const float* x, const float* y) {
    oracle* o = p;
    o->S = S; o->ids = ids; o->counts = counts; o->x = x; o->y = y;
    o->uq = calloc(S * o->c.world, sizeof(int64_t*));
    o->uq_n = calloc(S * o->c.world, sizeof(int64_t));
    o->loss = calloc(S ? S : 1, sizeof(double));
    o->grad = calloc((size_t)o->c.world * o->c.batch * o->c.slots * o->c.dim + 1, sizeof(float));
    o->pk = calloc(o->c.world, sizeof(int64_t*));
    o->pv = calloc(o->c.world, sizeof(float*));
    o->pn = calloc(o->c.world, sizeof(int64_t));
    o->cur = 0;
    return 0;
}

/* ---- schedule part of step s: (b) bucketing of Upd(s-1), (c) AdjustPriority, (d) age-out, (e) gate */
static void schedule(oracle* o, int64_t s) {
    const int L = o->c.lookahead;
    for (int i = 0; i < OR_NLISTS; i++) o->nl[i] = 0;
    /* (N3) epoch boundary: rows changing hotness are made clean first (reading R27) */
    if (s >= 1 && epoch_starts_at(o, s)) {
        for (int64_t i = 0; i < o->n; i++) {
            int64_t k = o->meta[i].key;
            int was = is_hot(o, k, s - 1), now = is_hot(o, k, s);
            if (was == now) continue;
            if (o->meta[i].state != OR_CLEAN) {
                push(o, OR_L_TRANSITION, k);
                if (s == o->c.skip_urgent_step) o->meta[i].state = OR_CLEAN; /* negative test: lost */
                else flush_row(o, i, 1);
            }
            if (was) memcpy(o->HG + i * o->c.dim, o->G + i * o->c.dim, o->c.dim * sizeof(float));
        }
        qsort(o->lists[OR_L_TRANSITION], o->nl[OR_L_TRANSITION], sizeof(int64_t), cmp_i64);
    }
    /* (b) rows updated at s-1: priority = next access (Eq. 1) */
    for (int64_t a = 0; a < o->n_upd; a++) {
        int64_t k = o->upd[a], i = find_row(o, k);
        if (o->meta[i].state == OR_CLEAN) continue; /* flushed by the transition above */
        int cold = !is_hot(o, k, s);
        if (o->c.write_through) { push(o, OR_L_URGENT, k); flush_row(o, i, cold); continue; }
        int32_t pr = next_access(o, k, s - 1);
        if (pr == OR_INF) { o->meta[i].state = OR_INFP; continue; }
        if (!needs_host(o, k, pr)) { o->meta[i].state = OR_EXEMPT; continue; }
        if (pr == s) {
            push(o, OR_L_URGENT, k);
            if (s == o->c.skip_urgent_step) { o->meta[i].state = OR_CLEAN; continue; } /* lost flush */
        } else {
            push(o, OR_L_DEFERRED, k); push(o, OR_L_DEFERRED_P, pr);
        }
        flush_row(o, i, cold);
    }
    /* (c) AdjustPriority INF -> t for dirty rows read at the newly prefetched step t */
    int64_t t = s + L - 1;
    if (t < o->S && t >= 1) {
        for (int g = 0; g < o->c.world; g++) {
            int64_t n; const int64_t* u = uniq(o, t, g, &n);
            for (int64_t q = 0; q < n; q++) {
                int64_t k = u[q], i = find_row(o, k);
                if (i < 0 || o->meta[i].state != OR_INFP) continue;
                if (needs_host(o, k, t)) {
                    push(o, OR_L_DEFERRED, k); push(o, OR_L_DEFERRED_P, t);
                    flush_row(o, i, !is_hot(o, k, s));
                } else {
                    o->meta[i].state = OR_EXEMPT;
                }
            }
        }
    }
    /* (d) age-out of cold rows still dirty with INF priority */
    for (int64_t i = 0; i < o->n; i++) {
        rowmeta* m = &o->meta[i];
        if (m->state == OR_INFP && !is_hot(o, m->key, s) && m->last_update <= s - 1 - o->c.age_out) {
            push(o, OR_L_AGEOUT, m->key);
            flush_row(o, i, 1);
        }
    }
    /* remaining dirty rows, for introspection */
    for (int64_t i = 0; i < o->n; i++) {
        if (o->meta[i].state == OR_INFP) push(o, OR_L_INF, o->meta[i].key);
        if (o->meta[i].state == OR_EXEMPT) push(o, OR_L_EXEMPT, o->meta[i].key);
    }
    qsort(o->lists[OR_L_URGENT], o->nl[OR_L_URGENT], sizeof(int64_t), cmp_i64);
    qsort(o->lists[OR_L_AGEOUT], o->nl[OR_L_AGEOUT], sizeof(int64_t), cmp_i64);
    qsort(o->lists[OR_L_INF], o->nl[OR_L_INF], sizeof(int64_t), cmp_i64);
    qsort(o->lists[OR_L_EXEMPT], o->nl[OR_L_EXEMPT], sizeof(int64_t), cmp_i64);
    /* deferred: sort (p, k) pairs */
    int64_t nd = o->nl[OR_L_DEFERRED];
    pair64* pr = malloc((nd ? nd : 1) * sizeof(pair64));
    for (int64_t a = 0; a < nd; a++) { pr[a].v = o->lists[OR_L_DEFERRED_P][a]; pr[a].p = o->lists[OR_L_DEFERRED][a]; }
    qsort(pr, nd, sizeof(pair64), cmp_pair);
    for (int64_t a = 0; a < nd; a++) { o->lists[OR_L_DEFERRED_P][a] = pr[a].v; o->lists[OR_L_DEFERRED][a] = pr[a].p; }
    free(pr);
    /* (e) gate: waits iff some dirty host-read row has priority s (the urgent set) */
    o->gate_wait = o->nl[OR_L_URGENT] > 0;
    /* invariant (2): every host read at s sees a clean, bit-identical host row */
    for (int g = 0; g < o->c.world; g++) {
        int64_t n; const int64_t* u = uniq(o, s, g, &n);
        for (int64_t q = 0; q < n; q++) {
            int64_t k = u[q];
            if (!host_reader(o, k, g, s)) continue;
            int64_t i = row(o, k);
            if (o->meta[i].state != OR_CLEAN || !host_fresh_w(o, i)) o->violations++;
        }
    }
}

/* ---- TransE glue (reading R26; §4.1, DGL-KE TransE_l2): slots of a
   sample are (h, r, t, neg); the negatives of a chunk of neg_chunk consecutive triples of
   a rank are shared by the chunk (tail corruption).  score = gamma - |h + r - x|_2;
   loss_b = softplus(-score(h,r,t)) + (1/nC) sum_j softplus(score(h,r,n_j)).
   Everything in fp64, sums in the written order; gradients rounded to fp32 once. */
static double sigm(double x) { return 1.0 / (1.0 + exp(-x)); }
static double softplus(double x) { return x > 0 ? x + log1p(exp(-x)) : log1p(exp(x)); }
static double transe(oracle* o, int64_t s, int64_t nb) {
    const int n = o->c.world, F = o->c.slots, B = o->c.batch, C = o->c.neg_chunk;
    const int64_t d = o->c.dim;
    const double gamma = o->c.gamma;
    double loss = 0.0;
    double* P = malloc(d * sizeof(double));
    double* v = malloc(d * sizeof(double));
    double* u = malloc(d * sizeof(double));
    double* gh = malloc(d * sizeof(double));
    double* gn = malloc((size_t)C * d * sizeof(double));
    for (int g = 0; g < n; g++) {
        const int64_t* id = step_ids(o, s, g);
        const int32_t cnt = o->counts[s * n + g];
        float* grad = o->grad + (int64_t)g * B * F * d;
        for (int b0 = 0; b0 < cnt; b0 += C) {
            const int b1 = b0 + C < cnt ? b0 + C : cnt, nC = b1 - b0;
            for (int64_t q = 0; q < (int64_t)nC * d; q++) gn[q] = 0.0;
            for (int b = b0; b < b1; b++) {
                int64_t ih = row(o, id[b * F + 0]), ir = row(o, id[b * F + 1]), it = row(o, id[b * F + 2]);
                const float *h = o->W + ih * d, *r = o->W + ir * d, *t = o->W + it * d;
                double dp = 0.0;
                for (int64_t k = 0; k < d; k++) {
                    P[k] = (double)h[k] + (double)r[k];
                    v[k] = P[k] - (double)t[k];
                    dp = dp + v[k] * v[k];
                }
                dp = sqrt(dp);
                const double sp = gamma - dp;
                loss += softplus(-sp);
                const double a = dp > 0.0 ? (1.0 - sigm(sp)) / dp : 0.0;
                for (int64_t k = 0; k < d; k++) gh[k] = a * v[k];
                for (int j = b0; j < b1; j++) {
                    const float* nj = o->W + row(o, id[j * F + 3]) * d;
                    double dj = 0.0;
                    for (int64_t k = 0; k < d; k++) {
                        u[k] = P[k] - (double)nj[k];
                        dj = dj + u[k] * u[k];
                    }
                    dj = sqrt(dj);
                    const double sj = gamma - dj;
                    loss += softplus(sj) / (double)nC;
                    const double w = dj > 0.0 ? sigm(sj) / dj / (double)nC : 0.0;
                    double* gj = gn + (int64_t)(j - b0) * d;
                    for (int64_t k = 0; k < d; k++) {
                        gh[k] = gh[k] - w * u[k];
                        gj[k] = gj[k] + w * u[k];
                    }
                }
                for (int64_t k = 0; k < d; k++) {
                    grad[(b * F + 0) * d + k] = (float)(gh[k] / (double)nb);
                    grad[(b * F + 1) * d + k] = (float)(gh[k] / (double)nb);
                    grad[(b * F + 2) * d + k] = (float)(-(a * v[k]) / (double)nb);
                }
            }
            for (int j = b0; j < b1; j++)
                for (int64_t k = 0; k < d; k++)
                    grad[(j * F + 3) * d + k] = (float)(gn[(int64_t)(j - b0) * d + k] / (double)nb);
        }
    }
    free(P); free(v); free(u); free(gh); free(gn);
    return loss;
}

/* ---- value part of step s: synchronous training (f)-(j) */
static void train(oracle* o, int64_t s) {
    const int n = o->c.world, F = o->c.slots, B = o->c.batch;
    const int64_t d = o->c.dim;
    int64_t nb = 0;
    for (int g = 0; g < n; g++) nb += o->counts[s * n + g];
    double loss = 0.0;
    /* materialise every row this step reads first: row() may grow (realloc) W, and the glue
       below holds pointers into W across several row() calls (TransE: h, r, t while looking
       up the negatives) */
    for (int g = 0; g < n; g++) {
        const int64_t* id = step_ids(o, s, g);
        for (int64_t i = 0; i < step_len(o, s, g); i++) row(o, id[i]);
    }
    float* S = malloc(d * sizeof(float));
    /* (f) forward + glue backward, all reads before any update */
    for (int g = 0; g < n; g++) {
        const int64_t* id = step_ids(o, s, g);
        int32_t cnt = o->counts[s * n + g];
        for (int b = 0; b < cnt; b++) {
            const float* xb = o->x + ((s * n + g) * (int64_t)B + b) * d;
            float yb = o->y[(s * n + g) * (int64_t)B + b];
            float* gr = o->grad + ((int64_t)g * B * F + (int64_t)b * F) * d;
            if (o->c.model == OR_MODEL_DOT) {
                for (int64_t j = 0; j < d; j++) S[j] = 0.0f;
                for (int f = 0; f < F; f++) {
                    int64_t ri = row(o, id[b * F + f]); const float* e = o->W + ri * d;
                    for (int64_t j = 0; j < d; j++) S[j] = S[j] + e[j];
                }
                double sq = 0.0, ee = 0.0, xs = 0.0;
                for (int64_t j = 0; j < d; j++) { sq += (double)S[j] * S[j]; xs += (double)xb[j] * S[j]; }
                for (int f = 0; f < F; f++) {
                    int64_t ri = row(o, id[b * F + f]); const float* e = o->W + ri * d;
                    for (int64_t j = 0; j < d; j++) ee += (double)e[j] * e[j];
                }
                double z = 0.5 * (sq - ee) + xs;
                double p = 1.0 / (1.0 + exp(-z));
                loss += (z > 0 ? z + log1p(exp(-z)) : log1p(exp(z))) - (double)yb * z;
                float c = (float)((p - (double)yb) / (double)nb);
                for (int f = 0; f < F; f++) {
                    int64_t ri = row(o, id[b * F + f]); const float* e = o->W + ri * d;
                    for (int64_t j = 0; j < d; j++) gr[f * d + j] = c * ((S[j] - e[j]) + xb[j]);
                }
            } else if (o->c.model == OR_MODEL_TRANSE) {
                continue;  /* whole chunks below */
            } else if (o->c.model == OR_MODEL_CONST) {  /* linear loss <x_b, e_f>: grad = x_b */
                for (int f = 0; f < F; f++)
                    for (int64_t j = 0; j < d; j++) gr[f * d + j] = xb[j];
            } else {                                    /* L2: 1/(2 nb) |e_f - x_b|^2 */
                float c = (float)(1.0 / (double)nb);
                for (int f = 0; f < F; f++) {
                    int64_t ri = row(o, id[b * F + f]); const float* e = o->W + ri * d;
                    for (int64_t j = 0; j < d; j++) {
                        float r = e[j] - xb[j];
                        loss += 0.5 * (double)r * r;
                        gr[f * d + j] = c * r;
                    }
                }
            }
        }
    }
    free(S);
    if (o->c.model == OR_MODEL_TRANSE) loss += transe(o, s, nb);
    o->loss[s] = nb ? loss / (double)nb : 0.0;
    /* (g) per-rank partials, positions ascending, sequential fp32 */
    for (int g = 0; g < n; g++) {
        int64_t m = step_len(o, s, g), u = 0;
        const int64_t* id = step_ids(o, s, g);
        pair64* a = malloc((m ? m : 1) * sizeof(pair64));
        for (int64_t i = 0; i < m; i++) { a[i].v = id[i]; a[i].p = i; }
        qsort(a, m, sizeof(pair64), cmp_pair);
        free(o->pk[g]); free(o->pv[g]);
        o->pk[g] = malloc((m ? m : 1) * sizeof(int64_t));
        o->pv[g] = malloc((m ? m : 1) * d * sizeof(float));
        const float* gr = o->grad + (int64_t)g * B * F * d;
        /* canonical fixed order (reading R23): occurrences of a row, positions
           ascending, are cut into chunks of OR_CHUNK; each chunk is summed
           sequentially and the chunk sums are added sequentially in order.
           (For <= OR_CHUNK occurrences this is the plain sequential sum.) */
        float* chunk = malloc(d * sizeof(float));
        int64_t i = 0;
        while (i < m) {
            int64_t e = i;
            while (e < m && a[e].v == a[i].v) e++;
            o->pk[g][u] = a[i].v;
            float* P = o->pv[g] + u * d;
            for (int64_t c0 = i; c0 < e; c0 += OR_CHUNK) {
                int64_t c1 = c0 + OR_CHUNK < e ? c0 + OR_CHUNK : e;
                memcpy(chunk, gr + a[c0].p * d, d * sizeof(float));
                for (int64_t q = c0 + 1; q < c1; q++)
                    for (int64_t j = 0; j < d; j++) chunk[j] = chunk[j] + gr[a[q].p * d + j];
                if (c0 == i) memcpy(P, chunk, d * sizeof(float));
                else for (int64_t j = 0; j < d; j++) P[j] = P[j] + chunk[j];
            }
            u++;
            i = e;
        }
        free(chunk);
        o->pn[g] = u;
        free(a);
    }
    /* (h) rows touched at s (any rank), ascending; g_k = sum over ranks ascending */
    int64_t tot = 0;
    for (int g = 0; g < n; g++) tot += o->pn[g];
    int64_t* all = malloc((tot ? tot : 1) * sizeof(int64_t));
    int64_t na = 0;
    for (int g = 0; g < n; g++) for (int64_t u = 0; u < o->pn[g]; u++) all[na++] = o->pk[g][u];
    qsort(all, na, sizeof(int64_t), cmp_i64);
    int64_t nu = 0;
    for (int64_t i = 0; i < na; i++) if (i == 0 || all[i] != all[i - 1]) all[nu++] = all[i];
    int64_t* cursor = calloc(n, sizeof(int64_t));
    float* gk = malloc(d * sizeof(float));
    const float lr = o->c.lr, eps = o->c.eps;
    for (int64_t a = 0; a < nu; a++) {
        int64_t k = all[a], i = row(o, k);
        int first = 1;
        for (int g = 0; g < n; g++) {
            if (cursor[g] < o->pn[g] && o->pk[g][cursor[g]] == k) {
                const float* P = o->pv[g] + cursor[g] * d;
                for (int64_t j = 0; j < d; j++) gk[j] = first ? P[j] : gk[j] + P[j];
                first = 0;
                cursor[g]++;
            }
        }
        /* a cold row is read from the host at update time: it must be fresh */
        if (!is_hot(o, k, s) && (o->meta[i].state != OR_CLEAN || !host_fresh_w(o, i) || !host_fresh_g(o, i)))
            o->violations++;
        /* (i) optimizer, elementwise fp32 */
        float* w = o->W + i * d;
        float* G = o->G + i * d;
        for (int64_t j = 0; j < d; j++) {
            if (o->c.opt == OR_SGD) {
                float t = lr * gk[j];
                w[j] = w[j] - t;
            } else {
                float sq = gk[j] * gk[j];
                G[j] = G[j] + sq;
                float num = lr * gk[j];
                float den = sqrtf(G[j]) + eps;
                w[j] = w[j] - num / den;
            }
        }
        /* (j) dirty, last update s */
        o->meta[i].state = OR_UPDATED;
        o->meta[i].last_update = (int32_t)s;
    }
    free(cursor); free(gk);
    free(o->upd);
    o->upd = all; o->n_upd = nu;
}

/* run the next step; returns its index or -1 past the end */
int64_t oracle_step(void* p) {
    oracle* o = p;
    if (o->cur >= o->S) return -1;
    int64_t s = o->cur++;
    schedule(o, s);
    train(o, s);
    for (int64_t a = 0; a < o->n_upd; a++) push(o, OR_L_UPDATED, o->upd[a]);
    return s;
}

/* end of training: every dirty row to the host (L1082-1083); hot rows also push G (R8) */
int64_t oracle_final_flush(void* p) {
    oracle* o = p;
    const int64_t last = o->cur > 0 ? o->cur - 1 : 0;
    for (int i = 0; i < OR_NLISTS; i++) o->nl[i] = 0;
    for (int64_t i = 0; i < o->n; i++) {
        if (o->meta[i].state != OR_CLEAN) {
            push(o, OR_L_FINAL, o->meta[i].key);
            flush_row(o, i, 1);
        }
        if (is_hot(o, o->meta[i].key, last)) {
            int64_t d = o->c.dim;
            memcpy(o->HG + i * d, o->G + i * d, d * sizeof(float));
        }
    }
    qsort(o->lists[OR_L_FINAL], o->nl[OR_L_FINAL], sizeof(int64_t), cmp_i64);
    o->n_upd = 0;
    return o->nl[OR_L_FINAL];
}

int64_t oracle_get_list(void* p, int which, int64_t* out, int64_t cap) {
    oracle* o = p;
    int64_t n = o->nl[which];
    if (out) memcpy(out, o->lists[which], (n < cap ? n : cap) * sizeof(int64_t));
    return n;
}
int oracle_gate_wait(void* p) { return ((oracle*)p)->gate_wait; }
double oracle_loss(void* p, int64_t s) { return ((oracle*)p)->loss[s]; }
int64_t oracle_violations(void* p) { return ((oracle*)p)->violations; }
int64_t oracle_n_rows_touched(void* p) { return ((oracle*)p)->n; }

/* dedup artefacts of rank g at step s: uniq ascending, inv[i] = index of ids[i] in uniq */
int64_t oracle_dedup(void* p, int64_t s, int32_t g, int64_t* out_uniq, int32_t* out_inv) {
    oracle* o = p;
    int64_t n; const int64_t* u = uniq(o, s, g, &n);
    if (out_uniq) memcpy(out_uniq, u, n * sizeof(int64_t));
    if (out_inv) {
        const int64_t* id = step_ids(o, s, g);
        for (int64_t i = 0; i < step_len(o, s, g); i++) {
            const int64_t* hit = bsearch(&id[i], u, n, sizeof(int64_t), cmp_i64);
            out_inv[i] = (int32_t)(hit - u);
        }
    }
    return n;
}
int32_t oracle_next_access(void* p, int64_t k, int64_t u) { return next_access(p, k, u); }
int32_t oracle_needs_host(void* p, int64_t k, int64_t t) { return needs_host(p, k, t); }
int32_t oracle_row_state(void* p, int64_t k) {
    oracle* o = p; int64_t i = find_row(o, k);
    return i < 0 ? OR_CLEAN : o->meta[i].state;
}

/* authoritative (synchronous) values */
void oracle_read_rows(void* p, const int64_t* ks, int64_t n, float* w, float* G) {
    oracle* o = p; int64_t d = o->c.dim;
    for (int64_t a = 0; a < n; a++) {
        int64_t i = row(o, ks[a]);
        if (w) memcpy(w + a * d, o->W + i * d, d * sizeof(float));
        if (G) memcpy(G + a * d, o->G + i * d, d * sizeof(float));
    }
}
/* simulated host table */
void oracle_host_rows(void* p, const int64_t* ks, int64_t n, float* w, float* G) {
    oracle* o = p; int64_t d = o->c.dim;
    for (int64_t a = 0; a < n; a++) {
        int64_t i = row(o, ks[a]);
        if (w) memcpy(w + a * d, o->Hw + i * d, d * sizeof(float));
        if (G) memcpy(G + a * d, o->HG + i * d, d * sizeof(float));
    }
}
/* last step: glue gradients of rank g [batch*slots][dim] */
void oracle_get_grad(void* p, int32_t g, float* out) {
    oracle* o = p;
    int64_t m = (int64_t)o->c.batch * o->c.slots * o->c.dim;
    memcpy(out, o->grad + g * m, m * sizeof(float));
}
/* last step: partials of rank g (keys ascending) */
int64_t oracle_get_partial(void* p, int32_t g, int64_t* keys, float* P) {
    oracle* o = p;
    if (keys) memcpy(keys, o->pk[g], o->pn[g] * sizeof(int64_t));
    if (P) memcpy(P, o->pv[g], o->pn[g] * o->c.dim * sizeof(float));
    return o->pn[g];
}
/* the init function, exposed for pins */
float oracle_init_value(void* p, int64_t k, int32_t j) { return init_w(p, k, j); }
