// cpu_apply_probe.c -- can host threads apply a drain's rows (34k random 128-B rows of a 4.3 GB
// table, from a packed log) fast enough to replace the GPU's zero-copy scatter?  THP vs 4K pages,
// memcpy vs non-temporal stores, 1..8 threads (persistent, spinning workers).
#include <immintrin.h>
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#include <sys/mman.h>
static double now() { struct timespec t; clock_gettime(CLOCK_MONOTONIC, &t); return t.tv_sec + t.tv_nsec * 1e-9; }
#define NROWS 33762577L
#define NPER 34000
static float* table; static float* packed; static int32_t* idx; static int nthr, nt_mode;
static volatile int go_gen = 0, done_cnt = 0;
static void* worker(void* a) {
    long t = (long)a; int seen = 0;
    for (;;) {
        while (go_gen == seen) _mm_pause();
        seen = go_gen; if (seen < 0) return 0;
        int lo = NPER * t / nthr, hi = NPER * (t + 1) / nthr;
        for (int i = lo; i < hi; i++) {
            float* dst = table + (int64_t)idx[i] * 32; const float* src = packed + (int64_t)i * 32;
            if (nt_mode) { for (int c = 0; c < 2; c++) _mm512_stream_si512((__m512i*)(dst + 16 * c), _mm512_load_si512((const __m512i*)(src + 16 * c))); }
            else memcpy(dst, src, 128);
        }
        if (nt_mode) _mm_sfence();
        __sync_fetch_and_add(&done_cnt, 1);
    }
}
int main() {
    for (int thp = 0; thp < 2; thp++) {
        table = mmap(0, NROWS * 128, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
        if (thp) madvise(table, NROWS * 128, MADV_HUGEPAGE); else madvise(table, NROWS * 128, MADV_NOHUGEPAGE);
        memset(table, 1, NROWS * 128);
        packed = aligned_alloc(64, NPER * 128L); memset(packed, 2, NPER * 128L);
        idx = malloc(NPER * 4);
        srand(1);
        for (nt_mode = 0; nt_mode < 2; nt_mode++)
        for (nthr = 1; nthr <= 8; nthr *= 2) {
            pthread_t th[16]; go_gen = 0; done_cnt = 0;
            for (long t = 0; t < nthr; t++) pthread_create(&th[t], 0, worker, (void*)t);
            double best = 1e9, sum = 0; int reps = 30;
            for (int rep = 0; rep < reps; rep++) {
                for (int i = 0; i < NPER; i++) idx[i] = ((uint64_t)rand() * 2654435761u) % NROWS;
                done_cnt = 0; double t0 = now(); __sync_synchronize(); go_gen = rep + 1;
                while (done_cnt < nthr) _mm_pause();
                double dt = now() - t0; if (dt < best) best = dt; sum += dt;
            }
            go_gen = -1; for (int t = 0; t < nthr; t++) pthread_join(th[t], 0);
            printf("%s %-6s threads %d: best %.1f us mean %.1f us for %d rows (%.1f GB/s)\n", thp ? "THP" : "4K ", nt_mode ? "nt" : "memcpy",
                   nthr, best * 1e6, sum / reps * 1e6, NPER, NPER * 128 / best / 1e9);
        }
        munmap(table, NROWS * 128);
    }
}
