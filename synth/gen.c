/*
 * synth/gen.c -- seeded synthetic DNA pairs (counter-based SplitMix64).
 *
 * Input generator shared by tests and bench for BOTH sides (oracle and CUDA
 * path).  It holds none of the method's arithmetic: it only draws base codes
 * A=0, T=1, G=2, C=3 i.i.d. uniform, optionally planting copies of the
 * query into the target so that scores reach the width cap (input
 * recipe).  The numpy version in synth/__init__.py is the readable
 * definition; this C version is the fast one and is cross-checked against it.
 *
 *   mix(k)   = SplitMix64 finaliser of k + 0x9E3779B97F4A7C15
 *   q[p][i]  = mix(seed ^ (0<<63) ^ (p<<24) ^ i) >> 62
 *   t[p][j]  = mix(seed ^ (1<<63) ^ (p<<24) ^ j) >> 62
 *   planted: sel = mix(seed ^ (3<<62) ^ p)
 *     (sel & 63) == 1 : t[p][j] = q[p][j mod m]                 (exact copy)
 *     (sel & 15) == 0 : t[p][j] = q[p][j mod m], substituted where
 *                       h = mix(seed ^ (1<<62) ^ (p<<24) ^ j), h % 10 == 0,
 *                       by (code + 1 + (h>>62) % 3) & 3          (10% mutated)
 */
#include <stdint.h>
#include <pthread.h>

static inline uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

typedef struct {
    uint64_t seed; int64_t p_begin, p_end, p_offset; int m, n, planted;
    uint8_t *q, *t;
} gjob_t;

static void *gen_worker(void *arg) {
    gjob_t *g = (gjob_t *)arg;
    for (int64_t lp = g->p_begin; lp < g->p_end; ++lp) {
        uint64_t p = (uint64_t)(lp + g->p_offset);
        uint8_t *q = g->q + lp * g->m, *t = g->t + lp * g->n;
        for (int i = 0; i < g->m; ++i)
            q[i] = (uint8_t)(mix(g->seed ^ (p << 24) ^ (uint64_t)i) >> 62);
        int kind = 0;
        if (g->planted) {
            uint64_t sel = mix(g->seed ^ (3ull << 62) ^ p);
            if ((sel & 63) == 1) kind = 2;
            else if ((sel & 15) == 0) kind = 1;
        }
        for (int j = 0; j < g->n; ++j) {
            if (kind == 0) {
                t[j] = (uint8_t)(mix(g->seed ^ (1ull << 63) ^ (p << 24) ^ (uint64_t)j) >> 62);
            } else {
                uint8_t c = q[j % g->m];
                if (kind == 1) {
                    uint64_t h = mix(g->seed ^ (1ull << 62) ^ (p << 24) ^ (uint64_t)j);
                    if (h % 10 == 0) c = (uint8_t)((c + 1 + (h >> 62) % 3) & 3);
                }
                t[j] = c;
            }
        }
    }
    return 0;
}

int synth_gen_pairs(uint64_t seed, int64_t num_pairs, int64_t p_offset, int m, int n,
                    int planted, uint8_t *q, uint8_t *t, int nthreads) {
    if (num_pairs <= 0) return 0;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    if (nthreads > num_pairs) nthreads = (int)num_pairs;
    pthread_t th[256]; gjob_t jb[256]; int ok[256] = {0};
    int64_t chunk = num_pairs / nthreads, rem = num_pairs % nthreads, p = 0;
    for (int k = 0; k < nthreads; ++k) {
        int64_t c = chunk + (k < rem);
        jb[k] = (gjob_t){seed, p, p + c, p_offset, m, n, planted, q, t};
        p += c;
    }
    for (int k = 1; k < nthreads; ++k)
        ok[k] = pthread_create(&th[k], 0, gen_worker, &jb[k]) == 0;
    for (int k = 1; k < nthreads; ++k)
        if (!ok[k]) gen_worker(&jb[k]);
    gen_worker(&jb[0]);
    for (int k = 1; k < nthreads; ++k)
        if (ok[k]) pthread_join(th[k], 0);
    return 0;
}
