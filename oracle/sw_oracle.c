/*
 * oracle/sw_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU Smith-Waterman used to check the CUDA
 * path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares no code, header,
 * table or constant with paper_conf_ipps_nishimurabin17_b200/ (the product),
 * and the product never loads it.
 *
 * Citations are lines of the paper text PAPER.md ("P:Lnnn"), i.e.
 * Nishimura, Bordim, Ito, Nakano, "Accelerating the Smith-Waterman Algorithm
 * Using Bitwise Parallel Bulk Computation Technique on GPU", IPDPSW 2017.
 *
 * Definition followed (Sec. III recurrence; Sec. III
 * "Sequential algorithm for the SWA"), with the API's signed constants
 * (reading R1: the paper subtracts gap/c2 as magnitudes, the API
 * passes signed scores match>0, mismatch<=0, gap<=0):
 *
 *   d[-1][j] = d[i][-1] = 0
 *   d[i][j]  = max(0, d[i-1][j] + gap, d[i][j-1] + gap,
 *                  d[i-1][j-1] + (x_i == y_j ? match : mismatch))
 *   best     = max over all cells (0 if none positive)
 *   out      = min(best, 2^score_bits - 1)  if score_bits > 0  (reading R3)
 *
 * Pins (tests/test_oracle.py): Table II cell by cell, brute-force
 * enumeration of every alignment path (oracle_brute_local below, which uses
 * no DP), match*LCS when gap = 0, match*longest-common-substring when the
 * penalties are huge, per-diagonal Kadane when only the gap is huge, closed
 * forms and invariants.
 *
 * Plain int32 arithmetic, one rolling row, no SIMD intrinsics.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

static int max2(int a, int b) { return a > b ? a : b; }

/* w(x_i, y_j) of P:L198 with signed API constants (reading R1). */
static int w_score(uint8_t xi, uint8_t yj, int match, int mismatch) {
    return xi == yj ? match : mismatch;
}

/*
 * Full (m+1) x (n+1) score matrix d, row-major, row 0 and column 0 the zero
 * borders of P:L202-204.  Used to reproduce Table II.
 */
void oracle_sw_matrix(const uint8_t *x, int m, const uint8_t *y, int n,
                      int match, int mismatch, int gap, int32_t *d) {
    int W = n + 1;
    for (int j = 0; j <= n; ++j) d[j] = 0;                 /* d[-1][j] = 0 */
    for (int i = 1; i <= m; ++i) {
        d[i * W] = 0;                                      /* d[i][-1] = 0 */
        for (int j = 1; j <= n; ++j) {
            int v = 0;
            v = max2(v, d[(i - 1) * W + j] + gap);         /* from above   */
            v = max2(v, d[i * W + j - 1] + gap);           /* from left    */
            v = max2(v, d[(i - 1) * W + j - 1] +
                            w_score(x[i - 1], y[j - 1], match, mismatch));
            d[i * W + j] = v;
        }
    }
}

/*
 * Maximum local score of one pair with one rolling row of n+1 ints
 * (P:L202-216 in row-major order).  row[j] holds d[i-1][j] before the update
 * of cell (i,j) and d[i][j] after it; diag keeps d[i-1][j-1].
 */
int oracle_sw_score(const uint8_t *x, int m, const uint8_t *y, int n,
                    int match, int mismatch, int gap) {
    int32_t stack_row[1025];
    int32_t *row = n + 1 <= 1025 ? stack_row
                                 : (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
    if (!row) return -1;
    for (int j = 0; j <= n; ++j) row[j] = 0;
    int best = 0;
    for (int i = 1; i <= m; ++i) {
        int diag = 0;          /* d[i-1][0] */
        int left = 0;          /* d[i][0]   */
        uint8_t xi = x[i - 1];
        for (int j = 1; j <= n; ++j) {
            int up = row[j];   /* d[i-1][j] */
            int v = 0;
            v = max2(v, up + gap);
            v = max2(v, left + gap);
            v = max2(v, diag + w_score(xi, y[j - 1], match, mismatch));
            diag = up;
            row[j] = v;
            left = v;
            if (v > best) best = v;
        }
    }
    if (row != stack_row) free(row);
    return best;
}

/* ------------------------------------------------------------------------ */
/* Batch driver: P pairs of fixed lengths, row-major [P][m] and
 * [P][n] byte codes.  Threads split contiguous pair ranges. */

typedef struct {
    const uint8_t *q, *t;
    int64_t p0, p1;
    int m, n, match, mismatch, gap, score_bits;
    int32_t *out;
} job_t;

static void *batch_worker(void *arg) {
    job_t *jb = (job_t *)arg;
    int64_t cap = jb->score_bits > 0 ? (((int64_t)1 << jb->score_bits) - 1) : -1;
    for (int64_t p = jb->p0; p < jb->p1; ++p) {
        int s = oracle_sw_score(jb->q + p * jb->m, jb->m, jb->t + p * jb->n, jb->n,
                                jb->match, jb->mismatch, jb->gap);
        if (cap >= 0 && s > cap) s = (int)cap;   /* reading R3 */
        jb->out[p] = s;
    }
    return NULL;
}

int oracle_sw_batch(const uint8_t *q, const uint8_t *t, int64_t num_pairs,
                    int m, int n, int match, int mismatch, int gap,
                    int score_bits, int32_t *out, int nthreads) {
    if (num_pairs <= 0) return 0;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    if ((int64_t)nthreads > num_pairs) nthreads = (int)num_pairs;
    pthread_t th[256];
    job_t jobs[256];
    int64_t chunk = num_pairs / nthreads, rem = num_pairs % nthreads, p = 0;
    for (int k = 0; k < nthreads; ++k) {
        int64_t cnt = chunk + (k < rem ? 1 : 0);
        jobs[k] = (job_t){q, t, p, p + cnt, m, n, match, mismatch, gap, score_bits, out};
        p += cnt;
    }
    int joined[256] = {0};
    for (int k = 1; k < nthreads; ++k) {
        if (pthread_create(&th[k], NULL, batch_worker, &jobs[k]) != 0)
            batch_worker(&jobs[k]);      /* could not spawn: run it here */
        else
            joined[k] = 1;
    }
    batch_worker(&jobs[0]);
    for (int k = 1; k < nthreads; ++k)
        if (joined[k]) pthread_join(th[k], NULL);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Brute force: enumerate EVERY alignment path of every pair of substrings
 * and take the best score (0 for the empty alignment).  No dynamic
 * programming, no combining of partial results at cells: each path is scored
 * on its own.  A path starts at any (i0, j0) and takes steps
 *   D: align x_i with y_j (score w),  U: x_i against a gap,  L: y_j against a gap
 * ("local-alignment": highly similar substrings; P:L194 gap moves).
 * Exponential -- only for m, n <= 8. */

typedef struct {
    const uint8_t *x, *y;
    int m, n, match, mismatch, gap;
    int best;
} brute_t;

static void brute_rec(brute_t *b, int i, int j, int score) {
    if (score > b->best) b->best = score;
    if (i < b->m && j < b->n)
        brute_rec(b, i + 1, j + 1, score + w_score(b->x[i], b->y[j], b->match, b->mismatch));
    if (i < b->m) brute_rec(b, i + 1, j, score + b->gap);
    if (j < b->n) brute_rec(b, i, j + 1, score + b->gap);
}

int oracle_brute_local(const uint8_t *x, int m, const uint8_t *y, int n,
                       int match, int mismatch, int gap) {
    if (m > 8 || n > 8) return -1;
    brute_t b = {x, y, m, n, match, mismatch, gap, 0};
    for (int i0 = 0; i0 <= m; ++i0)
        for (int j0 = 0; j0 <= n; ++j0) brute_rec(&b, i0, j0, 0);
    return b.best;
}
