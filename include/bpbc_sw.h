/*
 * bpbc_sw.h -- C ABI of the B200 (sm_100a) Bitwise Parallel Bulk Computation
 * (BPBC) of the Smith-Waterman algorithm.
 *
 * Paper: T. Nishimura, J. L. Bordim, Y. Ito, K. Nakano, "Accelerating the
 * Smith-Waterman Algorithm Using Bitwise Parallel Bulk Computation Technique
 * on GPU", IPDPS Workshops 2017.  "P:Lnnn" cites line nnn of its text
 * (PAPER.md); "Rk" cites reading k in DESIGN.md.
 *
 * Problem: num_pairs independent DNA pairs
 * (X_k, Y_k), all with the same lengths m and n, stored wordwise (one byte
 * per base, P:L350 / R15).  For each pair the library returns the maximum
 * local-alignment score of the Smith-Waterman recurrence
 *
 *   d[i][j] = max(0, d[i-1][j] + gap, d[i][j-1] + gap,
 *                 d[i-1][j-1] + (x_i == y_j ? match : mismatch)),
 *   d[-1][.] = d[.][-1] = 0,  score = min(max_ij d[i][j], 2^score_bits - 1)
 *
 * (signed API constants: paper c1 = match, c2 = -mismatch, paper gap = -gap,
 * R1; width cap R3).  Internally the pairs are bit-transposed 32 to a word
 * (bit k = pair k) and every cell update runs as a Boolean circuit on
 * bit-sliced s-bit scores, so one 32-bit logic op advances 32
 * alignments.
 *
 * Base codes (R18): A = 0, T = 1, G = 2, C = 3 (the paper's A=00,
 * T=01, G=10, C=11 with the H bit first).  Any byte > 3 is read as (c & 3)
 * and raises the sticky BPBC_FLAG_BAD_BASE flag.
 *
 * Conventions for every function:
 *   - returns a bpbc_status (0 = OK, < 0 error); never aborts, exits or
 *     throws; no function writes to caller memory on an argument error;
 *   - "device" pointers are CUDA device (or managed) memory of the ctx's
 *     device; "host" pointers are host memory (pinned gives the fastest
 *     copies);
 *   - asynchronous functions only ENQUEUE work on `stream` (a cudaStream_t,
 *     NULL = legacy default stream) and return; the caller keeps every
 *     buffer alive until the stream has completed that work;
 *   - no function synchronizes the whole device: the blocking ones wait
 *     only for work this ctx enqueued;
 *   - ctx-owned buffers (the workspace used when `workspace` is NULL) are
 *     ordered across streams by the library: a call on stream B after a
 *     call on stream A makes B wait for A's use of them (an event), so
 *     calls on different streams through one ctx never share them
 *     concurrently.  Caller-owned workspaces are the caller's to order
 *     (give concurrent streams separate workspaces);
 *   - a ctx is not thread-safe: use one ctx per device per host thread;
 *   - the environment is read once, in bpbc_sw_init (benchmark knobs only:
 *     BPBC_MAX_BLOCKS_PER_SM, BPBC_MIN_BLOCKS_PER_SM, BPBC_NO_EXACT_RUN, BPBC_WRAP,
 *     BPBC_CHUNKED_HOST, BPBC_FORCE_WIDTH -- see DESIGN.md 6.4); no call on
 *     the hot path reads it.
 */
#ifndef BPBC_SW_H
#define BPBC_SW_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bpbc_sw_ctx bpbc_sw_ctx;

typedef enum {
    BPBC_OK = 0,
    BPBC_ERR_INVALID_ARG = -1, /* bad pointer / size / constant / workspace      */
    BPBC_ERR_UNSUPPORTED = -2, /* valid but outside what this build supports     */
    BPBC_ERR_CUDA = -3,        /* a CUDA call failed; text in bpbc_sw_last_error */
    BPBC_ERR_OOM = -4,         /* device or host allocation failed               */
    BPBC_ERR_BAD_BASE = -5     /* returned by bpbc_sw_get_error_flags when a base
                                  code > 3 was seen since the last read */
} bpbc_status;

/* Sticky device flags (bpbc_sw_get_error_flags). */
#define BPBC_FLAG_BAD_BASE 0x1u /* a base code > 3 was packed (read as c & 3) */
#define BPBC_FLAG_STALL 0x2u    /* a device-side wait of the host-streamed or wrap-around
                                   schedule saw no progress for 20 s and gave up: the
                                   scores of that call are undefined (never expected;
                                   guards against hanging the GPU) */

/* Supported ranges of this build. */
#define BPBC_MIN_SCORE_BITS 4
#define BPBC_MAX_SCORE_BITS 16
#define BPBC_MAX_LEN (1 << 20)       /* m, n <= 2^20 */
#define BPBC_MAX_QUERY_LEN (1 << 16) /* min(m, n) <= 2^16 */

/* Binds the context to `cuda_device`, creates its device flag word, a
 * private stream for flag reads and queries the SM count; reads the
 * benchmark knobs from the environment (once).  No pair-sized allocation.
 * *out_ctx is set only on success. */
int bpbc_sw_init(int cuda_device, bpbc_sw_ctx **out_ctx);

/* Waits for the work this ctx enqueued (on every stream it used), then frees
 * everything the ctx owns (workspace, host-path buffers and streams, pinned
 * staging).  NULL is a no-op. */
int bpbc_sw_destroy(bpbc_sw_ctx *ctx);

/* Upper bound on the device workspace any bpbc_sw_score_batch* /
 * bpbc_sw_filter_batch call with these sizes needs, whatever its constants
 * and width: the bit-transposed planes 8 * ceil(P/32) * (m + n) bytes plus
 * padding (only plans that run the separate pack pass use them), the
 * per-lane partial maxima (2 KiB per 32-pair group, per 128 query rows), the
 * stripe boundary rows when min(m, n) > 128 (64 * max(m, n) bytes per
 * concurrent group stream, at most 1 GiB), the wrap-around schedule's warp
 * snapshots when the batch has few groups (<= 8192) of a long target, and the
 * filter's compaction scratch.  Pure host function. */
int bpbc_sw_workspace_bytes(int64_t num_pairs, int32_t m, int32_t n, size_t *bytes);

/* Exact device workspace of one call with these arguments (the plan the
 * call will run on ctx's device: circuit, kernel, schedule), <= the bound
 * above.  filter != 0: for bpbc_sw_filter_batch.  Errors as
 * bpbc_sw_score_batch's argument checks.  Host function (queries the
 * kernels' occupancy once). */
int bpbc_sw_workspace_bytes_for(bpbc_sw_ctx *ctx, int64_t num_pairs, int32_t m, int32_t n,
                                int32_t match, int32_t mismatch, int32_t gap,
                                int32_t score_bits, int32_t filter, size_t *bytes);

/*
 * The hot path (Steps 2-4): pack (W2B) -> bit-sliced wavefront
 * sweep with running max -> max over rows -> untranspose (B2W), all on the
 * device, enqueued on `stream`.
 *
 * query       device, uint8 [num_pairs][m] row-major base codes (X_k).
 * target      device, uint8 [num_pairs][n] row-major base codes (Y_k).
 * num_pairs   >= 0; 0 is a no-op.  Need not be a multiple of 32.
 * m, n        1 .. BPBC_MAX_LEN each; m > n is allowed (roles are swapped
 *             internally; the score is symmetric, R17).  min(m, n) <=
 *             BPBC_MAX_QUERY_LEN (else BPBC_ERR_UNSUPPORTED); above 256 the
 *             query rows are processed in stripes of 128.
 * match       >= 1                      (paper c1)
 * mismatch    <= 0                      (paper -c2)
 * gap         <= 0                      (paper -gap, linear per column)
 * score_bits  s in [4, 16]: width of the bit-sliced score.  match,
 *             -mismatch and -gap must each be <= 2^s - 1.  Results are
 *             min(score, 2^s - 1) exactly (R3).
 * out_scores  device, int32 [num_pairs].
 * workspace   device scratch owned by the caller of >= bpbc_sw_workspace_bytes_for
 *             (...) bytes (bpbc_sw_workspace_bytes is always enough), or NULL
 *             to use the ctx-owned buffer, grown on demand in stream order
 *             (cudaMallocAsync on `stream`; no device-wide sync).
 * stream      cudaStream_t to enqueue on.
 *
 * Errors (host-side, no device sync): INVALID_ARG for negative sizes, NULL
 * pointers with num_pairs > 0, out-of-range constants or a too-small
 * workspace; UNSUPPORTED for score_bits outside [4,16] or lengths beyond this
 * build; CUDA if a launch fails.  Bad base codes cannot be seen without a
 * sync: they set BPBC_FLAG_BAD_BASE.
 */
int bpbc_sw_score_batch(bpbc_sw_ctx *ctx, const uint8_t *query, const uint8_t *target,
                        int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                        int32_t mismatch, int32_t gap, int32_t score_bits,
                        int32_t *out_scores, void *workspace, size_t workspace_bytes,
                        void *stream);

/*
 * End-to-end variant with HOST buffers (the paper's Steps 1-5):
 * copies the inputs host->device, runs the hot path and copies the scores
 * device->host.  Plans of the fused single-warp kernel (min(m, n) <= 256)
 * run as ONE streamed launch on ctx-owned streams: the sweep runs on a
 * compute stream while the inputs are copied on a copy stream in waves, each
 * closed by a device-side progress write (cuStreamWriteValue32) the sweep
 * polls before it reads that wave.  Group-granular plans: a wave = one
 * 32-pair group per sweep stream (contiguous, since groups are assigned to
 * streams strided).  Wrap-around plans (few long groups): a
 * wave = a column block of every stream's copy timeline, moved by one launch
 * of a gather kernel that reads PINNED host rows directly (pageable inputs
 * are copied whole before the sweep).  Each ctx first checks once that a
 * kernel can see a stream write enqueued after its launch (not so under a
 * kernel-serialising profiler or CUDA_LAUNCH_BLOCKING=1); where it cannot,
 * and for the other plans, the batch is cut into chunks of whole waves that
 * flow through three ctx-owned buffer slots on three ctx-owned streams
 * (copy-in, kernels, copy-out), so the copy of chunk c+1 and the result copy
 * of chunk c-1 overlap the kernels of chunk c; the chunk plan uses the H2D
 * and cell rates this ctx measured on its previous host call.  Device-side
 * waits are bounded (20 s): a wait that times out makes this ctx rerun the
 * batch chunked.  A pageable out_scores goes through pinned staging.
 * Blocking: returns when out_scores is written.
 *
 * query, target  host, uint8 [num_pairs][m] / [num_pairs][n].
 * out_scores     host, int32 [num_pairs].
 * Other arguments as bpbc_sw_score_batch.
 */
int bpbc_sw_score_batch_host(bpbc_sw_ctx *ctx, const uint8_t *query, const uint8_t *target,
                             int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                             int32_t mismatch, int32_t gap, int32_t score_bits,
                             int32_t *out_scores);

/*
 * Same as bpbc_sw_score_batch / bpbc_sw_score_batch_host with the bases
 * 2-bit packed, 4 per byte (the paper's 2-bit code of P:L51, stored densely;
 * SURVEY.md NEXT-1): row k of query2 is ceil(m/4) bytes and base i of it is
 * bits [2(i%4), 2(i%4)+1] of byte i/4 (A=0, T=1, G=2, C=3; bits past the row
 * end are ignored).  target2 likewise with ceil(n/4) bytes per row.  Cuts the
 * input bytes (and the host->device copy of the _host variant) 4x; every code
 * is valid, so BPBC_FLAG_BAD_BASE is never raised.  Rows are read with
 * 16-byte loads when ceil(len/4) is a multiple of 16 and the buffer is 16-byte
 * aligned, byte by byte otherwise.
 */
int bpbc_sw_score_batch_packed2(bpbc_sw_ctx *ctx, const uint8_t *query2, const uint8_t *target2,
                                int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                                int32_t mismatch, int32_t gap, int32_t score_bits,
                                int32_t *out_scores, void *workspace, size_t workspace_bytes,
                                void *stream);
int bpbc_sw_score_batch_host_packed2(bpbc_sw_ctx *ctx, const uint8_t *query2,
                                     const uint8_t *target2, int64_t num_pairs, int32_t m,
                                     int32_t n, int32_t match, int32_t mismatch, int32_t gap,
                                     int32_t score_bits, int32_t *out_scores);

/*
 * Threshold filter (the paper's stated use: flag the pairs
 * whose maximum score exceeds a threshold and re-align only those, with
 * traceback, on the CPU).  Same hot path as bpbc_sw_score_batch with
 * the per-cell running maximum (2s logic ops) replaced by a sticky
 * "some cell > threshold" flag (s + 1 ops).
 *
 * threshold    0 <= threshold <= 2^score_bits - 2; a pair is flagged iff
 *              its maximum local score > threshold.
 * out_mask     device, uint32 [ceil(num_pairs/32)]: bit k of word g = flag of
 *              pair 32g+k (bits past num_pairs are 0).  Required.
 * out_indices  device, int64 [num_pairs] or NULL: the flagged pair indices in
 *              ascending order (the first *out_count entries are written).
 * out_count    device, int64 [1] or NULL: number of flagged pairs.
 * The compaction scratch is a section of the workspace (size it with
 * bpbc_sw_workspace_bytes_for(..., filter = 1, ...)).  Other arguments
 * and errors as bpbc_sw_score_batch; a threshold outside the range above is
 * INVALID_ARG.  Asynchronous on `stream`.
 */
int bpbc_sw_filter_batch(bpbc_sw_ctx *ctx, const uint8_t *query, const uint8_t *target,
                         int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                         int32_t mismatch, int32_t gap, int32_t score_bits, int32_t threshold,
                         uint32_t *out_mask, int64_t *out_indices, int64_t *out_count,
                         void *workspace, size_t workspace_bytes, void *stream);

/*
 * Wordwise comparator: the same scores computed WITHOUT
 * the bitwise technique -- ordinary integer DP cells, the paper's "GPU
 * wordwise" implementation (Table IV) written for sm_100a with
 * 16-bit SIMD (two pairs per warp register) -- so the BPBC path's gain can be
 * measured on the same GPU.  Returns the exact max local score (no width
 * cap).  min(m, n) <= 256 and the scores must fit 16 bits (else
 * UNSUPPORTED).  workspace: device, >= bpbc_sw_wordwise_workspace_bytes, or
 * NULL for the ctx-owned buffer.  Asynchronous on `stream`.
 */
int bpbc_sw_wordwise_workspace_bytes(int64_t num_pairs, size_t *bytes);
int bpbc_sw_score_batch_wordwise(bpbc_sw_ctx *ctx, const uint8_t *query, const uint8_t *target,
                                 int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                                 int32_t mismatch, int32_t gap, int32_t *out_scores,
                                 void *workspace, size_t workspace_bytes, void *stream);

/*
 * W2B step alone: bit-transpose base codes into planes.
 * codes   device, uint8 [num_pairs][len].
 * planes  device, uint32 [ceil(num_pairs/32)][len][2]: [g][i][0] = X^H_i,
 *         [g][i][1] = X^L_i of group g (bit k = pair 32g+k; pairs past
 *         num_pairs read as code 0).
 */
int bpbc_sw_pack(bpbc_sw_ctx *ctx, const uint8_t *codes, int64_t num_pairs, int32_t len,
                 uint32_t *planes, void *stream);

/*
 * Max-reduction + B2W step alone.
 * partial    device, uint32 [num_groups][lanes][s]: lanes bit-sliced s-bit
 *            values per 32-pair group (bit k of word b = bit b of pair k's
 *            value).
 * out        device, int32 [num_pairs] (num_pairs <= 32 * num_groups):
 *            out[32g+k] = min(max over lanes of the value of pair k, cap).
 * lanes in [1, 4096], s in [1, 16], cap >= 0.
 */
int bpbc_sw_untranspose(bpbc_sw_ctx *ctx, const uint32_t *partial, int64_t num_groups,
                        int32_t lanes, int32_t s, int64_t num_pairs, int32_t cap,
                        int32_t *out, void *stream);

/* Waits for the work this ctx enqueued on every stream it used since the
 * last read (not the whole device), returns the sticky flags in *flags (bit
 * 0 = BPBC_FLAG_BAD_BASE, bit 1 = BPBC_FLAG_STALL) and clears them.  Returns BPBC_ERR_BAD_BASE when
 * that bit was set (the scores of those calls used c & 3 for the bad codes,
 * R18), BPBC_OK otherwise; *flags is written in both cases. */
int bpbc_sw_get_error_flags(bpbc_sw_ctx *ctx, uint32_t *flags);

/* Description of the last sweep dispatch (for benchmarks and tests):
 * circuit 0 = exact offset circuit, 1 = saturating circuit; the score width
 * actually evaluated; rows per lane R; lanes per 32-pair group L; concurrent
 * group streams; and the bitwise-logic operations per word-cell of the
 * evaluated circuit (hand count). Any pointer may be NULL. */
int bpbc_sw_last_plan(bpbc_sw_ctx *ctx, int32_t *circuit, int32_t *width, int32_t *rows_per_lane,
                      int32_t *lanes, int64_t *streams, int32_t *ops_per_word_cell);

/* Kernels of this library the last bpbc_sw_score_batch / _filter_batch call
 * on this ctx launched (pack, sweep, epilogue kernels; the CUB scan of the
 * filter compaction counts as one), and whether its sweep was the fused
 * kernel that transposes the raw codes itself (1) or ran on packed planes
 * (0).  Either pointer may be NULL. */
int bpbc_sw_last_launches(bpbc_sw_ctx *ctx, int32_t *kernels, int32_t *fused);

/* Stream schedule of the last sweep: wrap = 1 if it used the wrap-around
 * schedule (streams take equal runs of the concatenated target columns and
 * hand split groups over as warp-state snapshots), 0 for the
 * group-granular split; blocks_per_sm = resident sweep blocks per SM the
 * plan chose; host_streamed = 1 if the last bpbc_sw_score_batch_host* call
 * ran as one streamed launch (below), 0 if chunked.  Any pointer may be
 * NULL. */
int bpbc_sw_last_schedule(bpbc_sw_ctx *ctx, int32_t *wrap, int64_t *blocks_per_sm,
                          int32_t *host_streamed);

/* Per-phase device timing, the columns of the paper's Table IV (P:L384-413:
 * W2B, SWA, B2W).  bpbc_sw_profile(ctx, 1) clears the accumulators and makes
 * every following bpbc_sw_score_batch* call record CUDA events around its
 * kernels on the call's stream; bpbc_sw_profile(ctx, 0) stops recording.
 * bpbc_sw_profile_read synchronizes the recorded events and returns the
 * summed milliseconds since the last read/enable:
 *   ms[0] = W2B (both packs), ms[1] = SWA (sweep), ms[2] = B2W (extract),
 *   ms[3] = their sum; *calls = number of calls recorded.  Then resets. */
int bpbc_sw_profile(bpbc_sw_ctx *ctx, int enable);
int bpbc_sw_profile_read(bpbc_sw_ctx *ctx, double ms[4], int64_t *calls);

/* Static text for a status code. */
const char *bpbc_sw_status_string(int status);

/* Text of the last CUDA error seen by this ctx ("" if none). */
const char *bpbc_sw_last_error(bpbc_sw_ctx *ctx);

#ifdef __cplusplus
}
#endif

#endif /* BPBC_SW_H */
