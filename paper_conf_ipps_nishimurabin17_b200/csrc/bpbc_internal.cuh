// bpbc_internal.cuh -- shared layout and launch declarations of the CUDA path.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "bpbc_sw.h"
#include "circuit.cuh"

namespace bpbc {

// Planes buffers carry padding so the sweep never bounds-checks its loads:
// the Y stream of a warp is read at virtual column J = tau - lane, which runs
// up to L columns before its first group and up to n + L columns past its
// last.
constexpr int64_t kYFrontPad = 512;  // uint2 words before Y plane 0 (multi-warp lag)
constexpr int64_t kXBackPad = 512;   // uint2 words after the last X group
constexpr int64_t kYBackPadExtra = 640;

enum Circuit : int { kExact = 0, kSat = 1 };
enum Mode : int { kModeMax = 0, kModeThreshold = 1 };  // running max / sticky flag
enum Consts : int { kC211 = 0, kCRun = 1 };
// Kernel kinds of the multi-warp and striped registries: exact (+2,-1,-1),
// saturating (+2,-1,-1), saturating runtime constants, exact runtime constants.
constexpr int kNumKinds = 4;
constexpr int kind_index(int circuit, int consts) {
  return circuit == kExact ? (consts == kC211 ? 0 : 3) : (consts == kC211 ? 1 : 2);
}
constexpr int kNumVariants = 8;  // circuit x consts x padded-rows
constexpr int variant_index(int circuit, int consts, bool pad) {
  return (circuit * 2 + consts) * 2 + (pad ? 1 : 0);
}

// Arguments of the sweep kernel (one struct, passed by value).
struct SweepArgs {
  const uint2* Xp;   // [G][m] (+kXBackPad) query planes {H, L}
  const uint2* Yp;   // points at Y plane 0 of group 0: [G][n], padded both sides
  uint32_t* Mpart;   // [G][L][S] per-lane partial maxima (bit-sliced)
  int64_t G;         // 32-pair groups
  int m, n;          // query rows (m <= L*R), target columns
  int64_t streams;   // number of group streams (one per L lanes)
  int64_t base;      // groups per stream: base or base+1
  int64_t rem;       //   (the first rem streams get base+1; planes / multi-warp /
                     //   striped kernels: contiguous ranges; the fused kernel:
                     //   stream st takes groups st, st + streams, ...)
  int64_t steps;     // wavefront steps = (base + (rem>0)) * stripes * n + L
  // long-query (striped) kernel only
  // fused single-warp kernel: the caller's raw codes (query rows m, target
  // rows n, after the R17 swap), u8 or 2-bit packed
  const uint8_t* qraw;
  const uint8_t* traw;
  int64_t qstride, tstride;  // bytes per row
  int64_t P;                 // pairs (rows of qraw / traw)
  int packed2;
  uint32_t* flags;           // sticky error flags (bad base codes)
  // threshold mode (bpbc_sw_filter_batch): bits of the compared threshold as
  // all-ones / all-zeros masks (tau + g for the exact circuit, tau otherwise)
  uint32_t tmask[16];
  int stripes;          // row stripes of kStripeRows per group (1 = short kernel)
  uint32_t* bnd;        // [streams][n][SP] stripe boundary rows
  const uint32_t* bzero;  // 16 zero words
  // Wrap-around schedule (fused single-warp kernel, L = 32, n % 32 == 0;
  // DESIGN.md 6.2): stream k owns the columns [k span, (k+1) span) of the
  // concatenation of all groups' columns (group g, column j -> g n + j),
  // processed as head piece -> whole groups -> tail piece; a group split
  // between two streams moves its whole warp state (a snapshot) through
  // `snap` once the earlier stream has finished its head.
  int wrap;             // 1: wrap-around schedule (streams = ceil(G n / span))
  int64_t span;         // columns per stream (multiple of 32, >= n)
  uint32_t* snap;       // [streams][kSnapWords][32] warp-state snapshots
  uint32_t* snap_flag;  // [streams] 1 once snapshot k is written (zeroed per call)
  // Host-streamed inputs (bpbc_sw_score_batch_host): *progress = waves the
  // copy stream has completed; nullptr = inputs resident.  Group-granular
  // fused kernel: wave h = the h-th group of every stream (groups
  // [h streams, (h+1) streams)).  Wrap-around kernel: wave 0 = every query
  // row + columns [0, blk_first) of every stream's copy timeline, wave i > 0
  // = columns [blk_first + (i-1) blk_rest, blk_first + i blk_rest).
  const uint32_t* progress;
  int64_t blk_first, blk_rest;
};

// Words of one lane's warp-state snapshot (wrap-around schedule): R rows x S
// planes of scores, S planes of the diagonal input, S planes of running max
// (or the threshold flag word).
__host__ __device__ constexpr int snap_words(int R, int S) { return (R + 2) * S; }
// The wrap-around schedule's groups bound (above it the group-granular split
// wastes < 1 %); snapshot slots are reserved for at most kWrapMaxStreams.
constexpr int64_t kWrapMaxGroups = 8192;
constexpr int64_t kWrapMaxStreams = 4096;

// Long queries: stripes of kStripeR rows per lane x 32 lanes (R = 2 stripes
// were measured 1.7x slower at C5).
constexpr int kStripeR = 4;
constexpr int kStripeRows = 32 * kStripeR;
// Multi-warp groups (sw_sweep_mw_kernel): (R rows per lane, W warps per group)
// (R = 2 variants splitting 128-row groups over two warps were measured
// slower than one R = 4 warp and removed.)
constexpr int kNumMw = 3;
constexpr int kMwR[kNumMw] = {4, 4, 4};
constexpr int kMwW[kNumMw] = {2, 4, 3};
// Groups per block of the multi-warp kernel: blocks hold a multiple of 4
// warps so the block's warps cover the SM's four schedulers evenly (warp w of
// a block issues from SMSP w % 4: 2- or 3-warp blocks left SMSPs idle).
__host__ __device__ constexpr int mw_groups_per_block(int W) { return W % 4 == 0 ? 1 : W % 2 == 0 ? 2 : 4; }
// Dynamic shared memory of a multi-warp block: per group, W - 1 boundary
// rings of 128 columns x 16 words and the 2-slot query-plane ring (W = 3:
// four groups, 88 KB, above the 48 KB static limit).
constexpr int kMwRingCols = 128, kMwRingWords = 16;
__host__ __device__ constexpr int mw_smem_bytes(int R, int W) {
  return mw_groups_per_block(W) *
         ((W - 1) * kMwRingCols * kMwRingWords * 4 + W * 2 * 32 * R * 8);
}
constexpr int kMaxShortRows = 256;     // m <= 256: the short kernel
constexpr int64_t kMaxStripeStreams = 4096;
constexpr int64_t kMaxBoundaryBytes = int64_t(1) << 30;

typedef void (*SweepLaunchFn)(const SweepArgs&, const KRun&, int grid, int block,
                              cudaStream_t stream);

// Registry of compiled sweep kernels: [variant_index][rl][S - 4].
constexpr int kNumRL = 4;  // (R, L) in {(2,16), (4,16), (4,32), (8,32)}
constexpr int kRLR[kNumRL] = {2, 4, 4, 8};
constexpr int kRLL[kNumRL] = {16, 16, 32, 32};
struct SweepEntry {
  SweepLaunchFn launch;
  const void* func;  // kernel pointer for occupancy queries
};
SweepEntry sweep_entry(int circuit, int consts, bool pad, int rl, int S);

// Registration hooks, one per (score width, mode): sweep.cu is compiled once
// per pair with -DBPBC_S=S -DBPBC_MODE=M.  tab: [variant][rl][S-4] of the
// short kernel, stab: [striped kind][S-4] (0 exact (+2,-1,-1), 1 saturating
// (+2,-1,-1), 2 saturating runtime constants), ptab: [variant][rl 0..1][S-4]
// of the planes kernel, wtab: [variant][rl - 2][S-4] of the wrap-around
// kernel (L = 32 tilings), htab: [pad][rl][S-4] of the host-streamed fused
// kernel (exact (+2,-1,-1) circuit; running-max objects only).
// (weak: a development build may compile a subset of the widths, `make
// WIDTHS="9 10"`; the missing widths then report BPBC_ERR_UNSUPPORTED)
#define BPBC_DECLARE_REG(S)                                                       \
  __attribute__((weak)) void register_sweep_s##S##_m0(SweepEntry (*tab)[kNumRL][13], SweepEntry (*stab)[13],    \
                                SweepEntry (*mtab)[kNumKinds][13], SweepEntry (*ptab)[2][13], \
                                SweepEntry (*wtab)[2][13], SweepEntry (*htab)[kNumRL][13]);   \
  __attribute__((weak)) void register_sweep_s##S##_m1(SweepEntry (*tab)[kNumRL][13], SweepEntry (*stab)[13],    \
                                SweepEntry (*mtab)[kNumKinds][13], SweepEntry (*ptab)[2][13], \
                                SweepEntry (*wtab)[2][13], SweepEntry (*htab)[kNumRL][13]);
BPBC_DECLARE_REG(4)
BPBC_DECLARE_REG(5)
BPBC_DECLARE_REG(6)
BPBC_DECLARE_REG(7)
BPBC_DECLARE_REG(8)
BPBC_DECLARE_REG(9)
BPBC_DECLARE_REG(10)
BPBC_DECLARE_REG(11)
BPBC_DECLARE_REG(12)
BPBC_DECLARE_REG(13)
BPBC_DECLARE_REG(14)
BPBC_DECLARE_REG(15)
BPBC_DECLARE_REG(16)
#undef BPBC_DECLARE_REG

// pack.cu: one launch packs up to two [num_pairs][len] code arrays (query and
// target); a job with codes == nullptr is skipped.
cudaError_t launch_pack2(const uint8_t* codes_a, int len_a, uint2* planes_a,
                         const uint8_t* codes_b, int len_b, uint2* planes_b, int64_t num_pairs,
                         uint32_t* flags, int num_sms, cudaStream_t stream,
                         bool packed2 = false);
cudaError_t launch_pack(const uint8_t* codes, int64_t num_pairs, int len, uint2* planes,
                        uint32_t* flags, int num_sms, cudaStream_t stream);
// filter.cu: threshold-mode epilogue (mask words, ascending indices, count)
size_t filter_scratch_bytes(int64_t num_groups);
cudaError_t launch_filter_finish(const uint32_t* partial, int64_t num_groups, int lanes,
                                 int64_t num_pairs, uint32_t* mask, int64_t* indices,
                                 int64_t* count, void* scratch, size_t scratch_bytes,
                                 int num_sms, cudaStream_t stream);
// wordwise.cu: the wordwise 16-bit SIMD comparator (NEXT-4)
size_t wordwise_workspace_bytes(int64_t num_pairs);
cudaError_t launch_wordwise(const uint8_t* q, const uint8_t* t, int64_t P, int mq, int nt,
                            int c1, int c2, int g, int32_t* out, void* ws, int num_sms,
                            cudaStream_t st);
// extract.cu
// score = min(max(untransposed max - offset, 0), cap)
// One wave [x0, x1) of every wrap-around stream's copy timeline, gathered
// from the caller's pinned host target rows (gather.cu).
cudaError_t launch_wrap_gather(const uint8_t* host_t, uint8_t* dev_t, int64_t P, int64_t G, int n,
                               int64_t ts, int64_t span, int64_t streams, int64_t x0, int64_t x1,
                               bool packed2, int num_sms, cudaStream_t st);
// Waits (<= timeout_ns) for *flag != 0 and writes whether it was seen
// (gather.cu: the streamed host path's concurrency probe).
cudaError_t launch_probe_wait(const uint32_t* flag, uint32_t* seen, uint64_t timeout_ns,
                              cudaStream_t st);
cudaError_t launch_extract(const uint32_t* partial, int64_t num_groups, int lanes, int s,
                           int64_t num_pairs, int32_t offset, int32_t cap, int32_t* out,
                           int num_sms, cudaStream_t stream);

}  // namespace bpbc
