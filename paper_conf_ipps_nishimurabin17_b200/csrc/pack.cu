// pack.cu -- W2B: wordwise base codes -> bit-transpose planes (P:L89-184,
// Step 2 of P:L356).
//
// The paper transposes 32x32 bit blocks on each thread with a swap/copy
// network (Fig. 1, Lemma 1, Table I: 127 logic ops per 32 2-bit characters).
// Here a warp transposes ACROSS its lanes with the transpose of
// transpose.cuh (shared with the fused sweep).  One warp handles one
// (group g, 128-position chunk) item as four 32-position quarters:
//   1. the warp reads the item's 32 rows x 128 code bytes with coalesced
//      16-byte loads (4 rows per instruction) into a shared stage, and lane
//      k takes pair 32g+k's 128 bytes from it (ragged items: every lane
//      loads its own row; 2-bit packed input: 4 x 8 B per lane);
//   2. per quarter: tr_fold_u8 folds the 32 bytes into two words H, L (the
//      high / low code bits of the 32 positions, in the fixed bit order
//      tr_pos_u8), tr_butterfly transposes the warp's 32x32 bit matrices, so
//      lane p holds the words whose bit k is pair 32g+k's code bit at
//      position tr_pos(p) -- exactly X^H_i / X^L_i of P:L53;
//   3. lane p stores uint2(H, L) to planes[g][c0 + tr_pos(p)]: the warp
//      writes one contiguous 256-byte block per quarter.
// HBM-bound: 1 byte read + 0.25 byte written per base.  Base codes > 3 are
// read as c & 3 and raise the sticky bad-base flag (R18).
#include "bpbc_internal.cuh"
#include "transpose.cuh"

namespace bpbc {
namespace {

constexpr int kPackQ = 4;  // 32-position quarters per warp item

struct PackJob {
  const uint8_t* codes;  // [num_pairs][stride]: u8 codes, or 2-bit packed
  uint2* planes;         // [G][len]
  int len;
  int64_t stride;        // bytes per row: len (u8) or ceil(len / 4) (packed2)
  int chunks;            // ceil(len / 128): an item covers 128 positions
  int64_t items;         // G * chunks
  bool packed2;          // 4 bases per byte (bpbc_sw_score_batch_packed2)
};

// Coalesced staging of one u8 item: the 32 rows x 128 bytes of group g at
// columns [c0, c0 + 128) are read 4 rows per instruction (8 lanes x 16 B per
// row: 4 cache lines per load instead of 32 when every lane reads its own
// row -- the L1 data pipe, not DRAM, limited that form) into a per-warp
// shared buffer with 144-byte rows (conflict-free 16-byte reads below).
constexpr int kStageRow = 32 * kPackQ + 16;

__global__ void __launch_bounds__(256) pack_kernel(const PackJob j0, const PackJob j1,
                                                   int64_t num_pairs,
                                                   uint32_t* __restrict__ flags) {
  __shared__ __align__(16) uint8_t stage[8][32 * kStageRow];  // [warp][row][byte]
  const int lane = threadIdx.x & 31;
  uint8_t* st = stage[threadIdx.x >> 5];
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  const int64_t total = j0.items + j1.items;
  uint32_t bad = 0;
  for (int64_t it = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; it < total;
       it += warps) {
    const bool second = it >= j0.items;  // warp-uniform
    const PackJob& J = second ? j1 : j0;
    const uint32_t li = uint32_t(second ? it - j0.items : it);  // < 2^31 (host check)
    const uint32_t gq = li / uint32_t(J.chunks);
    const int64_t g = gq;
    const int c0 = int(li - gq * uint32_t(J.chunks)) * (32 * kPackQ);
    const int64_t pair = g * 32 + lane;
    uint2* row = J.planes + g * J.len;
    if (J.packed2) {  // warp-uniform
      uint32_t w[kPackQ][2];
#pragma unroll
      for (int h = 0; h < kPackQ; ++h) {
        w[h][0] = w[h][1] = 0u;
        if (c0 + 32 * h < J.len) tr_load_p2(J.codes, J.stride, J.len, pair, num_pairs, c0 + 32 * h, w[h]);
      }
      const int pos = tr_pos_packed2(lane);
#pragma unroll
      for (int h = 0; h < kPackQ; ++h) {
        if (c0 + 32 * h >= J.len) break;  // warp-uniform
        uint32_t H, L;
        tr_fold_packed2(w[h][0], w[h][1], H, L);
        tr_butterfly(H, L, lane);
        if (c0 + 32 * h + pos < J.len) row[c0 + 32 * h + pos] = make_uint2(H, L);
      }
      continue;
    }
    uint32_t w[kPackQ][8];
    // whole aligned item of full rows: coalesced loads through the stage
    const bool whole = c0 + 32 * kPackQ <= J.len && (g + 1) * 32 <= num_pairs &&
                       (J.stride & 15) == 0 && (reinterpret_cast<uintptr_t>(J.codes) & 15) == 0;
    if (whole) {  // warp-uniform
      const uint8_t* src = J.codes + (g * 32) * J.stride + c0;
      uint4 v[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)  // rows 4i + lane / 8, bytes 16 (lane % 8)
        v[i] = __ldcs(reinterpret_cast<const uint4*>(src + (4 * i + (lane >> 3)) * J.stride) +
                      (lane & 7));
      __syncwarp();  // the previous item's stage reads -> these writes
#pragma unroll
      for (int i = 0; i < 8; ++i)
        *reinterpret_cast<uint4*>(st + (4 * i + (lane >> 3)) * kStageRow + 16 * (lane & 7)) = v[i];
      __syncwarp();
#pragma unroll
      for (int h = 0; h < kPackQ; ++h) {  // my row (pair 32g + lane), quarter h
        const uint4 a = *reinterpret_cast<const uint4*>(st + lane * kStageRow + 32 * h);
        const uint4 b = *reinterpret_cast<const uint4*>(st + lane * kStageRow + 32 * h + 16);
        w[h][0] = a.x; w[h][1] = a.y; w[h][2] = a.z; w[h][3] = a.w;
        w[h][4] = b.x; w[h][5] = b.y; w[h][6] = b.z; w[h][7] = b.w;
      }
    } else {
      // ragged / unaligned items: every lane loads its own row (all four
      // quarters before any is used)
#pragma unroll
      for (int h = 0; h < kPackQ; ++h) {
#pragma unroll
        for (int q = 0; q < 8; ++q) w[h][q] = 0u;
        if (c0 + 32 * h < J.len) tr_load_u8(J.codes, J.stride, J.len, pair, num_pairs, c0 + 32 * h, w[h]);
      }
    }
    const int pos = tr_pos_u8(lane);
#pragma unroll
    for (int h = 0; h < kPackQ; ++h) {
      if (c0 + 32 * h >= J.len) break;  // warp-uniform
      uint32_t H, L;
      tr_fold_u8(w[h], H, L, bad);
      tr_butterfly(H, L, lane);
      if (c0 + 32 * h + pos < J.len) row[c0 + 32 * h + pos] = make_uint2(H, L);
    }
  }
  if (__any_sync(0xFFFFFFFFu, bad != 0) && lane == 0) atomicOr(flags, BPBC_FLAG_BAD_BASE);
}

PackJob make_job(const uint8_t* codes, int64_t num_pairs, int len, uint2* planes, bool packed2) {
  PackJob J;
  J.codes = codes;
  J.planes = planes;
  J.len = len > 0 ? len : 1;
  J.packed2 = packed2;
  J.stride = packed2 ? (J.len + 3) / 4 : J.len;
  J.chunks = (J.len + 32 * kPackQ - 1) / (32 * kPackQ);
  J.items = (codes && len > 0) ? (num_pairs + 31) / 32 * J.chunks : 0;
  return J;
}

}  // namespace

cudaError_t launch_pack2(const uint8_t* codes_a, int len_a, uint2* planes_a,
                         const uint8_t* codes_b, int len_b, uint2* planes_b, int64_t num_pairs,
                         uint32_t* flags, int num_sms, cudaStream_t stream, bool packed2) {
  if (num_pairs <= 0) return cudaSuccess;
  const PackJob a = make_job(codes_a, num_pairs, len_a, planes_a, packed2);
  const PackJob b = make_job(codes_b, num_pairs, len_b, planes_b, packed2);
  const int64_t items = a.items + b.items;
  if (items == 0) return cudaSuccess;
  if (a.items >= (int64_t(1) << 31) || b.items >= (int64_t(1) << 31)) return cudaErrorInvalidValue;
  const int block = 256;
  int64_t grid = (items + 7) / 8;
  const int64_t cap = int64_t(num_sms) * 8;  // 8 blocks x 8 warps per SM, grid-stride
  if (grid > cap) grid = cap;
  pack_kernel<<<int(grid), block, 0, stream>>>(a, b, num_pairs, flags);
  return cudaGetLastError();
}

cudaError_t launch_pack(const uint8_t* codes, int64_t num_pairs, int len, uint2* planes,
                        uint32_t* flags, int num_sms, cudaStream_t stream) {
  if (num_pairs <= 0 || len <= 0) return cudaSuccess;
  return launch_pack2(codes, len, planes, nullptr, 0, nullptr, num_pairs, flags, num_sms, stream,
                      false);
}

}  // namespace bpbc
