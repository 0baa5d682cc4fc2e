// pack.cu -- W2B: wordwise base codes -> bit-transpose planes (P:L89-184,
// Step 2 of P:L356).
//
// The paper transposes 32x32 bit blocks on each thread with a swap/copy
// network (Fig. 1, Lemma 1, Table I: 127 logic ops per 32 2-bit characters).
// Here a warp transposes ACROSS its lanes.  One warp handles one
// (group g, 64-position chunk) item, as two 32-position halves:
//   1. lane k loads the 32 code bytes of pair 32g+k at each half (two 16-B
//      loads = one full sector per lane and half; all four loads are issued
//      before the first use);
//   2. it folds them into two words, H and L, holding the high / low code
//      bit of all 32 positions (3 integer multiply-adds per 16 bytes on the
//      FMA pipe, then one shift and one LOP3 per word).  The bit order inside
//      H/L is a fixed permutation pi of the positions (below);
//   3. a 5-stage butterfly (shfl_xor + funnel rotate + one LOP3 per stage
//      and plane) transposes the 32x32 bit matrices H and L of the warp, so
//      lane p ends with the words whose bit k is pair 32g+k's code bit at
//      position pi(p) -- exactly X^H_i / X^L_i of P:L53 for i = c0 + pi(p);
//   4. lane p stores uint2(H, L) to planes[g][c0 + pi(p)]: the warp writes
//      one contiguous 256-byte block.
// HBM-bound: 1 byte read + 0.25 byte written per base; ~40 ALU lane-ops per
// 32 bases (vs ~200 for a ballot per position).  Base codes > 3 are read as
// c & 3 and raise the sticky bad-base flag (R18).
#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

__device__ __forceinline__ uint32_t mad_lo(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t r;  // integer multiply-add: issues on the FMA pipe, not the ALU pipe
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  return r;
}
__device__ __forceinline__ uint32_t rotr(uint32_t x, uint32_t r) {
  return __funnelshift_r(x, x, r);
}

// Position held by bit i of the folded words (and, after the transpose, by
// lane i): t = w0 + 4 w1 + 16 w2 + 64 w3 puts code(4q+b) in bits 8b+2q,
// 8b+2q+1; t' does the same for positions 16..31; H takes t's odd bits and
// t''s odd bits shifted to the even slots, L likewise for the low bits.
__device__ __forceinline__ int pos_of_bit(int i) {
  const int b = i >> 3, q = (i >> 1) & 3;
  return (i & 1) ? 4 * q + b : 16 + 4 * q + b;
}

// Position held by bit i for 2-bit packed input (base i of a row in bits
// 2i, 2i+1 of its little-endian words): H takes word A's odd bits (positions
// 0..15) and word B's odd bits shifted to the even slots (16..31).
__device__ __forceinline__ int pos_of_bit_packed2(int i) { return (i & 1) ? (i >> 1) : 16 + (i >> 1); }

struct PackJob {
  const uint8_t* codes;  // [num_pairs][stride]: u8 codes, or 2-bit packed
  uint2* planes;         // [G][len]
  int len;
  int64_t stride;        // bytes per row: len (u8) or ceil(len / 4) (packed2)
  int chunks;            // ceil(len / 64): an item covers 64 positions
  int64_t items;         // G * chunks
  bool vec_ok;           // rows 16-byte aligned for the vector loads
  bool packed2;          // 4 bases per byte (bpbc_sw_score_batch_packed2)
};

// 32 code bytes of one lane's pair at positions [c0, c0+32) (zeros past the
// row end or past the last pair).
__device__ __forceinline__ void load32(const PackJob& J, int64_t pair, int64_t num_pairs, int c0,
                                       uint32_t (&w)[8]) {
  if (pair < num_pairs && J.vec_ok && c0 + 32 <= J.len) {
    const uint4* src = reinterpret_cast<const uint4*>(J.codes + pair * J.len + c0);
    const uint4 a = __ldcs(src), b = __ldcs(src + 1);  // streamed once
    w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w;
    w[4] = b.x; w[5] = b.y; w[6] = b.z; w[7] = b.w;
  } else {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      uint32_t v = 0;
#pragma unroll
      for (int bb = 0; bb < 4; ++bb) {
        const int pos = c0 + q * 4 + bb;
        if (pair < num_pairs && pos < J.len) v |= uint32_t(J.codes[pair * J.len + pos]) << (8 * bb);
      }
      w[q] = v;
    }
  }
}

// 2-bit packed bases of one lane's pair, positions [c0, c0+64): 4 words, 16
// bases each (bits past the row end are never stored).
__device__ __forceinline__ void load64_packed2(const PackJob& J, int64_t pair, int64_t num_pairs,
                                               int c0, uint32_t (&w)[4]) {
  const uint8_t* row = J.codes + pair * J.stride + c0 / 4;
  if (pair < num_pairs && J.vec_ok && c0 + 64 <= J.len) {
    const uint4 a = __ldcs(reinterpret_cast<const uint4*>(row));
    w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w;
  } else {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint32_t v = 0;
#pragma unroll
      for (int bb = 0; bb < 4; ++bb) {
        const int pos = c0 + 16 * q + 4 * bb;
        if (pair < num_pairs && pos < J.len) v |= uint32_t(row[4 * q + bb]) << (8 * bb);
      }
      w[q] = v;
    }
  }
}

// Transpose the (H, L) words of one 32-position chunk across the warp and
// store lane p's result at dst (position set by the caller's bit order).
__device__ __forceinline__ void butterfly_store(uint32_t H, uint32_t L, const uint32_t (&keep)[5],
                                                const uint32_t (&rot)[5], uint2* dst, bool ok) {
  // 32x32 bit transpose across the warp: stage j swaps the off-diagonal
  // j x j blocks between lanes l and l^j.  Lane l keeps its bits where
  // keep = 1 and takes the partner's word rotated by j into the others.
#pragma unroll
  for (int s = 0; s < 5; ++s) {
    const int j = 16 >> s;
    const uint32_t yh = rotr(__shfl_xor_sync(0xFFFFFFFFu, H, j), rot[s]);
    const uint32_t yl = rotr(__shfl_xor_sync(0xFFFFFFFFu, L, j), rot[s]);
    H = (H & keep[s]) | (yh & ~keep[s]);
    L = (L & keep[s]) | (yl & ~keep[s]);
  }
  if (ok) *dst = make_uint2(H, L);
}

// Fold, transpose across the warp and store one 32-position chunk.
__device__ __forceinline__ void transpose_store(uint32_t (&w)[8], const uint32_t (&keep)[5],
                                                const uint32_t (&rot)[5], uint2* dst, bool ok,
                                                uint32_t& bad) {
  bad |= (w[0] | w[1] | w[2] | w[3] | w[4] | w[5] | w[6] | w[7]) & 0xFCFCFCFCu;
#pragma unroll
  for (int q = 0; q < 8; ++q) w[q] &= 0x03030303u;
  const uint32_t t = mad_lo(w[3], 64u, mad_lo(w[2], 16u, mad_lo(w[1], 4u, w[0])));
  const uint32_t u = mad_lo(w[7], 64u, mad_lo(w[6], 16u, mad_lo(w[5], 4u, w[4])));
  uint32_t H = (t & 0xAAAAAAAAu) | ((u >> 1) & 0x55555555u);
  uint32_t L = ((t << 1) & 0xAAAAAAAAu) | (u & 0x55555555u);
  butterfly_store(H, L, keep, rot, dst, ok);
}


__global__ void __launch_bounds__(256) pack_kernel(const PackJob j0, const PackJob j1,
                                                   int64_t num_pairs,
                                                   uint32_t* __restrict__ flags) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  const int64_t total = j0.items + j1.items;
  // per-stage lane constants of the butterfly (see transpose_store)
  uint32_t keep[5], rot[5];
#pragma unroll
  for (int s = 0; s < 5; ++s) {
    const int j = 16 >> s;
    const uint32_t m = s == 0 ? 0x0000FFFFu : s == 1 ? 0x00FF00FFu : s == 2 ? 0x0F0F0F0Fu
                     : s == 3 ? 0x33333333u : 0x55555555u;
    keep[s] = (lane & j) ? ~m : m;
    rot[s] = (lane & j) ? j : 32 - j;
  }
  const int mypos = pos_of_bit(lane);
  uint32_t bad = 0;
  for (int64_t it = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; it < total;
       it += warps) {
    const bool second = it >= j0.items;  // warp-uniform
    const PackJob& J = second ? j1 : j0;
    const uint32_t li = uint32_t(second ? it - j0.items : it);  // < 2^31 (host check)
    const uint32_t gq = li / uint32_t(J.chunks);
    const int64_t g = gq;
    const int c0 = int(li - gq * uint32_t(J.chunks)) * 64;
    const int64_t pair = g * 32 + lane;
    uint2* row = J.planes + g * J.len;
    if (J.packed2) {  // warp-uniform: 16 bytes per lane cover 64 positions
      uint32_t w[4];
      load64_packed2(J, pair, num_pairs, c0, w);
      const int p2 = pos_of_bit_packed2(lane);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (c0 + 32 * h < J.len) {  // warp-uniform
          const uint32_t A = w[2 * h], B = w[2 * h + 1];
          const uint32_t H = (A & 0xAAAAAAAAu) | ((B >> 1) & 0x55555555u);
          const uint32_t L = ((A << 1) & 0xAAAAAAAAu) | (B & 0x55555555u);
          butterfly_store(H, L, keep, rot, row + c0 + 32 * h + p2, c0 + 32 * h + p2 < J.len);
        }
      }
      continue;
    }
    // both 32-position halves are loaded before either is used (64 B per
    // lane in flight)
    uint32_t w0[8], w1[8];
    load32(J, pair, num_pairs, c0, w0);
    load32(J, pair, num_pairs, c0 + 32, w1);
    transpose_store(w0, keep, rot, row + c0 + mypos, c0 + mypos < J.len, bad);
    if (c0 + 32 < J.len)  // warp-uniform
      transpose_store(w1, keep, rot, row + c0 + 32 + mypos, c0 + 32 + mypos < J.len, bad);
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
  J.chunks = (J.len + 63) / 64;
  J.items = (codes && len > 0) ? (num_pairs + 31) / 32 * J.chunks : 0;
  J.vec_ok = (J.stride % 16 == 0) && ((reinterpret_cast<uintptr_t>(codes) & 15) == 0);
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
