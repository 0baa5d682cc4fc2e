// transpose.cuh -- the warp bit transpose (W2B) shared by the
// standalone pack kernel (pack.cu) and the fused sweep (sweep.cu).
//
// A warp turns 32 code bytes of each of its 32 lanes (lane k = pair k of a
// 32-pair group, 32 consecutive positions) into the bit planes of those 32
// positions (bit k of a word = pair k):
//   1. fold: the 32 bytes become two words H, L holding the high / low code
//      bit of all 32 positions (3 integer multiply-adds per 16 bytes on the
//      FMA pipe, one shift and one LOP3 per word); the bit order inside H/L is
//      a fixed permutation of the positions (tr_pos_u8);
//   2. a 5-stage butterfly across the warp (per stage and plane: shfl_xor,
//      funnel rotate, one LOP3) transposes the two 32x32 bit matrices, so
//      lane p ends with the plane words of position tr_pos_*(p).
// 2-bit packed input (4 bases per byte, base i in bits 2i of the row's
// little-endian words) needs no fold: tr_fold_packed2.
#pragma once
#include <stdint.h>

namespace bpbc {

__device__ __forceinline__ uint32_t tr_mad_lo(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t r;  // integer multiply-add: issues on the FMA pipe, not the ALU pipe
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  return r;
}

// Position held by bit i of the folded words (and, after the transpose, by
// lane i): t = w0 + 4 w1 + 16 w2 + 64 w3 puts code(4q+b) in bits 8b+2q,
// 8b+2q+1; u does the same for positions 16..31; H takes t's odd bits and
// u's odd bits shifted to the even slots, L likewise for the low bits.
__device__ __forceinline__ int tr_pos_u8(int i) {
  const int b = i >> 3, q = (i >> 1) & 3;
  return (i & 1) ? 4 * q + b : 16 + 4 * q + b;
}
// Same for 2-bit packed input: H takes word A's odd bits (positions 0..15)
// and word B's odd bits shifted to the even slots (16..31).
__device__ __forceinline__ int tr_pos_packed2(int i) { return (i & 1) ? (i >> 1) : 16 + (i >> 1); }

// Fold 32 code bytes (w[q] byte b = position 4q + b) into H / L; codes are
// read as c & 3 (R18); returns the bits > 3 seen in `bad`.
__device__ __forceinline__ void tr_fold_u8(uint32_t (&w)[8], uint32_t& H, uint32_t& L,
                                           uint32_t& bad) {
  bad |= (w[0] | w[1] | w[2] | w[3] | w[4] | w[5] | w[6] | w[7]) & 0xFCFCFCFCu;
#pragma unroll
  for (int q = 0; q < 8; ++q) w[q] &= 0x03030303u;
  const uint32_t t = tr_mad_lo(w[3], 64u, tr_mad_lo(w[2], 16u, tr_mad_lo(w[1], 4u, w[0])));
  const uint32_t u = tr_mad_lo(w[7], 64u, tr_mad_lo(w[6], 16u, tr_mad_lo(w[5], 4u, w[4])));
  H = (t & 0xAAAAAAAAu) | ((u >> 1) & 0x55555555u);
  L = ((t << 1) & 0xAAAAAAAAu) | (u & 0x55555555u);
}

// 16 packed bases in A (positions 0..15) and B (16..31) -> H / L.
__device__ __forceinline__ void tr_fold_packed2(uint32_t A, uint32_t B, uint32_t& H, uint32_t& L) {
  H = (A & 0xAAAAAAAAu) | ((B >> 1) & 0x55555555u);
  L = ((A << 1) & 0xAAAAAAAAu) | (B & 0x55555555u);
}

// 32x32 bit transpose of H and L across the warp: stage j swaps the
// off-diagonal j x j blocks between lanes l and l^j.  Lane l keeps its bits
// where keep = 1 and takes the partner's word rotated by j into the others.
__device__ __forceinline__ void tr_butterfly(uint32_t& H, uint32_t& L, int lane) {
#pragma unroll
  for (int s = 0; s < 5; ++s) {
    const int j = 16 >> s;
    const uint32_t m = s == 0 ? 0x0000FFFFu : s == 1 ? 0x00FF00FFu : s == 2 ? 0x0F0F0F0Fu
                     : s == 3 ? 0x33333333u : 0x55555555u;
    const uint32_t keep = (lane & j) ? ~m : m;
    const uint32_t rot = (lane & j) ? j : 32 - j;
    const uint32_t ph = __shfl_xor_sync(0xFFFFFFFFu, H, j);
    const uint32_t pl = __shfl_xor_sync(0xFFFFFFFFu, L, j);
    const uint32_t yh = __funnelshift_r(ph, ph, rot);  // rotate right by rot
    const uint32_t yl = __funnelshift_r(pl, pl, rot);
    H = (H & keep) | (yh & ~keep);
    L = (L & keep) | (yl & ~keep);
  }
}

// Raw words of positions [c0, c0 + 32) of one row of a raw input (`stride`
// bytes per row, `len` positions): zeros past the row end and for rows >=
// nrows.  u8 codes: 8 words (byte b of w[q] = position 4q + b), two 16-byte
// streaming loads when the row segment is 16-byte aligned and whole; 2-bit
// packed: 2 words (positions 0..15, 16..31), one 8-byte load when aligned.
__device__ __forceinline__ void tr_load_u8(const uint8_t* base, int64_t stride, int len,
                                           int64_t row, int64_t nrows, int c0, uint32_t (&w)[8]) {
#pragma unroll
  for (int q = 0; q < 8; ++q) w[q] = 0u;
  if (row < nrows) {
    const uint8_t* p = base + row * stride + c0;
    if (c0 + 32 <= len && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
      const uint4 a = __ldcs(reinterpret_cast<const uint4*>(p));
      const uint4 b = __ldcs(reinterpret_cast<const uint4*>(p) + 1);
      w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w;
      w[4] = b.x; w[5] = b.y; w[6] = b.z; w[7] = b.w;
    } else {
#pragma unroll
      for (int q = 0; q < 8; ++q)
#pragma unroll
        for (int bb = 0; bb < 4; ++bb)
          if (c0 + 4 * q + bb < len) w[q] |= uint32_t(p[4 * q + bb]) << (8 * bb);
    }
  }
}
__device__ __forceinline__ void tr_load_p2(const uint8_t* base, int64_t stride, int len,
                                           int64_t row, int64_t nrows, int c0, uint32_t (&w)[2]) {
  w[0] = w[1] = 0u;
  if (row < nrows) {
    const uint8_t* p = base + row * stride + c0 / 4;
    if (c0 + 32 <= len && ((reinterpret_cast<uintptr_t>(p) & 7) == 0)) {
      const uint2 v = *reinterpret_cast<const uint2*>(p);
      w[0] = v.x;
      w[1] = v.y;
    } else {
#pragma unroll
      for (int q = 0; q < 2; ++q)
#pragma unroll
        for (int bb = 0; bb < 4; ++bb)
          if (c0 + 16 * q + 4 * bb < len) w[q] |= uint32_t(p[4 * q + bb]) << (8 * bb);
    }
  }
}

// The (pre-butterfly) H / L words of positions [c0, c0 + 32) of one row of a
// raw input (u8 codes or 2-bit packed).
__device__ __forceinline__ void tr_load_fold(const uint8_t* base, int64_t stride, int len,
                                             int64_t row, int64_t nrows, int c0, bool packed2,
                                             uint32_t& H, uint32_t& L, uint32_t& bad) {
  if (packed2) {
    uint32_t w[2];
    tr_load_p2(base, stride, len, row, nrows, c0, w);
    tr_fold_packed2(w[0], w[1], H, L);
    return;
  }
  uint32_t w[8];
  tr_load_u8(base, stride, len, row, nrows, c0, w);
  tr_fold_u8(w, H, L, bad);
}

}  // namespace bpbc
