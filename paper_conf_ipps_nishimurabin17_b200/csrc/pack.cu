// pack.cu -- W2B: wordwise base codes -> bit-transpose planes (P:L89-184,
// Step 2 of P:L356).
//
// The paper transposes 32x32 bit blocks with a swap/copy network (Fig. 1,
// Lemma 1, Table I: 127 logic ops per 32 2-bit characters).  On sm_100a the
// warp vote unit does a 32-lane bit gather in ONE instruction: lane k holds a
// character of pair 32g+k and __ballot_sync(pred) returns the word whose bit
// k is lane k's predicate -- exactly X^H_i / X^L_i of P:L53.  So one warp
// handles (group g, 32 consecutive positions): each lane loads the 32 bytes
// of its pair with two 16-byte loads (one full sector per lane), the warp
// issues 2 ballots per position, and lane p stores the plane pair of
// position p (one coalesced 256-byte store per warp).  HBM-bound: 1 byte
// read + 0.25 byte written per base.
#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

__global__ void __launch_bounds__(256) pack_kernel(const uint8_t* __restrict__ codes,
                                                   int64_t num_pairs, int len,
                                                   uint2* __restrict__ planes,
                                                   uint32_t* __restrict__ flags, int64_t items,
                                                   int chunks, bool vec_ok) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  uint32_t bad = 0;
  for (int64_t it = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; it < items;
       it += warps) {
    const int64_t g = it / chunks;
    const int c0 = int(it - g * chunks) * 32;
    const int64_t pair = g * 32 + lane;
    uint32_t w[8];
    if (pair < num_pairs && vec_ok && c0 + 32 <= len) {
      const uint4* src = reinterpret_cast<const uint4*>(codes + pair * len + c0);
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
          if (pair < num_pairs && pos < len) v |= uint32_t(codes[pair * len + pos]) << (8 * bb);
        }
        w[q] = v;
      }
    }
    uint32_t myh = 0, myl = 0;
#pragma unroll
    for (int p = 0; p < 32; ++p) {
      const uint32_t byte = w[p >> 2] >> (8 * (p & 3));
      bad |= byte & 0xFCu;
      const uint32_t h = __ballot_sync(0xFFFFFFFFu, byte & 2u);
      const uint32_t l = __ballot_sync(0xFFFFFFFFu, byte & 1u);
      if (lane == p) {
        myh = h;
        myl = l;
      }
    }
    if (c0 + lane < len) planes[g * len + c0 + lane] = make_uint2(myh, myl);
  }
  if (__any_sync(0xFFFFFFFFu, bad != 0) && lane == 0) atomicOr(flags, BPBC_FLAG_BAD_BASE);
}

}  // namespace

cudaError_t launch_pack(const uint8_t* codes, int64_t num_pairs, int len, uint2* planes,
                        uint32_t* flags, int num_sms, cudaStream_t stream) {
  if (num_pairs <= 0 || len <= 0) return cudaSuccess;
  const int64_t G = (num_pairs + 31) / 32;
  const int chunks = (len + 31) / 32;
  const int64_t items = G * chunks;
  const bool vec_ok = (len % 16 == 0) && ((reinterpret_cast<uintptr_t>(codes) & 15) == 0);
  const int block = 256;
  int64_t grid = (items + 7) / 8;
  const int64_t cap = int64_t(num_sms) * 8;  // 8 blocks x 8 warps per SM, grid-stride
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  pack_kernel<<<int(grid), block, 0, stream>>>(codes, num_pairs, len, planes, flags, items,
                                              chunks, vec_ok);
  return cudaGetLastError();
}

}  // namespace bpbc
