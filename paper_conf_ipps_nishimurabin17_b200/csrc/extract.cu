// extract.cu -- max reduction over rows + B2W untranspose (P:L370, P:L184,
// Step 4 of P:L360).
//
// Input: for every 32-pair group, `lanes` bit-sliced partial maxima (one per
// sweep lane, i.e. per stripe of query rows), s planes each.  The paper
// forwards R_{k,i} down the rows and lets the bottom thread write it
// (P:L370); here each lane of the sweep wrote its own partial and one warp
// per group finishes the job:
//   1. lane j takes max_B over partials j, j+32, ...;
//   2. a 5-step xor-butterfly of bit-sliced max_B (s shuffles + 2s LOP3 per
//      step) gives every lane the group maximum M;
//   3. lane k untransposes bit k: score_k = sum_b ((M_b >> k) & 1) << b
//      (P:L184), subtracts `offset` clamped at 0 (the exact circuit's
//      partials hold max D' = max H + g, circuit.cuh finish_exact), clamps
//      to `cap`, and the warp stores 32 scores (128 B).
#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

template <int S>
__device__ __forceinline__ void vmax(uint32_t (&a)[S], const uint32_t (&b)[S]) {
  runmax<S, false>(a, b, 0u);
}

template <int S>
__global__ void __launch_bounds__(256) extract_kernel(const uint32_t* __restrict__ partial,
                                                      int64_t num_groups, int lanes,
                                                      int64_t num_pairs, int32_t offset,
                                                      int32_t cap, int32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  for (int64_t g = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; g < num_groups;
       g += warps) {
    uint32_t M[S];
#pragma unroll
    for (int i = 0; i < S; ++i) M[i] = 0;
    const uint32_t* src = partial + g * int64_t(lanes) * S;
    for (int j = lane; j < lanes; j += 32) {
      uint32_t v[S];
#pragma unroll
      for (int i = 0; i < S; ++i) v[i] = src[int64_t(j) * S + i];
      vmax<S>(M, v);
    }
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
      uint32_t v[S];
#pragma unroll
      for (int i = 0; i < S; ++i) v[i] = __shfl_xor_sync(0xFFFFFFFFu, M[i], off);
      vmax<S>(M, v);
    }
    int32_t score = 0;
#pragma unroll
    for (int i = 0; i < S; ++i) score |= int32_t((M[i] >> lane) & 1u) << i;
    score = score > offset ? score - offset : 0;
    score = score < cap ? score : cap;
    const int64_t p = g * 32 + lane;
    if (p < num_pairs) out[p] = score;
  }
}

template <int S>
void launch_s(const uint32_t* partial, int64_t G, int lanes, int64_t P, int32_t offset,
              int32_t cap, int32_t* out, int grid, cudaStream_t st) {
  extract_kernel<S><<<grid, 256, 0, st>>>(partial, G, lanes, P, offset, cap, out);
}

}  // namespace

cudaError_t launch_extract(const uint32_t* partial, int64_t num_groups, int lanes, int s,
                           int64_t num_pairs, int32_t offset, int32_t cap, int32_t* out,
                           int num_sms, cudaStream_t stream) {
  if (num_groups <= 0) return cudaSuccess;
  int64_t grid = (num_groups + 7) / 8;
  const int64_t lim = int64_t(num_sms) * 8;
  if (grid > lim) grid = lim;
  typedef void (*Fn)(const uint32_t*, int64_t, int, int64_t, int32_t, int32_t, int32_t*, int,
                     cudaStream_t);
  static const Fn table[17] = {nullptr,     &launch_s<1>,  &launch_s<2>,  &launch_s<3>,
                               &launch_s<4>,  &launch_s<5>,  &launch_s<6>,  &launch_s<7>,
                               &launch_s<8>,  &launch_s<9>,  &launch_s<10>, &launch_s<11>,
                               &launch_s<12>, &launch_s<13>, &launch_s<14>, &launch_s<15>,
                               &launch_s<16>};
  if (s < 1 || s > 16) return cudaErrorInvalidValue;
  table[s](partial, num_groups, lanes, num_pairs, offset, cap, out, int(grid), stream);
  return cudaGetLastError();
}

}  // namespace bpbc
