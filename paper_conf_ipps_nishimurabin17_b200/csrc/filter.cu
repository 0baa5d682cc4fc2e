// filter.cu -- epilogue of the threshold filter (NEXT-2): the paper's use
// case of flagging pairs whose maximum score exceeds a threshold tau so that
// only those are re-aligned (with traceback) on the CPU.
//
// The sweep in threshold mode leaves one flag word per (group, stripe, lane):
// bit k = 1 iff some cell of pair 32g+k in that lane's rows exceeded tau.
//   1. filter_mask_kernel: one warp per group ORs the lane words
//      (__reduce_or_sync), clears the bits of pairs past num_pairs, stores the
//      group's mask word (bit k = pair 32g+k) and its popcount;
//   2. an exclusive prefix sum of the popcounts (CUB DeviceScan, a library
//      primitive) gives each group's first output slot;
//   3. filter_compact_kernel: lane k of the group's warp writes index 32g+k
//      at slot offset[g] + popc(mask & ((1 << k) - 1)) -- ascending order --
//      and the last group writes the total count.
#include <cub/device/device_scan.cuh>

#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

__global__ void __launch_bounds__(256) filter_mask_kernel(const uint32_t* __restrict__ partial,
                                                          int64_t num_groups, int lanes,
                                                          int64_t num_pairs,
                                                          uint32_t* __restrict__ mask,
                                                          int64_t* __restrict__ counts) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  for (int64_t g = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; g < num_groups;
       g += warps) {
    uint32_t w = 0;
    for (int j = lane; j < lanes; j += 32) w |= partial[g * lanes + j];
    w = __reduce_or_sync(0xFFFFFFFFu, w);
    const int64_t left = num_pairs - g * 32;
    if (left < 32) w &= (1u << left) - 1u;
    if (lane == 0) {
      mask[g] = w;
      if (counts) counts[g] = __popc(w);
    }
  }
}

__global__ void __launch_bounds__(256) filter_compact_kernel(const uint32_t* __restrict__ mask,
                                                             const int64_t* __restrict__ offsets,
                                                             int64_t num_groups,
                                                             int64_t* __restrict__ indices,
                                                             int64_t* __restrict__ count) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  for (int64_t g = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; g < num_groups;
       g += warps) {
    const uint32_t w = mask[g];
    if (indices && ((w >> lane) & 1u))
      indices[offsets[g] + __popc(w & ((1u << lane) - 1u))] = g * 32 + lane;
    if (count && g == num_groups - 1 && lane == 0) *count = offsets[g] + __popc(w);
  }
}

int grid_for(int64_t warps_needed, int num_sms) {
  int64_t grid = (warps_needed + 7) / 8;
  const int64_t lim = int64_t(num_sms) * 8;
  if (grid > lim) grid = lim;
  return grid < 1 ? 1 : int(grid);
}

}  // namespace

size_t filter_scratch_bytes(int64_t num_groups) {
  size_t temp = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, temp, static_cast<const int64_t*>(nullptr),
                                static_cast<int64_t*>(nullptr), num_groups);
  // counts[G], offsets[G], CUB temp storage; 256-byte aligned sections
  const size_t a = (size_t(num_groups) * 8 + 255) & ~size_t(255);
  return 2 * a + ((temp + 255) & ~size_t(255));
}

cudaError_t launch_filter_finish(const uint32_t* partial, int64_t num_groups, int lanes,
                                 int64_t num_pairs, uint32_t* mask, int64_t* indices,
                                 int64_t* count, void* scratch, size_t scratch_bytes,
                                 int num_sms, cudaStream_t stream) {
  if (num_groups <= 0) return cudaSuccess;
  const bool compact = indices || count;
  const size_t a = (size_t(num_groups) * 8 + 255) & ~size_t(255);
  int64_t* counts = compact ? static_cast<int64_t*>(scratch) : nullptr;
  int64_t* offsets =
      compact ? reinterpret_cast<int64_t*>(static_cast<uint8_t*>(scratch) + a) : nullptr;
  const int grid = grid_for(num_groups, num_sms);
  filter_mask_kernel<<<grid, 256, 0, stream>>>(partial, num_groups, lanes, num_pairs, mask,
                                                counts);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess || !compact) return e;
  void* temp = static_cast<uint8_t*>(scratch) + 2 * a;
  size_t temp_bytes = scratch_bytes > 2 * a ? scratch_bytes - 2 * a : 0;
  e = cub::DeviceScan::ExclusiveSum(temp, temp_bytes, counts, offsets, num_groups, stream);
  if (e != cudaSuccess) return e;
  filter_compact_kernel<<<grid, 256, 0, stream>>>(mask, offsets, num_groups, indices, count);
  return cudaGetLastError();
}

}  // namespace bpbc
