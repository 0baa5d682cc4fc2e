// gather.cu -- host -> device gather of one wave of the wrap-around
// schedule's copy timelines (bpbc_sw_score_batch_host).
//
// With the wrap-around schedule stream k of the sweep reads
// its target columns in the order of its "copy timeline": the head piece of
// group gz (columns [0, rb)), the whole groups in between, then the tail of
// group ga from column ra - 32.  A wave is the timeline range [x0, x1) of
// EVERY stream: up to ~3 pieces of 32 rows each per stream, i.e. thousands
// of small 2D regions per wave.  One launch of this kernel moves them all,
// reading the caller's PINNED host buffer directly over PCIe (mapped
// memory, unified addressing) with 16-byte (u8) or 8-byte (2-bit packed)
// loads: one block per sweep stream, which derives its own pieces from
// (span, n, G) exactly as the sweep does.  It runs on the copy stream beside
// the sweep (1 block per SM of 128 threads leaves room on every SM).
#include <stdint.h>

#include <type_traits>

#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

template <int VB>  // vector bytes: 16 (u8 rows) or 8 (2-bit packed rows)
__global__ void __launch_bounds__(256) wrap_gather_kernel(const uint8_t* __restrict__ host_t,
                                                          uint8_t* __restrict__ dev_t, int64_t P,
                                                          int64_t G, int n, int64_t ts,
                                                          int64_t span, int64_t streams,
                                                          int64_t x0, int64_t x1, int packed2) {
  using V = typename std::conditional<VB == 16, uint4, uint2>::type;
  const int64_t tot = G * n;
  for (int64_t k = blockIdx.x; k < streams; k += gridDim.x) {
    const int64_t V0 = k * span, V1 = V0 + span < tot ? V0 + span : tot;
    const int64_t ga = V0 / n, gz = V1 / n;
    const int64_t ra = V0 - ga * n, rb = V1 - gz * n;
    const int64_t g1 = ga + (ra > 0 ? 1 : 0), nf = gz - g1;
    // the pieces of this stream's timeline: (group, first column, timeline
    // start, columns); whole groups are one contiguous timeline run
    for (int part = 0; part < 3; ++part) {
      int64_t t0, len;
      if (part == 0) {  // head [0, rb) of group gz
        if (rb == 0) continue;
        t0 = 0;
        len = rb;
      } else if (part == 1) {  // whole groups g1 .. g1 + nf - 1
        if (nf <= 0) continue;
        t0 = rb;
        len = nf * n;
      } else {  // tail [ra - 32, n) of group ga
        if (ra == 0) continue;
        t0 = rb + nf * n;
        len = n - ra + 32;
      }
      const int64_t a0 = t0 > x0 ? t0 : x0;
      const int64_t a1 = t0 + len < x1 ? t0 + len : x1;
      if (a0 >= a1) continue;
      // walk [a0, a1) group by group (only the whole-groups part spans several)
      int64_t t = a0;
      while (t < a1) {
        int64_t gg, c_from, c_end;
        if (part == 0) {
          gg = gz;
          c_from = t - t0;
          c_end = rb;
        } else if (part == 1) {
          const int64_t j = (t - t0) / n;
          gg = g1 + j;
          c_from = (t - t0) - j * n;
          c_end = n;
        } else {
          gg = ga;
          c_from = ra - 32 + (t - t0);
          c_end = n;
        }
        const int64_t c_to = c_from + (a1 - t) < c_end ? c_from + (a1 - t) : c_end;
        const int64_t rows = P - gg * 32 < 32 ? P - gg * 32 : 32;
        // (column ranges are multiples of 32: whole vectors of either layout)
        const int64_t b0 = packed2 ? c_from / 4 : c_from;
        const int64_t b1 = packed2 ? (c_to + 3) / 4 : c_to;
        const int64_t nv = (b1 - b0) / VB;
        const int64_t base = gg * 32 * ts + b0;
        for (int64_t i = threadIdx.x; i < rows * nv; i += blockDim.x) {
          const int64_t r = i / nv, v = i - r * nv;
          const int64_t off = base + r * ts + v * VB;
          *reinterpret_cast<V*>(dev_t + off) = *reinterpret_cast<const V*>(host_t + off);
        }
        t += c_to - c_from;
      }
    }
  }
}

}  // namespace

cudaError_t launch_wrap_gather(const uint8_t* host_t, uint8_t* dev_t, int64_t P, int64_t G, int n,
                               int64_t ts, int64_t span, int64_t streams, int64_t x0, int64_t x1,
                               bool packed2, int num_sms, cudaStream_t st) {
  const int grid = int(streams < int64_t(num_sms) * 4 ? streams : int64_t(num_sms) * 4);
  if (packed2)
    wrap_gather_kernel<8><<<grid, 256, 0, st>>>(host_t, dev_t, P, G, n, ts, span, streams, x0, x1, 1);
  else
    wrap_gather_kernel<16><<<grid, 256, 0, st>>>(host_t, dev_t, P, G, n, ts, span, streams, x0, x1, 0);
  return cudaGetLastError();
}

}  // namespace bpbc

// ---------------------------------------------------------------------------
// Concurrency probe of the streamed host path: one thread waits (at most
// timeout_ns) for *flag to become non-zero, written by the copy stream AFTER
// this kernel's launch, and records in *seen whether it did.  Under a
// launch-serialising environment (a kernel profiler, CUDA_LAUNCH_BLOCKING)
// it times out and the host path takes its chunked form instead.
namespace bpbc {
namespace {
__global__ void probe_wait_kernel(const uint32_t* flag, uint32_t* seen, uint64_t timeout_ns) {
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  uint32_t v = 0;
  do {
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    if (v != 0) break;
    __nanosleep(1000);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < timeout_ns);
  *seen = v != 0 ? 1u : 0u;
}
}  // namespace

cudaError_t launch_probe_wait(const uint32_t* flag, uint32_t* seen, uint64_t timeout_ns,
                              cudaStream_t st) {
  probe_wait_kernel<<<1, 1, 0, st>>>(flag, seen, timeout_ns);
  return cudaGetLastError();
}
}  // namespace bpbc
