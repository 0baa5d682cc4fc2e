// wordwise.cu -- the wordwise comparator: the same
// Smith-Waterman DP computed with ordinary integer scores, the
// paper's "GPU wordwise" implementation (Table IV) written for
// sm_100a, so the bitwise (BPBC) path's gain can be measured on B200.
//
// B200 design: 16-bit SIMD.  One warp scores two pairs at once: every 32-bit
// register holds the same DP cell of pair A (low half) and pair B (high half),
// and the cell update uses the packed instructions VIMNMX.U16x2 (max) and
// VIADD.16x2 / IADD3 (add).  Scores are kept in offset form V = H + K0 with
// K0 = max(c2, g) so that no half ever goes negative (no borrow between
// halves):
//   nz = min(x ^ y, 1)              per half: 1 on a mismatch
//   D  = Vdiag + c1 - (c1 + c2) nz  = (diag + w) + K0           (IMAD + IADD3)
//   T  = max(Vup, Vleft) - g                                    (max, add)
//   V  = max(max(T, D), K0)         = max(0, ...) + K0          (2 max)
//   M  = max(M, D)                  running max on the diagonal term (as in
//                                   the bitwise kernel; max H = max(0, max D))
// The wavefront and streaming are the bitwise kernel's: lane l owns rows
// [lR, lR+R), works on column J = tau - l, receives the bottom row of lane
// l-1 with one shuffle per step, and walks a contiguous range of pair-pairs
// back to back.  Inputs are the caller's u8 codes (no transpose needed).
// Scores must fit 16 bits: K0 + match * min(m, n) <= 65535.
#include "bpbc_internal.cuh"

namespace bpbc {
namespace {

__device__ __forceinline__ uint32_t vmax2(uint32_t a, uint32_t b) { return __vmaxu2(a, b); }
__device__ __forceinline__ uint32_t vmin2(uint32_t a, uint32_t b) { return __vminu2(a, b); }

struct WordArgs {
  const uint8_t* q;  // [P][m] (m <= n after the role swap)
  const uint8_t* t;  // [P][n]
  uint32_t* Mpart;   // [units][32] packed partial maxima (D + K0)
  const uint8_t* dummy;  // readable bytes for lanes before their first unit
  int64_t P, units;  // units = ceil(P / 2)
  int m, n;
  int64_t streams, base, rem, steps;
  uint32_t c1pk, kpk, gpk, k0pk;  // packed c1, scalar c1 + c2, packed g, packed K0
};

template <int R, bool PAD>
__global__ void __launch_bounds__(128) wordwise_kernel(const WordArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t stream = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  if (stream >= a.streams) return;  // uniform per warp
  const int64_t Us = a.base + (stream < a.rem ? 1 : 0);
  const int64_t ub = stream * a.base + (stream < a.rem ? stream : a.rem);
  const uint32_t nz0 = lane != 0 ? 1u : 0u;  // lane 0 reads the border row (V = K0)
  const uint32_t top = lane != 0 ? 0u : a.k0pk;

  uint32_t V[R], vtop = a.k0pk, M = 0, xk[R], live[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    V[r] = a.k0pk;
    xk[r] = 0;
    live[r] = (!PAD || lane * R + r < a.m) ? 0xFFFFFFFFu : 0u;  // padded rows stay out of M
  }
  // target bytes of my current column in the unit's two pairs (a safe dummy
  // before my first unit and after my last one)
  const uint8_t* tA = a.dummy;  // 256 bytes of workspace, never more than 32 read
  const uint8_t* tB = a.dummy;
  int cnt = lane;
  int64_t ui = -1;
  for (int64_t tau = 0; tau < a.steps; ++tau) {
    const uint32_t upv = __shfl_up_sync(0xFFFFFFFFu, V[R - 1], 1) * nz0 + top;
    if (cnt == 0) {  // column 0 of my next unit (divergent, once per unit)
      if (ui >= 0 && ui < Us) a.Mpart[(ub + ui) * 32 + lane] = M;
      ++ui;
      int64_t u = ub + ui;
      u = u < a.units ? u : a.units - 1;
      const int64_t pA = 2 * u, pB = 2 * u + 1 < a.P ? 2 * u + 1 : 2 * u;
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int row = lane * R + r < a.m ? lane * R + r : a.m - 1;
        const uint32_t qa = a.q[pA * a.m + row] & 3u;  // codes > 3 read as c & 3 (R18)
        const uint32_t qb = a.q[pB * a.m + row] & 3u;
        xk[r] = qa | (qb << 16);
        V[r] = a.k0pk;
      }
      vtop = a.k0pk;
      M = 0;
      tA = a.t + pA * a.n;  // (past my last unit: re-reads a valid row)
      tB = a.t + pB * a.n;
      cnt = a.n;
    }
    --cnt;
    const uint32_t ypk = (uint32_t(__ldg(tA)) | (uint32_t(__ldg(tB)) << 16)) & 0x00030003u;
    ++tA;
    ++tB;
    uint32_t dg = vtop, u = upv;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint32_t nz = vmin2(xk[r] ^ ypk, 0x00010001u);
      const uint32_t D = dg + a.c1pk - nz * a.kpk;  // halves stay >= 0
      const uint32_t T = vmax2(u, V[r]) - a.gpk;      // >= K0 - g >= 0
      const uint32_t h = vmax2(vmax2(T, D), a.k0pk);
      M = vmax2(M, PAD ? (D & live[r]) : D);
      dg = V[r];
      V[r] = h;
      u = h;
    }
    vtop = upv;
  }
}

template <int R>
void launch_ww(const WordArgs& a, int grid, cudaStream_t st) {
  if (a.m == 32 * R)
    wordwise_kernel<R, false><<<grid, 128, 0, st>>>(a);
  else
    wordwise_kernel<R, true><<<grid, 128, 0, st>>>(a);
}

// max over the 32 lane partials of each unit -> two int32 scores.
__global__ void __launch_bounds__(256) wordwise_reduce_kernel(const uint32_t* __restrict__ Mpart,
                                                              int64_t units, int64_t P,
                                                              uint32_t k0, int32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  for (int64_t u = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; u < units; u += warps) {
    uint32_t v = Mpart[u * 32 + lane];
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) v = __vmaxu2(v, __shfl_xor_sync(0xFFFFFFFFu, v, off));
    if (lane < 2) {
      const int64_t p = 2 * u + lane;
      const int32_t d = int32_t(lane == 0 ? (v & 0xFFFFu) : (v >> 16)) - int32_t(k0);
      if (p < P) out[p] = d > 0 ? d : 0;
    }
  }
}

}  // namespace

size_t wordwise_workspace_bytes(int64_t num_pairs) {
  return size_t((num_pairs + 1) / 2) * 32 * 4 + 256;
}

cudaError_t launch_wordwise(const uint8_t* q, const uint8_t* t, int64_t P, int mq, int nt,
                            int c1, int c2, int g, int32_t* out, void* ws, int num_sms,
                            cudaStream_t st) {
  if (P <= 0) return cudaSuccess;
  const int R = (mq + 31) / 32;
  WordArgs a;
  a.q = q;
  a.t = t;
  a.Mpart = static_cast<uint32_t*>(ws);
  a.dummy = static_cast<const uint8_t*>(ws) + size_t((P + 1) / 2) * 32 * 4;
  a.P = P;
  a.units = (P + 1) / 2;
  a.m = mq;
  a.n = nt;
  const int k0 = c2 > g ? c2 : g;
  a.c1pk = uint32_t(c1) * 0x00010001u;
  a.kpk = uint32_t(c1 + c2);  // scalar: nz (0/1 per half) * kpk scales each half
  a.gpk = uint32_t(g) * 0x00010001u;
  a.k0pk = uint32_t(k0) * 0x00010001u;
  typedef void (*Fn)(const WordArgs&, int, cudaStream_t);
  static const Fn fns[9] = {nullptr, &launch_ww<1>, &launch_ww<2>, &launch_ww<3>, &launch_ww<4>,
                            &launch_ww<5>, &launch_ww<6>, &launch_ww<7>, &launch_ww<8>};
  static const void* funcs[9] = {nullptr,
                                 (const void*)&wordwise_kernel<1, true>, (const void*)&wordwise_kernel<2, true>,
                                 (const void*)&wordwise_kernel<3, true>, (const void*)&wordwise_kernel<4, true>,
                                 (const void*)&wordwise_kernel<5, true>, (const void*)&wordwise_kernel<6, true>,
                                 (const void*)&wordwise_kernel<7, true>, (const void*)&wordwise_kernel<8, true>};
  if (R < 1 || R > 8) return cudaErrorInvalidValue;
  int nb = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, funcs[R], 128, 0);
  if (e != cudaSuccess) return e;
  if (nb < 1) nb = 1;
  const int64_t cap = int64_t(num_sms) * nb * 4;
  a.streams = a.units < cap ? a.units : cap;
  a.base = a.units / a.streams;
  a.rem = a.units % a.streams;
  a.steps = (a.base + (a.rem > 0 ? 1 : 0)) * int64_t(nt) + 32;
  const int grid = int((a.streams + 3) / 4);
  e = cudaMemsetAsync(const_cast<uint8_t*>(a.dummy), 0, 256, st);  // read by idle lanes
  if (e != cudaSuccess) return e;
  fns[R](a, grid, st);
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  int64_t rgrid = (a.units + 7) / 8;
  if (rgrid > int64_t(num_sms) * 8) rgrid = int64_t(num_sms) * 8;
  wordwise_reduce_kernel<<<int(rgrid), 256, 0, st>>>(a.Mpart, a.units, P, uint32_t(k0), out);
  return cudaGetLastError();
}

}  // namespace bpbc
