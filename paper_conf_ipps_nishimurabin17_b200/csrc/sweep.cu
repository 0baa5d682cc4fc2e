// sweep.cu -- the BPBC Smith-Waterman cell sweep (the hot loop), sm_100a.
//
// Compiled once per score width S (-DBPBC_S=S) so the 13 widths build in
// parallel; each object registers its kernels in the dispatch table.
//
// What it computes ("BPBC parallel for SWA", and the per-thread
// program of P:L364-372): for every 32-pair group, the bit-sliced score
// tables D^l[i][j] cell by cell along anti-diagonals t = i + j
// (R7), keeping the running maximum R_{k,i} per row and
// writing it per lane for the max-reduction + B2W step (extract.cu).
//
// B200 design, not the paper's TITAN X one:
//   * one 32-pair group per L lanes (L = 16 or 32; 32/L groups per warp);
//     lane l owns query rows [l*R, l*R + R) and keeps their current scores
//     (R*S planes), its query bases (2R words) and its running max (S planes)
//     in registers for the whole group -- no shared memory on the path
//     (the paper hands rows over through shared memory);
//   * wavefront skew across lanes: at step tau lane l works on column
//     J = tau - l; the bottom-row scores move to lane l+1 with S
//     __shfl_up_sync per step (the paper names shuffles as the option);
//   * persistent streaming: each L-lane segment walks a contiguous range of
//     groups back to back as one virtual target of length Gs*n, so the
//     pipeline fill/drain (L-1 steps, the paper's (m-1)/(n+m-1) idle share)
//     is paid once per stream, not per group;
//   * the group switch of a lane (its column J hits a multiple of n) stores
//     its partial max and resets its state, branch-free (predicated) in the
//     phases that contain switches;
//   * the cell is a fixed LOP3 circuit (circuit.cuh): no branch on data.
#include "bpbc_internal.cuh"
#include "transpose.cuh"

#ifndef BPBC_S
#error "compile with -DBPBC_S=<score width>"
#endif
#ifndef BPBC_MODE
#error "compile with -DBPBC_MODE=<0 running max | 1 threshold flag>"
#endif

namespace bpbc {
namespace {

__device__ __forceinline__ uint32_t opaque(uint32_t v) {
  uint32_t r;
  asm volatile("mov.b32 %0, %1;" : "=r"(r) : "r"(v));
  return r;
}
__device__ __forceinline__ uint32_t mul_lo(uint32_t a, uint32_t b) {
  uint32_t r;
  asm("mul.lo.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t mul_hi(uint32_t a, uint32_t b) {
  uint32_t r;
  asm("mul.hi.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}

// Predicated global store / shared load (the predicate is pr != 0): forced
// into PTX predication so the group switch of kSwPred adds no branch.
__device__ __forceinline__ void st_if(uint32_t* p, uint32_t v, uint32_t pr) {
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q st.global.u32 [%0], %1; }" ::"l"(p), "r"(v),
               "r"(pr)
               : "memory");
}
__device__ __forceinline__ void lds2_if(const uint2* p, uint32_t& x, uint32_t& y, uint32_t pr) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(p));
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %3, 0; @q ld.shared.v2.u32 {%0, %1}, [%2]; }"
               : "+r"(x), "+r"(y)
               : "r"(s), "r"(pr)
               : "memory");
}

// Group-switch handling of a step (sw_sweep_kernel): none in the phase, a
// divergent branch, or branch-free predication.
enum : int { kSwNone = 0, kSwBranch = 1, kSwPred = 2 };
#ifndef BPBC_SWMODE
#define BPBC_SWMODE kSwPred
#endif
template <int V>
using SwMode = std::integral_constant<int, V>;

// Asynchronous 8-byte global -> shared copies (cp.async, no register
// staging): the next group's query planes are fetched while the current
// group runs, and read back with a short-latency LDS at the group switch.
__device__ __forceinline__ void cp_async8(void* smem, const void* gmem) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }


// Target chunk that straddles two groups of a stream (only when n % 32 != 0):
// lane k gathers positions col.. of pair 32g+k, continuing into pair
// 32 g_next + k (the stream's next group) after the row end; folded H / L as
// tr_load_fold.  Out of line: one copy per object instead of one per kernel
// instantiation.
__device__ __noinline__ uint3 gather_straddle(const uint8_t* traw, int64_t tstride, int n,
                                              int64_t P, int64_t g, int64_t g_next, bool has_next,
                                              int col, int lane, bool packed2) {
  uint32_t H, L, bad = 0;
  uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  const int64_t row0 = g * 32 + lane, row1 = g_next * 32 + lane;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    const bool next = col + i >= n;  // past this group's last column
    const int cc = col + i - (next ? n : 0);
    const int64_t row = next ? row1 : row0;
    uint32_t code = 0;
    if ((next ? has_next : true) && row < P) {
      code = packed2 ? (traw[row * tstride + cc / 4] >> (2 * (cc & 3))) & 3u
                     : traw[row * tstride + cc];
    }
    if (packed2) {  // place as a 2-bit field of the packed layout
      w[i >> 4] |= (code & 3u) << (2 * (i & 15));
    } else {
      w[i >> 2] |= (code & 0xFFu) << (8 * (i & 3));
    }
  }
  if (packed2) tr_fold_packed2(w[0], w[1], H, L);
  else tr_fold_u8(w, H, L, bad);
  return make_uint3(H, L, bad);  // by value: registers, no stack frame at the call
}

// Acquire / release accesses of the progress and snapshot flags.
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// Device-side waits are bounded: a wait that sees no progress for
// kSpinTimeoutNs (a copy or a peer warp that never comes, e.g. another
// kernel holding the SMs the wrap schedule's streams need) raises the sticky
// BPBC_FLAG_STALL and gives up instead of hanging the GPU; the scores of
// that call are then undefined and the host-buffer calls return
// BPBC_ERR_CUDA.  The vote keeps every decision warp-uniform.
constexpr uint64_t kSpinTimeoutNs = 20ull * 1000000000ull;
__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Host-streamed inputs: wait until *progress > w and return the value seen
// (0xFFFFFFFF after a timeout).  Out of line: the resident-input path never
// calls it and keeps its registers.
__device__ __noinline__ uint32_t spin_progress(const uint32_t* progress, uint32_t w, uint32_t* flags) {
  const uint64_t t0 = global_ns();
  while (true) {
    const uint32_t v = ld_acquire_gpu(progress);
    if (!__any_sync(0xFFFFFFFFu, v <= w)) return v;
    if (__any_sync(0xFFFFFFFFu, global_ns() - t0 > kSpinTimeoutNs)) {
      if ((threadIdx.x & 31) == 0) atomicOr(flags, BPBC_FLAG_STALL);
      return 0xFFFFFFFFu;
    }
    __nanosleep(512);
  }
}
// Wrap-around schedule: wait until the snapshot flag *f is set.
__device__ __noinline__ void spin_flag(const uint32_t* f, uint32_t* flags) {
  const uint64_t t0 = global_ns();
  while (__any_sync(0xFFFFFFFFu, ld_acquire_gpu(f) == 0)) {
    if (__any_sync(0xFFFFFFFFu, global_ns() - t0 > kSpinTimeoutNs)) {
      if ((threadIdx.x & 31) == 0) atomicOr(flags, BPBC_FLAG_STALL);
      return;
    }
    __nanosleep(256);
  }
}

// ---------------------------------------------------------------------------
// Per-lane state and the wavefront step of the fused single-warp sweeps
// (sw_sweep_kernel and sw_sweep_wrap_kernel share it).
//
// A lane owns query rows [sl R, sl R + R) of its segment's current group:
// their scores at the previous column (H, R x S planes), the up-row score of
// the previous column (dtop, the diagonal input of its first row), its
// running max (M) or threshold flag, its query bases (xh / xl), and the
// countdown to its next group switch.  All of it lives in registers.
template <int S, int R, int L, int CIRC, bool PAD, class K>
struct FusedLane {
  static constexpr int kMW = BPBC_MODE == kModeThreshold ? L : L * S;  // Mpart words per lane-group
  uint32_t H[R][S], dtop[S], M[S];
  uint32_t xh[R], xl[R], kill[R];
  uint32_t nz, z0;    // 0/1 multiplier of the received up-row; 0 (state reset on the FMA pipe)
  uint32_t flag;      // threshold mode: pairs with a cell > tau so far
  int cnt;            // steps until my next group starts (J % n == 0)
  int gi;             // my current group within the (sub-)stream
  int gsn;            // group ends stored in this (sub-)stream
  uint32_t* mdst;     // my partial-max slot of the current group, advanced at every switch
  int mstep;          // words from one group's slot to the next group's (kMW x group stride)
  const uint2* xrow;  // my query-plane slot 0 in the shared ring (+ slot * 32 * R)

  __device__ __forceinline__ void reset(int sl) {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      dtop[i] = 0;
      M[i] = 0;
#pragma unroll
      for (int r = 0; r < R; ++r) H[r][i] = 0;
    }
#pragma unroll
    for (int r = 0; r < R; ++r) xh[r] = xl[r] = 0;
    flag = 0;
    cnt = sl;
    gi = -1;
  }

  // One wavefront step with target planes y of my current column.  SW: the
  // step may be a lane's group switch (the warp runs phases in which no lane
  // switches without the per-step check): kSwBranch takes the switch in a
  // divergent branch, kSwPred runs it branch-free in every lane (predicated
  // stores and loads, state reset by a multiply with 0/1 on the FMA pipe), so
  // the two steps of an iteration stay one basic block the scheduler can
  // interleave.
  template <int SW>
  __device__ __forceinline__ void step(const uint2 y, const SweepArgs& a, const K& k) {
    uint32_t up[S];
#pragma unroll
    for (int i = 0; i < S; ++i) up[i] = mul_lo(__shfl_up_sync(0xFFFFFFFFu, H[R - 1][i], 1, L), nz);

    if constexpr (SW == kSwPred) {
      // keep = 0 at column 0 of my next group, else 1: the carry of
      // cnt + (2^31 - 1) into bit 31, taken as mul.hi so it stays on the FMA
      // pipe and ptxas cannot turn the resets below into selects
      const uint32_t keep = mul_hi(uint32_t(cnt) + 0x7FFFFFFFu, 2u);
      const bool sw = cnt == 0;
      const uint32_t st = (sw && unsigned(gi) < unsigned(gsn)) ? 1u : 0u;
      if constexpr (BPBC_MODE == kModeThreshold) {
        st_if(mdst, flag, st);
      } else {
#pragma unroll
        for (int i = 0; i < S; ++i) st_if(mdst + i, M[i], st);
      }
      mdst += st * mstep;
      gi += sw ? 1 : 0;
      flag = mul_lo(flag, keep);
#pragma unroll
      for (int i = 0; i < S; ++i) {
        M[i] = mul_lo(M[i], keep);
        dtop[i] = mul_lo(dtop[i], keep);
#pragma unroll
        for (int r = 0; r < R; ++r) H[r][i] = mul_lo(H[r][i], keep);
      }
      const uint2* xv = xrow + (gi & 1) * (32 * R);
#pragma unroll
      for (int r = 0; r < R; ++r) lds2_if(xv + r, xh[r], xl[r], sw ? 1u : 0u);
      cnt = (sw ? a.n : cnt) - 1;
    }
    if (SW == kSwBranch && cnt == 0) {  // column 0 of my next group (divergent, once per group)
      if (gi >= 0 && gi < gsn) {
        if constexpr (BPBC_MODE == kModeThreshold) {
          *mdst = flag;  // one flag word per lane
        } else {
          // exact circuit: M tracked D' = diag + w + g; extract subtracts g
#pragma unroll
          for (int i = 0; i < S; ++i) mdst[i] = M[i];
        }
        mdst += mstep;
      }
      ++gi;
      flag = mul_lo(flag, z0);
#pragma unroll
      for (int i = 0; i < S; ++i) {
        M[i] = mul_lo(M[i], z0);
        dtop[i] = mul_lo(dtop[i], z0);
#pragma unroll
        for (int r = 0; r < R; ++r) H[r][i] = mul_lo(H[r][i], z0);
      }
      const uint2* xv = xrow + (gi & 1) * (32 * R);
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint2 v = xv[r];
        xh[r] = v.x;
        xl[r] = v.y;
      }
      cnt = a.n;
    }
    if (SW == kSwBranch) --cnt;

    uint32_t dg[S], u[S];
#pragma unroll
    for (int i = 0; i < S; ++i) {
      dg[i] = dtop[i];
      u[i] = up[i];
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t hn[S], dn[S];
      // running max over the diagonal term (circuit.cuh finish_exact); padded
      // rows are masked out of it
      if constexpr (CIRC == kExact) {
        cell_exact<S, K, false>(u, H[r], dg, xh[r], xl[r], y.x, y.y, 0u, hn, dn, k);
      } else {
        cell_sat<S, K>(u, H[r], dg, xh[r], xl[r], y.x, y.y, hn, dn, k);
      }
      if constexpr (BPBC_MODE == kModeThreshold) {
        flag_gt<S, PAD>(flag, dn, a.tmask, kill[r]);
      } else {
        runmax<S, PAD>(M, dn, kill[r]);
      }
#pragma unroll
      for (int i = 0; i < S; ++i) {
        dg[i] = H[r][i];
        H[r][i] = hn[i];
        u[i] = hn[i];
      }
    }
#pragma unroll
    for (int i = 0; i < S; ++i) dtop[i] = up[i];
  }

  // The 32 steps of one phase; yb = my 32 target columns of the phase in the
  // shared ring.  A lane switches groups in this phase iff its countdown is
  // below 32.  Two copies of the step must fit the instruction cache together
  // (4 warps per SMSP run both): at R = 8 one copy is ~27 KB and two copies
  // measured 16 % slower (C3), so R = 8 keeps only the checked step.  Switch
  // steps run branch-free (kSwPred: C2 5 743 vs 5 643 GCUPS with the
  // divergent branch); the single R = 8 step runs in every phase and keeps
  // the branch (kSwPred there costs every step: C3 5 194 vs 5 429).
  //
  // R <= 4: one loop for every phase, whose iterations (two steps each) run
  // the switch copy only inside the phase's switch window [lo, hi] -- the
  // steps at which some lane of the warp reaches column 0 of its next group
  // (warp-uniform, two redux votes per phase).  The L lanes of a segment
  // switch at L consecutive steps, so with L = 16 at most half of a phase
  // runs the switch copy (m <= 64, where every phase or every other one has
  // switches); with L = 32 a switch phase is switch steps throughout.
  __device__ __forceinline__ void phase(const uint2* yb, const SweepArgs& a, const K& k) {
    if constexpr (R > 4) {
#pragma unroll 1
      for (int i = 0; i < 32; i += 2) {
        const uint2 y0 = yb[i], y1 = yb[i + 1];
        step<kSwBranch>(y0, a, k);
        step<kSwBranch>(y1, a, k);
      }
    } else {
      // (broadcast from lane 0 so the window test runs on the uniform datapath)
      const int lo = __shfl_sync(0xFFFFFFFFu, int(__reduce_min_sync(0xFFFFFFFFu, cnt < 32 ? unsigned(cnt) : 32u)), 0);
      const int hi = __shfl_sync(0xFFFFFFFFu, int(__reduce_max_sync(0xFFFFFFFFu, cnt < 32 ? unsigned(cnt) + 1 : 0u)), 0) - 1;
#pragma unroll 1
      for (int i = 0; i < 32; i += 2) {
        const uint2 y0 = yb[i], y1 = yb[i + 1];
        if (i + 1 >= lo && i <= hi) {
          step<BPBC_SWMODE>(y0, a, k);
          step<BPBC_SWMODE>(y1, a, k);
        } else {
          step<kSwNone>(y0, a, k);
          step<kSwNone>(y1, a, k);
          cnt -= 2;
        }
      }
    }
  }
};

// ---------------------------------------------------------------------------
// The single-warp sweep with the W2B transpose fused in:
// it reads the caller's raw codes (u8, or 2-bit packed) and builds the bit
// planes itself, so no separate pack pass and no planes in HBM.
//
//   * target: every 32 steps (a "phase") the warp transposes the next 32
//     columns of each segment's virtual target (tr_load_fold + tr_butterfly,
//     transpose.cuh) into a shared-memory ring of 128 columns, stored twice
//     (slots j and j + 128) so a lane's 32 reads of a phase never wrap; the
//     ring holds chunks p-1..p+2 and chunk p+2 is built at the start of phase
//     p, so reads never wait on it;
//   * query: the planes of a segment's next group are transposed into a
//     2-slot shared ring at a phase start after every lane has entered the
//     current group (and before lane 0 leaves it: needs n >= L + 32);
//   * a __syncwarp at each phase start orders the ring writes before reads.
// HS: host-streamed inputs (SweepArgs::progress) -- a separate instantiation,
// so the wave polling costs the resident-input kernels no registers.
template <int S, int R, int L, int CIRC, bool PAD, class K, bool HS = false>
__global__ void __launch_bounds__(128, R <= 4 ? 4 : 3) sw_sweep_kernel(const SweepArgs a, const K k) {
  constexpr int SEGS = 32 / L;
  constexpr int XCH = (L * R + 31) / 32;  // 32-row chunks of a group's query rows
  const int lane = threadIdx.x & 31;
  const int sl = lane & (L - 1);
  const int seg = lane / L;
  const int wib = threadIdx.x >> 5;
  const int64_t warp = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  if (warp * SEGS >= a.streams) return;  // uniform per warp

  // groups of segment s's stream (uniform per warp for each s): stream st
  // takes the groups st, st + streams, st + 2 streams, ... (strided, so the
  // h-th groups of all streams -- one "wave" -- are contiguous: the
  // host-streamed path copies the input wave by wave, a.progress)
  const int64_t gstr = a.streams;
  // (every stream has base or base + 1 groups: the first rem streams one more)
  auto seg_range = [&](int s, int64_t& gbs, int64_t& gss) {
    const int64_t st = warp * SEGS + s;
    gss = 0;
    gbs = 0;
    if (st < a.streams) {
      gss = a.base + (st < a.rem ? 1 : 0);
      gbs = st;
    }
  };
  // host-streamed inputs: wave h (group index h of every stream) may be read
  // once the copy stream has published a.progress > h (warp-uniform poll)
  uint32_t ready = 0;  // waves known to be in (HS)
  auto wait_wave = [&](int64_t h) {
    if constexpr (HS) {
      if (uint32_t(h) >= ready) ready = spin_progress(a.progress, uint32_t(h), a.flags);
    }
  };
  int64_t Gs, gb;
  seg_range(seg, gb, Gs);
  FusedLane<S, R, L, CIRC, PAD, K> ln;
  ln.nz = opaque(sl != 0 ? 1u : 0u);
  // multiplier 0 for the state reset at a group switch: the reset runs as
  // IMADs on the FMA pipe instead of register-pair clears on the ALU pipe,
  // which the cell circuits saturate
  ln.z0 = opaque(uint32_t(a.m) >> 31);  // 0 (m > 0), unknown to ptxas
#pragma unroll
  for (int r = 0; r < R; ++r) ln.kill[r] = PAD ? opaque((sl * R + r >= a.m) ? 0xFFFFFFFFu : 0u) : 0u;
  ln.reset(sl);
  __shared__ uint2 xring[4][2][32][R];        // [warp][slot][lane][row]
  __shared__ uint2 yring[4][SEGS][256];       // [warp][segment][column slot, doubled]
  uint2 (*xr)[32][R] = xring[wib];
  uint2 (*yr)[256] = yring[wib];
  const bool packed2 = a.packed2 != 0;
  const int mypos = packed2 ? tr_pos_packed2(lane) : tr_pos_u8(lane);
  uint32_t bad = 0;

  // Staged loads (ST: the R <= 4 tilings, m <= 128; R = 8 is register-bound):
  // with short groups every phase transposes a new query group and a target
  // chunk per segment,
  // and a load consumed right away exposes its HBM latency once per phase
  // (ncu, m = n = 32: 28 % of the warp stall samples sat in the phase
  // prologue, mostly long-scoreboard).  Whole, aligned 32-position chunks are
  // therefore fetched one phase ahead by cp.async into a per-lane shared
  // staging slot (no registers held across the phase) and folded from there
  // a phase later; everything else (ragged / straddling / unaligned chunks)
  // keeps the direct load.  A lane reads back only its own staged bytes, so
  // cp.async.wait_all orders them; the staging slot is rewritten only after
  // the fold has consumed the values read from it.
  constexpr bool ST = (L == 16) || (R == 4);
  constexpr int SSEG = ST ? SEGS : 1, SXCH = ST ? XCH : 1;
  __shared__ __align__(16) uint4 ystage[4][SSEG][32][2];        // [warp][segment][lane] 32 B
  __shared__ __align__(16) uint4 xstage[4][SSEG][SXCH][32][2];  // [warp][segment][chunk][lane]
  const bool y_al = packed2 ? ((a.tstride & 7) == 0 && (reinterpret_cast<uintptr_t>(a.traw) & 7) == 0)
                            : ((a.tstride & 15) == 0 && (reinterpret_cast<uintptr_t>(a.traw) & 15) == 0);
  const bool x_al = packed2 ? ((a.qstride & 7) == 0 && (reinterpret_cast<uintptr_t>(a.qraw) & 7) == 0)
                            : ((a.qstride & 15) == 0 && (reinterpret_cast<uintptr_t>(a.qraw) & 15) == 0);
  // raw bytes of positions [c0, c0 + 32) of one row -> my staging slot
  auto stage_row = [&](uint4* dst, const uint8_t* base, int64_t stride, int64_t row, int c0) {
    if (packed2) {
      cp_async8(dst, base + row * stride + c0 / 4);
    } else {
      const uint8_t* src = base + row * stride + c0;
      cp_async16(dst, src);
      cp_async16(dst + 1, src + 16);
    }
  };
  auto fold_staged = [&](const uint4* src, uint32_t& Hw, uint32_t& Lw) {
    if (packed2) {
      const uint2 v = *reinterpret_cast<const uint2*>(src);
      tr_fold_packed2(v.x, v.y, Hw, Lw);
    } else {
      const uint4 u0 = src[0], u1 = src[1];
      uint32_t w[8] = {u0.x, u0.y, u0.z, u0.w, u1.x, u1.y, u1.z, u1.w};
      tr_fold_u8(w, Hw, Lw, bad);
    }
  };
  // the fast (staged) case of target chunk c of segment s: one group, whole
  auto y_fast = [&](int s, int64_t c, int64_t& g, int& col, int64_t& h) {
    int64_t gbs, gss;
    seg_range(s, gbs, gss);
    const int64_t v0 = 32 * c;
    if (!y_al || v0 < 0 || v0 >= gss * a.n) return false;
    h = v0 / a.n;
    col = int(v0 - h * a.n);
    g = gbs + h * gstr;
    return col + 32 <= a.n;
  };
  auto issue_y = [&](int s, int64_t c) {
    if constexpr (ST) {
      int64_t g, h;
      int col;
      if (y_fast(s, c, g, col, h)) {
        wait_wave(h);
        if (g * 32 + lane < a.P) stage_row(ystage[wib][s][lane], a.traw, a.tstride, g * 32 + lane, col);
      }
    }
  };
  // target columns [32c, 32c + 32) of segment s's virtual target -> ring
  // (staged: the chunk's fast case was issued to the staging slot a phase
  // ago; the prologue's chunks 0 and 1 are loaded directly)
  auto build_y = [&](int s, int64_t c, bool staged) {
    int64_t gbs, gss;
    seg_range(s, gbs, gss);
    const int64_t v0 = 32 * c;  // first virtual column
    uint32_t Hw = 0, Lw = 0;
    int64_t fg = 0, fh = 0;
    int fcol = 0;
    if (ST && staged && y_fast(s, c, fg, fcol, fh)) {
      if (fg * 32 + lane < a.P) fold_staged(ystage[wib][ST ? s : 0][lane], Hw, Lw);
    } else if (v0 >= 0 && v0 < gss * a.n) {
      const int64_t h = v0 / a.n;
      const int col = int(v0 - h * a.n);
      const int64_t g = gbs + h * gstr;
      if (col + 32 <= a.n) {
        wait_wave(h);
        tr_load_fold(a.traw, a.tstride, a.n, g * 32 + lane, a.P, col, packed2, Hw, Lw, bad);
      } else {  // the chunk straddles two groups (n % 32 != 0; n >= 48)
        wait_wave(h + 1 < gss ? h + 1 : h);
        const uint3 r3 = gather_straddle(a.traw, a.tstride, a.n, a.P, g, g + gstr, h + 1 < gss,
                                         col, lane, packed2);
        Hw = r3.x;
        Lw = r3.y;
        bad |= r3.z;
      }
    }
    tr_butterfly(Hw, Lw, lane);
    const int slot = int((v0 + mypos) & 127);
    yr[s][slot] = make_uint2(Hw, Lw);
    yr[s][slot + 128] = make_uint2(Hw, Lw);
  };
  // query group of segment s's stream-relative group h
  auto x_group = [&](int s, int64_t h, bool& live) {
    int64_t gbs, gss;
    seg_range(s, gbs, gss);
    int64_t g = gbs + h * gstr;
    live = g < a.G;
    if (!live) g = gbs < a.G ? gbs : a.G - 1;  // past the stream's last group: unused
    return g;
  };
  auto issue_x = [&](int s, int64_t h) {
    if constexpr (ST) {
      bool live;
      const int64_t g = x_group(s, h, live);
      if (!x_al) return;
      if (live) wait_wave(h);
#pragma unroll
      for (int c = 0; c < XCH; ++c)
        if (32 * c + 32 <= a.m && g * 32 + lane < a.P)
          stage_row(xstage[wib][s][c][lane], a.qraw, a.qstride, g * 32 + lane, 32 * c);
    }
  };
  // query rows of segment s's group h (stream-relative) -> x slot h & 1
  auto build_x = [&](int s, int64_t h, bool staged) {
    bool live;
    const int64_t g = x_group(s, h, live);
    if (live) wait_wave(h);
#pragma unroll
    for (int c = 0; c < XCH; ++c) {
      uint32_t Hw = 0, Lw = 0;
      if (ST && staged && x_al && 32 * c + 32 <= a.m) {
        if (g * 32 + lane < a.P) fold_staged(xstage[wib][ST ? s : 0][ST ? c : 0][lane], Hw, Lw);
      } else {
        tr_load_fold(a.qraw, a.qstride, a.m, g * 32 + lane, a.P, 32 * c, packed2, Hw, Lw, bad);
      }
      tr_butterfly(Hw, Lw, lane);
      const int row = 32 * c + mypos;  // rows >= m are zero (tr_load_fold)
      if (row < L * R) xr[int(h & 1)][s * L + row / R][row % R] = make_uint2(Hw, Lw);
    }
  };

  ln.gsn = int(Gs);  // groups of my stream (< 2^31: P < 2^36)
  ln.mdst = a.Mpart + (gb * L + sl) * (ln.kMW / L);
  ln.mstep = int(ln.kMW * gstr);
  ln.xrow = &xr[0][lane][0];

  // prologue: the first group's query planes, target chunks -1 (zeros), 0, 1
  // (and, staged: the next group's query rows and target chunk 2 in flight)
#pragma unroll
  for (int s = 0; s < SEGS; ++s) {
    yr[s][lane] = yr[s][lane + 32] = yr[s][lane + 64] = yr[s][lane + 96] = make_uint2(0u, 0u);
    yr[s][lane + 128] = yr[s][lane + 160] = yr[s][lane + 192] = yr[s][lane + 224] =
        make_uint2(0u, 0u);
  }
  __syncwarp();
  int64_t xnext[SEGS];
#pragma unroll
  for (int s = 0; s < SEGS; ++s) {
    build_x(s, 0, false);
    xnext[s] = 1;
    issue_x(s, 1);
    build_y(s, 0, false);
    build_y(s, 1, false);
    issue_y(s, 2);
  }
  if constexpr (ST) cp_async_commit();
  const int64_t phases = a.steps / 32;  // a.steps is a multiple of 32
  if constexpr (ST) {
    // Staged phase prologue: the target position of the next chunk to issue
    // advances by 32 columns per phase (no 64-bit division per chunk), the
    // chunk to build carries its fast/g decision from its issue a phase ago,
    // and the folds of all segments' chunks come first so their butterflies
    // form one straight-line block (the shuffle latencies overlap; ncu at
    // m = n = 32: the per-phase transposes held 22 % of the stall samples).
    int yi_h[SEGS], yi_col[SEGS], yb_g[SEGS];
    bool yb_fast[SEGS];
    const int64_t c2 = 64;  // chunk 2, issued in the prologue above
#pragma unroll
    for (int s = 0; s < SEGS; ++s) {
      int64_t gbs, gss;
      seg_range(s, gbs, gss);
      const int h2 = int(c2 / a.n), col2 = int(c2 - int64_t(h2) * a.n);
      yb_fast[s] = y_al && h2 < gss && col2 + 32 <= a.n;
      yb_g[s] = int(gbs + int64_t(h2) * gstr);
      yi_h[s] = h2;
      yi_col[s] = col2 + 32;  // chunk 3
      if (yi_col[s] >= a.n) {
        yi_col[s] -= a.n;
        ++yi_h[s];
      }
    }
    constexpr int NX = SEGS * XCH;
    for (int64_t p = 0; p < phases; ++p) {
      cp_async_wait_all();  // (this lane's copies issued a phase ago)
      __syncwarp();         // this warp's ring writes of the previous phase -> reads
      // target chunk p + 2 of every segment: fold, then issue chunk p + 3
      uint32_t yH[SEGS], yL[SEGS];
#pragma unroll
      for (int s = 0; s < SEGS; ++s) {
        yH[s] = yL[s] = 0u;
        if (yb_fast[s]) {
          if (int64_t(yb_g[s]) * 32 + lane < a.P) fold_staged(ystage[wib][s][lane], yH[s], yL[s]);
        } else {
          int64_t gbs, gss;
          seg_range(s, gbs, gss);
          const int64_t v0 = 32 * (p + 2);
          if (v0 < gss * a.n) {  // (ragged / straddling chunk: direct load)
            const int64_t h = v0 / a.n;
            const int col = int(v0 - h * a.n);
            const int64_t g = gbs + h * gstr;
            if (col + 32 <= a.n) {
              wait_wave(h);
              tr_load_fold(a.traw, a.tstride, a.n, g * 32 + lane, a.P, col, packed2, yH[s], yL[s], bad);
            } else {
              wait_wave(h + 1 < gss ? h + 1 : h);
              const uint3 r3 = gather_straddle(a.traw, a.tstride, a.n, a.P, g, g + gstr,
                                               h + 1 < gss, col, lane, packed2);
              yH[s] = r3.x;
              yL[s] = r3.y;
              bad |= r3.z;
            }
          }
        }
        // issue chunk p + 3 (position advanced incrementally)
        int64_t gbs, gss;
        seg_range(s, gbs, gss);
        const bool fast = y_al && yi_h[s] < gss && yi_col[s] + 32 <= a.n;
        const int g = int(gbs + int64_t(yi_h[s]) * gstr);
        if (fast) {
          wait_wave(yi_h[s]);
          if (int64_t(g) * 32 + lane < a.P)
            stage_row(ystage[wib][s][lane], a.traw, a.tstride, int64_t(g) * 32 + lane, yi_col[s]);
        }
        yb_fast[s] = fast;
        yb_g[s] = g;
        yi_col[s] += 32;
        if (yi_col[s] >= a.n) {
          yi_col[s] -= a.n;
          ++yi_h[s];
        }
      }
#pragma unroll
      for (int s = 0; s < SEGS; ++s) tr_butterfly(yH[s], yL[s], lane);
#pragma unroll
      for (int s = 0; s < SEGS; ++s) {
        const int slot = int((32 * (p + 2) + mypos) & 127);
        yr[s][slot] = make_uint2(yH[s], yL[s]);
        yr[s][slot + 128] = make_uint2(yH[s], yL[s]);
      }
      // query group xnext of every segment (the segments' lanes switch at the
      // same step offsets, so the condition is warp-uniform and equal for all
      // segments): write slot h & 1 once every lane of the segment entered
      // group h - 1 (step (h-1) n + L); lane 0 needs it at step h n
      if ((xnext[0] - 1) * a.n + L <= 32 * p) {
        uint32_t xH[NX], xL[NX];
#pragma unroll
        for (int s = 0; s < SEGS; ++s) {
          bool live;
          const int64_t g = x_group(s, xnext[s], live);
          if (live) wait_wave(xnext[s]);
#pragma unroll
          for (int c = 0; c < XCH; ++c) {
            uint32_t& H = xH[s * XCH + c];
            uint32_t& Lw = xL[s * XCH + c];
            H = Lw = 0u;
            if (x_al && 32 * c + 32 <= a.m) {
              if (g * 32 + lane < a.P) fold_staged(xstage[wib][s][c][lane], H, Lw);
            } else {
              tr_load_fold(a.qraw, a.qstride, a.m, g * 32 + lane, a.P, 32 * c, packed2, H, Lw, bad);
            }
          }
          ++xnext[s];
          issue_x(s, xnext[s]);
        }
#pragma unroll
        for (int i = 0; i < NX; ++i) tr_butterfly(xH[i], xL[i], lane);
#pragma unroll
        for (int s = 0; s < SEGS; ++s) {
#pragma unroll
          for (int c = 0; c < XCH; ++c) {
            const int row = 32 * c + mypos;  // rows >= m are zero
            if (row < L * R)
              xr[int((xnext[s] - 1) & 1)][s * L + row / R][row % R] =
                  make_uint2(xH[s * XCH + c], xL[s * XCH + c]);
          }
        }
      }
      cp_async_commit();
      __syncwarp();
      ln.phase(&yr[seg][(32 * p - sl) & 127], a, k);  // my 32 columns of this phase
    }
  } else {
  for (int64_t p = 0; p < phases; ++p) {
    __syncwarp();  // this warp's ring writes of the previous phase -> reads
#pragma unroll
    for (int s = 0; s < SEGS; ++s) {
      build_y(s, p + 2, true);
      // group h's query may be written into slot h & 1 once every lane of
      // the segment has entered group h - 1 (step (h-1) n + L); lane 0 needs
      // it at step h n
      if ((xnext[s] - 1) * a.n + L <= 32 * p) {
        build_x(s, xnext[s], true);
        ++xnext[s];
      }
    }
    __syncwarp();
    ln.phase(&yr[seg][(32 * p - sl) & 127], a, k);  // my 32 columns of this phase
  }
  }
  if constexpr (ST) cp_async_wait_all();
  if (__any_sync(0xFFFFFFFFu, bad != 0) && lane == 0) atomicOr(a.flags, BPBC_FLAG_BAD_BASE);
}

// ---------------------------------------------------------------------------
// The fused single-warp sweep (L = 32) with the wrap-around schedule
// (SweepArgs::wrap): used when a batch has few long groups
// (the paper's shape), where a group-granular split leaves SMSPs with
// one or two groups' worth of work (at most 1024 / (592 x 2) = 86 % of the
// pipe for 1024 groups on 592 SMSPs).  Stream k owns the columns
// [k span, (k+1) span) of the concatenation of all groups' columns and runs
// them as up to three "sub-streams": the head of the group its range ends in
// (columns [0, rb), ending in a snapshot of the whole warp state), the whole
// groups in between, and the tail of the group its range starts in (columns
// [ra, n), resuming from the snapshot the previous stream wrote at the end of
// ITS head).  The snapshot is taken after the step in which lane 0 finished
// column rb - 1, so lane l holds the state of column rb - 1 - l, and the
// resuming warp's lane l continues at column ra - l: the wavefront moves
// between warps without a drain or refill.  McNaughton's wrap-around rule
// makes the tail start at least (span - n) columns after the head ends.
// Per sub-stream the body is sw_sweep_kernel's (same transposes, rings,
// switch handling and circuits).


// (no occupancy floor: the schedule runs it with few blocks per SM; the
// planner reads its occupancy)
template <int S, int R, int CIRC, bool PAD, class K>
__global__ void __launch_bounds__(128) sw_sweep_wrap_kernel(const SweepArgs a, const K k) {
  constexpr int L = 32;
  constexpr int XCH = (L * R + 31) / 32;  // 32-row chunks of a group's query rows
  constexpr int NSW = snap_words(R, S);
  const int lane = threadIdx.x & 31;
  // warp index broadcast from lane 0: provably warp-uniform, so the
  // sub-stream bookkeeping derived from it stays on the uniform datapath
  const int wib = __shfl_sync(0xFFFFFFFFu, int(threadIdx.x >> 5), 0);
  const int64_t warp = int64_t(blockIdx.x) * (blockDim.x >> 5) + wib;
  if (warp >= a.streams) return;  // uniform per warp

  FusedLane<S, R, L, CIRC, PAD, K> ln;
  ln.nz = opaque(lane != 0 ? 1u : 0u);
  ln.z0 = opaque(uint32_t(a.m) >> 31);  // 0 (m > 0), unknown to ptxas
#pragma unroll
  for (int r = 0; r < R; ++r) ln.kill[r] = PAD ? opaque((lane * R + r >= a.m) ? 0xFFFFFFFFu : 0u) : 0u;
  __shared__ uint2 xring[4][2][32][R];  // [warp][slot][lane][row]
  __shared__ uint2 yring[4][256];       // [warp][column slot, doubled]
  uint2 (*xr)[32][R] = xring[wib];
  uint2* yr = yring[wib];
  ln.xrow = &xr[0][lane][0];
  const bool packed2 = a.packed2 != 0;
  const int mypos = packed2 ? tr_pos_packed2(lane) : tr_pos_u8(lane);
  uint32_t bad = 0;

  // sub-stream bookkeeping (warp-uniform): first group g0, groups touched
  // nspan, the next target chunk (group offset yg, column ycol, position
  // ypos on the stream's copy timeline, whose piece ends at yend) and the
  // next query group xnext with the step xth from which it may be built
  int64_t g0 = 0, nspan = 0, yg = 0, xnext = 0, xth = 0, ypos = 0, yend = 0;
  int ycol = 0;
  // host-streamed inputs (bpbc_sw_score_batch_host): the copy stream moves
  // every stream's timeline in waves -- wave 0 = all query rows and columns
  // [0, blk_first) of every stream, wave i = [blk_first + (i-1) blk_rest,
  // blk_first + i blk_rest) -- and publishes the number of waves done in
  // *progress; a chunk is read once its wave is in (warp-uniform poll)
  uint32_t ready = a.progress ? 0u : 0xFFFFFFFFu;  // waves known to be in
  auto wait_wave = [&](int64_t w) {
    if (uint32_t(w) >= ready) ready = spin_progress(a.progress, uint32_t(w), a.flags);
  };
  // the next 32 target columns -> ring chunk c; advance (n % 32 == 0 here)
  auto build_y = [&](int64_t c) {
    uint32_t Hw = 0, Lw = 0;
    // (chunks past the piece are never used: skip the wait; resident inputs
    // never wait)
    if (a.progress != nullptr && ypos < yend) {
      const int64_t e = ypos + 32;
      // (wave 0 = [0, blk_first), wave i = up to blk_first + i blk_rest)
      wait_wave(e <= a.blk_first ? 0 : (e - a.blk_first + a.blk_rest - 1) / a.blk_rest);
    }
    if (yg < nspan)
      tr_load_fold(a.traw, a.tstride, a.n, (g0 + yg) * 32 + lane, a.P, ycol, packed2, Hw, Lw, bad);
    tr_butterfly(Hw, Lw, lane);
    const int slot = int((32 * c + mypos) & 127);
    yr[slot] = make_uint2(Hw, Lw);
    yr[slot + 128] = make_uint2(Hw, Lw);
    ycol += 32;
    ypos += 32;
    if (ycol >= a.n) {
      ycol -= a.n;
      ++yg;
    }
  };
  // query rows of group g0 + h -> x slot h & 1
  auto build_x = [&](int64_t h) {
    wait_wave(0);  // (all query rows come with wave 0)
    int64_t g = g0 + h;
    g = g < a.G ? g : a.G - 1;
#pragma unroll
    for (int c = 0; c < XCH; ++c) {
      uint32_t Hw = 0, Lw = 0;
      tr_load_fold(a.qraw, a.qstride, a.m, g * 32 + lane, a.P, 32 * c, packed2, Hw, Lw, bad);
      tr_butterfly(Hw, Lw, lane);
      const int row = 32 * c + mypos;  // rows >= m are zero (tr_load_fold)
      if (row < L * R) xr[int(h & 1)][row / R][row % R] = make_uint2(Hw, Lw);
    }
  };

  const int64_t tot = a.G * a.n;
  const int64_t V0 = warp * a.span;
  const int64_t V1 = V0 + a.span < tot ? V0 + a.span : tot;
  const int64_t ga = V0 / a.n, gz = V1 / a.n;
  const int ra = int(V0 - ga * a.n), rb = int(V1 - gz * a.n);
#pragma unroll 1
  for (int sub = 0; sub < 3; ++sub) {
    // ---- this sub-stream's groups, first column and boundary behaviour
    int c0 = 0;  // first column (of group g0)
    bool snap_in = false, snap_out = false;
    int64_t steps = 0, slot = 0;
    int gs = 0;  // group ends stored
    // (copy timeline of this stream: head [0, rb), whole groups [rb, rb +
    // nf n), tail [rb + nf n, rb + nf n + n - ra + 32) from column ra - 32)
    const int64_t nf = gz - (ga + (ra > 0 ? 1 : 0));
    if (sub == 0) {  // head of group gz: columns [0, rb), snapshot out
      if (rb == 0) continue;
      g0 = gz;
      nspan = 1;
      snap_out = true;
      slot = warp + 1;
      steps = rb;  // (a multiple of 32)
      ypos = 0;
      yend = rb;
    } else if (sub == 1) {  // whole groups
      g0 = ga + (ra > 0 ? 1 : 0);
      nspan = gz - g0;
      if (nspan <= 0) continue;
      gs = int(nspan);
      steps = (nspan * a.n + L + 31) / 32 * 32;
      ypos = rb;
      yend = rb + nf * a.n;
    } else {  // tail of group ga: columns [ra, n), snapshot in
      if (ra == 0) continue;
      g0 = ga;
      nspan = 1;
      gs = 1;
      c0 = ra;
      snap_in = true;
      slot = warp;
      steps = (a.n - ra + L + 31) / 32 * 32;
      ypos = rb + nf * a.n;  // chunk -1 (columns ra - 32 ..) opens the tail's range
      yend = ypos + (a.n - ra) + 32;
    }
    // ---- fresh state (a lane enters its first group at its switch step)
    ln.reset(lane);
    ln.gsn = gs;
    ln.mdst = a.Mpart + (g0 * L + lane) * (ln.kMW / L);
    ln.mstep = ln.kMW;

    // ---- prologue: first group's query planes, target chunks -1 (zeros, or
    // the columns before c0 when resuming), 0, 1
    __syncwarp();  // the previous sub-stream's ring reads -> these writes
    yr[lane] = yr[lane + 32] = yr[lane + 64] = yr[lane + 96] = make_uint2(0u, 0u);
    yr[lane + 128] = yr[lane + 160] = yr[lane + 192] = yr[lane + 224] = make_uint2(0u, 0u);
    __syncwarp();
    xnext = 1;
    xth = L - c0;  // group h may be built once (h-1) n - c0 + L <= 32 p
    build_x(0);
    yg = 0;
    ycol = c0;
    if (snap_in) {
      ycol = c0 - 32;  // (c0 >= 32)
      build_y(-1);
    }
    build_y(0);
    build_y(1);
    if (snap_in) {  // resume the warp state the previous stream left at column c0
      // (every lane polls; the vote keeps the loop warp-uniform)
      spin_flag(a.snap_flag + slot, a.flags);
      const uint32_t* src = a.snap + slot * (NSW * 32) + lane;
#pragma unroll
      for (int i = 0; i < S; ++i) {
#pragma unroll
        for (int r = 0; r < R; ++r) ln.H[r][i] = __ldcg(src + (r * S + i) * 32);
        ln.dtop[i] = __ldcg(src + (R * S + i) * 32);
        if constexpr (BPBC_MODE != kModeThreshold) ln.M[i] = __ldcg(src + ((R + 1) * S + i) * 32);
      }
      if constexpr (BPBC_MODE == kModeThreshold) ln.flag = __ldcg(src + (R + 1) * S * 32);
      ln.cnt = int(a.n - c0) + lane;
      ln.gi = 0;
      __syncwarp();  // build_x's ring writes (other lanes' rows) -> these reads
#pragma unroll
      for (int r = 0; r < R; ++r) {  // (slot 0, written by build_x above)
        const uint2 v = ln.xrow[r];
        ln.xh[r] = v.x;
        ln.xl[r] = v.y;
      }
    }

    const int64_t phases = steps / 32;  // steps is a multiple of 32
    for (int64_t p = 0; p < phases; ++p) {
      __syncwarp();  // this warp's ring writes of the previous phase -> reads
      build_y(p + 2);
      // group h's query may be written into slot h & 1 once every lane has
      // entered group h - 1; lane 0 needs it at its start
      if (xth <= 32 * p) {
        build_x(xnext);
        ++xnext;
        xth += a.n;
      }
      __syncwarp();
      ln.phase(&yr[(32 * p - lane) & 127], a, k);  // my 32 columns of this phase
    }
    if (snap_out) {  // hand the warp state to the stream that finishes this group
      uint32_t* dst = a.snap + slot * (NSW * 32) + lane;
#pragma unroll
      for (int i = 0; i < S; ++i) {
#pragma unroll
        for (int r = 0; r < R; ++r) __stcg(dst + (r * S + i) * 32, ln.H[r][i]);
        __stcg(dst + (R * S + i) * 32, ln.dtop[i]);
        if constexpr (BPBC_MODE != kModeThreshold) __stcg(dst + ((R + 1) * S + i) * 32, ln.M[i]);
      }
      if constexpr (BPBC_MODE == kModeThreshold) __stcg(dst + (R + 1) * S * 32, ln.flag);
      __threadfence();
      __syncwarp();
      if (lane == 0) st_release_gpu(a.snap_flag + slot, 1u);
    }
  }
  if (__any_sync(0xFFFFFFFFu, bad != 0) && lane == 0) atomicOr(a.flags, BPBC_FLAG_BAD_BASE);
}

// ---------------------------------------------------------------------------
// The single-warp sweep on pre-packed planes (pack_kernel output): used when
// the target is too short (n < L + 32) for the fused kernel's phase-granular
// query transposes.  Same wavefront and circuits.
template <int S, int R, int L, int CIRC, bool PAD, class K>
__global__ void __launch_bounds__(128) sw_sweep_planes_kernel(const SweepArgs a, const K k) {
  constexpr int SEGS = 32 / L;
  const int lane = threadIdx.x & 31;
  const int sl = lane & (L - 1);
  const int64_t warp = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  if (warp * SEGS >= a.streams) return;  // uniform per warp
  const int64_t stream = warp * SEGS + lane / L;

  int64_t Gs = 0, gb = 0;
  if (stream < a.streams) {
    Gs = a.base + (stream < a.rem ? 1 : 0);
    gb = stream * a.base + (stream < a.rem ? stream : a.rem);
  }
  // 1 for lanes that receive a real "up" row from the lane above, 0 for the
  // first lane of a segment (border d[-1][j] = 0).  Applied with an
  // integer multiply so it issues on the FMA pipe, not the logic pipe.
  // (volatile moves keep these opaque: the compiler may neither turn the
  // multiply into a logic-pipe select nor rematerialise the masks per step)
  const uint32_t nz = opaque(sl != 0 ? 1u : 0u);

  // kill[r] = all ones for padded rows (row >= m): their cells output 0.
  uint32_t kill[R];
#pragma unroll
  for (int r = 0; r < R; ++r) kill[r] = PAD ? opaque((sl * R + r >= a.m) ? 0xFFFFFFFFu : 0u) : 0u;

  uint32_t H[R][S];   // scores of my rows at the previous column (left)
  uint32_t dtop[S];   // up-row score at the previous column (diag of row 0)
  uint32_t M[S];      // running max of my rows
#pragma unroll
  for (int i = 0; i < S; ++i) {
    dtop[i] = 0;
    M[i] = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) H[r][i] = 0;
  }
  // my query planes: registers for the current group, a 2-slot shared ring
  // for the current and the next group (slot = group index & 1)
  __shared__ uint2 xring[4][2][32][R];  // [warp in block][slot][lane][row]
  uint2 (*ring)[32][R] = xring[threadIdx.x >> 5];
  uint32_t xh[R], xl[R];
  auto fetch_x = [&](int64_t gidx, int slot) {  // gidx: group index in the stream
    int64_t g = gb + gidx;
    g = g < a.G ? g : a.G - 1;
    const uint2* xp = a.Xp + g * a.m + sl * R;
#pragma unroll
    for (int r = 0; r < R; ++r) cp_async8(&ring[slot][lane][r], xp + r);
    cp_async_commit();
  };
  fetch_x(0, 0);
#pragma unroll
  for (int r = 0; r < R; ++r) xh[r] = xl[r] = 0;
  const uint2* yp = a.Yp + gb * a.n - sl;
  int cnt = sl;      // steps until my next group starts (J % n == 0)
  int64_t gi = -1;   // my current group within the stream
  uint32_t flag = 0; // threshold mode: pairs with a cell > tau so far

  // One wavefront step with target planes y of my current column.
  auto step = [&](const uint2 y) {
    uint32_t up[S];
#pragma unroll
    for (int i = 0; i < S; ++i) up[i] = mul_lo(__shfl_up_sync(0xFFFFFFFFu, H[R - 1][i], 1, L), nz);

    if (cnt == 0) {  // column 0 of my next group (divergent, once per group)
      if (gi >= 0 && gi < Gs) {
        if constexpr (BPBC_MODE == kModeThreshold) {
          a.Mpart[(gb + gi) * L + sl] = flag;  // one flag word per lane
        } else {
          uint32_t* dst = a.Mpart + ((gb + gi) * L + sl) * S;
          // exact circuit: M tracked D' = diag + w + g; extract subtracts g
#pragma unroll
          for (int i = 0; i < S; ++i) dst[i] = M[i];
        }
      }
      ++gi;
      flag = 0;
#pragma unroll
      for (int i = 0; i < S; ++i) {
        M[i] = 0;
        dtop[i] = 0;
#pragma unroll
        for (int r = 0; r < R; ++r) H[r][i] = 0;
      }
      cp_async_wait_all();  // my own copies of group gi (issued n steps ago)
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint2 v = ring[gi & 1][lane][r];
        xh[r] = v.x;
        xl[r] = v.y;
      }
      fetch_x(gi + 1, int((gi + 1) & 1));  // slot of group gi - 1, no longer read
      cnt = a.n;
    }
    --cnt;

    uint32_t dg[S], u[S];
#pragma unroll
    for (int i = 0; i < S; ++i) {
      dg[i] = dtop[i];
      u[i] = up[i];
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t hn[S], dn[S];
      // running max over the diagonal term (circuit.cuh finish_exact); padded
      // rows are masked out of it
      if constexpr (CIRC == kExact) {
        cell_exact<S, K, false>(u, H[r], dg, xh[r], xl[r], y.x, y.y, 0u, hn, dn, k);
      } else {
        cell_sat<S, K>(u, H[r], dg, xh[r], xl[r], y.x, y.y, hn, dn, k);
      }
      if constexpr (BPBC_MODE == kModeThreshold) {
        flag_gt<S, PAD>(flag, dn, a.tmask, kill[r]);
      } else {
        runmax<S, PAD>(M, dn, kill[r]);
      }
#pragma unroll
      for (int i = 0; i < S; ++i) {
        dg[i] = H[r][i];
        H[r][i] = hn[i];
        u[i] = hn[i];
      }
    }
#pragma unroll
    for (int i = 0; i < S; ++i) dtop[i] = up[i];
  };

  // Two steps per iteration with two target registers: each load lands in
  // its own register half an iteration before use, so no register move
  // waits on it (steps is rounded up to even; the pads cover the extra
  // column and an extra step past the last group stores nothing).
  uint2 y0 = __ldg(yp), y1;
  for (int64_t tau = 0; tau < a.steps; tau += 2) {
    y1 = __ldg(yp + tau + 1);
    step(y0);
    y0 = __ldg(yp + tau + 2);
    step(y1);
  }
}

__device__ __forceinline__ uint32_t mad_lo(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  return r;
}

// ---------------------------------------------------------------------------
// Long queries (m > 256 after the R17 swap): the query rows are cut into
// stripes of kStripeRows = L*R = 128 rows.  Every (group, stripe) pair is a
// "unit" of n columns; a stream walks units group-major (g0s0, g0s1, ...,
// g1s0, ...) exactly as the short kernel walks groups.  The bottom row of
// stripe k (S planes per column) is handed to the top lane of stripe k+1
// through a per-stream boundary buffer in global memory: the last lane stores
// it at column j, and lane 0 of the next unit loads it n - L steps later (so
// n > L is required, which holds because n >= m > 256).  Lane 0 of stripe 0
// reads a zero row instead (border d[-1][j] = 0).  The partial
// maxima go to Mpart[g][k][lane] (the extract kernel reduces stripes x lanes).
// Everything else is the short kernel (same circuits, same wavefront).
template <int S, int CIRC, class K, int R>
__global__ void __launch_bounds__(128) sw_sweep_striped_kernel(const SweepArgs a, const K k) {
  constexpr int L = 32, LR = L * R;
  constexpr int SP = (S + 3) / 4 * 4;  // boundary words per column (uint4 aligned)
  const int sl = threadIdx.x & 31;
  const int64_t warp = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  if (warp >= a.streams) return;  // uniform per warp
  const int64_t stream = warp;
  const int64_t Gs = a.base + (stream < a.rem ? 1 : 0);
  const int64_t gb = stream * a.base + (stream < a.rem ? stream : a.rem);
  const int stripes = a.stripes;
  const int64_t units = Gs * stripes;
  const uint32_t nz = opaque(sl != 0 ? 1u : 0u);
  uint32_t* bnd = a.bnd + stream * int64_t(a.n) * SP;  // [n][SP] of this stream
  const uint32_t* zero = a.bzero;                      // SP zero words

  uint32_t kill[R];
  uint32_t H[R][S], dtop[S], M[S], bnext[S];
#pragma unroll
  for (int i = 0; i < S; ++i) {
    dtop[i] = 0;
    M[i] = 0;
    bnext[i] = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) H[r][i] = 0;
  }
#pragma unroll
  for (int r = 0; r < R; ++r) kill[r] = 0;
  uint32_t xh[R], xl[R];
  __shared__ uint2 xring[4][2][32][R];  // next unit's query planes (cp.async)
  uint2 (*ring)[32][R] = xring[threadIdx.x >> 5];
  auto fetch_x = [&](int64_t u) {  // query planes of unit u (clamped) -> slot u & 1
    const int slot = int(u & 1);
    u = u < units ? u : units - 1;
    const int64_t g = gb + u / stripes;
    const int kk = int(u % stripes);
    const uint2* xp = a.Xp + g * a.m + kk * LR + sl * R;
#pragma unroll
    for (int r = 0; r < R; ++r) cp_async8(&ring[slot][sl][r], xp + r);
    cp_async_commit();
  };
  fetch_x(0);
#pragma unroll
  for (int r = 0; r < R; ++r) xh[r] = xl[r] = 0;
  const uint2* ycol = a.Yp;  // my current target column (valid dummy before unit 0)
  uint2 ynext = __ldg(ycol);
  uint2 yfirst = __ldg(a.Yp + gb * a.n);  // column 0 of my next unit
  const uint32_t* bcol = zero;  // boundary column I load next (lane 0 only)
  int bstep = 0;                // words to advance bcol per step (SP or 0)
  bool store_bnd = false;       // last lane, not the last stripe
  int cnt = sl;
  int64_t vi = -1;
  uint32_t flag = 0;  // threshold mode

  for (int64_t tau = 0; tau < a.steps; ++tau) {
    uint32_t up[S];
#pragma unroll
    for (int i = 0; i < S; ++i)
      up[i] = mad_lo(__shfl_up_sync(0xFFFFFFFFu, H[R - 1][i], 1), nz, bnext[i]);
    uint2 y;
    if (cnt == 0) {  // column 0 of my next unit (divergent, once per unit)
      if (vi >= 0 && vi < units) {
        const int64_t g = gb + vi / stripes;
        const int kk = int(vi % stripes);
        if constexpr (BPBC_MODE == kModeThreshold) {
          a.Mpart[(g * stripes + kk) * L + sl] = flag;
        } else {
          uint32_t* dst = a.Mpart + ((g * stripes + kk) * L + sl) * S;
          // exact circuit: M tracked D' = diag + w + g; extract subtracts g
#pragma unroll
          for (int i = 0; i < S; ++i) dst[i] = M[i];
        }
      }
      ++vi;
      flag = 0;
      const int64_t uc = vi < units ? vi : units - 1;
      const int64_t g = gb + uc / stripes;
      const int kk = int(uc % stripes);
#pragma unroll
      for (int i = 0; i < S; ++i) {
        M[i] = 0;
        dtop[i] = 0;
#pragma unroll
        for (int r = 0; r < R; ++r) H[r][i] = 0;
      }
      cp_async_wait_all();
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint2 v = ring[vi & 1][sl][r];
        xh[r] = v.x;
        xl[r] = v.y;
        kill[r] = (kk * LR + sl * R + r >= a.m) ? 0xFFFFFFFFu : 0u;
      }
      fetch_x(vi + 1);
      ycol = a.Yp + g * a.n;
      y = yfirst;
      {
        const int64_t un = vi + 1 < units ? vi + 1 : units - 1;
        yfirst = __ldg(a.Yp + (gb + un / stripes) * a.n);
      }
      const bool from_bnd = sl == 0 && kk > 0;
      bcol = from_bnd ? bnd : zero;
      bstep = from_bnd ? SP : 0;
      store_bnd = sl == L - 1 && kk + 1 < stripes;
      if (from_bnd) {  // column 0 of a lower stripe: up = boundary row 0
#pragma unroll
        for (int i = 0; i < S; ++i) up[i] = __ldcg(bnd + i);
      }
      cnt = a.n;
    } else {
      y = ynext;
      ++ycol;
    }
    --cnt;
    ynext = __ldg(ycol + 1);
    // boundary row for the next step (lane 0 of stripes > 0; zeros otherwise;
    // column 0 of a unit is loaded at the switch instead)
    {
      const uint32_t* bp = bcol + (cnt > 0 ? bstep : 0);
      const uint4* b4 = reinterpret_cast<const uint4*>(cnt > 0 ? bp : zero);
#pragma unroll
      for (int q = 0; q < SP / 4; ++q) {
        const uint4 v = __ldcg(b4 + q);
        if (4 * q + 0 < S) bnext[4 * q + 0] = v.x;
        if (4 * q + 1 < S) bnext[4 * q + 1] = v.y;
        if (4 * q + 2 < S) bnext[4 * q + 2] = v.z;
        if (4 * q + 3 < S) bnext[4 * q + 3] = v.w;
      }
      bcol = bp;
    }

    uint32_t dg[S], u[S];
#pragma unroll
    for (int i = 0; i < S; ++i) {
      dg[i] = dtop[i];
      u[i] = up[i];
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t hn[S], dn[S];
      if constexpr (CIRC == kExact) {
        cell_exact<S, K, false>(u, H[r], dg, xh[r], xl[r], y.x, y.y, 0u, hn, dn, k);
      } else {
        cell_sat<S, K>(u, H[r], dg, xh[r], xl[r], y.x, y.y, hn, dn, k);
      }
      if constexpr (BPBC_MODE == kModeThreshold) {
        flag_gt<S, true>(flag, dn, a.tmask, kill[r]);
      } else {
        runmax<S, true>(M, dn, kill[r]);
      }
#pragma unroll
      for (int i = 0; i < S; ++i) {
        dg[i] = H[r][i];
        H[r][i] = hn[i];
        u[i] = hn[i];
      }
    }
#pragma unroll
    for (int i = 0; i < S; ++i) dtop[i] = up[i];
    if (store_bnd) {  // my bottom row at this column, for the next stripe
      uint4* d4 = reinterpret_cast<uint4*>(bnd + (int64_t(a.n) - 1 - cnt) * SP);
#pragma unroll
      for (int q = 0; q < SP / 4; ++q) {
        uint4 v;
        v.x = 4 * q + 0 < S ? H[R - 1][4 * q + 0] : 0u;
        v.y = 4 * q + 1 < S ? H[R - 1][4 * q + 1] : 0u;
        v.z = 4 * q + 2 < S ? H[R - 1][4 * q + 2] : 0u;
        v.w = 4 * q + 3 < S ? H[R - 1][4 * q + 3] : 0u;
        __stcg(d4 + q, v);
      }
    }
    __syncwarp();  // orders the boundary store before lane 0's later load
  }
}

// ---------------------------------------------------------------------------
// Multi-warp groups: the W warps of a block share one group stream and warp w
// owns rows [w*32R, (w+1)*32R) of every group, running kMwLag steps behind
// warp w-1 (lane l of warp w works on column J = tau - l - w*kMwLag).  The
// bottom row of warp w (its lane 31) reaches lane 0 of warp w+1 through a
// ring of kMwRing columns in shared memory; a __syncthreads every 32 steps
// orders the writes before the reads: a column is read kMwLag - 31 = 33 steps
// (more than one 32-step phase) after it is written, and its slot is rewritten
// kMwRing - 33 = 95 steps after the read.  Used when a group's rows exceed one
// warp (m > 256, or wide planes) and to put more warps on few long groups (the
// paper's shape).  Same circuits and wavefront as the single-warp kernel.
constexpr int kMwLag = 64, kMwRing = kMwRingCols, kMwSP = kMwRingWords;  // boundary words per column (padded)

// Resident warps per SM the register budget is sized for: 16 (128 registers)
// while R*S <= 36 planes of row state; 12 (168 registers) up to 44, where 128
// registers cost more in schedule than a fourth warp per SMSP gains (C5 point,
// m = 512 at 11 bits: 4 751 vs 4 620 GCUPS; 9 bits: 16 warps 0.3 % faster);
// above that the register count decides.
template <int S, int R, int W>
constexpr int mw_min_blocks() {
  return R * S <= 36   ? 16 / (W * mw_groups_per_block(W))
         : R * S <= 44 ? 12 / (W * mw_groups_per_block(W))
                       : 1;
}

template <int S, int R, int W, int CIRC, class K>
__global__ void __launch_bounds__(32 * W * mw_groups_per_block(W), (mw_min_blocks<S, R, W>()))
    sw_sweep_mw_kernel(const SweepArgs a, const K k) {
  constexpr int LR = 32 * R;
  constexpr int GPB = mw_groups_per_block(W);  // group streams per block
  static_assert(GPB <= 4, "named barriers 1..4");
  static_assert(S <= kMwSP, "boundary row holds up to 16 planes");
  const int lane = threadIdx.x & 31;
  const int gib = (threadIdx.x >> 5) / W;  // group stream of this warp within the block
  const int wk = (threadIdx.x >> 5) % W;   // row block of this warp
  const int64_t stream = int64_t(blockIdx.x) * GPB + gib;

  // dynamic shared memory (mw_smem_bytes): [GPB][W-1][ring][SP] boundary rings,
  // then [GPB][W][2][32][R] query-plane rings
  extern __shared__ __align__(16) uint8_t mw_smem[];
  __shared__ __align__(16) uint32_t bzero[kMwSP];
  using Ring = uint32_t[W - 1][kMwRing][kMwSP];
  using XRing = uint2[W][2][32][R];
  Ring& bring = reinterpret_cast<Ring*>(mw_smem)[gib];
  XRing& xring = reinterpret_cast<XRing*>(mw_smem + GPB * sizeof(Ring))[gib];
  static_assert(GPB * (sizeof(Ring) + sizeof(XRing)) == mw_smem_bytes(R, W), "smem layout");
  if (threadIdx.x < kMwSP) bzero[threadIdx.x] = 0;
  __syncthreads();
  if (stream >= a.streams) return;  // uniform per group (its barrier is its own)
  const int64_t Gs = a.base + (stream < a.rem ? 1 : 0);
  const int64_t gb = stream * a.base + (stream < a.rem ? stream : a.rem);

  const uint32_t nz = opaque(lane != 0 ? 1u : 0u);
  const uint32_t z0 = opaque(uint32_t(a.m) >> 31);  // 0: state reset on the FMA pipe
  const int row0 = wk * LR + lane * R;
  uint32_t kill[R];
#pragma unroll
  for (int r = 0; r < R; ++r) kill[r] = opaque(row0 + r >= a.m ? 0xFFFFFFFFu : 0u);
  // lane 0 of warps > 0 reads the ring of warp wk-1 (mask keeps the others on
  // the zero row); lane 31 of warps < W-1 writes its own ring
  const bool reader = lane == 0 && wk > 0;
  const uint32_t* rbase = reader ? &bring[wk - 1][0][0] : bzero;
  const uint32_t rmask = reader ? uint32_t(kMwRing * kMwSP - 1) : 0u;
  const bool writer = lane == 31 && wk + 1 < W;
  uint32_t* wbase = &bring[wk < W - 1 ? wk : 0][0][0];
  // ring offset (words) of my current column J: (J mod kMwRing) * kMwSP
  uint32_t off = uint32_t(-(lane + wk * kMwLag)) * kMwSP;

  uint32_t H[R][S], dtop[S], M[S];
#pragma unroll
  for (int i = 0; i < S; ++i) {
    dtop[i] = 0;
    M[i] = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) H[r][i] = 0;
  }
  uint2 (*ring)[32][R] = xring[wk];
  uint32_t xh[R], xl[R];
  auto fetch_x = [&](int64_t gidx, int slot) {
    int64_t g = gb + gidx;
    g = g < a.G ? g : a.G - 1;
    const uint2* xp = a.Xp + g * a.m + row0;
#pragma unroll
    for (int r = 0; r < R; ++r) cp_async8(&ring[slot][lane][r], xp + r);
    cp_async_commit();
  };
  fetch_x(0, 0);
#pragma unroll
  for (int r = 0; r < R; ++r) xh[r] = xl[r] = 0;
  const uint2* yp = a.Yp + gb * a.n - lane - wk * kMwLag;
  int cnt = lane + wk * kMwLag;
  int64_t gi = -1;
  uint32_t flag = 0;

  auto step = [&](const uint2 y, auto SW) {  // SW: as in sw_sweep_kernel
    uint32_t up[S];
    {
      const uint4* b4 = reinterpret_cast<const uint4*>(rbase + (off & rmask));
#pragma unroll
      for (int q = 0; q < (S + 3) / 4; ++q) {
        const uint4 v = b4[q];
        const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (4 * q + e < S)
            up[4 * q + e] = mad_lo(__shfl_up_sync(0xFFFFFFFFu, H[R - 1][4 * q + e], 1), nz, w[e]);
      }
    }
    if (decltype(SW)::value && cnt == 0) {  // column 0 of my next group (divergent, once per group)
      if (gi >= 0 && gi < Gs) {
        if constexpr (BPBC_MODE == kModeThreshold) {
          a.Mpart[((gb + gi) * W + wk) * 32 + lane] = flag;
        } else {
          uint32_t* dst = a.Mpart + (((gb + gi) * W + wk) * 32 + lane) * S;
          // exact circuit: M tracked D' = diag + w + g; extract subtracts g
#pragma unroll
          for (int i = 0; i < S; ++i) dst[i] = M[i];
        }
      }
      ++gi;
      flag = mul_lo(flag, z0);
#pragma unroll
      for (int i = 0; i < S; ++i) {
        M[i] = mul_lo(M[i], z0);
        dtop[i] = mul_lo(dtop[i], z0);
#pragma unroll
        for (int r = 0; r < R; ++r) H[r][i] = mul_lo(H[r][i], z0);
      }
      cp_async_wait_all();
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const uint2 v = ring[gi & 1][lane][r];
        xh[r] = v.x;
        xl[r] = v.y;
      }
      fetch_x(gi + 1, int((gi + 1) & 1));
      cnt = a.n;
    }
    if (decltype(SW)::value) --cnt;
    uint32_t dg[S], u[S];
#pragma unroll
    for (int i = 0; i < S; ++i) {
      dg[i] = dtop[i];
      u[i] = up[i];
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      uint32_t hn[S], dn[S];
      if constexpr (CIRC == kExact) {
        cell_exact<S, K, false>(u, H[r], dg, xh[r], xl[r], y.x, y.y, 0u, hn, dn, k);
      } else {
        cell_sat<S, K>(u, H[r], dg, xh[r], xl[r], y.x, y.y, hn, dn, k);
      }
      if constexpr (BPBC_MODE == kModeThreshold) {
        flag_gt<S, true>(flag, dn, a.tmask, kill[r]);
      } else {
        runmax<S, true>(M, dn, kill[r]);
      }
#pragma unroll
      for (int i = 0; i < S; ++i) {
        dg[i] = H[r][i];
        H[r][i] = hn[i];
        u[i] = hn[i];
      }
    }
#pragma unroll
    for (int i = 0; i < S; ++i) dtop[i] = up[i];
    if (writer) {  // my bottom row at this column, for the next warp's lane 0
      uint4* d4 = reinterpret_cast<uint4*>(wbase + (off & uint32_t(kMwRing * kMwSP - 1)));
#pragma unroll
      for (int q = 0; q < (S + 3) / 4; ++q) {
        uint4 v;
        v.x = 4 * q + 0 < S ? H[R - 1][4 * q + 0] : 0u;
        v.y = 4 * q + 1 < S ? H[R - 1][4 * q + 1] : 0u;
        v.z = 4 * q + 2 < S ? H[R - 1][4 * q + 2] : 0u;
        v.w = 4 * q + 3 < S ? H[R - 1][4 * q + 3] : 0u;
        d4[q] = v;
      }
    }
    off += kMwSP;
  };

  uint2 y0 = __ldg(yp), y1;
  for (int64_t tau = 0; tau < a.steps; tau += 32) {
    if (__any_sync(0xFFFFFFFFu, cnt < 32)) {  // a lane of this warp switches groups
#pragma unroll 1
      for (int i = 0; i < 32; i += 2) {
        y1 = __ldg(yp + tau + i + 1);
        step(y0, std::true_type{});
        y0 = __ldg(yp + tau + i + 2);
        step(y1, std::true_type{});
      }
    } else {
#pragma unroll 1
      for (int i = 0; i < 32; i += 2) {
        y1 = __ldg(yp + tau + i + 1);
        step(y0, std::false_type{});
        y0 = __ldg(yp + tau + i + 2);
        step(y1, std::false_type{});
      }
      cnt -= 32;
    }
    // phase boundary: ring writes of this phase -> reads of the next (a named
    // barrier per group stream, so the groups of a block do not wait on each other)
    if (GPB == 1 || gib == 0) {  // literal barrier ids: ptxas reserves only these
      asm volatile("bar.sync 1, %0;" ::"n"(32 * W) : "memory");
    } else if (GPB == 2 || gib == 1) {
      asm volatile("bar.sync 2, %0;" ::"n"(32 * W) : "memory");
    } else if (gib == 2) {
      asm volatile("bar.sync 3, %0;" ::"n"(32 * W) : "memory");
    } else {
      asm volatile("bar.sync 4, %0;" ::"n"(32 * W) : "memory");
    }
  }
}

template <int S, int R, int W, int CIRC, class K>
void launch_mw(const SweepArgs& a, const KRun& kr, int grid, int block, cudaStream_t st) {
  // (the dispatch raised the kernel's dynamic shared memory limit, api.cu)
  constexpr int smem = mw_smem_bytes(R, W);
  if constexpr (K::kFixed) {
    sw_sweep_mw_kernel<S, R, W, CIRC, K><<<grid, block, smem, st>>>(a, K{});
  } else {
    sw_sweep_mw_kernel<S, R, W, CIRC, KRun><<<grid, block, smem, st>>>(a, kr);
  }
}

template <int S, int MV>
void reg_mw(SweepEntry (*mtab)[kNumKinds][13]) {
  constexpr int R = kMwR[MV], W = kMwW[MV];
  using K211 = KFix<2, 1, 1>;
  mtab[MV][0][S - 4] = {&launch_mw<S, R, W, kExact, K211>,
                        (const void*)&sw_sweep_mw_kernel<S, R, W, kExact, K211>};
  mtab[MV][1][S - 4] = {&launch_mw<S, R, W, kSat, K211>,
                        (const void*)&sw_sweep_mw_kernel<S, R, W, kSat, K211>};
  mtab[MV][2][S - 4] = {&launch_mw<S, R, W, kSat, KRun>,
                        (const void*)&sw_sweep_mw_kernel<S, R, W, kSat, KRun>};
  mtab[MV][3][S - 4] = {&launch_mw<S, R, W, kExact, KRun>,
                        (const void*)&sw_sweep_mw_kernel<S, R, W, kExact, KRun>};
}

template <int S, int R, int L, int CIRC, bool PAD, class K, bool HS = false>
void launch_sweep(const SweepArgs& a, const KRun& kr, int grid, int block, cudaStream_t st) {
  if constexpr (K::kFixed) {
    sw_sweep_kernel<S, R, L, CIRC, PAD, K, HS><<<grid, block, 0, st>>>(a, K{});
  } else {
    sw_sweep_kernel<S, R, L, CIRC, PAD, KRun, HS><<<grid, block, 0, st>>>(a, kr);
  }
}

// host-streamed instantiations (exact (+2,-1,-1) circuit, running max):
// htab[pad][rl][S - 4]
template <int S, int RL, bool PAD>
void reg_hs(SweepEntry (*htab)[kNumRL][13]) {
  constexpr int R = kRLR[RL], L = kRLL[RL];
  using K211 = KFix<2, 1, 1>;
  htab[PAD ? 1 : 0][RL][S - 4] = {&launch_sweep<S, R, L, kExact, PAD, K211, true>,
                                 (const void*)&sw_sweep_kernel<S, R, L, kExact, PAD, K211, true>};
}

template <int S, int CIRC, class K, int R>
void launch_striped(const SweepArgs& a, const KRun& kr, int grid, int block, cudaStream_t st) {
  if constexpr (K::kFixed) {
    sw_sweep_striped_kernel<S, CIRC, K, R><<<grid, block, 0, st>>>(a, K{});
  } else {
    sw_sweep_striped_kernel<S, CIRC, KRun, R><<<grid, block, 0, st>>>(a, kr);
  }
}

template <int S>
void reg_striped(SweepEntry (*stab)[13]) {
  constexpr int R = kStripeR;
  using K211 = KFix<2, 1, 1>;
  stab[0][S - 4] = {&launch_striped<S, kExact, K211, R>,
                    (const void*)&sw_sweep_striped_kernel<S, kExact, K211, R>};
  stab[1][S - 4] = {&launch_striped<S, kSat, K211, R>,
                    (const void*)&sw_sweep_striped_kernel<S, kSat, K211, R>};
  stab[2][S - 4] = {&launch_striped<S, kSat, KRun, R>,
                    (const void*)&sw_sweep_striped_kernel<S, kSat, KRun, R>};
  stab[3][S - 4] = {&launch_striped<S, kExact, KRun, R>,
                    (const void*)&sw_sweep_striped_kernel<S, kExact, KRun, R>};
}

template <int S, int R, int L, int CIRC, bool PAD, class K>
void launch_planes(const SweepArgs& a, const KRun& kr, int grid, int block, cudaStream_t st) {
  if constexpr (K::kFixed) {
    sw_sweep_planes_kernel<S, R, L, CIRC, PAD, K><<<grid, block, 0, st>>>(a, K{});
  } else {
    sw_sweep_planes_kernel<S, R, L, CIRC, PAD, KRun><<<grid, block, 0, st>>>(a, kr);
  }
}

template <int S, int RL, bool PAD>
void reg_planes(SweepEntry (*ptab)[2][13]) {
  constexpr int R = kRLR[RL], L = kRLL[RL];
  using K211 = KFix<2, 1, 1>;
  ptab[variant_index(kExact, kC211, PAD)][RL][S - 4] = {
      &launch_planes<S, R, L, kExact, PAD, K211>,
      (const void*)&sw_sweep_planes_kernel<S, R, L, kExact, PAD, K211>};
  ptab[variant_index(kSat, kC211, PAD)][RL][S - 4] = {
      &launch_planes<S, R, L, kSat, PAD, K211>,
      (const void*)&sw_sweep_planes_kernel<S, R, L, kSat, PAD, K211>};
  ptab[variant_index(kSat, kCRun, PAD)][RL][S - 4] = {
      &launch_planes<S, R, L, kSat, PAD, KRun>,
      (const void*)&sw_sweep_planes_kernel<S, R, L, kSat, PAD, KRun>};
  ptab[variant_index(kExact, kCRun, PAD)][RL][S - 4] = {
      &launch_planes<S, R, L, kExact, PAD, KRun>,
      (const void*)&sw_sweep_planes_kernel<S, R, L, kExact, PAD, KRun>};
}

template <int S, int R, int CIRC, bool PAD, class K>
void launch_wrap(const SweepArgs& a, const KRun& kr, int grid, int block, cudaStream_t st) {
  if constexpr (K::kFixed) {
    sw_sweep_wrap_kernel<S, R, CIRC, PAD, K><<<grid, block, 0, st>>>(a, K{});
  } else {
    sw_sweep_wrap_kernel<S, R, CIRC, PAD, KRun><<<grid, block, 0, st>>>(a, kr);
  }
}

// wrap-around kernels for the L = 32 tilings: wtab[variant][rl - 2][S - 4]
template <int S, int RL, bool PAD>
void reg_wrap(SweepEntry (*wtab)[2][13]) {
  static_assert(RL >= 2, "wrap-around schedule: L = 32 tilings only");
  constexpr int R = kRLR[RL];
  using K211 = KFix<2, 1, 1>;
  wtab[variant_index(kExact, kC211, PAD)][RL - 2][S - 4] = {
      &launch_wrap<S, R, kExact, PAD, K211>, (const void*)&sw_sweep_wrap_kernel<S, R, kExact, PAD, K211>};
  wtab[variant_index(kSat, kC211, PAD)][RL - 2][S - 4] = {
      &launch_wrap<S, R, kSat, PAD, K211>, (const void*)&sw_sweep_wrap_kernel<S, R, kSat, PAD, K211>};
  wtab[variant_index(kSat, kCRun, PAD)][RL - 2][S - 4] = {
      &launch_wrap<S, R, kSat, PAD, KRun>, (const void*)&sw_sweep_wrap_kernel<S, R, kSat, PAD, KRun>};
  if constexpr (!(RL == 3 && S >= 13)) {
    wtab[variant_index(kExact, kCRun, PAD)][RL - 2][S - 4] = {
        &launch_wrap<S, R, kExact, PAD, KRun>, (const void*)&sw_sweep_wrap_kernel<S, R, kExact, PAD, KRun>};
  }
}

template <int S, int RL, bool PAD>
void reg_rl(SweepEntry (*tab)[kNumRL][13]) {
  constexpr int R = kRLR[RL], L = kRLL[RL];
  using K211 = KFix<2, 1, 1>;
  tab[variant_index(kExact, kC211, PAD)][RL][S - 4] = {
      &launch_sweep<S, R, L, kExact, PAD, K211>,
      (const void*)&sw_sweep_kernel<S, R, L, kExact, PAD, K211>};
  tab[variant_index(kSat, kC211, PAD)][RL][S - 4] = {
      &launch_sweep<S, R, L, kSat, PAD, K211>,
      (const void*)&sw_sweep_kernel<S, R, L, kSat, PAD, K211>};
  tab[variant_index(kSat, kCRun, PAD)][RL][S - 4] = {
      &launch_sweep<S, R, L, kSat, PAD, KRun>,
      (const void*)&sw_sweep_kernel<S, R, L, kSat, PAD, KRun>};
  // exact circuit with runtime constants (g >= c2; single-warp plans only)
  if constexpr (!(RL == 3 && S >= 13)) {
    tab[variant_index(kExact, kCRun, PAD)][RL][S - 4] = {
        &launch_sweep<S, R, L, kExact, PAD, KRun>,
        (const void*)&sw_sweep_kernel<S, R, L, kExact, PAD, KRun>};
  }
}

}  // namespace

#define BPBC_CAT2(a, b) a##b
#define BPBC_CAT(a, b) BPBC_CAT2(a, b)
#define BPBC_REGNAME BPBC_CAT(BPBC_CAT(BPBC_CAT(register_sweep_s, BPBC_S), _m), BPBC_MODE)
void BPBC_REGNAME(SweepEntry (*tab)[kNumRL][13], SweepEntry (*stab)[13],
                  SweepEntry (*mtab)[kNumKinds][13], SweepEntry (*ptab)[2][13],
                  SweepEntry (*wtab)[2][13], SweepEntry (*htab)[kNumRL][13]) {
#if BPBC_MODE == 0
  reg_hs<BPBC_S, 0, false>(htab);
  reg_hs<BPBC_S, 1, false>(htab);
  reg_hs<BPBC_S, 2, false>(htab);
  reg_hs<BPBC_S, 3, false>(htab);
  reg_hs<BPBC_S, 0, true>(htab);
  reg_hs<BPBC_S, 1, true>(htab);
  reg_hs<BPBC_S, 2, true>(htab);
  reg_hs<BPBC_S, 3, true>(htab);
#else
  (void)htab;
#endif
  reg_wrap<BPBC_S, 2, false>(wtab);
  reg_wrap<BPBC_S, 2, true>(wtab);
  reg_wrap<BPBC_S, 3, false>(wtab);
  reg_wrap<BPBC_S, 3, true>(wtab);
  reg_planes<BPBC_S, 0, false>(ptab);
  reg_planes<BPBC_S, 1, false>(ptab);
  reg_planes<BPBC_S, 0, true>(ptab);
  reg_planes<BPBC_S, 1, true>(ptab);
  reg_mw<BPBC_S, 0>(mtab);
  reg_mw<BPBC_S, 1>(mtab);
  reg_mw<BPBC_S, 2>(mtab);
  reg_rl<BPBC_S, 0, false>(tab);
  reg_rl<BPBC_S, 1, false>(tab);
  reg_rl<BPBC_S, 2, false>(tab);
  reg_rl<BPBC_S, 3, false>(tab);
  reg_rl<BPBC_S, 0, true>(tab);
  reg_rl<BPBC_S, 1, true>(tab);
  reg_rl<BPBC_S, 2, true>(tab);
  reg_rl<BPBC_S, 3, true>(tab);
  reg_striped<BPBC_S>(stab);
}

}  // namespace bpbc
