// api.cu -- the C ABI (include/bpbc_sw.h): validation, workspace layout,
// circuit/width/tiling plan, kernel dispatch, host-buffer path.
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>
#include <new>
#include <vector>

#include "bpbc_internal.cuh"

struct bpbc_sw_ctx {
  int device = 0;
  int num_sms = 0;
  uint32_t* d_flags = nullptr;
  void* ws = nullptr;  // ctx-owned device workspace
  size_t ws_bytes = 0;
  // host path buffers
  uint8_t* d_q = nullptr;
  uint8_t* d_t = nullptr;
  int32_t* d_out = nullptr;
  size_t d_q_bytes = 0, d_t_bytes = 0, d_out_bytes = 0;
  // host path: two streams, chunk c of the batch runs on stream c % 2 with
  // its own workspace, so chunk c+1's H2D overlaps chunk c's kernels
  cudaStream_t host_streams[2] = {nullptr, nullptr};
  void* ws_h[2] = {nullptr, nullptr};
  void* fscratch = nullptr;  // filter compaction scratch (grown lazily)
  size_t fscratch_bytes = 0;
  size_t ws_h_bytes[2] = {0, 0};
  char err[512] = {0};
  // last plan
  int32_t plan_circuit = -1, plan_width = 0, plan_R = 0, plan_L = 0, plan_ops = 0;
  int32_t plan_kernels = 0, plan_fused = 0;  // kernels the last call launched; fused sweep?
  int64_t plan_streams = 0;
  // phase profiling (bpbc_sw_profile): 4 events per recorded call
  bool profiling = false;
  std::vector<cudaEvent_t> ev_pool;   // all events ever created
  std::vector<cudaEvent_t> ev_used;   // recorded since last read, 4 per call
  cudaEvent_t take_event() {
    if (ev_used.size() < ev_pool.size()) {
      cudaEvent_t e = ev_pool[ev_used.size()];
      ev_used.push_back(e);
      return e;
    }
    cudaEvent_t e = nullptr;
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
    ev_pool.push_back(e);
    ev_used.push_back(e);
    return e;
  }
};

namespace bpbc {
namespace {

SweepEntry g_table[2][kNumVariants][kNumRL][13];  // [mode][variant][rl][S - 4]
SweepEntry g_striped[2][kNumKinds][13];           // [mode][kind][S - 4]
SweepEntry g_mw[2][kNumMw][kNumKinds][13];        // [mode][(R, W)][kind][S - 4]
SweepEntry g_planes[2][kNumVariants][2][13];      // [mode][variant][rl 0..1][S - 4]
std::once_flag g_table_once;

void init_table() {
  memset(g_table, 0, sizeof(g_table));
  memset(g_striped, 0, sizeof(g_striped));
  memset(g_mw, 0, sizeof(g_mw));
  memset(g_planes, 0, sizeof(g_planes));
#define BPBC_REG(S)                                      \
  register_sweep_s##S##_m0(g_table[0], g_striped[0], g_mw[0], g_planes[0]); \
  register_sweep_s##S##_m1(g_table[1], g_striped[1], g_mw[1], g_planes[1]);
  BPBC_REG(4)
  BPBC_REG(5)
  BPBC_REG(6)
  BPBC_REG(7)
  BPBC_REG(8)
  BPBC_REG(9)
  BPBC_REG(10)
  BPBC_REG(11)
  BPBC_REG(12)
  BPBC_REG(13)
  BPBC_REG(14)
  BPBC_REG(15)
  BPBC_REG(16)
#undef BPBC_REG
}

int bit_length(int64_t v) {
  int b = 0;
  while (v > 0) {
    ++b;
    v >>= 1;
  }
  return b;
}

int cuda_fail(bpbc_sw_ctx* ctx, cudaError_t e, const char* what) {
  if (ctx) snprintf(ctx->err, sizeof(ctx->err), "%s: %s", what, cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? BPBC_ERR_OOM : BPBC_ERR_CUDA;
}

// Workspace layout; sizes in bytes, all
// offsets 256-byte aligned.
struct Layout {
  int64_t G = 0;
  int stripes = 1;             // 32-lane partial slots per group (multi-warp / striped)
  int64_t bnd_streams = 0;     // streams the boundary buffer has room for
  int64_t x_off = 0, y_off = 0, mp_off = 0, bnd_off = 0, zero_off = 0, total = 0;
};

int64_t align256(int64_t v) { return (v + 255) & ~int64_t(255); }

Layout layout(int64_t P, int mq, int nt) {
  Layout L;
  L.G = (P + 31) / 32;
  // room for the striped / multi-warp kernels' partials: 32 lanes per 128 rows
  L.stripes = (mq + kStripeRows - 1) / kStripeRows;
  // the global boundary buffer is only used by the sequential striped kernel
  const bool may_stripe = mq > 512 || (mq > 128 && getenv("BPBC_NO_MULTIWARP"));
  const int64_t xbytes = (L.G * mq + kXBackPad) * 8;
  const int64_t ybytes = (kYFrontPad + L.G * nt + nt + kYBackPadExtra) * 8;
  const int64_t mpbytes = L.G * L.stripes * 32 * 16 * 4;
  int64_t bnd_bytes = 0;
  if (may_stripe) {
    const int64_t per_stream = int64_t(nt) * 16 * 4;  // [n][16 words] at most
    int64_t st = L.G < kMaxStripeStreams ? L.G : kMaxStripeStreams;
    if (st * per_stream > kMaxBoundaryBytes) st = kMaxBoundaryBytes / per_stream;
    if (st < 1) st = 1;
    L.bnd_streams = st;
    bnd_bytes = st * per_stream;
  }
  L.x_off = 0;
  L.y_off = align256(xbytes);
  L.mp_off = L.y_off + align256(ybytes);
  L.bnd_off = L.mp_off + align256(mpbytes);
  L.zero_off = L.bnd_off + align256(bnd_bytes);
  L.total = L.zero_off + 256;
  return L;
}

struct Plan {
  int circuit, consts, rl, width, cap;
  bool pad;
  int ops;
};


// Choose the circuit, the evaluated width and the tiling.
int make_plan(int mq, int c1, int c2, int g, int S, Plan* p) {
  if (mq <= 32) p->rl = 0;
  else if (mq <= 64) p->rl = 1;
  else if (mq <= 128) p->rl = 2;
  else if (mq <= kMaxShortRows) p->rl = 3;
  else if (mq <= BPBC_MAX_QUERY_LEN) p->rl = -1;  // striped long-query kernel
  else return BPBC_ERR_UNSUPPORTED;
  p->pad = p->rl < 0 || mq != kRLR[p->rl] * kRLL[p->rl];
  const bool wide_r8 = p->rl == 3;  // R = 8 rows per lane: register-heavy at large S
  p->cap = (1 << S) - 1;
  const bool spec = (c1 == 2 && c2 == 1 && g == 1);
  // width of the saturating circuit: no saturation can happen at or above
  // bit_length(c1*mq); the constants must fit.
  int cmax = c1 > c2 ? c1 : c2;
  cmax = cmax > g ? cmax : g;
  int s_sat = bit_length(int64_t(c1) * mq);
  if (s_sat < bit_length(cmax)) s_sat = bit_length(cmax);
  if (s_sat < BPBC_MIN_SCORE_BITS) s_sat = BPBC_MIN_SCORE_BITS;
  if (s_sat > S) s_sat = S;
  const int cost_sat = 11 * s_sat + 2;
  if (g >= c2) {
    // exact offset circuit at the width no value can exceed: compile-time
    // (+2,-1,-1) 10S LOP3, runtime constants 12S + 1; taken when cheaper
    // than the saturating circuit
    int s_ex = bit_length(int64_t(c1) * mq + g);
    if (s_ex < BPBC_MIN_SCORE_BITS) s_ex = BPBC_MIN_SCORE_BITS;
    const int cost_ex = spec ? 10 * s_ex : 12 * s_ex + 1;
    const int cost_sat_k = spec ? cost_sat : 13 * s_sat + 4;
    static const bool no_exact_run = [] {  // A/B knob: BPBC_NO_EXACT_RUN=1
      const char* v = getenv("BPBC_NO_EXACT_RUN");
      return v != nullptr && *v != '\0' && *v != '0';
    }();
    const bool runtime_ok = !no_exact_run;
    if (s_ex <= BPBC_MAX_SCORE_BITS && cost_ex <= cost_sat_k && (spec || runtime_ok)) {
      p->circuit = kExact;
      p->consts = spec ? kC211 : kCRun;
      p->width = s_ex;
      p->ops = cost_ex;
      if (wide_r8 && s_ex >= 13) {
        p->rl = -1;
        p->pad = true;
      }
      return BPBC_OK;
    }
  }
  p->circuit = kSat;
  p->consts = spec ? kC211 : kCRun;
  p->width = s_sat;
  if (wide_r8 && s_sat >= 13) {  // R = 8 x 13+ planes spills: use 128-row stripes
    p->rl = -1;
    p->pad = true;
  }
  p->ops = spec ? cost_sat : 13 * s_sat + 4;  // runtime masks: +S (w), +S (ssub), +2
  return BPBC_OK;
}

int validate_common(int64_t P, int m, int n, int match, int mismatch, int gap, int S) {
  if (P < 0 || m < 1 || n < 1) return BPBC_ERR_INVALID_ARG;
  if (S < BPBC_MIN_SCORE_BITS || S > BPBC_MAX_SCORE_BITS) return BPBC_ERR_UNSUPPORTED;
  if (match < 1 || mismatch > 0 || gap > 0) return BPBC_ERR_INVALID_ARG;
  const int64_t cap = (int64_t(1) << S) - 1;
  if (match > cap || -int64_t(mismatch) > cap || -int64_t(gap) > cap) return BPBC_ERR_INVALID_ARG;
  if (m > BPBC_MAX_LEN || n > BPBC_MAX_LEN) return BPBC_ERR_UNSUPPORTED;
  if ((m < n ? m : n) > BPBC_MAX_QUERY_LEN) return BPBC_ERR_UNSUPPORTED;
  return BPBC_OK;
}

// The sweep kernel a plan runs and how many group streams fit on the device.
struct Dispatch {
  Plan plan;
  SweepEntry ent;
  bool striped;
  bool fused = false;   // single-warp kernel reading raw codes (no pack pass)
  int mw = -1;          // multi-warp variant (index into kMwR / kMwW), -1 = none
  int R, L, W = 1;      // rows per lane, lanes per group, warps per group
  int64_t cap_streams;  // resident streams (before the boundary-buffer cap)
};

// Multi-warp variant for this plan, or -1: long queries up to
// 512 rows (R = 4, one warp per 128 rows) and the wide-plane 129..256 case.
int pick_mw(int mq, const Plan& p) {
  if (p.rl >= 0 || mq > 512) return -1;  // single-warp plan, or sequential stripes
  const int W = (mq + 127) / 128 < 2 ? 2 : (mq + 127) / 128;  // one warp per 128 rows
  for (int i = 0; i < kNumMw; ++i)
    if (kMwR[i] == 4 && kMwW[i] == W) return i;
  return -1;
}

// Cap on resident sweep blocks per SM: BPBC_MAX_BLOCKS_PER_SM in the
// environment (tuning knob for benchmarks; read once), else none.
int max_blocks_env() {
  static const int v = [] {
    const char* e = getenv("BPBC_MAX_BLOCKS_PER_SM");
    return e ? atoi(e) : 0;
  }();
  return v;
}

int occupancy_blocks(const void* func) {  // cached per kernel
  static std::mutex mu;
  static std::vector<std::pair<const void*, int>> cache;
  {
    std::lock_guard<std::mutex> lk(mu);
    for (auto& kv : cache)
      if (kv.first == func) return kv.second;
  }
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, func, 128, 0) != cudaSuccess) return -1;
  if (nb < 1) nb = 1;
  std::lock_guard<std::mutex> lk(mu);
  cache.emplace_back(func, nb);
  return nb;
}

int make_dispatch(bpbc_sw_ctx* ctx, int mq, int nt, int c1, int c2, int g, int S, Dispatch* d,
                  int mode = kModeMax, int64_t G = 0) {
  int rc = make_plan(mq, c1, c2, g, S, &d->plan);
  if (rc != BPBC_OK) return rc;
  std::call_once(g_table_once, init_table);
  const Plan& plan = d->plan;
  d->striped = plan.rl < 0;
  d->ent = d->striped
               ? g_striped[mode][kind_index(plan.circuit, plan.consts)]
                          [plan.width - 4]
               : g_table[mode][variant_index(plan.circuit, plan.consts, plan.pad)][plan.rl]
                        [plan.width - 4];
  // single-warp plans: the fused kernel unless the target is too short for
  // its phase-granular query transposes (n < L + 32, only for L = 16)
  if (!d->striped) {
    // (a query build per group must fall on a phase start between "every
    // lane entered the previous group" and "lane 0 needs it": some multiple
    // of 32 in [(h-1) n + L, h n] -- always when n >= L + 31, and at h n
    // itself when n is a multiple of 32)
    d->fused = nt >= kRLL[plan.rl] + 32 || nt % 32 == 0;
    if (!d->fused) {
      if (plan.rl > 1) return BPBC_ERR_UNSUPPORTED;  // (cannot happen: n >= m > 64)
      d->ent = g_planes[mode][variant_index(plan.circuit, plan.consts, plan.pad)][plan.rl]
                       [plan.width - 4];
    }
  }
  if (!d->ent.launch) return BPBC_ERR_UNSUPPORTED;
  d->R = d->striped ? kStripeR : kRLR[plan.rl];
  d->L = d->striped ? 32 : kRLL[plan.rl];
  int nb = occupancy_blocks(d->ent.func);
  if (nb < 0) return cuda_fail(ctx, cudaGetLastError(), "occupancy");
  if (max_blocks_env() > 0 && nb > max_blocks_env()) nb = max_blocks_env();
  d->cap_streams = int64_t(ctx->num_sms) * nb * 4 * (32 / d->L);
  d->mw = getenv("BPBC_NO_MULTIWARP") ? -1 : pick_mw(mq, plan);
  if (d->mw >= 0) {
    const SweepEntry e =
        g_mw[mode][d->mw][kind_index(plan.circuit, plan.consts)]
            [plan.width - 4];
    if (e.launch) {
      d->ent = e;
      d->striped = false;
      d->fused = false;
      d->R = kMwR[d->mw];
      d->W = kMwW[d->mw];
      d->L = 32;
      int nbm = 0;
      const int gpb = mw_groups_per_block(d->W);
      const int smem = mw_smem_bytes(d->R, d->W);
      if (cudaFuncSetAttribute(e.func, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) !=
              cudaSuccess ||
          cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nbm, e.func, 32 * d->W * gpb, smem) !=
              cudaSuccess)
        return cuda_fail(ctx, cudaGetLastError(), "occupancy");
      if (nbm < 1) nbm = 1;
      d->cap_streams = int64_t(ctx->num_sms) * nbm * gpb;  // gpb group streams per block
    } else {
      d->mw = -1;
    }
  }
  return BPBC_OK;
}

// What the sweep produces: max scores (extract) or threshold flags (filter).
struct RunOut {
  int32_t* scores = nullptr;     // max mode
  int mode = kModeMax;
  int threshold = 0;             // threshold mode: flag pairs with score > threshold
  uint32_t* mask = nullptr;      //   [ceil(P/32)] flag words
  int64_t* indices = nullptr;    //   optional ascending flagged pair indices
  int64_t* count = nullptr;      //   optional number of flagged pairs
  void* scratch = nullptr;       //   compaction scratch (filter_scratch_bytes)
  size_t scratch_bytes = 0;
};

// Enqueue pack -> sweep -> extract (or the filter epilogue) on device buffers.
int run_device(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target, int64_t P, int m,
               int n, int match, int mismatch, int gap, int S, const RunOut& o, uint8_t* ws,
               cudaStream_t st, bool packed2) {
  // score is symmetric (R17): the shorter sequence plays the query (rows)
  const uint8_t* qx = query;
  const uint8_t* ty = target;
  int mq = m, nt = n;
  if (m > n) {
    qx = target;
    ty = query;
    mq = n;
    nt = m;
  }
  const int c1 = match, c2 = -mismatch, g = -gap;
  Dispatch dsp;
  int rc = make_dispatch(ctx, mq, nt, c1, c2, g, S, &dsp, o.mode, (P + 31) / 32);
  if (rc != BPBC_OK) return rc;
  const Plan& plan = dsp.plan;
  const Layout lay = layout(P, mq, nt);
  uint2* Xp = reinterpret_cast<uint2*>(ws + lay.x_off);
  uint2* Ybase = reinterpret_cast<uint2*>(ws + lay.y_off);
  uint2* Yp = Ybase + kYFrontPad;
  uint32_t* Mpart = reinterpret_cast<uint32_t*>(ws + lay.mp_off);

  // The planes-reading sweeps read the pads around the planes (columns before
  // / after a stream's groups, rows past m) and discard what they compute
  // from them; zero them so those reads are of initialised memory.
  if (!dsp.fused) {
    cudaError_t ez = cudaMemsetAsync(Ybase, 0, size_t(kYFrontPad) * 8, st);
    if (ez == cudaSuccess)
      ez = cudaMemsetAsync(Yp + lay.G * nt, 0, size_t(nt + kYBackPadExtra) * 8, st);
    if (ez == cudaSuccess) ez = cudaMemsetAsync(Xp + lay.G * mq, 0, size_t(kXBackPad) * 8, st);
    if (ez != cudaSuccess) return cuda_fail(ctx, ez, "memset(pads)");
  }
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  if (ctx->profiling)
    for (int i = 0; i < 4; ++i) ev[i] = ctx->take_event();
  if (ev[0]) cudaEventRecord(ev[0], st);
  cudaError_t e = cudaSuccess;
  if (!dsp.fused) {  // the fused kernel transposes the raw codes itself
    e = launch_pack2(qx, mq, Xp, ty, nt, Yp, P, ctx->d_flags, ctx->num_sms, st, packed2);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "pack");
  }

  if (ev[1]) cudaEventRecord(ev[1], st);
  const bool striped = dsp.striped;
  const SweepEntry ent = dsp.ent;
  const int R = dsp.R, L = dsp.L, W = dsp.W;
  const bool mw = dsp.mw >= 0;
  const int64_t segs = mw ? 1 : 32 / L;
  int64_t cap_streams = dsp.cap_streams;
  if (striped && lay.bnd_streams < 1) return BPBC_ERR_UNSUPPORTED;  // (layout/plan mismatch)
  if (striped && cap_streams > lay.bnd_streams) cap_streams = lay.bnd_streams;
  SweepArgs a;
  a.Xp = Xp;
  a.Yp = Yp;
  a.Mpart = Mpart;
  a.G = lay.G;
  a.m = mq;
  a.n = nt;
  // Streams come in whole blocks on every SM (4 warps x 32/L streams per
  // block, b blocks per SM).  The SMs are ALU-bound, so an SM's time is its
  // total work, modelled as b * 4 * segs * ceil(G / streams) groups.  Pick b
  // in [nb - 1, nb] minimising that (ties -> more warps for latency hiding);
  // the streams then split the groups as evenly as possible (base / rem).
  // (A finer model of the base / rem split ties b = 4 and 5 at C4, where
  // b = 5 measured 5 % slower; this one picks the measured-better b at C2
  // and C4.)
  {
    const int64_t per_block = mw ? mw_groups_per_block(W) : 4 * segs;
    const int64_t nb = cap_streams / (int64_t(ctx->num_sms) * per_block);
    int64_t best_b = nb > 0 ? nb : 1, best_t = -1;
    for (int64_t b = nb; b >= 1 && b >= nb - 1; --b) {
      const int64_t st_b = int64_t(ctx->num_sms) * b * per_block;
      const int64_t t = b * per_block * ((lay.G + st_b - 1) / st_b);
      // fewer blocks only when they save more than 1 % of the work: more
      // resident warps hide more of the circuit's dependency latency
      if (best_t < 0 || t * 100 < best_t * 99) {
        best_t = t;
        best_b = b;
      }
    }
    int64_t cap_b = int64_t(ctx->num_sms) * best_b * per_block;
    if (nb < 1 || cap_b > cap_streams) cap_b = cap_streams;  // boundary-buffer cap
    a.streams = lay.G < cap_b ? lay.G : cap_b;
  }
  a.base = lay.G / a.streams;
  a.rem = lay.G % a.streams;
  a.stripes = striped ? (mq + 32 * R - 1) / (32 * R) : 1;
  a.qraw = qx;
  a.traw = ty;
  a.qstride = packed2 ? (int64_t(mq) + 3) / 4 : mq;
  a.tstride = packed2 ? (int64_t(nt) + 3) / 4 : nt;
  a.P = P;
  a.packed2 = packed2 ? 1 : 0;
  a.flags = ctx->d_flags;
  a.bnd = reinterpret_cast<uint32_t*>(ws + lay.bnd_off);
  a.bzero = reinterpret_cast<const uint32_t*>(ws + lay.zero_off);
  a.steps = (a.base + (a.rem > 0 ? 1 : 0)) * a.stripes * int64_t(nt) + L;
  if (mw) a.steps += int64_t(W - 1) * 64 + 31;  // warp lag (kMwLag), then whole phases
  a.steps += a.steps & 1;  // the short kernel runs two steps per iteration
  if (mw || dsp.fused) a.steps = (a.steps + 31) / 32 * 32;  // whole 32-step phases
  if (striped) {
    e = cudaMemsetAsync(ws + lay.zero_off, 0, 256, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset(zero row)");
  }
  const int64_t warps = (a.streams + segs - 1) / segs;
  const int gpb = mw ? mw_groups_per_block(W) : 1;
  const int grid = mw ? int((a.streams + gpb - 1) / gpb) : int((warps + 3) / 4);
  const int block = mw ? 32 * W * gpb : 128;
  KRun kr;
  memset(&kr, 0, sizeof(kr));
  const int Wd = plan.width;
  for (int i = 0; i < 16; ++i) {
    kr.c1mask[i] = (c1 >> i) & 1 ? 0xFFFFFFFFu : 0u;
    kr.nmask[i] = ((((1 << Wd) - c2) & ((1 << Wd) - 1)) >> i) & 1 ? 0xFFFFFFFFu : 0u;
    kr.gmask[i] = (g >> i) & 1 ? 0xFFFFFFFFu : 0u;
  }
  kr.zmask = c2 == 0 ? 0xFFFFFFFFu : 0u;
  for (int i = 0; i < 16; ++i) {  // exact circuit operands (used when g >= c2)
    kr.amask[i] = ((c1 + g) >> i) & 1 ? 0xFFFFFFFFu : 0u;
    kr.bmask[i] = g >= c2 && ((g - c2) >> i) & 1 ? 0xFFFFFFFFu : 0u;
  }
  // threshold mode compares the diagonal term with tau (+ g for the exact
  // circuit, whose D' carries the offset g)
  const int tcmp = o.threshold + (plan.circuit == kExact ? g : 0);
  for (int i = 0; i < 16; ++i) a.tmask[i] = (tcmp >> i) & 1 ? 0xFFFFFFFFu : 0u;
  ent.launch(a, kr, grid, block, st);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(ctx, e, "sweep");
  if (ev[2]) cudaEventRecord(ev[2], st);
  if (o.mode == kModeThreshold) {
    e = launch_filter_finish(Mpart, lay.G, L * a.stripes * W, P, o.mask, o.indices, o.count,
                             o.scratch, o.scratch_bytes, ctx->num_sms, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "filter epilogue");
  } else {
    // the exact circuit's partial maxima carry the offset g (finish_exact)
    e = launch_extract(Mpart, lay.G, L * a.stripes * W, plan.width, P,
                       plan.circuit == kExact ? g : 0, plan.cap, o.scores, ctx->num_sms, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "extract");
  }
  if (ev[3]) cudaEventRecord(ev[3], st);

  ctx->plan_circuit = plan.circuit;
  ctx->plan_width = Wd;
  ctx->plan_R = R;
  ctx->plan_L = L * W;  // lanes per group (over all its warps)
  ctx->plan_ops = plan.ops;
  ctx->plan_streams = a.streams;
  ctx->plan_fused = dsp.fused ? 1 : 0;
  ctx->plan_kernels = (dsp.fused ? 0 : 1) + 1 + (o.mode == kModeThreshold
                                                     ? ((o.indices || o.count) ? 2 : 1)
                                                     : 1);
  return BPBC_OK;
}

int ensure_ws(bpbc_sw_ctx* ctx, size_t need) {
  if (ctx->ws_bytes >= need) return BPBC_OK;
  if (ctx->ws) {
    cudaDeviceSynchronize();
    cudaFree(ctx->ws);
    ctx->ws = nullptr;
    ctx->ws_bytes = 0;
  }
  cudaError_t e = cudaMalloc(&ctx->ws, need);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaMalloc(workspace)");
  ctx->ws_bytes = need;
  return BPBC_OK;
}

int grow(bpbc_sw_ctx* ctx, void** p, size_t* have, size_t need, const char* what) {
  if (*have >= need) return BPBC_OK;
  if (*p) {
    cudaDeviceSynchronize();
    cudaFree(*p);
    *p = nullptr;
    *have = 0;
  }
  cudaError_t e = cudaMalloc(p, need);
  if (e != cudaSuccess) return cuda_fail(ctx, e, what);
  *have = need;
  return BPBC_OK;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace
}  // namespace bpbc

using namespace bpbc;

namespace {

int score_batch_impl(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                        int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                        int32_t mismatch, int32_t gap, int32_t score_bits, int32_t* out_scores,
                        void* workspace, size_t workspace_bytes, void* stream, bool packed2) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_scores) return BPBC_ERR_INVALID_ARG;
  size_t need = 0;
  bpbc_sw_workspace_bytes(num_pairs, m, n, &need);
  DeviceGuard dg(ctx->device);
  uint8_t* ws;
  if (workspace) {
    if (workspace_bytes < need) return BPBC_ERR_INVALID_ARG;
    ws = static_cast<uint8_t*>(workspace);
  } else {
    rc = ensure_ws(ctx, need);
    if (rc != BPBC_OK) return rc;
    ws = static_cast<uint8_t*>(ctx->ws);
  }
  RunOut o;
  o.scores = out_scores;
  return run_device(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits, o, ws,
                    static_cast<cudaStream_t>(stream), packed2);
}

int score_batch_host_impl(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                             int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                             int32_t mismatch, int32_t gap, int32_t score_bits,
                             int32_t* out_scores, bool packed2) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_scores) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaError_t e;
  for (int i = 0; i < 2; ++i) {
    if (!ctx->host_streams[i]) {
      e = cudaStreamCreateWithFlags(&ctx->host_streams[i], cudaStreamNonBlocking);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamCreate");
    }
  }
  // bytes per row: one per base, or 4 bases per byte (packed2)
  const int64_t qs = packed2 ? (int64_t(m) + 3) / 4 : m, ts = packed2 ? (int64_t(n) + 3) / 4 : n;
  const size_t qb = size_t(num_pairs) * qs, tb = size_t(num_pairs) * ts,
               ob = size_t(num_pairs) * sizeof(int32_t);
  // Chunks in whole "waves" (one group per resident sweep stream, so every
  // stream of a chunk gets the same number of groups), growing 1, 2, 4, ...
  // waves: the first copy is short, later chunks amortise the pipeline fill.
  Dispatch dsp;
  rc = make_dispatch(ctx, m < n ? m : n, m < n ? n : m, match, -mismatch, -gap, score_bits,
                     &dsp);
  if (rc != BPBC_OK) return rc;
  const int64_t wave_pairs = dsp.cap_streams * 32;
  // copy-bound (u8 rows: ~1 byte per base vs ~50 GB/s H2D) -> equal chunks so
  // the last chunk's kernels are short; compute-bound (packed2) -> growing
  // chunks so the first copy is short.  Estimate: H2D s/pair vs sweep s/pair.
  const double h2d_s = double(qs + ts) / 50e9, sweep_s = double(m) * n / 5e12;
  std::vector<int64_t> bounds{0};
  if (h2d_s >= sweep_s) {
    const int64_t waves = (num_pairs + wave_pairs - 1) / wave_pairs;
    const int64_t per = (waves + 7) / 8;  // about 8 chunks of whole waves
    while (bounds.back() < num_pairs) {
      const int64_t left = num_pairs - bounds.back();
      bounds.push_back(bounds.back() + (left < per * wave_pairs ? left : per * wave_pairs));
    }
  } else {
    for (int64_t w = 1; bounds.back() < num_pairs; w = w < 8 ? 2 * w : 8) {
      const int64_t left = num_pairs - bounds.back();
      // fold a short remainder (< 1 wave) into this chunk
      const int64_t take = left <= (w + 1) * wave_pairs ? left : w * wave_pairs;
      bounds.push_back(bounds.back() + take);
    }
  }
  int64_t chunk = 0;
  for (size_t i = 1; i < bounds.size(); ++i)
    chunk = bounds[i] - bounds[i - 1] > chunk ? bounds[i] - bounds[i - 1] : chunk;
  size_t need = 0;
  bpbc_sw_workspace_bytes(chunk, m, n, &need);
  if ((rc = grow(ctx, (void**)&ctx->d_q, &ctx->d_q_bytes, qb, "cudaMalloc(q)")) != BPBC_OK) return rc;
  if ((rc = grow(ctx, (void**)&ctx->d_t, &ctx->d_t_bytes, tb, "cudaMalloc(t)")) != BPBC_OK) return rc;
  if ((rc = grow(ctx, (void**)&ctx->d_out, &ctx->d_out_bytes, ob, "cudaMalloc(out)")) != BPBC_OK)
    return rc;
  for (int i = 0; i < 2; ++i)
    if ((rc = grow(ctx, &ctx->ws_h[i], &ctx->ws_h_bytes[i], need, "cudaMalloc(workspace)")) !=
        BPBC_OK)
      return rc;
  for (size_t ci = 0; ci + 1 < bounds.size(); ++ci) {
    const int64_t c0 = bounds[ci], cp = bounds[ci + 1] - bounds[ci];
    cudaStream_t st = ctx->host_streams[ci & 1];
    e = cudaMemcpyAsync(ctx->d_q + c0 * qs, query + c0 * qs, size_t(cp * qs),
                        cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(ctx->d_t + c0 * ts, target + c0 * ts, size_t(cp * ts),
                          cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "H2D");
    RunOut o;
    o.scores = ctx->d_out + c0;
    rc = run_device(ctx, ctx->d_q + c0 * qs, ctx->d_t + c0 * ts, cp, m, n, match, mismatch, gap,
                    score_bits, o, static_cast<uint8_t*>(ctx->ws_h[ci & 1]), st, packed2);
    if (rc != BPBC_OK) return rc;
    e = cudaMemcpyAsync(out_scores + c0, ctx->d_out + c0, size_t(cp) * sizeof(int32_t),
                        cudaMemcpyDeviceToHost, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "D2H");
  }
  for (int i = 0; i < 2; ++i) {
    e = cudaStreamSynchronize(ctx->host_streams[i]);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "sync");
  }
  return BPBC_OK;
}

}  // namespace


extern "C" {

const char* bpbc_sw_status_string(int status) {
  switch (status) {
    case BPBC_OK: return "ok";
    case BPBC_ERR_INVALID_ARG: return "invalid argument";
    case BPBC_ERR_UNSUPPORTED: return "unsupported by this build";
    case BPBC_ERR_CUDA: return "CUDA error";
    case BPBC_ERR_OOM: return "out of memory";
    case BPBC_ERR_BAD_BASE: return "base code > 3 in input";
    default: return "unknown status";
  }
}

const char* bpbc_sw_last_error(bpbc_sw_ctx* ctx) { return ctx ? ctx->err : ""; }

int bpbc_sw_init(int cuda_device, bpbc_sw_ctx** out_ctx) {
  if (!out_ctx) return BPBC_ERR_INVALID_ARG;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaGetDeviceCount");
  if (cuda_device < 0 || cuda_device >= ndev) return BPBC_ERR_INVALID_ARG;
  bpbc_sw_ctx* ctx = new (std::nothrow) bpbc_sw_ctx();
  if (!ctx) return BPBC_ERR_OOM;
  ctx->device = cuda_device;
  DeviceGuard dg(cuda_device);
  e = cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  if (e == cudaSuccess) e = cudaMalloc(&ctx->d_flags, sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMemset(ctx->d_flags, 0, sizeof(uint32_t));
  if (e != cudaSuccess) {
    int rc = cuda_fail(ctx, e, "init");
    if (ctx->d_flags) cudaFree(ctx->d_flags);
    delete ctx;
    return rc;
  }
  *out_ctx = ctx;
  return BPBC_OK;
}

int bpbc_sw_destroy(bpbc_sw_ctx* ctx) {
  if (!ctx) return BPBC_OK;
  DeviceGuard dg(ctx->device);
  cudaDeviceSynchronize();
  if (ctx->ws) cudaFree(ctx->ws);
  if (ctx->d_flags) cudaFree(ctx->d_flags);
  if (ctx->d_q) cudaFree(ctx->d_q);
  if (ctx->d_t) cudaFree(ctx->d_t);
  if (ctx->d_out) cudaFree(ctx->d_out);
  for (int i = 0; i < 2; ++i) {
    if (ctx->host_streams[i]) cudaStreamDestroy(ctx->host_streams[i]);
    if (ctx->ws_h[i]) cudaFree(ctx->ws_h[i]);
  }
  if (ctx->fscratch) cudaFree(ctx->fscratch);
  for (cudaEvent_t e : ctx->ev_pool) cudaEventDestroy(e);
  delete ctx;
  return BPBC_OK;
}

int bpbc_sw_workspace_bytes(int64_t num_pairs, int32_t m, int32_t n, size_t* bytes) {
  if (!bytes || num_pairs < 0 || m < 1 || n < 1) return BPBC_ERR_INVALID_ARG;
  if (m > BPBC_MAX_LEN || n > BPBC_MAX_LEN) return BPBC_ERR_UNSUPPORTED;
  const int mq = m < n ? m : n, nt = m < n ? n : m;
  *bytes = size_t(layout(num_pairs, mq, nt).total);
  return BPBC_OK;
}

int bpbc_sw_score_batch(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                        int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                        int32_t mismatch, int32_t gap, int32_t score_bits, int32_t* out_scores,
                        void* workspace, size_t workspace_bytes, void* stream) {
  return score_batch_impl(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits,
                          out_scores, workspace, workspace_bytes, stream, false);
}

int bpbc_sw_filter_batch(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                         int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                         int32_t mismatch, int32_t gap, int32_t score_bits, int32_t threshold,
                         uint32_t* out_mask, int64_t* out_indices, int64_t* out_count,
                         void* workspace, size_t workspace_bytes, void* stream) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  // "score > threshold" is decidable at width s only below the cap (R3)
  if (threshold < 0 || int64_t(threshold) > (int64_t(1) << score_bits) - 2)
    return BPBC_ERR_INVALID_ARG;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_mask) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int64_t G = (num_pairs + 31) / 32;
  const int mq = m < n ? m : n;
  if (int64_t(threshold) >= int64_t(match) * mq) {  // no local alignment can exceed it
    cudaError_t e = cudaMemsetAsync(out_mask, 0, size_t(G) * 4, st);
    if (e == cudaSuccess && out_count) e = cudaMemsetAsync(out_count, 0, 8, st);
    return e == cudaSuccess ? BPBC_OK : cuda_fail(ctx, e, "memset");
  }
  size_t need = 0;
  bpbc_sw_workspace_bytes(num_pairs, m, n, &need);
  uint8_t* ws;
  if (workspace) {
    if (workspace_bytes < need) return BPBC_ERR_INVALID_ARG;
    ws = static_cast<uint8_t*>(workspace);
  } else {
    rc = ensure_ws(ctx, need);
    if (rc != BPBC_OK) return rc;
    ws = static_cast<uint8_t*>(ctx->ws);
  }
  RunOut o;
  o.mode = kModeThreshold;
  o.threshold = threshold;
  o.mask = out_mask;
  o.indices = out_indices;
  o.count = out_count;
  if (out_indices || out_count) {
    rc = grow(ctx, &ctx->fscratch, &ctx->fscratch_bytes, filter_scratch_bytes(G),
              "cudaMalloc(filter scratch)");
    if (rc != BPBC_OK) return rc;
    o.scratch = ctx->fscratch;
    o.scratch_bytes = ctx->fscratch_bytes;
  }
  return run_device(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits, o, ws,
                    st, false);
}

int bpbc_sw_wordwise_workspace_bytes(int64_t num_pairs, size_t* bytes) {
  if (!bytes || num_pairs < 0) return BPBC_ERR_INVALID_ARG;
  *bytes = wordwise_workspace_bytes(num_pairs);
  return BPBC_OK;
}

int bpbc_sw_score_batch_wordwise(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                                 int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                                 int32_t mismatch, int32_t gap, int32_t* out_scores,
                                 void* workspace, size_t workspace_bytes, void* stream) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, BPBC_MAX_SCORE_BITS);
  if (rc != BPBC_OK) return rc;
  const int mq = m < n ? m : n, nt = m < n ? n : m;
  const int c2 = -mismatch, g = -gap, k0 = c2 > g ? c2 : g;
  if (mq > 256) return BPBC_ERR_UNSUPPORTED;                       // R <= 8 rows per lane
  if (int64_t(k0) + int64_t(match) * mq + match + c2 > 65535) return BPBC_ERR_UNSUPPORTED;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_scores) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  const size_t need = wordwise_workspace_bytes(num_pairs);
  void* ws = workspace;
  if (ws) {
    if (workspace_bytes < need) return BPBC_ERR_INVALID_ARG;
  } else {
    rc = ensure_ws(ctx, need);
    if (rc != BPBC_OK) return rc;
    ws = ctx->ws;
  }
  const uint8_t* qx = m <= n ? query : target;  // the shorter sequence plays the rows (R17)
  const uint8_t* ty = m <= n ? target : query;
  cudaError_t e = launch_wordwise(qx, ty, num_pairs, mq, nt, match, c2, g, out_scores, ws,
                                  ctx->num_sms, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? BPBC_OK : cuda_fail(ctx, e, "wordwise");
}

int bpbc_sw_score_batch_packed2(bpbc_sw_ctx* ctx, const uint8_t* query2, const uint8_t* target2,
                                int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                                int32_t mismatch, int32_t gap, int32_t score_bits,
                                int32_t* out_scores, void* workspace, size_t workspace_bytes,
                                void* stream) {
  return score_batch_impl(ctx, query2, target2, num_pairs, m, n, match, mismatch, gap,
                          score_bits, out_scores, workspace, workspace_bytes, stream, true);
}

int bpbc_sw_score_batch_host(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                             int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                             int32_t mismatch, int32_t gap, int32_t score_bits,
                             int32_t* out_scores) {
  return score_batch_host_impl(ctx, query, target, num_pairs, m, n, match, mismatch, gap,
                               score_bits, out_scores, false);
}

int bpbc_sw_score_batch_host_packed2(bpbc_sw_ctx* ctx, const uint8_t* query2,
                                     const uint8_t* target2, int64_t num_pairs, int32_t m,
                                     int32_t n, int32_t match, int32_t mismatch, int32_t gap,
                                     int32_t score_bits, int32_t* out_scores) {
  return score_batch_host_impl(ctx, query2, target2, num_pairs, m, n, match, mismatch, gap,
                               score_bits, out_scores, true);
}

int bpbc_sw_pack(bpbc_sw_ctx* ctx, const uint8_t* codes, int64_t num_pairs, int32_t len,
                 uint32_t* planes, void* stream) {
  if (!ctx || num_pairs < 0 || len < 1) return BPBC_ERR_INVALID_ARG;
  if (num_pairs == 0) return BPBC_OK;
  if (!codes || !planes) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaError_t e = launch_pack(codes, num_pairs, len, reinterpret_cast<uint2*>(planes),
                              ctx->d_flags, ctx->num_sms, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? BPBC_OK : cuda_fail(ctx, e, "pack");
}

int bpbc_sw_untranspose(bpbc_sw_ctx* ctx, const uint32_t* partial, int64_t num_groups,
                        int32_t lanes, int32_t s, int64_t num_pairs, int32_t cap, int32_t* out,
                        void* stream) {
  if (!ctx || num_groups < 0 || lanes < 1 || lanes > 4096 || s < 1 || s > 16 || cap < 0 ||
      num_pairs < 0 || num_pairs > num_groups * 32)
    return BPBC_ERR_INVALID_ARG;
  if (num_groups == 0 || num_pairs == 0) return BPBC_OK;
  if (!partial || !out) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaError_t e = launch_extract(partial, num_groups, lanes, s, num_pairs, 0, cap, out,
                                 ctx->num_sms, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? BPBC_OK : cuda_fail(ctx, e, "untranspose");
}

int bpbc_sw_get_error_flags(bpbc_sw_ctx* ctx, uint32_t* flags) {
  if (!ctx || !flags) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  uint32_t v = 0;
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(&v, ctx->d_flags, sizeof(v), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemset(ctx->d_flags, 0, sizeof(uint32_t));
  if (e != cudaSuccess) return cuda_fail(ctx, e, "get_error_flags");
  *flags = v;
  return BPBC_OK;
}

int bpbc_sw_last_plan(bpbc_sw_ctx* ctx, int32_t* circuit, int32_t* width, int32_t* rows_per_lane,
                      int32_t* lanes, int64_t* streams, int32_t* ops_per_word_cell) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  if (circuit) *circuit = ctx->plan_circuit;
  if (width) *width = ctx->plan_width;
  if (rows_per_lane) *rows_per_lane = ctx->plan_R;
  if (lanes) *lanes = ctx->plan_L;
  if (streams) *streams = ctx->plan_streams;
  if (ops_per_word_cell) *ops_per_word_cell = ctx->plan_ops;
  return BPBC_OK;
}

int bpbc_sw_last_launches(bpbc_sw_ctx* ctx, int32_t* kernels, int32_t* fused) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  if (kernels) *kernels = ctx->plan_kernels;
  if (fused) *fused = ctx->plan_fused;
  return BPBC_OK;
}

int bpbc_sw_profile(bpbc_sw_ctx* ctx, int enable) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaDeviceSynchronize();
  ctx->ev_used.clear();
  ctx->profiling = enable != 0;
  return BPBC_OK;
}

int bpbc_sw_profile_read(bpbc_sw_ctx* ctx, double ms[4], int64_t* calls) {
  if (!ctx || !ms) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  for (int i = 0; i < 4; ++i) ms[i] = 0.0;
  const size_t nc = ctx->ev_used.size() / 4;
  for (size_t c = 0; c < nc; ++c) {
    cudaEvent_t* e = &ctx->ev_used[4 * c];
    cudaError_t err = cudaEventSynchronize(e[3]);
    if (err != cudaSuccess) return cuda_fail(ctx, err, "profile_read");
    float a = 0, b = 0, d = 0;
    cudaEventElapsedTime(&a, e[0], e[1]);
    cudaEventElapsedTime(&b, e[1], e[2]);
    cudaEventElapsedTime(&d, e[2], e[3]);
    ms[0] += a;
    ms[1] += b;
    ms[2] += d;
  }
  ms[3] = ms[0] + ms[1] + ms[2];
  if (calls) *calls = int64_t(nc);
  ctx->ev_used.clear();
  return BPBC_OK;
}

}  // extern "C"
