// api.cu -- the C ABI (include/bpbc_sw.h): validation, workspace layout,
// circuit/width/tiling/stream plan, kernel dispatch, host-buffer path.
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>
#include <new>
#include <vector>

#include "bpbc_internal.cuh"

namespace {

// A stream this ctx enqueued work on, and the event recorded after its last
// call there (bpbc_sw_get_error_flags waits for exactly these).
struct StreamEvent {
  cudaStream_t s;
  cudaEvent_t e;
};

// One buffer slot of the host-buffer path (bpbc_sw_score_batch_host*).
struct HostSlot {
  uint8_t* dq = nullptr;
  uint8_t* dt = nullptr;
  int32_t* dout = nullptr;
  void* ws = nullptr;
  size_t q_bytes = 0, t_bytes = 0, out_bytes = 0, ws_bytes = 0;
  cudaEvent_t h2d_done = nullptr, comp_done = nullptr, d2h_done = nullptr;
  // timing of the slot's last chunk: H2D start / end (copy-in stream),
  // kernels start / end (compute stream)
  cudaEvent_t th0 = nullptr, th1 = nullptr, tc0 = nullptr, tc1 = nullptr;
  bool used = false;
};
constexpr int kHostSlots = 3;

}  // namespace

struct bpbc_sw_ctx {
  int device = 0;
  int num_sms = 0;
  uint32_t* d_flags = nullptr;
  uint32_t* h_flags = nullptr;  // pinned
  cudaStream_t aux = nullptr;   // flag reads, frees
  // options (read once from the environment at init; benchmark knobs)
  int opt_max_blocks = 0;       // BPBC_MAX_BLOCKS_PER_SM: cap on resident sweep blocks / SM
  int opt_min_blocks = 0;       // BPBC_MIN_BLOCKS_PER_SM: floor (with the cap: forces b)
  bool opt_no_exact_run = false;  // BPBC_NO_EXACT_RUN: exact circuit only for (+2,-1,-1)
  int opt_wrap = -1;            // BPBC_WRAP: -1 auto, 0 never, 1 whenever valid
  bool opt_chunked_host = false;  // BPBC_CHUNKED_HOST: host path always in chunks
  bool opt_force_width = false;   // BPBC_FORCE_WIDTH: evaluate the circuit at score_bits
  // ctx-owned device workspace (workspace == NULL; the filter's compaction
  // scratch is a section of it): stream-ordered (cudaMallocAsync / cudaFreeAsync); a call on another
  // stream waits for buf_ev, the event after the last call that used them
  void* ws = nullptr;
  size_t ws_bytes = 0;
  cudaEvent_t buf_ev = nullptr;
  cudaStream_t buf_stream = nullptr;
  bool buf_used = false;
  std::vector<StreamEvent> pending;  // streams with work since the last flag read
  // host path: copy-in, compute and copy-out streams, kHostSlots buffer slots
  cudaStream_t hs_in = nullptr, hs_comp = nullptr, hs_out = nullptr;
  HostSlot slots[kHostSlots];
  int32_t* h_out = nullptr;  // pinned staging for pageable outputs
  size_t h_out_bytes = 0;
  // streamed host path: whole-batch device inputs / scores / workspace, the
  // wave progress word and its reset event, copy timing events
  uint8_t* s_q = nullptr;
  uint8_t* s_t = nullptr;
  int32_t* s_out = nullptr;
  void* s_ws = nullptr;
  size_t s_q_bytes = 0, s_t_bytes = 0, s_out_bytes = 0, s_ws_bytes = 0;
  uint32_t* progress = nullptr;
  int concurrency = -1;  // streamed host path: kernels see later copy-stream writes (probe)
  cudaEvent_t ev_reset = nullptr, ev_c0 = nullptr, ev_c1 = nullptr;
  double h2d_bps = 50e9;     // measured H2D bytes/s (updated after each host call)
  double cells_ps = 5e12;    // measured cell updates/s of the device path
  char err[512] = {0};
  // last plan
  int32_t plan_circuit = -1, plan_width = 0, plan_R = 0, plan_L = 0, plan_ops = 0;
  int32_t plan_kernels = 0, plan_fused = 0, plan_wrap = 0, plan_host_streamed = 0;
  int64_t plan_streams = 0, plan_blocks_per_sm = 0;
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
SweepEntry g_wrap[2][kNumVariants][2][13];        // [mode][variant][rl 2..3][S - 4]
SweepEntry g_hs[2][2][kNumRL][13];                // [mode][pad][rl][S - 4] host-streamed
std::once_flag g_table_once;

void init_table() {
  memset(g_table, 0, sizeof(g_table));
  memset(g_striped, 0, sizeof(g_striped));
  memset(g_mw, 0, sizeof(g_mw));
  memset(g_planes, 0, sizeof(g_planes));
  memset(g_wrap, 0, sizeof(g_wrap));
  memset(g_hs, 0, sizeof(g_hs));
#define BPBC_REG(S)                                                                           \
  if (register_sweep_s##S##_m0)                                                              \
    register_sweep_s##S##_m0(g_table[0], g_striped[0], g_mw[0], g_planes[0], g_wrap[0], g_hs[0]); \
  if (register_sweep_s##S##_m1)                                                              \
    register_sweep_s##S##_m1(g_table[1], g_striped[1], g_mw[1], g_planes[1], g_wrap[1], g_hs[1]);
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

int64_t align256(int64_t v) { return (v + 255) & ~int64_t(255); }
int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ---------------------------------------------------------------------------
// Plan: circuit, evaluated width, tiling.
struct Plan {
  int circuit, consts, rl, width, cap;
  bool pad;
  int ops;
};

int make_plan(int mq, int c1, int c2, int g, int S, bool no_exact_run, bool force_width, Plan* p) {
  if (mq <= 32) p->rl = 0;
  else if (mq <= 64) p->rl = 1;
  else if (mq <= 128) p->rl = 2;
  else if (mq <= kMaxShortRows) p->rl = 3;
  else if (mq <= BPBC_MAX_QUERY_LEN) p->rl = -1;  // striped / multi-warp long-query kernels
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
  if (s_sat > S || force_width) s_sat = S;  // (force_width: circuit-depth studies, DESIGN 6)
  const int cost_sat = 11 * s_sat + 2;
  if (g >= c2) {
    // exact offset circuit at the width no value can exceed: compile-time
    // (+2,-1,-1) 10S LOP3, runtime constants 12S + 1; taken when cheaper
    // than the saturating circuit
    int s_ex = bit_length(int64_t(c1) * mq + g);
    if (s_ex < BPBC_MIN_SCORE_BITS) s_ex = BPBC_MIN_SCORE_BITS;
    if (force_width && S > s_ex) s_ex = S;  // still exact at any width above
    const int cost_ex = spec ? 10 * s_ex : 12 * s_ex + 1;
    const int cost_sat_k = spec ? cost_sat : 13 * s_sat + 4;
    if (s_ex <= BPBC_MAX_SCORE_BITS && cost_ex <= cost_sat_k && (spec || !no_exact_run)) {
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

// ---------------------------------------------------------------------------
// Dispatch: the sweep kernel a plan runs, its launch shape and the split of
// the groups over its streams.
struct Dispatch {
  Plan plan;
  SweepEntry ent;
  bool striped = false;
  bool fused = false;   // single-warp kernel reading raw codes (no pack pass)
  int mw = -1;          // multi-warp variant (index into kMwR / kMwW), -1 = none
  int R = 0, L = 0, W = 1;  // rows per lane, lanes per group, warps per group
  int64_t G = 0;        // 32-pair groups
  int stripes = 1;      // 128-row stripes per group (striped kernel)
  // stream split
  int64_t streams = 0;  // group streams (or wrap-around streams)
  int64_t base = 0, rem = 0;  // group-granular: base or base + 1 groups per stream
  bool wrap = false;    // wrap-around schedule (fused, L = 32)
  int64_t span = 0;     // wrap: columns per stream
  int64_t steps = 0;    // group-granular: steps of every stream
  int grid = 0, block = 0;
  int64_t blocks_per_sm = 0;
};

// Multi-warp variant for this plan, or -1: long queries up to 512 rows (R =
// 4, one warp per 128 rows) and the wide-plane 129..256 case.
int pick_mw(int mq, const Plan& p) {
  if (p.rl >= 0 || mq > 512) return -1;  // single-warp plan, or sequential stripes
  const int W = (mq + 127) / 128 < 2 ? 2 : (mq + 127) / 128;  // one warp per 128 rows
  for (int i = 0; i < kNumMw; ++i)
    if (kMwR[i] == 4 && kMwW[i] == W) return i;
  return -1;
}

int occupancy_blocks(const void* func, int threads, int smem) {  // cached per kernel
  static std::mutex mu;
  static std::vector<std::pair<const void*, int>> cache;
  {
    std::lock_guard<std::mutex> lk(mu);
    for (auto& kv : cache)
      if (kv.first == func) return kv.second;
  }
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, func, threads, smem) != cudaSuccess)
    return -1;
  if (nb < 1) nb = 1;
  std::lock_guard<std::mutex> lk(mu);
  cache.emplace_back(func, nb);
  return nb;
}

// Relative logic-pipe throughput of an SMSP running w resident sweep warps
// (measured: per-SM active cycles of the paper shape, one vs two warps per
// SMSP: 0.956; C2 at two vs four warps per SMSP: 0.97).
double smsp_rate(int64_t w) { return w <= 1 ? 0.93 : w == 2 ? 0.97 : w == 3 ? 0.99 : 1.0; }

int64_t round32(int64_t v) { return (v + 31) / 32 * 32; }

// Stream split of a single-warp (fused / planes) or multi-warp plan:
// minimises the modelled time of the busiest SMSP, (warps per SMSP) x (steps
// per warp) / smsp_rate, over the blocks per SM b and the two schedules:
// group-granular (stream = consecutive whole groups) and wrap-around
// (stream = an equal run of the concatenated columns, fused L = 32 only).
void split_streams(const bpbc_sw_ctx* ctx, int nt, int64_t nb, int64_t nbw, Dispatch* d) {
  const int64_t sms = ctx->num_sms;
  const int64_t G = d->G;
  const bool mw = d->mw >= 0;
  const int64_t segs = mw ? 1 : 32 / d->L;
  const int64_t per_block = mw ? mw_groups_per_block(d->W) : 4 * segs;  // streams per block
  const int64_t warps_per_block = mw ? d->W * per_block : 4;
  const int64_t lag = mw ? int64_t(d->W - 1) * 64 + 31 : 0;
  const int64_t fill = d->L + lag;
  const int64_t units = d->stripes;  // sequential units per group (striped)
  // best group-granular and best wrap-around candidates
  double gg_cost = -1.0, wr_cost = -1.0;
  int64_t gg_streams = 0, gg_steps = 0, gg_bm = 0, wr_span = 0, wr_streams = 0, wr_b = 0;
  const int64_t bmin = ctx->opt_min_blocks > 0 && ctx->opt_min_blocks <= nb ? ctx->opt_min_blocks : 1;
  for (int64_t b = nb; b >= bmin; --b) {
    const int64_t S = sms * b * per_block;
    {  // group-granular: stream = consecutive whole groups
      int64_t streams, gps, bm;
      if (G >= S) {
        streams = S;
        gps = ceil_div(G, S);
        bm = b;
      } else {
        streams = G;
        gps = 1;
        bm = ceil_div(ceil_div(G, per_block), sms);  // blocks on the busiest SM
      }
      int64_t steps = gps * units * nt + fill;
      steps += steps & 1;
      if (mw || d->fused) steps = round32(steps);
      // warps sharing an SMSP: bm blocks x (warps per block / 4 SMSPs)
      const int64_t w = bm * warps_per_block / 4 > 0 ? bm * warps_per_block / 4 : 1;
      const double cost = double(w) * double(steps) / smsp_rate(w);
      if (gg_cost < 0 || cost < gg_cost * 0.999) {
        gg_cost = cost;
        gg_streams = streams;
        gg_steps = steps;
        gg_bm = bm;
      }
    }
    // wrap-around: streams take equal runs of the concatenated columns
    // (nbw: resident blocks of the wrap kernel, 0 = none compiled)
    const bool wrap_ok = d->fused && d->L == 32 && nt % 32 == 0 && G <= kWrapMaxGroups &&
                         S <= kWrapMaxStreams && G >= S && ctx->opt_wrap != 0 && b <= nbw;
    if (wrap_ok) {
      const int64_t span = round32(ceil_div(G * nt, S));
      const int64_t steps = span + 2 * d->L + 32;  // + fill of the whole-group run, drains
      const double cost = double(b) * double(steps) / smsp_rate(b);
      if (wr_cost < 0 || cost < wr_cost * 0.999) {
        wr_cost = cost;
        wr_span = span;
        wr_streams = ceil_div(G * nt, span);
        wr_b = b;
      }
    }
  }
  // wrap when forced (BPBC_WRAP=1) or when it saves more than 1 %
  d->wrap = wr_cost >= 0 && (ctx->opt_wrap == 1 || wr_cost < 0.99 * gg_cost);
  if (d->wrap) {
    d->span = wr_span;
    d->streams = wr_streams;
    d->steps = 0;
    d->blocks_per_sm = wr_b;
  } else {
    d->streams = gg_streams;
    d->steps = gg_steps;
    d->blocks_per_sm = gg_bm;
    d->base = G / d->streams;
    d->rem = G % d->streams;
  }
  if (mw) {
    const int gpb = mw_groups_per_block(d->W);
    d->grid = int(ceil_div(d->streams, gpb));
    d->block = 32 * d->W * gpb;
  } else {
    const int64_t warps = ceil_div(d->streams, segs);
    d->grid = int(ceil_div(warps, 4));
    d->block = 128;
  }
}

int make_dispatch(bpbc_sw_ctx* ctx, int64_t P, int mq, int nt, int c1, int c2, int g, int S,
                  int mode, Dispatch* d, bool host_streamed = false) {
  int rc = make_plan(mq, c1, c2, g, S, ctx->opt_no_exact_run, ctx->opt_force_width, &d->plan);
  if (rc != BPBC_OK) return rc;
  std::call_once(g_table_once, init_table);
  const Plan& plan = d->plan;
  d->G = (P + 31) / 32;
  d->striped = plan.rl < 0;
  d->ent = d->striped ? g_striped[mode][kind_index(plan.circuit, plan.consts)][plan.width - 4]
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
  // host-streamed inputs: the polling instantiation of the fused kernel
  // (the wrap kernel always polls when SweepArgs::progress is set)
  SweepEntry hs_ent{nullptr, nullptr};
  if (host_streamed && d->fused && plan.circuit == kExact && plan.consts == kC211)
    hs_ent = g_hs[mode][plan.pad ? 1 : 0][plan.rl][plan.width - 4];
  if (!d->ent.launch) return BPBC_ERR_UNSUPPORTED;
  d->R = d->striped ? kStripeR : kRLR[plan.rl];
  d->L = d->striped ? 32 : kRLL[plan.rl];
  d->mw = pick_mw(mq, plan);
  int threads = 128, smem = 0;
  if (d->mw >= 0) {
    const SweepEntry e = g_mw[mode][d->mw][kind_index(plan.circuit, plan.consts)][plan.width - 4];
    if (e.launch) {
      d->ent = e;
      d->striped = false;
      d->fused = false;
      d->R = kMwR[d->mw];
      d->W = kMwW[d->mw];
      d->L = 32;
      smem = mw_smem_bytes(d->R, d->W);
      threads = 32 * d->W * mw_groups_per_block(d->W);
      if (cudaFuncSetAttribute(e.func, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) !=
          cudaSuccess)
        return cuda_fail(ctx, cudaGetLastError(), "occupancy");
    } else {
      d->mw = -1;
    }
  }
  if (host_streamed && d->mw < 0) {
    if (!hs_ent.launch) return BPBC_ERR_UNSUPPORTED;  // (the caller takes the chunked path)
    d->ent = hs_ent;
  }
  int64_t nb = occupancy_blocks(d->ent.func, threads, smem);
  if (nb < 0) return cuda_fail(ctx, cudaGetLastError(), "occupancy");
  if (ctx->opt_max_blocks > 0 && nb > ctx->opt_max_blocks) nb = ctx->opt_max_blocks;
  if (d->striped) {
    d->stripes = (mq + kStripeRows - 1) / kStripeRows;
    // one warp per stream; the boundary buffer caps the streams
    int64_t cap = int64_t(ctx->num_sms) * nb * 4;
    const int64_t per_stream = int64_t(nt) * 16 * 4;
    int64_t st = cap < kMaxStripeStreams ? cap : kMaxStripeStreams;
    if (st * per_stream > kMaxBoundaryBytes) st = kMaxBoundaryBytes / per_stream;
    if (st < 1) st = 1;
    d->streams = d->G < st ? d->G : st;
    d->base = d->G / d->streams;
    d->rem = d->G % d->streams;
    d->steps = (d->base + (d->rem > 0 ? 1 : 0)) * d->stripes * int64_t(nt) + d->L;
    d->steps += d->steps & 1;
    d->grid = int(ceil_div(d->streams, 4));
    d->block = 128;
    d->blocks_per_sm = ceil_div(d->grid, ctx->num_sms);
    return BPBC_OK;
  }
  // the wrap-around kernel of this plan (L = 32 fused tilings), if any
  SweepEntry went{nullptr, nullptr};
  int64_t nbw = 0;
  if (d->fused && d->mw < 0 && plan.rl >= 2) {
    went = g_wrap[mode][variant_index(plan.circuit, plan.consts, plan.pad)][plan.rl - 2]
                 [plan.width - 4];
    if (went.launch) {
      nbw = occupancy_blocks(went.func, 128, 0);
      if (nbw < 0) return cuda_fail(ctx, cudaGetLastError(), "occupancy");
      if (ctx->opt_max_blocks > 0 && nbw > ctx->opt_max_blocks) nbw = ctx->opt_max_blocks;
    }
  }
  split_streams(ctx, nt, nb, nbw, d);
  if (d->wrap) d->ent = went;
  return BPBC_OK;
}

// ---------------------------------------------------------------------------
// Workspace layout, 256-byte aligned sections.  With a
// dispatch: exactly what that call uses; without (d == nullptr): an upper
// bound over every plan of (P, mq, nt).
struct Layout {
  int64_t x_off = 0, y_off = 0, mp_off = 0, bnd_off = 0, snap_off = 0, sflag_off = 0,
          zero_off = 0, fs_off = 0, total = 0;
  int64_t G = 0;
};

Layout layout(int64_t P, int mq, int nt, const Dispatch* d, bool filter) {
  Layout L;
  L.G = (P + 31) / 32;
  const int64_t G = L.G;
  const bool planes = d ? !d->fused : true;
  const int64_t xbytes = planes ? (G * mq + kXBackPad) * 8 : 0;
  const int64_t ybytes = planes ? (kYFrontPad + G * nt + nt + kYBackPadExtra) * 8 : 0;
  // per-lane partial maxima: lanes per group x S words
  int64_t mpwords;
  if (d) {
    mpwords = G * int64_t(d->L) * d->W * d->stripes * d->plan.width;
  } else {
    const int64_t stripes = (mq + kStripeRows - 1) / kStripeRows;
    mpwords = G * stripes * 32 * 16;
  }
  // stripe boundary rows (sequential striped kernel only)
  int64_t bnd_bytes = 0;
  const bool may_stripe = d ? d->striped : mq > 128;
  if (may_stripe) {
    const int64_t per_stream = int64_t(nt) * 16 * 4;
    int64_t st = d ? d->streams : (G < kMaxStripeStreams ? G : kMaxStripeStreams);
    if (st * per_stream > kMaxBoundaryBytes) st = kMaxBoundaryBytes / per_stream;
    if (st < 1) st = 1;
    bnd_bytes = st * per_stream;
  }
  // wrap-around snapshots and their flags
  int64_t snap_bytes = 0, sflag_bytes = 0;
  const bool may_wrap = d ? d->wrap : (mq > 64 && mq <= kMaxShortRows && nt % 32 == 0 &&
                                       G <= kWrapMaxGroups);
  if (may_wrap) {
    const int64_t st = d ? d->streams : (G < kWrapMaxStreams ? G : kWrapMaxStreams);
    const int64_t words = d ? snap_words(d->R, d->plan.width) : snap_words(mq <= 128 ? 4 : 8, 16);
    snap_bytes = (st + 1) * words * 32 * 4;
    sflag_bytes = (st + 1) * 4;
  }
  const int64_t fs_bytes = filter ? int64_t(filter_scratch_bytes(G)) : 0;
  L.x_off = 0;
  L.y_off = align256(xbytes);
  L.mp_off = L.y_off + align256(ybytes);
  L.bnd_off = L.mp_off + align256(mpwords * 4);
  L.snap_off = L.bnd_off + align256(bnd_bytes);
  L.sflag_off = L.snap_off + align256(snap_bytes);
  L.zero_off = L.sflag_off + align256(sflag_bytes);
  L.fs_off = L.zero_off + 256;
  L.total = L.fs_off + align256(fs_bytes);
  return L;
}

// ---------------------------------------------------------------------------
// Stream bookkeeping.

// Records "this ctx has work on st up to here" (for bpbc_sw_get_error_flags).
int note_stream(bpbc_sw_ctx* ctx, cudaStream_t st) {
  for (auto& se : ctx->pending)
    if (se.s == st) return cudaEventRecord(se.e, st) == cudaSuccess ? BPBC_OK : BPBC_ERR_CUDA;
  cudaEvent_t e = nullptr;
  cudaError_t err = cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  if (err == cudaSuccess) err = cudaEventRecord(e, st);
  if (err != cudaSuccess) return cuda_fail(ctx, err, "event");
  ctx->pending.push_back({st, e});
  return BPBC_OK;
}

// Before a call uses the ctx-owned buffers on st: wait for the last call that
// used them on another stream.
int buf_acquire(bpbc_sw_ctx* ctx, cudaStream_t st) {
  if (ctx->buf_used && ctx->buf_stream != st) {
    cudaError_t e = cudaStreamWaitEvent(st, ctx->buf_ev, 0);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamWaitEvent");
  }
  return BPBC_OK;
}

int buf_release(bpbc_sw_ctx* ctx, cudaStream_t st) {
  cudaError_t e = cudaEventRecord(ctx->buf_ev, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaEventRecord");
  ctx->buf_stream = st;
  ctx->buf_used = true;
  return BPBC_OK;
}

// Grow a device buffer in stream order on st (no device-wide sync): the old
// allocation is freed after everything already queued on st.
int grow_async(bpbc_sw_ctx* ctx, void** p, size_t* have, size_t need, cudaStream_t st,
               const char* what) {
  if (*have >= need) return BPBC_OK;
  cudaError_t e = cudaSuccess;
  if (*p) {
    e = cudaFreeAsync(*p, st);
    *p = nullptr;
    *have = 0;
    if (e != cudaSuccess) return cuda_fail(ctx, e, what);
  }
  e = cudaMallocAsync(p, need, st);
  if (e != cudaSuccess) {
    *p = nullptr;
    return cuda_fail(ctx, e, what);
  }
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

// ---------------------------------------------------------------------------
// What the sweep produces: max scores (extract) or threshold flags (filter).
struct RunOut {
  int32_t* scores = nullptr;     // max mode
  int mode = kModeMax;
  int threshold = 0;             // threshold mode: flag pairs with score > threshold
  uint32_t* mask = nullptr;      //   [ceil(P/32)] flag words
  int64_t* indices = nullptr;    //   optional ascending flagged pair indices
  int64_t* count = nullptr;      //   optional number of flagged pairs
  const uint32_t* progress = nullptr;  // host-streamed inputs: waves ready (SweepArgs)
  int64_t blk_first = 0, blk_rest = 0;  //   wrap-around copy timeline blocks
};

// Enqueue pack -> sweep -> extract (or the filter epilogue) on device buffers
// with a dispatch made for exactly this call; ws holds layout(P, mq, nt, &dsp).
int run_device(bpbc_sw_ctx* ctx, const Dispatch& dsp, const uint8_t* qx, const uint8_t* ty,
               int64_t P, int mq, int nt, int c1, int c2, int g, const RunOut& o, uint8_t* ws,
               cudaStream_t st, bool packed2) {
  const Plan& plan = dsp.plan;
  const Layout lay = layout(P, mq, nt, &dsp, o.mode == kModeThreshold);
  uint2* Xp = reinterpret_cast<uint2*>(ws + lay.x_off);
  uint2* Ybase = reinterpret_cast<uint2*>(ws + lay.y_off);
  uint2* Yp = Ybase + kYFrontPad;
  uint32_t* Mpart = reinterpret_cast<uint32_t*>(ws + lay.mp_off);

  cudaError_t e = cudaSuccess;
  // The planes-reading sweeps read the pads around the planes (columns before
  // / after a stream's groups, rows past m) and discard what they compute
  // from them; zero them so those reads are of initialised memory.
  if (!dsp.fused) {
    e = cudaMemsetAsync(Ybase, 0, size_t(kYFrontPad) * 8, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(Yp + lay.G * nt, 0, size_t(nt + kYBackPadExtra) * 8, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(Xp + lay.G * mq, 0, size_t(kXBackPad) * 8, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset(pads)");
  }
  if (dsp.wrap) {  // snapshot flags start at 0 every call
    e = cudaMemsetAsync(ws + lay.sflag_off, 0, size_t(dsp.streams + 1) * 4, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset(snapshot flags)");
  }
  if (dsp.striped) {
    e = cudaMemsetAsync(ws + lay.zero_off, 0, 256, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset(zero row)");
  }
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  if (ctx->profiling)
    for (int i = 0; i < 4; ++i) ev[i] = ctx->take_event();
  if (ev[0]) cudaEventRecord(ev[0], st);
  if (!dsp.fused) {  // the fused kernel transposes the raw codes itself
    e = launch_pack2(qx, mq, Xp, ty, nt, Yp, P, ctx->d_flags, ctx->num_sms, st, packed2);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "pack");
  }
  if (ev[1]) cudaEventRecord(ev[1], st);

  SweepArgs a;
  memset(&a, 0, sizeof(a));
  a.Xp = Xp;
  a.Yp = Yp;
  a.Mpart = Mpart;
  a.G = lay.G;
  a.m = mq;
  a.n = nt;
  a.streams = dsp.streams;
  a.base = dsp.base;
  a.rem = dsp.rem;
  a.steps = dsp.steps;
  a.stripes = dsp.stripes;
  a.qraw = qx;
  a.traw = ty;
  a.qstride = packed2 ? (int64_t(mq) + 3) / 4 : mq;
  a.tstride = packed2 ? (int64_t(nt) + 3) / 4 : nt;
  a.P = P;
  a.packed2 = packed2 ? 1 : 0;
  a.flags = ctx->d_flags;
  a.bnd = reinterpret_cast<uint32_t*>(ws + lay.bnd_off);
  a.bzero = reinterpret_cast<const uint32_t*>(ws + lay.zero_off);
  a.wrap = dsp.wrap ? 1 : 0;
  a.span = dsp.span;
  a.snap = reinterpret_cast<uint32_t*>(ws + lay.snap_off);
  a.snap_flag = reinterpret_cast<uint32_t*>(ws + lay.sflag_off);
  a.progress = o.progress;
  a.blk_first = o.blk_first;
  a.blk_rest = o.blk_rest;
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
  dsp.ent.launch(a, kr, dsp.grid, dsp.block, st);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(ctx, e, "sweep");
  if (ev[2]) cudaEventRecord(ev[2], st);
  const int lanes = dsp.L * dsp.stripes * dsp.W;
  if (o.mode == kModeThreshold) {
    const int64_t fs = int64_t(filter_scratch_bytes(lay.G));
    e = launch_filter_finish(Mpart, lay.G, lanes, P, o.mask, o.indices, o.count,
                             ws + lay.fs_off, size_t(fs), ctx->num_sms, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "filter epilogue");
  } else {
    // the exact circuit's partial maxima carry the offset g (finish_exact)
    e = launch_extract(Mpart, lay.G, lanes, plan.width, P, plan.circuit == kExact ? g : 0,
                       plan.cap, o.scores, ctx->num_sms, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "extract");
  }
  if (ev[3]) cudaEventRecord(ev[3], st);

  ctx->plan_circuit = plan.circuit;
  ctx->plan_width = Wd;
  ctx->plan_R = dsp.R;
  ctx->plan_L = dsp.L * dsp.W;  // lanes per group (over all its warps)
  ctx->plan_ops = plan.ops;
  ctx->plan_streams = dsp.streams;
  ctx->plan_fused = dsp.fused ? 1 : 0;
  ctx->plan_wrap = dsp.wrap ? 1 : 0;
  ctx->plan_blocks_per_sm = dsp.blocks_per_sm;
  ctx->plan_kernels = (dsp.fused ? 0 : 1) + 1 + (o.mode == kModeThreshold
                                                     ? ((o.indices || o.count) ? 2 : 1)
                                                     : 1);
  return BPBC_OK;
}

// Common front of the device-buffer entry points: validation, the R17 swap,
// the dispatch and the workspace (caller's, or the ctx's in stream order).
int device_call(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target, int64_t P, int m,
                int n, int match, int mismatch, int gap, int S, const RunOut& o, void* workspace,
                size_t workspace_bytes, cudaStream_t st, bool packed2) {
  // score is symmetric (R17): the shorter sequence plays the query (rows)
  const uint8_t* qx = m <= n ? query : target;
  const uint8_t* ty = m <= n ? target : query;
  const int mq = m <= n ? m : n, nt = m <= n ? n : m;
  const int c1 = match, c2 = -mismatch, g = -gap;
  Dispatch dsp;
  int rc = make_dispatch(ctx, P, mq, nt, c1, c2, g, S, o.mode, &dsp);
  if (rc != BPBC_OK) return rc;
  const size_t need = size_t(layout(P, mq, nt, &dsp, o.mode == kModeThreshold).total);
  uint8_t* ws;
  const bool own = workspace == nullptr;
  if (!own) {
    if (workspace_bytes < need) return BPBC_ERR_INVALID_ARG;
    ws = static_cast<uint8_t*>(workspace);
  } else {
    if ((rc = buf_acquire(ctx, st)) != BPBC_OK) return rc;
    rc = grow_async(ctx, &ctx->ws, &ctx->ws_bytes, need, st, "cudaMallocAsync(workspace)");
    if (rc != BPBC_OK) return rc;
    ws = static_cast<uint8_t*>(ctx->ws);
  }
  rc = run_device(ctx, dsp, qx, ty, P, mq, nt, c1, c2, g, o, ws, st, packed2);
  if (rc != BPBC_OK) return rc;
  if (own && (rc = buf_release(ctx, st)) != BPBC_OK) return rc;
  return note_stream(ctx, st);
}

}  // namespace
}  // namespace bpbc

using namespace bpbc;

namespace {

int score_batch_impl(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                     int64_t num_pairs, int32_t m, int32_t n, int32_t match, int32_t mismatch,
                     int32_t gap, int32_t score_bits, int32_t* out_scores, void* workspace,
                     size_t workspace_bytes, void* stream, bool packed2) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_scores) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  RunOut o;
  o.scores = out_scores;
  return device_call(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits, o,
                     workspace, workspace_bytes, static_cast<cudaStream_t>(stream), packed2);
}

// ---------------------------------------------------------------------------
// Host-buffer path (the paper's Steps 1-5): chunks of whole
// "waves" (one group per resident sweep stream) flow through kHostSlots
// buffer slots on three streams -- H2D of chunk c+1 and D2H of chunk c-1
// overlap the kernels of chunk c.

int slot_events(bpbc_sw_ctx* ctx, HostSlot& s) {
  cudaEvent_t* sync_evs[3] = {&s.h2d_done, &s.comp_done, &s.d2h_done};
  for (cudaEvent_t* e : sync_evs)
    if (!*e && cudaEventCreateWithFlags(e, cudaEventDisableTiming) != cudaSuccess)
      return cuda_fail(ctx, cudaGetLastError(), "event");
  cudaEvent_t* t_evs[4] = {&s.th0, &s.th1, &s.tc0, &s.tc1};
  for (cudaEvent_t* e : t_evs)
    if (!*e && cudaEventCreate(e) != cudaSuccess) return cuda_fail(ctx, cudaGetLastError(), "event");
  return BPBC_OK;
}

// cuStreamWriteValue32 (driver API, through the runtime's entry-point query:
// no link against libcuda): a 32-bit store ordered after the stream's
// previous work, with a memory barrier (flags 0), done by the GPU front end.
typedef int (*WriteValue32Fn)(void* stream, unsigned long long addr, unsigned int value,
                              unsigned int flags);
// host_streamed(): the kernel's device-side wait timed out (internal status)
constexpr int kStallRetry = -100;

WriteValue32Fn write_value32() {
  static WriteValue32Fn fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      f = nullptr;
    cudaGetLastError();
    return reinterpret_cast<WriteValue32Fn>(f);
  }();
  return fn;
}

// Host path as ONE streamed launch (fused group-granular plans): the whole
// batch's device buffers are filled wave by wave on the copy-in stream (a
// wave = the h-th group of every sweep stream = S consecutive groups, since
// the fused kernel assigns groups to streams strided), each followed by a
// device-side write of the wave count to `progress`; the sweep runs
// concurrently on the compute stream and polls `progress` before it touches
// a wave (SweepArgs::progress).  No per-chunk pipeline fill, the copy
// overlaps the kernels from the first wave on, and only the first wave's
// copy is exposed.  Returns BPBC_ERR_UNSUPPORTED when the device cannot do
// stream memory writes (the caller then uses the chunked path).
int host_streamed(bpbc_sw_ctx* ctx, const Dispatch& dsp, const uint8_t* qx, const uint8_t* ty,
                  int64_t P, int mq, int nt, int c1, int c2, int g, int64_t qs, int64_t ts,
                  int32_t* out_scores, bool packed2) {
  WriteValue32Fn wv = write_value32();
  if (!wv) return BPBC_ERR_UNSUPPORTED;
  cudaError_t e;
  int rc;
  cudaStream_t cin = ctx->hs_in, comp = ctx->hs_comp;
  const size_t need = size_t(layout(P, mq, nt, &dsp, false).total);
  if ((rc = grow_async(ctx, (void**)&ctx->s_q, &ctx->s_q_bytes, size_t(P * qs), comp,
                       "cudaMallocAsync(q)")) != BPBC_OK ||
      (rc = grow_async(ctx, (void**)&ctx->s_t, &ctx->s_t_bytes, size_t(P * ts), comp,
                       "cudaMallocAsync(t)")) != BPBC_OK ||
      (rc = grow_async(ctx, (void**)&ctx->s_out, &ctx->s_out_bytes, size_t(P) * 4, comp,
                       "cudaMallocAsync(out)")) != BPBC_OK ||
      (rc = grow_async(ctx, &ctx->s_ws, &ctx->s_ws_bytes, need, comp,
                       "cudaMallocAsync(workspace)")) != BPBC_OK)
    return rc;
  cudaEvent_t* evs[3] = {&ctx->ev_reset, &ctx->ev_c0, &ctx->ev_c1};
  for (int i = 0; i < 3; ++i)
    if (!*evs[i] && (e = (i == 0 ? cudaEventCreateWithFlags(evs[i], cudaEventDisableTiming)
                                 : cudaEventCreate(evs[i]))) != cudaSuccess)
      return cuda_fail(ctx, e, "event");
  if (!ctx->progress && (e = cudaMalloc(&ctx->progress, 256)) != cudaSuccess)
    return cuda_fail(ctx, e, "cudaMalloc(progress)");
  // Once per ctx: can a kernel see a stream write enqueued after its launch
  // on another stream?  (No under a kernel-serialising profiler or with
  // launch blocking: the streamed launch would then wait for copies that
  // are never started; BPBC_FLAG_STALL is the backstop.)
  if (ctx->concurrency < 0) {
    uint32_t* f = ctx->progress + 32;  // [flag, seen] in the progress block
    if ((e = cudaMemsetAsync(f, 0, 8, comp)) != cudaSuccess ||
        (e = cudaEventRecord(ctx->ev_reset, comp)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(cin, ctx->ev_reset, 0)) != cudaSuccess ||
        (e = launch_probe_wait(f, f + 1, 200ull * 1000000ull, comp)) != cudaSuccess)
      return cuda_fail(ctx, e, "concurrency probe");
    if (wv(cin, reinterpret_cast<unsigned long long>(f), 1u, 0) != 0) {
      cudaGetLastError();
      return BPBC_ERR_UNSUPPORTED;
    }
    uint32_t seen = 0;
    if ((e = cudaMemcpyAsync(ctx->h_flags + 1, f + 1, 4, cudaMemcpyDeviceToHost, comp)) !=
            cudaSuccess ||
        (e = cudaStreamSynchronize(comp)) != cudaSuccess ||
        (e = cudaStreamSynchronize(cin)) != cudaSuccess)
      return cuda_fail(ctx, e, "concurrency probe");
    seen = ctx->h_flags[1];
    ctx->concurrency = seen ? 1 : 0;
  }
  if (ctx->concurrency == 0) return BPBC_ERR_UNSUPPORTED;  // (the chunked path)
  // progress = 0 before the kernel starts; the copy stream's first write
  // comes after the reset (and after the allocations above)
  if ((e = cudaMemsetAsync(ctx->progress, 0, 4, comp)) != cudaSuccess ||
      (e = cudaEventRecord(ctx->ev_reset, comp)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(cin, ctx->ev_reset, 0)) != cudaSuccess)
    return cuda_fail(ctx, e, "progress reset");
  // The copy-in plan, as waves, each closed by a progress write of the waves
  // done; wave 0 is enqueued before the kernel, the rest after it (their
  // API calls then overlap the kernel).
  const int64_t S = dsp.streams;
  const int64_t G = (P + 31) / 32;
  std::vector<int64_t> wave_end;  // group-granular: group-wave boundaries
  int64_t blk_first = 0, blk_rest = 0, nwaves = 0;
  bool bulk = false;            // wrap-around, pageable inputs: two plain copies first
  const uint8_t* ty_dev = nullptr;  // wrap-around, pinned inputs: the gather kernel's view
  if (!dsp.wrap) {
    // copy waves of whole stream-waves (the h-th group of every stream is
    // group h S + st), one stream-wave each (at most 256 copy waves): the
    // kernel starts after the first and, when the copy is the slower side,
    // ends one stream-wave of compute after the last byte is in (growing
    // waves left the last, largest one's compute exposed: C2 u8 e2e 0.74 of
    // the H2D bound)
    const int64_t waves = (G + S - 1) / S;
    const int64_t per = (waves + 255) / 256;
    for (int64_t w1 = per; ; w1 += per) {
      wave_end.push_back(w1 < waves ? w1 : waves);
      if (w1 >= waves) break;
    }
    nwaves = int64_t(wave_end.size());
  } else {
    // every stream's copy timeline (head, whole groups, tail from column
    // ra - 32) moves in equal column blocks after a short first one, so all
    // streams can start after ~blk_first columns of copying; the copy rate
    // (~55 GB/s) stays ahead of the kernels' (~45 GB/s at the paper's shape).
    // A wave is ~3 small 2D regions per stream: one launch of the gather
    // kernel (gather.cu) reading the pinned host rows; pageable inputs (not
    // device-readable) are copied whole before the kernel instead (bulk).
    blk_first = 1024;
    blk_rest = 8192;
    const int64_t tl = dsp.span + nt + 64;  // longest timeline
    void* dp = nullptr;
    cudaPointerAttributes pa;
    if (cudaPointerGetAttributes(&pa, ty) == cudaSuccess && pa.type == cudaMemoryTypeHost &&
        cudaHostGetDevicePointer(&dp, const_cast<uint8_t*>(ty), 0) == cudaSuccess && dp) {
      ty_dev = static_cast<const uint8_t*>(dp);
    } else {
      cudaGetLastError();
      bulk = true;
      blk_first = tl;
    }
    nwaves = 1 + (tl - blk_first + blk_rest - 1) / blk_rest;
  }
  auto enqueue_wave = [&](int64_t w) -> int {
    cudaError_t ee = cudaSuccess;
    if (!dsp.wrap) {
      const int64_t g0w = (w == 0 ? 0 : wave_end[w - 1]) * S;
      const int64_t p0 = g0w * 32;
      const int64_t p1 = wave_end[w] * S * 32 < P ? wave_end[w] * S * 32 : P;
      ee = cudaMemcpyAsync(ctx->s_q + p0 * qs, qx + p0 * qs, size_t((p1 - p0) * qs),
                           cudaMemcpyHostToDevice, cin);
      if (ee == cudaSuccess)
        ee = cudaMemcpyAsync(ctx->s_t + p0 * ts, ty + p0 * ts, size_t((p1 - p0) * ts),
                             cudaMemcpyHostToDevice, cin);
    } else if (bulk) {
      ee = cudaMemcpyAsync(ctx->s_q, qx, size_t(P * qs), cudaMemcpyHostToDevice, cin);
      if (ee == cudaSuccess)
        ee = cudaMemcpyAsync(ctx->s_t, ty, size_t(P * ts), cudaMemcpyHostToDevice, cin);
    } else {
      if (w == 0)
        ee = cudaMemcpyAsync(ctx->s_q, qx, size_t(P * qs), cudaMemcpyHostToDevice, cin);
      const int64_t x0 = w == 0 ? 0 : blk_first + (w - 1) * blk_rest;
      const int64_t x1 = w == 0 ? blk_first : blk_first + w * blk_rest;
      if (ee == cudaSuccess)
        ee = launch_wrap_gather(ty_dev, ctx->s_t, P, G, nt, ts, dsp.span, S, x0, x1, packed2,
                                ctx->num_sms, cin);
    }
    if (ee != cudaSuccess) return cuda_fail(ctx, ee, "H2D");
    // the kernel's wave index: group-granular = stream-waves in (wave_end),
    // wrap-around = column blocks in (w + 1)
    const unsigned done = dsp.wrap ? unsigned(w + 1) : unsigned(wave_end[w]);
    if (wv(cin, reinterpret_cast<unsigned long long>(ctx->progress), done, 0) != 0) {
      cudaGetLastError();
      return BPBC_ERR_UNSUPPORTED;
    }
    return BPBC_OK;
  };
  cudaEventRecord(ctx->ev_c0, cin);
  if ((rc = enqueue_wave(0)) != BPBC_OK) return rc;
  RunOut o;
  o.scores = ctx->s_out;
  o.progress = ctx->progress;
  o.blk_first = blk_first;
  o.blk_rest = blk_rest;
  rc = run_device(ctx, dsp, ctx->s_q, ctx->s_t, P, mq, nt, c1, c2, g, o,
                  static_cast<uint8_t*>(ctx->s_ws), comp, packed2);
  if (rc != BPBC_OK) return rc;
  for (int64_t w = 1; w < nwaves; ++w)
    if ((rc = enqueue_wave(w)) != BPBC_OK) return rc;
  cudaEventRecord(ctx->ev_c1, cin);
  if ((e = cudaMemcpyAsync(out_scores, ctx->s_out, size_t(P) * 4, cudaMemcpyDeviceToHost, comp)) !=
      cudaSuccess)
    return cuda_fail(ctx, e, "D2H");
  if ((e = cudaStreamSynchronize(comp)) != cudaSuccess ||
      (e = cudaStreamSynchronize(cin)) != cudaSuccess)
    return cuda_fail(ctx, e, "sync");
  // a timed-out device wait (BPBC_FLAG_STALL stays set for get_error_flags)
  if ((e = cudaMemcpyAsync(ctx->h_flags, ctx->d_flags, sizeof(uint32_t), cudaMemcpyDeviceToHost,
                           comp)) != cudaSuccess ||
      (e = cudaStreamSynchronize(comp)) != cudaSuccess)
    return cuda_fail(ctx, e, "flags");
  if (*ctx->h_flags & BPBC_FLAG_STALL) {  // handled here, so cleared (BAD_BASE stays)
    *ctx->h_flags &= ~BPBC_FLAG_STALL;
    cudaMemcpyAsync(ctx->d_flags, ctx->h_flags, sizeof(uint32_t), cudaMemcpyHostToDevice, comp);
    cudaStreamSynchronize(comp);
    return kStallRetry;  // the caller reruns the batch on the chunked path
  }
  float ms = 0;
  if (cudaEventElapsedTime(&ms, ctx->ev_c0, ctx->ev_c1) == cudaSuccess && ms > 0 &&
      P * (qs + ts) > (1 << 20))
    ctx->h2d_bps = double(P * (qs + ts)) / (ms * 1e-3);
  cudaGetLastError();
  return BPBC_OK;
}

int score_batch_host_impl(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                          int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                          int32_t mismatch, int32_t gap, int32_t score_bits, int32_t* out_scores,
                          bool packed2) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  if (num_pairs == 0) return BPBC_OK;
  if (!query || !target || !out_scores) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  cudaError_t e;
  cudaStream_t* sts[3] = {&ctx->hs_in, &ctx->hs_comp, &ctx->hs_out};
  for (cudaStream_t* s : sts) {
    if (!*s) {
      e = cudaStreamCreateWithFlags(s, cudaStreamNonBlocking);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamCreate");
    }
  }
  for (auto& s : ctx->slots)
    if ((rc = slot_events(ctx, s)) != BPBC_OK) return rc;
  const uint8_t* qx = m <= n ? query : target;
  const uint8_t* ty = m <= n ? target : query;
  const int mq = m <= n ? m : n, nt = m <= n ? n : m;
  const int c1 = match, c2 = -mismatch, g = -gap;
  // bytes per row: one per base, or 4 bases per byte (packed2)
  const int64_t qs = packed2 ? (int64_t(mq) + 3) / 4 : mq, ts = packed2 ? (int64_t(nt) + 3) / 4 : nt;
  // a wave = one group per resident stream of the full-size plan
  Dispatch full;
  if ((rc = make_dispatch(ctx, num_pairs, mq, nt, c1, c2, g, score_bits, kModeMax, &full)) !=
      BPBC_OK)
    return rc;
  // fused plans (group-granular or wrap-around): one streamed launch
  Dispatch hsd;
  if (full.fused && full.mw < 0 && !ctx->opt_chunked_host &&
      make_dispatch(ctx, num_pairs, mq, nt, c1, c2, g, score_bits, kModeMax, &hsd, true) ==
          BPBC_OK) {
    // results: straight into a pinned output, else through pinned staging
    cudaPointerAttributes pa;
    const bool pinned = cudaPointerGetAttributes(&pa, out_scores) == cudaSuccess &&
                        pa.type == cudaMemoryTypeHost;
    cudaGetLastError();
    int32_t* dst = out_scores;
    if (!pinned) {
      const size_t ob = size_t(num_pairs) * 4;
      if (ctx->h_out_bytes < ob) {
        if (ctx->h_out) cudaFreeHost(ctx->h_out);
        ctx->h_out = nullptr;
        ctx->h_out_bytes = 0;
        if ((e = cudaMallocHost(&ctx->h_out, ob)) != cudaSuccess)
          return cuda_fail(ctx, e, "cudaMallocHost(out staging)");
        ctx->h_out_bytes = ob;
      }
      dst = ctx->h_out;
    }
    rc = host_streamed(ctx, hsd, qx, ty, num_pairs, mq, nt, c1, c2, g, qs, ts, dst, packed2);
    if (rc == kStallRetry) {
      // the kernel waited 20 s for copies that never came (the environment
      // serialised it against them): this ctx uses the chunked path from now on
      ctx->opt_chunked_host = true;
      rc = BPBC_ERR_UNSUPPORTED;
    }
    if (rc == BPBC_OK) {
      if (!pinned) memcpy(out_scores, ctx->h_out, size_t(num_pairs) * 4);
      ctx->plan_host_streamed = 1;
      return BPBC_OK;
    }
    if (rc != BPBC_ERR_UNSUPPORTED) return rc;
  }
  ctx->plan_host_streamed = 0;
  // (few groups: a chunk of them would leave SMSPs idle -- no chunking)
  const int64_t wave_pairs = full.wrap ? num_pairs : full.streams * 32;
  // Chunk plan from the measured rates.  Every chunk's
  // kernels pay one pipeline fill / drain (~L steps per stream), so chunks
  // are few and large:
  //  * copy-bound (H2D time per pair >= kernel time per pair): ~12 equal
  //    chunks -- the run takes the whole copy plus the last chunk's kernels;
  //  * compute-bound: chunks growing geometrically from one wave, by the
  //    factor the kernels outpace the copy (the copy of chunk c+1 hides
  //    under the kernels of chunk c), capped at 4x.
  const double h2d_s = double(qs + ts) / ctx->h2d_bps;
  const double comp_s = double(mq) * nt / ctx->cells_ps;
  const int64_t waves = ceil_div(num_pairs, wave_pairs);
  std::vector<int64_t> bounds{0};
  if (h2d_s >= comp_s) {
    const int64_t per = ceil_div(waves, 12);
    while (bounds.back() < num_pairs) {
      const int64_t left = num_pairs - bounds.back();
      bounds.push_back(bounds.back() + (left < per * wave_pairs ? left : per * wave_pairs));
    }
  } else {
    double f = comp_s / (h2d_s > 0 ? h2d_s : 1e-30);
    f = f < 1.25 ? 1.25 : (f > 4.0 ? 4.0 : f);
    double w = 1.0;
    while (bounds.back() < num_pairs) {
      const int64_t left = num_pairs - bounds.back();
      const int64_t wi = int64_t(w) > 0 ? int64_t(w) : 1;
      // fold a remainder shorter than the next chunk into this one
      const int64_t take = left <= int64_t(double(wi) * (1.0 + f)) * wave_pairs ? left
                                                                                : wi * wave_pairs;
      bounds.push_back(bounds.back() + take);
      w *= f;
    }
  }
  const int64_t nch = int64_t(bounds.size()) - 1;
  int64_t chunk = 0;
  for (int64_t i = 1; i <= nch; ++i)
    chunk = bounds[i] - bounds[i - 1] > chunk ? bounds[i] - bounds[i - 1] : chunk;
  size_t need = 0;
  {
    Dispatch dc;
    // the largest chunk's exact workspace; smaller chunks need no more
    if ((rc = make_dispatch(ctx, chunk, mq, nt, c1, c2, g, score_bits, kModeMax, &dc)) != BPBC_OK)
      return rc;
    need = size_t(layout(chunk, mq, nt, &dc, false).total);
    for (int64_t i = 1; i <= nch; ++i) {
      Dispatch di;
      if ((rc = make_dispatch(ctx, bounds[i] - bounds[i - 1], mq, nt, c1, c2, g, score_bits,
                              kModeMax, &di)) != BPBC_OK)
        return rc;
      const size_t ni = size_t(layout(bounds[i] - bounds[i - 1], mq, nt, &di, false).total);
      need = ni > need ? ni : need;
    }
  }
  // buffers of every slot (freed / grown in the compute stream's order; the
  // previous host call has completed, it synchronizes before returning)
  for (auto& s : ctx->slots) {
    if ((rc = grow_async(ctx, (void**)&s.dq, &s.q_bytes, size_t(chunk * qs), ctx->hs_comp,
                         "cudaMallocAsync(q)")) != BPBC_OK ||
        (rc = grow_async(ctx, (void**)&s.dt, &s.t_bytes, size_t(chunk * ts), ctx->hs_comp,
                         "cudaMallocAsync(t)")) != BPBC_OK ||
        (rc = grow_async(ctx, (void**)&s.dout, &s.out_bytes, size_t(chunk) * 4, ctx->hs_comp,
                         "cudaMallocAsync(out)")) != BPBC_OK ||
        (rc = grow_async(ctx, &s.ws, &s.ws_bytes, need, ctx->hs_comp,
                         "cudaMallocAsync(workspace)")) != BPBC_OK)
      return rc;
    s.used = false;
  }
  // allocations are ordered on hs_comp; the copy streams start after them
  cudaEvent_t ready = ctx->slots[0].comp_done;
  if ((e = cudaEventRecord(ready, ctx->hs_comp)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(ctx->hs_in, ready, 0)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(ctx->hs_out, ready, 0)) != cudaSuccess)
    return cuda_fail(ctx, e, "stream order");
  // results: straight into a pinned output, else through pinned staging
  cudaPointerAttributes pa;
  bool pinned_out = cudaPointerGetAttributes(&pa, out_scores) == cudaSuccess &&
                    pa.type == cudaMemoryTypeHost;
  cudaGetLastError();  // (clear a pageable-pointer query error)
  int32_t* dst = out_scores;
  if (!pinned_out) {
    const size_t ob = size_t(num_pairs) * 4;
    if (ctx->h_out_bytes < ob) {
      if (ctx->h_out) cudaFreeHost(ctx->h_out);
      ctx->h_out = nullptr;
      ctx->h_out_bytes = 0;
      if ((e = cudaMallocHost(&ctx->h_out, ob)) != cudaSuccess)
        return cuda_fail(ctx, e, "cudaMallocHost(out staging)");
      ctx->h_out_bytes = ob;
    }
    dst = ctx->h_out;
  }
  for (int64_t ci = 0; ci < nch; ++ci) {
    HostSlot& s = ctx->slots[ci % kHostSlots];
    const int64_t c0 = bounds[ci], cp = bounds[ci + 1] - bounds[ci];
    // H2D into the slot once its previous chunk's kernels are done
    if (s.used && (e = cudaStreamWaitEvent(ctx->hs_in, s.comp_done, 0)) != cudaSuccess)
      return cuda_fail(ctx, e, "wait");
    cudaEventRecord(s.th0, ctx->hs_in);
    e = cudaMemcpyAsync(s.dq, qx + c0 * qs, size_t(cp * qs), cudaMemcpyHostToDevice, ctx->hs_in);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(s.dt, ty + c0 * ts, size_t(cp * ts), cudaMemcpyHostToDevice, ctx->hs_in);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "H2D");
    cudaEventRecord(s.th1, ctx->hs_in);
    cudaEventRecord(s.h2d_done, ctx->hs_in);
    // kernels once the inputs are in and the slot's previous results are out
    if ((e = cudaStreamWaitEvent(ctx->hs_comp, s.h2d_done, 0)) != cudaSuccess ||
        (s.used && (e = cudaStreamWaitEvent(ctx->hs_comp, s.d2h_done, 0)) != cudaSuccess))
      return cuda_fail(ctx, e, "wait");
    Dispatch dc;
    if ((rc = make_dispatch(ctx, cp, mq, nt, c1, c2, g, score_bits, kModeMax, &dc)) != BPBC_OK)
      return rc;
    cudaEventRecord(s.tc0, ctx->hs_comp);
    RunOut o;
    o.scores = s.dout;
    rc = run_device(ctx, dc, s.dq, s.dt, cp, mq, nt, c1, c2, g, o, static_cast<uint8_t*>(s.ws),
                    ctx->hs_comp, packed2);
    if (rc != BPBC_OK) return rc;
    cudaEventRecord(s.tc1, ctx->hs_comp);
    cudaEventRecord(s.comp_done, ctx->hs_comp);
    // D2H of the 4-byte scores
    if ((e = cudaStreamWaitEvent(ctx->hs_out, s.comp_done, 0)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dst + c0, s.dout, size_t(cp) * 4, cudaMemcpyDeviceToHost,
                             ctx->hs_out)) != cudaSuccess)
      return cuda_fail(ctx, e, "D2H");
    cudaEventRecord(s.d2h_done, ctx->hs_out);
    s.used = true;
  }
  if ((e = cudaStreamSynchronize(ctx->hs_out)) != cudaSuccess ||
      (e = cudaStreamSynchronize(ctx->hs_comp)) != cudaSuccess ||
      (e = cudaStreamSynchronize(ctx->hs_in)) != cudaSuccess)
    return cuda_fail(ctx, e, "sync");
  // measured rates for the next call's chunk plan, from the events of the
  // last chunks (each slot's events describe its last chunk)
  {
    double hb = 0, hs = 0, cb = 0, cs = 0;
    for (int64_t ci = nch - 1; ci >= 0 && ci >= nch - kHostSlots; --ci) {
      HostSlot& s = ctx->slots[ci % kHostSlots];
      const int64_t cp = bounds[ci + 1] - bounds[ci];
      float a = 0, b = 0;
      if (cudaEventElapsedTime(&a, s.th0, s.th1) == cudaSuccess && a > 0) {
        hb += double(cp) * double(qs + ts);
        hs += a * 1e-3;
      }
      if (cudaEventElapsedTime(&b, s.tc0, s.tc1) == cudaSuccess && b > 0) {
        cb += double(cp) * double(mq) * double(nt);
        cs += b * 1e-3;
      }
    }
    if (hs > 0 && hb > double(1 << 20)) ctx->h2d_bps = hb / hs;
    if (cs > 0 && cb > 1e8) ctx->cells_ps = cb / cs;
  }
  cudaGetLastError();
  if (!pinned_out) memcpy(out_scores, ctx->h_out, size_t(num_pairs) * 4);
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

static int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return (v && *v) ? atoi(v) : dflt;
}

int bpbc_sw_init(int cuda_device, bpbc_sw_ctx** out_ctx) {
  if (!out_ctx) return BPBC_ERR_INVALID_ARG;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaGetDeviceCount");
  if (cuda_device < 0 || cuda_device >= ndev) return BPBC_ERR_INVALID_ARG;
  bpbc_sw_ctx* ctx = new (std::nothrow) bpbc_sw_ctx();
  if (!ctx) return BPBC_ERR_OOM;
  ctx->device = cuda_device;
  // benchmark knobs: read once here, never on the hot path
  ctx->opt_max_blocks = env_int("BPBC_MAX_BLOCKS_PER_SM", 0);
  ctx->opt_min_blocks = env_int("BPBC_MIN_BLOCKS_PER_SM", 0);
  ctx->opt_no_exact_run = env_int("BPBC_NO_EXACT_RUN", 0) != 0;
  ctx->opt_wrap = env_int("BPBC_WRAP", -1);
  ctx->opt_chunked_host = env_int("BPBC_CHUNKED_HOST", 0) != 0;

  ctx->opt_force_width = env_int("BPBC_FORCE_WIDTH", 0) != 0;
  DeviceGuard dg(cuda_device);
  e = cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  if (e == cudaSuccess) e = cudaMalloc(&ctx->d_flags, sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMemset(ctx->d_flags, 0, sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMallocHost(&ctx->h_flags, 2 * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->aux, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->buf_ev, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();  // the flag word is zero before any call
  if (e != cudaSuccess) {
    int rc = cuda_fail(ctx, e, "init");
    if (ctx->d_flags) cudaFree(ctx->d_flags);
    if (ctx->h_flags) cudaFreeHost(ctx->h_flags);
    if (ctx->aux) cudaStreamDestroy(ctx->aux);
    if (ctx->buf_ev) cudaEventDestroy(ctx->buf_ev);
    delete ctx;
    return rc;
  }
  *out_ctx = ctx;
  return BPBC_OK;
}

int bpbc_sw_destroy(bpbc_sw_ctx* ctx) {
  if (!ctx) return BPBC_OK;
  DeviceGuard dg(ctx->device);
  // wait for this ctx's own work only (not the whole device)
  for (auto& se : ctx->pending) {
    cudaEventSynchronize(se.e);
    cudaEventDestroy(se.e);
  }
  for (cudaStream_t s : {ctx->hs_in, ctx->hs_comp, ctx->hs_out})
    if (s) cudaStreamSynchronize(s);
  if (ctx->buf_used) cudaEventSynchronize(ctx->buf_ev);
  if (ctx->ws) cudaFreeAsync(ctx->ws, ctx->aux);
  {
    void* bufs[4] = {ctx->s_q, ctx->s_t, ctx->s_out, ctx->s_ws};
    for (void* p : bufs)
      if (p) cudaFreeAsync(p, ctx->aux);
    cudaEvent_t evs[3] = {ctx->ev_reset, ctx->ev_c0, ctx->ev_c1};
    for (cudaEvent_t ev : evs)
      if (ev) cudaEventDestroy(ev);
  }
  for (auto& s : ctx->slots) {
    void* bufs[4] = {s.dq, s.dt, s.dout, s.ws};
    for (void* p : bufs)
      if (p) cudaFreeAsync(p, ctx->aux);
    cudaEvent_t evs[7] = {s.h2d_done, s.comp_done, s.d2h_done, s.th0, s.th1, s.tc0, s.tc1};
    for (cudaEvent_t ev : evs)
      if (ev) cudaEventDestroy(ev);
  }
  cudaStreamSynchronize(ctx->aux);
  for (cudaStream_t s : {ctx->hs_in, ctx->hs_comp, ctx->hs_out})
    if (s) cudaStreamDestroy(s);
  if (ctx->d_flags) cudaFree(ctx->d_flags);
  if (ctx->progress) cudaFree(ctx->progress);
  if (ctx->h_flags) cudaFreeHost(ctx->h_flags);
  if (ctx->h_out) cudaFreeHost(ctx->h_out);
  if (ctx->aux) cudaStreamDestroy(ctx->aux);
  if (ctx->buf_ev) cudaEventDestroy(ctx->buf_ev);
  for (cudaEvent_t e : ctx->ev_pool) cudaEventDestroy(e);
  delete ctx;
  return BPBC_OK;
}

int bpbc_sw_workspace_bytes(int64_t num_pairs, int32_t m, int32_t n, size_t* bytes) {
  if (!bytes || num_pairs < 0 || m < 1 || n < 1) return BPBC_ERR_INVALID_ARG;
  if (m > BPBC_MAX_LEN || n > BPBC_MAX_LEN) return BPBC_ERR_UNSUPPORTED;
  const int mq = m < n ? m : n, nt = m < n ? n : m;
  *bytes = size_t(layout(num_pairs, mq, nt, nullptr, true).total);
  return BPBC_OK;
}

int bpbc_sw_workspace_bytes_for(bpbc_sw_ctx* ctx, int64_t num_pairs, int32_t m, int32_t n,
                                int32_t match, int32_t mismatch, int32_t gap, int32_t score_bits,
                                int32_t filter, size_t* bytes) {
  if (!ctx || !bytes) return BPBC_ERR_INVALID_ARG;
  int rc = validate_common(num_pairs, m, n, match, mismatch, gap, score_bits);
  if (rc != BPBC_OK) return rc;
  if (num_pairs == 0) {
    *bytes = 0;
    return BPBC_OK;
  }
  const int mq = m < n ? m : n, nt = m < n ? n : m;
  DeviceGuard dg(ctx->device);
  Dispatch d;
  rc = make_dispatch(ctx, num_pairs, mq, nt, match, -mismatch, -gap, score_bits,
                     filter ? kModeThreshold : kModeMax, &d);
  if (rc != BPBC_OK) return rc;
  *bytes = size_t(layout(num_pairs, mq, nt, &d, filter != 0).total);
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
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset");
    return note_stream(ctx, st);
  }
  RunOut o;
  o.mode = kModeThreshold;
  o.threshold = threshold;
  o.mask = out_mask;
  o.indices = out_indices;
  o.count = out_count;
  return device_call(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits, o,
                     workspace, workspace_bytes, st, false);
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
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const size_t need = wordwise_workspace_bytes(num_pairs);
  void* ws = workspace;
  const bool own = ws == nullptr;
  if (!own) {
    if (workspace_bytes < need) return BPBC_ERR_INVALID_ARG;
  } else {
    if ((rc = buf_acquire(ctx, st)) != BPBC_OK) return rc;
    if ((rc = grow_async(ctx, &ctx->ws, &ctx->ws_bytes, need, st,
                         "cudaMallocAsync(workspace)")) != BPBC_OK)
      return rc;
    ws = ctx->ws;
  }
  const uint8_t* qx = m <= n ? query : target;  // the shorter sequence plays the rows (R17)
  const uint8_t* ty = m <= n ? target : query;
  cudaError_t e = launch_wordwise(qx, ty, num_pairs, mq, nt, match, c2, g, out_scores, ws,
                                  ctx->num_sms, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "wordwise");
  if (own && (rc = buf_release(ctx, st)) != BPBC_OK) return rc;
  return note_stream(ctx, st);
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
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = launch_pack(codes, num_pairs, len, reinterpret_cast<uint2*>(planes),
                              ctx->d_flags, ctx->num_sms, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "pack");
  return note_stream(ctx, st);
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
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = launch_extract(partial, num_groups, lanes, s, num_pairs, 0, cap, out,
                                 ctx->num_sms, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "untranspose");
  return note_stream(ctx, st);
}

int bpbc_sw_get_error_flags(bpbc_sw_ctx* ctx, uint32_t* flags) {
  if (!ctx || !flags) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  // wait for this ctx's enqueued work on every stream it used (not the device)
  cudaError_t e = cudaSuccess;
  for (auto& se : ctx->pending) {
    cudaError_t e2 = cudaEventSynchronize(se.e);
    if (e == cudaSuccess) e = e2;
    cudaEventDestroy(se.e);
  }
  ctx->pending.clear();
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(ctx->h_flags, ctx->d_flags, sizeof(uint32_t), cudaMemcpyDeviceToHost,
                        ctx->aux);
  if (e == cudaSuccess) e = cudaMemsetAsync(ctx->d_flags, 0, sizeof(uint32_t), ctx->aux);
  if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->aux);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "get_error_flags");
  *flags = *ctx->h_flags;
  if (*flags & BPBC_FLAG_STALL) {
    snprintf(ctx->err, sizeof(ctx->err), "a device-side wait timed out (BPBC_FLAG_STALL)");
    return BPBC_ERR_CUDA;
  }
  return (*flags & BPBC_FLAG_BAD_BASE) ? BPBC_ERR_BAD_BASE : BPBC_OK;
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

int bpbc_sw_last_schedule(bpbc_sw_ctx* ctx, int32_t* wrap, int64_t* blocks_per_sm,
                          int32_t* host_streamed) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  if (wrap) *wrap = ctx->plan_wrap;
  if (blocks_per_sm) *blocks_per_sm = ctx->plan_blocks_per_sm;
  if (host_streamed) *host_streamed = ctx->plan_host_streamed;
  return BPBC_OK;
}

int bpbc_sw_profile(bpbc_sw_ctx* ctx, int enable) {
  if (!ctx) return BPBC_ERR_INVALID_ARG;
  DeviceGuard dg(ctx->device);
  // the events of earlier recorded calls are dropped: wait for them first
  for (cudaEvent_t e : ctx->ev_used) cudaEventSynchronize(e);
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
