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
  size_t ws_h_bytes[2] = {0, 0};
  char err[512] = {0};
  // last plan
  int32_t plan_circuit = -1, plan_width = 0, plan_R = 0, plan_L = 0, plan_ops = 0;
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

SweepEntry g_table[kNumVariants][kNumRL][13];
SweepEntry g_striped[3][13];
std::once_flag g_table_once;

void init_table() {
  memset(g_table, 0, sizeof(g_table));
  memset(g_striped, 0, sizeof(g_striped));
  register_striped_s4(g_striped);
  register_striped_s5(g_striped);
  register_striped_s6(g_striped);
  register_striped_s7(g_striped);
  register_striped_s8(g_striped);
  register_striped_s9(g_striped);
  register_striped_s10(g_striped);
  register_striped_s11(g_striped);
  register_striped_s12(g_striped);
  register_striped_s13(g_striped);
  register_striped_s14(g_striped);
  register_striped_s15(g_striped);
  register_striped_s16(g_striped);
  register_sweep_s4(g_table);
  register_sweep_s5(g_table);
  register_sweep_s6(g_table);
  register_sweep_s7(g_table);
  register_sweep_s8(g_table);
  register_sweep_s9(g_table);
  register_sweep_s10(g_table);
  register_sweep_s11(g_table);
  register_sweep_s12(g_table);
  register_sweep_s13(g_table);
  register_sweep_s14(g_table);
  register_sweep_s15(g_table);
  register_sweep_s16(g_table);
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
  int stripes = 1;             // > 1 only for the long-query (striped) kernel
  int64_t bnd_streams = 0;     // streams the boundary buffer has room for
  int64_t x_off = 0, y_off = 0, mp_off = 0, bnd_off = 0, zero_off = 0, total = 0;
};

int64_t align256(int64_t v) { return (v + 255) & ~int64_t(255); }

Layout layout(int64_t P, int mq, int nt) {
  Layout L;
  L.G = (P + 31) / 32;
  // room for the striped kernel whenever the plan may pick it (m > 128)
  L.stripes = mq > kStripeRows ? (mq + kStripeRows - 1) / kStripeRows : 1;
  const int64_t xbytes = (L.G * mq + kXBackPad) * 8;
  const int64_t ybytes = (kYFrontPad + L.G * nt + nt + kYBackPadExtra) * 8;
  const int64_t mpbytes = L.G * L.stripes * 32 * 16 * 4;
  int64_t bnd_bytes = 0;
  if (L.stripes > 1) {
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
  if (spec && g >= c2) {
    int s_ex = bit_length(int64_t(c1) * mq + g);
    if (s_ex < BPBC_MIN_SCORE_BITS) s_ex = BPBC_MIN_SCORE_BITS;
    if (s_ex <= BPBC_MAX_SCORE_BITS && 10 * s_ex <= cost_sat) {
      p->circuit = kExact;
      p->consts = kC211;
      p->width = s_ex;
      p->ops = 10 * s_ex;
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

// Enqueue pack -> sweep -> extract on device buffers.
int run_device(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target, int64_t P, int m,
               int n, int match, int mismatch, int gap, int S, int32_t* out, uint8_t* ws,
               cudaStream_t st) {
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
  Plan plan;
  int rc = make_plan(mq, c1, c2, g, S, &plan);
  if (rc != BPBC_OK) return rc;
  const Layout lay = layout(P, mq, nt);
  uint2* Xp = reinterpret_cast<uint2*>(ws + lay.x_off);
  uint2* Ybase = reinterpret_cast<uint2*>(ws + lay.y_off);
  uint2* Yp = Ybase + kYFrontPad;
  uint32_t* Mpart = reinterpret_cast<uint32_t*>(ws + lay.mp_off);

  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  if (ctx->profiling)
    for (int i = 0; i < 4; ++i) ev[i] = ctx->take_event();
  if (ev[0]) cudaEventRecord(ev[0], st);
  cudaError_t e = launch_pack2(qx, mq, Xp, ty, nt, Yp, P, ctx->d_flags, ctx->num_sms, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "pack");

  if (ev[1]) cudaEventRecord(ev[1], st);
  std::call_once(g_table_once, init_table);
  const bool striped = plan.rl < 0;
  const SweepEntry ent =
      striped ? g_striped[plan.circuit == kExact ? 0 : (plan.consts == kC211 ? 1 : 2)]
                         [plan.width - 4]
              : g_table[variant_index(plan.circuit, plan.consts, plan.pad)][plan.rl]
                       [plan.width - 4];
  if (!ent.launch) return BPBC_ERR_UNSUPPORTED;
  const int R = striped ? kStripeR : kRLR[plan.rl], L = striped ? 32 : kRLL[plan.rl];
  int nb = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, ent.func, 128, 0);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "occupancy");
  if (nb < 1) nb = 1;
  const int64_t segs = 32 / L;
  int64_t cap_streams = int64_t(ctx->num_sms) * nb * 4 * segs;
  if (striped && cap_streams > lay.bnd_streams) cap_streams = lay.bnd_streams;
  SweepArgs a;
  a.Xp = Xp;
  a.Yp = Yp;
  a.Mpart = Mpart;
  a.G = lay.G;
  a.m = mq;
  a.n = nt;
  a.streams = lay.G < cap_streams ? lay.G : cap_streams;
  a.base = lay.G / a.streams;
  a.rem = lay.G % a.streams;
  a.stripes = striped ? (mq + kStripeRows - 1) / kStripeRows : 1;
  a.bnd = reinterpret_cast<uint32_t*>(ws + lay.bnd_off);
  a.bzero = reinterpret_cast<const uint32_t*>(ws + lay.zero_off);
  a.steps = (a.base + (a.rem > 0 ? 1 : 0)) * a.stripes * int64_t(nt) + L;
  if (striped) {
    e = cudaMemsetAsync(ws + lay.zero_off, 0, 256, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "memset(zero row)");
  }
  const int64_t warps = (a.streams + segs - 1) / segs;
  const int grid = int((warps + 3) / 4);
  KRun kr;
  memset(&kr, 0, sizeof(kr));
  const int W = plan.width;
  for (int i = 0; i < 16; ++i) {
    kr.c1mask[i] = (c1 >> i) & 1 ? 0xFFFFFFFFu : 0u;
    kr.nmask[i] = ((((1 << W) - c2) & ((1 << W) - 1)) >> i) & 1 ? 0xFFFFFFFFu : 0u;
    kr.gmask[i] = (g >> i) & 1 ? 0xFFFFFFFFu : 0u;
  }
  kr.zmask = c2 == 0 ? 0xFFFFFFFFu : 0u;
  ent.launch(a, kr, grid, 128, st);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(ctx, e, "sweep");
  if (ev[2]) cudaEventRecord(ev[2], st);
  e = launch_extract(Mpart, lay.G, L * a.stripes, W, P, plan.cap, out, ctx->num_sms, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "extract");
  if (ev[3]) cudaEventRecord(ev[3], st);

  ctx->plan_circuit = plan.circuit;
  ctx->plan_width = W;
  ctx->plan_R = R;
  ctx->plan_L = L;
  ctx->plan_ops = plan.ops;
  ctx->plan_streams = a.streams;
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
  return run_device(ctx, query, target, num_pairs, m, n, match, mismatch, gap, score_bits,
                    out_scores, ws, static_cast<cudaStream_t>(stream));
}

int bpbc_sw_score_batch_host(bpbc_sw_ctx* ctx, const uint8_t* query, const uint8_t* target,
                             int64_t num_pairs, int32_t m, int32_t n, int32_t match,
                             int32_t mismatch, int32_t gap, int32_t score_bits,
                             int32_t* out_scores) {
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
  const size_t qb = size_t(num_pairs) * m, tb = size_t(num_pairs) * n,
               ob = size_t(num_pairs) * sizeof(int32_t);
  // chunks of >= 64K pairs (multiples of 32), at most 8
  int64_t nchunks = (num_pairs + 65535) / 65536;
  if (nchunks > 8) nchunks = 8;
  if (nchunks < 1) nchunks = 1;
  int64_t chunk = (num_pairs + nchunks - 1) / nchunks;
  chunk = (chunk + 31) / 32 * 32;
  size_t need = 0;
  bpbc_sw_workspace_bytes(chunk < num_pairs ? chunk : num_pairs, m, n, &need);
  if ((rc = grow(ctx, (void**)&ctx->d_q, &ctx->d_q_bytes, qb, "cudaMalloc(q)")) != BPBC_OK) return rc;
  if ((rc = grow(ctx, (void**)&ctx->d_t, &ctx->d_t_bytes, tb, "cudaMalloc(t)")) != BPBC_OK) return rc;
  if ((rc = grow(ctx, (void**)&ctx->d_out, &ctx->d_out_bytes, ob, "cudaMalloc(out)")) != BPBC_OK)
    return rc;
  for (int i = 0; i < 2; ++i)
    if ((rc = grow(ctx, &ctx->ws_h[i], &ctx->ws_h_bytes[i], need, "cudaMalloc(workspace)")) !=
        BPBC_OK)
      return rc;
  for (int64_t c0 = 0, ci = 0; c0 < num_pairs; c0 += chunk, ++ci) {
    const int64_t cp = num_pairs - c0 < chunk ? num_pairs - c0 : chunk;
    cudaStream_t st = ctx->host_streams[ci & 1];
    e = cudaMemcpyAsync(ctx->d_q + c0 * m, query + c0 * m, size_t(cp) * m,
                        cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(ctx->d_t + c0 * n, target + c0 * n, size_t(cp) * n,
                          cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "H2D");
    rc = run_device(ctx, ctx->d_q + c0 * m, ctx->d_t + c0 * n, cp, m, n, match, mismatch, gap,
                    score_bits, ctx->d_out + c0, static_cast<uint8_t*>(ctx->ws_h[ci & 1]), st);
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
  cudaError_t e = launch_extract(partial, num_groups, lanes, s, num_pairs, cap, out,
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
