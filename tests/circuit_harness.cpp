// circuit_harness.cpp -- TEST HARNESS (tests only): runs the product's cell
// circuits (paper_conf_ipps_nishimurabin17_b200/csrc/circuit.cuh, compiled
// for the host, lop3 emulated) so tests/test_circuit_host.py can check them
// against integer arithmetic and, through a row-major bit-sliced DP of one
// 32-pair group, against the oracle.
#include <stdint.h>
#include <string.h>

#include "../paper_conf_ipps_nishimurabin17_b200/csrc/circuit.cuh"

using namespace bpbc;

namespace {

KRun make_krun(int S, int c1, int c2, int g) {
  KRun k;
  memset(&k, 0, sizeof(k));
  for (int i = 0; i < 16; ++i) {
    k.c1mask[i] = (c1 >> i) & 1 ? 0xFFFFFFFFu : 0u;
    k.nmask[i] = ((((1 << S) - c2) & ((1 << S) - 1)) >> i) & 1 ? 0xFFFFFFFFu : 0u;
    k.gmask[i] = (g >> i) & 1 ? 0xFFFFFFFFu : 0u;
  }
  k.zmask = c2 == 0 ? 0xFFFFFFFFu : 0u;
  for (int i = 0; i < 16; ++i) {
    k.amask[i] = ((c1 + g) >> i) & 1 ? 0xFFFFFFFFu : 0u;
    k.bmask[i] = g >= c2 && ((g - c2) >> i) & 1 ? 0xFFFFFFFFu : 0u;
  }
  return k;
}

template <int S>
void slice(const int* v, uint32_t (&w)[S]) {  // 32 values -> S planes
  for (int i = 0; i < S; ++i) {
    w[i] = 0;
    for (int k = 0; k < 32; ++k) w[i] |= uint32_t((v[k] >> i) & 1) << k;
  }
}
template <int S>
void unslice(const uint32_t (&w)[S], int* v) {
  for (int k = 0; k < 32; ++k) {
    v[k] = 0;
    for (int i = 0; i < S; ++i) v[k] |= int((w[i] >> k) & 1) << i;
  }
}

// circuit: 0 exact (KFix<2,1,1>), 1 saturating KFix<2,1,1>, 2 saturating KRun,
// 3 exact KRun (g >= c2)
template <int S>
void cell(int circuit, const KRun& kr, const uint32_t (&up)[S], const uint32_t (&left)[S],
          const uint32_t (&diag)[S], uint32_t xh, uint32_t xl, uint32_t yh, uint32_t yl,
          uint32_t kill, uint32_t (&H)[S], uint32_t (&D)[S]) {
  using K = KFix<2, 1, 1>;
  if (circuit == 0) {
    if (kill) cell_exact<S, K, true>(up, left, diag, xh, xl, yh, yl, kill, H, D, K{});
    else cell_exact<S, K, false>(up, left, diag, xh, xl, yh, yl, 0u, H, D, K{});
  } else if (circuit == 3) {
    if (kill) cell_exact<S, KRun, true>(up, left, diag, xh, xl, yh, yl, kill, H, D, kr);
    else cell_exact<S, KRun, false>(up, left, diag, xh, xl, yh, yl, 0u, H, D, kr);
  } else if (circuit == 1) {
    cell_sat<S, K>(up, left, diag, xh, xl, yh, yl, H, D, K{});
  } else {
    cell_sat<S, KRun>(up, left, diag, xh, xl, yh, yl, H, D, kr);
  }
}

int imax(int a, int b) { return a > b ? a : b; }

template <int S>
long long exhaustive(int circuit, int c1, int c2, int g, int with_kill) {
  const KRun kr = make_krun(S, c1, c2, g);
  const int cap = (1 << S) - 1;
  long long bad = 0;
  int up[32], left[32], diag[32], ref[32], got[32], refd[32], gotd[32];
  uint32_t eword = 0;
  int cnt = 0;
  auto flush = [&](int n) {
    uint32_t U[S], Lf[S], D[S], H[S], Dt[S];
    slice<S>(up, U);
    slice<S>(left, Lf);
    slice<S>(diag, D);
    // x = A (code 0) everywhere; y = A where e = 0, T (code 1) where e = 1
    const uint32_t kill = with_kill ? 0xAAAAAAAAu : 0u;
    cell<S>(circuit, kr, U, Lf, D, 0u, 0u, 0u, eword, kill, H, Dt);
    unslice<S>(H, got);
    unslice<S>(Dt, gotd);
    for (int k = 0; k < n; ++k) {
      const int expect = (kill >> k) & 1 ? 0 : ref[k];
      if (got[k] != expect) ++bad;
      if (gotd[k] != refd[k]) ++bad;  // diagonal term (running-max input)
    }
  };
  for (int a = 0; a <= cap; ++a)
    for (int b = 0; b <= cap; ++b)
      for (int d = 0; d <= cap; ++d)
        for (int e = 0; e < 2; ++e) {
          int r;
          if (circuit == 0 || circuit == 3) {
            // exact circuit domain: no intermediate above the cap
            if (d + c1 + g > cap || a > cap - 0 || b > cap) continue;
            r = imax(0, imax(a - g, imax(b - g, d + (e ? -c2 : c1))));
            refd[cnt] = d + (e ? -c2 : c1) + g;  // D' = diag + w + g
          } else {
            const int T = imax(a, b);
            const int U = imax(T - g, 0);
            const int D = e ? imax(d - c2, 0) : (d + c1 > cap ? cap : d + c1);
            r = imax(U, D);
            refd[cnt] = D;
          }
          up[cnt] = a;
          left[cnt] = b;
          diag[cnt] = d;
          ref[cnt] = r;
          if (e) eword |= 1u << cnt;
          if (++cnt == 32) {
            flush(32);
            cnt = 0;
            eword = 0;
          }
        }
  if (cnt) flush(cnt);
  return bad;
}

// Row-major DP of one 32-pair group with the product's cell + running max
// (P:L336-338 with the fixes of R8).  xp: [m][2] (H, L), yp: [n][2].
template <int S>
void group_dp(int circuit, int c1, int c2, int g, const uint32_t* xp, int m, const uint32_t* yp,
              int n, uint32_t* Mout) {
  const KRun kr = make_krun(S, c1, c2, g);
  // prev[j] = H[i-1][j] planes, j = 0..n (j = 0 border)
  static uint32_t prev[4097][16], cur[4097][16];
  for (int j = 0; j <= n; ++j)
    for (int i = 0; i < S; ++i) prev[j][i] = 0;
  uint32_t M[S] = {0};
  for (int r = 0; r < m; ++r) {
    for (int i = 0; i < S; ++i) cur[0][i] = 0;
    for (int j = 1; j <= n; ++j) {
      uint32_t up[S], left[S], diag[S], H[S], D[S];
      for (int i = 0; i < S; ++i) {
        up[i] = prev[j][i];
        left[i] = cur[j - 1][i];
        diag[i] = prev[j - 1][i];
      }
      cell<S>(circuit, kr, up, left, diag, xp[2 * r], xp[2 * r + 1], yp[2 * (j - 1)],
              yp[2 * (j - 1) + 1], 0u, H, D);
      runmax<S, false>(M, D, 0u);  // max over the diagonal term (finish_exact)
      for (int i = 0; i < S; ++i) cur[j][i] = H[i];
    }
    for (int j = 0; j <= n; ++j)
      for (int i = 0; i < S; ++i) prev[j][i] = cur[j][i];
  }
  if (circuit == 0) {
    uint32_t F[S];
    finish_exact<S, 1>(M, F);  // KFix<2,1,1>: g = 1
    for (int i = 0; i < S; ++i) Mout[i] = F[i];
  } else if (circuit == 3) {  // max D' - g, floored at 0 (finish_exact with runtime g)
    uint32_t F[S];
    ssub_run<S>(M, kr.gmask, F);
    for (int i = 0; i < S; ++i) Mout[i] = F[i];
  } else {
    for (int i = 0; i < S; ++i) Mout[i] = M[i];
  }
}

}  // namespace

#define DISPATCH(S_, CALL)            \
  switch (S_) {                       \
    case 4: return CALL(4);           \
    case 5: return CALL(5);           \
    case 6: return CALL(6);           \
    case 7: return CALL(7);           \
    case 8: return CALL(8);           \
    case 9: return CALL(9);           \
    case 10: return CALL(10);         \
    case 11: return CALL(11);         \
    case 12: return CALL(12);         \
    case 13: return CALL(13);         \
    case 14: return CALL(14);         \
    case 15: return CALL(15);         \
    case 16: return CALL(16);         \
    default: return -1;               \
  }

extern "C" {

long long harness_exhaustive(int circuit, int S, int c1, int c2, int g, int with_kill) {
#define EX(s) exhaustive<s>(circuit, c1, c2, g, with_kill)
  DISPATCH(S, EX)
#undef EX
}

int harness_group_dp(int circuit, int S, int c1, int c2, int g, const uint32_t* xp, int m,
                     const uint32_t* yp, int n, uint32_t* Mout) {
  if (n > 4096) return -2;
#define GD(s) (group_dp<s>(circuit, c1, c2, g, xp, m, yp, n, Mout), 0)
  DISPATCH(S, GD)
#undef GD
}

// Truth-table self-check of the host lop3 emulation and the gate tables.
int harness_gate_tables(void) {
  int bad = 0;
  for (uint32_t a = 0; a < 2; ++a)
    for (uint32_t b = 0; b < 2; ++b)
      for (uint32_t c = 0; c < 2; ++c) {
        const uint32_t A = a ? ~0u : 0u, B = b ? ~0u : 0u, C = c ? ~0u : 0u;
        bad += lop3<kMajNa>(A, B, C) != (((~A & B) | (~A & C) | (B & C)));
        bad += lop3<kSel>(A, B, C) != (a ? B : C);
        bad += lop3<kOrXor>(A, B, C) != (A | (B ^ C));
        bad += lop3<kXor2>(A, B, C) != (A ^ B);
      }
  return bad;
}

}  // extern "C"
