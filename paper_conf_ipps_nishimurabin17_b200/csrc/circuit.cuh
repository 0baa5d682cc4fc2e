// circuit.cuh -- bit-sliced Boolean circuits of the BPBC Smith-Waterman cell.
//
// A value V of width S is held as S 32-bit planes V[0] (LSB) .. V[S-1]; bit k
// of every plane belongs to pair k of the 32-pair group.  Every
// function is a fixed, data-independent sequence of bitwise operations (the
// DP is oblivious).  Each gate is ONE explicit three-input logic op
// (PTX lop3.b32 -> SASS LOP3) with a compile-time truth table, so the
// operation count per cell is exactly the hand count below and the compiler
// cannot re-associate the circuit into more instructions.
//
// The paper's circuits (Sec. IV.A) are the starting point:
//   greaterthan -> lt(): borrow chain, MAJ(~a_i, b_i, p) per bit;
//   max_B -> lt() + mux(): 2 LOP3 per bit (paper: 9s-2 ops);
//   SSub_B -> borrow chain + masked difference, constant
//                           subtrahend folded into the truth tables;
//   add_B -> ripple carry with carry-in 0 (R4: the printed
//                           carry init a0 XOR b0 is wrong);
//   matching_B -> ONE adder whose operand bits are the literals
//                           0 / 1 / e / ~e chosen by the mismatch flag e;
//   SW -> cell_sat() (same structure) and cell_exact()
//                           (offset form, fewer operations).
// Both cells are specified in DESIGN.md ("Cell circuits") with their
// operation counts; tests/test_circuit_host.py runs these same functions on
// the host (lop3 is emulated there) against integer arithmetic.
#pragma once
#include <stdint.h>

#include <type_traits>
#include <utility>

#if defined(__CUDACC__)
#define BPBC_HD __host__ __device__ __forceinline__
#else
#define BPBC_HD inline
#endif

namespace bpbc {

// ---------------------------------------------------------------------------
// Gates.  Truth tables use the PTX convention: inputs a, b, c stand for the
// bytes 0xF0, 0xCC, 0xAA and the table is the expression evaluated on them.
constexpr uint32_t TA = 0xF0, TB = 0xCC, TC = 0xAA;
constexpr uint8_t T8(uint32_t v) { return (uint8_t)(v & 0xFF); }

template <uint8_t LUT>
BPBC_HD uint32_t lop3(uint32_t a, uint32_t b, uint32_t c) {
#if defined(__CUDA_ARCH__)
  uint32_t d;
  asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
  return d;
#else
  uint32_t d = 0;
#pragma unroll
  for (int t = 0; t < 8; ++t)
    if ((LUT >> t) & 1) d |= ((t & 4) ? a : ~a) & ((t & 2) ? b : ~b) & ((t & 1) ? c : ~c);
  return d;
#endif
}

constexpr uint8_t kXor2 = T8(TA ^ TB);                              // a ^ b
constexpr uint8_t kOrXor = T8(TA | (TB ^ TC));                      // a | (b ^ c)
constexpr uint8_t kMajNa = T8((~TA & TB) | (~TA & TC) | (TB & TC));  // MAJ(~a, b, c)
constexpr uint8_t kNaAndB = T8(~TA & TB);                           // ~a & b
constexpr uint8_t kSel = T8((TA & TB) | (~TA & TC));                // a ? b : c
constexpr uint8_t kAndNot = T8(TA & ~TB);                           // a & ~b

// Literal kinds of an adder operand bit chosen by the mismatch flag e:
// w = e ? B_i : A_i  ->  0, 1, e or ~e.
enum : int { kLit0 = 0, kLit1 = 1, kLitE = 2, kLitNE = 3 };
constexpr int lit_kind(uint32_t a_bit, uint32_t b_bit) {
  return a_bit == b_bit ? (a_bit ? kLit1 : kLit0) : (b_bit ? kLitE : kLitNE);
}
constexpr uint32_t lit_tt(int kind) {  // literal as a truth table over input b (= e)
  return kind == kLit0 ? 0u : kind == kLit1 ? 0xFFu : kind == kLitE ? TB : (~TB & 0xFFu);
}
// Adder gates with inputs (x, e, carry): x ^ w ^ c  and  MAJ(x, w, c).
template <int KIND>
constexpr uint8_t kSumLit = T8(TA ^ lit_tt(KIND) ^ TC);
template <int KIND>
constexpr uint8_t kCarryLit = T8((TA & lit_tt(KIND)) | (TA & TC) | (lit_tt(KIND) & TC));

// Compile-time loop: f(std::integral_constant<int, I>) for I in [0, N).
template <class F, int... I>
BPBC_HD void static_for_impl(F&& f, std::integer_sequence<int, I...>) {
  (f(std::integral_constant<int, I>{}), ...);
}
template <int N, class F>
BPBC_HD void static_for(F&& f) {
  static_for_impl(f, std::make_integer_sequence<int, N>{});
}

constexpr uint32_t bitmask(int v, int i) { return ((v >> i) & 1) ? 0xFFFFFFFFu : 0u; }

// ---------------------------------------------------------------------------
// Scoring constants (paper c1, c2, gap as magnitudes).

// Folded at compile time.
template <int C1, int C2, int G>
struct KFix {
  static constexpr bool kFixed = true;
  static constexpr int c1 = C1, c2 = C2, g = G;
};

// From kernel parameters: per-bit masks precomputed on the host, read by the
// gates from the constant bank.
struct KRun {
  static constexpr bool kFixed = false;
  uint32_t c1mask[16];  // bits of c1
  uint32_t nmask[16];   // bits of (2^S - c2) mod 2^S
  uint32_t gmask[16];   // bits of g
  uint32_t zmask;       // all ones iff c2 == 0
  uint32_t amask[16];   // exact circuit: bits of c1 + g (match operand)
  uint32_t bmask[16];   // exact circuit: bits of g - c2 (mismatch operand, g >= c2)
};

// ---------------------------------------------------------------------------
// p = 1 in lane k iff a_k < b_k: the borrow out of a - b.  The paper's
// greaterthan computes the same borrow and returns its
// complement.  S LOP3.
template <int S>
BPBC_HD uint32_t lt(const uint32_t (&a)[S], const uint32_t (&b)[S]) {
  uint32_t p = lop3<kNaAndB>(a[0], b[0], 0u);
#pragma unroll
  for (int i = 1; i < S; ++i) p = lop3<kMajNa>(a[i], b[i], p);
  return p;
}

// out = p ? b : a per lane (the per-bit mux of max_B).  S LOP3.
template <int S>
BPBC_HD void mux(uint32_t p, const uint32_t (&a)[S], const uint32_t (&b)[S], uint32_t (&out)[S]) {
#pragma unroll
  for (int i = 0; i < S; ++i) out[i] = lop3<kSel>(p, b[i], a[i]);
}

// Running maximum M = max(M, H) (R_{k,i} = max_B(d, R_{k,i})) over
// lanes whose kill bit is 0.  2S LOP3 (+1 if kill is not the constant 0).
template <int S, bool KILL>
BPBC_HD void runmax(uint32_t (&M)[S], const uint32_t (&H)[S], uint32_t kill) {
  uint32_t p = lt<S>(M, H);
  if constexpr (KILL) p = lop3<kAndNot>(p, kill, 0u);
  mux<S>(p, M, H, M);
}

// Threshold filter (NEXT-2, the paper's use case P:L231): sticky flag
// F |= (D > T) over lanes whose kill bit is 0.  T's bits come as all-ones /
// all-zeros masks tm[i] (kernel parameters, read from the constant bank by
// the gates).  The borrow out of T - D is lt(T, D) (S LOP3); + 1 to fold it
// into F.  Replaces the 2S-LOP3 running max when only "score > T" is needed.
template <int S, bool KILL>
BPBC_HD void flag_gt(uint32_t& F, const uint32_t (&D)[S], const uint32_t* tm, uint32_t kill) {
  uint32_t p = lop3<kNaAndB>(tm[0], D[0], 0u);
#pragma unroll
  for (int i = 1; i < S; ++i) p = lop3<kMajNa>(tm[i], D[i], p);
  if constexpr (KILL) {
    F = lop3<T8(TA | (TB & ~TC))>(F, p, kill);
  } else {
    F = lop3<T8(TA | TB)>(F, p, 0u);
  }
}

// e = (xH ^ yH) | (xL ^ yL): 1 where the 2-bit bases differ.
BPBC_HD uint32_t mismatch_flag(uint32_t xh, uint32_t xl, uint32_t yh, uint32_t yl) {
  return lop3<kOrXor>(lop3<kXor2>(xh, yh, 0u), xl, yl);
}

// U = max(X - G, 0) for a compile-time G, forced to 0 where kill = 1.
// Borrow chain b_{i+1} = MAJ(~X_i, G_i, b_i), output U_i = (X_i^G_i^b_i) & ~b_S.
// 2S - 1 LOP3 (G_0 = 0: b_1 = 0 is constant-folded by ptxas; G_0 = 1: see below).
//
// When G_0 = 1 the first borrow is b_1 = ~X_0: it is never materialised;
// its two consumers (b_2 and U_1) read X_0 with the inversion folded into
// their truth tables, which saves one gate (2S - 1 in total).
template <int S, int G, bool KILL>
BPBC_HD void ssub_const(const uint32_t (&X)[S], uint32_t kill, uint32_t (&U)[S]) {
  static_assert(S >= 3, "ssub_const needs S >= 3");
  constexpr bool kB1 = (G & 1) != 0;  // b_1 = ~X_0 (virtual)
  uint32_t b[S + 1];
  b[0] = 0u;
  b[1] = 0u;  // (unused when kB1)
  static_for<S>([&](auto I) {
    constexpr int i = decltype(I)::value;
    constexpr uint32_t g = (G >> i) & 1 ? 0xFFu : 0u;
    // borrow input b_i as seen by this gate: TB, or ~TB when it is X_0
    constexpr uint32_t bin = (kB1 && i == 1) ? (~TB & 0xFFu) : TB;
    constexpr uint32_t maj = (~TA & g) | (~TA & bin) | (g & bin);
    if constexpr (kB1 && i == 0) {
      // b_1 = ~X_0: folded into the consumers
    } else if constexpr (i == S - 1 && KILL) {
      // borrow out OR kill, still one gate: inputs (X_i, b_i, kill)
      constexpr uint8_t t = T8((maj & 0xFF) | TC);
      b[i + 1] = lop3<t>(X[i], (kB1 && i == 1) ? X[0] : b[i], kill);
    } else {
      constexpr uint8_t t = T8(maj);
      b[i + 1] = lop3<t>(X[i], (kB1 && i == 1) ? X[0] : b[i], 0u);
    }
  });
  static_for<S>([&](auto I) {
    constexpr int i = decltype(I)::value;
    constexpr uint32_t g = (G >> i) & 1 ? 0xFFu : 0u;
    constexpr uint32_t bin = (kB1 && i == 1) ? (~TB & 0xFFu) : TB;
    constexpr uint8_t t = T8((TA ^ g ^ bin) & ~TC);  // (X_i ^ G_i ^ b_i) & ~b_S
    U[i] = lop3<t>(X[i], (kB1 && i == 1) ? X[0] : b[i], b[S]);
  });
}

// Same with G from per-bit masks in memory (KRun).  3S LOP3.
template <int S>
BPBC_HD void ssub_run(const uint32_t (&X)[S], const uint32_t* gm, uint32_t (&U)[S]) {
  uint32_t b[S + 1], d[S];
  b[0] = 0u;
#pragma unroll
  for (int i = 0; i < S; ++i) {
    d[i] = lop3<T8(TA ^ TB ^ TC)>(X[i], gm[i], b[i]);
    b[i + 1] = lop3<kMajNa>(X[i], gm[i], b[i]);
  }
#pragma unroll
  for (int i = 0; i < S; ++i) U[i] = lop3<kAndNot>(d[i], b[S], 0u);
}

// ---------------------------------------------------------------------------
// Exact ("offset") cell.  Valid when c1*min(m,n) + g <= 2^S - 1 and g >= c2
// (then no intermediate overflows and nothing goes negative):
//   e  = (xH ^ yH) | (xL ^ yL)                  mismatch flag
//   D' = diag + (e ? g - c2 : c1 + g)           one ripple adder
//   X  = max(up, max(left, D'))                 two max_B
//   H  = max(X - g, 0)  = max(0, up-g, left-g, diag+w)
// kill forces H = 0 (rows past m).  LOP3 per word-cell with compile-time
// constants: 2 + (2S - 1) + 4S + (2S - 1) = 8S, 10S with the running max
// (S = 9: 90; the paper's Theorem 6 + Lemma 2 count 57S - 19 = 494).  With
// runtime constants (KRun, per-bit masks): the adder operand is selected per
// bit (+S), the gap subtract reads g's masks (3S): 10S + 1, 12S + 1 with the
// running max (the saturating runtime circuit costs 13S + 4).
//
// Dp receives D' (the diagonal term).  The running maximum is taken over D'
// instead of H (see finish_exact below), so it never waits for the
// comparator chain.
template <int S, class K, bool KILL>
BPBC_HD void cell_exact(const uint32_t (&up)[S], const uint32_t (&left)[S],
                        const uint32_t (&diag)[S], uint32_t xh, uint32_t xl, uint32_t yh,
                        uint32_t yl, uint32_t kill, uint32_t (&H)[S], uint32_t (&Dp)[S],
                        const K& k) {
  const uint32_t e = mismatch_flag(xh, xl, yh, yl);
  uint32_t D[S];
  uint32_t c = 0u;
  if constexpr (K::kFixed) {
    static_assert(K::g >= K::c2, "exact cell needs g >= c2");
    constexpr int A = K::c1 + K::g, B = K::g - K::c2;
    static_for<S>([&](auto I) {
      constexpr int i = decltype(I)::value;
      constexpr int kind = lit_kind((A >> i) & 1, (B >> i) & 1);
      D[i] = lop3<kSumLit<kind>>(diag[i], e, c);
      if constexpr (i + 1 < S) c = lop3<kCarryLit<kind>>(diag[i], e, c);
    });
  } else {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      const uint32_t w = lop3<kSel>(e, k.bmask[i], k.amask[i]);  // e ? g - c2 : c1 + g
      D[i] = lop3<T8(TA ^ TB ^ TC)>(diag[i], w, c);
      if (i + 1 < S) c = lop3<T8((TA & TB) | (TA & TC) | (TB & TC))>(diag[i], w, c);
    }
  }
  // X = max(up, max(left, D')): the inner max does not depend on `up` (the
  // previous row's fresh output), so only one comparator + mux + the gap
  // subtract sit on the row-to-row dependency chain (2S+1 deep instead of
  // 3S+2); same gate count as max(max(up, left), D').
  uint32_t T[S], X[S];
  mux<S>(lt<S>(left, D), left, D, T);
  mux<S>(lt<S>(up, T), up, T, X);
  if constexpr (K::kFixed) {
    ssub_const<S, K::g, KILL>(X, kill, H);
  } else {
    ssub_run<S>(X, k.gmask, H);
    if constexpr (KILL) {
#pragma unroll
      for (int i = 0; i < S; ++i) H[i] = lop3<kAndNot>(H[i], kill, 0u);
    }
  }
#pragma unroll
  for (int i = 0; i < S; ++i) Dp[i] = D[i];
}

// Maximum over cells taken on the diagonal term.  The cell holding the
// largest score H* > 0 got it from its diagonal input: if H* came from
// up - g or left - g, that neighbour would hold H* + g > H*.  Every D <= H.
// Hence max_ij H = max(0, max_ij D) with D = diag + w (saturating cell), and
// max_ij H = max(0, max_ij D' - g) with D' = diag + w + g (exact cell).  The
// lane keeps M over D (2S LOP3 per cell, as over H); for the exact circuit
// the sweep stores max D' and extract.cu subtracts g from the untransposed
// integer once per pair (finish_exact is the bit-sliced form of that step,
// used by the host circuit tests).  D is ready long before H, so the M chain
// runs beside the comparator chain instead of after it.
template <int S, int G>
BPBC_HD void finish_exact(const uint32_t (&Mp)[S], uint32_t (&M)[S]) {
  ssub_const<S, G, false>(Mp, 0u, M);
}

// ---------------------------------------------------------------------------
// Saturating cell (the paper's SW function, with the R3 / R4 / R19
// fixes).  Valid for any constants <= 2^S - 1.  It computes values that are
// <= the exact ones and equal to them below the cap, so that the maximum over
// all cells is exactly min(max_exact, 2^S - 1) (R3).
//   T = max(up, left);  U = max(T - g, 0)
//   D = e ? max(diag - c2, 0) : min(diag + c1, 2^S - 1)    (one adder)
//   H = max(D, U)
// LOP3 per word-cell with compile-time constants: 2 + 2S + 2S + 3S + 2S =
// 9S + 2, 11S + 2 with the running max.
// D receives the diagonal term (see finish_exact above).
template <int S, class K>
BPBC_HD void cell_sat(const uint32_t (&up)[S], const uint32_t (&left)[S],
                      const uint32_t (&diag)[S], uint32_t xh, uint32_t xl, uint32_t yh,
                      uint32_t yl, uint32_t (&H)[S], uint32_t (&D)[S], const K& k) {
  const uint32_t e = mismatch_flag(xh, xl, yh, yl);
  uint32_t T[S], U[S];
  mux<S>(lt<S>(up, left), up, left, T);
  if constexpr (K::kFixed) {
    ssub_const<S, K::g, false>(T, 0u, U);
  } else {
    ssub_run<S>(T, k.gmask, U);
  }
  uint32_t s[S];
  uint32_t c = 0u;
  if constexpr (K::kFixed) {
    constexpr int N = ((1 << S) - K::c2) & ((1 << S) - 1);  // mismatch operand
    static_for<S>([&](auto I) {
      constexpr int i = decltype(I)::value;
      constexpr int kind = lit_kind((K::c1 >> i) & 1, (N >> i) & 1);
      s[i] = lop3<kSumLit<kind>>(diag[i], e, c);
      c = lop3<kCarryLit<kind>>(diag[i], e, c);
    });
    if constexpr (K::c2 != 0) {
      // match: carry out = overflow -> all ones; mismatch: carry out = no
      // borrow -> keep, else 0.  Inputs (e, s_i, c).
      constexpr uint8_t t = T8((TA & (TB & TC)) | (~TA & (TB | TC)));
#pragma unroll
      for (int i = 0; i < S; ++i) D[i] = lop3<t>(e, s[i], c);
    } else {
      // mismatch adds 0 and never carries: D = s | c covers both cases (R19).
#pragma unroll
      for (int i = 0; i < S; ++i) D[i] = lop3<T8(TA | TB)>(s[i], c, 0u);
    }
  } else {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      const uint32_t w = lop3<kSel>(e, k.nmask[i], k.c1mask[i]);
      s[i] = lop3<T8(TA ^ TB ^ TC)>(diag[i], w, c);
      c = lop3<T8((TA & TB) | (TA & TC) | (TB & TC))>(diag[i], w, c);
    }
    // a = ~e | c | z, o = ~e & c; D_i = (s_i & a) | o   (c2 == 0 -> z = ~0, R19)
    const uint32_t a = lop3<T8(~TA | TB | TC)>(e, c, k.zmask);
    const uint32_t o = lop3<T8(~TA & TB)>(e, c, 0u);
#pragma unroll
    for (int i = 0; i < S; ++i) D[i] = lop3<T8((TA & TB) | TC)>(s[i], a, o);
  }
  mux<S>(lt<S>(U, D), U, D, H);
}

}  // namespace bpbc
