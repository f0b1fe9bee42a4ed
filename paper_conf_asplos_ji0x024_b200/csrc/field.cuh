// Field layer: Montgomery arithmetic over F_p on radix-2^W limbs.
//
// What it computes is PAPER.md Alg. 2: C = A*B*R^-1 mod p with the
// word-serial m[i] = C[i]*n'_0.  How it computes it is B200-specific
// (DESIGN.md "Field layer"):
//   * limbs are W = 30 (29 for MNT4-753) bits in 32-bit registers, R = 2^(W*L);
//   * every limb product is one IMAD.WIDE.U32 (32x32 -> 64 with 64-bit addend), which
//     runs at the full 64/clk/SM IMAD rate on sm_100a, whereas IMAD.HI.U32 runs at
//     half rate (microbench/imad_peak.cu); a column of products accumulates in a 64-bit
//     register with no carry propagation (finely-integrated product scanning, the FIPS
//     variant PAPER.md:119 cites from [23]);
//   * lazy reduction: values are kept in [0, B*p) with B <= KMAX and
//     limbs normalised (< 2^W); a Montgomery product of inputs < 10p is < 2p
//     (tools/gen_params.py asserts it per curve).  Only values leaving the library are
//     fully reduced.
#pragma once
#include <cstdint>
#include "params.h"

typedef unsigned long long u64;

#define DEVI __device__ __forceinline__

#ifndef MSM_FMUL2_LAT
#define MSM_FMUL2_LAT 0  // A/B: fmul2 columns with the a*b chain split in two (6 chains per warp)
#endif

#ifndef MSM_FSQR_AS_MUL
#define MSM_FSQR_AS_MUL 0
#endif

// One IMAD.WIDE.U32 (a*b + c, 64-bit addend).  The product is an explicit PTX
// mul.wide.u32 and the add is C++: ptxas then emits a clean IMAD.WIDE.U32 chain.
// (An inline-asm mad.wide.u32 chain gets re-associated into IMAD.WIDE + IADD3 trees,
// and a C++ (u64)a*b with a constant b becomes a 64x64 multiply with dead hi-word
// adds — both checked with cuobjdump -sass.)
DEVI u64 mad_wide(uint32_t a, uint32_t b, u64 c) {
  u64 p;
  asm("mul.wide.u32 %0, %1, %2;" : "=l"(p) : "r"(a), "r"(b));
  return p + c;
}

template <class C>
struct Fp {
  static constexpr int L = C::L;
  uint32_t v[C::L];
};

// ---- r = a*b*R^-1 mod p (lazy: result < 2p for inputs < 10p) ----
// Column k of the product scan (FIPS) accumulates, as IMAD.WIDE.U32 chains,
//   the a*b terms  a_i b_{k-i}   (SQR: a_i (2a_{k-i}) for i < k-i, plus a_{k/2}^2)
//   the m*p terms  m_i p_{k-i}   (i < k), then m_k = t_k n'_0 mod 2^W and + m_k p_0 (k < L).
// A 64-bit accumulator holds MAXT = floor(2^64 / 2^(2W)) - 1 products of W-bit limbs plus
// the incoming carry; a column with more terms splits them over two accumulators (a*b
// and m*p) whose carries travel separately.  Edge columns (few terms) use one chain and
// a cheaper epilogue.
// One column as a template instance: every index below is a compile-time constant, so
// the whole product scan is straight-line code on registers (no reliance on the loop
// unroller, which gives up on 25 large column bodies and then spills m[] to local memory).
// LAT (latency mode, for single-thread serial tails): the a*b products of a column form
// two chains that start from 0 — independent of every earlier column — and the carry is
// added afterwards, so a lone warp overlaps the columns instead of walking one long
// dependency chain (2 extra ALU ops per column, irrelevant off the throughput path).
// Shape of product-scan column K: a*b terms i in [lo, hiA], m*p terms i in [lo, hiM] plus
// m_K p_0 (K < L).  A 64-bit accumulator holds MAXT products of W-bit limbs plus a carry;
// a column with more terms splits a*b and m*p over two accumulators ("split").
template <class C>
__host__ __device__ constexpr bool col_single(int K) {
  const int L = C::L, W = C::W;
  const int MAXT = (W == 30) ? 15 : (W == 29 ? 63 : 255);
  const int lo = K - L + 1 > 0 ? K - L + 1 : 0;
  const int hiA = K < L - 1 ? K : L - 1;
  const int hiM = (K - 1) < (L - 1) ? K - 1 : L - 1;
  const int nA = hiA - lo + 1;
  const int nM = (hiM >= lo ? hiM - lo + 1 : 0) + (K < L ? 1 : 0);
  return (C::NACC == 1) || (nA + nM <= MAXT);
}

template <class C, int K>
struct ColShape {
  static constexpr int L = C::L;
  static constexpr int lo = K - L + 1 > 0 ? K - L + 1 : 0;
  static constexpr int hiA = K < L - 1 ? K : L - 1;
  static constexpr int hiM = (K - 1) < (L - 1) ? K - 1 : L - 1;
  static constexpr bool single = col_single<C>(K);
  static constexpr bool prev_split = K > 0 && !col_single<C>(K - 1);
};

template <class C, bool SQR, bool LAT, int K>
DEVI void fmul_step(uint32_t* r, const uint32_t* a, const uint32_t* b, const uint32_t* a2, uint32_t* m, u64& cA, u64& cM) {
  using S = ColShape<C, K>;
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  constexpr int lo = S::lo, hiA = S::hiA, hiM = S::hiM;
  constexpr bool single = S::single, PREV_SPLIT = S::prev_split;
  u64 accA;
  if constexpr (LAT) {
    u64 e0 = 0, e1 = 0;
    if constexpr (SQR) {
#pragma unroll
      for (int i = lo; i < K - i; i++) {
        if ((i - lo) & 1) e1 = mad_wide(a[i], a2[K - i], e1);
        else e0 = mad_wide(a[i], a2[K - i], e0);
      }
      if constexpr ((K & 1) == 0) e1 = mad_wide(a[K >> 1], a[K >> 1], e1);
    } else {
#pragma unroll
      for (int i = lo; i <= hiA; i++) {
        if ((i - lo) & 1) e1 = mad_wide(a[i], b[K - i], e1);
        else e0 = mad_wide(a[i], b[K - i], e0);
      }
    }
    accA = e0 + e1 + cA;
  } else {
    accA = cA;
    if constexpr (SQR) {
#pragma unroll
      for (int i = lo; i < K - i; i++) accA = mad_wide(a[i], a2[K - i], accA);
      if constexpr ((K & 1) == 0) accA = mad_wide(a[K >> 1], a[K >> 1], accA);
    } else {
#pragma unroll
      for (int i = lo; i <= hiA; i++) accA = mad_wide(a[i], b[K - i], accA);
    }
  }
  u64 nA_carry, nM_carry;
  if constexpr (single) {
    u64 acc = PREV_SPLIT ? accA + cM : accA;
#pragma unroll
    for (int i = lo; i <= hiM; i++) acc = mad_wide(m[i], C::P(K - i), acc);
    if constexpr (K < L) {
      m[K] = ((uint32_t)acc * C::N0) & MASK;
      acc = mad_wide(m[K], C::P(0), acc);
    } else {
      r[K - L] = (uint32_t)acc & MASK;
    }
    nA_carry = acc >> W;
    nM_carry = 0;
  } else {
    u64 accM = PREV_SPLIT ? cM : 0;
#pragma unroll
    for (int i = lo; i <= hiM; i++) accM = mad_wide(m[i], C::P(K - i), accM);
    if constexpr (K < L) {
      uint32_t s = (uint32_t)accA + (uint32_t)accM;
      m[K] = (s * C::N0) & MASK;
      accM = mad_wide(m[K], C::P(0), accM);
      uint32_t loA = (uint32_t)accA & MASK, loM = (uint32_t)accM & MASK;
      nA_carry = accA >> W;
      nM_carry = (accM >> W) + ((loA + loM) >> W);
    } else {
      uint32_t s = ((uint32_t)accA & MASK) + ((uint32_t)accM & MASK);
      r[K - L] = s & MASK;
      nA_carry = accA >> W;
      nM_carry = (accM >> W) + (s >> W);
    }
  }
  if constexpr (K == 2 * L - 2) r[L - 1] = (uint32_t)(single ? nA_carry : nA_carry + nM_carry);
  cA = nA_carry;
  cM = nM_carry;
}

// One column per template instance: every index is a compile-time constant, so the whole
// product scan is straight-line code on registers (no reliance on the loop unroller, which
// gives up on 25 large column bodies and then spills m[] to local memory).
template <class C, bool SQR, bool LAT, int K>
DEVI void fmul_cols(uint32_t* r, const uint32_t* a, const uint32_t* b, const uint32_t* a2, uint32_t* m, u64 cA, u64 cM) {
  fmul_step<C, SQR, LAT, K>(r, a, b, a2, m, cA, cM);
  if constexpr (K + 1 < 2 * C::L - 1) fmul_cols<C, SQR, LAT, K + 1>(r, a, b, a2, m, cA, cM);
}

// Two independent products column-interleaved: four accumulation chains instead of two,
// so the IMAD.WIDE latency of one product's column hides behind the other's (ILP without
// more warps; the accumulation kernel runs at 2 warps per scheduler).  r1 / r2 may alias
// their OWN inputs only (as for fmul), never the other product's inputs.
template <class C, bool SQR, int K>
DEVI void fmul2_cols(uint32_t* r1, const uint32_t* a1, const uint32_t* b1, const uint32_t* a21, uint32_t* m1,
                     u64 cA1, u64 cM1, uint32_t* r2, const uint32_t* a2, const uint32_t* b2, const uint32_t* a22,
                     uint32_t* m2, u64 cA2, u64 cM2) {
  fmul_step<C, SQR, MSM_FMUL2_LAT != 0, K>(r1, a1, b1, a21, m1, cA1, cM1);
  fmul_step<C, SQR, MSM_FMUL2_LAT != 0, K>(r2, a2, b2, a22, m2, cA2, cM2);
  if constexpr (K + 1 < 2 * C::L - 1)
    fmul2_cols<C, SQR, K + 1>(r1, a1, b1, a21, m1, cA1, cM1, r2, a2, b2, a22, m2, cA2, cM2);
}

// Three independent products column-interleaved (six accumulation chains in split
// columns): the PACC groups {PPP, Q, ZZ'} and {ZZZ', T, E} each need only values of the
// previous group, so a warp can keep three products in flight (ILP at 2 warps/scheduler).
template <class C, int K>
DEVI void fmul3_cols(uint32_t* r1, const uint32_t* a1, const uint32_t* b1, uint32_t* m1, u64 cA1, u64 cM1,
                     uint32_t* r2, const uint32_t* a2, const uint32_t* b2, uint32_t* m2, u64 cA2, u64 cM2,
                     uint32_t* r3, const uint32_t* a3, const uint32_t* b3, uint32_t* m3, u64 cA3, u64 cM3) {
  fmul_step<C, false, false, K>(r1, a1, b1, a1, m1, cA1, cM1);
  fmul_step<C, false, false, K>(r2, a2, b2, a2, m2, cA2, cM2);
  fmul_step<C, false, false, K>(r3, a3, b3, a3, m3, cA3, cM3);
  if constexpr (K + 1 < 2 * C::L - 1)
    fmul3_cols<C, K + 1>(r1, a1, b1, m1, cA1, cM1, r2, a2, b2, m2, cA2, cM2, r3, a3, b3, m3, cA3, cM3);
}

// r1 = a1*b1, r2 = a2*b2, r3 = a3*b3 (same contract as fmul; each r may alias its OWN inputs only)
template <class C>
DEVI void fmul3(uint32_t* r1, const uint32_t* a1, const uint32_t* b1, uint32_t* r2, const uint32_t* a2,
                const uint32_t* b2, uint32_t* r3, const uint32_t* a3, const uint32_t* b3) {
  constexpr int L = C::L;
  uint32_t m1[L], m2[L], m3[L];
  fmul3_cols<C, 0>(r1, a1, b1, m1, 0ull, 0ull, r2, a2, b2, m2, 0ull, 0ull, r3, a3, b3, m3, 0ull, 0ull);
}

// ---- r = (a*b + c*d) * R^-1 mod p with ONE Montgomery reduction (lazy reduction of a
// sum of products): the a*b, c*d and m*p terms of a column accumulate in three
// IMAD.WIDE chains (each <= L products of < 2^(2W), within MAXT), their low words are added
// for m_K, and the three carries travel separately.  Saves the L^2 + L reduction products of
// a second multiplication.  Bound: for inputs with a*b + c*d < 68 p^2 the result is < 2p on
// every curve here (R/p >= 2^9.3).
template <class C, int K>
DEVI void fsum_step(uint32_t* r, const uint32_t* a, const uint32_t* b, const uint32_t* c, const uint32_t* d, uint32_t* m,
                    u64& cA, u64& cB, u64& cM) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  constexpr int lo = K - L + 1 > 0 ? K - L + 1 : 0;
  constexpr int hiA = K < L - 1 ? K : L - 1;
  constexpr int hiM = (K - 1) < (L - 1) ? K - 1 : L - 1;
  u64 accA = cA, accB = cB, accM = cM;
#pragma unroll
  for (int i = lo; i <= hiA; i++) {
    accA = mad_wide(a[i], b[K - i], accA);
    accB = mad_wide(c[i], d[K - i], accB);
  }
#pragma unroll
  for (int i = lo; i <= hiM; i++) accM = mad_wide(m[i], C::P(K - i), accM);
  const uint32_t t = ((uint32_t)accA & MASK) + ((uint32_t)accB & MASK);  // < 2^(W+1)
  if constexpr (K < L) {
    const uint32_t s = t + ((uint32_t)accM & MASK);                        // < 3 * 2^W
    m[K] = (s * C::N0) & MASK;
    accM = mad_wide(m[K], C::P(0), accM);
    const uint32_t s2 = t + ((uint32_t)accM & MASK);                       // 0, 2^W or 2^(W+1)
    cM = (accM >> W) + (s2 >> W);
  } else {
    const uint32_t s = t + ((uint32_t)accM & MASK);
    r[K - L] = s & MASK;
    cM = (accM >> W) + (s >> W);
  }
  cA = accA >> W;
  cB = accB >> W;
  if constexpr (K == 2 * L - 2) r[L - 1] = (uint32_t)(cA + cB + cM);
}

template <class C, int K>
DEVI void fsum_cols(uint32_t* r, const uint32_t* a, const uint32_t* b, const uint32_t* c, const uint32_t* d, uint32_t* m,
                    u64 cA, u64 cB, u64 cM) {
  fsum_step<C, K>(r, a, b, c, d, m, cA, cB, cM);
  if constexpr (K + 1 < 2 * C::L - 1) fsum_cols<C, K + 1>(r, a, b, c, d, m, cA, cB, cM);
}

// r = a*b + c*d (Montgomery), r may alias any input
template <class C>
DEVI void fmul_sum(uint32_t* r, const uint32_t* a, const uint32_t* b, const uint32_t* c, const uint32_t* d) {
  uint32_t m[C::L], t[C::L];
  fsum_cols<C, 0>(t, a, b, c, d, m, 0ull, 0ull, 0ull);
#pragma unroll
  for (int i = 0; i < C::L; i++) r[i] = t[i];
}

#ifndef MSM_ROWS
#define MSM_ROWS 0  // A/B: MNT4-753 products by operand scanning (fmul_rows) instead of columns
#endif

// Operand scanning with delayed carries, for the 27-limb field: row i adds a_i * b and
// m_i * p into 64-bit column accumulators T[i..i+L) — L independent IMAD.WIDE chains per
// row instead of one 54-deep chain per column (MNT4-753's accumulation is latency-bound:
// r01 ncu "wait" 5.5 stalls per issue at 2 warps per scheduler).  m_i = T_i n'_0 mod 2^W
// (T_i complete: every earlier row has added its terms and its carry), then T_{i+1} +=
// T_i >> W.  A column gets <= 2L products of (2^W + 3)^2 plus carries < 2^35: < 2^64 for
// W = 29, L = 27.  Same result and bounds as the column form.
template <class C>
DEVI void fmul_rows(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  u64 T[2 * L];
#pragma unroll
  for (int k = 0; k < 2 * L; k++) T[k] = 0;
#pragma unroll
  for (int i = 0; i < L; i++) {
#pragma unroll
    for (int j = 0; j < L; j++) T[i + j] = mad_wide(a[i], b[j], T[i + j]);
    const uint32_t m = ((uint32_t)T[i] * C::N0) & MASK;
#pragma unroll
    for (int j = 0; j < L; j++)
      if (C::P(j) != 0u) T[i + j] = mad_wide(m, C::P(j), T[i + j]);
    T[i + 1] += T[i] >> W;
  }
  u64 c = 0;
#pragma unroll
  for (int k = 0; k < L - 1; k++) {
    const u64 v = T[L + k] + c;
    r[k] = (uint32_t)v & MASK;
    c = v >> W;
  }
  r[L - 1] = (uint32_t)c;
}

template <class C, bool SQR, bool LAT = false>
DEVI void fmul_impl(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  if constexpr (MSM_ROWS != 0 && C::L > 13) {
    fmul_rows<C>(r, a, b);
    return;
  }
  constexpr int L = C::L;
  uint32_t m[L];
  uint32_t a2[L];
  if constexpr (SQR) {
#pragma unroll
    for (int i = 0; i < L; i++) a2[i] = a[i] << 1;
  }
  fmul_cols<C, SQR, LAT, 0>(r, a, b, a2, m, 0ull, 0ull);
}

#ifndef MSM_FMUL2_SKEW
#define MSM_FMUL2_SKEW 0  // A/B: product 2's column scan trails product 1's by this many columns
#endif
// Skewed interleave: while one product is in its few-term edge columns (latency-bound
// m_K epilogues), the other is in its many-term middle columns (independent IMAD.WIDE).
template <class C, bool SQR, int K, int D>
DEVI void fmul2_skew_cols(uint32_t* r1, const uint32_t* a1, const uint32_t* b1, const uint32_t* a21, uint32_t* m1,
                          u64& cA1, u64& cM1, uint32_t* r2, const uint32_t* a2, const uint32_t* b2,
                          const uint32_t* a22, uint32_t* m2, u64& cA2, u64& cM2) {
  constexpr int NC = 2 * C::L - 1;
  if constexpr (K < NC) fmul_step<C, SQR, MSM_FMUL2_LAT != 0, K>(r1, a1, b1, a21, m1, cA1, cM1);
  if constexpr (K >= D && K - D < NC) fmul_step<C, SQR, MSM_FMUL2_LAT != 0, K - D>(r2, a2, b2, a22, m2, cA2, cM2);
  if constexpr (K + 1 < NC + D)
    fmul2_skew_cols<C, SQR, K + 1, D>(r1, a1, b1, a21, m1, cA1, cM1, r2, a2, b2, a22, m2, cA2, cM2);
}

// r1 = a1*b1, r2 = a2*b2 (SQR: r1 = a1^2, r2 = a2^2), same contract as fmul
template <class C, bool SQR = false>
DEVI void fmul2(uint32_t* r1, const uint32_t* a1, const uint32_t* b1, uint32_t* r2, const uint32_t* a2, const uint32_t* b2) {
  if constexpr (MSM_ROWS != 0 && C::L > 13) {  // each product already has L-way ILP
    fmul_rows<C>(r1, a1, b1);
    fmul_rows<C>(r2, a2, b2);
    return;
  }
  constexpr int L = C::L;
  uint32_t m1[L], m2[L], d1[L], d2[L];
  if constexpr (SQR) {
#pragma unroll
    for (int i = 0; i < L; i++) { d1[i] = a1[i] << 1; d2[i] = a2[i] << 1; }
  }
  if constexpr (MSM_FMUL2_SKEW > 0 && C::L <= 13) {
    u64 cA1 = 0, cM1 = 0, cA2 = 0, cM2 = 0;
    fmul2_skew_cols<C, SQR, 0, MSM_FMUL2_SKEW>(r1, a1, b1, d1, m1, cA1, cM1, r2, a2, b2, d2, m2, cA2, cM2);
  } else {
    fmul2_cols<C, SQR, 0>(r1, a1, b1, d1, m1, 0ull, 0ull, r2, a2, b2, d2, m2, 0ull, 0ull);
  }
}

template <class C>
DEVI void fmul(uint32_t* r, const uint32_t* a, const uint32_t* b) { fmul_impl<C, false>(r, a, b); }

// latency-mode multiplication / squaring (serial tails: window combine, finalisation)
template <class C>
DEVI void fmul_lat(uint32_t* r, const uint32_t* a, const uint32_t* b) { fmul_impl<C, false, true>(r, a, b); }
template <class C>
DEVI void fsqr_lat(uint32_t* r, const uint32_t* a) { fmul_impl<C, true, true>(r, a, a); }

// r = a^2 (same contract as fmul): L(L+1)/2 products instead of L^2
template <class C>
DEVI void fsqr(uint32_t* r, const uint32_t* a) {
#if MSM_FSQR_AS_MUL
  fmul_impl<C, false>(r, a, a);
#else
  fmul_impl<C, true>(r, a, a);
#endif
}

// r = a + b (no reduction; bound(r) = bound(a) + bound(b) <= KMAX)
template <class C>
DEVI void fadd(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  uint32_t c = 0;
#pragma unroll
  for (int i = 0; i < L - 1; i++) {
    uint32_t s = a[i] + b[i] + c;
    r[i] = s & MASK;
    c = s >> W;
  }
  r[L - 1] = a[L - 1] + b[L - 1] + c;
}

// r = a - b + K*p   (requires bound(b) <= K; bound(r) = bound(a) + K)
template <class C, int K>
DEVI void fsub(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  static_assert(K < C::KMAX, "K*p not tabulated");
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  int32_t c = 0;
#pragma unroll
  for (int i = 0; i < L - 1; i++) {
    int32_t s = (int32_t)(a[i] - b[i] + C::KP(K, i)) + c;
    r[i] = (uint32_t)s & MASK;
    c = s >> W;
  }
  r[L - 1] = (uint32_t)((int32_t)(a[L - 1] - b[L - 1] + C::KP(K, L - 1)) + c);
}

// ---- carry-deferred add / subtract (one-step carries: every limb independent, so the
// glue between the PACC's multiplication pairs is ~3 dependent ALU ops deep instead of a
// 13-step carry chain).  Outputs are "semi-normalised": limbs <= 2^W + 3 (the top limb
// unmasked), which every multiplication accepts (a column of <= MAXT products of
// (2^W + 3)^2 still fits 64 bits) and the exact fsub/fadd normalise again.  They are NOT
// valid inputs for fis_zero / fequal / fcsub (those need normalised limbs).
// r = a + b  (a, b limbs <= 2^W + 3; bound(r) = bound(a) + bound(b))
template <class C>
DEVI void fadd_fast(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  uint32_t s[L];
#pragma unroll
  for (int i = 0; i < L; i++) s[i] = a[i] + b[i];
  r[0] = s[0] & MASK;
#pragma unroll
  for (int i = 1; i < L - 1; i++) r[i] = (s[i] & MASK) + (s[i - 1] >> W);
  r[L - 1] = s[L - 1] + (s[L - 2] >> W);
}

// r = a - b + (K+1)*p  (a normalised (limbs < 2^W), b limbs <= 2^W + 3, bound(b) <= K;
// bound(r) = bound(a) + K + 1).  (K+1)*p is added in a borrow-proof limb form
// D_0 = kp_0 + 2^(W+1), D_i = kp_i + 2^(W+1) - 2, D_(L-1) = kp_(L-1) - 2 (same value), so
// every limb difference is non-negative and < 2^32; the extra p keeps the value >= p, so
// the top limb stays non-negative after the one-step carries.
template <class C, int K>
DEVI void fsub_fast(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  static_assert(K + 1 < C::KMAX, "(K+1)*p not tabulated");
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  uint32_t s[L];
  s[0] = a[0] - b[0] + (C::KP(K + 1, 0) + (2u << W));
#pragma unroll
  for (int i = 1; i < L - 1; i++) s[i] = a[i] - b[i] + (C::KP(K + 1, i) + (2u << W) - 2u);
  s[L - 1] = a[L - 1] - b[L - 1] + (C::KP(K + 1, L - 1) - 2u);
  r[0] = s[0] & MASK;
#pragma unroll
  for (int i = 1; i < L - 1; i++) r[i] = (s[i] & MASK) + (s[i - 1] >> W);
  r[L - 1] = s[L - 1] + (s[L - 2] >> W);
}

// r = K*p - a   (negation; requires bound(a) <= K)
template <class C, int K>
DEVI void fneg(uint32_t* r, const uint32_t* a) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  int32_t c = 0;
#pragma unroll
  for (int i = 0; i < L - 1; i++) {
    int32_t s = (int32_t)(C::KP(K, i) - a[i]) + c;
    r[i] = (uint32_t)s & MASK;
    c = s >> W;
  }
  r[L - 1] = (uint32_t)((int32_t)(C::KP(K, L - 1) - a[L - 1]) + c);
}

template <class C>
DEVI void fcopy(uint32_t* r, const uint32_t* a) {
#pragma unroll
  for (int i = 0; i < C::L; i++) r[i] = a[i];
}

template <class C>
DEVI void fset_one(uint32_t* r) {
#pragma unroll
  for (int i = 0; i < C::L; i++) r[i] = C::ONE(i);
}

template <class C>
DEVI void fzero(uint32_t* r) {
#pragma unroll
  for (int i = 0; i < C::L; i++) r[i] = 0;
}

// a == b as limb vectors (both normalised)
template <class C>
DEVI bool flimbs_eq(const uint32_t* a, const uint32_t* b) {
  uint32_t d = 0;
#pragma unroll
  for (int i = 0; i < C::L; i++) d |= a[i] ^ b[i];
  return d == 0;
}

// a == 0 (mod p) for a lazy value a < K*p.
// a = j*p  <=>  a[0]*p^-1 = j (mod 2^W) and the limbs equal those of j*p.  The fast
// reject costs one IMAD + one compare; the full compare runs only when j < K.
template <class C, int K>
DEVI bool fis_zero(const uint32_t* a) {
  static_assert(K <= C::KMAX, "K*p not tabulated");
  constexpr uint32_t MASK = (1u << C::W) - 1;
  uint32_t j = (a[0] * C::PINV) & MASK;
  if (j >= (uint32_t)K) return false;
  uint32_t d = 0;
#pragma unroll
  for (int i = 0; i < C::L; i++) d |= a[i] ^ C::KPc()[j * C::L + i];
  return d == 0;
}

// a == b (mod p) for lazy a, b < K*p
template <class C, int K>
DEVI bool fequal(const uint32_t* a, const uint32_t* b) {
  uint32_t t[C::L];
  fsub<C, K>(t, a, b);
  return fis_zero<C, 2 * K>(t);
}

// conditional subtraction: if a >= k*p then a -= k*p (a normalised)
template <class C, int k>
DEVI void fcsub(uint32_t* a) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
  uint32_t t[L];
  int32_t c = 0;
#pragma unroll
  for (int i = 0; i < L; i++) {
    int32_t s = (int32_t)(a[i] - C::KP(k, i)) + c;
    t[i] = (uint32_t)s & MASK;
    c = s >> W;
  }
  if (c >= 0) {
#pragma unroll
    for (int i = 0; i < L; i++) a[i] = t[i];
  }
}

// full reduction to the canonical representative in [0, p), for a < 16p
template <class C>
DEVI void freduce(uint32_t* a) {
  fcsub<C, 8>(a);
  fcsub<C, 4>(a);
  fcsub<C, 2>(a);
  fcsub<C, 1>(a);
}

// radix-2^W limbs <-> 32-bit words (canonical values)
template <class C>
DEVI void from_words32(uint32_t* r, const uint32_t* w) {
  constexpr int L = C::L, W = C::W;
  constexpr uint32_t MASK = (1u << W) - 1;
#pragma unroll
  for (int i = 0; i < L; i++) {
    const int bit = i * W, wi = bit >> 5, sh = bit & 31;
    uint32_t lo = wi < C::L32 ? w[wi] : 0u;
    uint32_t hi = (wi + 1) < C::L32 ? w[wi + 1] : 0u;
    uint32_t v = sh ? ((lo >> sh) | (hi << (32 - sh))) : lo;
    r[i] = v & MASK;
  }
}

template <class C>
DEVI void to_words32(uint32_t* w, const uint32_t* a) {
  constexpr int L = C::L, W = C::W;
#pragma unroll
  for (int j = 0; j < C::L32; j++) {
    uint32_t v = 0;
#pragma unroll
    for (int i = 0; i < L; i++) {
      const int lo = i * W;  // limb i covers bits [lo, lo+W)
      if (lo + W <= 32 * j || lo >= 32 * j + 32) continue;
      const int sh = lo - 32 * j;
      v |= sh >= 0 ? (a[i] << sh) : (a[i] >> (-sh));
    }
    w[j] = v;
  }
}

// Montgomery form: x -> x*R mod p  (x canonical), and back (result canonical)
template <class C>
DEVI void fto_mont(uint32_t* r, const uint32_t* x) {
  uint32_t r2[C::L];
#pragma unroll
  for (int i = 0; i < C::L; i++) r2[i] = C::R2(i);
  fmul<C>(r, x, r2);
}

template <class C>
DEVI void ffrom_mont(uint32_t* r, const uint32_t* a) {
  uint32_t one[C::L];
  one[0] = 1;
#pragma unroll
  for (int i = 1; i < C::L; i++) one[i] = 0;
  fmul<C>(r, a, one);
  freduce<C>(r);
}

template <class C>
__device__ __noinline__ void fmul_ni(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  uint32_t x[C::L], y[C::L], z[C::L];
  fcopy<C>(x, a);
  fcopy<C>(y, b);
  fmul<C>(z, x, y);
  fcopy<C>(r, z);
}

// Multiplication as used by the EC layer: always inlined.  (An out-of-line copy for
// MNT4-753 compiled faster, but sm_100a keeps the stack pointer in a uniform register, so
// a warp whose lanes diverge between a path with a call and one touching the stack
// corrupts local memory — compute-sanitizer caught it.  Rule in this code base: calls to
// __noinline__ functions only from warp-uniform control flow.)
template <class C, bool LAT = false>
DEVI void fmul_e(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  if constexpr (LAT) fmul_lat<C>(r, a, b);
  else fmul<C>(r, a, b);
}
template <class C, bool LAT = false>
DEVI void fsqr_e(uint32_t* r, const uint32_t* a) {
  if constexpr (LAT) fsqr_lat<C>(r, a);
  else fsqr<C>(r, a);
}

// r = a^(p-2) = a^-1 (Montgomery form in and out; a != 0 mod p), Fermat (PAPER.md silent;
// used only for the final affine normalisation)
template <class C>
__device__ __noinline__ void finv(uint32_t* r, const uint32_t* a) {
  uint32_t acc[C::L];
  fset_one<C>(acc);
  for (int wi = C::L32 - 1; wi >= 0; wi--) {
    const uint32_t e = C::PM2c()[wi];
    for (int b = 31; b >= 0; b--) {
      fsqr_lat<C>(acc, acc);
      if ((e >> b) & 1u) fmul_lat<C>(acc, acc, a);
    }
  }
  fcopy<C>(r, acc);
}

// r = a^-1 (Montgomery form in and out; a != 0 mod p) by binary GCD on canonical 32-bit
// words (PAPER.md is silent on inversion; R19), for the single-thread final
// normalisation (a7), where Fermat's ~|p| serial latency-mode products dominate (0.75 ms
// for BLS12-381).  Round 2: the batched form of Pornin ("Optimized binary GCD for modular
// inversion", 2020): the binary-GCD step (a odd: if a < b swap (a,u),(b,v); a -= b,
// u -= v; then a /= 2, u /= 2 mod p) runs 30 times on 62-bit approximations of a and b
// (their low 30 bits, exact, and their top 32 bits), recording the steps as a 2x2 matrix
// of signed factors (|f| + |g| <= 2^30); then (a, b) <- (f0 a + g0 b, f1 a + g1 b) / 2^30
// (negated if an approximate comparison made one negative) and (u, v) likewise mod p.
// ceil((2|p| - 1) / 30) batches suffice; invariants a == u*y, b == v*y (mod p), and b = 1,
// v = y^-1 at the end.  Variable time: the MSM result is not secret.  Input words
// y = canonical(aR) = aR mod p; output (aR)^-1, then two Montgomery products by R^2 give
// a^-1 R.
template <int N>
DEVI uint32_t inv_words_bits(const uint32_t* w, int pos) {  // bits [pos, pos + 32) of w
  const int q = pos >> 5, sh = pos & 31;
  const uint32_t lo = q < N ? w[q] : 0u, hi = q + 1 < N ? w[q + 1] : 0u;
  return sh ? (lo >> sh) | (hi << (32 - sh)) : lo;
}
// r = (f x + g y) / 2^30 (exact), |r| returned with neg = sign; N words
template <int N>
DEVI void inv_lin_shift(uint32_t* r, const uint32_t* x, const uint32_t* y, int64_t f, int64_t g, bool& neg) {
  uint32_t t[N + 1];
  int64_t c = 0;
#pragma unroll
  for (int i = 0; i < N; i++) {
    const int64_t s = f * (int64_t)x[i] + g * (int64_t)y[i] + c;
    t[i] = (uint32_t)s;
    c = s >> 32;
  }
  t[N] = (uint32_t)c;
  neg = c < 0;
  if (neg) {  // two's complement over N + 1 words
    uint32_t cy = 1;
#pragma unroll
    for (int i = 0; i <= N; i++) {
      const uint64_t s2 = (uint64_t)(~t[i]) + cy;
      t[i] = (uint32_t)s2;
      cy = (uint32_t)(s2 >> 32);
    }
  }
#pragma unroll
  for (int i = 0; i < N; i++) r[i] = (t[i] >> 30) | (t[i + 1] << 2);
}
// r = (f x + g y) / 2^30 mod p, x, y in [0, p), r in [0, p); minv = -p^-1 mod 2^30
template <int N>
DEVI void inv_lin_mod(uint32_t* r, const uint32_t* x, const uint32_t* y, int64_t f, int64_t g,
                      const uint32_t* p, uint32_t minv) {
  uint32_t t[N + 1];
  int64_t c = 0;
#pragma unroll
  for (int i = 0; i < N; i++) {
    const int64_t s = f * (int64_t)x[i] + g * (int64_t)y[i] + c;
    t[i] = (uint32_t)s;
    c = s >> 32;
  }
  t[N] = (uint32_t)c;
  const uint32_t q = (t[0] * minv) & 0x3fffffffu;  // t + q p == 0 mod 2^30
  uint64_t cy = 0;
#pragma unroll
  for (int i = 0; i < N; i++) {
    cy += (uint64_t)q * p[i] + t[i];
    t[i] = (uint32_t)cy;
    cy >>= 32;
  }
  t[N] += (uint32_t)cy;  // two's complement top word; the true value is in (-2^30 p, 2^31 p)
  uint32_t w[N + 1];
#pragma unroll
  for (int i = 0; i < N; i++) w[i] = (t[i] >> 30) | (t[i + 1] << 2);
  w[N] = (uint32_t)((int32_t)t[N] >> 30);  // r in (-p, 2p)
  if ((int32_t)w[N] < 0) {  // += p
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < N; i++) { s += (uint64_t)w[i] + p[i]; w[i] = (uint32_t)s; s >>= 32; }
    w[N] += (uint32_t)s;
  } else {  // -= p if >= p
    bool ge = w[N] != 0;
    if (!ge) {
      bool done = false;
      ge = true;
#pragma unroll
      for (int i = N - 1; i >= 0; i--)
        if (!done && w[i] != p[i]) { ge = w[i] > p[i]; done = true; }
    }
    if (ge) {
      int64_t s = 0;
#pragma unroll
      for (int i = 0; i < N; i++) { s = (int64_t)w[i] - p[i] + (s >> 32); w[i] = (uint32_t)s; }
    }
  }
#pragma unroll
  for (int i = 0; i < N; i++) r[i] = w[i];
}

template <class C>
__device__ __noinline__ void finv_bgcd(uint32_t* r, const uint32_t* a) {
  constexpr int N = C::L32;
  uint32_t t[C::L], ua[N], ub[N], u[N], v[N], p[N];
  fcopy<C>(t, a);
  freduce<C>(t);
  to_words32<C>(ua, t);
  uint32_t nz = 0;
#pragma unroll
  for (int i = 0; i < N; i++) { p[i] = C::P32c()[i]; ub[i] = p[i]; u[i] = i == 0; v[i] = 0; nz |= ua[i]; }
  if (nz == 0) {  // a == 0 mod p has no inverse: return 0 rather than loop
    fzero<C>(r);
    return;
  }
  uint32_t pinv = p[0];  // p^-1 mod 2^32 by Newton (p odd: correct to 3 bits, doubling)
#pragma unroll
  for (int k = 0; k < 4; k++) pinv *= 2u - p[0] * pinv;
  const uint32_t minv = (0u - pinv) & 0x3fffffffu;
  const int pbits = 32 * N - __clz(p[N - 1]);
  const int batches = (2 * pbits - 1 + 29) / 30;
  for (int it = 0; it < batches; it++) {
    int top = N - 1;
    while (top > 0 && (ua[top] | ub[top]) == 0) top--;
    const int len = 32 * top + 32 - __clz(ua[top] | ub[top]);
    const int nb = len > 62 ? len : 62;
    uint64_t A = (ua[0] & 0x3fffffffu) | ((uint64_t)inv_words_bits<N>(ua, nb - 32) << 30);
    uint64_t B = (ub[0] & 0x3fffffffu) | ((uint64_t)inv_words_bits<N>(ub, nb - 32) << 30);
    int64_t f0 = 1, g0 = 0, f1 = 0, g1 = 1;
    for (int j = 0; j < 30; j++) {
      if (A & 1u) {
        if (A < B) {
          const uint64_t T = A; A = B; B = T;
          int64_t q = f0; f0 = f1; f1 = q;
          q = g0; g0 = g1; g1 = q;
        }
        A -= B;
        f0 -= f1;
        g0 -= g1;
      }
      A >>= 1;
      f1 *= 2;
      g1 *= 2;
    }
    uint32_t na[N], nb2[N];
    bool neg_a, neg_b;
    inv_lin_shift<N>(na, ua, ub, f0, g0, neg_a);
    inv_lin_shift<N>(nb2, ua, ub, f1, g1, neg_b);
    if (neg_a) { f0 = -f0; g0 = -g0; }
    if (neg_b) { f1 = -f1; g1 = -g1; }
    uint32_t nu[N], nv[N];
    inv_lin_mod<N>(nu, u, v, f0, g0, p, minv);
    inv_lin_mod<N>(nv, u, v, f1, g1, p, minv);
#pragma unroll
    for (int i = 0; i < N; i++) { ua[i] = na[i]; ub[i] = nb2[i]; u[i] = nu[i]; v[i] = nv[i]; }
  }
  uint32_t w[C::L], r2[C::L];
  from_words32<C>(w, v);  // b == 1: v = y^-1
#pragma unroll
  for (int i = 0; i < C::L; i++) r2[i] = C::R2(i);
  fmul_lat<C>(w, w, r2);  // a^-1 R^-1 -> a^-1
  fmul_lat<C>(r, w, r2);  // a^-1 -> a^-1 R
}
