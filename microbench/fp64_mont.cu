// B200 FP64-pipe Montgomery multiplication A/B (BLS12-381), for the a1 field layer.
//
// B200 (sm_100a) still has a full-rate FP64 pipe — 64 DFMA/clk/SM measured by
// microbench/dfma_probe.cu — that the IMAD-only field layer leaves idle.  A 49x49-bit
// limb product fits a DFMA exactly when split at 2^49 with round-toward-zero:
//     hb = fma_rz(a, b, 2^101)   = 2^101 + floor(ab / 2^49) * 2^49    (ulp of [2^101,2^102) is 2^49)
//     nh = 2^101 - hb            = -floor(ab / 2^49) * 2^49           (exact)
//     lo = fma(a, b, nh)         = ab mod 2^49                        (exact)
// so a column of products accumulates exactly in doubles (all sums < 2^53).
//
// `fpm`: word-serial Montgomery (Alg. 2, FIPS column order) on L = 8 limbs of
// W = 49 bits, R_fp = 2^392.  The operand a enters scaled by 4 (free in the radix
// conversion), so fpm(4a, b) = a*b*2^-390 mod p: the SAME Montgomery domain (R = 2^390)
// and the same lazy bound (inputs < 10p -> output < 2p) as the library's radix-2^30 IMAD
// path (`fips`, csrc/field.cuh).  Values stay in the library's radix-2^30 u32 form; the
// FP path converts at its inputs and output.
//
// Variants (each thread: dependent chains x <- x*y, ITERS iterations):
//   fips     1 chain, library IMAD path
//   fips2    2 chains, library fmul2 (column-interleaved pair)
//   fp       1 chain, FP64 path (with radix conversions)
//   hyb2     2 chains: one IMAD (fmul) + one FP64 — both pipes at once
//   hyb3     3 chains: fmul2 (IMAD pair) + one FP64
// Every result is checked bit-for-bit (after full reduction) against a fips-only chain.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o microbench/fp64_mont microbench/fp64_mont.cu
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_ji0x024_b200/csrc/field.cuh"

using C = BLS12_381_params;
constexpr int L = 13, W = 30;
constexpr int FL = 8, FW = 49;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

DEVI double fpP(int i) {
  constexpr double t[8] = {281474976688811.0, 378962144386303.0, 67658748461055.0, 541948005064406.0,
                           409809928605995.0, 477301282618147.0, 562513631276702.0, 223374201970.0};
  return t[i];
}
constexpr double FP_N0 = 562937068322813.0;  // -p^-1 mod 2^49
constexpr double C101 = 0x1p101, C52 = 0x1p52;

// lo_acc += ab mod 2^49 ; hi_acc += floor(ab / 2^49)     (a, b < 2^50, ab < 2^99)
DEVI void prod_acc(double a, double b, double& lo_acc, double& hi_acc) {
  const double hb = __fma_rz(a, b, C101);
  const double nh = __dsub_rn(C101, hb);
  const double lo = __fma_rn(a, b, nh);
  lo_acc = __dadd_rn(lo_acc, lo);
  hi_acc = __fma_rn(nh, -0x1p-49, hi_acc);
}
// x (integer, 0 <= x < 2^53) = q*2^49 + r
DEVI void split49(double x, double& q, double& r) {
  const double qb = __fma_rz(x, 0x1p-49, C52);
  q = __dsub_rn(qb, C52);
  r = __fma_rn(q, -0x1p49, x);
}
// t * N0 mod 2^49
DEVI double mulmod49(double t) {
  const double hb = __fma_rz(t, FP_N0, C101);
  const double nh = __dsub_rn(C101, hb);
  return __fma_rn(t, FP_N0, nh);
}

// r = a*b*2^-392 mod p (lazy), a, b: 8 limbs < 2^49 (SQR: b ignored, a*a)
template <bool SQR>
DEVI void fpm(double* r, const double* a, const double* b) {
  double m[FL];
  double a2[FL];
  if constexpr (SQR) {
#pragma unroll
    for (int i = 0; i < FL; i++) a2[i] = __dadd_rn(a[i], a[i]);
  }
  double ab_cur = 0, ab_nxt = 0, mp_cur = 0, mp_nxt = 0, carry = 0;
#pragma unroll
  for (int k = 0; k < 2 * FL - 1; k++) {
    ab_cur = ab_nxt; ab_nxt = 0;
    mp_cur = mp_nxt; mp_nxt = 0;
    const int lo = k - FL + 1 > 0 ? k - FL + 1 : 0;
    const int hi = k < FL - 1 ? k : FL - 1;
    if constexpr (SQR) {
#pragma unroll
      for (int i = lo; i <= hi; i++) {
        const int j = k - i;
        if (i < j) prod_acc(a2[i], a[j], ab_cur, ab_nxt);
        else if (i == j) prod_acc(a[i], a[i], ab_cur, ab_nxt);
      }
    } else {
#pragma unroll
      for (int i = lo; i <= hi; i++) prod_acc(a[i], b[k - i], ab_cur, ab_nxt);
    }
    const int mhi = (k - 1) < (FL - 1) ? (k - 1) : (FL - 1);
#pragma unroll
    for (int i = lo; i <= mhi; i++) prod_acc(m[i], fpP(k - i), mp_cur, mp_nxt);
    double q1, r1, q2, r2, q3, t;
    split49(ab_cur, q1, r1);
    split49(mp_cur, q2, r2);
    const double u = __dadd_rn(__dadd_rn(r1, r2), carry);
    split49(u, q3, t);
    carry = __dadd_rn(__dadd_rn(q1, q2), q3);
    if (k < FL) {
      m[k] = mulmod49(t);
      const double hb = __fma_rz(m[k], fpP(0), C101);
      const double nh = __dsub_rn(C101, hb);
      const double l0 = __fma_rn(m[k], fpP(0), nh);      // t + l0 in {0, 2^49}
      carry = __fma_rn(__dadd_rn(t, l0), 0x1p-49, carry);
      mp_nxt = __fma_rn(nh, -0x1p-49, mp_nxt);
    } else {
      r[k - FL] = t;
    }
  }
  r[FL - 1] = __dadd_rn(__dadd_rn(ab_nxt, mp_nxt), carry);
}

// radix-2^30 u32 limbs (value < 2^392 / SCALE) -> 8 doubles of 49 bits, value * 2^SH
template <int SH>
DEVI void to_fp(double* d, const uint32_t* x) {
#pragma unroll
  for (int j = 0; j < FL; j++) {
    const int s = FW * j - SH;  // first bit of x in this limb (may be negative for j = 0)
    uint64_t v;
    if (s < 0) {
      v = ((uint64_t)x[0] | ((uint64_t)x[1] << 30)) << (-s);
    } else {
      const int i0 = s / 30, sh = s % 30;
      uint64_t w = (uint64_t)x[i0];
      if (i0 + 1 < L) w |= (uint64_t)x[i0 + 1] << 30;
      w >>= sh;
      if (i0 + 2 < L && 60 - sh < 49) w |= (uint64_t)x[i0 + 2] << (60 - sh);
      v = w;
    }
    v &= (1ull << FW) - 1;
    d[j] = __dsub_rn(__longlong_as_double((long long)(v | 0x4330000000000000ull)), C52);
  }
}
// 8 doubles (normalised limbs < 2^49, value < 2^390) -> radix-2^30 u32 limbs
DEVI void from_fp(uint32_t* x, const double* d) {
  uint64_t v[FL];
#pragma unroll
  for (int j = 0; j < FL; j++) v[j] = (uint64_t)__double_as_longlong(__dadd_rn(d[j], C52)) & ((1ull << 52) - 1);
#pragma unroll
  for (int i = 0; i < L; i++) {
    const int s = 30 * i, j0 = s / FW, sh = s % FW;
    uint64_t w = v[j0] >> sh;
    if (j0 + 1 < FL && FW - sh < 30) w |= v[j0 + 1] << (FW - sh);
    x[i] = (uint32_t)w & ((1u << 30) - 1);
  }
}

// a*b*2^-390 in the library's domain, through the FP64 pipe
DEVI void fmul_fp(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  double da[FL], db[FL], dr[FL];
  to_fp<2>(da, a);
  to_fp<0>(db, b);
  fpm<false>(dr, da, db);
  from_fp(r, dr);
}

constexpr int ITERS = 256;
enum { V_FIPS = 0, V_FIPS2, V_FP, V_HYB2, V_HYB3, V_COUNT };
const char* VNAME[] = {"fips", "fips2", "fp", "hyb2", "hyb3"};
constexpr int VMULTS[] = {1, 2, 1, 2, 3};

template <int V>
__global__ void __launch_bounds__(128, 1) k_bench(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, int n) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n) return;
  uint32_t x1[L], x2[L], x3[L], y[L];
#pragma unroll
  for (int i = 0; i < L; i++) { x1[i] = in[t * 2 * L + i]; y[i] = in[t * 2 * L + L + i]; x2[i] = x1[i]; x3[i] = x1[i]; }
#pragma unroll 1
  for (int it = 0; it < ITERS; it++) {
    if constexpr (V == V_FIPS) fmul<C>(x1, x1, y);
    if constexpr (V == V_FIPS2) fmul2<C>(x1, x1, y, x2, x2, y);
    if constexpr (V == V_FP) fmul_fp(x1, x1, y);
    if constexpr (V == V_HYB2) { fmul<C>(x1, x1, y); fmul_fp(x2, x2, y); }
    if constexpr (V == V_HYB3) { fmul2<C>(x1, x1, y, x2, x2, y); fmul_fp(x3, x3, y); }
  }
  constexpr int NM = V == V_HYB3 ? 3 : (V == V_FIPS2 || V == V_HYB2) ? 2 : 1;
  freduce<C>(x1); freduce<C>(x2); freduce<C>(x3);
#pragma unroll
  for (int i = 0; i < L; i++) {
    out[(size_t)t * 3 * L + i] = x1[i];
    out[(size_t)t * 3 * L + L + i] = NM > 1 ? x2[i] : x1[i];
    out[(size_t)t * 3 * L + 2 * L + i] = NM > 2 ? x3[i] : x1[i];
  }
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int n = sms * 1024;  // 8 warps per SM x 4... enough residency for every variant
  uint32_t* h = new uint32_t[(size_t)n * 2 * L];
  uint64_t s = 0x9e3779b97f4a7c15ull;
  for (size_t i = 0; i < (size_t)n * 2 * L; i++) {
    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
    h[i] = (uint32_t)s & ((1u << 30) - 1);
  }
  for (int t = 0; t < n; t++) {  // values < 2^370 < p (canonical, < 2p lazily)
    h[(size_t)t * 2 * L + 12] = 0; h[(size_t)t * 2 * L + 2 * L - 1] = 0;
  }
  uint32_t *din, *dout;
  CK(cudaMalloc(&din, (size_t)n * 2 * L * 4));
  CK(cudaMalloc(&dout, (size_t)n * 3 * L * 4));
  CK(cudaMemcpy(din, h, (size_t)n * 2 * L * 4, cudaMemcpyHostToDevice));
  uint32_t* ref = new uint32_t[(size_t)n * 3 * L];
  uint32_t* got = new uint32_t[(size_t)n * 3 * L];
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto launch = [&](int v) {
    const int blocks = (n + 127) / 128;
    switch (v) {
      case V_FIPS: k_bench<V_FIPS><<<blocks, 128>>>(din, dout, n); break;
      case V_FIPS2: k_bench<V_FIPS2><<<blocks, 128>>>(din, dout, n); break;
      case V_FP: k_bench<V_FP><<<blocks, 128>>>(din, dout, n); break;
      case V_HYB2: k_bench<V_HYB2><<<blocks, 128>>>(din, dout, n); break;
      default: k_bench<V_HYB3><<<blocks, 128>>>(din, dout, n); break;
    }
  };
  launch(V_FIPS);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(ref, dout, (size_t)n * 3 * L * 4, cudaMemcpyDeviceToHost));
  for (int v = 0; v < V_COUNT; v++) {
    launch(v);
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    const int reps = 5;
    for (int r = 0; r < reps; r++) launch(v);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= reps;
    CK(cudaMemcpy(got, dout, (size_t)n * 3 * L * 4, cudaMemcpyDeviceToHost));
    size_t bad = 0;
    for (int t = 0; t < n; t++)
      for (int c = 0; c < VMULTS[v]; c++)
        for (int i = 0; i < L; i++) bad += got[(size_t)t * 3 * L + c * L + i] != ref[(size_t)t * 3 * L + i];
    const double mults = (double)n * ITERS * VMULTS[v];
    printf("{\"variant\":\"%s\",\"ms\":%.3f,\"gmults_per_s\":%.2f,\"mismatched_words\":%zu,\"threads\":%d}\n", VNAME[v], ms,
           mults / (ms * 1e-3) / 1e9, bad, n);
  }
  return 0;
}
