// MSM kernels.  All templated on the curve parameter struct C.
//
// Data layout in HBM (per device shard):
//   pts      [n][PW] u32      affine (x, y), Montgomery form, radix-2^W limbs, x then y,
//                             padded to PW = round_up(2L, 4) words (16-B aligned records)
//   scal     [n][S] u32       scalars k_i, canonical little-endian 32-bit words
//   goff     [F+1] u32        F = nwin * NB flat buckets f = j*NB + b (NB = 2^(c-1) + 1);
//                             exclusive prefix sum of the bucket counts over ALL windows
//   cursor   [F] u32          scatter cursors (goff copy, consumed by atomics)
//   sorted   [M] u32          point index | sign << 31, grouped by flat bucket
//   buckets  [F] Xyzz         bucket sums B_{j,b} (valid where the bucket is non-empty)
#pragma once
#include <cooperative_groups.h>

#include "ec.cuh"

namespace msmk {

constexpr uint32_t SIGN_BIT = 0x80000000u;

#ifndef MSM_ACC_MINB
#define MSM_ACC_MINB 1  // min resident 128-thread blocks per SM for k_accumulate (register cap)
#endif
#ifndef MSM_SUM_WARP
#define MSM_SUM_WARP 1  // k_sum_groups as a warp shuffle tree per group (0: one thread per group)
#endif
#ifndef MSM_SEG_MINB
#define MSM_SEG_MINB 1
#endif
#ifndef MSM_SEG_MINB_BIG
#define MSM_SEG_MINB_BIG 1  // A/B: min resident blocks of k_bucket_segments for MNT4-753 (register cap)
#endif

template <class C>
struct Layout {
  static constexpr int PW = ((2 * C::L + 3) / 4) * 4;  // words per stored affine point
  static constexpr int XW = 4 * C::L;                   // words per XYZZ point
};

// ---------------------------------------------------------------------------------------
// XYZZ load/store (plain word arrays; XYZZ records are 4L words)
template <class C>
DEVI void load_xyzz(Xyzz<C>& A, const uint32_t* __restrict__ p) {
#pragma unroll
  for (int i = 0; i < C::L; i++) {
    A.X[i] = p[i];
    A.Y[i] = p[C::L + i];
    A.ZZ[i] = p[2 * C::L + i];
    A.ZZZ[i] = p[3 * C::L + i];
  }
}
template <class C>
DEVI void store_xyzz(uint32_t* __restrict__ p, const Xyzz<C>& A) {
#pragma unroll
  for (int i = 0; i < C::L; i++) {
    p[i] = A.X[i];
    p[C::L + i] = A.Y[i];
    p[2 * C::L + i] = A.ZZ[i];
    p[3 * C::L + i] = A.ZZZ[i];
  }
}

// gather one stored affine point with 16-B vector loads
template <class C>
DEVI void load_point(uint32_t* x, uint32_t* y, const uint32_t* __restrict__ pts, uint32_t idx) {
  constexpr int PW = Layout<C>::PW;
  uint32_t w[PW];
  const uint4* src = reinterpret_cast<const uint4*>(pts + (size_t)idx * PW);
#pragma unroll
  for (int q = 0; q < PW / 4; q++) {
    uint4 v = __ldg(src + q);
    w[4 * q] = v.x; w[4 * q + 1] = v.y; w[4 * q + 2] = v.z; w[4 * q + 3] = v.w;
  }
#pragma unroll
  for (int i = 0; i < C::L; i++) { x[i] = w[i]; y[i] = w[C::L + i]; }
}

// ---------------------------------------------------------------------------------------
// a0: canonical affine words -> Montgomery radix-2^W, on-curve check (context creation)
//     in: [n][2*L32] words, (0,0) = O.   err |= 1 for an off-curve point, 2 for x/y >= p.
template <class C>
__global__ void k_points_to_mont(uint32_t* __restrict__ pts, const uint32_t* __restrict__ in,
                                 size_t n, uint32_t* err) {
  constexpr int L = C::L, PW = Layout<C>::PW;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint32_t xw[C::L32], yw[C::L32];
#pragma unroll
  for (int k = 0; k < C::L32; k++) { xw[k] = in[i * 2 * C::L32 + k]; yw[k] = in[i * 2 * C::L32 + C::L32 + k]; }
  uint32_t nz = 0;
#pragma unroll
  for (int k = 0; k < C::L32; k++) nz |= xw[k] | yw[k];
  uint32_t x[L], y[L], out[PW];
#pragma unroll
  for (int k = 0; k < PW; k++) out[k] = 0;
  if (nz) {
    // range check x, y < p (canonical input)
    bool ltx = false, lty = false, decx = false, decy = false;
#pragma unroll
    for (int k = C::L32 - 1; k >= 0; k--) {
      const uint32_t pk = C::P32c()[k];
      if (!decx && xw[k] != pk) { ltx = xw[k] < pk; decx = true; }
      if (!decy && yw[k] != pk) { lty = yw[k] < pk; decy = true; }
    }
    if (!ltx || !lty) atomicOr(err, 2u);
    // y = 0 would be read as O by the accumulation: such a point has order 2 (on
    // BLS12-377, (p-1, 0) lies on the curve) and is outside the prime-order subgroup
    uint32_t ynz = 0;
#pragma unroll
    for (int k = 0; k < C::L32; k++) ynz |= yw[k];
    if (!ynz) atomicOr(err, 1u);
    from_words32<C>(x, xw);
    from_words32<C>(y, yw);
    fto_mont<C>(x, x);
    fto_mont<C>(y, y);
    // y^2 == x^3 + a x + b
    uint32_t l[L], r[L], t[L], b[L];
    fsqr_e<C>(l, y);
    fsqr_e<C>(t, x);
    fmul_e<C>(r, t, x);
    if constexpr (!C::A_ZERO) {
      uint32_t a[L];
#pragma unroll
      for (int k = 0; k < L; k++) a[k] = C::A_M(k);
      fmul_e<C>(t, a, x);
      fadd<C>(r, r, t);
    }
#pragma unroll
    for (int k = 0; k < L; k++) b[k] = C::B_M(k);
    fadd<C>(r, r, b);
    if (!fequal<C, 6>(l, r)) atomicOr(err, 1u);
#pragma unroll
    for (int k = 0; k < L; k++) { out[k] = x[k]; out[L + k] = y[k]; }
  }
  uint4* dst = reinterpret_cast<uint4*>(pts + i * PW);
#pragma unroll
  for (int q = 0; q < PW / 4; q++) dst[q] = make_uint4(out[4 * q], out[4 * q + 1], out[4 * q + 2], out[4 * q + 3]);
}

// ---------------------------------------------------------------------------------------
// f3: precomputed window table ("in window j, the point P_i is replaced with
// 2^{js} P_i"; :161 "bucket-reduce and window-reduce are commutative with precomputation").
// Row j of the table is 2^c times row j-1, built at context creation in two passes per
// chunk of points:
//   k_pre_dbl   tmp[i] = 2^c * src[i]         (c XYZZ doublings, dbl-2008-s-1)
//   k_pre_norm  dst[i] = affine(tmp[i])       (batch inversion: one Fermat inverse per
//                                               PRE_K points, Montgomery's trick)
// O (stored as x = y = 0) stays O.  Output values are < 2p (products), as PACC requires.
constexpr int PRE_K = 32;

template <class C>
__global__ void __launch_bounds__(128) k_pre_dbl(const uint32_t* __restrict__ src, size_t cnt, int c,
                                                 uint32_t* __restrict__ tmp) {
  constexpr int XW = Layout<C>::XW;
  const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= cnt) return;
  uint32_t x[C::L], y[C::L];
  load_point<C>(x, y, src, (uint32_t)i);
  Xyzz<C> A;
  if (fis_zero<C, 2>(y)) xyzz_set_zero<C>(A);
  else xyzz_from_affine<C>(A, x, y);
  for (int s = 0; s < c; s++) {
    Xyzz<C> T = A;
    xyzz_dbl<C>(A, T);
  }
  store_xyzz<C>(tmp + i * XW, A);
}

// thread t normalises points [t*PRE_K, (t+1)*PRE_K) of tmp into dst; the prefix products
// are parked in dst's records (PW >= L words) between the two sweeps.  Trip counts are
// warp-uniform (tail lanes use d = 1) so the out-of-line finv is called convergently.
template <class C>
__global__ void __launch_bounds__(128) k_pre_norm(const uint32_t* __restrict__ tmp, size_t cnt,
                                                  uint32_t* __restrict__ dst) {
  constexpr int L = C::L, XW = Layout<C>::XW, PW = Layout<C>::PW;
  const size_t t = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t i0 = t * PRE_K;
  uint32_t acc[L], d[L], zz[L], zzz[L];
  fset_one<C>(acc);
  for (int k = 0; k < PRE_K; k++) {
    const size_t i = i0 + k;
    if (i < cnt) {
      const uint32_t* q = tmp + i * XW;
#pragma unroll
      for (int w = 0; w < L; w++) { zz[w] = q[2 * L + w]; zzz[w] = q[3 * L + w]; }
      fmul<C>(d, zz, zzz);
      if (fis_zero<C, 2>(d)) fset_one<C>(d);
      fmul<C>(acc, acc, d);
#pragma unroll
      for (int w = 0; w < L; w++) dst[i * PW + w] = acc[w];
    }
  }
  uint32_t inv[L];
  finv<C>(inv, acc);  // (prod d)^-1
  for (int k = PRE_K - 1; k >= 0; k--) {
    const size_t i = i0 + k;
    if (i < cnt) {
      const uint32_t* q = tmp + i * XW;
      uint32_t X[L], Y[L], prev[L], ik[L], out[PW];
#pragma unroll
      for (int w = 0; w < L; w++) { X[w] = q[w]; Y[w] = q[L + w]; zz[w] = q[2 * L + w]; zzz[w] = q[3 * L + w]; }
      if (k > 0) {
#pragma unroll
        for (int w = 0; w < L; w++) prev[w] = dst[(i - 1) * PW + w];
      } else {
        fset_one<C>(prev);
      }
      fmul<C>(ik, inv, prev);  // 1 / (ZZ * ZZZ)
      fmul<C>(d, zz, zzz);
      const bool inf = fis_zero<C, 2>(d);
      if (!inf) fmul<C>(inv, inv, d);
#pragma unroll
      for (int w = 0; w < PW; w++) out[w] = 0;
      if (!inf) {
        uint32_t s[L];
        fmul<C>(s, zzz, ik);     // 1/ZZ
        fmul<C>(out, X, s);      // x = X / ZZ
        fmul<C>(s, zz, ik);      // 1/ZZZ
        fmul<C>(out + L, Y, s);  // y = Y / ZZZ
      }
      uint4* o4 = reinterpret_cast<uint4*>(dst + i * PW);
#pragma unroll
      for (int w = 0; w < PW / 4; w++) o4[w] = make_uint4(out[4 * w], out[4 * w + 1], out[4 * w + 2], out[4 * w + 3]);
    }
  }
}

// ---------------------------------------------------------------------------------------
// a2: signed c-bit digits (R6):  nwin = floor(λ/c) + 1;  d_j = chunk_j + carry;
//     for j < nwin-1: d_j > 2^(c-1) -> d_j -= 2^c, carry = 1.  Top digit never negated.
template <class C>
struct ScalarReg {
  uint32_t w[C::S];
};

template <class C>
DEVI void load_scalar(ScalarReg<C>& k, const uint32_t* __restrict__ scal, size_t i) {
  if constexpr (C::S % 4 == 0) {
    const uint4* src = reinterpret_cast<const uint4*>(scal + i * C::S);
#pragma unroll
    for (int q = 0; q < C::S / 4; q++) {
      uint4 v = __ldg(src + q);
      k.w[4 * q] = v.x; k.w[4 * q + 1] = v.y; k.w[4 * q + 2] = v.z; k.w[4 * q + 3] = v.w;
    }
  } else {
#pragma unroll
    for (int q = 0; q < C::S; q++) k.w[q] = scal[i * C::S + q];
  }
}

// k < r ?
template <class C>
DEVI bool scalar_in_range(const ScalarReg<C>& k) {
  bool lt = false, dec = false;
#pragma unroll
  for (int q = C::S - 1; q >= 0; q--) {
    const uint32_t rq = C::R32c()[q];
    if (!dec && k.w[q] != rq) { lt = k.w[q] < rq; dec = true; }
  }
  return lt;
}

// Walks the windows of one scalar, calling f(j, bucket, negative) for non-zero digits.
// cp = c | (G - 1) << 8 | g << 16 packs the f1 bucket split ("splits the
// buckets into GPUs-per-window parts"): with G > 1 only digits |d| = G*q + g are emitted,
// as local bucket q (weight G*q + g in the bucket reduce).  G = 1: every digit, bucket |d|.
template <class C, class F>
DEVI void for_each_digit(const ScalarReg<C>& k, int cp, int nwin, F&& f) {
  const int c = cp & 0xff;
  const uint32_t G = ((uint32_t)(cp >> 8) & 0xffu) + 1u, g = (uint32_t)(cp >> 16) & 0xffu;
  const uint32_t half = 1u << (c - 1), cmask = (1u << c) - 1u;
  // the scalar is consumed by funnel shifts (S SHF per window; c <= 24 < 32), instead of
  // selecting the window's words with runtime indices (~4S ALU ops per window)
  uint32_t w[C::S];
#pragma unroll
  for (int q = 0; q < C::S; q++) w[q] = k.w[q];
  uint32_t carry = 0;
  for (int j = 0; j < nwin; j++) {
    uint32_t d = (w[0] & cmask) + carry;
#pragma unroll
    for (int q = 0; q < C::S - 1; q++) w[q] = __funnelshift_r(w[q], w[q + 1], c);
    w[C::S - 1] >>= c;
    bool neg = false;
    if (j < nwin - 1 && d > half) {
      d = (1u << c) - d;
      neg = true;
      carry = 1;
    } else {
      carry = 0;
    }
    if (G == 1) {
      if (d) f(j, d, neg);
    } else if (d >= g && d != 0) {
      const uint32_t q = (d - g) / G;
      if (q * G + g == d) f(j, q, neg);
    }
  }
}

// Flat bucket of digit (j, b): j*wstride + b, with wstride = NB (one bucket set per window)
// or 0 (precomputed table, f3: all windows share one set).  The sorted entry of point i in
// window j is (i + j*istride) | sign<<31 with istride = 0, or n (row j of the table).
// histogram: counts[j*wstride + b] += 1 for every non-zero digit.  err |= 4 for k >= r.
template <class C>
__global__ void k_digit_counts(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                               uint32_t wstride, uint32_t* __restrict__ counts, uint32_t* err) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  ScalarReg<C> k;
  load_scalar<C>(k, scal, i);
  if (!scalar_in_range<C>(k)) { atomicOr(err, 4u); return; }
  for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool) { atomicAdd(counts + (size_t)j * wstride + b, 1u); });
}

// scatter: sorted[cursor[f]++] = i | sign << 31
template <class C>
__global__ void k_digit_scatter(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                                uint32_t wstride, uint32_t istride, uint32_t* __restrict__ cursor,
                                uint32_t* __restrict__ sorted) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  ScalarReg<C> k;
  load_scalar<C>(k, scal, i);
  if (!scalar_in_range<C>(k)) return;
  for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool neg) {
    uint32_t pos = atomicAdd(cursor + (size_t)j * wstride + b, 1u);
    sorted[pos] = ((uint32_t)i + (uint32_t)j * istride) | (neg ? SIGN_BIT : 0u);
  });
}

// debug: digits[i][j] (signed int32)
template <class C>
__global__ void k_digits_debug(const uint32_t* __restrict__ scal, size_t n, int c, int nwin, int32_t* out) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  ScalarReg<C> k;
  load_scalar<C>(k, scal, i);
  for (int j = 0; j < nwin; j++) out[i * nwin + j] = 0;
  for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool neg) { out[i * nwin + j] = neg ? -(int32_t)b : (int32_t)b; });
}

// ---------------------------------------------------------------------------------------
// exclusive scan of counts[0..F) -> goff[0..F], cursor[0..F)   (three-phase)
constexpr int SCAN_THREADS = 1024;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t v, uint32_t* smem, uint32_t* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) smem[wid] = x;
  __syncthreads();
  if (wid == 0) {
    uint32_t s = lane < (int)(blockDim.x >> 5) ? smem[lane] : 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    smem[lane] = s;
  }
  __syncthreads();
  uint32_t warp_prefix = wid ? smem[wid - 1] : 0u;
  if (total) *total = smem[(blockDim.x >> 5) - 1];
  __syncthreads();
  return warp_prefix + x - v;
}

static __global__ void k_bin_sort_impl(const uint32_t* __restrict__ binOff, const uint32_t* __restrict__ binIdx,
                                       const uint16_t* __restrict__ binFine, int shift, uint32_t nbin, uint32_t NB,
                                       uint32_t* __restrict__ goff, uint32_t* __restrict__ sorted) {
  extern __shared__ uint32_t cnt[];
  __shared__ uint32_t warp_sums[32];
  const uint32_t fb = blockIdx.x;
  const uint32_t j = fb / nbin, bin = fb % nbin;
  const uint32_t e0 = binOff[fb], e1 = binOff[fb + 1];
  const uint32_t nfine = 1u << shift;
  for (uint32_t i = threadIdx.x; i < nfine; i += blockDim.x) cnt[i] = 0;
  __syncthreads();
  // loads batched U per thread (memory-level parallelism), then the smem atomics
  constexpr int U = 8;
  for (uint32_t e = e0 + threadIdx.x; e < e1; e += blockDim.x * U) {
    uint32_t fv[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const uint32_t ee = e + u * blockDim.x;
      fv[u] = ee < e1 ? (uint32_t)__ldg(binFine + ee) : 0xFFFFFFFFu;
    }
#pragma unroll
    for (int u = 0; u < U; u++)
      if (fv[u] != 0xFFFFFFFFu) atomicAdd(cnt + fv[u], 1u);
  }
  __syncthreads();
  // exclusive scan of cnt[0..nfine): each thread owns a contiguous chunk
  const uint32_t per = (nfine + blockDim.x - 1) / blockDim.x;
  const uint32_t c0 = threadIdx.x * per, c1 = min(c0 + per, nfine);
  uint32_t sum = 0;
  for (uint32_t i = c0; i < c1; i++) sum += cnt[i];
  uint32_t run = block_exclusive_scan(sum, warp_sums, nullptr);
  for (uint32_t i = c0; i < c1; i++) {
    const uint32_t v = cnt[i];
    cnt[i] = run;
    const uint32_t b = (bin << shift) + i;
    if (b < NB) goff[(size_t)j * NB + b] = e0 + run;
    run += v;
  }
  __syncthreads();
  for (uint32_t e = e0 + threadIdx.x; e < e1; e += blockDim.x * U) {
    uint32_t fv[U], iv[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const uint32_t ee = e + u * blockDim.x;
      const bool ok = ee < e1;
      fv[u] = ok ? (uint32_t)__ldg(binFine + ee) : 0xFFFFFFFFu;
      iv[u] = ok ? __ldg(binIdx + ee) : 0u;
    }
#pragma unroll
    for (int u = 0; u < U; u++)
      if (fv[u] != 0xFFFFFFFFu) sorted[e0 + atomicAdd(cnt + fv[u], 1u)] = iv[u];
  }
}

static __global__ void k_scan_reduce(const uint32_t* __restrict__ counts, size_t F, uint32_t* __restrict__ tile_sums) {
  __shared__ uint32_t smem[32];
  size_t base = (size_t)blockIdx.x * SCAN_TILE + (size_t)threadIdx.x * SCAN_ITEMS;
  uint32_t s = 0;
#pragma unroll
  for (int q = 0; q < SCAN_ITEMS; q++)
    if (base + q < F) s += counts[base + q];
  uint32_t tot;
  block_exclusive_scan(s, smem, &tot);
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = tot;
}

// single block: exclusive scan of tile sums in place (ntiles arbitrary), writes total
static __global__ void k_scan_tiles(uint32_t* tile_sums, size_t ntiles, uint32_t* total_out) {
  __shared__ uint32_t smem[32];
  uint32_t carry = 0;
  for (size_t base = 0; base < ntiles; base += blockDim.x) {
    size_t i = base + threadIdx.x;
    uint32_t v = i < ntiles ? tile_sums[i] : 0u;
    uint32_t tot;
    uint32_t ex = block_exclusive_scan(v, smem, &tot);
    if (i < ntiles) tile_sums[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) *total_out = carry;
}

static __global__ void k_scan_apply(const uint32_t* __restrict__ counts, size_t F, const uint32_t* __restrict__ tile_sums,
                             uint32_t* __restrict__ goff, uint32_t* __restrict__ cursor) {
  __shared__ uint32_t smem[32];
  size_t base = (size_t)blockIdx.x * SCAN_TILE + (size_t)threadIdx.x * SCAN_ITEMS;
  uint32_t v[SCAN_ITEMS];
  uint32_t s = 0;
#pragma unroll
  for (int q = 0; q < SCAN_ITEMS; q++) {
    v[q] = base + q < F ? counts[base + q] : 0u;
    s += v[q];
  }
  uint32_t ex = block_exclusive_scan(s, smem, nullptr) + tile_sums[blockIdx.x];
#pragma unroll
  for (int q = 0; q < SCAN_ITEMS; q++) {
    if (base + q < F) {
      goff[base + q] = ex;
      cursor[base + q] = ex;
    }
    ex += v[q];
  }
}

// ---------------------------------------------------------------------------------------
// a3, binned (default): two-level counting sort, the B200 form of the paper's hierarchical
// bucket scatter (§3.2.1, Alg. 3).  With c up to 22 a window has 2^21 buckets,
// far beyond shared memory (the paper's scheme stops at s = 14), so buckets are
// grouped into coarse bins of 2^shift buckets (flat bin fb = j*nbin + (b >> shift),
// nwin*nbin <= ~13K so a per-block bin histogram fits in shared memory):
//   k_bin_count   per-block smem histogram over bins -> one global atomic per (block, bin)
//   scan          bin offsets
//   k_bin_scatter per-block smem ranks; one atomic per (block, bin) reserves a contiguous
//                 run; entries (idx|sign, fine = b mod 2^shift) land in short runs per bin
//   k_bin_sort    one block per bin: smem counting sort on `fine` (2^shift counters),
//                 writes goff for the bin's buckets and the final sorted indices, all inside
//                 the bin's own contiguous output range.
constexpr int BIN_THREADS = 512;
constexpr int BIN_PTS = 16;                      // points per thread per tile
constexpr int BIN_TILE = BIN_THREADS * BIN_PTS;  // 8192 points per block: ~8 entries per bin per block

template <class C>
__global__ void __launch_bounds__(BIN_THREADS) k_bin_count(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                                                           int shift, uint32_t FB, uint32_t wstride,
                                                           uint32_t* __restrict__ binCount, uint32_t* err) {
  extern __shared__ uint32_t hist[];
  for (uint32_t i = threadIdx.x; i < FB; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const size_t base = (size_t)blockIdx.x * BIN_TILE;
  bool bad = false;
  for (int q = 0; q < BIN_PTS; q++) {
    const size_t i = base + (size_t)q * BIN_THREADS + threadIdx.x;
    if (i >= n) break;
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) { bad = true; continue; }
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool) { atomicAdd(hist + (uint32_t)j * wstride + (b >> shift), 1u); });
  }
  if (bad) atomicOr(err, 4u);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < FB; i += blockDim.x)
    if (hist[i]) atomicAdd(binCount + i, hist[i]);
}

template <class C>
__global__ void __launch_bounds__(BIN_THREADS) k_bin_scatter(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                                                             int shift, uint32_t FB, uint32_t wstride, uint32_t istride,
                                                             uint32_t* __restrict__ binCursor,
                                                             uint32_t* __restrict__ binIdx, uint16_t* __restrict__ binFine) {
  extern __shared__ uint32_t sm[];
  uint32_t* hist = sm;
  uint32_t* base = sm + FB;
  for (uint32_t i = threadIdx.x; i < FB; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const size_t tile = (size_t)blockIdx.x * BIN_TILE;
  for (int q = 0; q < BIN_PTS; q++) {
    const size_t i = tile + (size_t)q * BIN_THREADS + threadIdx.x;
    if (i >= n) break;
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) continue;
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool) { atomicAdd(hist + (uint32_t)j * wstride + (b >> shift), 1u); });
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < FB; i += blockDim.x) {
    const uint32_t h = hist[i];
    base[i] = h ? atomicAdd(binCursor + i, h) : 0u;
    hist[i] = 0;
  }
  __syncthreads();
  const uint32_t fmask = (1u << shift) - 1u;
  for (int q = 0; q < BIN_PTS; q++) {
    const size_t i = tile + (size_t)q * BIN_THREADS + threadIdx.x;
    if (i >= n) break;
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) continue;
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool neg) {
      const uint32_t fb = (uint32_t)j * wstride + (b >> shift);
      const uint32_t pos = base[fb] + atomicAdd(hist + fb, 1u);
      binIdx[pos] = ((uint32_t)i + (uint32_t)j * istride) | (neg ? SIGN_BIT : 0u);
      binFine[pos] = (uint16_t)(b & fmask);
    });
  }
}

// k_bin_sort_impl (one block per flat bin, nfine = 2^shift <= 8192) is defined with the
// scan helpers above.

#include "sort3.cuh"
#include "sort4.cuh"


// ---------------------------------------------------------------------------------------
// number of non-empty flat buckets (statistics only)
static __global__ void k_count_nonempty(const uint32_t* __restrict__ goff, size_t F, unsigned long long* out) {
  size_t f = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned v = (f < F && goff[f + 1] != goff[f]) ? 1u : 0u;
  v = __reduce_add_sync(0xffffffffu, v);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(out, (unsigned long long)v);
}

// ---------------------------------------------------------------------------------------
// a4: bucket accumulation (PACC, Alg. 4), load-balanced over equal slices of `sorted`.
//   Thread t owns entries [t*slice, min((t+1)*slice, M)).  Runs of equal flat bucket f are
//   accumulated in registers.  A bucket whose first entry lies in the slice is written to
//   buckets[f] (complete, or the owner's partial); a slice that starts inside a bucket
//   writes its partial to carry[t] (carry_f[t] = f) for k_fixup.
// Gathers the point of a sorted entry; negates y for a negative digit.  Returns false for
// the point at infinity (stored as x = y = 0).  A stored y is 0 only for O: points with
// y = 0 (order 2) are rejected at context creation (k_points_to_mont).
template <class C>
DEVI bool point_for_entry(uint32_t* x, uint32_t* y, const uint32_t* __restrict__ pts, uint32_t e) {
  load_point<C>(x, y, pts, e & ~SIGN_BIT);
  if (fis_zero<C, 2>(y)) return false;
  if (e & SIGN_BIT) fneg<C, 2>(y, y);
  return true;
}

#ifndef MSM_ACC_PREFETCH
#define MSM_ACC_PREFETCH 3  // next point gather: 3 registers (L <= 13), 2/1 L1 prefetch, 0 none
#endif
#ifndef MSM_ACC_PADD
#define MSM_ACC_PADD 0  // f4 ablation: PADD (Alg. 1) with Z = 1 operand instead of PACC (Alg. 4)
#endif
#ifndef MSM_ACC_SYNC
#define MSM_ACC_SYNC 1  // k_accumulate_sync (256-thread blocks in per-iteration lockstep) for L <= 13
#endif
#ifndef MSM_ACC_SYNC_ALL
// lockstep accumulation for MNT4-753 too (L1 prefetch there): r01 measured it slower
// (253.7 vs 249.0 ms); in r02, after the small-n block spreading and the reduce changes,
// it is faster — accumulate 240.2 -> 228.2 ms, C5 279.2 -> 267.9 ms
#define MSM_ACC_SYNC_ALL 1
#endif
#ifndef MSM_SEG_SYNC
#define MSM_SEG_SYNC 0  // A/B: k_bucket_segments with 256-thread blocks in per-bucket lockstep
#endif
constexpr int SEG_NT = MSM_SEG_SYNC ? 256 : 128;
#ifndef MSM_ACC_SMEM
#define MSM_ACC_SMEM 0  // A/B: k_accumulate_smem (operands in shared-memory slots, one fmul2 body)
#endif
#ifndef MSM_ACC_TRIPLE
#define MSM_ACC_TRIPLE 0  // k_accumulate: PACC in groups 2,2,3,3 (xyzz_acc_hot3) instead of 5 pairs
#endif
#ifndef MSM_ACC_DUAL
#define MSM_ACC_DUAL 1  // k_accumulate: column-interleaved multiplication pairs (xyzz_acc_hot)
#endif

// L1 prefetch of the (at most two) 128-B lines holding the stored point of entry e
template <class C>
DEVI void prefetch_point(const uint32_t* __restrict__ pts, uint32_t e) {
  const char* a = reinterpret_cast<const char*>(pts + (size_t)(e & ~SIGN_BIT) * Layout<C>::PW);
  asm volatile("prefetch.global.L1 [%0];" ::"l"(a));
  asm volatile("prefetch.global.L1 [%0];" ::"l"(a + Layout<C>::PW * 4 - 4));
}

template <class C>
DEVI void acc_start(Xyzz<C>& acc, const uint32_t* x, const uint32_t* y, bool ok) {
  if (ok) xyzz_from_affine<C>(acc, x, y);
  else xyzz_set_zero<C>(acc);
}

// largest f with goff[f] <= e (goff non-decreasing, goff[0] = 0, e < goff[F])
DEVI uint32_t find_bucket(const uint32_t* __restrict__ goff, uint32_t F, uint32_t e) {
  uint32_t lo = 0, hi = F;  // invariant goff[lo] <= e < goff[hi]
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (__ldg(goff + mid) <= e) lo = mid; else hi = mid;
  }
  return lo;
}

template <class C>
__global__ void __launch_bounds__(128, MSM_ACC_MINB) k_accumulate(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted,
                                                    const uint32_t* __restrict__ goff, uint32_t F,
                                                    uint32_t* __restrict__ buckets, uint32_t* __restrict__ carry_pts,
                                                    int32_t* __restrict__ carry_f, uint32_t nthreads,
                                                    uint32_t* __restrict__ nlong) {
  constexpr int XW = Layout<C>::XW;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0) *nlong = 0;  // long-run list of k_fixup (same stream, later kernel)
  if (t >= nthreads) return;
  // equal slices of the M entries actually present (M <= n*nwin: zero digits are skipped)
  const uint32_t M = __ldg(goff + F);
  const uint32_t slice = M ? (M + nthreads - 1) / nthreads : 1u;
  const uint64_t e0l = (uint64_t)t * slice;
  if (e0l >= M) { carry_f[t] = -1; return; }
  const uint32_t e0 = (uint32_t)e0l;
  const uint32_t e1 = (uint32_t)(e0l + slice < (uint64_t)M ? e0l + slice : (uint64_t)M);
  uint32_t f = find_bucket(goff, F, e0);
  uint32_t end = __ldg(goff + f + 1);
  bool head = __ldg(goff + f) < e0;
  Xyzz<C> acc;
  uint32_t x[C::L], y[C::L];
  bool ok = point_for_entry<C>(x, y, pts, __ldg(sorted + e0));
  acc_start<C>(acc, x, y, ok);
  int32_t my_carry = -1;
  // Gather of the next entry's stored point (PF, A/B-able with MSM_ACC_PREFETCH):
  //   3  into REGISTERS one PACC ahead (index read two ahead) — default for L <= 13.  The
  //      first use of a gathered point was the top stall site of the kernel (ncu source
  //      view: the zero test of y waiting on the gather, ~4 % of samples) even with an L1
  //      prefetch, because the L1 hit latency itself sat on the critical path; 26 more
  //      registers keep 8 warps/SM.  MNT4-753 (L = 27, already at 255 registers) keeps 1.
  //   2  L1 prefetch two PACCs ahead;  1  L1 prefetch one PACC ahead;  0  none.
  constexpr int PF = (MSM_ACC_PREFETCH == 3 && C::L > 13) ? 1 : MSM_ACC_PREFETCH;
  uint32_t nx[C::L], ny[C::L];
  uint32_t ent1 = 0, ent2 = 0, ent3 = 0;
  if constexpr (PF > 0) {
    ent1 = e0 + 1 < e1 ? __ldg(sorted + e0 + 1) : 0u;
    ent2 = e0 + 2 < e1 ? __ldg(sorted + e0 + 2) : 0u;
    if constexpr (PF == 3) {
      if (e0 + 1 < e1) load_point<C>(nx, ny, pts, ent1 & ~SIGN_BIT);
    } else {
      if (e0 + 1 < e1) prefetch_point<C>(pts, ent1);
    }
    if constexpr (PF == 2) {
      ent3 = e0 + 3 < e1 ? __ldg(sorted + e0 + 3) : 0u;
      if (e0 + 2 < e1) prefetch_point<C>(pts, ent2);
    }
  }
  for (uint32_t e = e0 + 1; e < e1; e++) {
    uint32_t ent;
    if constexpr (PF == 3) {
      ent = ent1;
      ent1 = ent2;
      fcopy<C>(x, nx);
      fcopy<C>(y, ny);
      if (e + 1 < e1) load_point<C>(nx, ny, pts, ent1 & ~SIGN_BIT);
      if (e + 2 < e1) ent2 = __ldg(sorted + e + 2);
      ok = !fis_zero<C, 2>(y);
      if (ok && (ent & SIGN_BIT)) fneg<C, 2>(y, y);
    } else {
      if constexpr (PF == 2) {
        ent = ent1;
        ent1 = ent2;
        ent2 = ent3;
        if (e + 2 < e1) prefetch_point<C>(pts, ent2);
        if (e + 3 < e1) ent3 = __ldg(sorted + e + 3);
      } else if constexpr (PF == 1) {
        ent = ent1;
        ent1 = ent2;
        if (e + 1 < e1) prefetch_point<C>(pts, ent1);
        if (e + 2 < e1) ent2 = __ldg(sorted + e + 2);
      } else {
        ent = __ldg(sorted + e);
      }
      ok = point_for_entry<C>(x, y, pts, ent);
    }
    if (e == end) {
      if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, acc); my_carry = (int32_t)f; head = false; }
      else store_xyzz<C>(buckets + (size_t)f * XW, acc);
      do { f++; end = __ldg(goff + f + 1); } while (end <= e);
      acc_start<C>(acc, x, y, ok);
    } else if (ok) {
#if MSM_ACC_PADD
      {  // f4 ablation (Fig. 12): general PADD (Alg. 1, 14 mults) instead of PACC
        Xyzz<C> Pt;
        xyzz_from_affine<C>(Pt, x, y);
        xyzz_add<C>(acc, acc, Pt);
      }
#elif MSM_ACC_DUAL
      if (MSM_ACC_TRIPLE ? xyzz_acc_hot3<C>(acc, x, y) : xyzz_acc_hot<C>(acc, x, y)) {  // rare: the point equals the accumulator
        Xyzz<C> T = acc;
        xyzz_dbl<C>(acc, T);
      }
#else
      xyzz_acc<C>(acc, x, y);
#endif
    }
  }
  if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, acc); my_carry = (int32_t)f; }
  else store_xyzz<C>(buckets + (size_t)f * XW, acc);
  carry_f[t] = my_carry;
}

// ---------------------------------------------------------------------------------------
// a4 variant (MSM_ACC_SYNC, A/B): 256-thread blocks, one per SM (2 warps per scheduler as
// in k_accumulate), with a block barrier at the top of every PACC iteration so the two
// warps of each scheduler walk the ~90 KB straight-line PACC code in lockstep and share
// instruction fetches (ncu: no_instruction is 17 % of k_accumulate's stall samples, spread
// evenly over the straight-line code).  Every thread runs the same number of iterations
// (the uniform slice length); threads without work only take part in the barriers.
#ifndef MSM_ACC_SYNC_NT
#define MSM_ACC_SYNC_NT 256  // A/B: 384 = 3 warps per scheduler (<= 168 registers)
#endif
constexpr int ACC_SYNC_NT = MSM_ACC_SYNC_NT;
// DIRECT (batch-affine front end, baff.cuh): entry e's point is pts[e] itself (the folded
// affine points, bucket-major), no index and no sign.
template <bool DIRECT>
DEVI uint32_t entry_at(const uint32_t* __restrict__ sorted, uint32_t e) {
  if constexpr (DIRECT) return e;
  else return __ldg(sorted + e);
}

// INIT (chunked host scalars, engine.cu): the buckets already hold the sums of earlier
// chunks, so a thread that owns a bucket's first entry starts from the stored bucket (O
// if it was empty) and adds the entry by PACC instead of starting from the entry; the loop
// then begins at the slice's first entry (every lane one more iteration, still uniform).
template <class C, bool DIRECT = false, bool INIT = false>
__global__ void __launch_bounds__(ACC_SYNC_NT, 1) k_accumulate_sync(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted,
                                                    const uint32_t* __restrict__ goff, uint32_t F,
                                                    uint32_t* __restrict__ buckets, uint32_t* __restrict__ carry_pts,
                                                    int32_t* __restrict__ carry_f, uint32_t nthreads,
                                                    uint32_t* __restrict__ nlong) {
  constexpr int XW = Layout<C>::XW;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0) *nlong = 0;
  const uint32_t M = __ldg(goff + F);
  const uint32_t slice = M ? (M + nthreads - 1) / nthreads : 1u;
  const uint64_t e0l = (uint64_t)t * slice;
  const bool active = t < nthreads && e0l < M;
  if (t < nthreads && !active) carry_f[t] = -1;
  const uint32_t e0 = active ? (uint32_t)e0l : 0u;
  const uint32_t e1 = active ? (uint32_t)(e0l + slice < (uint64_t)M ? e0l + slice : (uint64_t)M) : 0u;
  uint32_t f = 0, end = 0;
  bool head = false, ok = false;
  Xyzz<C> acc;
  uint32_t x[C::L], y[C::L], nx[C::L], ny[C::L];
  uint32_t ent1 = 0, ent2 = 0;
  int32_t my_carry = -1;
  // next point into registers one PACC ahead (L <= 13), or an L1 prefetch for MNT4-753
  // whose 255 registers leave no room for it
  constexpr bool REGPF = C::L <= 13;
  // INIT: the first entry goes through the loop (q = 0) like every other one
  constexpr uint32_t Q0 = INIT ? 0u : 1u;
  if (active) {
    f = find_bucket(goff, F, e0);
    end = __ldg(goff + f + 1);
    head = __ldg(goff + f) < e0;
    if constexpr (INIT) {
      if (head) xyzz_set_zero<C>(acc);
      else load_xyzz<C>(acc, buckets + (size_t)f * XW);
    } else {
      ok = point_for_entry<C>(x, y, pts, entry_at<DIRECT>(sorted, e0));
      acc_start<C>(acc, x, y, ok);
    }
    ent1 = e0 + Q0 < e1 ? entry_at<DIRECT>(sorted, e0 + Q0) : 0u;
    ent2 = e0 + Q0 + 1 < e1 ? entry_at<DIRECT>(sorted, e0 + Q0 + 1) : 0u;
    if constexpr (REGPF) {
      if (e0 + Q0 < e1) load_point<C>(nx, ny, pts, ent1 & ~SIGN_BIT);
    } else {
      if (e0 + Q0 < e1) prefetch_point<C>(pts, ent1);
    }
  }
  for (uint32_t q = Q0; q < slice; q++) {
    __syncthreads();
    const uint32_t e = e0 + q;
    if (!active || e >= e1) continue;
    const uint32_t ent = ent1;
    ent1 = ent2;
    if constexpr (REGPF) {
      fcopy<C>(x, nx);
      fcopy<C>(y, ny);
      if (e + 1 < e1) load_point<C>(nx, ny, pts, ent1 & ~SIGN_BIT);
      if (e + 2 < e1) ent2 = entry_at<DIRECT>(sorted, e + 2);
      ok = !fis_zero<C, 2>(y);
      if (ok && (ent & SIGN_BIT)) fneg<C, 2>(y, y);
    } else {
      if (e + 1 < e1) prefetch_point<C>(pts, ent1);
      if (e + 2 < e1) ent2 = entry_at<DIRECT>(sorted, e + 2);
      ok = point_for_entry<C>(x, y, pts, ent);
    }
    if constexpr (INIT) {
      if (e == end) {
        if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, acc); my_carry = (int32_t)f; head = false; }
        else store_xyzz<C>(buckets + (size_t)f * XW, acc);
        do { f++; end = __ldg(goff + f + 1); } while (end <= e);
        load_xyzz<C>(acc, buckets + (size_t)f * XW);
      }
      if (ok) {
        if (xyzz_acc_hot<C>(acc, x, y)) {
          Xyzz<C> T = acc;
          xyzz_dbl<C>(acc, T);
        }
      }
    } else {
      if (e == end) {
        if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, acc); my_carry = (int32_t)f; head = false; }
        else store_xyzz<C>(buckets + (size_t)f * XW, acc);
        do { f++; end = __ldg(goff + f + 1); } while (end <= e);
        acc_start<C>(acc, x, y, ok);
      } else if (ok) {
        if (xyzz_acc_hot<C>(acc, x, y)) {
          Xyzz<C> T = acc;
          xyzz_dbl<C>(acc, T);
        }
      }
    }
  }
  if (active) {
    if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, acc); my_carry = (int32_t)f; }
    else store_xyzz<C>(buckets + (size_t)f * XW, acc);
    carry_f[t] = my_carry;
  }
}

#ifndef MSM_BAFF
#define MSM_BAFF 0  // batch-affine a4 front end (ablation, baff.cuh): instantiated only with -DMSM_BAFF=1
#endif
#include "baff.cuh"

// ---------------------------------------------------------------------------------------
// a4 variant (MSM_ACC_SMEM, A/B): the PAPER.md:267 idea — big integers cached in shared
// memory instead of registers — taken to its end.  The accumulator and every PACC
// temporary live in per-thread shared-memory slots; the ten multiplications are five
// steps of ONE column-interleaved fmul2 body (squarings as multiplications) whose operands
// are loaded from slots chosen per step, so the hot loop is a few KB of code instead of
// ~100 KB (ncu: no_instruction is the second stall of k_accumulate) and needs far fewer
// registers.  Slot layout: word (slot*L + i) of thread t at smem[(slot*L + i)*ACC_NT + t].
constexpr int ACC_NT = 128;
constexpr int ACC_SLOTS = 10;  // X Y ZZ ZZZ P R PP V PPP Q
enum { SX = 0, SY, SZZ, SZZZ, SP, SR, SPP, SV, SPPP, SQ };

// operand slots (a1, b1, a2, b2) of the step program, 4 bits each: steps 0-4 are PACC
// (Alg. 4), steps 5-9 the doubling dbl-2008-s-1 (a = 0 curves) for the rare acc == P case
static __constant__ uint32_t ACC_OPS[10] = {
    (SPPP) | (SZZ << 4) | (SQ << 8) | (SZZZ << 12),
    (SP) | (SP << 4) | (SR << 8) | (SR << 12),
    (SPP) | (SP << 4) | (SX << 8) | (SPP << 12),
    (SZZ) | (SPP << 4) | (SY << 8) | (SPPP << 12),
    (SZZZ) | (SPPP << 4) | (SR << 8) | (SQ << 12),
    (SP) | (SP << 4) | (SX << 8) | (SX << 12),
    (SP) | (SR << 4) | (SX << 8) | (SR << 12),
    (SR) | (SZZ << 4) | (SV << 8) | (SZZZ << 12),
    (SV) | (SY << 4) | (SQ << 8) | (SQ << 12),
    (SQ) | (SPP << 4) | (SQ << 8) | (SQ << 12)};

template <class C>
DEVI void sload(uint32_t* v, const uint32_t* sb, int slot) {
#pragma unroll
  for (int i = 0; i < C::L; i++) v[i] = sb[(slot * C::L + i) * ACC_NT];
}
template <class C>
DEVI void sstore(uint32_t* sb, int slot, const uint32_t* v) {
#pragma unroll
  for (int i = 0; i < C::L; i++) sb[(slot * C::L + i) * ACC_NT] = v[i];
}
template <class C>
DEVI void sload_xyzz(Xyzz<C>& A, const uint32_t* sb) {
  sload<C>(A.X, sb, SX); sload<C>(A.Y, sb, SY); sload<C>(A.ZZ, sb, SZZ); sload<C>(A.ZZZ, sb, SZZZ);
}
template <class C>
DEVI void sstore_xyzz(uint32_t* sb, const Xyzz<C>& A) {
  sstore<C>(sb, SX, A.X); sstore<C>(sb, SY, A.Y); sstore<C>(sb, SZZ, A.ZZ); sstore<C>(sb, SZZZ, A.ZZZ);
}
template <class C>
DEVI bool s_is_zero(const uint32_t* sb, int slot) {
  uint32_t v[C::L];
  sload<C>(v, sb, slot);
  return fis_zero<C, 2>(v);
}

// acc(slots X..ZZZ) += (x, y) held in slots PPP, Q: Alg. 4 with the bounds of
// xyzz_acc_hot, as a program of multiplication pairs through ONE fmul2 body.
//   step 0  U2 = x ZZ,  S2 = y ZZZ       P = U2 - X, R = S2 - Y (zero tests)
//   step 1  PP = P P,   V = R R
//   step 2  PPP = PP P, Q = X PP          X' = V - PPP - 2Q, D = Q - X'
//   step 3  ZZ' = ZZ PP, T = Y PPP
//   step 4  ZZZ' = ZZZ PPP, E = R D       Y' = E - T
// acc == (x, y) (P = R = 0) continues with the doubling of acc (xyzz_dbl's formula/bounds):
//   pre     U = 2Y                        (< 8p)
//   step 5  V = U U,    X^2 = X X
//   step 6  W = U V,    S = X V           M = 3 X^2
//   step 7  ZZ' = V ZZ, ZZZ' = W ZZZ
//   step 8  WY = W Y,   M^2               X' = M^2 - 2S, D = S - X'
//   step 9  E = M D     (pair slot idle)  Y' = E - WY
template <class C>
DEVI void s_pacc(uint32_t* sb) {
  constexpr int L = C::L;
  static_assert(C::A_ZERO, "smem step program: a = 0 curves");
  // the step bounds are opaque to the optimiser, so the loop stays a loop (one fmul2 body)
  int step, stop;
  asm volatile("mov.u32 %0, 0;" : "=r"(step));
  asm volatile("mov.u32 %0, 5;" : "=r"(stop));
#pragma unroll 1
  for (; step < stop; step++) {
    const uint32_t ops = ACC_OPS[step];
    uint32_t a1[L], b1[L], a2[L], b2[L], r1[L], r2[L];
    sload<C>(a1, sb, ops & 15);
    sload<C>(b1, sb, (ops >> 4) & 15);
    sload<C>(a2, sb, (ops >> 8) & 15);
    sload<C>(b2, sb, (ops >> 12) & 15);
    fmul2<C>(r1, a1, b1, r2, a2, b2);
    switch (step) {
      case 0:
        sload<C>(a1, sb, SX);
        sload<C>(a2, sb, SY);
        fsub<C, 8>(r1, r1, a1);  // P = U2 - X    < 10p
        fsub<C, 4>(r2, r2, a2);  // R = S2 - Y    < 6p
        if (fis_zero<C, 10>(r1)) {
          if (fis_zero<C, 6>(r2)) {  // acc == (x, y): double acc instead
            fadd<C>(b1, a2, a2);     // U = 2Y < 8p
            sstore<C>(sb, SP, b1);
            step = 4;
            stop = 10;
          } else {                   // acc == -(x, y): O
            fzero<C>(a1);
#pragma unroll
            for (int q = 0; q < 4; q++) sstore<C>(sb, q, a1);
            stop = 0;
          }
          break;
        }
        sstore<C>(sb, SP, r1);
        sstore<C>(sb, SR, r2);
        break;
      case 1:
        sstore<C>(sb, SPP, r1);  // PP < 2p
        sstore<C>(sb, SV, r2);   // V  < 2p
        break;
      case 2:
        sload<C>(a1, sb, SV);
        fadd<C>(b1, r1, r2);
        fadd<C>(b1, b1, r2);     // PPP + 2Q      < 6p
        fsub<C, 6>(b2, a1, b1);  // X' = V - PPP - 2Q < 8p
        fsub<C, 8>(a2, r2, b2);  // D = Q - X'    < 10p
        sstore<C>(sb, SPPP, r1);
        sstore<C>(sb, SX, b2);
        sstore<C>(sb, SQ, a2);
        break;
      case 3:
        sstore<C>(sb, SZZ, r1);  // ZZ' < 2p
        sstore<C>(sb, SV, r2);   // T   < 2p
        break;
      case 4:
        sload<C>(a1, sb, SV);
        fsub<C, 2>(b1, r2, a1);  // Y' = E - T    < 4p
        sstore<C>(sb, SZZZ, r1);
        sstore<C>(sb, SY, b1);
        break;
      case 5:
        sstore<C>(sb, SR, r1);   // V = U^2 < 2p
        sstore<C>(sb, SPP, r2);  // X^2 < 2p
        break;
      case 6:
        sstore<C>(sb, SV, r1);    // W = U V < 2p
        sstore<C>(sb, SPPP, r2);  // S = X V < 2p
        sload<C>(a1, sb, SPP);
        fadd<C>(b1, a1, a1);
        fadd<C>(b1, b1, a1);      // M = 3 X^2 < 6p
        sstore<C>(sb, SQ, b1);
        break;
      case 7:
        sstore<C>(sb, SZZ, r1);   // ZZ' = V ZZ < 2p
        sstore<C>(sb, SZZZ, r2);  // ZZZ' = W ZZZ < 2p
        break;
      case 8:
        sstore<C>(sb, SR, r1);    // WY < 2p
        sload<C>(a1, sb, SPPP);   // S
        fadd<C>(b1, a1, a1);      // 2S < 4p
        fsub<C, 4>(b2, r2, b1);   // X' = M^2 - 2S < 6p
        fsub<C, 6>(a2, a1, b2);   // D = S - X' < 8p
        sstore<C>(sb, SX, b2);
        sstore<C>(sb, SPP, a2);
        break;
      default:
        sload<C>(a1, sb, SR);
        fsub<C, 2>(b1, r1, a1);   // Y' = M D - WY < 4p
        sstore<C>(sb, SY, b1);
        break;
    }
  }
}

template <class C>
DEVI void s_start(uint32_t* sb, const uint32_t* x, const uint32_t* y, bool ok) {
  Xyzz<C> A;
  if (ok) xyzz_from_affine<C>(A, x, y);
  else xyzz_set_zero<C>(A);
  sstore_xyzz<C>(sb, A);
}

template <class C>
__global__ void __launch_bounds__(ACC_NT, MSM_ACC_MINB) k_accumulate_smem(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted,
                                                    const uint32_t* __restrict__ goff, uint32_t F,
                                                    uint32_t* __restrict__ buckets, uint32_t* __restrict__ carry_pts,
                                                    int32_t* __restrict__ carry_f, uint32_t nthreads,
                                                    uint32_t* __restrict__ nlong) {
  constexpr int XW = Layout<C>::XW;
  extern __shared__ uint32_t acc_smem[];
  uint32_t* sb = acc_smem + threadIdx.x;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0) *nlong = 0;
  if (t >= nthreads) return;
  const uint32_t M = __ldg(goff + F);
  const uint32_t slice = M ? (M + nthreads - 1) / nthreads : 1u;
  const uint64_t e0l = (uint64_t)t * slice;
  if (e0l >= M) { carry_f[t] = -1; return; }
  const uint32_t e0 = (uint32_t)e0l;
  const uint32_t e1 = (uint32_t)(e0l + slice < (uint64_t)M ? e0l + slice : (uint64_t)M);
  uint32_t f = find_bucket(goff, F, e0);
  uint32_t end = __ldg(goff + f + 1);
  bool head = __ldg(goff + f) < e0;
  uint32_t x[C::L], y[C::L];
  bool ok = point_for_entry<C>(x, y, pts, __ldg(sorted + e0));
  s_start<C>(sb, x, y, ok);
  int32_t my_carry = -1;
  uint32_t ent1 = e0 + 1 < e1 ? __ldg(sorted + e0 + 1) : 0u;
  uint32_t ent2 = e0 + 2 < e1 ? __ldg(sorted + e0 + 2) : 0u;
  if (e0 + 1 < e1) prefetch_point<C>(pts, ent1);
  Xyzz<C> A;
  for (uint32_t e = e0 + 1; e < e1; e++) {
    const uint32_t ent = ent1;
    ent1 = ent2;
    if (e + 1 < e1) prefetch_point<C>(pts, ent1);
    if (e + 2 < e1) ent2 = __ldg(sorted + e + 2);
    ok = point_for_entry<C>(x, y, pts, ent);
    if (e == end) {
      sload_xyzz<C>(A, sb);
      if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, A); my_carry = (int32_t)f; head = false; }
      else store_xyzz<C>(buckets + (size_t)f * XW, A);
      do { f++; end = __ldg(goff + f + 1); } while (end <= e);
      s_start<C>(sb, x, y, ok);
    } else if (ok) {
      if (s_is_zero<C>(sb, SZZ)) {
        s_start<C>(sb, x, y, true);
      } else {
        sstore<C>(sb, SPPP, x);
        sstore<C>(sb, SQ, y);
        s_pacc<C>(sb);
      }
    }
  }
  sload_xyzz<C>(A, sb);
  if (head) { store_xyzz<C>(carry_pts + (size_t)t * XW, A); my_carry = (int32_t)f; }
  else store_xyzz<C>(buckets + (size_t)f * XW, A);
  carry_f[t] = my_carry;
}

// Calls to __noinline__ EC functions below are made from warp-uniform control flow only
// (loops with warp-uniform trip counts; per-lane differences become O operands): sm_100a
// keeps the stack pointer in a uniform register, and lanes diverging around a call corrupt
// local memory (found with compute-sanitizer).
template <class C>
DEVI void xyzz_select(Xyzz<C>& R, const Xyzz<C>& A, bool take) {
  if (take) R = A;
  else xyzz_set_zero<C>(R);
}

// Carries of one bucket are consecutive (slices are in entry order).  Run leaders of short
// runs (<= FIX_SHORT carries) add them serially into buckets[f]; longer runs (a bucket
// spanning many slices: heavy buckets of skewed scalars, or a top window holding only the
// carry digit) go to a list for k_fixup_long's block-wide tree.
constexpr int FIX_SHORT = 8;
constexpr int FIX_THREADS = 256;

template <class C>
__global__ void k_fixup(uint32_t* __restrict__ buckets, const uint32_t* __restrict__ carry_pts,
                        const int32_t* __restrict__ carry_f, uint32_t nthreads,
                        uint32_t* __restrict__ nlong, uint32_t* __restrict__ longs) {
  constexpr int XW = Layout<C>::XW;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  const int32_t f = t < nthreads ? carry_f[t] : -1;
  bool leader = f >= 0 && (t == 0 || carry_f[t - 1] != f);
  uint32_t R = 0;
  if (leader) {
    while (R <= FIX_SHORT && t + R < nthreads && carry_f[t + R] == f) R++;
    if (R > FIX_SHORT) {
      longs[atomicAdd(nlong, 1u)] = t;
      leader = false;
    }
  }
  const unsigned mask = __ballot_sync(0xffffffffu, leader);
  if (!leader) return;
  Xyzz<C> s, b;
  load_xyzz<C>(s, carry_pts + (size_t)t * XW);
  uint32_t u = t + 1;
  bool more = u < nthreads && carry_f[u] == f;
  while (__any_sync(mask, more)) {
    if (more) load_xyzz<C>(b, carry_pts + (size_t)u * XW);
    else xyzz_set_zero<C>(b);
    __syncwarp(mask);
    xyzz_add_ni<C>(s, s, b);
    if (more) {
      u++;
      more = u < nthreads && carry_f[u] == f;
    }
  }
  load_xyzz<C>(b, buckets + (size_t)f * XW);
  __syncwarp(mask);
  xyzz_add_ni<C>(s, s, b);
  store_xyzz<C>(buckets + (size_t)f * XW, s);
}

// one block per long run (grid-stride over the list of run leaders): strided partial sums
// while the run lasts (a bucket's carries are one contiguous run, so membership
// carry_f[t] == f is exact for t >= t0), then a shared-memory tree; every lane calls the
// adds (O operands where idle).
template <class C>
__global__ void __launch_bounds__(FIX_THREADS) k_fixup_long(uint32_t* __restrict__ buckets, const uint32_t* __restrict__ carry_pts,
                                                            const int32_t* __restrict__ carry_f, uint32_t nthreads,
                                                            const uint32_t* __restrict__ nlong, const uint32_t* __restrict__ longs) {
  constexpr int XW = Layout<C>::XW;
  extern __shared__ uint32_t red[];  // [FIX_THREADS][XW]
  const uint32_t cnt = *nlong;
  for (uint32_t q = blockIdx.x; q < cnt; q += gridDim.x) {
    const uint32_t t0 = longs[q];
    const int32_t f = carry_f[t0];
    Xyzz<C> s, b;
    xyzz_set_zero<C>(s);
    for (uint32_t base = t0;; base += FIX_THREADS) {
      const uint32_t u = base + threadIdx.x;
      const bool in = u < nthreads && carry_f[u] == f;
      if (!__syncthreads_or(in)) break;
      if (in) load_xyzz<C>(b, carry_pts + (size_t)u * XW);
      else xyzz_set_zero<C>(b);
      xyzz_add_ni<C>(s, s, b);
    }
    store_xyzz<C>(red + threadIdx.x * XW, s);
    __syncthreads();
    for (int h = FIX_THREADS / 2; h >= 1; h >>= 1) {
      if ((int)threadIdx.x < (h < 32 ? 32 : h)) {
        if ((int)threadIdx.x < h) {
          load_xyzz<C>(s, red + threadIdx.x * XW);
          load_xyzz<C>(b, red + (threadIdx.x + h) * XW);
        } else {
          xyzz_set_zero<C>(s);
          xyzz_set_zero<C>(b);
        }
        xyzz_add_ni<C>(s, s, b);
      }
      __syncthreads();
      if ((int)threadIdx.x < h) store_xyzz<C>(red + threadIdx.x * XW, s);
      __syncthreads();
    }
    if (threadIdx.x < 32) {
      if (threadIdx.x == 0) {
        load_xyzz<C>(s, red);
        load_xyzz<C>(b, buckets + (size_t)f * XW);
      } else {
        xyzz_set_zero<C>(s);
        xyzz_set_zero<C>(b);
      }
      xyzz_add_ni<C>(s, s, b);
      if (threadIdx.x == 0) store_xyzz<C>(buckets + (size_t)f * XW, s);
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------------------
// a5: bucket reduce W_j = sum_{b=1}^{2^(c-1)} b * B_{j,b}.
//   Segment t of window j covers buckets [lo, hi] = [1 + t*seg, min((t+1)*seg, 2^(c-1))]:
//   descending running sum gives run = sum B_b and tri = sum (b - lo + 1) B_b;
//   the segment's contribution is tri + (lo - 1) * run  (small-scalar double-and-add).
// R = k * A by double-and-add over `bits` bits (warp-uniform trip count and call sequence)
template <class C, bool LAT = false>
DEVI void xyzz_mul_small(Xyzz<C>& R, const Xyzz<C>& A, uint32_t k, int bits) {
  xyzz_set_zero<C>(R);
  Xyzz<C> Z;
  for (int b = bits - 1; b >= 0; b--) {
    xyzz_dbl_sel_ni<C, LAT>(R, R);
    xyzz_select<C>(Z, A, (k >> b) & 1u);
    xyzz_add_sel_ni<C, LAT>(R, R, Z);
  }
}

// Segment t of set j covers local buckets [lo, lo + seg), lo = t*seg, of the NB local
// buckets 0..NB-1 (bucket q has weight alpha*q + beta: alpha = 1, beta = 0 without the f1
// split, alpha = G, beta = g with it).  Descending running sums give
//   run = sum_q B_q,   tri = sum_q (q - lo) B_q          (2 PADD per bucket)
// and the segment's share of W_j = sum_q (alpha q + beta) B_q is
//   alpha*tri + (alpha*lo + beta)*run.
// LAT: latency-mode products — chosen when the segments fill less than half a wave (small
// n: a few warps walk the serial chains; ops_impl.cuh)
template <class C, bool LAT = false>
__global__ void __launch_bounds__(SEG_NT, MSM_SEG_SYNC ? 1 : (C::L > 13 ? MSM_SEG_MINB_BIG : MSM_SEG_MINB)) k_bucket_segments(const uint32_t* __restrict__ buckets, const uint32_t* __restrict__ goff,
                                                         int nwin, uint32_t NB, uint32_t seg, uint32_t nseg,
                                                         uint32_t alpha, uint32_t beta,
                                                         uint32_t* __restrict__ out) {
  constexpr int XW = Layout<C>::XW;
  const uint32_t gid = blockIdx.x * blockDim.x + threadIdx.x;
  // MSM_SEG_SYNC: lanes past the last segment stay (as O segments) for the block barriers
  const bool live = gid < (uint32_t)nwin * nseg;
  if (!MSM_SEG_SYNC && !live) return;
  const uint32_t j = live ? gid / nseg : 0u, t = live ? gid % nseg : 0u;
  const uint32_t lo = t * seg;
  Xyzz<C> run, tri, B;
  xyzz_set_zero<C>(run);
  xyzz_set_zero<C>(tri);
  // uniform trip count `seg`; buckets past NB - 1 and empty buckets contribute O
  for (uint32_t q = seg; q-- > 0;) {
    if (MSM_SEG_SYNC) __syncthreads();  // lockstep: shared instruction fetch (see k_accumulate_sync)
    const uint32_t b = lo + q;
    const size_t f = (size_t)j * NB + b;
    // goff == nullptr (chunked host scalars): every bucket was written (zeroed = O first)
    const bool ne = live && b < NB && (goff == nullptr || __ldg(goff + f + 1) != __ldg(goff + f));
    if (ne) load_xyzz<C>(B, buckets + f * XW);
    else xyzz_set_zero<C>(B);
    xyzz_add_hot<C, LAT>(run, run, B);
    if (q > 0) xyzz_add_hot<C, LAT>(tri, tri, run);  // warp-uniform: q is the same in every lane
  }
  if (alpha > 1) {  // warp-uniform
    xyzz_mul_small<C, LAT>(B, tri, alpha, 32 - __clz(alpha));
    tri = B;
  }
  const uint32_t kmax = alpha * (NB - 1) + beta;
  xyzz_mul_small<C, LAT>(B, run, alpha * lo + beta, 32 - __clz(kmax | 1u));
  xyzz_add_sel_ni<C, LAT>(tri, tri, B);
  if (live) store_xyzz<C>(out + (size_t)gid * XW, tri);
}

// out[j*nout + g] = sum of in[j*nin + g*group .. + group)   (per window)
template <class C>
__global__ void __launch_bounds__(128) k_sum_groups(const uint32_t* __restrict__ in, uint32_t nin, uint32_t group,
                                                    uint32_t nout, int nwin, uint32_t* __restrict__ out) {
  constexpr int XW = Layout<C>::XW;
  const uint32_t gid = blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= (uint32_t)nwin * nout) return;
  const uint32_t j = gid / nout, g = gid % nout;
  Xyzz<C> s, b;
  xyzz_set_zero<C>(s);
  for (uint32_t q = 0; q < group; q++) {
    const uint32_t i = g * group + q;
    if (i < nin) load_xyzz<C>(b, in + ((size_t)j * nin + i) * XW);
    else xyzz_set_zero<C>(b);
    xyzz_add_ni<C>(s, s, b);
  }
  store_xyzz<C>(out + (size_t)gid * XW, s);
}

// The same sums with one warp per group (MSM_SUM_WARP, default): lane q loads input q of the
// group and a five-step shuffle tree adds them, so each level of the tree costs 5 serial
// PADDs instead of 32.  Every lane runs every add (lanes past the live half add copies of
// themselves; only lane 0's sum is stored), so the out-of-line PADD is called convergently.
template <class C>
__global__ void __launch_bounds__(128) k_sum_groups_warp(const uint32_t* __restrict__ in, uint32_t nin, uint32_t group,
                                                         uint32_t nout, int nwin, uint32_t* __restrict__ out) {
  constexpr int XW = Layout<C>::XW, L = C::L;
  const uint32_t gid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (gid >= (uint32_t)nwin * nout) return;  // warp-uniform
  const uint32_t j = gid / nout, g = gid % nout;
  Xyzz<C> s, b;
  const uint32_t i = g * group + lane;
  if (lane < group && i < nin) load_xyzz<C>(s, in + ((size_t)j * nin + i) * XW);
  else xyzz_set_zero<C>(s);
#pragma unroll 1
  for (int off = 16; off >= 1; off >>= 1) {
#pragma unroll
    for (int k = 0; k < L; k++) {
      b.X[k] = __shfl_down_sync(0xffffffffu, s.X[k], off);
      b.Y[k] = __shfl_down_sync(0xffffffffu, s.Y[k], off);
      b.ZZ[k] = __shfl_down_sync(0xffffffffu, s.ZZ[k], off);
      b.ZZZ[k] = __shfl_down_sync(0xffffffffu, s.ZZZ[k], off);
    }
    if (lane + off >= 32) xyzz_set_zero<C>(b);
    xyzz_add_ni<C>(s, s, b);
  }
  if (lane == 0) store_xyzz<C>(out + (size_t)gid * XW, s);
}

// ---------------------------------------------------------------------------------------
// a6: window combine Q = sum_j 2^(j c) W_j (Horner), one thread.  Writes the XYZZ partial.
template <class C>
__global__ void k_window_combine(const uint32_t* __restrict__ W, int nwin, int c, uint32_t* __restrict__ partial) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  constexpr int XW = Layout<C>::XW;
  Xyzz<C> Q, B;
  load_xyzz<C>(Q, W + (size_t)(nwin - 1) * XW);
  // single thread: inline latency-mode EC ops (no divergence, so no call hazard)
  for (int j = nwin - 2; j >= 0; j--) {
    for (int s = 0; s < c; s++) {
      Xyzz<C> T = Q;
      xyzz_dbl<C, true>(Q, T);
    }
    load_xyzz<C>(B, W + (size_t)j * XW);
    xyzz_add<C, true>(Q, Q, B);
  }
  store_xyzz<C>(partial, Q);
}

// a7: sum G partial XYZZ points, normalise to canonical affine 32-bit words
template <class C>
__global__ void k_finalize(const uint32_t* __restrict__ partials, int count, uint32_t* __restrict__ result) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  constexpr int XW = Layout<C>::XW;
  Xyzz<C> Q, B;
  xyzz_set_zero<C>(Q);
  for (int g = 0; g < count; g++) {
    load_xyzz<C>(B, partials + (size_t)g * XW);
    xyzz_add<C, true>(Q, Q, B);
  }
  xyzz_to_affine_words<C>(result, result + C::L32, Q);
}

// normalise an array of XYZZ points to affine words (debug: bucket / window sums)
template <class C>
__global__ void k_to_affine(const uint32_t* __restrict__ in, size_t n, uint32_t* __restrict__ out) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  constexpr int XW = Layout<C>::XW;
  Xyzz<C> A;
  load_xyzz<C>(A, in + i * XW);
  xyzz_to_affine_words<C>(out + i * 2 * C::L32, out + i * 2 * C::L32 + C::L32, A);
}

// ---------------------------------------------------------------------------------------
// Synthetic point generator (bench / large tests; not on the MSM path):
//   P_i = (e0 + i*delta) G = E0 + i*D, with E0 = e0 G, D = delta G computed by one thread.
template <class C>
DEVI void xyzz_mul_words(Xyzz<C>& R, const Xyzz<C>& A, const uint32_t* k, int nwords) {
  xyzz_set_zero<C>(R);
  Xyzz<C> Z;
  for (int w = nwords - 1; w >= 0; w--) {
    for (int b = 31; b >= 0; b--) {
      xyzz_dbl_ni<C>(R, R);
      xyzz_select<C>(Z, A, (k[w] >> b) & 1u);
      xyzz_add_ni<C>(R, R, Z);
    }
  }
}

// base: G in canonical affine words; e0w / dw: S words each.  out2: [2] XYZZ (E0, D)
template <class C>
__global__ void k_gen_bases(const uint32_t* __restrict__ gw, const uint32_t* __restrict__ e0w,
                            const uint32_t* __restrict__ dw, uint32_t* __restrict__ out2) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  constexpr int XW = Layout<C>::XW;
  uint32_t x[C::L], y[C::L];
  from_words32<C>(x, gw);
  from_words32<C>(y, gw + C::L32);
  fto_mont<C>(x, x);
  fto_mont<C>(y, y);
  Xyzz<C> G, R;
  xyzz_from_affine<C>(G, x, y);
  uint32_t k[C::S];
  for (int q = 0; q < C::S; q++) k[q] = e0w[q];
  xyzz_mul_words<C>(R, G, k, C::S);
  store_xyzz<C>(out2, R);
  for (int q = 0; q < C::S; q++) k[q] = dw[q];
  xyzz_mul_words<C>(R, G, k, C::S);
  store_xyzz<C>(out2 + XW, R);
}

// uniform-ish scalars in [0, r) for the small-n window-size autotune (engine.cu): hashed
// words, the top word reduced below r's top word
template <class C>
__global__ void k_rand_scalars(uint32_t* __restrict__ out, size_t n, uint32_t seed) {
  const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  for (int q = 0; q < C::S; q++) {
    uint32_t x = (uint32_t)i * 0x9E3779B9u ^ (uint32_t)(i >> 32) * 0xC2B2AE35u ^ (uint32_t)q * 0x85EBCA6Bu ^ seed;
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    out[i * C::S + q] = q == C::S - 1 ? x % C::R32c()[C::S - 1] : x;
  }
}

// thread t generates points [t*chunk, min((t+1)*chunk, n)) as canonical affine words
template <class C>
__global__ void __launch_bounds__(128) k_gen_points(const uint32_t* __restrict__ bases, size_t n, uint32_t chunk,
                                                    uint32_t* __restrict__ out) {
  constexpr int XW = Layout<C>::XW;
  const size_t t = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t i0 = t * chunk;
  if (i0 >= n) return;
  Xyzz<C> E0, D, P, T;
  load_xyzz<C>(E0, bases);
  load_xyzz<C>(D, bases + XW);
  uint32_t kw[2] = {(uint32_t)i0, (uint32_t)(i0 >> 32)};
  xyzz_mul_words<C>(T, D, kw, 2);
  xyzz_add_ni<C>(P, E0, T);
  uint32_t w[2 * C::L32];
  for (uint32_t q = 0; q < chunk; q++) {  // uniform trip count; tail lanes compute and drop
    const size_t i = i0 + q;
    xyzz_to_affine_words<C>(w, w + C::L32, P);
    if (i < n)
      for (int k = 0; k < 2 * C::L32; k++) out[i * 2 * C::L32 + k] = w[k];
    xyzz_add_ni<C>(P, P, D);
  }
}

// ---------------------------------------------------------------------------------------
// debug kernels for the field / EC layers (tests only)
enum { DBG_MUL = 0, DBG_SQR = 1, DBG_ADD = 2, DBG_SUB = 3, DBG_INV = 4, DBG_NEG = 5, DBG_INV_BGCD = 6, DBG_SUM_ABBA = 7,
       DBG_SUM_ABAA = 8 };

template <class C>
__global__ void k_debug_field(int op, const uint32_t* __restrict__ a, const uint32_t* __restrict__ b, size_t n,
                              uint32_t* __restrict__ out) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  constexpr int L = C::L;
  uint32_t x[L], y[L], r[L];
  from_words32<C>(x, a + i * C::L32);
  from_words32<C>(y, b + i * C::L32);
  fto_mont<C>(x, x);
  fto_mont<C>(y, y);
  switch (op) {
    case DBG_MUL: fmul_e<C>(r, x, y); break;
    case DBG_SQR: fsqr_e<C>(r, x); break;
    case DBG_ADD: fadd<C>(r, x, y); break;
    case DBG_SUB: fsub<C, 2>(r, x, y); break;
    case DBG_INV: finv<C>(r, x); break;
    case DBG_INV_BGCD: finv_bgcd<C>(r, x); break;
    case DBG_SUM_ABBA: fmul_sum<C>(r, x, y, y, x); break;  // 2ab (one reduction)
    case DBG_SUM_ABAA: fmul_sum<C>(r, x, y, x, x); break;  // a(b + a)
    default: fneg<C, 2>(r, x); break;
  }
  ffrom_mont<C>(r, r);
  to_words32<C>(out + i * C::L32, r);
}

enum { DBG_EC_ACC = 0, DBG_EC_ADD = 1, DBG_EC_DBL = 2 };

// P, Q affine canonical words (2*L32), (0,0) = O; z1, z2 non-zero scalars (L32 words) used to
// randomise the XYZZ representatives: (x z^2, y z^3, z^2, z^3).
template <class C>
DEVI void debug_xyzz_in(Xyzz<C>& A, const uint32_t* P, const uint32_t* zw) {
  constexpr int L = C::L;
  uint32_t x[L], y[L], z[L], z2[L], z3[L];
  from_words32<C>(x, P);
  from_words32<C>(y, P + C::L32);
  uint32_t nz = 0;
  for (int k = 0; k < 2 * C::L32; k++) nz |= P[k];
  if (!nz) { xyzz_set_zero<C>(A); return; }
  from_words32<C>(z, zw);
  fto_mont<C>(x, x);
  fto_mont<C>(y, y);
  fto_mont<C>(z, z);
  fsqr_e<C>(z2, z);
  fmul_e<C>(z3, z2, z);
  fmul_e<C>(A.X, x, z2);
  fmul_e<C>(A.Y, y, z3);
  fcopy<C>(A.ZZ, z2);
  fcopy<C>(A.ZZZ, z3);
}

template <class C>
__global__ void k_debug_ec(int op, const uint32_t* __restrict__ P, const uint32_t* __restrict__ Q,
                           const uint32_t* __restrict__ z, size_t n, uint32_t* __restrict__ out) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  constexpr int L = C::L;
  const uint32_t* p = P + i * 2 * C::L32;
  const uint32_t* q = Q + i * 2 * C::L32;
  Xyzz<C> A, B, R;
  debug_xyzz_in<C>(A, p, z + i * 2 * C::L32);
  if (op == DBG_EC_ACC) {
    uint32_t x[L], y[L];
    from_words32<C>(x, q);
    from_words32<C>(y, q + C::L32);
    fto_mont<C>(x, x);
    fto_mont<C>(y, y);
    R = A;
    uint32_t nz = 0;
    for (int k = 0; k < 2 * C::L32; k++) nz |= q[k];
    if (nz) xyzz_acc_ni<C>(R, x, y);
  } else if (op == DBG_EC_ADD) {
    debug_xyzz_in<C>(B, q, z + i * 2 * C::L32 + C::L32);
    xyzz_add_ni<C>(R, A, B);
  } else {
    xyzz_dbl_ni<C>(R, A);
  }
  xyzz_to_affine_words<C>(out + i * 2 * C::L32, out + i * 2 * C::L32 + C::L32, R);
}

}  // namespace msmk
