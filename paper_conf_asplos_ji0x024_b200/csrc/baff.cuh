// a4 front end: batch-affine pairwise bucket additions (included by msm_kernels.cuh).
//
// What it computes is PAPER.md §3.2.2's bucket-sum B_b = sum of the points of bucket b
// (P:221), unchanged; how is B200-specific (DESIGN.md §5 "Batch-affine front end").  Two
// affine additions share one field inversion by Montgomery's trick, so an affine addition
// costs 6 multiplications (1 prefix product, 2 inverse updates, lambda, lambda^2, y3) plus
// its share of one Fermat inversion per batch, against 10 for a PACC (Alg. 4).
//
// Status: ablation, off by default (MSM_OPT_ACC_MODE = 1 selects it).  Bit-exact, but on
// B200 it ran at 8.2 G field mults/s against PACC's 22.3 (BLS12-381 2^26: front end 503 ms
// for 3/4 of the additions, vs 327 ms for all of them with PACC): the affine glue per
// addition (two equality tests, three reductions to [0, 2p), scratch round trips) costs as
// many instructions as the multiplications it saves, and the per-batch Fermat inversion is a
// serial chain (ncu: profiles/r02/baff_ncu_summary.txt).
//
// k_baff2 folds every group of 4 consecutive entries of a bucket into one affine point in
// two pairwise levels (4 -> 2 -> 1), each level one batch over the thread's outputs with a
// single inversion; the quarter-size result is then accumulated by the PACC kernel as
// before (k_accumulate_sync<DIRECT>).  Bucket f with c_f entries becomes ceil(c_f / 4)
// points at goff4[f] (exclusive scan of the ceil(c_f / 4)).
//
// Affine pair (P1, P2) -> P1 + P2 (formulas from the group law, Formula (1) P:90):
//   x1 != x2:            lambda = (y2 - y1) / (x2 - x1)
//   x1 == x2, y1 == y2:  lambda = (3 x1^2 + a) / (2 y1)                   (doubling)
//   x1 == x2, y1 != y2:  O                    (denominator replaced by 1)
//   P1 or P2 = O:        the other point      (denominator replaced by 1)
//   x3 = lambda^2 - x1 - x2,   y3 = lambda (x1 - x3) - y1.
// O is stored as (0, 0); a stored point with y = 0 is O (y = 0 points are rejected at
// context creation).  Bounds (lazy, multiples of p): inputs x, y < 2p; outputs reduced to
// [0, 2p) so the PACC kernel sees the same bounds as for table points.
#pragma once

// r = a^(p-2) = a^-1 (Montgomery form; a != 0), Fermat with throughput-mode products.
// Called once per batch from warp-uniform control flow (every lane runs every batch loop).
template <class C>
__device__ __noinline__ void finv_thr(uint32_t* r, const uint32_t* a) {
  uint32_t acc[C::L], b[C::L];
  fcopy<C>(b, a);
  fset_one<C>(acc);
  for (int wi = C::L32 - 1; wi >= 0; wi--) {
    const uint32_t e = C::PM2c()[wi];
    for (int bit = 31; bit >= 0; bit--) {
      fsqr<C>(acc, acc);
      if ((e >> bit) & 1u) fmul<C>(acc, acc, b);  // exponent bits: uniform across lanes
    }
  }
  fcopy<C>(r, acc);
}

constexpr int BAFF_NT = 128;

enum { PAIR_ADD = 0, PAIR_DBL = 1, PAIR_COPY1 = 2, PAIR_COPY2 = 3, PAIR_O = 4 };

// Classifies (P1, P2) and returns the denominator of lambda (1 when no field division is
// needed).  ok1/ok2: P1/P2 are not O.
template <class C>
DEVI int pair_den(uint32_t* den, const uint32_t* x1, const uint32_t* y1, bool ok1, const uint32_t* x2,
                  const uint32_t* y2, bool ok2) {
  int mode;
  if (!ok1 && !ok2) mode = PAIR_O;
  else if (!ok1) mode = PAIR_COPY2;
  else if (!ok2) mode = PAIR_COPY1;
  else if (fequal<C, 2>(x1, x2)) mode = fequal<C, 2>(y1, y2) ? PAIR_DBL : PAIR_O;
  else mode = PAIR_ADD;
  if (mode == PAIR_ADD) fsub<C, 2>(den, x2, x1);        // < 4p
  else if (mode == PAIR_DBL) fadd<C>(den, y1, y1);       // < 4p
  else fset_one<C>(den);
  return mode;
}

// Two pairs at once: (x3, y3)_q = P1_q + P2_q given inv_q = 1/den_q (mode_q from pair_den),
// q = a, b, with every product issued as a column-interleaved pair (fmul2).  Outputs are
// reduced to [0, 2p); O -> (0, 0).  x3/y3 may alias x1/y1 of the same pair.
template <class C>
DEVI void pair_num(uint32_t* num, int mode, const uint32_t* x1, const uint32_t* y1, const uint32_t* y2) {
  if (mode == PAIR_DBL) {            // rare: 3 x1^2 + a
    uint32_t t[C::L];
    fsqr<C>(t, x1);                  // < 2p
    fadd<C>(num, t, t);
    fadd<C>(num, num, t);            // < 6p
    if constexpr (!C::A_ZERO) {
      uint32_t a[C::L];
#pragma unroll
      for (int i = 0; i < C::L; i++) a[i] = C::A_M(i);
      fadd<C>(num, num, a);          // < 7p
    }
  } else {
    fsub<C, 2>(num, y2, y1);         // < 4p
  }
}

template <class C>
DEVI void pair_select(uint32_t* x3, uint32_t* y3, int mode, const uint32_t* xs, const uint32_t* ys, const uint32_t* x1,
                      const uint32_t* y1, const uint32_t* x2, const uint32_t* y2) {
  if (mode == PAIR_ADD || mode == PAIR_DBL) {
    fcopy<C>(x3, xs);
    fcopy<C>(y3, ys);
  } else if (mode == PAIR_COPY1) {
    fcopy<C>(x3, x1);
    fcopy<C>(y3, y1);
  } else if (mode == PAIR_COPY2) {
    fcopy<C>(x3, x2);
    fcopy<C>(y3, y2);
  } else {
    fzero<C>(x3);
    fzero<C>(y3);
  }
}

template <class C>
DEVI void pair_finish2(uint32_t* xa3, uint32_t* ya3, int ma, const uint32_t* inva, const uint32_t* xa1, const uint32_t* ya1,
                       const uint32_t* xa2, const uint32_t* ya2, uint32_t* xb3, uint32_t* yb3, int mb,
                       const uint32_t* invb, const uint32_t* xb1, const uint32_t* yb1, const uint32_t* xb2,
                       const uint32_t* yb2) {
  constexpr int L = C::L;
  uint32_t na[L], nb[L], la[L], lb[L], ta[L], tb[L];
  pair_num<C>(na, ma, xa1, ya1, ya2);
  pair_num<C>(nb, mb, xb1, yb1, yb2);
  fmul2<C>(la, na, inva, lb, nb, invb);           // lambda < 2p
  fmul2<C, true>(ta, la, la, tb, lb, lb);         // lambda^2 < 2p
  fadd<C>(na, xa1, xa2);
  fadd<C>(nb, xb1, xb2);                          // < 4p
  fsub<C, 4>(ta, ta, na);
  fsub<C, 4>(tb, tb, nb);                         // x3 < 6p
  fcsub<C, 4>(ta); fcsub<C, 2>(ta);
  fcsub<C, 4>(tb); fcsub<C, 2>(tb);               // x3 < 2p
  fsub<C, 2>(na, xa1, ta);
  fsub<C, 2>(nb, xb1, tb);                        // x1 - x3 < 4p
  fmul2<C>(la, la, na, lb, lb, nb);               // < 2p
  fsub<C, 2>(na, la, ya1);
  fsub<C, 2>(nb, lb, yb1);                        // y3 < 4p
  fcsub<C, 2>(na);
  fcsub<C, 2>(nb);                                // y3 < 2p
  pair_select<C>(xa3, ya3, ma, ta, na, xa1, ya1, xa2, ya2);
  pair_select<C>(xb3, yb3, mb, tb, nb, xb1, yb1, xb2, yb2);
}

// c4[f] = ceil((goff[f+1] - goff[f]) / 4)
static __global__ void k_group4_counts(const uint32_t* __restrict__ goff, size_t F, uint32_t* __restrict__ c4) {
  const size_t f = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (f < F) c4[f] = (goff[f + 1] - goff[f] + 3u) >> 2;
}

// Scratch of thread t (T threads): word w of slot j at ((j * width + w) * T + t), so the
// lanes of a warp touch consecutive words (coalesced).
struct BaffScratch {
  uint32_t* base;
  uint32_t T;
  DEVI uint32_t* at(size_t region, uint32_t j, int width, int w, uint32_t t) const {
    return base + region + ((size_t)j * width + w) * T + t;
  }
};

template <class C>
DEVI void sc_store(const BaffScratch& s, size_t region, uint32_t j, int width, int off, uint32_t t, const uint32_t* v) {
#pragma unroll
  for (int w = 0; w < C::L; w++) *s.at(region, j, width, off + w, t) = v[w];
}
template <class C>
DEVI void sc_load(const BaffScratch& s, size_t region, uint32_t j, int width, int off, uint32_t t, uint32_t* v) {
#pragma unroll
  for (int w = 0; w < C::L; w++) v[w] = *s.at(region, j, width, off + w, t);
}

template <class C>
DEVI void store_affine(uint32_t* __restrict__ dst, const uint32_t* x, const uint32_t* y) {
  constexpr int L = C::L, PW = Layout<C>::PW;
  uint32_t rec[PW];
#pragma unroll
  for (int w = 0; w < PW; w++) rec[w] = 0;
#pragma unroll
  for (int w = 0; w < L; w++) { rec[w] = x[w]; rec[L + w] = y[w]; }
  uint4* d4 = reinterpret_cast<uint4*>(dst);
#pragma unroll
  for (int q = 0; q < PW / 4; q++) d4[q] = make_uint4(rec[4 * q], rec[4 * q + 1], rec[4 * q + 2], rec[4 * q + 3]);
}

// Gathers the stored point of sorted entry `ent` (index | sign << 31): y negated for a
// negative digit; returns false for O.
template <class C>
DEVI bool baff_gather(uint32_t* x, uint32_t* y, const uint32_t* __restrict__ pts, uint32_t ent) {
  load_point<C>(x, y, pts, ent & 0x7FFFFFFFu);
  if (fis_zero<C, 2>(y)) return false;
  if (ent & 0x80000000u) fneg<C, 2>(y, y);
  return true;
}

// Level-1 pair s (0/1) of group (g0, k): entries g0+2s, g0+2s+1 of `sorted`; absent
// entries are O.
template <class C>
DEVI void baff_level1_pair(uint32_t* x1, uint32_t* y1, bool& ok1, uint32_t* x2, uint32_t* y2, bool& ok2,
                           const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted, uint32_t g0, uint32_t k,
                           int s) {
  const uint32_t a = 2u * s;
  ok1 = a < k ? baff_gather<C>(x1, y1, pts, __ldg(sorted + g0 + a)) : false;
  ok2 = a + 1 < k ? baff_gather<C>(x2, y2, pts, __ldg(sorted + g0 + a + 1)) : false;
  if (!ok1) { fzero<C>(x1); fzero<C>(y1); }
  if (!ok2) { fzero<C>(x2); fzero<C>(y2); }
}

// L2 prefetch of the (<= 4) stored points of group (g0, k)
template <class C>
DEVI void baff_prefetch_group(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted, uint32_t g0,
                              uint32_t k) {
  for (uint32_t a = 0; a < k; a++) {
    const char* p = reinterpret_cast<const char*>(pts + (size_t)(__ldg(sorted + g0 + a) & 0x7FFFFFFFu) * Layout<C>::PW);
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p + Layout<C>::PW * 4 - 4));
  }
}

// group (g0, k) of output o walking buckets from f (goff4 non-decreasing)
DEVI void baff_group(const uint32_t* __restrict__ goff, const uint32_t* __restrict__ goff4, uint32_t& f, uint32_t o,
                     uint32_t& g0, uint32_t& k) {
  while (__ldg(goff4 + f + 1) <= o) f++;
  const uint32_t b0 = __ldg(goff + f);
  const uint32_t c = __ldg(goff + f + 1) - b0;
  const uint32_t i4 = 4u * (o - __ldg(goff4 + f));
  g0 = b0 + i4;
  k = min(4u, c - i4);
}

// Folds groups of 4 entries per bucket into one affine point each (out: [M4][PW], M4 =
// goff4[F]).  Persistent grid of T threads; thread t handles batches t, t+T, ... of B
// consecutive outputs, as two independent chains (outputs [0, B/2) and [B/2, B) of the
// batch) so that every product is issued in a column-interleaved pair (fmul2) — one
// inversion per batch and level covers both chains.  Every thread runs the same number of
// batch iterations (idle ones on empty batches), so the out-of-line inversion is called
// convergently.
template <class C>
__global__ void __launch_bounds__(BAFF_NT, 1) k_baff2(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sorted,
                                                      const uint32_t* __restrict__ goff, const uint32_t* __restrict__ goff4,
                                                      uint32_t F, uint32_t B, uint32_t* __restrict__ out,
                                                      uint32_t* __restrict__ scratch) {
  constexpr int L = C::L, PW = Layout<C>::PW;
  const uint32_t T = gridDim.x * blockDim.x;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  const BaffScratch sc{scratch, T};
  // regions (words per thread-slot): pre1 [2B][L], r1 [2B][2L], pre2 [B][L], meta [B][2]
  const size_t R_PRE1 = 0, R_R1 = (size_t)2 * B * L * T, R_PRE2 = R_R1 + (size_t)2 * B * 2 * L * T,
               R_META = R_PRE2 + (size_t)B * L * T;
  const uint32_t H = B / 2;
  const uint32_t M4 = __ldg(goff4 + F);
  const uint32_t nbatch = (M4 + B - 1) / B;
  const uint32_t iters = (nbatch + T - 1) / T;
  for (uint32_t it = 0; it < iters; it++) {
    const uint32_t batch = t + it * T;
    const uint32_t o0 = batch * B;
    const uint32_t nout = o0 < M4 ? min(B, M4 - o0) : 0u;
    const uint32_t nA = min(nout, H), nB = nout > H ? nout - H : 0u;  // chain a: [0, nA), chain b: [H, H + nB)
    uint32_t accA[L], accB[L], denA[L], denB[L];
    uint32_t xa1[L], ya1[L], xa2[L], ya2[L], xb1[L], yb1[L], xb2[L], yb2[L];
    // ---- level 1 forward: groups of each output, den of its two pairs, prefix products
    fset_one<C>(accA);
    fset_one<C>(accB);
    uint32_t fa = 0, fb = 0, ga = 0, ka = 0, gb = 0, kb = 0;
    if (nA) {
      fa = find_bucket(goff4, F, o0);
      baff_group(goff, goff4, fa, o0, ga, ka);
    }
    if (nB) {
      fb = find_bucket(goff4, F, o0 + H);
      baff_group(goff, goff4, fb, o0 + H, gb, kb);
    }
    for (uint32_t j = 0; j < nA; j++) {
      const bool hb = j < nB;
      *sc.at(R_META, j, 2, 0, t) = ga;
      *sc.at(R_META, j, 2, 1, t) = ka;
      if (hb) {
        *sc.at(R_META, H + j, 2, 0, t) = gb;
        *sc.at(R_META, H + j, 2, 1, t) = kb;
      }
      // groups of the next outputs, and their points into L2 while this one computes
      uint32_t gan = 0, kan = 0, gbn = 0, kbn = 0;
      if (j + 1 < nA) { baff_group(goff, goff4, fa, o0 + j + 1, gan, kan); baff_prefetch_group<C>(pts, sorted, gan, kan); }
      if (j + 1 < nB) { baff_group(goff, goff4, fb, o0 + H + j + 1, gbn, kbn); baff_prefetch_group<C>(pts, sorted, gbn, kbn); }
#pragma unroll 1
      for (int s = 0; s < 2; s++) {
        bool a1, a2, b1, b2;
        baff_level1_pair<C>(xa1, ya1, a1, xa2, ya2, a2, pts, sorted, ga, ka, s);
        baff_level1_pair<C>(xb1, yb1, b1, xb2, yb2, b2, pts, sorted, gb, hb ? kb : 0u, s);
        pair_den<C>(denA, xa1, ya1, a1, xa2, ya2, a2);
        pair_den<C>(denB, xb1, yb1, b1, xb2, yb2, b2);
        sc_store<C>(sc, R_PRE1, 2 * j + s, L, 0, t, accA);
        sc_store<C>(sc, R_PRE1, 2 * (H + j) + s, L, 0, t, accB);
        fmul2<C>(accA, accA, denA, accB, accB, denB);
      }
      ga = gan; ka = kan; gb = gbn; kb = kbn;
    }
    uint32_t invA[L], invB[L], pa[L], pb[L];
    fmul<C>(pa, accA, accB);
    finv_thr<C>(pb, pa);                       // 1 / (accA accB)
    fmul2<C>(invA, pb, accB, invB, pb, accA);  // 1 / accA, 1 / accB
    // ---- level 1 backward: results into r1
    for (uint32_t j = nA; j-- > 0;) {
      const bool hb = j < nB;
      const uint32_t ga_ = *sc.at(R_META, j, 2, 0, t), ka_ = *sc.at(R_META, j, 2, 1, t);
      const uint32_t gb_ = hb ? *sc.at(R_META, H + j, 2, 0, t) : 0u, kb_ = hb ? *sc.at(R_META, H + j, 2, 1, t) : 0u;
      if (j > 0) {
        baff_prefetch_group<C>(pts, sorted, *sc.at(R_META, j - 1, 2, 0, t), *sc.at(R_META, j - 1, 2, 1, t));
        if (j - 1 < nB) baff_prefetch_group<C>(pts, sorted, *sc.at(R_META, H + j - 1, 2, 0, t), *sc.at(R_META, H + j - 1, 2, 1, t));
      }
#pragma unroll 1
      for (int s = 1; s >= 0; s--) {
        bool a1, a2, b1, b2;
        baff_level1_pair<C>(xa1, ya1, a1, xa2, ya2, a2, pts, sorted, ga_, ka_, s);
        baff_level1_pair<C>(xb1, yb1, b1, xb2, yb2, b2, pts, sorted, gb_, kb_, s);
        const int ma = pair_den<C>(denA, xa1, ya1, a1, xa2, ya2, a2);
        const int mb = pair_den<C>(denB, xb1, yb1, b1, xb2, yb2, b2);
        uint32_t ia[L], ib[L];
        sc_load<C>(sc, R_PRE1, 2 * j + s, L, 0, t, pa);
        sc_load<C>(sc, R_PRE1, 2 * (H + j) + s, L, 0, t, pb);
        fmul2<C>(ia, invA, pa, ib, invB, pb);
        fmul2<C>(invA, invA, denA, invB, invB, denB);
        pair_finish2<C>(xa1, ya1, ma, ia, xa1, ya1, xa2, ya2, xb1, yb1, mb, ib, xb1, yb1, xb2, yb2);
        sc_store<C>(sc, R_R1, 2 * j + s, 2 * L, 0, t, xa1);
        sc_store<C>(sc, R_R1, 2 * j + s, 2 * L, L, t, ya1);
        if (hb) {
          sc_store<C>(sc, R_R1, 2 * (H + j) + s, 2 * L, 0, t, xb1);
          sc_store<C>(sc, R_R1, 2 * (H + j) + s, 2 * L, L, t, yb1);
        }
      }
    }
    // ---- level 2 forward
    fset_one<C>(accA);
    fset_one<C>(accB);
    for (uint32_t j = 0; j < nA; j++) {
      const bool hb = j < nB;
      sc_load<C>(sc, R_R1, 2 * j, 2 * L, 0, t, xa1);
      sc_load<C>(sc, R_R1, 2 * j, 2 * L, L, t, ya1);
      sc_load<C>(sc, R_R1, 2 * j + 1, 2 * L, 0, t, xa2);
      sc_load<C>(sc, R_R1, 2 * j + 1, 2 * L, L, t, ya2);
      if (hb) {
        sc_load<C>(sc, R_R1, 2 * (H + j), 2 * L, 0, t, xb1);
        sc_load<C>(sc, R_R1, 2 * (H + j), 2 * L, L, t, yb1);
        sc_load<C>(sc, R_R1, 2 * (H + j) + 1, 2 * L, 0, t, xb2);
        sc_load<C>(sc, R_R1, 2 * (H + j) + 1, 2 * L, L, t, yb2);
      }
      pair_den<C>(denA, xa1, ya1, !fis_zero<C, 2>(ya1), xa2, ya2, !fis_zero<C, 2>(ya2));
      pair_den<C>(denB, xb1, yb1, hb && !fis_zero<C, 2>(yb1), xb2, yb2, hb && !fis_zero<C, 2>(yb2));
      sc_store<C>(sc, R_PRE2, j, L, 0, t, accA);
      sc_store<C>(sc, R_PRE2, H + j, L, 0, t, accB);
      fmul2<C>(accA, accA, denA, accB, accB, denB);
    }
    fmul<C>(pa, accA, accB);
    finv_thr<C>(pb, pa);
    fmul2<C>(invA, pb, accB, invB, pb, accA);
    // ---- level 2 backward: results to out
    for (uint32_t j = nA; j-- > 0;) {
      const bool hb = j < nB;
      sc_load<C>(sc, R_R1, 2 * j, 2 * L, 0, t, xa1);
      sc_load<C>(sc, R_R1, 2 * j, 2 * L, L, t, ya1);
      sc_load<C>(sc, R_R1, 2 * j + 1, 2 * L, 0, t, xa2);
      sc_load<C>(sc, R_R1, 2 * j + 1, 2 * L, L, t, ya2);
      if (hb) {
        sc_load<C>(sc, R_R1, 2 * (H + j), 2 * L, 0, t, xb1);
        sc_load<C>(sc, R_R1, 2 * (H + j), 2 * L, L, t, yb1);
        sc_load<C>(sc, R_R1, 2 * (H + j) + 1, 2 * L, 0, t, xb2);
        sc_load<C>(sc, R_R1, 2 * (H + j) + 1, 2 * L, L, t, yb2);
      }
      const int ma = pair_den<C>(denA, xa1, ya1, !fis_zero<C, 2>(ya1), xa2, ya2, !fis_zero<C, 2>(ya2));
      const int mb = pair_den<C>(denB, xb1, yb1, hb && !fis_zero<C, 2>(yb1), xb2, yb2, hb && !fis_zero<C, 2>(yb2));
      uint32_t ia[L], ib[L];
      sc_load<C>(sc, R_PRE2, j, L, 0, t, pa);
      sc_load<C>(sc, R_PRE2, H + j, L, 0, t, pb);
      fmul2<C>(ia, invA, pa, ib, invB, pb);
      fmul2<C>(invA, invA, denA, invB, invB, denB);
      pair_finish2<C>(xa1, ya1, ma, ia, xa1, ya1, xa2, ya2, xb1, yb1, mb, ib, xb1, yb1, xb2, yb2);
      store_affine<C>(out + (size_t)(o0 + j) * PW, xa1, ya1);
      if (hb) store_affine<C>(out + (size_t)(o0 + H + j) * PW, xb1, yb1);
    }
  }
}
