// a3, three-level staged counting sort (§3.2.1, Alg. 3).
// Included inside namespace msmk by msm_kernels.cuh.
//
// The paper's bucket scatter ranks points per bucket in shared memory and reserves one
// global range per (block, bucket) with one atomic (Alg. 3 lines 12-15), which
// stops at s = 14 on A100 shared memory.  With c up to 24 a bucket set has up to
// 2^23 buckets, so on B200 the scatter is split into three passes over a flat key
// f = j*ws + b (the entry's flat bucket), each pass writing only long coalesced runs:
//   P1  k_s3_part1   scalars -> (key, value) partitioned by the top b1 key bits: per tile
//                    of E_T entries, shared-memory ranks, one global atomic per (tile, bin),
//                    entries staged in shared memory in bin order and written as runs;
//   P2  k_s3_count2 + scan + k_s3_part2: the P1 output, in tiles that never straddle a
//                    P1 bin, partitioned by the next b2 bits the same way (sub-bin starts
//                    from a global scan of the per-(bin, sub-bin) counts);
//   P3  k_s3_part3   one block per sub-bin (2^b3 buckets, ~4-8K entries): a complete
//                    counting sort in shared memory, written contiguously, plus goff.
// The (i, j) entry value is (i + j*istride) | sign<<31 as in the other sort variants (i
// offset by ibase when the scalars arrive in chunks: engine.cu, chunked host H2D).
// Why: the two-level binned sort (k_bin_scatter) wrote 6-B entries at random positions
// of 8K bins; ncu measured 28.7 GB DRAM writes for 4.4 GB of entries at 2^26 (partial
// sectors evicted before they fill) -- 31 ms of a 40 ms sort.

constexpr int S3_THREADS = 512;
constexpr int S3_TILE = 12288;       // staged entries per tile (96 KB of keys + values)
constexpr int S3_CAP = 12288;        // largest sub-bin P3 sorts in shared memory
constexpr int S3_MAXB = 512;         // max bins per partition pass (b1, b2 <= 9)
constexpr int S3_MAXFINE = 4096;     // max buckets per sub-bin (b3 <= 12)

// Entry loops over [e0, e1) with stride blockDim.x, S3_U loads in flight per thread: the
// P2/P3 passes were global-load-latency bound (ncu: long_scoreboard ~35-49 stalls per
// issue, 14-17 % issue) with one key load outstanding per thread.
constexpr int S3_U = 8;
template <class KT, class F>
__device__ __forceinline__ void s3_for_keys(const KT* __restrict__ keys, uint32_t e0, uint32_t e1, F&& f) {
  for (uint32_t eb = e0 + threadIdx.x; eb < e1; eb += S3_U * blockDim.x) {
    uint32_t k[S3_U];
#pragma unroll
    for (int u = 0; u < S3_U; u++) {
      const uint32_t e = eb + u * blockDim.x;
      k[u] = e < e1 ? (uint32_t)__ldg(keys + e) : 0u;
    }
#pragma unroll
    for (int u = 0; u < S3_U; u++)
      if (eb + u * blockDim.x < e1) f(k[u]);
  }
}
template <class KT, class F>
__device__ __forceinline__ void s3_for_entries(const KT* __restrict__ keys, const uint32_t* __restrict__ vals,
                                               uint32_t e0, uint32_t e1, F&& f) {
  for (uint32_t eb = e0 + threadIdx.x; eb < e1; eb += S3_U * blockDim.x) {
    uint32_t k[S3_U], v[S3_U];
#pragma unroll
    for (int u = 0; u < S3_U; u++) {
      const uint32_t e = eb + u * blockDim.x;
      k[u] = e < e1 ? (uint32_t)__ldg(keys + e) : 0u;
      v[u] = e < e1 ? __ldg(vals + e) : 0u;
    }
#pragma unroll
    for (int u = 0; u < S3_U; u++)
      if (eb + u * blockDim.x < e1) f(k[u], v[u]);
  }
}

// exclusive scan of cnt[0..N) in place (N <= blockDim.x * per-thread chunk); returns total
__device__ __forceinline__ uint32_t s3_block_scan(uint32_t* cnt, uint32_t N, uint32_t* warp_sums) {
  const uint32_t per = (N + blockDim.x - 1) / blockDim.x;
  const uint32_t c0 = min(threadIdx.x * per, N), c1 = min(c0 + per, N);
  uint32_t sum = 0;
  for (uint32_t i = c0; i < c1; i++) sum += cnt[i];
  uint32_t total;
  uint32_t run = block_exclusive_scan(sum, warp_sums, &total);
  for (uint32_t i = c0; i < c1; i++) {
    const uint32_t v = cnt[i];
    cnt[i] = run;
    run += v;
  }
  __syncthreads();
  return total;
}

// P1 histogram: binCount[f >> sh1] over all digits (tiles of BIN_TILE points); err |= 4
// for k >= r
template <class C>
__global__ void __launch_bounds__(S3_THREADS) k_s3_count1(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                                                          uint32_t ws, int sh1, uint32_t NC1,
                                                          uint32_t* __restrict__ binCount, uint32_t* err) {
  __shared__ uint32_t hist[S3_MAXB];
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const size_t base = (size_t)blockIdx.x * (S3_THREADS * 16);
  bool bad = false;
  for (int q = 0; q < 16; q++) {
    const size_t i = base + (size_t)q * S3_THREADS + threadIdx.x;
    if (i >= n) break;
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) { bad = true; continue; }
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool) { atomicAdd(hist + ((j * ws + b) >> sh1), 1u); });
  }
  if (bad) atomicOr(err, 4u);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x)
    if (hist[i]) atomicAdd(binCount + i, hist[i]);
}

// P1: tile = tp points (tp * nwin <= S3_TILE entries)
// KT: P1 keys leave as the flat key's low sh1 bits (the bin is the position), u16 when
// sh1 <= 16 (round 2: 6 instead of 8 bytes per entry through P2)
template <class C, class KT>
__global__ void __launch_bounds__(S3_THREADS) k_s3_part1(const uint32_t* __restrict__ scal, size_t n, int c, int nwin,
                                                         uint32_t ws, uint32_t istride, int sh1, uint32_t NC1, uint32_t tp,
                                                         uint32_t* __restrict__ binCursor,
                                                         KT* __restrict__ keys, uint32_t* __restrict__ vals,
                                                         uint32_t ibase = 0) {
  extern __shared__ uint32_t sm[];
  uint32_t* skey = sm;                 // [S3_TILE]
  uint32_t* sval = sm + S3_TILE;       // [S3_TILE]
  __shared__ uint32_t loc[S3_MAXB], cur[S3_MAXB], gbase[S3_MAXB], warp_sums[32];
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) cur[i] = 0;
  __syncthreads();
  const size_t p0 = (size_t)blockIdx.x * tp;
  const size_t p1 = min(p0 + tp, n);
  for (size_t i = p0 + threadIdx.x; i < p1; i += blockDim.x) {
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) continue;
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool) { atomicAdd(cur + ((j * ws + b) >> sh1), 1u); });
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) {
    const uint32_t h = cur[i];
    gbase[i] = h ? atomicAdd(binCursor + i, h) : 0u;
    loc[i] = h;
  }
  __syncthreads();
  const uint32_t E = s3_block_scan(loc, NC1, warp_sums);
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) cur[i] = loc[i];
  __syncthreads();
  for (size_t i = p0 + threadIdx.x; i < p1; i += blockDim.x) {
    ScalarReg<C> k;
    load_scalar<C>(k, scal, i);
    if (!scalar_in_range<C>(k)) continue;
    for_each_digit<C>(k, c, nwin, [&](int j, uint32_t b, bool neg) {
      const uint32_t f = j * ws + b;
      const uint32_t pos = atomicAdd(cur + (f >> sh1), 1u);
      skey[pos] = f;
      sval[pos] = ((uint32_t)i + ibase + (uint32_t)j * istride) | (neg ? SIGN_BIT : 0u);
    });
  }
  __syncthreads();
  const uint32_t lowmask = sh1 >= 32 ? ~0u : (1u << sh1) - 1u;
  for (uint32_t p = threadIdx.x; p < E; p += blockDim.x) {
    const uint32_t f = skey[p], bin = f >> sh1;
    const uint32_t o = gbase[bin] + (p - loc[bin]);
    keys[o] = (KT)(f & lowmask);
    vals[o] = sval[p];
  }
}

// P2 work is cut into tiles of <= S3_TILE entries that never straddle a P1 bin, so heavy
// bins (skewed scalars; with the f3 table the top window's small digits all land in the
// lowest buckets) spread over many blocks.  tileStart[b] = first tile of P1 bin b.
static __global__ void k_s3_tiles(const uint32_t* __restrict__ binOff, uint32_t NC1, uint32_t* __restrict__ tileStart) {
  __shared__ uint32_t cnt[S3_MAXB], warp_sums[32];
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x)
    cnt[i] = (binOff[i + 1] - binOff[i] + S3_TILE - 1) / S3_TILE;
  __syncthreads();
  const uint32_t total = s3_block_scan(cnt, NC1, warp_sums);
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) tileStart[i] = cnt[i];
  if (threadIdx.x == 0) tileStart[NC1] = total;
}

// tile t -> its P1 bin and entry range; false past the last tile
__device__ __forceinline__ bool s3_tile(const uint32_t* __restrict__ tileStart, const uint32_t* __restrict__ binOff,
                                        uint32_t NC1, uint32_t t, uint32_t& bin, uint32_t& e0, uint32_t& e1) {
  if (t >= tileStart[NC1]) return false;
  uint32_t lo = 0, hi = NC1;  // largest bin with tileStart[bin] <= t (tileStart non-decreasing)
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (tileStart[mid] <= t) lo = mid; else hi = mid;
  }
  while (lo + 1 < NC1 && tileStart[lo + 1] <= t) lo++;  // skip empty bins sharing the start
  bin = lo;
  e0 = binOff[bin] + (t - tileStart[bin]) * S3_TILE;
  e1 = min(e0 + S3_TILE, binOff[bin + 1]);
  return true;
}

// P2 histogram: subCount[bin*NC2 + s] for s = (f >> sh2) & (NC2 - 1)
template <class KT>
__global__ void __launch_bounds__(S3_THREADS) k_s3_count2(const uint32_t* __restrict__ tileStart,
                                                          const uint32_t* __restrict__ binOff, uint32_t NC1,
                                                          int sh2, uint32_t NC2, const KT* __restrict__ keys,
                                                          uint32_t* __restrict__ subCount) {
  __shared__ uint32_t hist[S3_MAXB];
  uint32_t bin, e0, e1;
  if (!s3_tile(tileStart, binOff, NC1, blockIdx.x, bin, e0, e1)) return;
  const uint32_t mask = NC2 - 1;
  for (uint32_t i = threadIdx.x; i < NC2; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  s3_for_keys(keys, e0, e1, [&](uint32_t f) { atomicAdd(hist + ((f >> sh2) & mask), 1u); });
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < NC2; i += blockDim.x)
    if (hist[i]) atomicAdd(subCount + (size_t)bin * NC2 + i, hist[i]);
}

// P2 scatter: per tile, shared-memory ranks by sub-bin, one global atomic per (tile,
// sub-bin) on subCursor (initialised to the global sub-bin starts), staged coalesced runs.
// P2 keys leave as the low sh2 = b3 bits (u16; b3 <= 12)
template <class KT>
__global__ void __launch_bounds__(S3_THREADS) k_s3_part2(const uint32_t* __restrict__ tileStart,
                                                         const uint32_t* __restrict__ binOff, uint32_t NC1,
                                                         int sh2, uint32_t NC2,
                                                         const KT* __restrict__ keys, const uint32_t* __restrict__ vals,
                                                         uint32_t* __restrict__ subCursor,
                                                         uint16_t* __restrict__ keys2, uint32_t* __restrict__ vals2) {
  extern __shared__ uint32_t sm[];
  uint32_t* skey = sm;
  uint32_t* sval = sm + S3_TILE;
  __shared__ uint32_t loc[S3_MAXB], cur[S3_MAXB], gbase[S3_MAXB], warp_sums[32];
  uint32_t bin, e0, e1;
  if (!s3_tile(tileStart, binOff, NC1, blockIdx.x, bin, e0, e1)) return;
  const uint32_t mask = NC2 - 1;
  for (uint32_t i = threadIdx.x; i < NC2; i += blockDim.x) cur[i] = 0;
  __syncthreads();
  s3_for_keys(keys, e0, e1, [&](uint32_t f) { atomicAdd(cur + ((f >> sh2) & mask), 1u); });
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < NC2; i += blockDim.x) {
    const uint32_t h = cur[i];
    gbase[i] = h ? atomicAdd(subCursor + (size_t)bin * NC2 + i, h) : 0u;
    loc[i] = h;
  }
  __syncthreads();
  const uint32_t E = s3_block_scan(loc, NC2, warp_sums);
  for (uint32_t i = threadIdx.x; i < NC2; i += blockDim.x) cur[i] = loc[i];
  __syncthreads();
  s3_for_entries(keys, vals, e0, e1, [&](uint32_t f, uint32_t v) {
    const uint32_t pos = atomicAdd(cur + ((f >> sh2) & mask), 1u);
    skey[pos] = f;
    sval[pos] = v;
  });
  __syncthreads();
  const uint32_t lowmask = (1u << sh2) - 1u;
  for (uint32_t p = threadIdx.x; p < E; p += blockDim.x) {
    const uint32_t f = skey[p], sb = (f >> sh2) & mask;
    const uint32_t o = gbase[sb] + (p - loc[sb]);
    keys2[o] = (uint16_t)(f & lowmask);
    vals2[o] = sval[p];
  }
}

// P3: block = sub-bin q covering buckets [q << b3, (q+1) << b3) of [subOff[q], end_q);
// writes goff for its buckets (< F) and the final values in bucket order.
// Oversized sub-bins (> S3_CAP entries: skewed scalars, or a top window of lambda mod c
// bits piling n entries into a few buckets) leave their scatter to k_s3_big: P3 writes their
// bucket starts into gcur and lists them in big[1..big[0]].
static __global__ void __launch_bounds__(256) k_s3_part3(const uint32_t* __restrict__ subOff, int b3, uint32_t F,
                                                         const uint16_t* __restrict__ keys2, const uint32_t* __restrict__ vals2,
                                                         uint32_t* __restrict__ goff, uint32_t* __restrict__ sorted,
                                                         uint32_t* __restrict__ gcur, uint32_t* __restrict__ big) {
  extern __shared__ uint32_t sm[];
  uint32_t* sval = sm;                  // [S3_CAP] staged values (bucket order)
  uint32_t* cnt = sm + S3_CAP;          // [2^b3]
  __shared__ uint32_t warp_sums[32];
  const uint32_t q = blockIdx.x;
  const uint32_t e0 = subOff[q], e1 = subOff[q + 1];  // subOff[nsub] = M
  const uint32_t nf = 1u << b3, fmask = nf - 1, fbase = q << b3;
  if (e1 - e0 > (uint32_t)S3_CAP) {  // oversized: counted, scanned and scattered by k_s3_big_*
    for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x)
      if (fbase + i < F) gcur[fbase + i] = 0;
    if (threadIdx.x == 0) big[1 + atomicAdd(big, 1u)] = q;
    return;
  }
  for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) cnt[i] = 0;
  __syncthreads();
  s3_for_keys(keys2, e0, e1, [&](uint32_t f) { atomicAdd(cnt + (f & fmask), 1u); });
  __syncthreads();
  s3_block_scan(cnt, nf, warp_sums);
  for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x)
    if (fbase + i < F) goff[fbase + i] = e0 + cnt[i];
  __syncthreads();
  const uint32_t len = e1 - e0;
  if (len <= (uint32_t)S3_CAP) {
    s3_for_entries(keys2, vals2, e0, e1, [&](uint32_t f, uint32_t v) { sval[atomicAdd(cnt + (f & fmask), 1u)] = v; });
    __syncthreads();
    for (uint32_t p = threadIdx.x; p < len; p += blockDim.x) sorted[e0 + p] = sval[p];
  }
}

// Oversized sub-bins, step 1: per-bucket counts by many blocks (chunks of S3_BIG_CH
// entries, shared-memory histogram, one global atomic per (chunk, bucket)) into gcur.
constexpr uint32_t S3_BIG_CH = 8192;
static __global__ void __launch_bounds__(256) k_s3_big_count(const uint32_t* __restrict__ subOff, int b3,
                                                             const uint16_t* __restrict__ keys2,
                                                             uint32_t* __restrict__ gcur, const uint32_t* __restrict__ big) {
  __shared__ uint32_t cnt[S3_MAXFINE];
  const uint32_t nbig = big[0];
  const uint32_t nf = 1u << b3, fmask = nf - 1;
  uint32_t off = 0;
  for (uint32_t t = 0; t < nbig; t++) {
    const uint32_t q = big[1 + t];
    const uint32_t e0 = subOff[q], e1 = subOff[q + 1], fbase = q << b3;
    const uint32_t nch = (e1 - e0 + S3_BIG_CH - 1) / S3_BIG_CH;
    // chunks of all listed sub-bins are dealt round-robin over the blocks (global chunk
    // index off + ch), so many small oversized sub-bins (the f3 top window's low buckets)
    // run in parallel instead of one after another
    const uint32_t ch0 = (blockIdx.x + gridDim.x - off % gridDim.x) % gridDim.x;
    off += nch;
    for (uint32_t ch = ch0; ch < nch; ch += gridDim.x) {
      const uint32_t c0 = e0 + ch * S3_BIG_CH, c1 = min(c0 + S3_BIG_CH, e1);
      for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) cnt[i] = 0;
      __syncthreads();
      s3_for_keys(keys2, c0, c1, [&](uint32_t f) { atomicAdd(cnt + (f & fmask), 1u); });
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x)
        if (cnt[i]) atomicAdd(gcur + fbase + i, cnt[i]);
      __syncthreads();
    }
  }
}

// step 2: one block per oversized sub-bin scans its bucket counts into goff and the cursors
static __global__ void __launch_bounds__(256) k_s3_big_scan(const uint32_t* __restrict__ subOff, int b3, uint32_t F,
                                                            uint32_t* __restrict__ gcur, const uint32_t* __restrict__ big,
                                                            uint32_t* __restrict__ goff) {
  __shared__ uint32_t cnt[S3_MAXFINE], warp_sums[32];
  const uint32_t nbig = big[0];
  const uint32_t nf = 1u << b3;
  for (uint32_t t = blockIdx.x; t < nbig; t += gridDim.x) {
    const uint32_t q = big[1 + t];
    const uint32_t e0 = subOff[q], fbase = q << b3;
    for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) cnt[i] = fbase + i < F ? gcur[fbase + i] : 0u;
    __syncthreads();
    s3_block_scan(cnt, nf, warp_sums);
    for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x)
      if (fbase + i < F) goff[fbase + i] = gcur[fbase + i] = e0 + cnt[i];
    __syncthreads();
  }
}

// step 3, the scatter: every block takes chunks of S3_BIG_CH entries of every listed
// sub-bin, counts them per bucket in shared memory, reserves one range per (chunk, bucket)
// with a global atomic on the bucket's cursor, and writes the entries there (a run per
// bucket of the chunk: the degenerate one-bucket case writes whole chunks contiguously).
// Was: one block counting and scattering the whole sub-bin (BLS12-377 2^24 at c = 21, ~n
// entries in bucket 1: a 24 ms sort).
static __global__ void __launch_bounds__(256) k_s3_big(const uint32_t* __restrict__ subOff, int b3,
                                                       const uint16_t* __restrict__ keys2, const uint32_t* __restrict__ vals2,
                                                       uint32_t* __restrict__ gcur, const uint32_t* __restrict__ big,
                                                       uint32_t* __restrict__ sorted) {
  __shared__ uint32_t cnt[S3_MAXFINE], gb[S3_MAXFINE];
  const uint32_t nbig = big[0];
  const uint32_t nf = 1u << b3, fmask = nf - 1;
  uint32_t off = 0;
  for (uint32_t t = 0; t < nbig; t++) {
    const uint32_t q = big[1 + t];
    const uint32_t e0 = subOff[q], e1 = subOff[q + 1];
    const uint32_t fbase = q << b3;
    const uint32_t nch = (e1 - e0 + S3_BIG_CH - 1) / S3_BIG_CH;
    // chunks of all listed sub-bins are dealt round-robin over the blocks (global chunk
    // index off + ch), so many small oversized sub-bins (the f3 top window's low buckets)
    // run in parallel instead of one after another
    const uint32_t ch0 = (blockIdx.x + gridDim.x - off % gridDim.x) % gridDim.x;
    off += nch;
    for (uint32_t ch = ch0; ch < nch; ch += gridDim.x) {
      const uint32_t c0 = e0 + ch * S3_BIG_CH, c1 = min(c0 + S3_BIG_CH, e1);
      for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) cnt[i] = 0;
      __syncthreads();
      s3_for_keys(keys2, c0, c1, [&](uint32_t f) { atomicAdd(cnt + (f & fmask), 1u); });
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < nf; i += blockDim.x) {
        const uint32_t h = cnt[i];
        gb[i] = h ? atomicAdd(gcur + fbase + i, h) : 0u;
        cnt[i] = 0;
      }
      __syncthreads();
      s3_for_entries(keys2, vals2, c0, c1, [&](uint32_t f, uint32_t v) {
        const uint32_t k = f & fmask;
        sorted[gb[k] + atomicAdd(cnt + k, 1u)] = v;
      });
      __syncthreads();
    }
  }
}
