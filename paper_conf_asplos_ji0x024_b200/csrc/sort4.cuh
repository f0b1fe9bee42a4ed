// a3, two-pass cluster counting sort (§3.2.1, Alg. 3).
// Included inside namespace msmk by msm_kernels.cuh, after sort3.cuh.
//
// Alg. 3 ranks a block's entries per bucket in shared memory and reserves one global range
// per (block, bucket) with one atomic.  B200's bucket sets (2^23 buckets at
// c = 24 with the f3 table) are far beyond one block's shared memory, and the three-level
// sort3.cuh moved every entry through HBM twice as an 8-byte (key, value) pair (ncu at
// 2^26: 34 GB of DRAM traffic for 5.1 GB of algorithmic bytes).  Here the rank is taken
// by a thread-block CLUSTER of S4_CL CTAs whose shared memories (DSMEM) act as one:
//   count  k_s4_count   scalars -> per-bin counts (bin = flat bucket >> b2, <= 8192 bins)
//   P1     k_s4_part1   scalars -> entries partitioned into bins; per CLUSTER tile one
//                       global atomic per (tile, bin), taken by the bin's owner CTA after
//                       summing the S4_CL local histograms through DSMEM; the S4_CL CTAs'
//                       fragments of a bin are adjacent and written together, so L2 merges
//                       them into full sectors.  An entry leaves P1 as 6 bytes: the
//                       bucket's low b2 bits (u16) and the value (u32).
//   P2     k_s4_part2   one cluster per bin (2^b2 buckets, <= S4_CL * S4_CAP entries in a
//                       round): local histograms, a cluster-wide scan over the bin's buckets
//                       through DSMEM (goff), and every CTA writes its entries, staged in
//                       bucket order, at their final positions.  Oversized bins (skewed
//                       scalars; the f3 table's top window lands in the lowest buckets) take
//                       a histogram sweep first, then rounds with running per-bucket offsets.
// HBM per entry: P1 writes 6 B, P2 reads 6 B and writes the 4-B value; the scalars are read
// twice (count, P1).  The (i, j) entry value is (i + j*istride) | sign<<31 as everywhere.
namespace cg = cooperative_groups;  // <cooperative_groups.h>: included by msm_kernels.cuh

constexpr int S4_CL = 8;              // CTAs per cluster (portable maximum)
constexpr int S4_THREADS = 1024;
constexpr int S4_CAP = 24576;         // P2 entries per CTA per round (staged: 144 KB)
constexpr int S4_MAXBIN = 8192;       // P1 bins (counters in shared memory)
constexpr int S4_MAXNBK = 4096;       // buckets per bin (b2 <= 12)
constexpr int S4_SMEM = 232000;       // dynamic shared memory budget per CTA (bytes)
constexpr int S4_U = 8;               // loads in flight per thread in the P2 sweep loop
constexpr int S4_THREADS2 = 512;      // P2 threads; each holds S4_IT entries of a round in registers
constexpr int S4_IT = S4_CAP / S4_THREADS2;

// P1 slots per CTA for NC1 bins: 12 B of counters per bin; per slot 14 B (the unsorted
// digit u32 + its rank u16, the staged key u32 + value u32)
__host__ __device__ inline uint32_t s4_t1(uint32_t NC1) {
  const uint32_t t = (uint32_t)((S4_SMEM - 12u * NC1 - 64u) / 14u);
  return t & ~511u;
}

// count: binCount[f >> b2] over all digits; err |= 4 for k >= r
template <class C>
__global__ void __launch_bounds__(512) k_s4_count(const uint32_t* __restrict__ scal, size_t n, int cp, int nwin,
                                                  uint32_t ws, int b2, uint32_t NC1, uint32_t* __restrict__ binCount,
                                                  uint32_t* err) {
  extern __shared__ uint32_t hist[];
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  constexpr int U = C::S <= 8 ? 4 : 1;  // scalars in flight per thread
  const size_t base = (size_t)blockIdx.x * (512 * 16);
  bool bad = false;
#pragma unroll 1
  for (int q0 = 0; q0 < 16; q0 += U) {
    ScalarReg<C> k[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const size_t i = base + (size_t)(q0 + u) * 512 + threadIdx.x;
      if (i < n) load_scalar<C>(k[u], scal, i);
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      const size_t i = base + (size_t)(q0 + u) * 512 + threadIdx.x;
      if (i >= n) continue;
      if (!scalar_in_range<C>(k[u])) { bad = true; continue; }
      for_each_digit<C>(k[u], cp, nwin, [&](int j, uint32_t b, bool) { atomicAdd(hist + ((j * ws + b) >> b2), 1u); });
    }
  }
  if (bad) atomicOr(err, 4u);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x)
    if (hist[i]) atomicAdd(binCount + i, hist[i]);
}

// P1: CTA = tp points (tp * nwin <= s4_t1(NC1) slots); cluster = S4_CL consecutive CTAs.
// Digits are extracted once: slot (point, window) keeps the flat key and its rank within
// (CTA, bin) (the return value of the counting atomic), so after the cluster exchange and
// the local scan every entry moves to its staged position without a second atomic.
template <class C>
__global__ void __cluster_dims__(S4_CL, 1, 1) __launch_bounds__(S4_THREADS, 1)
    k_s4_part1(const uint32_t* __restrict__ scal, size_t n, int cp, int nwin, uint32_t ws, uint32_t istride, int b2,
               uint32_t NC1, uint32_t tp, uint32_t* __restrict__ binCursor, uint16_t* __restrict__ keys,
               uint32_t* __restrict__ vals, uint32_t ibase = 0) {
  extern __shared__ uint32_t sm[];
  const uint32_t T1 = s4_t1(NC1);
  uint32_t* cnt = sm;              // [NC1] local counts (read remotely), then local bin starts
  uint32_t* gbase = cnt + NC1;     // [NC1] global start of this CTA's fragment (owner-written)
  uint32_t* gadj = gbase + NC1;    // [NC1] gbase - local start
  uint32_t* U = gadj + NC1;        // [T1] slot -> flat key | sign << 31, ~0 = no entry
  uint32_t* Tk = U + T1;           // [T1] staged flat keys (bin order)
  uint32_t* Tv = Tk + T1;          // [T1] staged values
  uint16_t* R = reinterpret_cast<uint16_t*>(Tv + T1);  // [T1] slot -> rank within (CTA, bin)
  __shared__ uint32_t warp_sums[32];
  cg::cluster_group cl = cg::this_cluster();
  const uint32_t rank = cl.block_rank();
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) cnt[i] = 0;
  __syncthreads();
  const size_t p0 = min((size_t)blockIdx.x * tp, n);
  const uint32_t npts = (uint32_t)(min(p0 + tp, n) - p0);
  for (uint32_t pl = threadIdx.x; pl < npts; pl += blockDim.x) {
    ScalarReg<C> k;
    load_scalar<C>(k, scal, p0 + pl);
    uint32_t* u = U + pl * nwin;
    uint16_t* rr = R + pl * nwin;
    for (int j = 0; j < nwin; j++) u[j] = ~0u;
    if (!scalar_in_range<C>(k)) continue;
    for_each_digit<C>(k, cp, nwin, [&](int j, uint32_t b, bool neg) {
      const uint32_t f = j * ws + b;
      rr[j] = (uint16_t)atomicAdd(cnt + (f >> b2), 1u);
      u[j] = f | (neg ? SIGN_BIT : 0u);
    });
  }
  cl.sync();  // (A) every CTA's counts visible cluster-wide
  {  // owner of bins [o0, o1): one global reservation per (cluster tile, bin)
    const uint32_t per = (NC1 + S4_CL - 1) / S4_CL;
    const uint32_t o0 = min(rank * per, NC1), o1 = min(o0 + per, NC1);
    for (uint32_t b = o0 + threadIdx.x; b < o1; b += blockDim.x) {
      uint32_t c[S4_CL], tot = 0;
#pragma unroll
      for (int q = 0; q < S4_CL; q++) {
        c[q] = cl.map_shared_rank(cnt, q)[b];
        tot += c[q];
      }
      uint32_t g = tot ? atomicAdd(binCursor + b, tot) : 0u;
#pragma unroll
      for (int q = 0; q < S4_CL; q++) {
        cl.map_shared_rank(gbase, q)[b] = g;
        g += c[q];
      }
    }
  }
  cl.sync();  // (B) gbase written; no remote access after this point
  const uint32_t E = s3_block_scan(cnt, NC1, warp_sums);  // cnt -> local bin starts
  for (uint32_t i = threadIdx.x; i < NC1; i += blockDim.x) gadj[i] = gbase[i] - cnt[i];
  const uint32_t ns = npts * (uint32_t)nwin;
  const uint32_t magic = 0xffffffffu / (uint32_t)nwin + 1u;  // s / nwin exact for s * nwin < 2^32
  for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) {
    const uint32_t f = U[s];
    if (f == ~0u) continue;
    const uint32_t fb = f & ~SIGN_BIT;
    const uint32_t pos = cnt[fb >> b2] + R[s];
    const uint32_t pl = nwin == 1 ? s : __umulhi(s, magic);
    const uint32_t j = s - pl * (uint32_t)nwin;
    Tk[pos] = fb;
    Tv[pos] = ((uint32_t)(p0 + pl) + ibase + j * istride) | (f & SIGN_BIT);
  }
  __syncthreads();
  const uint32_t mask = (1u << b2) - 1u;
  for (uint32_t p = threadIdx.x; p < E; p += blockDim.x) {
    const uint32_t fb = Tk[p];
    const uint32_t o = gadj[fb >> b2] + p;
    keys[o] = (uint16_t)(fb & mask);
    vals[o] = Tv[p];
  }
}

// entries [e0, e1) with stride blockDim.x, S4_U loads in flight per thread
template <class F>
__device__ __forceinline__ void s4_for_keys(const uint16_t* __restrict__ keys, uint32_t e0, uint32_t e1, F&& f) {
  for (uint32_t eb = e0 + threadIdx.x; eb < e1; eb += S4_U * blockDim.x) {
    uint32_t k[S4_U];
#pragma unroll
    for (int u = 0; u < S4_U; u++) {
      const uint32_t e = eb + u * blockDim.x;
      k[u] = e < e1 ? (uint32_t)__ldg(keys + e) : 0u;
    }
#pragma unroll
    for (int u = 0; u < S4_U; u++)
      if (eb + u * blockDim.x < e1) f(k[u]);
  }
}
template <class F>
__device__ __forceinline__ void s4_for_entries(const uint16_t* __restrict__ keys, const uint32_t* __restrict__ vals,
                                               uint32_t e0, uint32_t e1, F&& f) {
  for (uint32_t eb = e0 + threadIdx.x; eb < e1; eb += S4_U * blockDim.x) {
    uint32_t k[S4_U], v[S4_U];
#pragma unroll
    for (int u = 0; u < S4_U; u++) {
      const uint32_t e = eb + u * blockDim.x;
      k[u] = e < e1 ? (uint32_t)__ldg(keys + e) : 0u;
      v[u] = e < e1 ? __ldg(vals + e) : 0u;
    }
#pragma unroll
    for (int u = 0; u < S4_U; u++)
      if (eb + u * blockDim.x < e1) f(k[u], v[u]);
  }
}

// Exclusive scan of the owners' ranges across the cluster: every CTA holds own[0..per)
// (its buckets' totals); on return own[i] = start of bucket rank*per + i relative to the
// bin, and the function returns nothing else.  Contains two cluster barriers.
__device__ __forceinline__ void s4_cluster_scan(cg::cluster_group& cl, uint32_t* own, uint32_t per, uint32_t* range_sum,
                                                uint32_t* warp_sums) {
  const uint32_t T = s3_block_scan(own, per, warp_sums);
  if (threadIdx.x == 0) *range_sum = T;
  cl.sync();
  uint32_t prefix = 0;
  const uint32_t rank = cl.block_rank();
  for (uint32_t q = 0; q < rank; q++) prefix += *cl.map_shared_rank(range_sum, q);
  for (uint32_t i = threadIdx.x; i < per; i += blockDim.x) own[i] += prefix;
  __syncthreads();
}

// P2: cluster b = bin b, buckets f in [b << b2, (b+1) << b2) (those < F get goff).
static __global__ void __cluster_dims__(S4_CL, 1, 1) __launch_bounds__(S4_THREADS2, 1)
    k_s4_part2(const uint32_t* __restrict__ binOff, int b2, uint32_t F, const uint16_t* __restrict__ keys,
               const uint32_t* __restrict__ vals, uint32_t* __restrict__ goff, uint32_t* __restrict__ sorted) {
  extern __shared__ uint32_t sm[];
  const uint32_t NBK = 1u << b2;
  uint32_t* cnt = sm;                              // [NBK] round counts, then local starts
  uint32_t* cur = cnt + NBK;                       // [NBK] local cursors
  uint32_t* base = cur + NBK;                      // [NBK] global start of this CTA's fragment (owner-written)
  uint32_t* sval = base + NBK;                     // [S4_CAP] staged values (bucket order)
  uint16_t* skey = reinterpret_cast<uint16_t*>(sval + S4_CAP);  // [S4_CAP] staged bucket
  __shared__ uint32_t own[S4_MAXNBK / S4_CL];      // owner: bucket starts (absolute)
  __shared__ uint32_t run[S4_MAXNBK / S4_CL];      // owner: entries already placed (rounds)
  __shared__ uint32_t warp_sums[32], range_sum;
  cg::cluster_group cl = cg::this_cluster();
  const uint32_t rank = cl.block_rank();
  const uint32_t bin = blockIdx.x / S4_CL;
  const uint32_t e0 = binOff[bin], e1 = binOff[bin + 1], len = e1 - e0;
  const uint32_t fbase = bin << b2;
  const uint32_t per = NBK / S4_CL, k0 = rank * per;
  if (len == 0) {  // uniform over the cluster: no barrier is reached
    for (uint32_t k = threadIdx.x; k < per; k += blockDim.x)
      if (fbase + k0 + k < F) goff[fbase + k0 + k] = e0;
    return;
  }
  constexpr uint32_t RCAP = (uint32_t)S4_CL * S4_CAP;
  const bool heavy = len > RCAP;
  if (heavy) {  // histogram sweep over the whole bin -> bucket starts, goff
    for (uint32_t k = threadIdx.x; k < NBK; k += blockDim.x) cnt[k] = 0;
    __syncthreads();
    const uint32_t cs = (len + S4_CL - 1) / S4_CL;
    const uint32_t c0 = e0 + min(rank * cs, len), c1 = e0 + min((rank + 1) * cs, len);
    s4_for_keys(keys, c0, c1, [&](uint32_t k) { atomicAdd(cnt + k, 1u); });
    cl.sync();
    for (uint32_t k = threadIdx.x; k < per; k += blockDim.x) {
      uint32_t t = 0;
#pragma unroll
      for (int q = 0; q < S4_CL; q++) t += cl.map_shared_rank(cnt, q)[k0 + k];
      own[k] = t;
      run[k] = 0;
    }
    __syncthreads();
    s4_cluster_scan(cl, own, per, &range_sum, warp_sums);
    for (uint32_t k = threadIdx.x; k < per; k += blockDim.x) {
      own[k] += e0;
      if (fbase + k0 + k < F) goff[fbase + k0 + k] = own[k];
    }
    cl.sync();  // all remote reads of cnt done before it is reused
  }
  for (uint32_t r0 = e0; r0 < e1; r0 += RCAP) {
    const uint32_t rl = min(RCAP, e1 - r0);
    const uint32_t cs = (rl + S4_CL - 1) / S4_CL;
    const uint32_t c0 = r0 + min(rank * cs, rl), c1 = r0 + min((rank + 1) * cs, rl);
    for (uint32_t k = threadIdx.x; k < NBK; k += blockDim.x) cnt[k] = 0;
    // the CTA's chunk (<= S4_CAP entries) in registers: two 16-bit keys per word, 0xffff = none
    uint32_t kk[S4_IT / 2], vv[S4_IT];
#pragma unroll
    for (int u = 0; u < S4_IT; u++) {
      const uint32_t e = c0 + u * S4_THREADS2 + threadIdx.x;
      const uint32_t k = e < c1 ? (uint32_t)__ldg(keys + e) : 0xffffu;
      vv[u] = e < c1 ? __ldg(vals + e) : 0u;
      if (u & 1) kk[u >> 1] |= k << 16; else kk[u >> 1] = k;
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < S4_IT; u++) {
      const uint32_t k = (kk[u >> 1] >> (16 * (u & 1))) & 0xffffu;
      if (k != 0xffffu) atomicAdd(cnt + k, 1u);
    }
    cl.sync();  // (A) round counts visible
    if (!heavy) {  // single round: bucket starts from this round's totals
      for (uint32_t k = threadIdx.x; k < per; k += blockDim.x) {
        uint32_t t = 0;
#pragma unroll
        for (int q = 0; q < S4_CL; q++) t += cl.map_shared_rank(cnt, q)[k0 + k];
        own[k] = t;
        run[k] = 0;
      }
      __syncthreads();
      s4_cluster_scan(cl, own, per, &range_sum, warp_sums);
      for (uint32_t k = threadIdx.x; k < per; k += blockDim.x) {
        own[k] += e0;
        if (fbase + k0 + k < F) goff[fbase + k0 + k] = own[k];
      }
      __syncthreads();
    }
    for (uint32_t k = threadIdx.x; k < per; k += blockDim.x) {  // per-CTA fragment starts
      uint32_t g = own[k] + run[k];
#pragma unroll
      for (int q = 0; q < S4_CL; q++) {
        const uint32_t c = cl.map_shared_rank(cnt, q)[k0 + k];
        cl.map_shared_rank(base, q)[k0 + k] = g;
        g += c;
      }
      run[k] = g - own[k];
    }
    cl.sync();  // (B) bases written
    const uint32_t E = s3_block_scan(cnt, NBK, warp_sums);
    for (uint32_t k = threadIdx.x; k < NBK; k += blockDim.x) cur[k] = cnt[k];
    __syncthreads();
#pragma unroll
    for (int u = 0; u < S4_IT; u++) {
      const uint32_t k = (kk[u >> 1] >> (16 * (u & 1))) & 0xffffu;
      if (k != 0xffffu) {
        const uint32_t pos = atomicAdd(cur + k, 1u);
        sval[pos] = vv[u];
        skey[pos] = (uint16_t)k;
      }
    }
    __syncthreads();
    for (uint32_t p = threadIdx.x; p < E; p += blockDim.x) {
      const uint32_t k = skey[p];
      sorted[base[k] + (p - cnt[k])] = sval[p];
    }
    if (r0 + RCAP < e1) cl.sync();  // (C) next round reuses cnt/base (read remotely above)
  }
}
