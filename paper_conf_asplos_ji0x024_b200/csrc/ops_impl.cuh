// Per-curve implementation of msmrt::CurveOps: launches the kernels of msm_kernels.cuh.
// Included by exactly one translation unit per curve (curve_*.cu).
#pragma once
#include <algorithm>
#include <cmath>

#include "msm_kernels.cuh"
#include "runtime.h"

namespace msmrt {

using namespace msmk;

#ifndef MSM_SEG_UNI
#define MSM_SEG_UNI 0  // A/B (with MSM_UNI_ALL=1): call-based PADD in the bucket reduce at every n
#endif

template <class C>
struct Ops final : CurveOps {
  // k_accumulate_sync (lockstep blocks, register-prefetched gathers) for L <= 13; MNT4-753
  // keeps k_accumulate (255 registers already; no room for the prefetched point)
  static constexpr bool kAccSync = MSM_ACC_SYNC != 0 && (C::L <= 13 || MSM_ACC_SYNC_ALL != 0);
  // batch-affine front end (baff.cuh) for L <= 13 (MNT4-753's 27-limb pairs would spill)
  // Built only with -DMSM_BAFF=1 (an ablation, off by default: compile time and speed,
  // DESIGN.md §7b); without it MSM_OPT_ACC_MODE = 1 returns MSM_ERR_UNIMPLEMENTED.
  static constexpr bool kBaff = MSM_BAFF != 0 && kAccSync && C::L <= 13;
  bool has_baff() const override { return kBaff; }
  static constexpr uint32_t kBaffB = 256;  // outputs per batch (one inversion per level)
  static constexpr int XW_ = Layout<C>::XW;
  static constexpr int PW_ = Layout<C>::PW;
  int L32() const override { return C::L32; }
  int S() const override { return C::S; }
  int lambda() const override { return C::LAMBDA; }
  int PW() const override { return PW_; }
  int XW() const override { return XW_; }

  void points_to_mont(Shard& s, const uint32_t* in_dev, size_t n) override {
    if (n == 0) return;
    k_points_to_mont<C><<<(unsigned)cdiv(n, 128), 128, 0, s.stream>>>(s.pts, in_dev, n, s.err);
    CK(cudaGetLastError());
  }

  void free_scratch(Shard& s) override {
    dfree(s.counts); dfree(s.goff); dfree(s.cursor); dfree(s.sorted); dfree(s.buckets);
    dfree(s.carry_pts); dfree(s.carry_f); dfree(s.segA); dfree(s.segB); dfree(s.W); dfree(s.tiles);
    dfree(s.binCount); dfree(s.binOff); dfree(s.binCursor); dfree(s.binIdx); dfree(s.binFine);
    dfree(s.nlong); dfree(s.longs);
    dfree(s.s3Count); dfree(s.s3Off); dfree(s.s3Cursor); dfree(s.s3Sub);
    dfree(s.s3SubCount); dfree(s.s3SubCursor); dfree(s.s3Tiles); dfree(s.s3Big);
    dfree(s.s3k1); dfree(s.s3v1); dfree(s.s3k2); dfree(s.s3v2);
    dfree(s.s4Count); dfree(s.s4Off); dfree(s.s4Cursor); dfree(s.s4k); dfree(s.s4v);
    dfree(s.c4); dfree(s.goff4); dfree(s.cursor4); dfree(s.out4); dfree(s.baff_scratch);
    s.baff = 0;
  }

  void free_table(Shard& s) override {
    dfree(s.table);
    s.table_c = 0;
  }

  // f3: table[j][i] = 2^(j c) P_i for j < nwin (k_pre_dbl + k_pre_norm per chunk of points)
  void build_table(Shard& s) {
    const size_t n = s.n;
    dalloc(&s.table, std::max<size_t>(1, (size_t)s.nwin * n) * PW_);
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    CK(cudaEventRecord(e0, s.stream));
    if (n) CK(cudaMemcpyAsync(s.table, s.pts, n * PW_ * 4, cudaMemcpyDeviceToDevice, s.stream));
    const size_t chunk = std::min<size_t>(std::max<size_t>(n, 1), (size_t)1 << 22);
    uint32_t* tmp = nullptr;
    dalloc(&tmp, chunk * XW_);
    for (int j = 1; j < s.nwin && n; j++) {
      for (size_t off = 0; off < n; off += chunk) {
        const size_t cnt = std::min(chunk, n - off);
        const uint32_t* src = s.table + ((size_t)(j - 1) * n + off) * PW_;
        uint32_t* dst = s.table + ((size_t)j * n + off) * PW_;
        k_pre_dbl<C><<<(unsigned)cdiv(cnt, 128), 128, 0, s.stream>>>(src, cnt, s.c, tmp);
        k_pre_norm<C><<<(unsigned)cdiv(cdiv(cnt, PRE_K), 128), 128, 0, s.stream>>>(tmp, cnt, dst);
        CK(cudaGetLastError());
      }
    }
    CK(cudaEventRecord(e1, s.stream));
    CK(cudaStreamSynchronize(s.stream));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    s.table_ms = ms;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    dfree(tmp);
    s.table_c = s.c;
  }

  void configure(const Options& o, Shard& s, int c, int pre) override {
    CK(cudaSetDevice(s.dev));
    free_scratch(s);
    s.c = c;
    s.nwin = num_windows(C::LAMBDA, c);
    s.pre = pre;
    s.nset = pre ? 1 : s.nwin;
    s.split_G = o.split_G;
    s.split_g = o.split_g;
    s.c_arg = c | ((o.split_G - 1) << 8) | (o.split_g << 16);
    s.NB = (1u << (c - 1)) / (uint32_t)o.split_G + 1;
    s.F = (size_t)s.nset * s.NB;
    s.ntiles = cdiv(s.F, SCAN_TILE);
    // a3 variant: the staged three-level sort for large entry counts, the binned two-level
    // sort below ~2^21 entries (fewer launches)
    const size_t Mmax0 = s.n * (size_t)s.nwin;
    s.sort_mode = o.sort ? o.sort : (Mmax0 >= ((size_t)1 << 21) ? 3 : 2);
    if (s.sort_mode == 4) {
      // bins of 2^b2 flat buckets holding ~85 % of one cluster round (S4_CL * S4_CAP entries)
      // on average; <= S4_MAXBIN bins, b2 in [3, 12] (else the three-level sort)
      const double per_bucket = (double)std::max<size_t>(Mmax0 / (size_t)o.split_G, 1) / (double)std::max<size_t>(s.F, 1);
      int b2 = (int)std::floor(std::log2(0.85 * S4_CL * S4_CAP / std::max(per_bucket, 1e-9)));
      b2 = std::max(3, std::min(b2, 12));
      while (b2 < 12 && ((s.F - 1) >> b2) + 1 > (size_t)S4_MAXBIN) b2++;
      s.s4_b2 = b2;
      s.s4_NC1 = (uint32_t)(((s.F - 1) >> b2) + 1);
      if (s.s4_NC1 > (uint32_t)S4_MAXBIN) s.sort_mode = 3;
    }
    s.shift = 0;
    while (s.shift < 13 && (size_t)s.nset * (((size_t)(s.NB - 1) >> s.shift) + 1) > 13000) s.shift++;
    s.nbin = (uint32_t)(((size_t)(s.NB - 1) >> s.shift) + 1);
    s.FB = (uint32_t)s.nset * s.nbin;
    s.ntiles_bin = cdiv(s.FB, SCAN_TILE);
    CK(cudaFuncSetAttribute(k_bin_count<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(s.FB * 4)));
    CK(cudaFuncSetAttribute(k_bin_scatter<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(2 * s.FB * 4)));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, s.dev));
    const int sms = prop.multiProcessorCount;
    s.sms = sms;
    int bps = 0;
#if MSM_ACC_SMEM
    constexpr int acc_smem = ACC_SLOTS * C::L * ACC_NT * 4;
    CK(cudaFuncSetAttribute(k_accumulate_smem<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, acc_smem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_accumulate_smem<C>, 128, acc_smem));
#else
    if constexpr (kAccSync) {
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_accumulate_sync<C>, ACC_SYNC_NT, 0));
      bps *= ACC_SYNC_NT / 128;  // in units of 128 threads below
    } else {
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_accumulate<C>, 128, 0));
    }
#endif
    if (bps < 1) bps = 1;
    const size_t resident = (size_t)sms * bps * 128;
    const size_t Mmax = s.n * (size_t)s.nwin;
    size_t T = o.threads > 0 ? (size_t)o.threads : std::min(resident, std::max<size_t>(1, cdiv(Mmax, 16)));
    if (T < 1) T = 1;
    s.slice = (uint32_t)std::max<size_t>(1, cdiv(Mmax, T));
    s.acc_threads = (uint32_t)std::max<size_t>(1, cdiv(Mmax, s.slice));
    // bucket-reduce segments
    int bps2 = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps2, k_bucket_segments<C, false>, SEG_NT, 0));
    bps2 *= SEG_NT / 128;  // in units of 128 threads below
    if (bps2 < 1) bps2 = 1;
    const size_t resident2 = (size_t)sms * bps2 * 128;
    const size_t nb = s.NB;  // local buckets 0..NB-1 (bucket 0 is empty without the f1 split)
    // one segment per resident thread (full occupancy, no tail wave); >= 4 buckets each
    uint32_t seg = o.seg > 0 ? (uint32_t)o.seg : (uint32_t)std::max<size_t>(4, cdiv((size_t)s.nset * nb, resident2));
    s.seg = seg;
    s.nseg = (uint32_t)cdiv(nb, seg);
    // small n (segments below half a wave): k_bucket_segments<C, true> runs the shared
    // out-of-line PADD body (MSM_SHARED_NI, ec.cuh); the call-based PADD (MSM_UNI_ALL) and
    // r01's inline latency-mode products measured slower (C1 reduce 0.253 -> 0.269 ms)
    s.seg_lat = ((MSM_UNI_ALL || MSM_SHARED_NI) && (MSM_SEG_UNI || (size_t)s.nset * s.nseg * 2 < resident2)) ? 1 : 0;
    if (!pre) free_table(s);
    else if (!s.table || s.table_c != c) {
      free_table(s);
      build_table(s);
    }
    s.baff = (kBaff && o.acc_mode == 1) ? 1 : 0;  // auto (2) = PACC only: the front end measured slower
    if constexpr (kBaff) if (s.baff) {
      int bpb = 0;
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bpb, k_baff2<C>, BAFF_NT, 0));
      if (bpb < 1) bpb = 1;
      s.baff_T = (uint32_t)(sms * bpb * BAFF_NT);
      s.baff_B = kBaffB;
      const size_t M4max = Mmax / 4 + s.F + 1;
      dalloc(&s.c4, s.F);
      dalloc(&s.goff4, s.F + 1);
      dalloc(&s.cursor4, s.F);
      dalloc(&s.out4, M4max * PW_);
      dalloc(&s.baff_scratch, (size_t)s.baff_T * s.baff_B * (7 * C::L + 2));
    }
    dalloc(&s.counts, s.F);
    dalloc(&s.goff, s.F + 1);
    dalloc(&s.cursor, s.F);
    dalloc(&s.sorted, Mmax);
    dalloc(&s.buckets, s.F * XW_);
    dalloc(&s.carry_pts, (size_t)s.acc_threads * XW_);
    dalloc(&s.carry_f, s.acc_threads);
    dalloc(&s.nlong, 1);
    dalloc(&s.longs, s.acc_threads);
    CK(cudaFuncSetAttribute(k_fixup_long<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, FIX_THREADS * XW_ * 4));
    dalloc(&s.segA, (size_t)s.nset * s.nseg * XW_);
    dalloc(&s.segB, (size_t)s.nset * cdiv(s.nseg, 32) * XW_);
    dalloc(&s.W, (size_t)s.nset * XW_);
    dalloc(&s.tiles, std::max(std::max(s.ntiles, s.ntiles_bin), cdiv((size_t)1 << 18, SCAN_TILE)) + 1);
    if (s.sort_mode == 3) {
      // key bits: b3 resolved per sub-bin in shared memory (~8K entries per sub-bin),
      // b1, b2 <= 9 per partition pass
      int KB = 1;
      while (((size_t)1 << KB) < s.F) KB++;
      int b3 = (int)std::lround(std::log2(8192.0 * (double)s.F / (double)std::max<size_t>(Mmax / (size_t)s.split_G, 1)));
      b3 = std::max(1, std::min(b3, 12));
      b3 = std::min(b3, KB);
      if (KB - b3 > 18) b3 = KB - 18;
      const int rest = KB - b3;
      s.s3_b2 = std::min(9, rest / 2);
      s.s3_b1 = rest - s.s3_b2;
      // P1 keys are the flat key's low b2 + b3 bits: u16 when <= 16 (move bits into b1 if it
      // has room; b2 only shrinks, so b2 <= 9 still holds)
      if (s.s3_b2 + b3 > 16 && KB - 16 <= 9) {
        s.s3_b1 = KB - 16;
        s.s3_b2 = rest - s.s3_b1;
      }
      s.s3_b3 = b3;
      s.s3_k16 = s.s3_b2 + b3 <= 16 ? 1 : 0;
      const size_t NC1 = (size_t)1 << s.s3_b1, NC2 = (size_t)1 << s.s3_b2;
      dalloc(&s.s3Count, NC1);
      dalloc(&s.s3Off, NC1 + 1);
      dalloc(&s.s3Cursor, NC1);
      dalloc(&s.s3Sub, NC1 * NC2 + 1);
      dalloc(&s.s3SubCount, NC1 * NC2);
      dalloc(&s.s3SubCursor, NC1 * NC2);
      dalloc(&s.s3Tiles, NC1 + 1);
      dalloc(&s.s3Big, NC1 * NC2 + 1);
      dalloc(&s.s3k1, Mmax);
      dalloc(&s.s3v1, Mmax);
      dalloc(&s.s3k2, Mmax);
      dalloc(&s.s3v2, Mmax);
      CK(cudaFuncSetAttribute(k_s3_part1<C, uint16_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * S3_TILE * 4));
      CK(cudaFuncSetAttribute(k_s3_part1<C, uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * S3_TILE * 4));
      CK(cudaFuncSetAttribute(k_s3_part2<uint16_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * S3_TILE * 4));
      CK(cudaFuncSetAttribute(k_s3_part2<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * S3_TILE * 4));
      CK(cudaFuncSetAttribute(k_s3_part3, cudaFuncAttributeMaxDynamicSharedMemorySize, (S3_CAP + S3_MAXFINE) * 4));
    }
    if (s.sort_mode == 4) {
      const size_t NC1 = s.s4_NC1;
      dalloc(&s.s4Count, NC1);
      dalloc(&s.s4Off, NC1 + 1);
      dalloc(&s.s4Cursor, NC1);
      dalloc(&s.s4k, Mmax);
      dalloc(&s.s4v, Mmax);
      CK(cudaFuncSetAttribute(k_s4_count<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(NC1 * 4)));
      CK(cudaFuncSetAttribute(k_s4_part1<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)(12 * NC1 + 14 * (size_t)s4_t1((uint32_t)NC1))));
      CK(cudaFuncSetAttribute(k_s4_part2, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * S4_MAXNBK * 4 + S4_CAP * 6));
    }
    if (s.sort_mode == 2) {
      dalloc(&s.binCount, s.FB);
      dalloc(&s.binOff, s.FB + 1);
      dalloc(&s.binCursor, s.FB);
      dalloc(&s.binIdx, Mmax);
      dalloc(&s.binFine, Mmax);
    }
  }

  int enqueue_pipeline(Shard& s, const uint32_t* scal, bool timed) override {
    return enqueue_range(s, scal, s.n, 0, false, true, s.goff, timed);
  }

  // Chunked host scalars (engine.cu): chunk k of the shard's points [ibase, ibase + n)
  // is sorted and accumulated INTO the bucket set (zeroed before chunk 0; INIT
  // accumulation from chunk 1 on), so its H2D overlaps the previous chunk's work; the
  // last chunk runs the bucket reduce over every bucket (goff = nullptr) and a6.
  bool can_chunk(const Shard& s) const override {
    return kAccSync && C::L <= 13 && !s.baff && (s.sort_mode == 3 || s.sort_mode == 4) && MSM_ACC_SMEM == 0;
  }
  int enqueue_chunk(Shard& s, const uint32_t* scal, size_t n, size_t ibase, bool first, bool last, bool timed) override {
    if (first) CK(cudaMemsetAsync(s.buckets, 0, s.F * XW_ * sizeof(uint32_t), s.stream));
    return enqueue_range(s, scal, n, (uint32_t)ibase, !first, last, nullptr, timed);
  }

  int enqueue_range(Shard& s, const uint32_t* scal, size_t n, uint32_t ibase, bool init, bool reduce,
                    const uint32_t* red_goff, bool timed) {
    cudaStream_t st = s.stream;
    int launches = 0;
    // flat-bucket / flat-bin stride per window and table-row stride (f3: one shared set)
    const uint32_t ws = s.pre ? 0u : s.NB, wsb = s.pre ? 0u : s.nbin, istride = s.pre ? (uint32_t)s.n : 0u;  // table row stride (all points of the shard)
    const uint32_t* pts = s.pre ? s.table : s.pts;
    if (timed) CK(cudaEventRecord(s.ev[EV_H2D], st));
    // a2 + a3: digits, histogram, scan, scatter
    if (s.sort_mode == 4) {
      const uint32_t NC1 = s.s4_NC1;
      const int b2 = s.s4_b2;
      CK(cudaMemsetAsync(s.s4Count, 0, NC1 * sizeof(uint32_t), st));
      if (n) {
        k_s4_count<C><<<(unsigned)cdiv(n, 512 * 16), 512, NC1 * 4, st>>>(scal, n, s.c_arg, s.nwin, ws, b2, NC1, s.s4Count,
                                                                          s.err);
        launches++;
      }
      const size_t nt = cdiv(NC1, SCAN_TILE);
      k_scan_reduce<<<(unsigned)nt, SCAN_THREADS, 0, st>>>(s.s4Count, NC1, s.tiles);
      k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, nt, s.s4Off + NC1);
      k_scan_apply<<<(unsigned)nt, SCAN_THREADS, 0, st>>>(s.s4Count, NC1, s.tiles, s.s4Off, s.s4Cursor);
      launches += 3;
      if (n) {
        const uint32_t tp = std::max<uint32_t>(1, s4_t1(NC1) / (uint32_t)s.nwin);
        const size_t ctas = cdiv(cdiv(n, tp), S4_CL) * S4_CL;
        k_s4_part1<C><<<(unsigned)ctas, S4_THREADS, 12 * NC1 + 14 * s4_t1(NC1), st>>>(
            scal, n, s.c_arg, s.nwin, ws, istride, b2, NC1, tp, s.s4Cursor, s.s4k, s.s4v, ibase);
        launches++;
      }
      CK(cudaMemcpyAsync(s.goff + s.F, s.s4Off + NC1, 4, cudaMemcpyDeviceToDevice, st));
      k_s4_part2<<<(unsigned)(NC1 * S4_CL), S4_THREADS2, 3 * (4u << b2) + S4_CAP * 6, st>>>(s.s4Off, b2, (uint32_t)s.F,
                                                                                         s.s4k, s.s4v, s.goff, s.sorted);
      launches++;
    } else if (s.sort_mode == 3) {
      const uint32_t NC1 = 1u << s.s3_b1, NC2 = 1u << s.s3_b2;
      const int sh1 = s.s3_b2 + s.s3_b3;
      CK(cudaMemsetAsync(s.s3Count, 0, NC1 * sizeof(uint32_t), st));
      if (n) {
        k_s3_count1<C><<<(unsigned)cdiv(n, S3_THREADS * 16), S3_THREADS, 0, st>>>(scal, n, s.c_arg, s.nwin, ws, sh1, NC1,
                                                                               s.s3Count, s.err);
        launches++;
      }
      const size_t nt = cdiv(NC1, SCAN_TILE);
      k_scan_reduce<<<(unsigned)nt, SCAN_THREADS, 0, st>>>(s.s3Count, NC1, s.tiles);
      k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, nt, s.s3Off + NC1);
      k_scan_apply<<<(unsigned)nt, SCAN_THREADS, 0, st>>>(s.s3Count, NC1, s.tiles, s.s3Off, s.s3Cursor);
      launches += 3;
      const uint32_t tp = (uint32_t)std::max(1, S3_TILE / s.nwin);
      uint16_t* k1s = reinterpret_cast<uint16_t*>(s.s3k1);
      uint16_t* k2s = reinterpret_cast<uint16_t*>(s.s3k2);
      if (n) {
        if (s.s3_k16)
          k_s3_part1<C, uint16_t><<<(unsigned)cdiv(n, tp), S3_THREADS, 2 * S3_TILE * 4, st>>>(
              scal, n, s.c_arg, s.nwin, ws, istride, sh1, NC1, tp, s.s3Cursor, k1s, s.s3v1, ibase);
        else
          k_s3_part1<C, uint32_t><<<(unsigned)cdiv(n, tp), S3_THREADS, 2 * S3_TILE * 4, st>>>(
              scal, n, s.c_arg, s.nwin, ws, istride, sh1, NC1, tp, s.s3Cursor, s.s3k1, s.s3v1, ibase);
        launches++;
      }
      const unsigned maxTiles = (unsigned)(cdiv(std::max<size_t>(n * (size_t)s.nwin, 1), S3_TILE) + NC1);
      const size_t nsub = (size_t)NC1 * NC2, nts = cdiv(nsub, SCAN_TILE);
      k_s3_tiles<<<1, S3_THREADS, 0, st>>>(s.s3Off, NC1, s.s3Tiles);
      CK(cudaMemsetAsync(s.s3SubCount, 0, nsub * sizeof(uint32_t), st));
      if (s.s3_k16)
        k_s3_count2<uint16_t><<<maxTiles, S3_THREADS, 0, st>>>(s.s3Tiles, s.s3Off, NC1, s.s3_b3, NC2, k1s, s.s3SubCount);
      else
        k_s3_count2<uint32_t><<<maxTiles, S3_THREADS, 0, st>>>(s.s3Tiles, s.s3Off, NC1, s.s3_b3, NC2, s.s3k1, s.s3SubCount);
      k_scan_reduce<<<(unsigned)nts, SCAN_THREADS, 0, st>>>(s.s3SubCount, nsub, s.tiles);
      k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, nts, s.s3Sub + nsub);
      k_scan_apply<<<(unsigned)nts, SCAN_THREADS, 0, st>>>(s.s3SubCount, nsub, s.tiles, s.s3Sub, s.s3SubCursor);
      if (s.s3_k16)
        k_s3_part2<uint16_t><<<maxTiles, S3_THREADS, 2 * S3_TILE * 4, st>>>(s.s3Tiles, s.s3Off, NC1, s.s3_b3, NC2, k1s,
                                                                            s.s3v1, s.s3SubCursor, k2s, s.s3v2);
      else
        k_s3_part2<uint32_t><<<maxTiles, S3_THREADS, 2 * S3_TILE * 4, st>>>(s.s3Tiles, s.s3Off, NC1, s.s3_b3, NC2, s.s3k1,
                                                                            s.s3v1, s.s3SubCursor, k2s, s.s3v2);
      CK(cudaMemcpyAsync(s.goff + s.F, s.s3Off + NC1, 4, cudaMemcpyDeviceToDevice, st));
      CK(cudaMemsetAsync(s.s3Big, 0, sizeof(uint32_t), st));
      k_s3_part3<<<(unsigned)nsub, 256, (S3_CAP + (1u << s.s3_b3)) * 4, st>>>(s.s3Sub, s.s3_b3, (uint32_t)s.F, k2s,
                                                                             s.s3v2, s.goff, s.sorted, s.cursor, s.s3Big);
      k_s3_big_count<<<(unsigned)(2 * s.sms), 256, 0, st>>>(s.s3Sub, s.s3_b3, k2s, s.cursor, s.s3Big);
      k_s3_big_scan<<<(unsigned)s.sms, 256, 0, st>>>(s.s3Sub, s.s3_b3, (uint32_t)s.F, s.cursor, s.s3Big, s.goff);
      k_s3_big<<<(unsigned)(2 * s.sms), 256, 0, st>>>(s.s3Sub, s.s3_b3, k2s, s.s3v2, s.cursor, s.s3Big, s.sorted);
      launches += 10;
    } else if (s.sort_mode == 2) {
      CK(cudaMemsetAsync(s.binCount, 0, s.FB * sizeof(uint32_t), st));
      const unsigned tiles = (unsigned)cdiv(std::max<size_t>(n, 1), BIN_TILE);
      if (n) {
        k_bin_count<C><<<tiles, BIN_THREADS, s.FB * 4, st>>>(scal, n, s.c_arg, s.nwin, s.shift, s.FB, wsb, s.binCount, s.err);
        launches++;
      }
      k_scan_reduce<<<(unsigned)s.ntiles_bin, SCAN_THREADS, 0, st>>>(s.binCount, s.FB, s.tiles);
      k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, s.ntiles_bin, s.binOff + s.FB);
      k_scan_apply<<<(unsigned)s.ntiles_bin, SCAN_THREADS, 0, st>>>(s.binCount, s.FB, s.tiles, s.binOff, s.binCursor);
      launches += 3;
      if (n) {
        k_bin_scatter<C><<<tiles, BIN_THREADS, 2 * s.FB * 4, st>>>(scal, n, s.c_arg, s.nwin, s.shift, s.FB, wsb, istride,
                                                                  s.binCursor, s.binIdx, s.binFine);
        launches++;
      }
      CK(cudaMemcpyAsync(s.goff + s.F, s.binOff + s.FB, 4, cudaMemcpyDeviceToDevice, st));
      const uint32_t nfine = 1u << s.shift;
      const unsigned sort_threads = nfine >= 1024 ? 1024 : 256;
      k_bin_sort_impl<<<s.FB, sort_threads, nfine * 4, st>>>(s.binOff, s.binIdx, s.binFine, s.shift, s.nbin, s.NB,
                                                              s.goff, s.sorted);
      launches++;
    } else {
      CK(cudaMemsetAsync(s.counts, 0, s.F * sizeof(uint32_t), st));
      if (n) {
        k_digit_counts<C><<<(unsigned)cdiv(n, 256), 256, 0, st>>>(scal, n, s.c_arg, s.nwin, ws, s.counts, s.err);
        launches++;
      }
      k_scan_reduce<<<(unsigned)s.ntiles, SCAN_THREADS, 0, st>>>(s.counts, s.F, s.tiles);
      k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, s.ntiles, s.goff + s.F);
      k_scan_apply<<<(unsigned)s.ntiles, SCAN_THREADS, 0, st>>>(s.counts, s.F, s.tiles, s.goff, s.cursor);
      launches += 3;
      if (n) {
        k_digit_scatter<C><<<(unsigned)cdiv(n, 256), 256, 0, st>>>(scal, n, s.c_arg, s.nwin, ws, istride, s.cursor, s.sorted);
        launches++;
      }
    }
    CK(cudaGetLastError());
    if (timed) CK(cudaEventRecord(s.ev[EV_SORT], st));
    // a4 front end: groups of 4 entries per bucket -> one affine point (batch-affine)
    const uint32_t* acc_pts = pts;
    const uint32_t* acc_goff = s.goff;
    if constexpr (kBaff) {
      if (s.baff) {
        k_group4_counts<<<(unsigned)cdiv(s.F, 256), 256, 0, st>>>(s.goff, s.F, s.c4);
        k_scan_reduce<<<(unsigned)s.ntiles, SCAN_THREADS, 0, st>>>(s.c4, s.F, s.tiles);
        k_scan_tiles<<<1, 1024, 0, st>>>(s.tiles, s.ntiles, s.goff4 + s.F);
        k_scan_apply<<<(unsigned)s.ntiles, SCAN_THREADS, 0, st>>>(s.c4, s.F, s.tiles, s.goff4, s.cursor4);
        k_baff2<C><<<s.baff_T / BAFF_NT, BAFF_NT, 0, st>>>(pts, s.sorted, s.goff, s.goff4, (uint32_t)s.F, s.baff_B,
                                                            s.out4, s.baff_scratch);
        launches += 5;
        CK(cudaGetLastError());
        acc_pts = s.out4;
        acc_goff = s.goff4;
      }
    }
    if (timed) CK(cudaEventRecord(s.ev[EV_BAFF], st));
    // Small n: the accumulation and reduce threads are few (C1: ~2.8 K accumulation threads =
    // 11 blocks of 256), and 8 warps of one SM then share its IMAD pipe while 137 SMs idle
    // (ncu: 144 us for 17 PACC per thread).  Halve the block size (down to one warp) until the
    // blocks cover the SMs.
    auto spread = [&](size_t threads, uint32_t nt) {
      uint32_t bs = nt;
      while (bs > 32 && cdiv(std::max<size_t>(threads, 1), bs) < (size_t)s.sms) bs >>= 1;
      return bs;
    };
    const uint32_t anb = spread(s.acc_threads, kAccSync ? ACC_SYNC_NT : 128);
    // a4: accumulate + fixup
#if MSM_ACC_SMEM
    k_accumulate_smem<C><<<(unsigned)cdiv(s.acc_threads, 128), 128, ACC_SLOTS * C::L * ACC_NT * 4, st>>>(pts, s.sorted, s.goff, (uint32_t)s.F,
#else
    if constexpr (kAccSync) {
      // (INIT and DIRECT instantiations only where they can run: each copy of this kernel
      // is ~100 KB of code and minutes of MNT4-753 compile time)
      if (C::L <= 13 && init) {
        if constexpr (C::L <= 13)
          k_accumulate_sync<C, false, true><<<(unsigned)cdiv(s.acc_threads, anb), anb, 0, st>>>(
              pts, s.sorted, s.goff, (uint32_t)s.F, s.buckets, s.carry_pts, s.carry_f, s.acc_threads, s.nlong);
      } else if (kBaff && s.baff) {
        if constexpr (kBaff)
          k_accumulate_sync<C, true><<<(unsigned)cdiv(s.acc_threads, anb), anb, 0, st>>>(
              acc_pts, s.sorted, acc_goff, (uint32_t)s.F, s.buckets, s.carry_pts, s.carry_f, s.acc_threads, s.nlong);
      } else
        k_accumulate_sync<C><<<(unsigned)cdiv(s.acc_threads, anb), anb, 0, st>>>(
            pts, s.sorted, s.goff, (uint32_t)s.F, s.buckets, s.carry_pts, s.carry_f, s.acc_threads, s.nlong);
    } else
      k_accumulate<C><<<(unsigned)cdiv(s.acc_threads, anb), anb, 0, st>>>(pts, s.sorted, s.goff, (uint32_t)s.F,
#endif
                                                                        s.buckets, s.carry_pts, s.carry_f, s.acc_threads,
                                                                        s.nlong);
    launches++;
    CK(cudaGetLastError());
    if (timed) CK(cudaEventRecord(s.ev[EV_ACC], st));
    k_fixup<C><<<(unsigned)cdiv(s.acc_threads, 128), 128, 0, st>>>(s.buckets, s.carry_pts, s.carry_f, s.acc_threads,
                                                                   s.nlong, s.longs);
    k_fixup_long<C><<<(unsigned)s.sms, FIX_THREADS, FIX_THREADS * XW_ * 4, st>>>(s.buckets, s.carry_pts, s.carry_f,
                                                                                s.acc_threads, s.nlong, s.longs);
    launches += 2;
    CK(cudaGetLastError());
    if (timed) CK(cudaEventRecord(s.ev[EV_FIX], st));
    if (!reduce) return launches;
    // a5: bucket reduce
    const uint32_t total = (uint32_t)s.nset * s.nseg;
    const uint32_t snb = MSM_SEG_SYNC ? (uint32_t)SEG_NT : spread(total, SEG_NT);
    if (s.seg_lat)
      k_bucket_segments<C, true><<<(unsigned)cdiv(total, snb), snb, 0, st>>>(
          s.buckets, red_goff, s.nset, s.NB, s.seg, s.nseg, (uint32_t)s.split_G, (uint32_t)s.split_g, s.segA);
    else
      k_bucket_segments<C, false><<<(unsigned)cdiv(total, snb), snb, 0, st>>>(
          s.buckets, red_goff, s.nset, s.NB, s.seg, s.nseg, (uint32_t)s.split_G, (uint32_t)s.split_g, s.segA);
    launches++;
    uint32_t nin = s.nseg;
    uint32_t* src = s.segA;
    uint32_t* dst = s.segB;
    while (nin > 1) {
      const uint32_t group = nin > 32 ? 32 : nin;
      const uint32_t nout = (uint32_t)cdiv(nin, group);
      uint32_t* out = nout == 1 ? s.W : dst;
#if MSM_SUM_WARP
      k_sum_groups_warp<C><<<(unsigned)cdiv((size_t)s.nset * nout * 32, 128), 128, 0, st>>>(src, nin, group, nout, s.nset, out);
#else
      k_sum_groups<C><<<(unsigned)cdiv((size_t)s.nset * nout, 128), 128, 0, st>>>(src, nin, group, nout, s.nset, out);
#endif
      launches++;
      nin = nout;
      std::swap(src, dst);
      if (nout == 1) { src = s.W; break; }
    }
    if (src != s.W) CK(cudaMemcpyAsync(s.W, src, (size_t)s.nset * XW_ * 4, cudaMemcpyDeviceToDevice, st));
    CK(cudaGetLastError());
    if (timed) CK(cudaEventRecord(s.ev[EV_RED], st));
    // a6: window combine
    k_window_combine<C><<<1, 32, 0, st>>>(s.W, s.nset, s.c, s.partial);
    launches++;
    CK(cudaGetLastError());
    if (timed) CK(cudaEventRecord(s.ev[EV_COMB], st));
    return launches;
  }

  void enqueue_finalize(const uint32_t* partials, int count, uint32_t* result, cudaStream_t st) override {
    k_finalize<C><<<1, 32, 0, st>>>(partials, count, result);
    CK(cudaGetLastError());
  }

  void gen_points(const uint32_t* e0, const uint32_t* delta, size_t n, uint32_t* out) override {
    uint32_t *g, *e, *d, *bases;
    dalloc(&g, 2 * C::L32);
    dalloc(&e, C::S);
    dalloc(&d, C::S);
    dalloc(&bases, 2 * XW_);
    try {
      CK(cudaMemcpy(g, C::G_h, 2 * C::L32 * 4, cudaMemcpyHostToDevice));
      CK(cudaMemcpy(e, e0, C::S * 4, cudaMemcpyHostToDevice));
      CK(cudaMemcpy(d, delta, C::S * 4, cudaMemcpyHostToDevice));
      k_gen_bases<C><<<1, 32>>>(g, e, d, bases);
      CK(cudaGetLastError());
      const uint32_t chunk = 64;
      const size_t threads = cdiv(n, chunk);
      if (threads) k_gen_points<C><<<(unsigned)cdiv(threads, 128), 128>>>(bases, n, chunk, out);
      CK(cudaGetLastError());
      CK(cudaDeviceSynchronize());
    } catch (...) {
      dfree(g); dfree(e); dfree(d); dfree(bases);
      throw;
    }
    dfree(g); dfree(e); dfree(d); dfree(bases);
  }

  void debug_field(int op, const uint32_t* a, const uint32_t* b, size_t n, uint32_t* out) override {
    uint32_t *da, *db, *dout;
    const size_t w = n * C::L32;
    dalloc(&da, w); dalloc(&db, w); dalloc(&dout, w);
    CK(cudaMemcpy(da, a, w * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(db, b, w * 4, cudaMemcpyHostToDevice));
    k_debug_field<C><<<(unsigned)cdiv(n, 128), 128>>>(op, da, db, n, dout);
    CK(cudaGetLastError());
    CK(cudaMemcpy(out, dout, w * 4, cudaMemcpyDeviceToHost));
    dfree(da); dfree(db); dfree(dout);
  }

  void debug_ec(int op, const uint32_t* P, const uint32_t* Q, const uint32_t* z, size_t n, uint32_t* out) override {
    uint32_t *dP, *dQ, *dz, *dout;
    const size_t w = n * 2 * C::L32;
    dalloc(&dP, w); dalloc(&dQ, w); dalloc(&dz, w); dalloc(&dout, w);
    CK(cudaMemcpy(dP, P, w * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dQ, Q, w * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dz, z, w * 4, cudaMemcpyHostToDevice));
    k_debug_ec<C><<<(unsigned)n, 1>>>(op, dP, dQ, dz, n, dout);  // one lane per warp: divergent EC paths
    CK(cudaGetLastError());
    CK(cudaMemcpy(out, dout, w * 4, cudaMemcpyDeviceToHost));
    dfree(dP); dfree(dQ); dfree(dz); dfree(dout);
  }

  void debug_digits(int c, const uint32_t* scal, size_t n, int32_t* out) override {
    const int nwin = num_windows(C::LAMBDA, c);
    uint32_t* ds;
    int32_t* dout;
    dalloc(&ds, n * C::S);
    dalloc(&dout, n * nwin);
    CK(cudaMemcpy(ds, scal, n * C::S * 4, cudaMemcpyHostToDevice));
    k_digits_debug<C><<<(unsigned)cdiv(n, 128), 128>>>(ds, n, c, nwin, dout);
    CK(cudaGetLastError());
    CK(cudaMemcpy(out, dout, n * nwin * 4, cudaMemcpyDeviceToHost));
    dfree(ds); dfree(dout);
  }

  long count_nonempty(Shard& s) override {
    unsigned long long* d;
    dalloc(&d, 1);
    CK(cudaMemsetAsync(d, 0, 8, s.stream));
    k_count_nonempty<<<(unsigned)cdiv(s.F, 256), 256, 0, s.stream>>>(s.goff, s.F, d);
    unsigned long long h = 0;
    CK(cudaMemcpyAsync(&h, d, 8, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaStreamSynchronize(s.stream));
    dfree(d);
    return (long)h;
  }

  void rand_scalars(Shard& s, uint32_t* out, size_t n, uint32_t seed) override {
    if (!n) return;
    k_rand_scalars<C><<<(unsigned)cdiv(n, 128), 128, 0, s.stream>>>(out, n, seed);
    CK(cudaGetLastError());
  }

  void to_affine(const uint32_t* in, size_t n, uint32_t* out, cudaStream_t st) override {
    if (!n) return;
    k_to_affine<C><<<(unsigned)cdiv(n, 64), 64, 0, st>>>(in, n, out);
    CK(cudaGetLastError());
  }
};

}  // namespace msmrt
