// Host runtime types shared by the C-ABI layer (engine.cu) and the per-curve kernel
// translation units (curve_*.cu).  Host C++ only.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../../include/msm.h"

namespace msmrt {

struct CudaError {
  int code;
};

#define CK(call)                                                                         \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess) {                                                             \
      if (getenv("MSM_DEBUG")) fprintf(stderr, "msm: %s -> %s (%s:%d)\n", #call,        \
                                       cudaGetErrorString(e_), __FILE__, __LINE__);      \
      throw ::msmrt::CudaError{e_ == cudaErrorMemoryAllocation ? MSM_ERR_OOM : MSM_ERR_CUDA}; \
    }                                                                                    \
  } while (0)

inline size_t cdiv(size_t a, size_t b) { return (a + b - 1) / b; }

template <class T>
void dalloc(T** p, size_t count) {
  *p = nullptr;
  if (count == 0) count = 1;
  CK(cudaMalloc((void**)p, count * sizeof(T)));
}
template <class T>
void dfree(T*& p) {
  if (p) cudaFree(p);
  p = nullptr;
}

enum { EV_START, EV_H2D, EV_SORT, EV_BAFF, EV_ACC, EV_FIX, EV_RED, EV_COMB, EV_END, EV_COUNT };

// One device's share of a context: its points, scratch and stream.
struct Shard {
  int dev = 0;
  size_t off = 0, n = 0;
  cudaStream_t stream = nullptr;
  cudaEvent_t ev[EV_COUNT] = {};
  // chunked host scalars: copy stream and one event per chunk (created on first use)
  cudaStream_t cstream = nullptr;
  cudaEvent_t cev[8] = {};
  int chunks_used = 1;
  // small-n launch path: a2..a6 captured once into a CUDA graph and replayed while the
  // configuration (gen) and the device scalar pointer stay the same (engine.cu)
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t gexec = nullptr;
  const uint32_t* g_scal = nullptr;
  const uint32_t* last_scal = nullptr;
  int gen = 0, g_gen = -1, g_launches = 0;
  // configuration (depends on c)
  int c = 0, nwin = 0;
  int pre = 0;         // precomputed window table in use (f3): one bucket set for all windows
  int nset = 0;        // bucket sets: nwin (pre = 0) or 1 (pre = 1)
  uint32_t NB = 0;     // (local) buckets per set incl. bucket 0 = 2^(c-1)/G + 1
  int split_G = 1, split_g = 0;  // f1 bucket split: part g of G
  int c_arg = 0;       // c | (G-1) << 8 | g << 16 for the digit kernels (for_each_digit)
  size_t F = 0;        // flat buckets = nset * NB
  uint32_t acc_threads = 0, slice = 0;
  uint32_t seg = 0, nseg = 0;
  int seg_lat = 0;     // bucket reduce with latency-mode products (small n)
  size_t ntiles = 0;
  // binned sort geometry (a3): flat bins fb = j*nbin + (b >> shift), FB = nwin*nbin
  int sort_mode = 0, shift = 0;  // effective a3 variant (1, 2, 3 or 4)
  uint32_t nbin = 0, FB = 0;
  size_t ntiles_bin = 0;
  // device buffers
  uint32_t *pts = nullptr, *scal = nullptr, *counts = nullptr, *goff = nullptr, *cursor = nullptr,
           *sorted = nullptr, *buckets = nullptr, *carry_pts = nullptr, *segA = nullptr, *segB = nullptr,
           *W = nullptr, *partial = nullptr, *partials = nullptr, *tiles = nullptr, *err = nullptr,
           *result = nullptr;
  int32_t* carry_f = nullptr;
  uint32_t* nlong = nullptr;   // k_fixup long-run list: count, and the runs' first carries
  uint32_t* longs = nullptr;
  int sms = 148;
  uint32_t *binCount = nullptr, *binOff = nullptr, *binCursor = nullptr, *binIdx = nullptr;
  uint16_t* binFine = nullptr;
  // three-level staged sort (sort3.cuh): key bits b1 + b2 + b3 >= bits(F - 1)
  int s3_b1 = 0, s3_b2 = 0, s3_b3 = 0;
  int s3_k16 = 0;  // P1 keys as u16 (b2 + b3 <= 16)
  uint32_t *s3Count = nullptr, *s3Off = nullptr, *s3Cursor = nullptr, *s3Sub = nullptr,
           *s3k1 = nullptr, *s3v1 = nullptr, *s3k2 = nullptr, *s3v2 = nullptr, *s3SubCount = nullptr,
           *s3SubCursor = nullptr, *s3Tiles = nullptr, *s3Big = nullptr;
  // two-pass cluster sort (sort4.cuh): bins of 2^s4_b2 flat buckets
  int s4_b2 = 0;
  uint32_t s4_NC1 = 0;
  uint32_t *s4Count = nullptr, *s4Off = nullptr, *s4Cursor = nullptr, *s4v = nullptr;
  uint16_t* s4k = nullptr;
  uint32_t* host_err = nullptr;  // pinned
  // f3 precomputation: table[j][i] = 2^(j c) P_i, affine device form,
  // [nwin][n][PW] words; built for window size table_c, kept across runs.
  uint32_t* table = nullptr;
  int table_c = 0;
  float table_ms = 0;
  // batch-affine front end of a4 (baff.cuh): groups of 4 entries per bucket folded into one
  // affine point (out4 [M4][PW], offsets goff4), then PACC over out4
  int baff = 0;
  uint32_t *c4 = nullptr, *goff4 = nullptr, *cursor4 = nullptr, *out4 = nullptr, *baff_scratch = nullptr;
  uint32_t baff_T = 0, baff_B = 0;
};

struct Options {
  int c = 0, threads = 0, seg = 0;
  int sort = 0;  // a3 variant: 0 auto, 1 direct global atomics (ablation), 2 two-level binned,
                 // 3 three-level staged (sort3.cuh), 4 two-pass cluster (sort4.cuh)
  int pre = 2;   // f3 precomputation: 0 off, 1 on, 2 auto (on when the table fits in memory)
  int split_G = 1, split_g = 0;  // f1: this context sums only buckets |d| = G*q + g
  int acc_mode = 2;  // a4: 0 PACC only, 1 batch-affine front end + PACC (ablation), 2 auto (= 0, measured faster)
  int chunks = 0;    // host-scalar H2D chunks per msm_run: 0 auto, 1 one copy, K >= 2 (engine.cu)
  int tuned_c = 0;   // window size measured best at context creation (small n, c auto; engine.cu)
};

// Per-curve kernels behind a virtual interface (one instance per curve, curve_*.cu).
struct CurveOps {
  virtual ~CurveOps() {}
  virtual int L32() const = 0;
  virtual int S() const = 0;
  virtual int lambda() const = 0;
  virtual int PW() const = 0;
  virtual int XW() const = 0;
  virtual void points_to_mont(Shard& s, const uint32_t* in_dev, size_t n) = 0;
  // (re)allocates the scratch for window size c; pre = 1 uses (and if needed builds) the
  // f3 precomputed table
  virtual void configure(const Options& o, Shard& s, int c, int pre) = 0;
  virtual void free_scratch(Shard& s) = 0;
  virtual void free_table(Shard& s) = 0;
  // enqueue a2..a6 on s.stream for the shard's scalars; the partial ends in s.partial.
  // Returns the number of kernels launched.
  virtual int enqueue_pipeline(Shard& s, const uint32_t* scal_dev, bool timed) = 0;
  // chunked host scalars: whether this shard's configuration supports it, and one chunk
  // (points [ibase, ibase + n) of the shard, scalars already on the device at scal_dev)
  virtual bool can_chunk(const Shard& s) const = 0;
  virtual int enqueue_chunk(Shard& s, const uint32_t* scal_dev, size_t n, size_t ibase, bool first, bool last,
                            bool timed) = 0;
  virtual void enqueue_finalize(const uint32_t* partials_dev, int count, uint32_t* result_dev, cudaStream_t st) = 0;
  virtual void gen_points(const uint32_t* e0, const uint32_t* delta, size_t n, uint32_t* out) = 0;
  virtual void debug_field(int op, const uint32_t* a, const uint32_t* b, size_t n, uint32_t* out) = 0;
  virtual void debug_ec(int op, const uint32_t* P, const uint32_t* Q, const uint32_t* z, size_t n, uint32_t* out) = 0;
  virtual void debug_digits(int c, const uint32_t* scal, size_t n, int32_t* out) = 0;
  virtual void to_affine(const uint32_t* in_dev, size_t n, uint32_t* out_dev, cudaStream_t st) = 0;
  virtual long count_nonempty(Shard& s) = 0;
  virtual bool has_baff() const = 0;
  virtual void rand_scalars(Shard& s, uint32_t* out_dev, size_t n, uint32_t seed) = 0;
};

inline int num_windows(int lambda, int c) { return lambda / c + 1; }

// weak: a development build (tools/build.py --dev) may link a subset of the curve TUs;
// a missing curve then reports MSM_ERR_CURVE.  The release build links all four.
__attribute__((weak)) CurveOps* make_ops_bn254();
__attribute__((weak)) CurveOps* make_ops_bls12_377();
__attribute__((weak)) CurveOps* make_ops_bls12_381();
__attribute__((weak)) CurveOps* make_ops_mnt4_753();

}  // namespace msmrt
