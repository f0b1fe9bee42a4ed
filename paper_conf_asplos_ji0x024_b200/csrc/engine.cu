// Host runtime and C ABI of libmsm.so (include/msm.h).
//
// One context = n points sharded over G devices (contiguous shards).  Per
// device the MSM pipeline of SURVEY.md §3.3 runs on the shard's own stream:
//   H2D scalars -> k_digit_counts -> scan (3 kernels) -> k_digit_scatter      (a2, a3)
//   -> k_accumulate -> k_fixup                                                (a4)
//   -> k_bucket_segments -> k_sum_groups (x levels)                           (a5)
//   -> k_window_combine                                                       (a6)
// then the G partial XYZZ points meet on device 0 (peer copies) for k_finalize (a7).
// For one-process-per-GPU jobs the caller gathers msm_run_partial() outputs itself
// (torch.distributed / NCCL) and calls msm_finalize().
#include <algorithm>
#include <cmath>
#include <cstring>
#include <memory>
#include <mutex>
#include <new>
#include <thread>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "runtime.h"

using namespace msmrt;

static thread_local int g_last_error = MSM_OK;

struct msm_context {
  int curve = 0;
  size_t n = 0;
  int ngpus = 1;
  std::vector<Shard> shards;
  Options opt;
  msm_stats stats{};
  CurveOps* ops = nullptr;
  int launches = 0;
  // pipelined submit/wait (single shard): ring of MSM_MAX_INFLIGHT result slots
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied = nullptr;
  cudaEvent_t ev_done[MSM_MAX_INFLIGHT] = {};
  uint32_t* d_result[MSM_MAX_INFLIGHT] = {};
  uint32_t* h_result = nullptr;  // pinned [MSM_MAX_INFLIGHT][2*L32 + 1] (last word: error flags)
  long next_ticket = 0, next_wait = 0;
  uint32_t* h_run = nullptr;     // pinned [2*L32 + 1]: msm_run's result and error word (one D2H)
  bool stats_pending = false;    // msm_stats of the last run are read lazily (msm_get_stats)
  int graph = 1;                 // MSM_OPT_GRAPH: small-n CUDA-graph replay allowed
  bool last_graphed = false;     // the last run replayed a graph: no per-stage events
};

namespace {

bool is_device_ptr(const void* p, int* dev) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
    if (dev) *dev = a.device;
    return true;
  }
  return false;
}

// NVTX range for the duration of an ABI call (visible in nsys / ncu --nvtx timelines; the
// header-only NVTX v3 API costs nothing when no tool is attached).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// Restores the caller's current device when an ABI call returns (the library switches
// devices per shard; the caller's torch/CUDA state must not change under it).
struct DeviceGuard {
  int dev = -1;
  DeviceGuard() {
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); dev = -1; }
  }
  ~DeviceGuard() {
    if (dev >= 0) cudaSetDevice(dev);
  }
};

// Orders `stream` (on device `dev`) after all work already submitted to the legacy default
// stream of device `src_dev` — where torch (default stream) and synchronous CUDA calls put
// the producers of device-resident inputs.  Inputs written on other non-blocking streams
// must be complete before the call (include/msm.h, "Ordering").
std::mutex g_order_mu;
cudaEvent_t g_order_ev[64] = {};
void order_after_legacy(int src_dev, int dev, cudaStream_t stream) {
  if (src_dev < 0 || src_dev >= 64) return;
  std::lock_guard<std::mutex> lk(g_order_mu);
  CK(cudaSetDevice(src_dev));
  if (!g_order_ev[src_dev]) CK(cudaEventCreateWithFlags(&g_order_ev[src_dev], cudaEventDisableTiming));
  CK(cudaEventRecord(g_order_ev[src_dev], cudaStreamLegacy));
  CK(cudaSetDevice(dev));
  CK(cudaStreamWaitEvent(stream, g_order_ev[src_dev], 0));
}

// Pippenger cost model, in units of one PACC (10 field mults):
//   per window n PACC ("ceil(lambda/s)(N + 2^{s+1})"), plus a sort cost per
//   entry, plus the bucket reduce (2 PADD per bucket, measured ~4.4 PACC-equivalents per
//   bucket on B200, r01 bench) over 2^(c-1) buckets per bucket set.  With the f3 table all
//   windows share one bucket set, so larger c pays off.
//   Each bucket-reduce segment (>= 4 buckets, at most one per resident thread, ~37.9 K on
//   148 SMs) also ends with a small-scalar multiplication of ~c doublings + adds on one
//   thread (~2.3 PACC-equivalents per bit): a per-segment latency term that makes large c
//   lose at small n (C2, n = 2^20: c = 16 beats c = 20, r01 sweep).
//   bucket_cost: reduce cost per bucket in units of one entry's accumulation — 4.4 for the
//   8..13-limb curves.  For MNT4-753 the reduce per bucket is dearer (out-of-line 27-limb
//   PADD: 52.7 ms for 2^22 buckets) but the accumulation per entry grows as c shrinks
//   (r02, n = 2^22: 1.79 / 1.96 / 2.27 ns per entry at c = 23 / 22 / 21; step 304.7 /
//   330.1 / 373.8 ms), which this model does not capture; 3.5 keeps c = 23 there.
double plan_cost(size_t n, int lambda, int c, bool pre, double bucket_cost = 4.4) {
  const double nwin = num_windows(lambda, c);
  const double sets = pre ? 1.0 : nwin;
  const double buckets = sets * std::ldexp(1.0, c - 1);
  const double segs = std::min(buckets / 4.0, 37888.0);
  return nwin * (double)n * 1.12 + buckets * bucket_cost + segs * c * 2.3;
}

// device bytes of the f3 table and of the per-run scratch for window size c
size_t table_bytes(size_t n, int lambda, int c, int PW) { return (size_t)num_windows(lambda, c) * n * PW * 4; }
size_t scratch_bytes(size_t n, int lambda, int c, int XW, bool pre) {
  const size_t nwin = num_windows(lambda, c);
  const size_t sets = pre ? 1 : nwin;
  const size_t NB = ((size_t)1 << (c - 1)) + 1;
  // sort + sorted entries (~22 B/entry), bucket set(s), and the batch-affine front end:
  // ceil(count/4) folded points per bucket (<= entries/4 + buckets, ~28 B/entry at PW = 28)
  // plus its per-thread batch scratch (<= 2 GB)
  return n * nwin * (22 + (size_t)XW * 4 / 7) + sets * NB * ((size_t)XW * 4 + 12 + (size_t)XW * 2) +
         ((size_t)1 << 28) + ((size_t)2 << 30);
}

// Chooses (c, pre) for one shard: opt.c / opt.pre when fixed; otherwise the cheapest
// configuration whose device memory fits (the f3 table needs nwin*n < 2^31 entries too).
void plan_shard(const Options& o, const Shard& s, int lambda, int PW, int XW, int* c_out, int* pre_out,
                double bucket_cost) {
  size_t fr = 0, tot = 0;
  CK(cudaSetDevice(s.dev));
  CK(cudaMemGetInfo(&fr, &tot));
  size_t held = 0;  // this shard's current table and scratch are freed before reallocation
  if (s.table) held += table_bytes(s.n, lambda, s.table_c, PW);
  if (s.sorted) held += scratch_bytes(s.n, lambda, s.c, XW, s.pre);
  const double budget = 0.92 * (double)(fr + held) - (double)(2ull << 30);
  auto fits = [&](int c, bool pre) {
    double need = (double)scratch_bytes(s.n, lambda, c, XW, pre);
    if (pre) need += (double)table_bytes(s.n, lambda, c, PW);
    return need <= budget;
  };
  // Entry counts (goff, cursors, M) are 32-bit and a sorted entry holds its point index in
  // 31 bits: (table row j)*n + i with the f3 table, i without it.  Every c whose nwin*n
  // entries could overflow either is skipped (n < 2^31 is checked at create).
  auto indexable = [&](int c) { return (double)num_windows(lambda, c) * (double)s.n < 2147483647.0; };
  const int cmin = o.c > 0 ? o.c : 4, cmax = o.c > 0 ? o.c : 24;
  double best = 1e300;
  int bc = o.c > 0 ? o.c : 8, bp = 0;
  bool any_fit = false;
  for (int pass = 0; pass < 2 && best == 1e300; pass++) {
    // pass 0 requires the memory fit of every candidate; pass 1 (nothing fits) lets an
    // explicitly chosen configuration try its allocation (MSM_ERR_OOM if it fails)
    for (int pre = 0; pre <= 1; pre++) {
      if ((o.pre == 0 && pre) || (o.pre == 1 && !pre)) continue;
      for (int c = cmin; c <= cmax; c++) {
        if (o.c <= 0 && c > 22 && !pre) continue;  // per-window bucket sets beyond 2^21
        if (!indexable(c)) continue;
        const bool fit = fits(c, pre);
        any_fit |= fit;
        if (pass == 0 && !fit && (o.pre == 2 || o.c <= 0)) continue;
        const double cost = s.n == 0 ? (double)c : plan_cost(s.n, lambda, c, pre, bucket_cost);
        if (cost < best) { best = cost; bc = c; bp = pre; }
      }
    }
    if (o.pre == 2 && o.c <= 0) break;  // fully automatic: only configurations that fit
  }
  if (best == 1e300) throw CudaError{any_fit ? MSM_ERR_ARG : MSM_ERR_OOM};
  *c_out = bc;
  *pre_out = bp;
}

CurveOps* ops_for(int curve) {
  switch (curve) {
    case MSM_BN254: return make_ops_bn254 ? make_ops_bn254() : nullptr;
    case MSM_BLS12_377: return make_ops_bls12_377 ? make_ops_bls12_377() : nullptr;
    case MSM_BLS12_381: return make_ops_bls12_381 ? make_ops_bls12_381() : nullptr;
    case MSM_MNT4_753: return make_ops_mnt4_753 ? make_ops_mnt4_753() : nullptr;
    default: return nullptr;
  }
}

void destroy_shard(CurveOps* ops, Shard& s) {
  cudaSetDevice(s.dev);
  if (s.stream) cudaStreamSynchronize(s.stream);
  if (ops) {
    ops->free_scratch(s);
    ops->free_table(s);
  }
  dfree(s.pts); dfree(s.scal); dfree(s.partial); dfree(s.partials); dfree(s.err); dfree(s.result);
  if (s.host_err) cudaFreeHost(s.host_err);
  s.host_err = nullptr;
  for (auto& e : s.ev)
    if (e) { cudaEventDestroy(e); e = nullptr; }
  for (auto& e : s.cev)
    if (e) { cudaEventDestroy(e); e = nullptr; }
  if (s.gexec) cudaGraphExecDestroy(s.gexec);
  if (s.graph) cudaGraphDestroy(s.graph);
  s.gexec = nullptr;
  s.graph = nullptr;
  if (s.cstream) cudaStreamSynchronize(s.cstream), cudaStreamDestroy(s.cstream);
  s.cstream = nullptr;
  if (s.stream) cudaStreamDestroy(s.stream);
  s.stream = nullptr;
}

int apply_window_bits(msm_context* ctx) {
  Options o = ctx->opt;
  // the tuned c is a timing result, so it may differ between processes: the f1 bucket split
  // needs the same c (the same digits) in every part, so it keeps the deterministic model
  if (o.c == 0 && o.tuned_c > 0 && o.split_G == 1) o.c = o.tuned_c;
  for (auto& s : ctx->shards) {
    int c = 0, pre = 0;
    plan_shard(o, s, ctx->ops->lambda(), ctx->ops->PW(), ctx->ops->XW(), &c, &pre,
               ctx->ops->L32() > 12 ? 3.5 : 4.4);
    ctx->ops->configure(o, s, c, pre);
    s.gen++;  // invalidates the captured graph
  }
  return MSM_OK;
}

// Small n (2^10 <= n <= 2^17, one shard, c automatic): the cost model is a throughput
// model, but here the MSM is a chain of dependent EC operations whose length depends on c in
// ways it does not capture (the top window's lambda mod c bits pile n extra entries into a
// few buckets -> long carry runs; the reduce's weight multiplication grows with c).  A
// sweep (profiles/r02/small_n_c_sweep.txt: BN254 2^10 best c = 6 at 0.54 ms vs the model's
// c = 10 at 0.69 ms; 2^12 c = 5; 2^14 c = 16; BLS12-381 2^16 c = 8) is non-monotonic, so the
// context measures instead: each candidate c runs twice on hashed scalars and the fastest
// second run wins (FFTW-style planning; ~0.1 s at creation).  MSM_NO_AUTOTUNE=1 disables it.
void autotune_c(msm_context* ctx) {
  Shard& s = ctx->shards[0];
  std::vector<int> cands = {5, 6, 7, 8, 10, 12, 14, 16};
  if (std::find(cands.begin(), cands.end(), s.c) == cands.end()) cands.push_back(s.c);
  ctx->ops->rand_scalars(s, s.scal, s.n, 0x5eed1234u);
  float best = 1e30f;
  int bc = s.c;
  for (int c : cands) {
    ctx->opt.tuned_c = c;
    apply_window_bits(ctx);
    float ms = 0;
    for (int rep = 0; rep < 2; rep++) {
      CK(cudaMemsetAsync(s.err, 0, 4, s.stream));
      CK(cudaEventRecord(s.ev[EV_START], s.stream));
      ctx->ops->enqueue_pipeline(s, s.scal, false);
      ctx->ops->enqueue_finalize(s.partial, 1, s.result, s.stream);
      CK(cudaEventRecord(s.ev[EV_END], s.stream));
      CK(cudaEventSynchronize(s.ev[EV_END]));
      CK(cudaEventElapsedTime(&ms, s.ev[EV_START], s.ev[EV_END]));
    }
    if (ms < best) { best = ms; bc = c; }
  }
  ctx->opt.tuned_c = bc;
  apply_window_bits(ctx);
}

// Small MSMs are launch-bound (C1: ~25 kernels for ~0.1 ms of GPU work), so for shards of
// <= 2^17 points with device scalars on the shard's own device, a2..a6 are captured into a
// CUDA graph the second time the same scalar buffer is seen, and replayed after that.
constexpr size_t GRAPH_MAX_N = (size_t)1 << 17;
// A replayed graph has no per-stage events: the stage events are recorded after it (the
// stats then show the whole a2..a6 time as sort_ms and 0 for the later stages), which also
// keeps EV_SORT valid for msm_submit's copy-stream ordering.
void graph_launch(Shard& s, bool timed) {
  if (timed) CK(cudaEventRecord(s.ev[EV_H2D], s.stream));
  CK(cudaGraphLaunch(s.gexec, s.stream));
  if (timed)
    for (int e : {EV_SORT, EV_BAFF, EV_ACC, EV_FIX, EV_RED, EV_COMB}) CK(cudaEventRecord(s.ev[e], s.stream));
}
int enqueue_graphed(msm_context* ctx, Shard& s, const uint32_t* sc, bool timed) {
  const bool same = sc == s.last_scal;
  s.last_scal = sc;
  if (s.gexec && s.g_gen == s.gen && s.g_scal == sc) {
    graph_launch(s, timed);
    return s.g_launches;
  }
  if (!same) return ctx->ops->enqueue_pipeline(s, sc, timed);
  if (s.gexec) cudaGraphExecDestroy(s.gexec);
  if (s.graph) cudaGraphDestroy(s.graph);
  s.gexec = nullptr;
  s.graph = nullptr;
  CK(cudaStreamBeginCapture(s.stream, cudaStreamCaptureModeThreadLocal));
  int launched = 0;
  try {
    launched = ctx->ops->enqueue_pipeline(s, sc, false);  // no event nodes in the graph
  } catch (...) {
    cudaGraph_t g = nullptr;
    cudaStreamEndCapture(s.stream, &g);
    if (g) cudaGraphDestroy(g);
    throw;
  }
  CK(cudaStreamEndCapture(s.stream, &s.graph));
  CK(cudaGraphInstantiate(&s.gexec, s.graph, 0));
  s.g_gen = s.gen;
  s.g_scal = sc;
  s.g_launches = launched;
  graph_launch(s, timed);
  return launched;
}

// scalar pointer for shard s: device-resident on the shard's device -> use directly,
// otherwise copy into s.scal (H2D or peer).
const uint32_t* stage_scalars(msm_context* ctx, Shard& s, const uint32_t* scalars, bool is_dev, int src_dev) {
  const size_t S = ctx->ops->S();
  const uint32_t* src = scalars + s.off * S;
  const size_t bytes = s.n * S * 4;
  if (s.n == 0) return s.scal;
  if (is_dev && src_dev == s.dev && ((uintptr_t)src % 16) == 0) return src;
  if (is_dev) {
    if (src_dev == s.dev) CK(cudaMemcpyAsync(s.scal, src, bytes, cudaMemcpyDeviceToDevice, s.stream));
    else CK(cudaMemcpyPeerAsync(s.scal, s.dev, src, src_dev, bytes, s.stream));
  } else {
    CK(cudaMemcpyAsync(s.scal, src, bytes, cudaMemcpyHostToDevice, s.stream));
  }
  return s.scal;
}

// Host scalars in K chunks (the bucket work "can be efficiently pipelined"
// with the transfers): chunk k's H2D runs on the shard's copy stream while the compute
// stream sorts and accumulates chunk k-1 into the bucket set.  Chunk sizes grow by 4x
// (n/4^(K-1), 3n/4^(K-1), 12n/4^(K-1), ...): the GPU work of a chunk (~6 GB/s of scalars
// at 2^26) outlasts the next chunk's copy (25-50 GB/s), so only the first, smallest copy
// stays on the critical path.  Each later chunk costs one extra PACC per non-empty bucket
// (INIT accumulation from the stored bucket).
int h2d_chunks(msm_context* ctx, const Shard& s) {
  const int want = ctx->opt.chunks;
  if (want == 1 || s.n == 0 || !ctx->ops->can_chunk(s)) return 1;
  // auto: from 2^22 points (BLS12-377 2^24: 103.8 -> 99.0 ms; at 2^20 it is neutral,
  // 9.28 vs 9.32 ms, profiles/r02b/configs.jsonl)
  if (want == 0) return s.n >= ((size_t)1 << 22) ? 3 : 1;
  return std::min(want, 8);
}

int run_chunked(msm_context* ctx, Shard& s, const uint32_t* host_src, int K, bool timed) {
  const size_t S = ctx->ops->S();
  if (!s.cstream) CK(cudaStreamCreateWithFlags(&s.cstream, cudaStreamNonBlocking));
  for (int k = 0; k < K; k++)
    if (!s.cev[k]) CK(cudaEventCreateWithFlags(&s.cev[k], cudaEventDisableTiming));
  // the copy stream must not overwrite s.scal while an earlier MSM on s.stream reads it
  CK(cudaEventRecord(s.cev[0], s.stream));
  CK(cudaStreamWaitEvent(s.cstream, s.cev[0], 0));
  const double T = std::pow(4.0, K - 1);
  int launched = 0;
  size_t lo = 0;
  for (int k = 0; k < K; k++) {
    const size_t hi = k == K - 1 ? s.n : std::min(s.n, (size_t)std::llround((double)s.n * std::pow(4.0, k) / T));
    if (hi < lo) continue;
    CK(cudaMemcpyAsync(s.scal + lo * S, host_src + lo * S, (hi - lo) * S * 4, cudaMemcpyHostToDevice, s.cstream));
    CK(cudaEventRecord(s.cev[k], s.cstream));
    CK(cudaStreamWaitEvent(s.stream, s.cev[k], 0));
    launched += ctx->ops->enqueue_chunk(s, s.scal + lo * S, hi - lo, lo, k == 0, k == K - 1, timed && k == K - 1);
    lo = hi;
  }
  return launched;
}

int check_errors(msm_context* ctx) {
  uint32_t e = 0;
  for (auto& s : ctx->shards) {
    CK(cudaSetDevice(s.dev));
    CK(cudaMemcpyAsync(s.host_err, s.err, 4, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaStreamSynchronize(s.stream));
    e |= *s.host_err;
  }
  if (e & 4u) return MSM_ERR_SCALAR;
  if (e & 3u) return MSM_ERR_POINT;
  return MSM_OK;
}

// runs a2..a6 on every shard; partials end in shard0.partials[g]
int run_all(msm_context* ctx, const uint32_t* scalars, bool gather_to_dev0) {
  int src_dev = -1;
  const bool is_dev = ctx->n ? is_device_ptr(scalars, &src_dev) : false;
  ctx->launches = 0;
  const int XW = ctx->ops->XW();
  Shard& s0 = ctx->shards[0];
  const size_t G = ctx->shards.size();
  std::vector<int> launched(G, 0), rc(G, MSM_OK);
  auto one = [&](size_t g) {
    Shard& s = ctx->shards[g];
    try {
      CK(cudaSetDevice(s.dev));
      const bool timed = g == 0;
      if (is_dev) order_after_legacy(src_dev, s.dev, s.stream);
      if (timed) CK(cudaEventRecord(s.ev[EV_START], s.stream));
      CK(cudaMemsetAsync(s.err, 0, 4, s.stream));
      const int K = is_dev ? 1 : h2d_chunks(ctx, s);
      s.chunks_used = K;
      if (K > 1) {
        NvtxRange nr("chunked H2D + a2..a6 (shard)");
        launched[g] = run_chunked(ctx, s, scalars + s.off * ctx->ops->S(), K, timed);
      } else {
        const uint32_t* sc = stage_scalars(ctx, s, scalars, is_dev, src_dev);
        NvtxRange nr("enqueue a2..a6 (shard)");
        static const bool no_graph = getenv("MSM_NO_GRAPH") != nullptr;  // A/B
        bool graphed = false;
        if (!no_graph && ctx->graph && is_dev && src_dev == s.dev && s.n <= GRAPH_MAX_N && sc != s.scal) {
          launched[g] = enqueue_graphed(ctx, s, sc, timed);
          graphed = s.gexec && s.g_scal == sc && s.g_gen == s.gen;
        } else {
          launched[g] = ctx->ops->enqueue_pipeline(s, sc, timed);
        }
        if (g == 0) ctx->last_graphed = graphed;
      }
    } catch (const CudaError& e) {
      rc[g] = e.code;
    } catch (...) {
      rc[g] = MSM_ERR_CUDA;
    }
  };
  if (G > 1 && ctx->n && !is_dev) {
    // host scalars: one host thread per shard, so the (possibly pageable, hence
    // host-synchronous) H2D copies of the shards run in parallel over their own links
    std::vector<std::thread> th;
    for (size_t g = 0; g < G; g++) th.emplace_back(one, g);
    for (auto& t : th) t.join();
  } else {
    for (size_t g = 0; g < G; g++) one(g);
  }
  for (size_t g = 0; g < G; g++) {
    if (rc[g] != MSM_OK) throw CudaError{rc[g]};
    ctx->launches += launched[g];
  }
  if (gather_to_dev0) {
    for (size_t g = 0; g < ctx->shards.size(); g++) {
      Shard& s = ctx->shards[g];
      if (g == 0) {
        CK(cudaSetDevice(s0.dev));
        CK(cudaMemcpyAsync(s0.partials, s0.partial, XW * 4, cudaMemcpyDeviceToDevice, s0.stream));
      } else {
        CK(cudaSetDevice(s.dev));
        CK(cudaEventRecord(s.ev[EV_END], s.stream));
        CK(cudaSetDevice(s0.dev));
        CK(cudaStreamWaitEvent(s0.stream, s.ev[EV_END], 0));
        CK(cudaMemcpyPeerAsync(s0.partials + g * XW, s0.dev, s.partial, s.dev, XW * 4, s0.stream));
      }
    }
  }
  return MSM_OK;
}

void collect_stats(msm_context* ctx) {
  Shard& s = ctx->shards[0];
  CK(cudaSetDevice(s.dev));
  CK(cudaEventSynchronize(s.ev[EV_END]));
  auto el = [&](int a, int b) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, s.ev[a], s.ev[b]) != cudaSuccess) { cudaGetLastError(); ms = -1; }
    return ms;
  };
  msm_stats& st = ctx->stats;
  st.h2d_ms = el(EV_START, EV_H2D);
  st.sort_ms = el(EV_H2D, EV_SORT);
  st.accumulate_ms = el(EV_SORT, EV_ACC);
  st.baff_ms = el(EV_SORT, EV_BAFF);
  st.fixup_ms = el(EV_ACC, EV_FIX);
  st.reduce_ms = el(EV_FIX, EV_RED);
  st.combine_ms = el(EV_RED, EV_COMB);
  if (ctx->last_graphed)  // a replayed graph has no per-stage events: a2..a6 unknown (-1)
    st.sort_ms = st.accumulate_ms = st.baff_ms = st.fixup_ms = st.reduce_ms = st.combine_ms = -1.0f;
  st.finalize_ms = el(EV_COMB, EV_END);
  st.total_ms = el(EV_START, EV_END);
  st.window_bits = s.c;
  st.nwin = s.nwin;
  st.acc_threads = (int)s.acc_threads;
  st.acc_launches = ctx->launches;
  uint32_t M = 0;
  cudaMemcpy(&M, s.goff + s.F, 4, cudaMemcpyDeviceToHost);
  st.entries = M;
  st.precompute = s.pre;
  st.table_ms = s.table_ms;
  st.baff = s.baff;
  uint32_t M4 = M;
  if (s.baff) cudaMemcpy(&M4, s.goff4 + s.F, 4, cudaMemcpyDeviceToHost);
  st.entries_acc = M4;
}

// Every ABI call that touches a device runs through guarded(): C++ exceptions become
// MSM_ERR_* codes and the caller's current device is restored on return.
template <class F>
int guarded(F&& f) {
  DeviceGuard guard;
  try {
    return f();
  } catch (const CudaError& e) {
    return e.code;
  } catch (const std::bad_alloc&) {
    return MSM_ERR_OOM;
  } catch (...) {
    return MSM_ERR_CUDA;
  }
}

// small per-device scratch for msm_finalize (kept across calls; no cudaMalloc when timed)
struct FinalizeScratch {
  uint32_t* partials = nullptr;
  size_t cap = 0;
  uint32_t* result = nullptr;
  cudaStream_t stream = nullptr;
};
std::mutex g_fin_mu;
FinalizeScratch g_fin[64];

}  // namespace

// =========================================================================================
extern "C" {

int msm_field_words(int curve) {
  CurveOps* o = ops_for(curve);
  return o ? o->L32() : MSM_ERR_CURVE;
}
int msm_scalar_words(int curve) {
  CurveOps* o = ops_for(curve);
  return o ? o->S() : MSM_ERR_CURVE;
}
int msm_scalar_bits(int curve) {
  CurveOps* o = ops_for(curve);
  return o ? o->lambda() : MSM_ERR_CURVE;
}
int msm_partial_words(int curve) {
  CurveOps* o = ops_for(curve);
  return o ? o->XW() : MSM_ERR_CURVE;
}

int msm_device_count(void) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

int msm_last_error(void) { return g_last_error; }

const char* msm_error_string(int code) {
  switch (code) {
    case MSM_OK: return "ok";
    case MSM_ERR_ARG: return "invalid argument";
    case MSM_ERR_CURVE: return "unknown curve";
    case MSM_ERR_CUDA: return "CUDA error";
    case MSM_ERR_OOM: return "device out of memory";
    case MSM_ERR_NCCL: return "NCCL error";
    case MSM_ERR_POINT: return "point not on curve or not canonical";
    case MSM_ERR_SCALAR: return "scalar >= r";
    case MSM_ERR_UNIMPLEMENTED: return "unimplemented";
    case MSM_ERR_NO_DEVICE: return "no (or not enough) CUDA devices";
    default: return "unknown error";
  }
}

msm_context* msm_context_create(int curve, const uint32_t* points, size_t n, int ngpus) {
  g_last_error = MSM_OK;
  const int ndev = msm_device_count();
  if (ndev < 1) { g_last_error = MSM_ERR_NO_DEVICE; return nullptr; }
  if (ngpus < 1 || ngpus > 64) { g_last_error = MSM_ERR_ARG; return nullptr; }
  if (ngpus > ndev) { g_last_error = MSM_ERR_NO_DEVICE; return nullptr; }
  // shard g on device (current + g) mod ndev: a one-process-per-GPU caller that selected
  // cuda:LOCAL_RANK gets its context there
  int base = 0;
  if (cudaGetDevice(&base) != cudaSuccess) { cudaGetLastError(); base = 0; }
  int devs[64];
  for (int g = 0; g < ngpus; g++) devs[g] = (base + g) % ndev;
  return msm_context_create_on(curve, points, n, ngpus, devs);
}

msm_context* msm_context_create_on(int curve, const uint32_t* points, size_t n, int ngpus, const int* devices) {
  NvtxRange nvtx_("msm_context_create");
  g_last_error = MSM_OK;
  DeviceGuard guard;
  CurveOps* ops = ops_for(curve);
  if (!ops) { g_last_error = MSM_ERR_CURVE; return nullptr; }
  if (ngpus < 1 || ngpus > 64 || !devices || (n > 0 && !points) || n >= 0x80000000ull) { g_last_error = MSM_ERR_ARG; return nullptr; }
  const int ndev = msm_device_count();
  if (ndev < 1) { g_last_error = MSM_ERR_NO_DEVICE; return nullptr; }
  for (int g = 0; g < ngpus; g++)
    if (devices[g] < 0 || devices[g] >= ndev) { g_last_error = MSM_ERR_NO_DEVICE; return nullptr; }
  auto* ctx = new msm_context();
  ctx->curve = curve;
  ctx->n = n;
  ctx->ngpus = ngpus;
  ctx->ops = ops;
  ctx->shards.resize(ngpus);
  int rc = guarded([&]() -> int {
    int src_dev = -1;
    const bool in_dev = n ? is_device_ptr(points, &src_dev) : false;
    const size_t pw_in = 2 * (size_t)ops->L32();
    for (int g = 0; g < ngpus; g++) {
      Shard& s = ctx->shards[g];
      s.dev = devices[g];
      s.off = (size_t)((unsigned __int128)n * g / ngpus);
      s.n = (size_t)((unsigned __int128)n * (g + 1) / ngpus) - s.off;
      CK(cudaSetDevice(s.dev));
      CK(cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking));
      for (auto& e : s.ev) CK(cudaEventCreate(&e));
      dalloc(&s.pts, s.n * ops->PW());
      dalloc(&s.scal, s.n * ops->S());
      dalloc(&s.partial, ops->XW());
      dalloc(&s.err, 1);
      dalloc(&s.result, 2 * ops->L32());
      if (g == 0) dalloc(&s.partials, (size_t)ngpus * ops->XW());
      CK(cudaMallocHost((void**)&s.host_err, 4));
      CK(cudaMemsetAsync(s.err, 0, 4, s.stream));
      if (s.n) {
        const uint32_t* src = points + s.off * pw_in;
        if (in_dev) order_after_legacy(src_dev, s.dev, s.stream);
        if (in_dev && src_dev == s.dev) {
          ops->points_to_mont(s, src, s.n);
        } else {
          uint32_t* tmp;
          dalloc(&tmp, s.n * pw_in);
          if (in_dev) CK(cudaMemcpyPeerAsync(tmp, s.dev, src, src_dev, s.n * pw_in * 4, s.stream));
          else CK(cudaMemcpyAsync(tmp, src, s.n * pw_in * 4, cudaMemcpyHostToDevice, s.stream));
          ops->points_to_mont(s, tmp, s.n);
          CK(cudaStreamSynchronize(s.stream));
          dfree(tmp);
        }
      }
    }
    int e = check_errors(ctx);
    if (e != MSM_OK) return e;
    if (ngpus > 1) {
      for (int a = 0; a < ngpus; a++)
        for (int b = 0; b < ngpus; b++) {
          const int da = ctx->shards[a].dev, db = ctx->shards[b].dev;
          if (da == db) continue;  // logical shards on one device
          int ok = 0;
          cudaDeviceCanAccessPeer(&ok, da, db);
          if (ok) {
            cudaSetDevice(da);
            cudaError_t pe = cudaDeviceEnablePeerAccess(db, 0);
            if (pe != cudaSuccess) cudaGetLastError();  // already enabled
          }
        }
    }
    const int e2 = apply_window_bits(ctx);
    if (e2 != MSM_OK) return e2;
    static const bool no_tune = getenv("MSM_NO_AUTOTUNE") != nullptr;
    if (!no_tune && ngpus == 1 && n >= ((size_t)1 << 10) && n <= ((size_t)1 << 17)) autotune_c(ctx);
    return MSM_OK;
  });
  if (rc != MSM_OK) {
    g_last_error = rc;
    for (auto& s : ctx->shards) destroy_shard(ops, s);
    delete ctx;
    return nullptr;
  }
  return ctx;
}

void msm_context_destroy(msm_context* ctx) {
  if (!ctx) return;
  DeviceGuard guard;
  if (ctx->copy_stream) {
    cudaSetDevice(ctx->shards[0].dev);
    cudaStreamSynchronize(ctx->shards[0].stream);
    cudaStreamSynchronize(ctx->copy_stream);
    cudaStreamDestroy(ctx->copy_stream);
    cudaEventDestroy(ctx->ev_copied);
    for (int q = 0; q < MSM_MAX_INFLIGHT; q++) {
      cudaEventDestroy(ctx->ev_done[q]);
      dfree(ctx->d_result[q]);
    }
    cudaFreeHost(ctx->h_result);
  }
  if (ctx->h_run) cudaFreeHost(ctx->h_run);
  for (auto& s : ctx->shards) destroy_shard(ctx->ops, s);
  delete ctx;
}

int msm_run(msm_context* ctx, const uint32_t* scalars, uint32_t* result) {
  NvtxRange nvtx_("msm_run");
  if (!ctx || !result || (ctx->n && !scalars)) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    run_all(ctx, scalars, true);
    Shard& s0 = ctx->shards[0];
    CK(cudaSetDevice(s0.dev));
    ctx->ops->enqueue_finalize(s0.partials, (int)ctx->shards.size(), s0.result, s0.stream);
    ctx->launches++;
    CK(cudaEventRecord(s0.ev[EV_END], s0.stream));
    ctx->stats_pending = true;
    const int L32 = ctx->ops->L32();
    if (ctx->shards.size() == 1) {  // one round trip: result and error word together
      if (!ctx->h_run) CK(cudaMallocHost((void**)&ctx->h_run, (2 * 24 + 1) * 4));
      CK(cudaMemcpyAsync(ctx->h_run, s0.result, 2 * L32 * 4, cudaMemcpyDeviceToHost, s0.stream));
      CK(cudaMemcpyAsync(ctx->h_run + 2 * L32, s0.err, 4, cudaMemcpyDeviceToHost, s0.stream));
      CK(cudaStreamSynchronize(s0.stream));
      const uint32_t e = ctx->h_run[2 * L32];
      if (e & 4u) return MSM_ERR_SCALAR;
      if (e & 3u) return MSM_ERR_POINT;
      std::memcpy(result, ctx->h_run, 2 * L32 * 4);
      return MSM_OK;
    }
    const int e = check_errors(ctx);
    if (e != MSM_OK) return e;
    CK(cudaMemcpy(result, s0.result, 2 * L32 * 4, cudaMemcpyDeviceToHost));
    return MSM_OK;
  });
}

int msm_run_partial(msm_context* ctx, const uint32_t* scalars, uint32_t* partial) {
  NvtxRange nvtx_("msm_run_partial");
  if (!ctx || !partial || (ctx->n && !scalars) || ctx->shards.size() != 1) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    run_all(ctx, scalars, false);
    Shard& s0 = ctx->shards[0];
    CK(cudaSetDevice(s0.dev));
    CK(cudaEventRecord(s0.ev[EV_END], s0.stream));
    const int e = check_errors(ctx);
    ctx->stats_pending = true;
    if (e != MSM_OK) return e;
    int pdev = -1;
    if (is_device_ptr(partial, &pdev)) {
      if (pdev == s0.dev) CK(cudaMemcpyAsync(partial, s0.partial, ctx->ops->XW() * 4, cudaMemcpyDeviceToDevice, s0.stream));
      else CK(cudaMemcpyPeerAsync(partial, pdev, s0.partial, s0.dev, ctx->ops->XW() * 4, s0.stream));
      CK(cudaStreamSynchronize(s0.stream));
    } else {
      CK(cudaMemcpy(partial, s0.partial, ctx->ops->XW() * 4, cudaMemcpyDeviceToHost));
    }
    return MSM_OK;
  });
}

long msm_submit(msm_context* ctx, const uint32_t* scalars) {
  NvtxRange nvtx_("msm_submit");
  if (!ctx || (ctx->n && !scalars) || ctx->shards.size() != 1) return MSM_ERR_ARG;
  if (ctx->next_ticket - ctx->next_wait >= MSM_MAX_INFLIGHT) return MSM_ERR_ARG;
  const int rc = guarded([&]() -> int {
    Shard& s = ctx->shards[0];
    const int L32 = ctx->ops->L32();
    CK(cudaSetDevice(s.dev));
    if (!ctx->copy_stream) {
      CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
      CK(cudaEventCreateWithFlags(&ctx->ev_copied, cudaEventDisableTiming));
      for (int q = 0; q < MSM_MAX_INFLIGHT; q++) {
        CK(cudaEventCreateWithFlags(&ctx->ev_done[q], cudaEventDisableTiming));
        dalloc(&ctx->d_result[q], 2 * L32);
      }
      CK(cudaMallocHost((void**)&ctx->h_result, MSM_MAX_INFLIGHT * (2 * L32 + 1) * 4));
    }
    const int q = (int)(ctx->next_ticket % MSM_MAX_INFLIGHT);
    const size_t bytes = s.n * (size_t)ctx->ops->S() * 4;
    int src_dev = -1;
    const bool is_dev = bytes && is_device_ptr(scalars, &src_dev);
    // an MSM submitted into an empty pipeline has no earlier MSM to hide its upload behind:
    // it takes the chunked upload of msm_run (§6a) instead of one copy before its sort
    const int K = (!is_dev && ctx->next_wait == ctx->next_ticket) ? h2d_chunks(ctx, s) : 1;
    s.chunks_used = K;
    if (K > 1) {
      // s.scal is free: nothing is in flight (the chunks' copies follow s.stream's work)
      CK(cudaEventRecord(s.ev[EV_START], s.stream));
      CK(cudaMemsetAsync(s.err, 0, 4, s.stream));
      ctx->launches = run_chunked(ctx, s, scalars + s.off * ctx->ops->S(), K, true);
    } else {
      // copy stream: wait until the previous MSM's sort has consumed s.scal (EV_SORT is
      // re-recorded by every pipeline, so this waits on the latest one), then H2D
      CK(cudaStreamWaitEvent(ctx->copy_stream, s.ev[EV_SORT], 0));
      if (is_dev) order_after_legacy(src_dev, s.dev, ctx->copy_stream);
      if (bytes) CK(cudaMemcpyAsync(s.scal, scalars + s.off * ctx->ops->S(), bytes, cudaMemcpyDefault, ctx->copy_stream));
      CK(cudaEventRecord(ctx->ev_copied, ctx->copy_stream));
      // compute stream: a2..a6 on the staged scalars, then finalise into result slot q
      CK(cudaStreamWaitEvent(s.stream, ctx->ev_copied, 0));
      CK(cudaEventRecord(s.ev[EV_START], s.stream));
      CK(cudaMemsetAsync(s.err, 0, 4, s.stream));
      ctx->launches = ctx->ops->enqueue_pipeline(s, s.scal, true);
    }
    ctx->ops->enqueue_finalize(s.partial, 1, ctx->d_result[q], s.stream);
    ctx->launches++;
    CK(cudaEventRecord(s.ev[EV_END], s.stream));
    uint32_t* h = ctx->h_result + q * (2 * L32 + 1);
    CK(cudaMemcpyAsync(h, ctx->d_result[q], 2 * L32 * 4, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaMemcpyAsync(h + 2 * L32, s.err, 4, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaEventRecord(ctx->ev_done[q], s.stream));
    return MSM_OK;
  });
  return rc == MSM_OK ? ctx->next_ticket++ : (long)rc;
}

int msm_wait(msm_context* ctx, long ticket, uint32_t* result) {
  if (!ctx || !result || ticket != ctx->next_wait || ticket >= ctx->next_ticket) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    Shard& s = ctx->shards[0];
    const int L32 = ctx->ops->L32();
    const int q = (int)(ticket % MSM_MAX_INFLIGHT);
    CK(cudaSetDevice(s.dev));
    CK(cudaEventSynchronize(ctx->ev_done[q]));
    ctx->next_wait++;
    if (ticket + 1 == ctx->next_ticket) {
      collect_stats(ctx);
      ctx->stats_pending = false;
    }
    const uint32_t* h = ctx->h_result + q * (2 * L32 + 1);
    const uint32_t e = h[2 * L32];
    if (e & 4u) return MSM_ERR_SCALAR;
    if (e & 3u) return MSM_ERR_POINT;
    std::memcpy(result, h, 2 * L32 * 4);
    return MSM_OK;
  });
}

int msm_finalize(int curve, const uint32_t* partials, int count, uint32_t* result) {
  NvtxRange nvtx_("msm_finalize");
  CurveOps* ops = ops_for(curve);
  if (!ops) return MSM_ERR_CURVE;
  if (count < 0 || (count > 0 && !partials) || !result) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    if (dev < 0 || dev >= 64) return MSM_ERR_ARG;
    std::lock_guard<std::mutex> lk(g_fin_mu);
    FinalizeScratch& fs = g_fin[dev];
    const size_t words = (size_t)std::max(count, 1) * ops->XW();
    if (!fs.stream) CK(cudaStreamCreateWithFlags(&fs.stream, cudaStreamNonBlocking));
    if (fs.cap < words) {
      dfree(fs.partials);
      dalloc(&fs.partials, words);
      fs.cap = words;
    }
    if (!fs.result) dalloc(&fs.result, 2 * 24);
    const uint32_t* src = fs.partials;
    int pdev = -1;
    if (count > 0) {
      if (is_device_ptr(partials, &pdev)) order_after_legacy(pdev, dev, fs.stream);
      if (pdev == dev) src = partials;
      else CK(cudaMemcpyAsync(fs.partials, partials, (size_t)count * ops->XW() * 4,
                              pdev >= 0 ? cudaMemcpyDefault : cudaMemcpyHostToDevice, fs.stream));
    }
    ops->enqueue_finalize(src, count, fs.result, fs.stream);
    CK(cudaMemcpyAsync(result, fs.result, 2 * ops->L32() * 4, cudaMemcpyDeviceToHost, fs.stream));
    CK(cudaStreamSynchronize(fs.stream));
    return MSM_OK;
  });
}

int msm_set_option(msm_context* ctx, int key, long value) {
  if (!ctx) return MSM_ERR_ARG;
  switch (key) {
    case MSM_OPT_WINDOW_BITS:
      if (value != 0 && (value < 2 || value > 24)) return MSM_ERR_ARG;
      ctx->opt.c = (int)value;
      break;
    case MSM_OPT_ACC_THREADS:
      if (value < 0) return MSM_ERR_ARG;
      ctx->opt.threads = (int)value;
      break;
    case MSM_OPT_SEG_LEN:
      if (value < 0 || value > (1 << 20)) return MSM_ERR_ARG;
      ctx->opt.seg = (int)value;
      break;
    case MSM_OPT_SORT:
      if (value < 0 || value > 4) return MSM_ERR_ARG;
      ctx->opt.sort = (int)value;
      break;
    case MSM_OPT_PRECOMPUTE:
      if (value < 0 || value > 2) return MSM_ERR_ARG;
      ctx->opt.pre = (int)value;
      break;
    case MSM_OPT_SPLIT_PARTS:
      if (value < 1 || value > 256) return MSM_ERR_ARG;
      ctx->opt.split_G = (int)value;
      if (ctx->opt.split_g >= ctx->opt.split_G) ctx->opt.split_g = 0;
      break;
    case MSM_OPT_SPLIT_INDEX:
      if (value < 0 || value >= ctx->opt.split_G) return MSM_ERR_ARG;
      ctx->opt.split_g = (int)value;
      break;
    case MSM_OPT_ACC_MODE:
      if (value < 0 || value > 2) return MSM_ERR_ARG;
      if (value == 1 && !ctx->ops->has_baff()) return MSM_ERR_UNIMPLEMENTED;
      ctx->opt.acc_mode = (int)value;
      break;
    case MSM_OPT_H2D_CHUNKS:
      if (value < 0 || value > 8) return MSM_ERR_ARG;
      ctx->opt.chunks = (int)value;
      return MSM_OK;  // no reconfiguration
    case MSM_OPT_GRAPH:
      if (value < 0 || value > 1) return MSM_ERR_ARG;
      ctx->graph = (int)value;
      return MSM_OK;
    default:
      return MSM_ERR_ARG;
  }
  return guarded([&]() -> int { return apply_window_bits(ctx); });
}

long msm_get_option(msm_context* ctx, int key) {
  if (!ctx) return MSM_ERR_ARG;
  switch (key) {
    case MSM_OPT_WINDOW_BITS: return ctx->shards[0].c;
    case MSM_OPT_ACC_THREADS: return ctx->shards[0].acc_threads;
    case MSM_OPT_SEG_LEN: return ctx->shards[0].seg;
    case MSM_OPT_SORT: return ctx->shards[0].sort_mode;
    case MSM_OPT_NWIN: return ctx->shards[0].nwin;
    case MSM_OPT_PRECOMPUTE: return ctx->shards[0].pre;
    case MSM_OPT_NSETS: return ctx->shards[0].nset;
    case MSM_OPT_SPLIT_PARTS: return ctx->opt.split_G;
    case MSM_OPT_SPLIT_INDEX: return ctx->opt.split_g;
    case MSM_OPT_ACC_MODE: return ctx->shards[0].baff;
    case MSM_OPT_H2D_CHUNKS: return ctx->shards[0].chunks_used;
    case MSM_OPT_GRAPH: return ctx->graph;
    case MSM_OPT_DEVICE: return ctx->shards[0].dev;
    case MSM_OPT_NGPUS: return (long)ctx->shards.size();
    case MSM_OPT_NONEMPTY: {
      long v = MSM_ERR_CUDA;
      guarded([&]() -> int { CK(cudaSetDevice(ctx->shards[0].dev)); v = ctx->ops->count_nonempty(ctx->shards[0]); return MSM_OK; });
      return v;
    }
    default: return MSM_ERR_ARG;
  }
}

int msm_get_stats(const msm_context* ctx, msm_stats* out) {
  if (!ctx || !out) return MSM_ERR_ARG;
  if (ctx->stats_pending) {  // read the events and counters of the last run now, not in msm_run
    msm_context* c = const_cast<msm_context*>(ctx);
    const int rc = guarded([&]() -> int {
      collect_stats(c);
      return MSM_OK;
    });
    if (rc != MSM_OK) return rc;
    c->stats_pending = false;
  }
  *out = ctx->stats;
  return MSM_OK;
}

int msm_shard_info(const msm_context* ctx, int g, int* device, size_t* offset, size_t* count) {
  if (!ctx || g < 0 || g >= (int)ctx->shards.size()) return MSM_ERR_ARG;
  const Shard& s = ctx->shards[g];
  if (device) *device = s.dev;
  if (offset) *offset = s.off;
  if (count) *count = s.n;
  return MSM_OK;
}

void* msm_get_stream(msm_context* ctx, int dev) {
  if (!ctx || dev < 0 || dev >= (int)ctx->shards.size()) return nullptr;
  return (void*)ctx->shards[dev].stream;
}

int msm_gen_points(int curve, const uint32_t* e0, const uint32_t* delta, size_t n, uint32_t* out) {
  CurveOps* ops = ops_for(curve);
  if (!ops) return MSM_ERR_CURVE;
  if (!e0 || !delta || (n && !out)) return MSM_ERR_ARG;
  if (n && !is_device_ptr(out, nullptr)) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    ops->gen_points(e0, delta, n, out);
    return MSM_OK;
  });
}

int msm_debug_field(int curve, int op, const uint32_t* a, const uint32_t* b, size_t n, uint32_t* out) {
  CurveOps* ops = ops_for(curve);
  if (!ops) return MSM_ERR_CURVE;
  if (!a || !b || !out || op < 0 || op > 8) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    ops->debug_field(op, a, b, n, out);
    return MSM_OK;
  });
}

int msm_debug_ec(int curve, int op, const uint32_t* P, const uint32_t* Q, const uint32_t* z, size_t n, uint32_t* out) {
  CurveOps* ops = ops_for(curve);
  if (!ops) return MSM_ERR_CURVE;
  if (!P || !Q || !z || !out || op < 0 || op > 2) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    ops->debug_ec(op, P, Q, z, n, out);
    return MSM_OK;
  });
}

int msm_debug_digits(int curve, int c, const uint32_t* scalars, size_t n, int32_t* out) {
  CurveOps* ops = ops_for(curve);
  if (!ops) return MSM_ERR_CURVE;
  if (!scalars || !out || c < 2 || c > 30) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    ops->debug_digits(c, scalars, n, out);
    return MSM_OK;
  });
}

int msm_debug_windows(msm_context* ctx, const uint32_t* scalars, uint32_t* windows, uint32_t* buckets) {
  if (!ctx || !windows || (ctx->n && !scalars) || ctx->shards.size() != 1) return MSM_ERR_ARG;
  return guarded([&]() -> int {
    run_all(ctx, scalars, false);
    Shard& s = ctx->shards[0];
    CK(cudaSetDevice(s.dev));
    CK(cudaEventRecord(s.ev[EV_END], s.stream));
    int e = check_errors(ctx);
    if (e != MSM_OK) return e;
    const int L32 = ctx->ops->L32();
    uint32_t* dout;
    dalloc(&dout, (size_t)s.nset * 2 * L32);
    ctx->ops->to_affine(s.W, s.nset, dout, s.stream);
    CK(cudaMemcpyAsync(windows, dout, (size_t)s.nset * 2 * L32 * 4, cudaMemcpyDeviceToHost, s.stream));
    CK(cudaStreamSynchronize(s.stream));
    dfree(dout);
    if (buckets) {
      std::vector<uint32_t> goff(s.F + 1);
      CK(cudaMemcpy(goff.data(), s.goff, (s.F + 1) * 4, cudaMemcpyDeviceToHost));
      dalloc(&dout, s.F * 2 * L32);
      ctx->ops->to_affine(s.buckets, s.F, dout, s.stream);
      CK(cudaMemcpyAsync(buckets, dout, s.F * 2 * L32 * 4, cudaMemcpyDeviceToHost, s.stream));
      CK(cudaStreamSynchronize(s.stream));
      dfree(dout);
      for (size_t f = 0; f < s.F; f++)
        if (goff[f + 1] == goff[f]) std::memset(buckets + f * 2 * L32, 0, 2 * L32 * 4);
    }
    return MSM_OK;
  });
}

}  // extern "C"
