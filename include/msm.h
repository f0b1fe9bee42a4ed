/*
 * msm.h — C ABI of the B200-native multi-scalar multiplication library (libmsm.so).
 *
 * Operation (§2.2): given fixed curve points P_i and per-call scalars k_i,
 *     Q = sum_{i<n} k_i * P_i      in G1 of the selected curve,
 * computed by Pippenger's bucket method (§2.3, :141-143) with signed c-bit
 * windows, a per-window bucket counting sort (§3.2.1, Alg. 3), XYZZ bucket
 * accumulation (Alg. 4, §3.2.2), bucket reduce and window combine,
 * points sharded over GPUs with the partial results gathered and added.
 *
 * Encoding (all integers are arrays of little-endian 32-bit words):
 *   base-field element   L32 = msm_field_words(curve) words, canonical (< p)
 *   affine point         2*L32 words: x then y.  (0, 0) encodes the point at infinity O
 *                        (it is on none of the four curves because b != 0).  A point with
 *                        y = 0 (order 2; it exists on BLS12-377: (p-1, 0)) is outside the
 *                        prime-order subgroup and rejected with MSM_ERR_POINT.
 *   scalar               S = msm_scalar_words(curve) words, canonical (< r)
 *   result               2*L32 words, canonical affine; O -> (0, 0)
 *   partial (XYZZ)       msm_partial_words(curve) words: the library's internal projective
 *                        form (Montgomery radix-2^W limbs); only meaningful as input to
 *                        msm_finalize of the same curve.
 * Word counts: BN254 L32=8 S=8; BLS12-377 12/8; BLS12-381 12/8; MNT4-753 24/24.
 *
 * Pointers: a pointer argument documented "host or device" is classified with
 * cudaPointerGetAttributes; device pointers must be 16-byte aligned.  The library never
 * keeps a caller pointer past the call that receives it.
 *
 * Errors: every int-returning call returns MSM_OK (0) or a negative MSM_ERR_* code; no
 * C++ exception or abort crosses the ABI.  Create returns NULL on failure and the code is
 * available from msm_last_error() (thread-local).  After MSM_ERR_SCALAR or MSM_ERR_POINT
 * the context stays usable; after MSM_ERR_CUDA it should be destroyed.
 *
 * Threading: one call at a time per context; distinct contexts are independent.
 *
 * Devices: every call restores the caller's current CUDA device before it returns.  A
 * context's shard g lives on device (current device at create + g) mod device-count, so a
 * one-process-per-GPU caller that selected cuda:LOCAL_RANK gets its context there;
 * msm_context_create_on takes an explicit device per shard.
 *
 * Ordering of device-resident inputs: before reading a device pointer argument the
 * library orders its own (non-blocking) streams after all work already submitted to the
 * legacy default stream of the pointer's device — where torch's default stream and
 * synchronous CUDA calls run.  Inputs produced on other non-blocking streams must be
 * complete (synchronised by the caller) before the call.  Calls return only after their
 * device outputs are written (msm_submit: results are read through msm_wait).
 */
#ifndef MSM_H
#define MSM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { MSM_BN254 = 0, MSM_BLS12_377 = 1, MSM_BLS12_381 = 2, MSM_MNT4_753 = 3 } msm_curve;

enum {
  MSM_OK = 0,
  MSM_ERR_ARG = -1,           /* NULL pointer, bad size or option                       */
  MSM_ERR_CURVE = -2,         /* unknown curve id                                       */
  MSM_ERR_CUDA = -3,          /* CUDA runtime error                                     */
  MSM_ERR_OOM = -4,           /* device allocation failed                               */
  MSM_ERR_NCCL = -5,          /* reserved: the library itself makes no NCCL calls; the
                                 one-process-per-GPU gather runs in the caller's process
                                 group (paper_conf_asplos_ji0x024_b200/dist.py)           */
  MSM_ERR_POINT = -6,         /* an input point is not on the curve or not canonical    */
  MSM_ERR_SCALAR = -7,        /* a scalar is >= r                                       */
  MSM_ERR_UNIMPLEMENTED = -8,
  MSM_ERR_NO_DEVICE = -9      /* no CUDA device / fewer devices than requested          */
};

/* Options for msm_set_option / msm_get_option. */
enum {
  MSM_OPT_WINDOW_BITS = 1,    /* c in [2, 24]; 0 = automatic (cost model). Reallocates scratch. */
  MSM_OPT_ACC_THREADS = 2,    /* accumulation threads per device; 0 = automatic            */
  MSM_OPT_SEG_LEN = 3,        /* buckets per bucket-reduce segment; 0 = automatic          */
  MSM_OPT_SORT = 4,           /* a3 variant: 0 = auto (default: 3 for >= 2^21 entries, else 2),
                                 1 = direct global atomics (ablation), 2 = two-level binned,
                                 3 = three-level staged (coalesced runs), 4 = two-pass
                                 thread-block-cluster sort (ablation: half the HBM traffic of
                                 3, slower on B200); get returns 1..4          */
  MSM_OPT_PRECOMPUTE = 5,     /* f3 window table 2^(jc) P_i: 0 off, 1 on,
                                 2 auto (default: on when the table fits in device memory).
                                 With it all windows share one bucket set; building the table
                                 costs ~c*nwin doublings per point at create / option change;
                                 get returns the mode in use (0/1).                          */
  MSM_OPT_SPLIT_PARTS = 6,    /* f1 bucket split (§3.2.2: "splits the buckets
                                 into GPUs-per-window parts"): G in [1, 256], default 1.  With
                                 G > 1 this context sums only the buckets |d| = G*q + g
                                 (g = MSM_OPT_SPLIT_INDEX) of every bucket set, over ALL n points
                                 and scalars; msm_run_partial then returns that part's share and
                                 msm_finalize over the G parts' partials gives the MSM.  The
                                 interleaved (b mod G) assignment balances the parts even though
                                 the top window's digits sit in low buckets.                  */
  MSM_OPT_SPLIT_INDEX = 7,    /* f1: this context's part g in [0, G), default 0               */
  MSM_OPT_ACC_MODE = 8,       /* a4 bucket accumulation: 0 = PACC only (Alg. 4 per entry),
                                 1 = batch-affine front end (groups of 4 entries of a bucket
                                 folded into one affine point by pairwise additions sharing
                                 one inversion per batch, Montgomery's trick) then PACC,
                                 2 = auto (default: 0 — on B200 the front end's affine glue and
                                 per-batch inversion made it 1.8x slower; mode 1
                                 exists for BN254 and BLS12-377/381 as an ablation);
                                 get returns the mode in use (0/1)                           */
  MSM_OPT_H2D_CHUNKS = 9,     /* host scalars in msm_run / msm_run_partial: copy them in K
                                 chunks of growing size (n/4^(K-1), 3n/4^(K-1), 12n/4^(K-1),
                                 ...) on a copy stream, each sorted and accumulated INTO the
                                 bucket set while the next one uploads ("can be
                                 efficiently pipelined"); 0 = auto (default: K = 3 for
                                 n >= 2^22 per shard where supported: BN254, BLS12-377/381 with
                                 the staged or cluster sort), 1 = one copy before the MSM,
                                 2..8 = K.  Device scalars are never chunked.  Get returns the
                                 K used by the last run on shard 0.  No reconfiguration.      */
  MSM_OPT_GRAPH = 10,         /* 1 (default) = shards of <= 2^17 points with device scalars
                                 replay a2..a6 as a CUDA graph once the same scalar buffer is
                                 seen twice (the stage times of such runs read -1 in
                                 msm_stats, the total stays valid); 0 = always launch kernels */
  MSM_OPT_NWIN = 101,         /* (get only) number of windows floor(lambda/c) + 1           */
  MSM_OPT_NSETS = 103,        /* (get only) bucket sets: nwin, or 1 with the f3 table        */
  MSM_OPT_NONEMPTY = 102,     /* (get only) non-empty buckets of the last run on shard 0    */
  MSM_OPT_DEVICE = 104,       /* (get only) CUDA device of shard 0 (msm_shard_info: any shard) */
  MSM_OPT_NGPUS = 105         /* (get only) number of shards G                              */
};

/* Per-stage device times of the last msm_run on device 0 (CUDA events), milliseconds. */
typedef struct {
  float h2d_ms;         /* scalar upload (0 for device-resident scalars)   */
  float sort_ms;        /* a2+a3: digits, histogram, scan, scatter         */
  float accumulate_ms;  /* a4: bucket accumulation (k_accumulate)          */
  float fixup_ms;       /* a4: boundary partial fix-up (k_fixup)           */
  float reduce_ms;      /* a5: bucket reduce                               */
  float combine_ms;     /* a6: window combine                              */
  float finalize_ms;    /* a7: gather + final add + normalisation          */
  float total_ms;       /* whole msm_run on device 0                       */
  int window_bits;      /* c used                                          */
  int nwin;             /* windows                                         */
  int acc_threads;      /* threads of k_accumulate                         */
  int acc_launches;     /* kernels launched by the last run (all devices)  */
  uint64_t entries;     /* sorted (bucket, point) entries = PACC + bucket starts, device 0 */
  int precompute;       /* f3 table in use on device 0                     */
  float table_ms;       /* time of the last f3 table build on device 0     */
  float baff_ms;        /* a4 batch-affine front end (part of accumulate_ms) */
  int baff;             /* batch-affine front end in use                   */
  uint64_t entries_acc; /* points entering the PACC stage (= entries without the front end) */
} msm_stats;

typedef struct msm_context msm_context;

/* Sizes of the encodings above (negative MSM_ERR_CURVE for an unknown curve). */
int msm_field_words(int curve);
int msm_scalar_words(int curve);
int msm_scalar_bits(int curve);    /* lambda = bit length of r (Table 1) */
int msm_partial_words(int curve);

/* Number of visible CUDA devices (0 when none). */
int msm_device_count(void);

/*
 * Create a context holding n points sharded over devices 0..ngpus-1 in contiguous shards
 * [floor(g*n/G), floor((g+1)*n/G)).  `points` (host or device, n*2*L32 words) is copied,
 * converted to the device representation and checked on the curve; the caller keeps
 * ownership.  n may be 0.  All scratch for msm_run is allocated here.
 * Returns NULL on error (msm_last_error(): MSM_ERR_ARG/CURVE/NO_DEVICE/OOM/CUDA/POINT).
 */
msm_context* msm_context_create(int curve, const uint32_t* points, size_t n, int ngpus);

/*
 * As msm_context_create with an explicit CUDA device per shard: devices[g] in
 * [0, msm_device_count()).  A device may repeat: several shards then share it ("logical
 * shards" — each with its own stream and scratch, the gather a same-device copy); this is
 * how the multi-shard path (per-shard pipelines, cross-shard gather of the partials,
 * final add) is exercised on a one-GPU machine.
 * Returns NULL on error (msm_last_error(): also MSM_ERR_NO_DEVICE for a bad device id).
 */
msm_context* msm_context_create_on(int curve, const uint32_t* points, size_t n, int ngpus, const int* devices);

/* Shard g of the context: its device and its contiguous point range [offset, offset+count). */
int msm_shard_info(const msm_context* ctx, int g, int* device, size_t* offset, size_t* count);

/* NULL-safe; frees all device memory and streams of the context. */
void msm_context_destroy(msm_context* ctx);

/*
 * Q = sum k_i P_i.  `scalars`: n*S words, host or device.  Each shard reads its slice
 * [offset, offset+count): in place when it is on the shard's device (16-B aligned),
 * otherwise by a peer (NVLink) or host copy; host slices are uploaded by one host thread
 * per shard in parallel.  The G partial sums then meet on shard 0's device (peer copies
 * of 4L words each — the gather of PAPER.md:163) for the final add and normalisation.
 * `result`: host buffer of 2*L32 words (written only on MSM_OK).
 * Synchronous.  Returns MSM_OK, MSM_ERR_SCALAR (some k_i >= r), MSM_ERR_ARG, MSM_ERR_CUDA.
 */
int msm_run(msm_context* ctx, const uint32_t* scalars, uint32_t* result);

/*
 * The per-process half of a multi-process MSM (one process per GPU, ngpus == 1 contexts):
 * computes this context's partial sum sum_{i in shard} k_i P_i and writes it in XYZZ form
 * (msm_partial_words words) to `partial` (host or device).  Synchronous.
 */
int msm_run_partial(msm_context* ctx, const uint32_t* scalars, uint32_t* partial);

/*
 * Adds `count` XYZZ partials (host or device, count*msm_partial_words words) and writes
 * the canonical affine result to the host buffer `result`.  Runs on the current device.
 */
int msm_finalize(int curve, const uint32_t* partials, int count, uint32_t* result);

/*
 * Pipelined MSMs on one context (ngpus == 1), for a stream of MSMs over the same points
 * (the proving workload): msm_submit enqueues one MSM — H2D copy of its
 * scalars on a copy stream, the a2..a7 kernels on the compute stream — and returns a
 * ticket (>= 0) without waiting.  The copy of MSM t+1's scalars starts as soon as MSM t's
 * sort stage has consumed the device scalar buffer, so it overlaps MSM t's accumulation.
 * msm_wait(ctx, ticket, result) blocks until MSM `ticket` is done and writes its canonical
 * affine result (2*L32 host words).  At most MSM_MAX_INFLIGHT tickets may be outstanding
 * (submitted, not yet waited for); tickets must be waited for in submission order.
 * `scalars`: host (pinned memory copies at full PCIe rate) or device; the caller keeps the
 * buffer valid and unmodified until msm_wait of that ticket returns.
 * Errors: msm_submit returns MSM_ERR_ARG (NULL, ngpus > 1, too many outstanding) or a CUDA
 * code; msm_wait returns MSM_ERR_ARG (not the oldest outstanding ticket), MSM_ERR_SCALAR
 * (some k_i >= r: no result written; later tickets are unaffected) or a CUDA code.
 * Statistics (msm_get_stats) describe the most recently waited-for MSM when it was also
 * the most recently submitted one.
 */
#define MSM_MAX_INFLIGHT 2
long msm_submit(msm_context* ctx, const uint32_t* scalars);
int msm_wait(msm_context* ctx, long ticket, uint32_t* result);

int msm_set_option(msm_context* ctx, int key, long value);
long msm_get_option(msm_context* ctx, int key);
int msm_get_stats(const msm_context* ctx, msm_stats* out);

/* cudaStream_t of device `dev` of the context (as void*), for event timing by callers. */
void* msm_get_stream(msm_context* ctx, int dev);

int msm_last_error(void);
const char* msm_error_string(int code);

/*
 * Synthetic input generator (not on the MSM path; used by bench.py and large tests):
 * writes P_i = (e0 + i*delta) * G, i < n, as canonical affine words to `out` (device
 * pointer, n*2*L32 words) on the current device.  e0, delta: S words each (host).
 */
int msm_gen_points(int curve, const uint32_t* e0, const uint32_t* delta, size_t n, uint32_t* out);

/*
 * Test-only entry points (host buffers; run on the current device; synchronous).
 *   msm_debug_field: op 0 mul, 1 sqr, 2 add, 3 sub, 4 inv (Fermat), 5 neg, 6 inv (binary
 *     extended Euclid, the one the final normalisation uses), 7 a*b + b*a and 8 a*b + a*a
 *     (sum of two products under one Montgomery reduction, fmul_sum) on n canonical elements
 *     a[i], b[i] (L32 words each); out[i] canonical (inv of 0 is 0 for op 6).
 *   msm_debug_ec: op 0 acc (P + Q via Alg. 4 with P in XYZZ scaled by z1), 1 add (Alg. 1,
 *     both scaled by z1/z2), 2 dbl; P, Q affine (2*L32 words, (0,0) = O); z: 2*L32 words
 *     per element (z1, z2 non-zero canonical); out: affine.
 *   msm_debug_digits: signed digits, out[i*nwin + j] (int32), nwin = floor(lambda/c)+1.
 *   msm_debug_windows: runs msm_run's pipeline on the context (ngpus == 1) and writes the
 *     per-set sums W_s = sum_b b*B_{s,b} (nsets = msm_get_option(MSM_OPT_NSETS) affine
 *     points: the window sums W_j without the f3 table, the whole MSM with it) to `windows`;
 *     if `buckets` is non-NULL also the bucket sums B_{s,b} for b = 0..2^(c-1)
 *     (nsets*(2^(c-1)+1) affine points, O where empty).
 */
int msm_debug_field(int curve, int op, const uint32_t* a, const uint32_t* b, size_t n, uint32_t* out);
int msm_debug_ec(int curve, int op, const uint32_t* P, const uint32_t* Q, const uint32_t* z, size_t n,
                 uint32_t* out);
int msm_debug_digits(int curve, int c, const uint32_t* scalars, size_t n, int32_t* out);
int msm_debug_windows(msm_context* ctx, const uint32_t* scalars, uint32_t* windows, uint32_t* buckets);

#ifdef __cplusplus
}
#endif

#endif /* MSM_H */
