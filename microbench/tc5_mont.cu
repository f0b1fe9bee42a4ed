// f2 on Blackwell tensor cores (§4.3): the m x p
// half of Montgomery multiplication (Alg. 2 line 4) on tcgen05.mma .kind::i8 with s32
// accumulators in TMEM, against the same product on IMAD.WIDE (BLS12-381).
//
// The paper puts m*n on 8-bit tensor-core MMAs with the constant modulus as matB (P:277:
// practical only because matB is constant) and compacts the column sums afterwards
// (P:279-283).  Here, per CTA of 128 threads (one 381-bit product per thread):
//   A   = the 128 threads' m values as bytes, 128 x 64 (K-major, canonical no-swizzle
//         layout: 8-row x 16-byte core matrices, LBO = 128 B between K chunks, SBO =
//         512 B between row groups), written by the threads to shared memory
//   B   = the Toeplitz byte matrix of p, 112 x 64 (B[n][k] = p_byte[n - k]), constant
//   D   = A * B^T in TMEM: 128 lanes x 112 s32 columns (column j = sum_k m_k p_{j-k})
// one elected thread issues two MMAs (K = 32 each) and commits to an mbarrier; every
// thread then reads its row with tcgen05.ld (32x32b) and compacts the 97 column sums into
// 26 radix-2^30 limbs (64-bit windows of 4 columns, one carry pass).
// `imad` computes the identical 26-limb product with 169 IMAD.WIDE (column sums, one
// carry pass).  Both variants run a dependent chain m <- f(m * p) for ITERS steps and the
// final values are compared word for word.  All mbarrier waits are bounded (a wrong
// descriptor gives wrong numbers or a flagged timeout, never a hang).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o microbench/tc5_mont microbench/tc5_mont.cu
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

#define DEVI __device__ __forceinline__
typedef unsigned long long u64;

constexpr int L = 13, W = 30, NL = 26;
constexpr uint32_t MASK = (1u << W) - 1;
constexpr int TM = 128, TN = 112, TK = 64;
constexpr int ITERS = 1024;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__constant__ uint32_t P30[L];       // p, radix 2^30
__constant__ uint8_t PB[TN * TK];   // Toeplitz B (n-major rows of K bytes), canonical layout image

DEVI u64 madw(uint32_t a, uint32_t b, u64 c) {
  u64 p;
  asm("mul.wide.u32 %0, %1, %2;" : "=l"(p) : "r"(a), "r"(b));
  return p + c;
}

// next m from the product (26 limbs): low 390 bits, perturbed per thread (dependency chain)
DEVI void next_m(uint32_t* m, const uint32_t* U, uint32_t salt) {
#pragma unroll
  for (int i = 0; i < L; i++) m[i] = (U[i] ^ (salt * (i + 1))) & MASK;
}

// ---- IMAD reference: U = m * p (26 radix-2^30 limbs)
DEVI void mp_imad(uint32_t* U, const uint32_t* m) {
  u64 carry = 0;
#pragma unroll
  for (int k = 0; k < 2 * L - 1; k++) {
    u64 acc = carry;
#pragma unroll
    for (int i = 0; i < L; i++)
      if (k - i >= 0 && k - i < L) acc = madw(m[i], P30[k - i], acc);
    U[k] = (uint32_t)acc & MASK;
    carry = acc >> W;
  }
  U[2 * L - 1] = (uint32_t)carry;
}

__global__ void __launch_bounds__(128) k_imad(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, int n) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n) return;
  uint32_t m[L], U[NL];
#pragma unroll
  for (int i = 0; i < L; i++) m[i] = in[t * L + i];
#pragma unroll 1
  for (int it = 0; it < ITERS; it++) {
    mp_imad(U, m);
    next_m(m, U, t * 2654435761u + it);
  }
#pragma unroll
  for (int i = 0; i < NL; i++) out[(size_t)t * NL + i] = U[i];
}

// ---- tcgen05 variant
DEVI uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

DEVI uint64_t make_desc(uint32_t saddr) {
  // SmemDescriptor (cute/arch/mma_sm100_desc.hpp): start>>4 [0,14), LBO>>4 [16,30),
  // SBO>>4 [32,46), version 1 [46,48), base offset 0, lbo mode 0, layout SWIZZLE_NONE (0)
  const uint64_t start = (saddr >> 4) & 0x3FFF;
  const uint64_t lbo = (128 >> 4) & 0x3FFF, sbo = (512 >> 4) & 0x3FFF;
  return start | (lbo << 16) | (sbo << 32) | (1ull << 46);
}

// InstrDescriptor for kind::i8: c_format S32 (2) [4,6), a/b unsigned (0), K-major,
// n_dim = N>>3 [17,23), m_dim = M>>4 [24,29)
constexpr uint32_t IDESC = (2u << 4) | ((uint32_t)(TN >> 3) << 17) | ((uint32_t)(TM >> 4) << 24);

__global__ void __launch_bounds__(128, 1) k_tc(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, int n,
                                               uint32_t* __restrict__ flags) {
  __shared__ __align__(1024) uint8_t sA[TM * TK];
  __shared__ __align__(1024) uint8_t sB[TN * TK];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t tmem_base;
  const int tid = threadIdx.x;
  const int t = blockIdx.x * blockDim.x + tid;
  // B image (constant) into shared memory
  for (int i = tid; i < TN * TK / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(sB)[i] = reinterpret_cast<const uint4*>(PB)[i];
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (tid < 32) {  // one warp allocates 128 TMEM columns
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(&tmem_base)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base;
  const uint64_t dA = make_desc(smem_u32(sA)), dB = make_desc(smem_u32(sB));
  uint32_t m[L], U[NL];
  const bool live = t < n;
#pragma unroll
  for (int i = 0; i < L; i++) m[i] = live ? in[t * L + i] : 0u;
  uint32_t phase = 0, bad = 0;
#pragma unroll 1
  for (int it = 0; it < ITERS; it++) {
    // m -> 13 little-endian 32-bit words (390 bits) -> row tid of A (canonical layout)
    uint32_t w[16];
#pragma unroll
    for (int j = 0; j < 16; j++) {
      const int bit = 32 * j, li = bit / W, sh = bit % W;
      uint32_t v = 0;
      if (li < L) v = m[li] >> sh;
      if (li + 1 < L) v |= m[li + 1] << (W - sh);
      if (li + 2 < L && 2 * W - sh < 32) v |= m[li + 2] << (2 * W - sh);
      w[j] = (j < 13) ? v : 0u;
    }
    if (true) {  // 390 bits: clear bits >= 390 of word 12
      w[12] &= (1u << (390 - 384)) - 1;
    }
    uint8_t* rowbase = sA + (tid >> 3) * 512 + (tid & 7) * 16;
#pragma unroll
    for (int kc = 0; kc < 4; kc++)
      *reinterpret_cast<uint4*>(rowbase + kc * 128) = make_uint4(w[4 * kc], w[4 * kc + 1], w[4 * kc + 2], w[4 * kc + 3]);
    asm volatile("fence.proxy.async.shared::cta;");
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;");
#pragma unroll
      for (int kk = 0; kk < 2; kk++) {
        const uint64_t a = dA + (uint64_t)((kk * 256) >> 4), b = dB + (uint64_t)((kk * 256) >> 4);
        const uint32_t acc = kk ? 1u : 0u;
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n"
            ::"r"(tmem), "l"(a), "l"(b), "r"(IDESC), "r"(acc));
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mbar)));
    }
    // bounded wait for the MMA completion
    uint32_t done = 0;
    for (int spin = 0; spin < (1 << 22) && !done; spin++) {
      asm volatile(
          "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
          : "=r"(done) : "r"(smem_u32(&mbar)), "r"(phase));
    }
    if (!done) bad = 1;
    phase ^= 1;
    asm volatile("tcgen05.fence::after_thread_sync;");
    // my row: TMEM lane (warp*32 + lane) = tid; columns 0..111 (two x64 loads: 0..127)
    uint32_t d[128];
    const uint32_t taddr = tmem + ((uint32_t)(tid & ~31) << 16);
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x64.b32 {"
        "%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,"
        "%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63},"
        " [%64];"
        : "=r"(d[0]), "=r"(d[1]), "=r"(d[2]), "=r"(d[3]), "=r"(d[4]), "=r"(d[5]), "=r"(d[6]), "=r"(d[7]), "=r"(d[8]),
          "=r"(d[9]), "=r"(d[10]), "=r"(d[11]), "=r"(d[12]), "=r"(d[13]), "=r"(d[14]), "=r"(d[15]), "=r"(d[16]),
          "=r"(d[17]), "=r"(d[18]), "=r"(d[19]), "=r"(d[20]), "=r"(d[21]), "=r"(d[22]), "=r"(d[23]), "=r"(d[24]),
          "=r"(d[25]), "=r"(d[26]), "=r"(d[27]), "=r"(d[28]), "=r"(d[29]), "=r"(d[30]), "=r"(d[31]), "=r"(d[32]),
          "=r"(d[33]), "=r"(d[34]), "=r"(d[35]), "=r"(d[36]), "=r"(d[37]), "=r"(d[38]), "=r"(d[39]), "=r"(d[40]),
          "=r"(d[41]), "=r"(d[42]), "=r"(d[43]), "=r"(d[44]), "=r"(d[45]), "=r"(d[46]), "=r"(d[47]), "=r"(d[48]),
          "=r"(d[49]), "=r"(d[50]), "=r"(d[51]), "=r"(d[52]), "=r"(d[53]), "=r"(d[54]), "=r"(d[55]), "=r"(d[56]),
          "=r"(d[57]), "=r"(d[58]), "=r"(d[59]), "=r"(d[60]), "=r"(d[61]), "=r"(d[62]), "=r"(d[63])
        : "r"(taddr));
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x64.b32 {"
        "%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,"
        "%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63},"
        " [%64];"
        : "=r"(d[64]), "=r"(d[65]), "=r"(d[66]), "=r"(d[67]), "=r"(d[68]), "=r"(d[69]), "=r"(d[70]), "=r"(d[71]),
          "=r"(d[72]), "=r"(d[73]), "=r"(d[74]), "=r"(d[75]), "=r"(d[76]), "=r"(d[77]), "=r"(d[78]), "=r"(d[79]),
          "=r"(d[80]), "=r"(d[81]), "=r"(d[82]), "=r"(d[83]), "=r"(d[84]), "=r"(d[85]), "=r"(d[86]), "=r"(d[87]),
          "=r"(d[88]), "=r"(d[89]), "=r"(d[90]), "=r"(d[91]), "=r"(d[92]), "=r"(d[93]), "=r"(d[94]), "=r"(d[95]),
          "=r"(d[96]), "=r"(d[97]), "=r"(d[98]), "=r"(d[99]), "=r"(d[100]), "=r"(d[101]), "=r"(d[102]), "=r"(d[103]),
          "=r"(d[104]), "=r"(d[105]), "=r"(d[106]), "=r"(d[107]), "=r"(d[108]), "=r"(d[109]), "=r"(d[110]),
          "=r"(d[111]), "=r"(d[112]), "=r"(d[113]), "=r"(d[114]), "=r"(d[115]), "=r"(d[116]), "=r"(d[117]),
          "=r"(d[118]), "=r"(d[119]), "=r"(d[120]), "=r"(d[121]), "=r"(d[122]), "=r"(d[123]), "=r"(d[124]),
          "=r"(d[125]), "=r"(d[126]), "=r"(d[127])
        : "r"(taddr + 64));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();  // TMEM D free for the next MMA; A free for the next m
    // compaction: 97 byte-column sums (each < 2^22) -> 25 32-bit words -> 26 radix-2^30 limbs
    uint32_t o32[26];
    u64 c = 0;
#pragma unroll
    for (int q = 0; q < 25; q++) {
      u64 v = c + (u64)d[4 * q] + ((u64)d[4 * q + 1] << 8) + ((u64)d[4 * q + 2] << 16) + ((u64)d[4 * q + 3] << 24);
      o32[q] = (uint32_t)v;
      c = v >> 32;
    }
    o32[25] = (uint32_t)c;
#pragma unroll
    for (int i = 0; i < NL; i++) {
      const int bit = W * i, wi = bit >> 5, sh = bit & 31;
      uint32_t v = o32[wi] >> sh;
      if (sh && wi + 1 < 26) v |= o32[wi + 1] << (32 - sh);
      U[i] = v & MASK;
    }
    next_m(m, U, t * 2654435761u + it);
  }
  if (live) {
#pragma unroll
    for (int i = 0; i < NL; i++) out[(size_t)t * NL + i] = U[i];
  }
  if (bad) atomicOr(flags, 1u);
  __syncthreads();
  if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

int main() {
  // p (BLS12-381) in radix 2^30 and as bytes
  const uint32_t p30[L] = {0x3fffaaabu, 0x27fbffffu, 0x153ffffbu, 0x2affffacu, 0x30f6241eu, 0x034a83dau, 0x112bf673u,
                           0x12e13ce1u, 0x2cd76477u, 0x1ed90d2eu, 0x29a4b1bau, 0x3a8e5ff9u, 0x001a0111u};
  uint8_t pbytes[64] = {0};
  for (int b = 0; b < 390; b++) {
    const uint32_t bit = (p30[b / 30] >> (b % 30)) & 1u;
    pbytes[b / 8] |= (uint8_t)(bit << (b % 8));
  }
  // Toeplitz B (N x K, K-major), canonical no-swizzle image: row n, k chunk kc at
  // (n/8)*512 + kc*128 + (n%8)*16
  static uint8_t img[TN * TK];
  memset(img, 0, sizeof(img));
  for (int nn = 0; nn < TN; nn++)
    for (int k = 0; k < TK; k++) {
      const int j = nn - k;
      const uint8_t v = (j >= 0 && j < 49) ? pbytes[j] : 0;
      img[(nn / 8) * 512 + (k / 16) * 128 + (nn % 8) * 16 + (k % 16)] = v;
    }
  CK(cudaMemcpyToSymbol(P30, p30, sizeof(p30)));
  CK(cudaMemcpyToSymbol(PB, img, sizeof(img)));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int n = sms * 128 * 8;
  uint32_t* h = new uint32_t[(size_t)n * L];
  uint64_t s = 0x9e3779b97f4a7c15ull;
  for (size_t i = 0; i < (size_t)n * L; i++) {
    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
    h[i] = (uint32_t)s & MASK;
  }
  uint32_t *din, *d1, *d2, *flags;
  CK(cudaMalloc(&din, (size_t)n * L * 4));
  CK(cudaMalloc(&d1, (size_t)n * NL * 4));
  CK(cudaMalloc(&d2, (size_t)n * NL * 4));
  CK(cudaMalloc(&flags, 4));
  CK(cudaMemset(flags, 0, 4));
  CK(cudaMemcpy(din, h, (size_t)n * L * 4, cudaMemcpyHostToDevice));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float ms_imad = 0, ms_tc = 0;
  const int reps = 5;
  k_imad<<<n / 128, 128>>>(din, d1, n);
  CK(cudaDeviceSynchronize());
  cudaEventRecord(e0);
  for (int r = 0; r < reps; r++) k_imad<<<n / 128, 128>>>(din, d1, n);
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  cudaEventElapsedTime(&ms_imad, e0, e1);
  k_tc<<<n / 128, 128>>>(din, d2, n, flags);
  CK(cudaDeviceSynchronize());
  cudaEventRecord(e0);
  for (int r = 0; r < reps; r++) k_tc<<<n / 128, 128>>>(din, d2, n, flags);
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  cudaEventElapsedTime(&ms_tc, e0, e1);
  uint32_t hf = 0;
  CK(cudaMemcpy(&hf, flags, 4, cudaMemcpyDeviceToHost));
  uint32_t* r1 = new uint32_t[(size_t)n * NL];
  uint32_t* r2 = new uint32_t[(size_t)n * NL];
  CK(cudaMemcpy(r1, d1, (size_t)n * NL * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(r2, d2, (size_t)n * NL * 4, cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (size_t i = 0; i < (size_t)n * NL; i++) bad += r1[i] != r2[i];
  const double prods = (double)n * ITERS;
  printf("{\"variant\":\"imad m*p\",\"ms\":%.3f,\"g_products_per_s\":%.2f}\n", ms_imad / reps, prods / (ms_imad / reps * 1e-3) / 1e9);
  printf("{\"variant\":\"tcgen05 i8 m*p + TMEM + compaction\",\"ms\":%.3f,\"g_products_per_s\":%.2f,\"mismatched_words\":%zu,"
         "\"wait_timeouts\":%u,\"threads\":%d}\n", ms_tc / reps, prods / (ms_tc / reps * 1e-3) / 1e9, bad, hf, n);
  return 0;
}
