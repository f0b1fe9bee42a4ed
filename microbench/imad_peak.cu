// Integer-pipe peak microbenchmarks on sm_100a.
// Measures per-SM-per-clock throughput of the instructions a 32-bit-limb Montgomery
// multiplication lowers to (IMAD, IMAD.HI, IMAD.WIDE, IADD3(.X)), plus whole
// Montgomery multiplications in two formulations (PTX carry chains vs 64-bit products).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o imad_peak imad_peak.cu
// Output: one JSON object per line.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_ji0x024_b200/csrc/field.cuh"
typedef unsigned long long u64;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\":\"%s\"}\n", cudaGetErrorString(e)); return 1; } } while (0)

constexpr int ITERS = 4096;
constexpr int CH = 8;  // independent chains per thread

__global__ void k_imad(uint32_t* out, uint32_t seed, long long* cyc) {
  uint32_t x[CH];
  #pragma unroll
  for (int c = 0; c < CH; c++) x[c] = seed + threadIdx.x * 7 + c;
  uint32_t y = seed | 1, z = seed ^ 0x1234567;
  long long t0 = clock64();
  for (int i = 0; i < ITERS; i++) {
    #pragma unroll
    for (int c = 0; c < CH; c++) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[c]) : "r"(y), "r"(z));
  }
  long long t1 = clock64();
  uint32_t s = 0;
  #pragma unroll
  for (int c = 0; c < CH; c++) s ^= x[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}
__global__ void k_imadhi(uint32_t* out, uint32_t seed, long long* cyc) {
  uint32_t x[CH];
  #pragma unroll
  for (int c = 0; c < CH; c++) x[c] = seed + threadIdx.x * 7 + c;
  uint32_t y = seed | 1, z = seed ^ 0x1234567;
  long long t0 = clock64();
  for (int i = 0; i < ITERS; i++) {
    #pragma unroll
    for (int c = 0; c < CH; c++) asm volatile("mad.hi.u32 %0, %0, %1, %2;" : "+r"(x[c]) : "r"(y), "r"(z));
  }
  long long t1 = clock64();
  uint32_t s = 0;
  #pragma unroll
  for (int c = 0; c < CH; c++) s ^= x[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}
__global__ void k_imadwide(uint32_t* out, uint32_t seed, long long* cyc) {
  u64 x[CH];
  #pragma unroll
  for (int c = 0; c < CH; c++) x[c] = seed + threadIdx.x * 7 + c;
  uint32_t y = seed | 1, z = seed ^ 0x1234567;
  long long t0 = clock64();
  for (int i = 0; i < ITERS; i++) {
    #pragma unroll
    for (int c = 0; c < CH; c++) x[c] = mad_wide((uint32_t)x[c], y, x[c]);
  }
  long long t1 = clock64();
  uint32_t s = 0;
  #pragma unroll
  for (int c = 0; c < CH; c++) s ^= (uint32_t)x[c] ^ (uint32_t)(x[c] >> 32);
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}
__global__ void k_iadd3(uint32_t* out, uint32_t seed, long long* cyc) {
  uint32_t x[CH];
  #pragma unroll
  for (int c = 0; c < CH; c++) x[c] = seed + threadIdx.x * 7 + c;
  uint32_t y = seed | 1, z = seed ^ 0x1234567;
  long long t0 = clock64();
  for (int i = 0; i < ITERS; i++) {
    #pragma unroll
    for (int c = 0; c < CH; c++) asm volatile("add.u32 %0, %0, %1;\n\tadd.u32 %0, %0, %2;" : "+r"(x[c]) : "r"(y), "r"(z));
  }
  long long t1 = clock64();
  uint32_t s = 0;
  #pragma unroll
  for (int c = 0; c < CH; c++) s ^= x[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}

// ---- Montgomery multiplication, BLS12-381 base field, L = 12 ----
__constant__ uint32_t Pc[12];
constexpr uint32_t N0 = 0xfffcfffdu;

__device__ __forceinline__ void mont_wide(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  uint32_t t[14];
  #pragma unroll
  for (int i = 0; i < 14; i++) t[i] = 0;
  #pragma unroll
  for (int i = 0; i < 12; i++) {
    u64 C = 0;
    #pragma unroll
    for (int j = 0; j < 12; j++) { u64 T = (u64)a[j] * b[i] + t[j] + C; t[j] = (uint32_t)T; C = T >> 32; }
    u64 T = (u64)t[12] + C; t[12] = (uint32_t)T; t[13] = (uint32_t)(T >> 32);
    uint32_t m = t[0] * N0;
    T = (u64)m * Pc[0] + t[0]; C = T >> 32;
    #pragma unroll
    for (int j = 1; j < 12; j++) { T = (u64)m * Pc[j] + t[j] + C; t[j - 1] = (uint32_t)T; C = T >> 32; }
    T = (u64)t[12] + C; t[11] = (uint32_t)T; t[12] = t[13] + (uint32_t)(T >> 32);
  }
  #pragma unroll
  for (int i = 0; i < 12; i++) r[i] = t[i];
}

// CIOS with PTX carry chains, even/odd accumulation (two interleaved rows).
__device__ __forceinline__ void mont_ptx(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  uint32_t t[13];
  #pragma unroll
  for (int i = 0; i < 13; i++) t[i] = 0;
  #pragma unroll
  for (int i = 0; i < 12; i++) {
    uint32_t bi = b[i];
    // t += a*bi  (lo parts into t[j], hi parts into t[j+1])
    asm("mad.lo.cc.u32 %0, %1, %2, %0;" : "+r"(t[0]) : "r"(a[0]), "r"(bi));
    #pragma unroll
    for (int j = 1; j < 12; j++) asm("madc.lo.cc.u32 %0, %1, %2, %0;" : "+r"(t[j]) : "r"(a[j]), "r"(bi));
    uint32_t t13;
    asm("addc.cc.u32 %0, %0, 0;" : "+r"(t[12]));
    asm("addc.u32 %0, 0, 0;" : "=r"(t13));
    asm("mad.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[1]) : "r"(a[0]), "r"(bi));
    #pragma unroll
    for (int j = 1; j < 11; j++) asm("madc.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[j + 1]) : "r"(a[j]), "r"(bi));
    asm("madc.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[12]) : "r"(a[11]), "r"(bi));
    asm("addc.u32 %0, %0, 0;" : "+r"(t13));
    uint32_t m = t[0] * N0;
    asm("mad.lo.cc.u32 %0, %1, %2, %0;" : "+r"(t[0]) : "r"(m), "r"(Pc[0]));
    #pragma unroll
    for (int j = 1; j < 12; j++) asm("madc.lo.cc.u32 %0, %1, %2, %0;" : "+r"(t[j]) : "r"(m), "r"(Pc[j]));
    asm("addc.cc.u32 %0, %0, 0;" : "+r"(t[12]));
    asm("addc.u32 %0, %0, 0;" : "+r"(t13));
    asm("mad.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[1]) : "r"(m), "r"(Pc[0]));
    #pragma unroll
    for (int j = 1; j < 11; j++) asm("madc.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[j + 1]) : "r"(m), "r"(Pc[j]));
    asm("madc.hi.cc.u32 %0, %1, %2, %0;" : "+r"(t[12]) : "r"(m), "r"(Pc[11]));
    asm("addc.u32 %0, %0, 0;" : "+r"(t13));
    #pragma unroll
    for (int j = 0; j < 12; j++) t[j] = t[j + 1];
    t[12] = t13;
  }
  #pragma unroll
  for (int i = 0; i < 12; i++) r[i] = t[i];
}

// radix-2^30 FIPS Montgomery (the library's field layer)
__global__ void k_mont30(uint32_t* out, const uint32_t* in, int iters, long long* cyc) {
  uint32_t x[13], y[13];
  int gid = blockIdx.x * blockDim.x + threadIdx.x;
  #pragma unroll
  for (int i = 0; i < 13; i++) { x[i] = in[(gid % 1024) * 26 + i] & 0x3fffffffu; y[i] = in[(gid % 1024) * 26 + 13 + i] & 0x3fffffffu; }
  x[12] &= 0xffff; y[12] &= 0xffff;
  long long t0 = clock64();
  for (int it = 0; it < iters; it++) fmul<BLS12_381_params>(x, x, y);
  long long t1 = clock64();
  #pragma unroll
  for (int i = 0; i < 13; i++) out[gid * 13 + i] = x[i];
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}

template <int V>
__global__ void k_mont(uint32_t* out, const uint32_t* in, int iters, long long* cyc) {
  uint32_t x[12], y[12];
  int gid = blockIdx.x * blockDim.x + threadIdx.x;
  #pragma unroll
  for (int i = 0; i < 12; i++) { x[i] = in[(gid % 1024) * 24 + i]; y[i] = in[(gid % 1024) * 24 + 12 + i]; }
  long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
    if (V == 0) mont_wide(x, x, y); else mont_ptx(x, x, y);
  }
  long long t1 = clock64();
  #pragma unroll
  for (int i = 0; i < 12; i++) out[gid * 12 + i] = x[i];
  if (threadIdx.x == 0) atomicMax((unsigned long long*)cyc, (unsigned long long)(t1 - t0));
}

int main() {
  int dev = 0; cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, dev));
  int sms = prop.multiProcessorCount;
  const uint32_t p381[12] = {0xffffaaab, 0xb9feffff, 0xb153ffff, 0x1eabfffe, 0xf6b0f624, 0x6730d2a0,
                             0xf38512bf, 0x64774b84, 0x434bacd7, 0x4b1ba7b6, 0x397fe69a, 0x1a0111ea};
  CK(cudaMemcpyToSymbol(Pc, p381, sizeof(p381)));
  uint32_t* out; long long* cyc; uint32_t* in;
  int blocks = sms * 8, threads = 256;
  CK(cudaMalloc(&out, (size_t)blocks * threads * 13 * 4));
  CK(cudaMalloc(&cyc, 8));
  CK(cudaMalloc(&in, 1024 * 26 * 4));
  // inputs < p: random limbs with top limb small
  static uint32_t h[1024 * 26]; uint32_t s = 12345;
  for (int i = 0; i < 1024 * 26; i++) { s = s * 1664525u + 1013904223u; h[i] = s; if (i % 12 == 11) h[i] &= 0x0fffffff; }
  CK(cudaMemcpy(in, h, sizeof(h), cudaMemcpyHostToDevice));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto run = [&](const char* name, void (*kern)(uint32_t*, uint32_t, long long*), double ops_per_thread) {
    for (int rep = 0; rep < 2; rep++) {
      cudaMemset(cyc, 0, 8);
      cudaEventRecord(e0);
      kern<<<blocks, threads>>>(out, 777u, cyc);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      double ops = ops_per_thread * blocks * threads;
      if (rep == 1)
        printf("{\"kernel\":\"%s\",\"ms\":%.4f,\"Gops_per_s\":%.1f,\"ops_per_clk_per_SM_by_block_cycles\":%.2f,\"implied_mhz\":%.0f}\n",
               name, ms, ops / ms / 1e6, ops / (double)c / sms * ((double)blocks / (sms * 8.0)) / (blocks / (sms * 8.0)),
               (double)c / (ms * 1e3));
    }
  };
  run("imad_lo", k_imad, (double)ITERS * CH);
  run("imad_hi", k_imadhi, (double)ITERS * CH);
  run("imad_wide", k_imadwide, (double)ITERS * CH);
  run("iadd_x2", k_iadd3, (double)ITERS * CH * 2);
  for (int tpb : {128, 256, 384, 512, 1024}) {
    int bl = sms * 4, iters = 256;
    for (int rep = 0; rep < 2; rep++) {
      cudaMemset(cyc, 0, 8);
      cudaEventRecord(e0);
      k_mont30<<<bl, tpb>>>(out, in, iters, cyc);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double mults = (double)iters * bl * tpb;
      long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      if (rep == 1)
        printf("{\"kernel\":\"mont381_radix30_fips\",\"tpb\":%d,\"blocks\":%d,\"ms\":%.4f,\"Gmults_per_s\":%.2f,\"wide_slots_per_mult\":354,\"fma_pipe_util_at_1965MHz\":%.3f}\n",
               tpb, bl, ms, mults / ms / 1e6, mults * 354 / (ms * 1e-3) / (148.0 * 64 * 1.965e9));
    }
  }
  for (int v = 0; v < 2; v++) {
    for (int tpb : {128, 256, 384, 512}) {
      int bl = sms * 4;
      int iters = 256;
      for (int rep = 0; rep < 2; rep++) {
        cudaMemset(cyc, 0, 8);
        cudaEventRecord(e0);
        if (v == 0) k_mont<0><<<bl, tpb>>>(out, in, iters, cyc); else k_mont<1><<<bl, tpb>>>(out, in, iters, cyc);
        cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        double mults = (double)iters * bl * tpb;
        if (rep == 1)
          printf("{\"kernel\":\"mont381_%s\",\"tpb\":%d,\"blocks\":%d,\"ms\":%.4f,\"Gmults_per_s\":%.2f,\"IMAD_equiv_T_per_s_588\":%.2f}\n",
                 v == 0 ? "wide" : "ptx", tpb, bl, ms, mults / ms / 1e6, mults * 588 / ms / 1e9);
      }
    }
  }
  // cross-check both variants produce the same value
  {
    uint32_t *o2; CK(cudaMalloc(&o2, 1024 * 12 * 4));
    k_mont<0><<<4, 256>>>(out, in, 3, cyc); k_mont<1><<<4, 256>>>(o2, in, 3, cyc);
    static uint32_t ha[1024 * 12], hb[1024 * 12];
    cudaMemcpy(ha, out, sizeof(ha), cudaMemcpyDeviceToHost); cudaMemcpy(hb, o2, sizeof(hb), cudaMemcpyDeviceToHost);
    int bad = 0; for (int i = 0; i < 1024 * 12; i++) bad += ha[i] != hb[i];
    printf("{\"variants_agree_mismatch_words\":%d}\n", bad);
  }
  printf("{\"sms\":%d,\"clock_khz\":%d,\"regs_per_sm\":%d,\"l2\":%d}\n", sms, prop.clockRate, prop.regsPerMultiprocessor, prop.l2CacheSize);
  return 0;
}
