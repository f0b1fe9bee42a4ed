// f2 (§4.3): tensor-core Montgomery A/B on sm_100a.
//
// The paper moves the m x n half of Montgomery multiplication (Alg. 2 line 4) onto
// 8-bit tensor-core MMAs with the constant modulus n as matB ("practical only when
// matB is constant"), then compacts the 32-bit column sums.  North_star:
// keep it "only if an ncu A/B run shows it beats the IMAD path".  Three BLS12-381
// multiplications, all with R = 2^390 (radix-2^30, L = 13) so their results agree mod p:
//
//   fips   the library's field layer (csrc/field.cuh: word-serial m_k, IMAD.WIDE columns)
//   sep    separated Montgomery on IMAD: T = a*b, m = (T mod R)*n' mod R, U = m*p,
//          r = (T + U) / R  — the algebra the tensor-core variant needs (m must be known
//          in full before an MMA can multiply it)
//   tc     as sep, with U = m*p on mma.sync.m16n8k32.u8 (s32 accumulate): the 32 lanes of
//          a warp hold 32 independent multiplications = two 16-row A tiles of m bytes
//          (K = 64), B = the Toeplitz byte matrix of p (K x 104), 2 x 2 x 13 MMAs per warp;
//          column sums are packed in pairs (c0 + c1 << 8 < 2^31, the paper's compaction)
//          and routed back to the owning lane through shared memory.
//
// Each thread runs x <- x*y for ITERS dependent multiplications; every result is checked
// against fips (congruent mod p).  Output: one JSON object per line.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o tc_mont tc_mont.cu
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_ji0x024_b200/csrc/field.cuh"

using C = BLS12_381_params;
constexpr int L = 13, W = 30;
constexpr uint32_t MASK = (1u << W) - 1;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\":\"%s\",\"line\":%d}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__constant__ uint32_t NPc[L];   // n' = -p^-1 mod 2^390, radix 2^30
__constant__ uint32_t PLc[L];   // p, radix 2^30

// T = a*b: 26 normalised 30-bit limbs (column sums of <= 13 products < 13*2^60 + carry < 2^64)
DEVI void mul_full(uint32_t* T, const uint32_t* a, const uint32_t* b) {
  u64 carry = 0;
#pragma unroll
  for (int k = 0; k < 2 * L - 1; k++) {
    u64 acc = carry;
#pragma unroll
    for (int i = 0; i < L; i++)
      if (k - i >= 0 && k - i < L) acc = mad_wide(a[i], b[k - i], acc);
    T[k] = (uint32_t)acc & MASK;
    carry = acc >> W;
  }
  T[2 * L - 1] = (uint32_t)carry;
}

// m = (T mod 2^390) * n' mod 2^390 (lower triangle: 91 products)
DEVI void mul_m(uint32_t* m, const uint32_t* T) {
  u64 carry = 0;
#pragma unroll
  for (int k = 0; k < L; k++) {
    u64 acc = carry;
#pragma unroll
    for (int i = 0; i <= k; i++) acc = mad_wide(T[i], NPc[k - i], acc);
    m[k] = (uint32_t)acc & MASK;
    carry = acc >> W;
  }
}

// r = (T + m*p) / 2^390 with m*p on IMAD (sep)
DEVI void redc_imad(uint32_t* r, const uint32_t* T, const uint32_t* m) {
  u64 carry = 0;
#pragma unroll
  for (int k = 0; k < 2 * L; k++) {
    u64 acc = carry + T[k];
#pragma unroll
    for (int i = 0; i < L; i++)
      if (k - i >= 0 && k - i < L) acc = mad_wide(m[i], PLc[k - i], acc);
    if (k >= L) r[k - L] = (uint32_t)acc & MASK;
    carry = acc >> W;
  }
}

DEVI void fmul_sep(uint32_t* r, const uint32_t* a, const uint32_t* b) {
  uint32_t T[2 * L], m[L];
  mul_full(T, a, b);
  mul_m(m, T);
  redc_imad(r, T, m);
}

// ---- tensor-core m*p ----
constexpr int NT = 13;      // 8-column N tiles: 104 >= 49 + 48 byte columns
constexpr int AST = 20;     // A row stride in words (16 used; 20 = conflict-free quad reads)
constexpr int OST = 52;     // packed-output row stride in words (4 per N tile)
constexpr int TPB = 128, WPB = TPB / 32;

DEVI void mma_u8(int* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.u8.u8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+r"(c[0]), "+r"(c[1]), "+r"(c[2]), "+r"(c[3])
               : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

struct TcSmem {
  uint32_t A[WPB][32 * AST];
  uint32_t O[WPB][32 * OST];
  uint2 B[2][NT][32];  // B fragments per (k-step, N tile, lane)
};

DEVI void fmul_tc(uint32_t* r, const uint32_t* a, const uint32_t* b, TcSmem& sm) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, g = lane >> 2, t = lane & 3;
  uint32_t T[2 * L], m[L];
  mul_full(T, a, b);
  mul_m(m, T);
  // m (390 bits) -> 13 little-endian 32-bit words (bytes 0..51; K = 64, tail zero)
  uint32_t* Arow = sm.A[w] + lane * AST;
#pragma unroll
  for (int j = 0; j < 16; j++) {
    uint32_t v = 0;
#pragma unroll
    for (int i = 0; i < L; i++) {
      const int lo = i * W;
      if (lo + W <= 32 * j || lo >= 32 * j + 32) continue;
      const int sh = lo - 32 * j;
      v |= sh >= 0 ? (m[i] << sh) : (m[i] >> (-sh));
    }
    Arow[j] = v;
  }
  __syncwarp();
  uint32_t af[2][2][4];
#pragma unroll
  for (int h = 0; h < 2; h++)
#pragma unroll
    for (int s = 0; s < 2; s++) {
      const uint32_t* r0 = sm.A[w] + (16 * h + g) * AST + 8 * s;
      const uint32_t* r1 = sm.A[w] + (16 * h + g + 8) * AST + 8 * s;
      af[h][s][0] = r0[t]; af[h][s][1] = r1[t]; af[h][s][2] = r0[4 + t]; af[h][s][3] = r1[4 + t];
    }
#pragma unroll
  for (int q = 0; q < NT; q++) {
    const uint2 b0 = sm.B[0][q][lane], b1 = sm.B[1][q][lane];
#pragma unroll
    for (int h = 0; h < 2; h++) {
      int c[4] = {0, 0, 0, 0};
      mma_u8(c, af[h][0], b0.x, b0.y);
      mma_u8(c, af[h][1], b1.x, b1.y);
      // paper's compaction: adjacent byte columns fold into one word (< 49*255^2*257 < 2^31)
      sm.O[w][(16 * h + g) * OST + 4 * q + t] = (uint32_t)c[0] + ((uint32_t)c[1] << 8);
      sm.O[w][(16 * h + g + 8) * OST + 4 * q + t] = (uint32_t)c[2] + ((uint32_t)c[3] << 8);
    }
  }
  __syncwarp();
  // Z = T + sum_{q,t} V_{q,t} 2^(64q + 16t); r = Z >> 390
  u64 acc[28];
#pragma unroll
  for (int i = 0; i < 28; i++) acc[i] = i < 2 * L ? T[i] : 0;
  const uint4* orow = reinterpret_cast<const uint4*>(sm.O[w] + lane * OST);
#pragma unroll
  for (int q = 0; q < NT; q++) {
    const uint4 v4 = orow[q];
    const uint32_t vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
    for (int tt = 0; tt < 4; tt++) {
      const int bit = 64 * q + 16 * tt, li = bit / W, sh = bit % W;
      acc[li] += (u64)vv[tt] << sh;
    }
  }
  u64 carry = 0;
#pragma unroll
  for (int i = 0; i < 28; i++) {
    const u64 v = acc[i] + carry;
    if (i >= L && i < 2 * L) r[i - L] = (uint32_t)v & MASK;
    carry = v >> W;
  }
  __syncwarp();
}

template <int V>
__global__ void __launch_bounds__(TPB) k_bench(uint32_t* out, const uint32_t* in, int iters, const uint2* btab) {
  __shared__ TcSmem sm;
  if (V == 2) {
    for (int i = threadIdx.x; i < 2 * NT * 32; i += TPB) (&sm.B[0][0][0])[i] = btab[i];
    __syncthreads();
  }
  uint32_t x[L], y[L];
  const int gid = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int i = 0; i < L; i++) { x[i] = in[(gid % 4096) * 2 * L + i]; y[i] = in[(gid % 4096) * 2 * L + L + i]; }
  for (int it = 0; it < iters; it++) {
    if (V == 0) fmul<C>(x, x, y);
    else if (V == 1) fmul_sep(x, x, y);
    else fmul_tc(x, x, y, sm);
  }
  freduce<C>(x);
#pragma unroll
  for (int i = 0; i < L; i++) out[(size_t)gid * L + i] = x[i];
}

// ---- host: constants ----
static void to_limbs30(uint32_t* l, const uint32_t* w32, int nw) {
  for (int i = 0; i < L; i++) {
    uint32_t v = 0;
    for (int b = 0; b < W; b++) {
      const int bit = i * W + b, wi = bit / 32;
      if (wi < nw && ((w32[wi] >> (bit % 32)) & 1)) v |= 1u << b;
    }
    l[i] = v;
  }
}
static void mul_lo_h(uint32_t* r, const uint32_t* a, const uint32_t* b) {  // mod 2^390
  unsigned __int128 carry = 0;
  uint32_t t[L];
  for (int k = 0; k < L; k++) {
    unsigned __int128 acc = carry;
    for (int i = 0; i <= k; i++) acc += (u64)a[i] * b[k - i];
    t[k] = (uint32_t)acc & MASK;
    carry = acc >> W;
  }
  memcpy(r, t, sizeof(t));
}

int main() {
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  const int sms = prop.multiProcessorCount;
  const uint32_t p381[12] = {0xffffaaab, 0xb9feffff, 0xb153ffff, 0x1eabfffe, 0xf6b0f624, 0x6730d2a0,
                             0xf38512bf, 0x64774b84, 0x434bacd7, 0x4b1ba7b6, 0x397fe69a, 0x1a0111ea};
  uint32_t pl[L]; to_limbs30(pl, p381, 12);
  // x = p^-1 mod 2^390 by Newton (x <- x(2 - p x)), then n' = -x
  uint32_t x[L] = {1}, t[L], two[L] = {2};
  for (int it = 0; it < 10; it++) {
    mul_lo_h(t, pl, x);
    int64_t br = 0;  // t = 2 - t
    for (int i = 0; i < L; i++) { int64_t v = (int64_t)two[i] - t[i] - br; br = v < 0; t[i] = (uint32_t)(v + (br << W)) & MASK; }
    mul_lo_h(x, x, t);
  }
  uint32_t np[L]; { int64_t br = 0; for (int i = 0; i < L; i++) { int64_t v = -(int64_t)x[i] - br; br = v < 0; np[i] = (uint32_t)(v + (br << W)) & MASK; } }
  mul_lo_h(t, pl, np);  // p * n' == -1 mod 2^390
  for (int i = 0; i < L; i++) if (t[i] != MASK) { printf("{\"error\":\"n' check\"}\n"); return 1; }
  CK(cudaMemcpyToSymbol(NPc, np, sizeof(np)));
  CK(cudaMemcpyToSymbol(PLc, pl, sizeof(pl)));
  // B fragments: B[k][n] = pbyte[n - k] for 0 <= n - k < 48 (m16n8k32 .col: b0 rows 4t..4t+3, b1 rows 16+4t.., col g)
  uint8_t pb[48]; memcpy(pb, p381, 48);
  static uint2 btab[2 * NT * 32];
  for (int s = 0; s < 2; s++)
    for (int q = 0; q < NT; q++)
      for (int lane = 0; lane < 32; lane++) {
        const int g = lane >> 2, tq = lane & 3;
        uint32_t r[2] = {0, 0};
        for (int half = 0; half < 2; half++)
          for (int i = 0; i < 4; i++) {
            const int k = 32 * s + 16 * half + 4 * tq + i, n = 8 * q + g, d = n - k;
            if (d >= 0 && d < 48) r[half] |= (uint32_t)pb[d] << (8 * i);
          }
        btab[(s * NT + q) * 32 + lane] = make_uint2(r[0], r[1]);
      }
  uint2* dbt; CK(cudaMalloc(&dbt, sizeof(btab)));
  CK(cudaMemcpy(dbt, btab, sizeof(btab), cudaMemcpyHostToDevice));
  // inputs: random < 2^380 (< p), radix 2^30
  static uint32_t h[4096 * 2 * L]; uint64_t s = 0x9e3779b97f4a7c15ull;
  for (int e = 0; e < 4096 * 2; e++) {
    uint32_t w32[12];
    for (int i = 0; i < 12; i++) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; w32[i] = (uint32_t)s; }
    w32[11] &= 0x0fffffff;
    to_limbs30(h + e * L, w32, 12);
  }
  uint32_t* din; CK(cudaMalloc(&din, sizeof(h)));
  CK(cudaMemcpy(din, h, sizeof(h), cudaMemcpyHostToDevice));
  const int blocks = sms * 8, iters = 128;
  const size_t nthr = (size_t)blocks * TPB;
  uint32_t *o0, *o1;
  CK(cudaMalloc(&o0, nthr * L * 4)); CK(cudaMalloc(&o1, nthr * L * 4));
  static uint32_t hr0[148 * 8 * TPB * L], hr1[148 * 8 * TPB * L];
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[3] = {"fips_imad (library)", "separated_imad", "separated_tc_mma_u8"};
  for (int v = 0; v < 3; v++) {
    float best = 1e30f;
    for (int rep = 0; rep < 3; rep++) {
      cudaEventRecord(e0);
      if (v == 0) k_bench<0><<<blocks, TPB>>>(o0, din, iters, dbt);
      else if (v == 1) k_bench<1><<<blocks, TPB>>>(o1, din, iters, dbt);
      else k_bench<2><<<blocks, TPB>>>(o1, din, iters, dbt);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    CK(cudaGetLastError());
    long mism = 0;
    if (v > 0) {
      CK(cudaMemcpy(hr0, o0, nthr * L * 4, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(hr1, o1, nthr * L * 4, cudaMemcpyDeviceToHost));
      for (size_t i = 0; i < nthr * L; i++) mism += hr0[i] != hr1[i];
    }
    cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, v == 0 ? (const void*)k_bench<0> : v == 1 ? (const void*)k_bench<1> : (const void*)k_bench<2>);
    const double mults = (double)iters * nthr;
    printf("{\"variant\":\"%s\",\"ms\":%.4f,\"Gmults_per_s\":%.2f,\"regs\":%d,\"mismatched_words_vs_fips\":%ld,\"threads\":%zu,\"iters\":%d}\n",
           names[v], best, mults / best / 1e6, fa.numRegs, mism, nthr, iters);
  }
  return 0;
}
