// Occupancy probe for the field layer (BLS12-381, csrc/field.cuh): G mult/s of
//   fmul   one dependent product chain per thread (x <- x*y)
//   fmul2  two independent chains per thread, column-interleaved (the PACC kernel's form)
// at a FORCED number of resident 128-thread blocks per SM (dynamic shared memory is sized
// so that only B blocks fit), B = 1..8.  Separates "warps per scheduler" from everything
// else the PACC kernel does (gathers, add/sub glue, bucket bookkeeping).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o occ_probe occ_probe.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_ji0x024_b200/csrc/field.cuh"

using C = BLS12_381_params;
constexpr int L = C::L;

template <int V>
__global__ void __launch_bounds__(128) k_occ(uint32_t* out, const uint32_t* in, int iters) {
  extern __shared__ uint32_t pad[];
  uint32_t x[L], y[L], u[L], v[L];
  const int gid = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int i = 0; i < L; i++) {
    x[i] = in[(gid % 1024) * 4 * L + i];
    y[i] = in[(gid % 1024) * 4 * L + L + i];
    u[i] = in[(gid % 1024) * 4 * L + 2 * L + i];
    v[i] = in[(gid % 1024) * 4 * L + 3 * L + i];
  }
  for (int it = 0; it < iters; it++) {
    if (V == 0) fmul<C>(x, x, y);
    else fmul2<C>(x, x, y, u, u, v);
  }
#pragma unroll
  for (int i = 0; i < L; i++) out[(size_t)gid * L + i] = x[i] ^ u[i];
  if (threadIdx.x == 0 && gid == -1) pad[0] = 0;
}

int main() {
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, 0);
  const int sms = prop.multiProcessorCount;
  const size_t smem_sm = prop.sharedMemPerMultiprocessor;
  uint32_t *in, *out;
  cudaMalloc(&in, 1024 * 4 * L * 4);
  cudaMalloc(&out, (size_t)sms * 40 * 128 * L * 4);
  static uint32_t h[1024 * 4 * L];
  uint32_t s = 1;
  for (int i = 0; i < 1024 * 4 * L; i++) { s = s * 1664525u + 1013904223u; h[i] = (s >> 2) & 0x3fffffffu; if (i % L == L - 1) h[i] &= 0xffff; }
  cudaMemcpy(in, h, sizeof(h), cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(k_occ<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(k_occ<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int V = 0; V < 2; V++) {
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, V ? (const void*)k_occ<1> : (const void*)k_occ<0>);
    for (int B : {1, 2, 3, 4, 5, 6, 8}) {
      size_t sm = smem_sm / B - 2048;  // only B blocks fit per SM
      if (sm > 200 * 1024) sm = 200 * 1024;
      int bps = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, V ? k_occ<1> : k_occ<0>, 128, sm);
      const int blocks = sms * bps * 4, iters = 64;
      float best = 1e30f;
      for (int rep = 0; rep < 3; rep++) {
        cudaEventRecord(e0);
        if (V) k_occ<1><<<blocks, 128, sm>>>(out, in, iters);
        else k_occ<0><<<blocks, 128, sm>>>(out, in, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      const double mults = (double)blocks * 128 * iters * (V ? 2 : 1);
      printf("{\"variant\":\"%s\",\"regs\":%d,\"blocks_per_sm\":%d,\"warps_per_sm\":%d,\"ms\":%.3f,\"Gmults_per_s\":%.2f,\"err\":\"%s\"}\n",
             V ? "fmul2" : "fmul", fa.numRegs, bps, bps * 4, best, mults / best / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
