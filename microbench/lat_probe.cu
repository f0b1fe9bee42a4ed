// Single-thread latency of one Montgomery multiplication (dependent chain x = x*y):
// throughput-mode vs latency-mode column scheduling (csrc/field.cuh).
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_asplos_ji0x024_b200/csrc/field.cuh"
template <int V>
__global__ void k(uint32_t* out, const uint32_t* in, int iters, long long* cyc) {
  uint32_t x[13], y[13];
  for (int i = 0; i < 13; i++) { x[i] = in[i] & 0x3fffffff; y[i] = in[13 + i] & 0x3fffffff; }
  x[12] &= 0xffff; y[12] &= 0xffff;
  long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
    if (V == 0) fmul<BLS12_381_params>(x, x, y);
    else if (V == 1) fmul_lat<BLS12_381_params>(x, x, y);
    else if (V == 2) fsqr<BLS12_381_params>(x, x);
    else fsqr_lat<BLS12_381_params>(x, x);
  }
  long long t1 = clock64();
  for (int i = 0; i < 13; i++) out[i] = x[i];
  *cyc = t1 - t0;
}
int main() {
  uint32_t *in, *out; long long* cyc;
  cudaMalloc(&in, 26 * 4); cudaMalloc(&out, 13 * 4); cudaMalloc(&cyc, 8);
  uint32_t h[26]; for (int i = 0; i < 26; i++) h[i] = 0x12345678u * (i + 1);
  cudaMemcpy(in, h, sizeof(h), cudaMemcpyHostToDevice);
  const char* names[4] = {"fmul", "fmul_lat", "fsqr", "fsqr_lat"};
  for (int v = 0; v < 4; v++) {
    for (int rep = 0; rep < 2; rep++) {
      if (v == 0) k<0><<<1, 1>>>(out, in, 1000, cyc);
      if (v == 1) k<1><<<1, 1>>>(out, in, 1000, cyc);
      if (v == 2) k<2><<<1, 1>>>(out, in, 1000, cyc);
      if (v == 3) k<3><<<1, 1>>>(out, in, 1000, cyc);
      long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      if (rep) printf("{\"op\":\"%s\",\"cycles_per_op_single_thread\":%.1f}\n", names[v], c / 1000.0);
    }
  }
  return 0;
}
