// Pipe-rate probe (sm_100a): DFMA alone, IMAD.WIDE alone, and both interleaved in one
// instruction stream — are the FP64 and IMAD pipes independent on B200, and at what rate?
// Each thread runs NCH independent chains; results are kept live through a final store.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o microbench/dfma_probe microbench/dfma_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int NCH = 8;
constexpr int ITERS = 4096;

__global__ void k_dfma(double* out, double a0, double b0) {
  double acc[NCH];
#pragma unroll
  for (int c = 0; c < NCH; c++) acc[c] = a0 + threadIdx.x + c;
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < NCH; c++) acc[c] = fma(acc[c], b0, 0.5);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < NCH; c++) s += acc[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__device__ __forceinline__ unsigned long long madw(uint32_t a, uint32_t b, unsigned long long c) {
  unsigned long long p;
  asm volatile("mul.wide.u32 %0, %1, %2;" : "=l"(p) : "r"(a), "r"(b));
  return p + c;
}

__global__ void k_imadw(unsigned long long* out, uint32_t a0, uint32_t b0) {
  unsigned long long acc[NCH];
  uint32_t a[NCH];
#pragma unroll
  for (int c = 0; c < NCH; c++) { acc[c] = threadIdx.x + c; a[c] = a0 + c * 7 + threadIdx.x; }
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < NCH; c++) acc[c] = madw(a[c], b0 + (uint32_t)acc[c], acc[c]);
  }
  unsigned long long s = 0;
#pragma unroll
  for (int c = 0; c < NCH; c++) s += acc[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_mix(double* out, unsigned long long* out2, double a0, double b0, uint32_t ia, uint32_t ib) {
  double acc[NCH];
  unsigned long long iacc[NCH];
  uint32_t a[NCH];
#pragma unroll
  for (int c = 0; c < NCH; c++) { acc[c] = a0 + threadIdx.x + c; iacc[c] = threadIdx.x + c; a[c] = ia + c; }
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < NCH; c++) {
      acc[c] = fma(acc[c], b0, 0.5);
      iacc[c] = madw(a[c], ib + (uint32_t)iacc[c], iacc[c]);
    }
  }
  double s = 0;
  unsigned long long t = 0;
#pragma unroll
  for (int c = 0; c < NCH; c++) { s += acc[c]; t += iacc[c]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  out2[blockIdx.x * blockDim.x + threadIdx.x] = t;
}

// 64-bit integer add throughput (how does nvcc lower u64 +?)
__global__ void k_iadd64(unsigned long long* out, unsigned long long a0) {
  unsigned long long acc[NCH];
#pragma unroll
  for (int c = 0; c < NCH; c++) acc[c] = a0 * (threadIdx.x + c);
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < NCH; c++) acc[c] = acc[c] + acc[(c + 1) % NCH];
  }
  unsigned long long s = 0;
#pragma unroll
  for (int c = 0; c < NCH; c++) s += acc[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int blocks = sms * 8, threads = 256;
  double* d;
  unsigned long long* u;
  cudaMalloc(&d, blocks * threads * 8);
  cudaMalloc(&u, blocks * threads * 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const double ops = (double)blocks * threads * ITERS * NCH;
  auto run = [&](const char* name, auto launch, double per) {
    launch();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    for (int r = 0; r < 5; r++) launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= 5;
    const double rate = ops * per / (ms * 1e-3);
    printf("%-10s %8.3f ms  %8.2f T ops/s  %6.1f /clk/SM (at %d MHz)\n", name, ms, rate / 1e12,
           rate / sms / (clk * 1e3), clk / 1000);
  };
  run("dfma", [&] { k_dfma<<<blocks, threads>>>(d, 1.0, 0.999999); }, 1.0);
  run("imad.wide", [&] { k_imadw<<<blocks, threads>>>(u, 12345u, 777u); }, 1.0);
  run("mix(each)", [&] { k_mix<<<blocks, threads>>>(d, u, 1.0, 0.999999, 3u, 5u); }, 1.0);
  run("iadd64", [&] { k_iadd64<<<blocks, threads>>>(u, 3ull); }, 1.0);
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
