// Throughput probe for the integer ops the mapper's hot loop is made of.
// Each kernel runs NREG independent cyclic chains of one op kind; the per-SM rate in
// lane-ops per SM clock is derived from clock64() deltas and the wall rate from events.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define NREG 16
#define ITERS 4096

template <int OP>
__global__ void __launch_bounds__(256) probe(uint32_t* out, uint32_t seed, unsigned long long* cyc) {
  uint32_t r[NREG];
#pragma unroll
  for (int i = 0; i < NREG; ++i) r[i] = seed * (threadIdx.x + 1) * (i + 7) + blockIdx.x;
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < NREG; ++i) {
      uint32_t a = r[i], b = r[(i + 1) % NREG], c = r[(i + 5) % NREG];
      if (OP == 0) r[i] = max(a, b);                 // IMNMX / VIMNMX
      if (OP == 1) r[i] = min(a, min(b, c));         // VIMNMX3
      if (OP == 2) r[i] = a + b + c;                 // IADD3 (or IMAD.IADD)
      if (OP == 3) r[i] = a * b + c;                 // IMAD
      if (OP == 4) { r[i] = (i & 1) ? min(a, min(b, c)) : max(a, b); }  // 1:1 mix
    }
  }
  long long t1 = clock64();
  uint32_t acc = 0;
#pragma unroll
  for (int i = 0; i < NREG; ++i) acc ^= r[i];
  if (acc == 0x12345678u) out[0] = acc;
  if (threadIdx.x == 0) atomicMax(cyc, (unsigned long long)(t1 - t0));
}

template <int OP>
void run(const char* name, int sms) {
  uint32_t* out; unsigned long long* cyc;
  cudaMalloc(&out, 4); cudaMalloc(&cyc, 8);
  int blocks = sms * 8, threads = 256;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int w = 0; w < 3; ++w) probe<OP><<<blocks, threads>>>(out, 3, cyc);
  cudaMemset(cyc, 0, 8);
  cudaEventRecord(e0);
  probe<OP><<<blocks, threads>>>(out, 3, cyc);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double ops = (double)blocks * threads * ITERS * NREG;
  // per SM: ops executed by the CTAs resident on it (8 CTAs x 256 thr all co-resident)
  double per_sm_clk = (double)8 * threads * ITERS * NREG / (double)c;
  printf("%-8s %.4e lane-ops/s  %.2f lane-ops/clk/SM  (max cta cycles %llu, %.3f ms, eff clk %.0f MHz)\n",
         name, ops / (ms * 1e-3), per_sm_clk, c, ms, c / (ms * 1e3));
}

int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  printf("%s sms=%d clock=%d kHz\n", p.name, p.multiProcessorCount, p.clockRate);
  int s = p.multiProcessorCount;
  run<0>("max2", s); run<1>("min3", s); run<2>("iadd3", s); run<3>("imad", s); run<4>("mix", s);
  run<0>("max2", s); run<1>("min3", s);
  return 0;
}
