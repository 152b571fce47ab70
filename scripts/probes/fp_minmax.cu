// Throughput of fp32 min/max vs the integer VIMNMX3 (measurement only): can exact integer
// makespans below 2^24 be maxed / folded on another pipe than the integer ALU?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 fp_minmax.cu -o /tmp/fp_minmax
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kRegs = 16, kIters = 4096;

__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float r;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
  return r;
}
__device__ __forceinline__ float fmin3(float a, float b, float c) {
  float r;
  asm("min.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
  return r;
}

template <int OP>
__global__ void __launch_bounds__(256) k(float* out, unsigned* iout, unsigned seed, unsigned long long* cyc) {
  float f[kRegs];
  unsigned u[kRegs];
#pragma unroll
  for (int i = 0; i < kRegs; ++i) {
    u[i] = seed * (threadIdx.x + 1) * (i + 7) + blockIdx.x;
    f[i] = (float)(u[i] & 0xffff);
  }
  const long long t0 = clock64();
  for (int it = 0; it < kIters; ++it) {
#pragma unroll
    for (int i = 0; i < kRegs; ++i) {
      if (OP == 0) u[i] = __vimin3_u32(u[i], u[(i + 1) % kRegs], u[(i + 5) % kRegs]);
      if (OP == 1) f[i] = fmaxf(f[i], f[(i + 1) % kRegs]);
      if (OP == 2) f[i] = fmin3(f[i], f[(i + 1) % kRegs], f[(i + 5) % kRegs]);
      if (OP == 3) {
        u[i] = __vimin3_u32(u[i], u[(i + 1) % kRegs], u[(i + 5) % kRegs]);
        f[i] = fmin3(f[i], f[(i + 1) % kRegs], f[(i + 5) % kRegs]);
      }
      if (OP == 4) f[i] = f[i] + f[(i + 1) % kRegs];  // FADD
    }
  }
  const long long t1 = clock64();
  float acc = 0;
  unsigned ua = 0;
#pragma unroll
  for (int i = 0; i < kRegs; ++i) { acc += f[i]; ua ^= u[i]; }
  if (acc == 1234.5f) out[0] = acc;
  if (ua == 0x12345678u) iout[0] = ua;
  if (threadIdx.x == 0) atomicMax(cyc, (unsigned long long)(t1 - t0));
}

template <int OP>
void run(const char* name, int sms) {
  float* out; unsigned* iout; unsigned long long* cyc;
  cudaMalloc(&out, 4); cudaMalloc(&iout, 4); cudaMalloc(&cyc, 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int blocks = sms * 8, threads = 256;
  for (int w = 0; w < 3; ++w) k<OP><<<blocks, threads>>>(out, iout, 3, cyc);
  cudaMemset(cyc, 0, 8);
  cudaEventRecord(e0);
  k<OP><<<blocks, threads>>>(out, iout, 3, cyc);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  const double ops = (double)kIters * kRegs * (OP == 3 ? 2 : 1);
  printf("{\"op\": \"%s\", \"lane_ops_per_clk_sm\": %.2f, \"eff_mhz\": %.0f, \"ms\": %.3f}\n", name,
         8.0 * threads * ops / (double)c, (double)c / (ms * 1e3), ms);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run<0>("VIMNMX3 u32", sms);
  run<1>("fmaxf f32 2-input", sms);
  run<2>("min.f32 3-input", sms);
  run<3>("VIMNMX3 u32 + min.f32 3-input interleaved (2 ops)", sms);
  run<4>("FADD f32", sms);
  return 0;
}
