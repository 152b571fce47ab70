// probe.cu -- integer-pipe throughput probe: the denominator of the
// mapper's roofline, measured on the same GPU and at the same clocks as the search.
//
// Each op kind runs 16 independent cyclic chains per thread at full occupancy (8 CTAs x
// 256 threads per SM); lane-ops per SM clock come from clock64() deltas, the wall rate
// from CUDA events on the launching stream. Op kinds:
//   0 VIMNMX (2-input min/max)   1 VIMNMX3 (3-input)   2 IADD3   3 IMAD
//   4 VIMNMX3 + IMAD interleaved (are the ALU and FMA pipes issued concurrently?)
//   5 IMAD.HI (signed, opaque multiplier): the sign-mask step of an FMA-pipe max
//   6 max on the FMA pipe (IMAD, IMAD.HI, IMAD: 3 instructions per max) interleaved
//     1:1 with VIMNMX on the ALU pipe
#include "kernels.h"

namespace mcl {

namespace {
constexpr int kRegs = 16;
constexpr int kIters = 4096;

__device__ __forceinline__ int32_t mulhi_s32(int32_t a, int32_t b) {
  int32_t r;
  asm volatile("mul.hi.s32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}

// max(a, b) for a, b < 2^31 on the FMA pipe: nd = b - a, m = sign mask of nd, r = b + nd*m
__device__ __forceinline__ uint32_t max_fma(uint32_t a, uint32_t b, int32_t one, int32_t neg1) {
  int32_t nd, r;
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(nd) : "r"((int32_t)a), "r"(neg1), "r"((int32_t)b));
  const int32_t m = mulhi_s32(nd, one);
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(r) : "r"(nd), "r"(m), "r"((int32_t)b));
  return (uint32_t)r;
}

template <int OP>
__global__ void __launch_bounds__(256) probe_kernel(uint32_t* out, uint32_t seed,
                                                    unsigned long long* cyc) {
  const int32_t one = (int32_t)(seed >> 1), neg1 = -one;  // seed == 3: opaque 1 and -1
  uint32_t r[kRegs], s[kRegs];
#pragma unroll
  for (int i = 0; i < kRegs; ++i) {
    r[i] = seed * (threadIdx.x + 1) * (i + 7) + blockIdx.x;
    s[i] = r[i] ^ 0x9e3779b9u;
  }
  const long long t0 = clock64();
  for (int it = 0; it < kIters; ++it) {
#pragma unroll
    for (int i = 0; i < kRegs; ++i) {
      const uint32_t a = r[i], b = r[(i + 1) % kRegs], c = r[(i + 5) % kRegs];
      if (OP == 0) r[i] = max(a, b);
      if (OP == 1) r[i] = __vimin3_u32(a, b, c);
      if (OP == 2) r[i] = a + b + c;
      if (OP == 3) r[i] = a * b + c;
      if (OP == 4) {
        r[i] = __vimin3_u32(a, b, c);
        s[i] = s[i] * s[(i + 1) % kRegs] + s[(i + 3) % kRegs];
      }
      if (OP == 5) r[i] = (uint32_t)mulhi_s32((int32_t)a, (int32_t)b);
      if (OP == 6) {
        r[i] = max(a, b);
        s[i] = max_fma(s[i], s[(i + 1) % kRegs], one, neg1);  // throughput only
      }
    }
  }
  const long long t1 = clock64();
  uint32_t acc = 0;
#pragma unroll
  for (int i = 0; i < kRegs; ++i) acc ^= r[i] ^ ((OP == 4 || OP == 6) ? s[i] : 0u);
  if (acc == 0x12345678u) out[0] = acc;
  if (threadIdx.x == 0) atomicMax(cyc, (unsigned long long)(t1 - t0));
}

template <int OP>
cudaError_t run(int sms, cudaStream_t st, double* rate, double* per_clk, double* mhz) {
  uint32_t* out = nullptr;
  unsigned long long* cyc = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  cudaError_t err = cudaMalloc(&out, 4);
  if (err == cudaSuccess) err = cudaMalloc(&cyc, 8);
  if (err == cudaSuccess) err = cudaEventCreate(&e0);
  if (err == cudaSuccess) err = cudaEventCreate(&e1);
  const int ctas_per_sm = 8, threads = 256, blocks = sms * ctas_per_sm;
  if (err == cudaSuccess) {
    for (int w = 0; w < 3; ++w) probe_kernel<OP><<<blocks, threads, 0, st>>>(out, 3, cyc);
    cudaMemsetAsync(cyc, 0, 8, st);
    cudaEventRecord(e0, st);
    probe_kernel<OP><<<blocks, threads, 0, st>>>(out, 3, cyc);
    cudaEventRecord(e1, st);
    err = cudaEventSynchronize(e1);
  }
  if (err == cudaSuccess) {
    float ms = 0;
    unsigned long long c = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    err = cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    // lane-ops: op 4 counts both instructions; op 6 counts 1 ALU max + 1 FMA-pipe max
    const double ops_per_thread = (double)kIters * kRegs * ((OP == 4 || OP == 6) ? 2 : 1);
    *rate = (double)blocks * threads * ops_per_thread / (ms * 1e-3);
    *per_clk = (double)ctas_per_sm * threads * ops_per_thread / (double)c;
    *mhz = (double)c / (ms * 1e3);
  }
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (out) cudaFree(out);
  if (cyc) cudaFree(cyc);
  return err;
}
}  // namespace

cudaError_t probe_alu(int op, int sms, cudaStream_t st, double* rate, double* per_clk,
                      double* mhz) {
  switch (op) {
    case 0: return run<0>(sms, st, rate, per_clk, mhz);
    case 1: return run<1>(sms, st, rate, per_clk, mhz);
    case 2: return run<2>(sms, st, rate, per_clk, mhz);
    case 3: return run<3>(sms, st, rate, per_clk, mhz);
    case 4: return run<4>(sms, st, rate, per_clk, mhz);
    case 5: return run<5>(sms, st, rate, per_clk, mhz);
    case 6: return run<6>(sms, st, rate, per_clk, mhz);
    default: return cudaErrorInvalidValue;
  }
}

// Timing aid (mcl_set_timing_hold): keeps the stream busy while the host enqueues the
// start event and the search launch, so the events measure device execution only.
__global__ void hold_kernel(uint64_t ns) {
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    __nanosleep(500);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < ns);
}

cudaError_t launch_hold(uint64_t ns, cudaStream_t st) {
  hold_kernel<<<1, 1, 0, st>>>(ns);
  return cudaGetLastError();
}

// Launch floor: what CUDA events around a kernel that does nothing report, timed as the
// search kernels are timed (a 200 us hold first, so the events bracket device execution).
// One CTA per SM of 512 threads (the pooled batch kernel's shape). Also the events alone.
__global__ void empty_kernel(int* never) {
  if (never && threadIdx.x == 1023) *never = 1;  // never true: 512 threads
}

cudaError_t probe_launch_floor(int sms, cudaStream_t st, int reps, double* empty_us,
                               double* events_us) {
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  cudaError_t err = cudaEventCreate(&e0);
  if (err == cudaSuccess) err = cudaEventCreate(&e1);
  double sum_k = 0, sum_e = 0;
  for (int kind = 0; kind < 2 && err == cudaSuccess; ++kind) {
    for (int i = 0; i < reps + 3 && err == cudaSuccess; ++i) {
      hold_kernel<<<1, 1, 0, st>>>(200000);
      cudaEventRecord(e0, st);
      if (kind == 0) empty_kernel<<<sms, 512, 0, st>>>(nullptr);
      cudaEventRecord(e1, st);
      err = cudaEventSynchronize(e1);
      float ms = 0;
      if (err == cudaSuccess) err = cudaEventElapsedTime(&ms, e0, e1);
      if (i >= 3) (kind == 0 ? sum_k : sum_e) += ms * 1e3;
    }
  }
  if (err == cudaSuccess) {
    *empty_us = sum_k / reps;
    *events_us = sum_e / reps;
  }
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  return err;
}

}  // namespace mcl
