// score.cu -- makespan of GIVEN mappings (NEXT-3: policy baselines such as ROUND_ROBIN,
// "the next available device when the scheduler is triggered", PAPER.md L584-587, L620-624,
// and the static hint-based choices of SS V.B, L1086-1116, are scored against the optimum).
//
// One thread per epoch: loads start at the optional base loads, every queue adds its
// composed cost C = K + X on its device (serialised on a device), and
// the makespan is the max over devices (L1048-1052). 64-bit arithmetic; HBM-bound.
#include "common.cuh"
#include "kernels.h"

namespace mcl {

// Compile-time D keeps the per-device loads in registers (a runtime-indexed array of 16 went
// to the stack: 128 bytes of local memory per thread).
template <int D>
__global__ void __launch_bounds__(256) score_kernel(uint32_t Q, uint64_t E,
                                                    const uint64_t* __restrict__ K,
                                                    const uint64_t* __restrict__ X,
                                                    const uint64_t* __restrict__ base,
                                                    const uint8_t* __restrict__ mapping,
                                                    uint64_t* __restrict__ makespan,
                                                    volatile uint32_t* flags) {
  uint32_t status = 0;
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E;
       e += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t load[D];
#pragma unroll
    for (int d = 0; d < D; ++d) load[d] = 0;
    if (base) {
#pragma unroll
      for (int d = 0; d < D; ++d) {
        const uint64_t b = base[e * D + d];
        if (b >= kEntryLimit) status |= kFlagRange;
        load[d] = b;
      }
    }
    for (uint32_t q = 0; q < Q; ++q) {
      const uint32_t dq = mapping[e * Q + q];
      if (dq >= (uint32_t)D) {
        status |= kFlagBadMapping;
        continue;
      }
      const uint64_t k = K[(e * Q + q) * D + dq], x = X[(e * Q + q) * D + dq];
      if (k >= kEntryLimit || x >= kEntryLimit) status |= kFlagRange;
      const uint64_t c = k + x;
#pragma unroll
      for (int d = 0; d < D; ++d) load[d] += (dq == (uint32_t)d) ? c : 0;
    }
    uint64_t ms = 0;
#pragma unroll
    for (int d = 0; d < D; ++d) ms = max(ms, load[d]);
    makespan[e] = ms;
  }
  if (__any_sync(0xffffffffu, status != 0)) {
    const uint32_t all = __reduce_or_sync(0xffffffffu, status);
    if ((threadIdx.x & 31) == 0) raise_flag(flags, all);
  }
}

cudaError_t launch_score(uint32_t Q, uint32_t D, uint64_t E, const uint64_t* K, const uint64_t* X,
                         const uint64_t* base, const uint8_t* mapping, uint64_t* makespan,
                         volatile uint32_t* flags, cudaStream_t st) {
  uint64_t grid = (E + 255) / 256;
  if (grid > 148 * 16) grid = 148 * 16;
  if (grid == 0) grid = 1;
  switch (D) {
#define MCL_SCORE_CASE(DD) \
  case DD: score_kernel<DD><<<(unsigned)grid, 256, 0, st>>>(Q, E, K, X, base, mapping, makespan, flags); break;
    MCL_SCORE_CASE(1) MCL_SCORE_CASE(2) MCL_SCORE_CASE(3) MCL_SCORE_CASE(4)
    MCL_SCORE_CASE(5) MCL_SCORE_CASE(6) MCL_SCORE_CASE(7) MCL_SCORE_CASE(8)
    MCL_SCORE_CASE(9) MCL_SCORE_CASE(10) MCL_SCORE_CASE(11) MCL_SCORE_CASE(12)
    MCL_SCORE_CASE(13) MCL_SCORE_CASE(14) MCL_SCORE_CASE(15) MCL_SCORE_CASE(16)
#undef MCL_SCORE_CASE
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace mcl
