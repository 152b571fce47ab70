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

// Static command-queue scheduling (SCHED_AUTO_STATIC): "we statically
// decide the command queue schedules based only on the device profiles ... [using] the
// command queue properties (compute intensive, memory intensive, or I/O intensive) as the
// selection criterion and [choose] the best available device for the given command queue"
// (reading R18). Thread per (epoch, queue): among the queue's eligible devices,
// the one whose device-profile cost for the queue's class is lowest (ties: lowest device).
// No kernel profiles and no search: the policy baseline the mapper is compared with.
__global__ void __launch_bounds__(256) static_map_kernel(uint32_t Q, uint32_t D, uint64_t EQ,
                                                         const uint8_t* __restrict__ hints,
                                                         uint32_t num_classes,
                                                         const uint64_t* __restrict__ score,
                                                         const uint16_t* __restrict__ elig,
                                                         uint8_t* __restrict__ mapping,
                                                         volatile uint32_t* flags) {
  __shared__ uint64_t s_score[kMaxDevices * kMaxDevices];
  for (uint32_t t = threadIdx.x; t < num_classes * D; t += blockDim.x) s_score[t] = score[t];
  __syncthreads();
  uint32_t status = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < EQ;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t c = hints[i];
    const uint32_t m = elig ? (uint32_t)elig[i] : 0u;
    uint32_t best_d = 0xffu;
    uint64_t best = ~0ull;
    if (c >= num_classes) {
      status |= kFlagBadHint;
    } else {
      for (uint32_t d = 0; d < D; ++d) {
        if (m != 0 && !((m >> d) & 1u)) continue;
        const uint64_t v = s_score[c * D + d];
        if (best_d == 0xffu || v < best) {  // strict: the lowest device among equal scores
          best = v;
          best_d = d;
        }
      }
      if (best_d == 0xffu) status |= kFlagInfeasible;
    }
    mapping[i] = (uint8_t)best_d;
  }
  if (__any_sync(0xffffffffu, status != 0)) {
    const uint32_t all = __reduce_or_sync(0xffffffffu, status);
    if ((threadIdx.x & 31) == 0) raise_flag(flags, all);
  }
}

cudaError_t launch_static_map(uint32_t Q, uint32_t D, uint64_t E, const uint8_t* hints,
                              uint32_t num_classes, const uint64_t* score, const uint16_t* elig,
                              uint8_t* mapping, volatile uint32_t* flags, cudaStream_t st) {
  const uint64_t EQ = E * Q;
  uint64_t grid = (EQ + 255) / 256;
  if (grid > 148 * 16) grid = 148 * 16;
  if (grid == 0) grid = 1;
  static_map_kernel<<<(unsigned)grid, 256, 0, st>>>(Q, D, EQ, hints, num_classes, score, elig, mapping, flags);
  return cudaGetLastError();
}

}  // namespace mcl
