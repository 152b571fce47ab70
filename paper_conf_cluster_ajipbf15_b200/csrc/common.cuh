// common.cuh -- device-side helpers shared by the mapper kernels (product path only).
//
// Result of a search (one thread, warp, CTA, epoch): the lexicographic minimum of
// (makespan, mapping index) -- PAPER.md L1048-1056 ("ideal queue-device mapping that
// minimizes the concurrent execution time") with ties to the lowest index
// (BASELINE.json north_star; reading R6).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "kernels.h"

namespace mcl {

constexpr uint64_t kNone = ~0ull;              // "no candidate" (both fields)
constexpr uint64_t kEntryLimit = 1ull << 48;   // entries must be < 2^48 (reading R10)

// Status bits written by kernels into the handle's host-mapped status word.
enum : uint32_t {
  kFlagRange = 1u,     // some cost entry >= 2^48
  kFlagNeedU64 = 2u,   // some epoch's bound sum_q max_d C >= 2^32: rerun with 64-bit loads
  kFlagNoPack = 4u,    // makespan does not fit beside the index in one u64 key (NCCL path)
};

__device__ __forceinline__ bool cand_less(const Cand& a, const Cand& b) {
  return a.ms < b.ms || (a.ms == b.ms && a.idx < b.idx);
}

__device__ __forceinline__ Cand cand_min(const Cand& a, const Cand& b) {
  return cand_less(b, a) ? b : a;
}

__device__ __forceinline__ Cand warp_min(Cand c) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    Cand o;
    o.ms = __shfl_xor_sync(0xffffffffu, c.ms, off);
    o.idx = __shfl_xor_sync(0xffffffffu, c.idx, off);
    c = cand_min(c, o);
  }
  return c;
}

// CTA-wide minimum; every thread must call it. Returns the result in thread 0.
// `red` is shared scratch of >= 32 Cand.
__device__ __forceinline__ Cand block_min(Cand c, Cand* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int nwarps = (blockDim.x + 31) >> 5;
  c = warp_min(c);
  if (nwarps == 1) return c;
  __syncthreads();  // protect `red` against a previous use
  if (lane == 0) red[warp] = c;
  __syncthreads();
  if (warp == 0) {
    c = (lane < nwarps) ? red[lane] : Cand{kNone, kNone};
    c = warp_min(c);
  }
  return c;
}

__device__ __forceinline__ void raise_flag(volatile uint32_t* flags, uint32_t bit) {
  if (flags) atomicOr((uint32_t*)flags, bit);
}

// Bits needed to hold every index of an N-mapping space (N >= 1): ceil(log2(N)).
__host__ __device__ __forceinline__ int index_bits(uint64_t N) {
  int b = 0;
  while (b < 64 && (N - 1) >> b) ++b;
  return b;
}

__device__ __forceinline__ void write_epoch(const EpochOut& o, uint64_t e, uint32_t Q, uint32_t D,
                                            int ibits, const Cand& c, volatile uint32_t* flags) {
  if (o.key) {
    // multi-GPU: publish the packed key; outputs are decoded after the all-reduce
    const bool fits = (ibits == 0) || (c.ms < (1ull << (64 - ibits)));
    if (!fits) raise_flag(flags, kFlagNoPack);
    o.key[e] = fits ? ((ibits == 0 ? 0ull : (c.ms << ibits)) | c.idx) : kNone;
    if (o.pair) {
      o.pair[2 * e] = c.ms;
      o.pair[2 * e + 1] = c.idx;
    }
    return;
  }
  o.index[e] = c.idx;
  o.makespan[e] = c.ms;
  if (o.mapping) {
    uint64_t rest = c.idx;
    for (int q = (int)Q - 1; q >= 0; --q) {
      o.mapping[e * Q + (uint64_t)q] = (uint8_t)(rest % D);
      rest /= D;
    }
  }
}

}  // namespace mcl
