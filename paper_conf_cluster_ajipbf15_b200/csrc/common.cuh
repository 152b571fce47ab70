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
constexpr int kMaxDevices = 16;                // D <= 16 (include/mcl.h)
constexpr int kMaxQueues = 32;                 // Q <= 32
constexpr uint64_t kEntryLimit = 1ull << 48;   // entries must be < 2^48 (reading R10)

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

// Epoch prologue, run by ONE WARP after C64[Q][D] = K + X is in shared memory (a1):
//  * base loads (constrained variant, NEXT-3): s_base[d] = base_e[d] (0 without them) --
//    load already on device d from queues outside the pool (SCHED_OFF);
//  * eligibility: a forbidden entry C64[q][d] (mask != 0 and bit d clear) is replaced by
//    INF = UB_f + 1, where UB_f = max_d base + sum_q max over q's eligible d of C is an upper
//    bound of every feasible makespan; a mapping using a forbidden entry then has a load
//    >= INF > any feasible makespan, so the argmin (and its lowest-index tie rule) ranges
//    over feasible mappings only;
//  * returns UB = max_d base + sum_q max_d C64 (after masking): every makespan is <= UB,
//    which decides 32- vs 64-bit load arithmetic.
// status |= kFlagRange (a base load >= 2^48) / kFlagInfeasible (a queue with no eligible
// device below D). Q <= 32, D <= 16: lane q handles queue q.
// *s_feasible receives UB_f when masks are given (a candidate above it is infeasible: only
// possible in a sub-range search whose range holds no feasible mapping), else kNone.
__device__ __forceinline__ uint64_t epoch_prologue(uint64_t* C64, uint32_t Q, uint32_t D,
                                                   const uint64_t* base_e, const uint16_t* elig_e,
                                                   uint64_t* s_base, uint32_t* status,
                                                   uint64_t* s_feasible) {
  const int lane = threadIdx.x & 31;
  uint64_t b = 0;
  if (lane < (int)D) {
    b = base_e ? base_e[lane] : 0;
    s_base[lane] = b;
  }
  const bool bad_base = __any_sync(0xffffffffu, b >= kEntryLimit);
  uint64_t bmax = b;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) bmax = max(bmax, __shfl_xor_sync(0xffffffffu, bmax, off));
  uint32_t mask = 0;
  uint64_t row_f = 0;  // max over eligible devices
  bool feasible = true;
  if (lane < (int)Q) {
    mask = elig_e ? (uint32_t)elig_e[lane] : 0u;
    bool any = false;
    for (uint32_t d = 0; d < D; ++d)
      if (mask == 0 || ((mask >> d) & 1u)) {
        row_f = max(row_f, C64[lane * D + d]);
        any = true;
      }
    feasible = any;
  }
  const bool infeasible = __any_sync(0xffffffffu, !feasible);
  uint64_t ubf = row_f;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) ubf += __shfl_xor_sync(0xffffffffu, ubf, off);
  ubf += bmax;
  uint64_t row = 0;
  if (lane < (int)Q) {
    for (uint32_t d = 0; d < D; ++d) {
      if (mask != 0 && !((mask >> d) & 1u)) C64[lane * D + d] = ubf + 1;  // INF
      row = max(row, C64[lane * D + d]);
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) row += __shfl_xor_sync(0xffffffffu, row, off);
  if (lane == 0) {
    if (bad_base) *status |= kFlagRange;
    if (infeasible) *status |= kFlagInfeasible;
    *s_feasible = elig_e ? ubf : kNone;
  }
  __syncwarp();
  return row + bmax;
}

// Public outputs of epoch e: index, makespan and (optionally) the index's base-D digits,
// queue 0 most significant (reading R2); 0xFF bytes for "no mapping" (kNone).
__device__ __forceinline__ void write_result(uint64_t* index, uint64_t* makespan, uint8_t* mapping,
                                             uint64_t e, uint32_t Q, uint32_t D, uint64_t idx,
                                             uint64_t ms) {
  index[e] = idx;
  makespan[e] = ms;
  if (mapping) {
    uint64_t rest = idx;
    for (int q = (int)Q - 1; q >= 0; --q) {
      mapping[e * Q + (uint64_t)q] = (idx == kNone) ? 0xFF : (uint8_t)(rest % D);
      rest /= D;
    }
  }
}

// `feasible`: candidates above it are infeasible (constrained sub-range searches) and are
// reported as (kNone, kNone); kNone when unconstrained.
__device__ __forceinline__ void write_epoch(const EpochOut& o, uint64_t e, uint32_t Q, uint32_t D,
                                            int ibits, Cand c, volatile uint32_t* flags,
                                            uint64_t feasible = kNone) {
  if (c.ms != kNone && c.ms > feasible) c = Cand{kNone, kNone};
  if (o.key) {
    // multi-GPU: publish the packed key; outputs are decoded after the all-reduce. A
    // makespan that does not fit beside the index publishes kNone: it is larger than every
    // key that fits, so it can only be the global minimum if no rank's candidate fits --
    // which the decode step detects on the REDUCED key (identical on every rank, so every
    // rank takes the same two-step decision; a local flag could differ between ranks).
    const bool none = (c.ms == kNone);
    const bool fits = none || (ibits == 0) || (c.ms < (1ull << (64 - ibits)));
    o.key[e] = (fits && !none) ? ((ibits == 0 ? 0ull : (c.ms << ibits)) | c.idx) : kNone;
    if (o.pair) {
      o.pair[2 * e] = c.ms;
      o.pair[2 * e + 1] = c.idx;
    }
    return;
  }
  write_result(o.index, o.makespan, o.mapping, e, Q, D, c.idx, c.ms);
}

}  // namespace mcl
