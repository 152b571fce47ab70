// peer.cuh -- fused cross-GPU exchange at the end of a sharded search kernel (SURVEY SS8(f)
// NEXT-2; include/mcl.h mcl_peer_export / mcl_peer_import).
//
// Replaces "search kernel -> ncclAllReduce(MIN) -> decode kernel" by one kernel: when the
// last CTA of this rank's search is done (every epoch's packed key written locally), it
// runs exchange ROUNDS over NVLink / NVSwitch peer memory. Round R:
//   1. add this rank's value of every epoch to region R % 2 of EVERY rank's slab with a
//      system-scope atomicMin (the reduction happens in the owners' memory);
//   2. fence (system scope), then add 1 to every rank's signal counter;
//   3. wait until this rank's counter reaches world * (R + 1): all ranks' values are in;
//   4. read the global minimum of every epoch from this rank's own region, and reset the
//      region's words to kNone (UINT64_MAX) for round R + 2.
// Why one reset per round is enough: other ranks write region R % 2 again only in round
// R + 2, which they enter after the barrier of round R + 1, which needs this rank's signal
// of round R + 1 -- issued after the reset in program order, behind a system fence.
// Every rank runs the same rounds (identical inputs; the two-step decision below depends
// only on reduced values), so the counters stay in lock-step. The number of completed
// rounds lives in the slab (word 1), so the host never tracks it.
//
// Values: round A = the packed keys (makespan << ibits | index; kNone when a makespan does
// not fit). If some epoch's reduced key is kNone, no rank's candidate fitted and two more
// rounds give the lexicographic minimum: B = the makespans, C = the indices of the ranks
// whose makespan equals the global one (the NCCL path's two-step, reduce.cu).
#pragma once
#include "common.cuh"

namespace mcl {

__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Reductions without a returned value (RED): no round trip per contribution.
__device__ __forceinline__ void red_min_relaxed_sys(uint64_t* p, uint64_t v) {
  asm volatile("red.relaxed.sys.global.min.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void red_add_relaxed_sys(uint64_t* p, uint64_t v) {
  asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }

__device__ __forceinline__ uint32_t atom_add_acq_rel_gpu(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}

// One exchange round (steps 1-3), run by the whole last CTA. value(e) is this rank's
// contribution for epoch e. Returns false if some rank did not signal within the timeout.
// Ordering: the contributions (relaxed, system scope, any thread of the CTA) come before
// the barrier; thread 0 then fences (acq_rel, system scope) and signals every rank, so a rank whose
// ACQUIRE load sees the signal also sees every contribution (causality through the CTA
// barrier and the release/acquire pair, PTX memory model).
template <typename F>
static __device__ bool peer_round(const PeerArgs& p, uint64_t R, uint64_t E, F value) {
  const uint64_t region = kPeerHeaderWords + (R & 1) * p.cap;
  __syncthreads();  // values computed by other threads of the CTA are visible
  for (uint64_t i = threadIdx.x; i < E * (uint64_t)p.world; i += blockDim.x) {
    const uint64_t e = i / (uint64_t)p.world;
    const int r = (int)(i % (uint64_t)p.world);
    const uint64_t v = value(e);
    if (v != kNone) red_min_relaxed_sys(p.slabs[r] + region + e, v);
  }
  __syncthreads();
  __shared__ int s_ok;
  if (threadIdx.x == 0) {
    fence_acq_rel_sys();  // release pattern: one fence, then relaxed signals to every rank
    for (int r = 0; r < p.world; ++r) red_add_relaxed_sys(p.slabs[r], 1ull);
    const uint64_t want = (R + 1) * (uint64_t)p.world;
    const uint64_t t0 = global_ns();
    int ok = 1;
    while (ld_acquire_sys(p.mine) < want) {
      if (global_ns() - t0 > p.timeout_ns) {
        ok = 0;
        break;
      }
      __nanosleep(64);
    }
    s_ok = ok;
  }
  __syncthreads();
  return s_ok != 0;
}

// Read-and-reset epoch e of this rank's region of round R (step 4).
__device__ __forceinline__ uint64_t peer_take(const PeerArgs& p, uint64_t R, uint64_t e) {
  volatile uint64_t* w = p.mine + kPeerHeaderWords + (R & 1) * p.cap + e;
  const uint64_t v = *w;
  *w = kNone;
  return v;
}

// Called by EVERY CTA of a sharded search kernel after its last epoch. The last CTA to get
// here runs the exchange and writes the public outputs o.index / o.makespan / o.mapping
// from the global result. `abandoned`: this CTA skipped an epoch on an input error or for
// the 64-bit rerun; then the whole exchange is skipped (identical on every rank, since all
// ranks see the same inputs). Only GPU-scope ordering is needed up to here: the other CTAs'
// keys (written by their thread 0) are read by this GPU's last CTA alone, so an acq_rel
// counter increment replaces fences. Measured on one B200 (scripts/archive/collective_compare.sh,
// scripts/archive/peer_tail_bench.cu): a system-scope fence per CTA plus a read of the host-mapped
// status word made the tail ~17 us; as written it adds ~6 us to the search kernel at
// world = 1 -- a chain of dependent memory round trips (round counter, keys, reduction,
// fence, signal, poll, read-back, outputs), of which the counting and one round alone are
// ~2 us in isolation.
static __device__ __forceinline__ void peer_finish(const PeerArgs& p, const EpochOut& o, uint64_t E,
                                                   uint32_t Q, uint32_t D, int ibits,
                                                   volatile uint32_t* flags, bool abandoned) {
  __shared__ bool s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    if (abandoned) atomicOr(&p.kdone[1], 1u);
    s_last = (atom_add_acq_rel_gpu(&p.kdone[0], 1u) == gridDim.x * gridDim.y * gridDim.z - 1);
  }
  __syncthreads();
  if (!s_last) return;
  const bool skip = *reinterpret_cast<volatile uint32_t*>(&p.kdone[1]) != 0;
  __syncthreads();
  if (threadIdx.x == 0) {  // self-reset for the next call
    p.kdone[0] = 0;
    p.kdone[1] = 0;
  }
  if (skip) return;

  uint64_t R = *reinterpret_cast<volatile uint64_t*>(p.mine + 1);
  const uint64_t mask = (ibits >= 64) ? ~0ull : ((1ull << ibits) - 1);
  // round A: packed keys
  if (!peer_round(p, R, E, [&](uint64_t e) { return ld_relaxed_gpu(o.key + e); })) {
    if (threadIdx.x == 0) raise_flag(flags, kFlagPeerTimeout);
    return;
  }
  int unpacked = 0;
  for (uint64_t e = threadIdx.x; e < E; e += blockDim.x) {
    const uint64_t k = peer_take(p, R, e);
    if (k == kNone) {
      unpacked = 1;
      continue;
    }
    const uint64_t ms = (ibits == 0) ? k : (ibits >= 64 ? 0 : (k >> ibits));
    write_result(o.index, o.makespan, o.mapping, e, Q, D, k & mask, ms);
  }
  ++R;
  if (__syncthreads_or(unpacked)) {
    // round B: global makespans
    if (!peer_round(p, R, E, [&](uint64_t e) { return ld_relaxed_gpu(o.pair + 2 * e); })) {
      if (threadIdx.x == 0) raise_flag(flags, kFlagPeerTimeout);
      return;
    }
    for (uint64_t e = threadIdx.x; e < E; e += blockDim.x) p.gms[e] = peer_take(p, R, e);
    ++R;
    // round C: lowest index among the ranks holding the global makespan
    if (!peer_round(p, R, E, [&](uint64_t e) {
          return (ld_relaxed_gpu(o.pair + 2 * e) == p.gms[e]) ? ld_relaxed_gpu(o.pair + 2 * e + 1) : kNone;
        })) {
      if (threadIdx.x == 0) raise_flag(flags, kFlagPeerTimeout);
      return;
    }
    for (uint64_t e = threadIdx.x; e < E; e += blockDim.x)
      write_result(o.index, o.makespan, o.mapping, e, Q, D, peer_take(p, R, e), p.gms[e]);
    ++R;
    if (threadIdx.x == 0) raise_flag(flags, kFlagTwoStep);
  }
  __syncthreads();
  if (threadIdx.x == 0) *reinterpret_cast<volatile uint64_t*>(p.mine + 1) = R;
}

}  // namespace mcl
