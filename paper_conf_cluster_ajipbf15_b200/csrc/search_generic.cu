// search_generic.cu -- generic exhaustive mapper search for any Q <= 32, D <= 16 with
// 64-bit loads (the correctness path for shapes outside the register-blocked kernel, and
// for D = 1 / Q < 3).
//
// Work unit: a ROW = the D mappings that share the first Q-1 digits (the last queue's
// digit k varies). Each thread walks a contiguous range of rows with an odometer, keeps
// its device loads L[d] of queues 0..Q-2 in shared memory (runtime-indexed), and scores
// every mapping of the row as max(M, L[k] + C[Q-1][k]) with M = max_d L[d] -- equal to
// max_d of the loads with queue Q-1 placed on k because every cost is >= 0
// (serialise on a device, concurrent across devices).
#include "common.cuh"
#include "kernels.h"
#include "peer.cuh"

namespace mcl {

__global__ void __launch_bounds__(256) search_generic_kernel(GenericArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q, D = a.D;
  const int nthr = blockDim.x, tid = threadIdx.x;
  // layout: C64[Q*D] | L[D*nthr] u64 | red[32] Cand | dig[(Q-1)*nthr] u8
  uint64_t* C64 = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* L = C64 + Q * D;
  Cand* red = reinterpret_cast<Cand*>(L + (size_t)D * nthr);
  uint8_t* dig = reinterpret_cast<uint8_t*>(red + 32);
  __shared__ uint32_t s_status;
  __shared__ bool s_last;
  __shared__ uint64_t s_base[kMaxDevices];
  __shared__ uint64_t s_feas;

  bool abandoned = false;  // an epoch skipped on an input error (peer exchange skipped too)
  for (uint64_t e = blockIdx.y; e < a.E; e += gridDim.y) {
    __syncthreads();
    if (tid == 0) s_status = 0;
    __syncthreads();
    const uint64_t* Ke = a.K + e * Q * D;
    const uint64_t* Xe = a.X + e * Q * D;
    for (uint32_t t = tid; t < Q * D; t += nthr) {
      const uint64_t k = Ke[t], x = Xe[t];
      if (k >= kEntryLimit || x >= kEntryLimit) s_status = kFlagRange;
      C64[t] = k + x;  // a1: aggregate cost
    }
    __syncthreads();
    if (tid < 32)  // base loads and eligibility masking (constrained variant); 64-bit loads
      epoch_prologue(C64, Q, D, a.base ? a.base + e * D : nullptr, a.elig ? a.elig + e * Q : nullptr,
                     s_base, &s_status, &s_feas);
    __syncthreads();
    if (s_status) {
      if (tid == 0 && blockIdx.x == 0) raise_flag(a.flags, s_status);
      abandoned = true;
      continue;
    }
    const uint64_t nr = a.rhi - a.rlo;
    const uint64_t T_all = (uint64_t)gridDim.x * nthr;
    const uint64_t gt = (uint64_t)blockIdx.x * nthr + tid;
    const uint64_t per = nr / T_all, rem = nr % T_all;
    uint64_t row = a.rlo + gt * per + (gt < rem ? gt : rem);
    uint64_t nleft = per + (gt < rem ? 1 : 0);
    const uint64_t* Clast = C64 + (Q - 1) * D;

    Cand best{kNone, kNone};
    if (nleft) {
      for (uint32_t d = 0; d < D; ++d) L[d * nthr + tid] = s_base[d];
      uint64_t r = row;
      for (int q = (int)Q - 2; q >= 0; --q) {  // decode the first row's digits
        const uint32_t dq = (uint32_t)(r % D);
        r /= D;
        dig[q * nthr + tid] = (uint8_t)dq;
        L[dq * nthr + tid] += C64[q * D + dq];
      }
      while (true) {
        uint64_t M = 0;
        for (uint32_t d = 0; d < D; ++d) M = max(M, L[d * nthr + tid]);
        for (uint32_t k = 0; k < D; ++k) {
          const uint64_t v = max(M, L[k * nthr + tid] + Clast[k]);
          if (v < best.ms) {  // strict: rows and k ascend, so the first minimum is kept
            best.ms = v;
            best.idx = row * D + k;
          }
        }
        if (--nleft == 0) break;
        ++row;
        for (int q = (int)Q - 2; q >= 0; --q) {  // odometer over queues 0..Q-2
          const uint32_t old = dig[q * nthr + tid];
          const uint32_t nw = (old + 1 == D) ? 0u : old + 1;
          dig[q * nthr + tid] = (uint8_t)nw;
          L[old * nthr + tid] -= C64[q * D + old];
          L[nw * nthr + tid] += C64[q * D + nw];
          if (nw != 0) break;
        }
      }
    }
    Cand c = block_min(best, red);
    if (gridDim.x == 1) {
      if (tid == 0) write_epoch(a.out, e, Q, D, a.ibits, c, a.flags, s_feas);
      continue;
    }
    if (tid == 0) {
      a.scratch[e * gridDim.x + blockIdx.x] = c;
      __threadfence();
      s_last = (atomicAdd(&a.done[e], 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last) {
      __threadfence();
      Cand r{kNone, kNone};
      for (uint32_t t = tid; t < gridDim.x; t += nthr) {
        const volatile uint64_t* o =
            reinterpret_cast<const volatile uint64_t*>(&a.scratch[e * gridDim.x + t]);
        r = cand_min(r, Cand{o[0], o[1]});
      }
      r = block_min(r, red);
      if (tid == 0) {
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags, s_feas);
        a.done[e] = 0;
      }
    }
  }
  if (a.peer.world) peer_finish(a.peer, a.out, a.E, Q, D, a.ibits, a.flags, abandoned);  // NEXT-2
}

size_t generic_smem_bytes(uint32_t Q, uint32_t D, int threads) {
  size_t b = (size_t)Q * D * 8 + (size_t)D * threads * 8 + 32 * sizeof(Cand) +
             (size_t)(Q > 1 ? Q - 1 : 0) * threads;
  return (b + 15) & ~size_t(15);
}

cudaError_t launch_generic(const GenericArgs& a, dim3 grid, int threads, size_t smem,
                           cudaStream_t st) {
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(search_generic_kernel, smem, cache);
  if (err != cudaSuccess) return err;
  search_generic_kernel<<<grid, threads, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace mcl
