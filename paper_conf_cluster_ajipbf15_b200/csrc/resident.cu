// resident.cu -- a resident mapper for online decisions (cfg1-sized searches).
//
// The paper's mapper runs at every scheduling epoch, inside the runtime's scheduler thread,
// and its decision is on the application's critical path (the search
// must stay "negligible"). A launch per decision costs a kernel launch, the launch ramp and
// a stream synchronisation (~15 us per call, SS12), far more than scoring 81
// mappings. Here ONE warp stays resident on the GPU and serves decisions from a mailbox in
// pinned, device-mapped host memory: the host writes an epoch batch's K and X and then a
// request number; the warp (polling the request number over PCIe) reads the inputs in
// place, scores every mapping (the same definition as every other path: C = K + X,
// PAPER.md L2106-2118; loads per device, makespan = max over devices, L1048-1052; argmin
// with the lowest index on ties) and answers with one record per epoch of three words
// (index, makespan, packed digits), each stored whole and tagged with the request number,
// so the host accepts the answer without a fence or a separate done flag (kernels.h,
// ResidentArgs). No launch, no copy engine, no stream synchronisation per decision.
//
// Shape: any Q <= 16, D <= 16 with D^Q <= 8192: one warp up to 4096 mappings (lane l scores
// mappings l, l + 32, ... in increasing order keeping its first strict minimum, then five
// shuffle rounds of the lexicographic (makespan, index) minimum), 8 warps above (the same per
// warp, then the warps' minima in shared memory; thread 0 alone polls the mailbox). The
// kernel exits when the host sets `stop`, or after `idle_ns` without a request (the host
// relaunches it on demand).
#include "common.cuh"
#include "kernels.h"

namespace mcl {

namespace {

__device__ __forceinline__ uint64_t ld_acquire_sys64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_sys64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_sys64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t now_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Lowest-index minimum makespan of one epoch (C = [Q][D] composed costs in shared memory),
// by the NT = 32 * W threads: thread t scores m = t, t + NT, ... in increasing order
// (strict <), then five shuffle rounds of the lexicographic (makespan, index) minimum per
// warp and, for W > 1, one more over the warps' results in shared memory (every thread
// returns the epoch's result). QT, DT > 0: shape fixed at compile time (digits by constant
// division, loads in registers by static selects); 0: runtime shape (loads in this
// thread's shared-memory row).
template <int QT, int DT, int W>
__device__ __forceinline__ void score_epoch(const uint64_t* C, uint32_t Qr, uint32_t Dr, uint32_t N,
                                            uint64_t* sL, uint64_t* s_wms, uint32_t* s_wm,
                                            uint64_t& best_ms, uint32_t& best_m) {
  constexpr uint32_t NT = 32u * W;
  const uint32_t tid = threadIdx.x;
  const int lane = threadIdx.x & 31;
  uint64_t bms = ~0ull;
  uint32_t bm = 0xffffffffu;
  if constexpr (QT > 0) {
    // Thread t walks a contiguous range of PREFIXES (the digits of queues 0..QT-2) in
    // increasing order, stepping an odometer over them (loads updated by one-hot selects,
    // static register indices); for each prefix the DT leaves of the last queue are scored
    // with static k: makespan = max(L[k] + C[QT-1][k], max of the other devices' loads).
    // About 5x fewer instructions than decoding every mapping from scratch.
    uint64_t c[QT][DT];
#pragma unroll
    for (int q = 0; q < QT; ++q)
#pragma unroll
      for (int d = 0; d < DT; ++d) c[q][d] = C[q * DT + d];
    const uint32_t P = N / DT;  // prefixes (N = DT^QT)
    const uint32_t per = (P + NT - 1) / NT;
    const uint32_t p0 = min(P, tid * per), p1 = min(P, p0 + per);
    if (p0 < p1) {
      uint32_t dig[QT > 1 ? QT - 1 : 1];
      uint64_t L[DT];
#pragma unroll
      for (int d = 0; d < DT; ++d) L[d] = 0;
      uint32_t rest = p0;
#pragma unroll
      for (int q = QT - 2; q >= 0; --q) {  // queue 0 is the most significant digit
        const uint32_t dq = rest % DT;
        rest /= DT;
        dig[q] = dq;
#pragma unroll
        for (int d = 0; d < DT; ++d) L[d] += (dq == (uint32_t)d) ? c[q][d] : 0;  // a3
      }
      for (uint32_t pp = p0; pp < p1; ++pp) {
#pragma unroll
        for (int k = 0; k < DT; ++k) {  // a4: leaves of this prefix, increasing index
          uint64_t mo = 0;
#pragma unroll
          for (int d = 0; d < DT; ++d)
            if (d != k) mo = max(mo, L[d]);
          const uint64_t ms = max(mo, L[k] + c[QT - 1][k]);
          if (ms < bms) {  // a5: strict, so the thread keeps its lowest index of a tie
            bms = ms;
            bm = pp * DT + (uint32_t)k;
          }
        }
#pragma unroll
        for (int q = QT - 2; q >= 0; --q) {  // odometer step to the next prefix
          const uint32_t old = dig[q];
          const uint32_t nw = (old + 1 == (uint32_t)DT) ? 0u : old + 1;
#pragma unroll
          for (int d = 0; d < DT; ++d)
            L[d] += ((nw == (uint32_t)d) ? c[q][d] : 0) - ((old == (uint32_t)d) ? c[q][d] : 0);
          dig[q] = nw;
          if (nw != 0) break;
        }
      }
    }
  } else {
    for (uint32_t m = tid; m < N; m += NT) {
      for (uint32_t d = 0; d < Dr; ++d) sL[d] = 0;
      uint32_t rest = m;
      for (int q = (int)Qr - 1; q >= 0; --q) {
        const uint32_t dq = rest % Dr;
        rest /= Dr;
        sL[dq] += C[q * Dr + dq];
      }
      uint64_t ms = 0;
      for (uint32_t d = 0; d < Dr; ++d) ms = max(ms, sL[d]);
      if (ms < bms) {
        bms = ms;
        bm = m;
      }
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {  // lexicographic (makespan, index) minimum
    const uint64_t oms = __shfl_xor_sync(0xffffffffu, bms, off);
    const uint32_t om = __shfl_xor_sync(0xffffffffu, bm, off);
    if (oms < bms || (oms == bms && om < bm)) {
      bms = oms;
      bm = om;
    }
  }
  if constexpr (W > 1) {  // across the warps (every warp's lane 0 holds its minimum)
    const int w = (int)(tid >> 5);
    if (lane == 0) {
      s_wms[w] = bms;
      s_wm[w] = bm;
    }
    __syncthreads();
    bms = s_wms[0];
    bm = s_wm[0];
#pragma unroll
    for (int v = 1; v < W; ++v) {
      const uint64_t oms = s_wms[v];
      const uint32_t om = s_wm[v];
      if (oms < bms || (oms == bms && om < bm)) {
        bms = oms;
        bm = om;
      }
    }
    __syncthreads();  // s_wms / s_wm are rewritten by the next epoch
  }
  best_ms = bms;
  best_m = bm;
}

}  // namespace

template <int QT, int DT, int W>
__global__ void __launch_bounds__(32 * W) resident_kernel(ResidentArgs a) {
  extern __shared__ __align__(16) uint64_t s_res[];
  constexpr uint32_t NT = 32u * W;
  const uint32_t tid = threadIdx.x;
  const uint32_t Q = QT > 0 ? QT : a.Q, D = DT > 0 ? DT : a.D, N = a.N, QD = Q * D;
  uint64_t* sC = s_res;                                  // [cap][Q][D] composed costs
  uint64_t* sL = s_res + (size_t)a.cap * QD + tid * 16;  // generic shapes: this thread's loads
  __shared__ uint64_t s_req;                             // W > 1: the request, broadcast
  __shared__ uint32_t s_quit;
  __shared__ uint64_t s_wms[W];                          // W > 1: per-warp minima
  __shared__ uint32_t s_wm[W];
  ResidentBox* box = a.box;
  uint32_t last = a.seq0;
  uint64_t t_idle = now_ns();
  for (;;) {
    // ---- wait for a request: thread 0 polls one word (number, epochs, stop) over PCIe ----
    uint64_t req = 0;
    uint32_t quit = 0;
    if (tid == 0) {
      // one acquire load of the request word at a time: measured, several relaxed loads
      // in flight (4 or 8, staggered), a pause between polls, or polling tagged inputs
      // together with the request word only add latency (SS7, resident mapper)
      for (;;) {
        req = ld_acquire_sys64(&box->req);
        if (req >> 63) {
          quit = 1;
          break;
        }
        if ((uint32_t)req != last) break;
        if (now_ns() - t_idle > a.idle_ns) {
          quit = 2;
          break;
        }
      }
    }
    if constexpr (W == 1) {
      quit = __shfl_sync(0xffffffffu, quit, 0);
      req = __shfl_sync(0xffffffffu, req, 0);
    } else {  // the other warps wait at the barrier (no polling of their own)
      if (tid == 0) {
        s_req = req;
        s_quit = quit;
      }
      __syncthreads();
      req = s_req;
      quit = s_quit;
    }
    if (quit) {
      if (tid == 0) {
        box->exit_reason = quit;
        st_release_sys(&box->alive, 0u);
      }
      return;
    }
    const uint32_t seq = (uint32_t)req, E = (uint32_t)(req >> 32) & 0xffffu;
    last = seq;
#ifdef MCL_RESIDENT_TRACE
    const uint64_t tr0 = now_ns();
#endif
    // ---- inputs, read in place from host memory after the acquire (a1: C = K + X) ----
    uint32_t status = 0;
    if (E > a.cap || E == 0) status |= kFlagBadModel;
    const uint32_t n = (E <= a.cap ? E : 0u) * QD;
    bool bad = false;
    for (uint32_t i0 = tid; i0 < n; i0 += 4 * NT) {  // 8 loads in flight per thread (PCIe)
      uint64_t k[4], x[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t i = i0 + NT * u;
        k[u] = i < n ? ld_relaxed_sys64(a.K + i) : 0;
        x[u] = i < n ? ld_relaxed_sys64(a.X + i) : 0;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t i = i0 + NT * u;
        bad |= (k[u] >= kEntryLimit) | (x[u] >= kEntryLimit);
        if (i < n) sC[i] = k[u] + x[u];
      }
    }
    if constexpr (W == 1) {
      if (__any_sync(0xffffffffu, bad)) status |= kFlagRange;
      __syncwarp();
    } else {
      if (__syncthreads_or(bad)) status |= kFlagRange;
    }
#ifdef MCL_RESIDENT_TRACE
    const uint64_t tr1 = now_ns();
#endif
    // digit width b: the smallest b with D <= 2^b (0 for D = 1); Q * b <= 16 for D^Q <= 8192
    const uint32_t b = D <= 1 ? 0u : 32u - __clz(D - 1);
    for (uint32_t e = 0; e < (status == 0 ? E : 1u); ++e) {
      uint64_t ms = 0;
      uint32_t idx = 0;
      if (status == 0) score_epoch<QT, DT, W>(sC + (size_t)e * QD, Q, D, N, sL, s_wms, s_wm, ms, idx);
      uint64_t* rec = a.rec + (size_t)e * kResidentRecWords;
      if (tid == 0) {
        st_relaxed_sys64(rec + 0, ((uint64_t)seq << 32) | ((uint64_t)status << 16) | idx);
      } else if (tid == 1) {
        st_relaxed_sys64(rec + 1, ((uint64_t)(seq & 0x7ffu) << 53) | ms);
      } else if (tid == 2) {  // a7: digits of the index, queue 0 most significant
        uint32_t rest = idx, packed = 0;
        for (int q = (int)Q - 1; q >= 0; --q) {
          packed |= (rest % D) << (q * b);
          rest /= D;
        }
        st_relaxed_sys64(rec + 2, ((uint64_t)seq << 32) | packed);
      }
    }
#ifdef MCL_RESIDENT_TRACE
    if (tid == 0) {
      box->trace[0] = tr0;
      box->trace[1] = tr1;
      box->trace[2] = now_ns();
      box->trace[3] = box->trace[2];
    }
#endif
    t_idle = now_ns();
  }
}

// Decisions above kResidentWarpMappings (e.g. the paper's FT: 8 queues x 3 devices = 6561
// mappings) are scored by 8 warps: one warp alone took 44 us per 8 x 3 decision, more than
// a launch per call (19 us device-resident).
#ifndef MCL_RESIDENT_WARP_MAPPINGS
#define MCL_RESIDENT_WARP_MAPPINGS 4096
#endif
constexpr uint32_t kResidentWarpMappings = MCL_RESIDENT_WARP_MAPPINGS;
#ifndef MCL_RESIDENT_WIDE
#define MCL_RESIDENT_WIDE 8
#endif
constexpr int kResidentWide = MCL_RESIDENT_WIDE;

cudaError_t launch_resident(const ResidentArgs& a, cudaStream_t st) {
  const bool wide = a.N > kResidentWarpMappings;
  void (*k)(ResidentArgs) = wide ? resident_kernel<0, 0, kResidentWide> : resident_kernel<0, 0, 1>;
  bool generic = true;
  switch (a.Q * 100 + a.D) {  // compile-time shapes of small decisions (cfg1: 4 x 3; FT: 8 x 3)
#define MCL_RES_CASE(QQ, DD)                                                              \
  case QQ * 100 + DD:                                                                     \
    k = wide ? resident_kernel<QQ, DD, kResidentWide> : resident_kernel<QQ, DD, 1>;       \
    generic = false;                                                                      \
    break;
    MCL_RES_CASE(2, 2) MCL_RES_CASE(2, 3) MCL_RES_CASE(2, 4) MCL_RES_CASE(3, 2) MCL_RES_CASE(3, 3)
    MCL_RES_CASE(3, 4) MCL_RES_CASE(4, 2) MCL_RES_CASE(4, 3) MCL_RES_CASE(4, 4) MCL_RES_CASE(5, 3)
    MCL_RES_CASE(5, 4) MCL_RES_CASE(6, 3) MCL_RES_CASE(6, 4) MCL_RES_CASE(8, 2) MCL_RES_CASE(8, 3)
#undef MCL_RES_CASE
    default: break;
  }
  const uint32_t threads = 32u * (wide ? kResidentWide : 1);
  // composed costs of up to cap epochs, plus one 16-entry load row per thread for the
  // generic (runtime-shape) kernel
  const size_t smem = ((size_t)a.cap * a.Q * a.D + (generic ? threads * 16 : 0)) * sizeof(uint64_t);
  // the compile-time shapes need at most 64 x 8 x 4 entries (16 KB, under the default
  // 48 KB); only the generic kernels (one cache each) may need the larger opt-in
  if (generic) {
    static SmemAttrCache cache[2];
    cudaError_t err = ensure_smem(k, smem, cache[wide ? 1 : 0]);
    if (err != cudaSuccess) return err;
  }
  k<<<1, threads, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace mcl
