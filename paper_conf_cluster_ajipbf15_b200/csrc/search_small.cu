// search_small.cu -- batched search for tiny index spaces (D^Q <= 81), one thread per epoch
// (FDM-Seismology 2 queues x 3 devices x 10^6 epochs, and cfg1).
//
// The work per epoch is a handful of integer ops; the kernel is bound by HBM (96 B of
// costs in, 18 B of results out per epoch at Q=2, D=3). A persistent grid streams tiles of
// blockDim.x epochs: one elected thread moves a tile's K and X slabs global -> shared with
// cp.async.bulk (the TMA bulk-copy engine, SASS UBLKCP) completing on mbarriers, several
// stages deep so tiles are in flight while the current one is scored. Each thread then
// scores its epoch's D^Q mappings from shared memory with compile-time digits (so every
// load index is static), in increasing index order with a strict '<' (lowest index wins
// ties, BASELINE.json north_star), and writes its outputs coalesced.
#include "common.cuh"
#include "kernels.h"

namespace mcl {

namespace {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

template <int Q, int D>
struct Pow {
  static constexpr int N = D * Pow<Q - 1, D>::N;
};
template <int D>
struct Pow<0, D> {
  static constexpr int N = 1;
};

}  // namespace

constexpr int kMaxSmallStages = 16;  // tiles in flight per CTA (TMA bulk copies), upper bound

template <int Q, int D>
__global__ void __launch_bounds__(256) search_small_kernel(SmallArgs a, int use_tma, int kSmallStages) {
  constexpr int QD = Q * D;
  constexpr int N = Pow<Q, D>::N;
  constexpr bool kVec = (QD % 2) == 0;  // a row of QD u64 is a whole number of 16-B vectors
  extern __shared__ __align__(128) unsigned char smem_raw[];
  __shared__ __align__(8) uint64_t full[kMaxSmallStages];
  const int TE = blockDim.x, tid = threadIdx.x;
  const size_t slab = (size_t)TE * QD;  // u64 per array per stage
  uint64_t* sbase = reinterpret_cast<uint64_t*>(smem_raw);
  auto sK = [&](int s) { return sbase + (size_t)(2 * s) * slab; };
  auto sX = [&](int s) { return sbase + (size_t)(2 * s + 1) * slab; };

  const uint64_t E = a.E;
  const uint64_t ntiles = (E + TE - 1) / TE;
  // a tile goes through TMA iff it is full (the ragged last tile uses plain loads) and the
  // caller's pointers are 16-byte aligned (use_tma)
  auto tile_tma = [&](uint64_t t) { return use_tma && (t + 1) * TE <= E; };
  auto issue = [&](uint64_t t, int s) {
    const uint32_t bytes = (uint32_t)(slab * 8);
    fence_proxy_async();
    mbar_expect_tx(&full[s], 2 * bytes);
    bulk_g2s(sK(s), a.K + t * slab, bytes, &full[s]);
    bulk_g2s(sX(s), a.X + t * slab, bytes, &full[s]);
  };
  if (tid == 0) {
    for (int s = 0; s < kSmallStages; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // prologue: up to kSmallStages of this CTA's tiles in flight
  if (tid == 0) {
    uint64_t t = blockIdx.x;
    for (int s = 0; s < kSmallStages && t < ntiles; ++s, t += gridDim.x)
      if (tile_tma(t)) issue(t, s);
  }
  uint32_t phase_bits = 0;  // bit s = parity to wait for on stage s
  bool bad = false;
  int s = 0;
  for (uint64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    if (tile_tma(t)) {
      mbar_wait(&full[s], (phase_bits >> s) & 1u);
      phase_bits ^= 1u << s;
    } else {
      const uint64_t n = (E - t * TE < (uint64_t)TE) ? E - t * TE : (uint64_t)TE;
      for (uint64_t j = tid; j < n * QD; j += TE) {
        sK(s)[j] = a.K[t * slab + j];
        sX(s)[j] = a.X[t * slab + j];
      }
      __syncthreads();
    }
    const uint64_t e = t * TE + tid;
    if (e < E) {
      uint64_t kv[QD], xv[QD];
      const uint64_t* k = sK(s) + (size_t)tid * QD;
      const uint64_t* x = sX(s) + (size_t)tid * QD;
      if (kVec) {  // 16-byte shared loads; a 48-B row stride keeps each quarter-warp conflict-free
#pragma unroll
        for (int j = 0; j < QD; j += 2) {
          const ulonglong2 k2 = *reinterpret_cast<const ulonglong2*>(k + j);
          const ulonglong2 x2 = *reinterpret_cast<const ulonglong2*>(x + j);
          kv[j] = k2.x;
          kv[j + 1] = k2.y;
          xv[j] = x2.x;
          xv[j + 1] = x2.y;
        }
      } else {
#pragma unroll
        for (int j = 0; j < QD; ++j) {
          kv[j] = k[j];
          xv[j] = x[j];
        }
      }
      uint64_t C[Q][D];
#pragma unroll
      for (int q = 0; q < Q; ++q)
#pragma unroll
        for (int d = 0; d < D; ++d) {
          bad |= (kv[q * D + d] >= kEntryLimit) | (xv[q * D + d] >= kEntryLimit);
          C[q][d] = kv[q * D + d] + xv[q * D + d];  // a1: aggregate cost
        }
      uint64_t best = kNone;
      uint32_t bi = 0;
#pragma unroll
      for (int m = 0; m < N; ++m) {
        uint64_t L[D];
#pragma unroll
        for (int d = 0; d < D; ++d) L[d] = 0;
        int rest = m;
#pragma unroll
        for (int q = Q - 1; q >= 0; --q) {
          const int dq = rest % D;
          rest /= D;
          L[dq] += C[q][dq];
        }
        uint64_t ms = L[0];
#pragma unroll
        for (int d = 1; d < D; ++d) ms = max(ms, L[d]);
        if (ms < best) {
          best = ms;
          bi = (uint32_t)m;
        }
      }
      a.index[e] = bi;
      a.makespan[e] = best;
      if (a.mapping) {
        uint32_t rest = bi;
#pragma unroll
        for (int q = Q - 1; q >= 0; --q) {
          a.mapping[e * Q + q] = (uint8_t)(rest % D);
          rest /= D;
        }
      }
    }
    __syncthreads();  // stage s is consumed: refill it with this CTA's tile kSmallStages ahead
    const uint64_t tn = t + (uint64_t)kSmallStages * gridDim.x;
    if (tid == 0 && tn < ntiles && tile_tma(tn)) issue(tn, s);
    s = (s + 1 == kSmallStages) ? 0 : s + 1;
  }
  if (__any_sync(0xffffffffu, bad) && (tid & 31) == 0) raise_flag(a.flags, kFlagRange);
}

namespace {
// A few epochs (cfg1: one scheduling decision, 81 mappings): one WARP per epoch instead of
// one thread, so the D^Q mappings are scored 32 at a time (lane l: l, l + 32, ...) and the
// decision's latency is a few dependent steps plus five shuffles, not a serial loop of 81.
// Lexicographic (makespan, index) through the packed key ms << 7 | m (D^Q <= 81 < 128;
// ms < 2^51 for Q <= 4 entries below 2^48 each).
template <int Q, int D>
__global__ void __launch_bounds__(32) search_tiny_kernel(SmallArgs a) {
  constexpr int QD = Q * D;
  constexpr int N = Pow<Q, D>::N;
  static_assert(N <= 128 && Q <= 4, "packed key: 7 index bits, ms < 2^51");
  const uint64_t e = blockIdx.x;
  const int lane = threadIdx.x;
  __shared__ uint64_t C[QD];
  bool bad = false;
  if (lane < QD) {
    const uint64_t k = a.K[e * QD + lane], x = a.X[e * QD + lane];
    bad = (k >= kEntryLimit) | (x >= kEntryLimit);
    C[lane] = k + x;  // a1: aggregate cost
  }
  __syncwarp();
  if (__any_sync(0xffffffffu, bad)) {
    if (lane == 0) raise_flag(a.flags, kFlagRange);
    return;
  }
  uint64_t key = ~0ull;
  for (int m = lane; m < N; m += 32) {  // increasing m: the first strict minimum is kept
    uint64_t L[D];
#pragma unroll
    for (int d = 0; d < D; ++d) L[d] = 0;
    int rest = m;
#pragma unroll
    for (int q = Q - 1; q >= 0; --q) {
      const int dq = rest % D;
      rest /= D;
#pragma unroll
      for (int d = 0; d < D; ++d) L[d] += (dq == d) ? C[q * D + d] : 0;
    }
    uint64_t ms = L[0];
#pragma unroll
    for (int d = 1; d < D; ++d) ms = max(ms, L[d]);
    key = min(key, (ms << 7) | (uint64_t)m);
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) key = min(key, __shfl_xor_sync(0xffffffffu, key, off));
  const uint32_t idx = (uint32_t)(key & 127);
  if (lane == 0) {
    a.index[e] = idx;
    a.makespan[e] = key >> 7;
  }
  if (a.mapping && lane < Q) {  // digits of the index, queue 0 most significant
    uint32_t rest = idx;
    for (int q = Q - 1; q > lane; --q) rest /= D;
    a.mapping[e * Q + lane] = (uint8_t)(rest % D);
  }
}

constexpr uint64_t kTinyMaxEpochs = 64;  // up to this many epochs: a warp per epoch

template <int Q, int D>
cudaError_t launch_small_t(const SmallArgs& a, int num_sms, cudaStream_t st, int* grid_out,
                           int* threads_out) {
  if (a.E <= kTinyMaxEpochs) {
    search_tiny_kernel<Q, D><<<(unsigned)a.E, 32, 0, st>>>(a);
    *grid_out = (int)a.E;
    *threads_out = 32;
    return cudaGetLastError();
  }
  // tile = one epoch per thread; tiny batches (cfg1: one epoch) get a single warp.
  // Defaults from the cfg3 sweep (scripts/archive/sweep_small.sh, profiles/r01/sweep_small.txt):
  // 128-epoch tiles, 2 stages, 4 CTAs per SM (8 tiles in flight per SM) was fastest;
  // MCL_SMALL_{THREADS,STAGES,CTAS_PER_SM} override them for tuning.
  static const int kThreads = env_int("MCL_SMALL_THREADS", 128, 32, 256);
  static const int kStages = env_int("MCL_SMALL_STAGES", 2, 1, kMaxSmallStages);
  static const int kCtasCap = env_int("MCL_SMALL_CTAS_PER_SM", 4, 1, 32);
  const int threads = a.E >= (uint64_t)kThreads ? kThreads : (int)((a.E + 31) / 32 * 32);
  const size_t smem = (size_t)kStages * 2 * threads * Q * D * 8;
  auto k = search_small_kernel<Q, D>;
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  static std::atomic<int> occ_full[64];  // CTAs per SM at full tiles, per device (0 = unknown)
  int dev = 0;
  cudaGetDevice(&dev);
  int per_sm = 1;
  if (threads == kThreads) {
    per_sm = occ_full[dev & 63].load(std::memory_order_relaxed);
    if (per_sm == 0) {
      err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, threads, smem);
      if (err != cudaSuccess) return err;
      if (per_sm < 1) per_sm = 1;
      occ_full[dev & 63].store(per_sm, std::memory_order_relaxed);
    }
    if (per_sm > kCtasCap) per_sm = kCtasCap;
  }
  const uint64_t ntiles = (a.E + threads - 1) / threads;
  uint64_t grid = (uint64_t)num_sms * per_sm;
  if (grid > ntiles) grid = ntiles;
  const int use_tma = ((reinterpret_cast<uintptr_t>(a.K) | reinterpret_cast<uintptr_t>(a.X)) & 15) == 0;
  k<<<(unsigned)grid, threads, smem, st>>>(a, use_tma, kStages);
  *grid_out = (int)grid;
  *threads_out = threads;
  return cudaGetLastError();
}
}  // namespace

bool small_supported(uint32_t Q, uint32_t D) {
  return (Q == 2 && (D >= 2 && D <= 4)) || (Q == 3 && (D >= 2 && D <= 4)) ||
         (Q == 4 && (D == 2 || D == 3));
}

cudaError_t launch_small(const SmallArgs& a, int num_sms, cudaStream_t st, int* grid_out,
                         int* threads_out) {
  const uint32_t key = a.Q * 100 + a.D;
  switch (key) {
    case 202: return launch_small_t<2, 2>(a, num_sms, st, grid_out, threads_out);
    case 203: return launch_small_t<2, 3>(a, num_sms, st, grid_out, threads_out);
    case 204: return launch_small_t<2, 4>(a, num_sms, st, grid_out, threads_out);
    case 302: return launch_small_t<3, 2>(a, num_sms, st, grid_out, threads_out);
    case 303: return launch_small_t<3, 3>(a, num_sms, st, grid_out, threads_out);
    case 304: return launch_small_t<3, 4>(a, num_sms, st, grid_out, threads_out);
    case 402: return launch_small_t<4, 2>(a, num_sms, st, grid_out, threads_out);
    case 403: return launch_small_t<4, 3>(a, num_sms, st, grid_out, threads_out);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mcl
