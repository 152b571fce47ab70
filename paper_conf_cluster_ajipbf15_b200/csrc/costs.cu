// costs.cu -- cost-table construction: the mapper's inputs K and X built on
// the GPU from the kernel profiles, the epochs' kernel lists and the device profiles.
//
//  K[e][q][d] = sum over the kernel invocations enqueued to queue q in epoch e of
//               profile[kernel][d]   (kernel profiler; "the aggregate
//               performance vector of the epoch", L1154-1158)
//  X[e][q][d] = 0                                     data on d, or a copy cached on d
//                                                     (data caching, L1309-1321)
//             = t_h2d(d, bytes)                       data in host memory
//             = t_d2h(src, bytes) + t_h2d(d, bytes)   data on another device: "a D2H-H2D
//                                                     double operation via the host", L1293-1301
//  with no H2D/D2H leg for a device flagged host_shared, and t(curve, b) = ceil(b / bw(b))
//  ns, bw linearly interpolated between the sampled sizes and clamped at the ends ("simple
//  interpolation techniques", L905-907). The curves are per (host socket, device) ("all the
//  CPU socket-device combinations", L897-901; nonuniform host-device distances, L1349-1361):
//  a queue's host memory is on socket host_socket[e][q], whose curves both legs use (DESIGN.md
//  R19). fp64 with explicitly rounded operations (no FMA contraction), so the result is
//  bit-identical to a plain IEEE evaluation. Range (R10): a profile entry >= 2^48, or a kernel
//  sum reaching 2^48, raises kFlagRange (lists of >= 2^16 invocations check every addition,
//  shorter ones cannot wrap a u64 and are checked once).
//
// Tiles of 256 (epoch, queue) pairs per CTA, one thread per pair: it sums its invocations'
// profile rows and interpolates the curves (sizes and bandwidths in shared memory; one
// segment search serves every device because the sample sizes are shared). Memory-bound:
// reads ids / offsets / bytes / source / cached once, writes 2 x D x 8 bytes per pair.
#include "common.cuh"
#include "kernels.h"

namespace mcl {

namespace {

__device__ __forceinline__ double lerp_bw(const double* __restrict__ bw, uint32_t i, double f,
                                          bool clamp_lo, bool clamp_hi, uint32_t M) {
  if (clamp_lo) return bw[0];
  if (clamp_hi) return bw[M - 1];
  return __dadd_rn(bw[i], __dmul_rn(f, __dsub_rn(bw[i + 1], bw[i])));
}

__device__ __forceinline__ uint64_t transfer_ns(uint64_t bytes, double bw) {
  if (bytes == 0) return 0;
  return (uint64_t)ceil(__ddiv_rn(__ull2double_rn(bytes), bw));
}

}  // namespace

constexpr int kCostTile = 256;        // (epoch, queue) pairs per CTA tile (= blockDim.x)
constexpr int kProfCapBytes = 32768;  // profile table staged when it fits
// Row stride of the staged profile table in u64 words: odd, so the rows of a warp's random
// kernel ids spread over 16 bank pairs instead of 32 / (2 D) (a stride of 4 words put every
// row on one of 4 bank groups: 8-way conflicts on each 64-bit row load).
template <int D>
__host__ __device__ constexpr int prof_stride() { return D % 2 ? D : D + 1; }

// Memory pipeline: a persistent CTA walks its tiles with each thread's next pair (CSR
// offsets, bytes, source, cached mask) loaded into registers while the current pair is
// computed, so the loads of tile t + 1 are in flight during tile t -- no block barriers in
// the tile loop. Invocation ids are read straight from global memory through L1 (the lists
// of a warp's pairs are adjacent, so a warp's reads of one list position share lines);
// profile rows and bandwidth curves come from shared memory. Outputs go through a per-warp
// shared buffer so every store instruction writes 32 consecutive words.
template <int D>
__global__ void __launch_bounds__(kCostTile) build_costs_kernel(CostArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t M = a.M;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // layout: outK[kCostTile*D] u64 | outX[kCostTile*D] u64 | sizes[M] u64 | h2d[S][D][M] f64 |
  //         d2h[S][D][M] f64 | prof[num_kernels][D] u64 (if it fits)
  const uint32_t S = a.S;
  uint64_t* s_outK = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* s_outX = s_outK + (size_t)kCostTile * D;
  uint64_t* s_sizes = s_outX + (size_t)kCostTile * D;
  double* s_h2d = reinterpret_cast<double*>(s_sizes + M);
  double* s_d2h = s_h2d + (size_t)S * D * M;
  uint64_t* s_prof = reinterpret_cast<uint64_t*>(s_d2h + (size_t)S * D * M);
  constexpr int PS = prof_stride<D>();
  const bool prof_in_smem = (size_t)a.num_kernels * PS * 8 <= (size_t)kProfCapBytes;
  for (uint32_t t = tid; t < M; t += blockDim.x) s_sizes[t] = a.sizes[t];
  for (uint32_t t = tid; t < S * D * M; t += blockDim.x) {
    s_h2d[t] = a.h2d[t];
    s_d2h[t] = a.d2h[t];
  }
  // Profiles that all fit 32 bits (kernel times below 4.3 s) are staged as u32 rows of odd
  // stride PS32: one 4-byte shared load per (id, device) instead of an 8-byte one, half the
  // shared-memory wavefronts of the sum; the sums stay 64-bit.
  constexpr int PS32 = D % 2 ? D : D + 1;
  uint32_t* s_prof32 = reinterpret_cast<uint32_t*>(s_prof);
  bool fits32 = false;
  __shared__ uint32_t s_pmax;  // largest entry of a 32-bit table
  if (tid == 0) s_pmax = 0;
  if (prof_in_smem) {
    bool big = false;
    uint32_t pm = 0;
    for (uint32_t t = tid; t < a.num_kernels * D; t += blockDim.x) {
      big |= (a.profile[t] >> 32) != 0;
      pm = max(pm, (uint32_t)a.profile[t]);
    }
    pm = __reduce_max_sync(0xffffffffu, pm);
    if (lane == 0 && pm) atomicMax(&s_pmax, pm);
    fits32 = !__syncthreads_or(big);
    if (fits32) {
      for (uint32_t t = tid; t < a.num_kernels * D; t += blockDim.x)
        s_prof32[(t / D) * PS32 + t % D] = (uint32_t)a.profile[t];
    }
    else
      for (uint32_t t = tid; t < a.num_kernels * D; t += blockDim.x) s_prof[(t / D) * PS + t % D] = a.profile[t];
  }
  __syncthreads();
  const uint64_t* prof = prof_in_smem ? s_prof : a.profile;
  uint32_t status = 0;
  if (blockIdx.x == 0) {  // model validation (once)
    if (tid == 0) {
      for (uint32_t i = 0; i + 1 < M; ++i)
        if (!(s_sizes[i] < s_sizes[i + 1])) status |= kFlagBadModel;
      for (uint32_t i = 0; i < S * D * M; ++i)
        if (!(s_h2d[i] > 0.0) || !(s_d2h[i] > 0.0)) status |= kFlagBadModel;
      if (a.offsets[a.EQ] != a.nnz) status |= kFlagBadModel;
    }
    for (uint32_t t = tid; t < a.num_kernels * D; t += blockDim.x)
      if (a.profile[t] >= kEntryLimit) status |= kFlagRange;  // every entry, invoked or not
  }

  // this thread's pair of a tile, loaded one tile ahead
  uint64_t n_j0 = 0, n_j1 = 0, n_bytes = 0;
  int32_t n_src = 0;
  uint32_t n_cached = 0, n_sock = 0;
  auto fetch = [&](uint64_t tile) {
    const uint64_t eq = tile * kCostTile + tid;
    if (eq < a.EQ) {
      n_j0 = a.offsets[eq];
      n_j1 = a.offsets[eq + 1];
      n_bytes = a.bytes[eq];
      n_src = a.source[eq];
      n_cached = a.cached ? (uint32_t)a.cached[eq] : 0u;
      n_sock = a.host_socket ? (uint32_t)a.host_socket[eq] : 0u;
    }
  };
  const uint64_t ntiles = (a.EQ + kCostTile - 1) / kCostTile;
  if (blockIdx.x < ntiles) fetch(blockIdx.x);
  for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const uint64_t j0 = n_j0, j1 = n_j1, bytes = n_bytes;
    const int32_t src = n_src;
    const uint32_t cached = n_cached, sock = n_sock;
    if (tile + gridDim.x < ntiles) fetch(tile + gridDim.x);
    const uint64_t eq = tile * kCostTile + tid;
    if (eq < a.EQ) {
      // ---- kernel part: sum of the invoked kernels' profile rows ----
      uint64_t k[D];
#pragma unroll
      for (int d = 0; d < D; ++d) k[d] = 0;
      bool ok = j0 <= j1 && j1 <= a.nnz;
      if (ok && j1 - j0 >= 65536u) {
        // a long list could wrap a u64 sum of entries < 2^48: check every addition, stop at
        // 2^48 (the range error), as the definition's running sum does
        for (uint64_t j = j0; j < j1 && ok; ++j) {
          const uint32_t kid = __ldg(a.ids + j);
          if (kid >= a.num_kernels) {
            ok = false;
            break;
          }
          bool over = false;
#pragma unroll
          for (int d = 0; d < D; ++d) {
            if (k[d] < kEntryLimit) k[d] += a.profile[(uint64_t)kid * D + d];
            over |= k[d] >= kEntryLimit;
          }
          if (over) {
            status |= kFlagRange;
            break;
          }
        }
      } else if (ok && fits32 && a.num_kernels != 0 && j1 - j0 < (1ull << 31) &&
                 (uint64_t)(j1 - j0) * s_pmax < (1ull << 32)) {
        // the list's sums fit 32 bits (n x largest entry < 2^32): 32-bit accumulators and
        // 32-bit positions; ids are clamped into the table and checked once after the loop
        // (an id >= num_kernels flags the pair, as the early exit below does)
        const uint32_t n = (uint32_t)(j1 - j0), kcap = a.num_kernels - 1;
        const uint32_t* ids = a.ids + j0;
        uint32_t k32[D];
#pragma unroll
        for (int d = 0; d < D; ++d) k32[d] = 0;
        uint32_t idmax = 0;
        auto add_id = [&](uint32_t kid) {
          idmax = max(idmax, kid);
          const uint32_t* row = s_prof32 + (size_t)min(kid, kcap) * PS32;
#pragma unroll
          for (int d = 0; d < D; ++d) k32[d] += row[d];
        };
#pragma unroll 4
        for (uint32_t t = 0; t < n; ++t) add_id(__ldg(ids + t));
        ok = idmax <= kcap;
#pragma unroll
        for (int d = 0; d < D; ++d) k[d] = ok ? k32[d] : 0;
      } else if (ok && fits32) {
#pragma unroll 4
        for (uint64_t j = j0; j < j1; ++j) {
          const uint32_t kid = __ldg(a.ids + j);
          if (kid >= a.num_kernels) {
            ok = false;
            break;
          }
          const uint32_t* row = s_prof32 + (size_t)kid * PS32;
#pragma unroll
          for (int d = 0; d < D; ++d) k[d] += row[d];
        }
      } else if (ok) {
#pragma unroll 4
        for (uint64_t j = j0; j < j1; ++j) {
          const uint32_t kid = __ldg(a.ids + j);
          if (kid >= a.num_kernels) {
            ok = false;
            break;
          }
          const uint64_t* row = prof + (uint64_t)kid * (prof_in_smem ? PS : D);
#pragma unroll
          for (int d = 0; d < D; ++d) k[d] += row[d];
        }
      }
      // ---- transfer part ----
      ok = ok && src >= -1 && src < (int32_t)D && sock < S;
      if (!ok) status |= kFlagBadModel;
      const double* h2d_s = s_h2d + (size_t)(ok ? sock : 0) * D * M;
      const double* d2h_s = s_d2h + (size_t)(ok ? sock : 0) * D * M;
      const bool clo = bytes <= s_sizes[0], chi = bytes >= s_sizes[M - 1];
      uint32_t seg = 0;
      double f = 0.0;
      if (ok && !clo && !chi) {
        // binary search for sizes[seg] <= bytes < sizes[seg + 1]
        uint32_t l = 0, r = M - 1;  // sizes[l] <= bytes < sizes[r]
        while (r - l > 1) {
          const uint32_t mid = (l + r) >> 1;
          if (s_sizes[mid] <= bytes) l = mid; else r = mid;
        }
        seg = l;
        f = __ddiv_rn(__ull2double_rn(bytes - s_sizes[seg]),
                      __ull2double_rn(s_sizes[seg + 1] - s_sizes[seg]));
      }
      uint64_t down = 0;
      if (ok && src >= 0 && !((a.host_shared >> src) & 1u))
        down = transfer_ns(bytes, lerp_bw(d2h_s + (size_t)src * M, seg, f, clo, chi, M));
#pragma unroll
      for (int d = 0; d < D; ++d) {
        uint64_t x = 0;
        if (ok && !(src == d || ((cached >> d) & 1u))) {
          const uint64_t up = ((a.host_shared >> d) & 1u)
                                  ? 0
                                  : transfer_ns(bytes, lerp_bw(h2d_s + (size_t)d * M, seg, f, clo, chi, M));
          x = down + up;
        }
        if (k[d] >= kEntryLimit || x >= kEntryLimit) status |= kFlagRange;
        s_outK[(size_t)tid * D + d] = k[d];
        s_outX[(size_t)tid * D + d] = x;
      }
    }
    // ---- coalesced stores: the warp's 32 pairs are 32 * D consecutive words ----
    __syncwarp();
    const uint64_t base = tile * kCostTile + (uint64_t)warp * 32;
    if (base < a.EQ) {
      const uint32_t np = (uint32_t)((a.EQ - base < 32) ? a.EQ - base : 32);
      const uint64_t* sk = s_outK + (size_t)warp * 32 * D;
      const uint64_t* sx = s_outX + (size_t)warp * 32 * D;
      for (uint32_t w = lane; w < np * D; w += 32) {
        a.K[base * D + w] = sk[w];
        a.X[base * D + w] = sx[w];
      }
    }
    __syncwarp();  // the buffer is rewritten by the next tile
  }
  if (__any_sync(0xffffffffu, status != 0)) {
    const uint32_t all = __reduce_or_sync(0xffffffffu, status);
    if ((tid & 31) == 0) raise_flag(a.flags, all);
  }
}

namespace {
template <int D>
cudaError_t launch_build_costs_t(const CostArgs& a, int num_sms, cudaStream_t st) {
  size_t smem = 2 * (size_t)kCostTile * D * 8 + (size_t)a.M * 8 + 2 * (size_t)a.S * D * a.M * 8;
  if ((size_t)a.num_kernels * prof_stride<D>() * 8 <= (size_t)kProfCapBytes)
    smem += (size_t)a.num_kernels * prof_stride<D>() * 8;
  auto k = build_costs_kernel<D>;
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  // resident CTAs per SM at this shared-memory size (persistent grid); the last query is
  // cached per device, keyed by the size (it depends on sockets, samples and the profile)
  static std::atomic<uint64_t> occ[64];
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t hit = occ[dev & 63].load(std::memory_order_relaxed);
  int per_sm = (hit >> 8) == (uint64_t)smem + 1 ? (int)(hit & 0xff) : 0;
  if (per_sm == 0) {
    err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kCostTile, smem);
    if (err != cudaSuccess) return err;
    per_sm = per_sm < 1 ? 1 : (per_sm > 255 ? 255 : per_sm);
    occ[dev & 63].store((((uint64_t)smem + 1) << 8) | (uint64_t)per_sm, std::memory_order_relaxed);
  }
  uint64_t grid = (a.EQ + kCostTile - 1) / kCostTile;
  const uint64_t cap = (uint64_t)num_sms * per_sm;
  if (grid > cap) grid = cap;
  if (grid == 0) grid = 1;
  k<<<(unsigned)grid, kCostTile, smem, st>>>(a);
  return cudaGetLastError();
}
}  // namespace

cudaError_t launch_build_costs(const CostArgs& a, int num_sms, cudaStream_t st) {
  switch (a.D) {
#define MCL_COST_CASE(DD) \
  case DD: return launch_build_costs_t<DD>(a, num_sms, st);
    MCL_COST_CASE(1) MCL_COST_CASE(2) MCL_COST_CASE(3) MCL_COST_CASE(4)
    MCL_COST_CASE(5) MCL_COST_CASE(6) MCL_COST_CASE(7) MCL_COST_CASE(8)
    MCL_COST_CASE(9) MCL_COST_CASE(10) MCL_COST_CASE(11) MCL_COST_CASE(12)
    MCL_COST_CASE(13) MCL_COST_CASE(14) MCL_COST_CASE(15) MCL_COST_CASE(16)
#undef MCL_COST_CASE
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mcl
