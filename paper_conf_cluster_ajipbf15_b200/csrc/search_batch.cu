// search_batch.cu -- batched exhaustive search with compile-time (Q, D) (
// cfg2: 8 queues x 4 devices x 10^4 epochs), in two forms:
//   * search_pool_kernel (below; the default for device-resident batches of >= 2 epochs per
//     SM): one 16-warp CTA per SM whose warps claim sub-epoch parts of the SM's epochs;
//   * search_batch_kernel (first): one WARP per epoch -- pinned host inputs read in place
//     (its per-warp next-epoch prefetch hides PCIe latency) and smaller batches.
//
// Same scoring core as search_blocked.cu (blocked_core.cuh: the D^4 leaves of a
// super-block folded into one running minimum, one integer max per mapping; PAPER.md
// L1048-1052 loads / makespan, L2106-2118 C = K + X), but the per-epoch work around it is
// cut to what a warp-sized epoch needs, because with 4^8 = 65,536 mappings per epoch that
// setup is a fifth of the instructions in the CTA-per-epoch kernel:
//   * persistent warps stride over the epochs; the next epoch's K and X are loaded into
//     registers while the current one is searched (no load latency in the prologue);
//   * warp-synchronous setup, no outer tables: the chunk digits (queues 0..Q-6) come from
//     compile-time divisions of the chunk index, the one-hot prefix vectors from selects
//     on the cost table;
//   * lane l walks chunks l, l + 32, ... (D^2 blocks each, the super-block path), keeping
//     the first strict minimum of its own increasing sequence; the warp takes the
//     lexicographic minimum of (makespan, super-block index), and re-scans only that
//     super-block (lane x * D + i takes the leaves (x, i, *, *); one ballot) for the
//     lowest leaf index.
// Wave quantisation: whole waves of epochs (one per warp) run first; the epochs of the last,
// partial wave go one per CTA, its warps splitting the epoch's super-blocks and merging
// their keys through shared memory (no global atomics or fences). A batch below one wave
// runs one warp per epoch.
// Mapping index m = ((chunk * D + y) * D + x) * D^3 + leaf, queue 0 most significant
// (R6): chunk = digits of queues 0..Q-6, y = queue Q-5, x = queue Q-4, leaf =
// queues Q-3..Q-1.
#include <algorithm>
#include <type_traits>

#include "blocked_core.cuh"

namespace mcl {

#ifdef MCL_TRACE
// Measurement build only (-DMCL_TRACE): per warp and unit (<= 8 units), %globaltimer at the
// unit's start, after its tables, after the walk and after the finish, plus the SM id.
__device__ unsigned long long g_mcl_btrace[4096 * 4][8][4];
__device__ unsigned int g_mcl_bsm[4096 * 4];
__device__ unsigned long long g_mcl_ptrace[1024][4];  // SM-pooled kernel, per CTA
__device__ __forceinline__ unsigned long long btrace_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define MCL_BTRACE(unit, slot)                                                         \
  do {                                                                                 \
    if (lane == 0 && gw < 4096 * 4 && (unit) < 8) g_mcl_btrace[gw][unit][slot] = btrace_ns(); \
  } while (0)
#else
#define MCL_BTRACE(unit, slot) \
  do {                         \
  } while (0)
#endif

namespace {

template <int B, int E>
struct IPow {
  static constexpr uint64_t v = (uint64_t)B * IPow<B, E - 1>::v;
};
template <int B>
struct IPow<B, 0> {
  static constexpr uint64_t v = 1;
};

constexpr int kBatchWarps = 4;  // warps per CTA (each its own epochs)

}  // namespace

template <int Q, int D>
__global__ void __launch_bounds__(32 * kBatchWarps, 4) search_batch_kernel(BatchArgs a) {
  using T = uint32_t;
  constexpr int QD = Q * D;
  constexpr uint32_t kChunks = (uint32_t)IPow<D, Q - 5>::v;  // chunks of D^2 blocks per epoch
  constexpr uint32_t kSb = kChunks * D;                      // super-blocks per epoch
  static_assert(QD <= 64, "two cost entries per lane");
  static_assert(Q >= 6, "chunks need queues 0..Q-6");
  static_assert(D * D <= 32, "finish: one lane per (x, i) pair of a super-block");
  __shared__ __align__(16) uint64_t sC64[kBatchWarps][QD];
  __shared__ __align__(16) T sC[kBatchWarps][QD];
  __shared__ __align__(16) T sIn[kBatchWarps][8 * D];
  // one-hot rows of the outer queues 0..Q-5: sV[q][x][d] = C[q][x] if d == x else 0, so a
  // digit's prefix contribution is one vector load instead of D compare-and-selects
  constexpr int kVN = (Q - 4) * D * D;
  __shared__ __align__(16) T sV[kBatchWarps][kVN];
  __shared__ uint64_t s_key[2][kBatchWarps];  // split epochs: each warp's key (double-buffered)
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  uint64_t* C64 = sC64[wib];
  T* Cs = sC[wib];
  T* in = sIn[wib];
  const uint32_t one = a.one;
  const uint64_t nwarps = (uint64_t)gridDim.x * kBatchWarps;
  const uint64_t gw = (uint64_t)blockIdx.x * kBatchWarps + wib;
  // This warp's units: whole epochs gw, gw + nwarps, ... below e_full, then the CTA's
  // split epochs e_full + blockIdx.x, + gridDim.x, ... There are split epochs only when
  // e_full is a multiple of nwarps, so the CTA's warps then share one unit sequence (the
  // barrier of a split epoch is reached by all of them).
  const uint64_t n_whole = a.e_full > gw ? (a.e_full - gw + nwarps - 1) / nwarps : 0;
  auto unit_epoch = [&](uint64_t i) -> uint64_t {
    return i < n_whole ? gw + i * nwarps : a.e_full + blockIdx.x + (i - n_whole) * gridDim.x;
  };

  // prefetch of an epoch's costs: entries lane and lane + 32
  uint64_t k0 = 0, x0 = 0, k1 = 0, x1 = 0;
  auto prefetch = [&](uint64_t ep) {
    const uint64_t* Ke = a.K + ep * QD;
    const uint64_t* Xe = a.X + ep * QD;
    if (lane < QD) { k0 = Ke[lane]; x0 = Xe[lane]; }
    if (lane + 32 < QD) { k1 = Ke[lane + 32]; x1 = Xe[lane + 32]; }
  };
  if (unit_epoch(0) < a.E) prefetch(unit_epoch(0));

  const T* c4 = in + 7 * D;
  // prefix loads of chunk c: one-hot costs of queues 0..Q-6 on their digits' devices
  T* V = sV[wib];
  auto chunk_base = [&](uint32_t c, T (&b)[D]) {
#pragma unroll
    for (int d = 0; d < D; ++d) b[d] = 0;
#pragma unroll
    for (int q = Q - 6; q >= 0; --q) {
      const uint32_t dq = c % D;
      c /= D;
      const T* row = V + (q * D + dq) * D;
#pragma unroll
      for (int d = 0; d < D; ++d) b[d] = add_f(b[d], row[d], one);
    }
  };
  // prefix loads of super-block sb = chunk * D + y
  auto sb_base = [&](uint32_t sb, T (&b)[D]) {
    T b2[D];
    chunk_base(sb / D, b2);
    const T* row = V + ((Q - 5) * D + sb % D) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) b[d] = add_f(b2[d], row[d], one);
  };
  // a warp's lexicographic minimum of (makespan << 32 | super-block)
  // (two 32-bit warp reductions, REDUX: the minimum makespan, then the lowest super-block
  // among the lanes holding it -- the same key as a 64-bit shuffle tree, in fewer steps)
  auto warp_key = [&](T best, uint32_t best_sb) {
    const uint32_t g = __reduce_min_sync(0xffffffffu, (uint32_t)best);
    const uint32_t sb = __reduce_min_sync(0xffffffffu, (uint32_t)best == g ? best_sb : 0xffffffffu);
    return ((uint64_t)g << 32) | sb;
  };
  // The lowest leaf inside the winning super-block, then the outputs (a5, a7). Leaf
  // (x, i, j, k) of the super-block has offset ((x * D + i) * D + j) * D + k: lane
  // x * D + i takes the D^2 leaves (j, k) in order with loads P' = base + C[Q-4][x] on x +
  // A[i] on i and forms max(M', P'_j + B_j, P'_k + C_k) (j, k static; one sum when j == k;
  // M' = max P' covers the untouched devices); one ballot finds the lowest lane holding the
  // target, so the rescan is one pass instead of up to D rounds of block re-scans.
  auto finish = [&](uint64_t e, uint64_t key) {
    const T target = (T)(key >> 32);
    const uint32_t sb = (uint32_t)key;
    T base[D];
    sb_base(sb, base);
    const uint32_t x = (uint32_t)lane / D, i = (uint32_t)lane % D;
    T PB[D], PC[D];
    T Mp = 0;
#pragma unroll
    for (int d = 0; d < D; ++d) {
      T v = base[d];
      if (x == (uint32_t)d) v += c4[d];
      if (i == (uint32_t)d) v += in[0 * D + d];
      Mp = max2(Mp, v);
      PB[d] = v + in[1 * D + d];
      PC[d] = v + in[2 * D + d];
    }
    uint32_t hit = 0xffffffffu;
#pragma unroll
    for (int j = D - 1; j >= 0; --j)
#pragma unroll
      for (int k = D - 1; k >= 0; --k) {
        const T v = (j == k) ? max2(Mp, PB[j] + in[2 * D + j]) : max3(Mp, PB[j], PC[k]);
        if (v == target) hit = (uint32_t)(j * D + k);
      }
    const uint32_t m = __ballot_sync(0xffffffffu, lane < D * D && hit != 0xffffffffu);
    uint64_t idx = kNone;
    if (m) {
      const int src = __ffs(m) - 1;
      const uint32_t t = __shfl_sync(0xffffffffu, hit, src);
      idx = (uint64_t)sb * (uint64_t)(D * D * D * D) + (uint64_t)src * (D * D) + t;
    }
    if (lane == 0) {
      a.index[e] = idx;
      a.makespan[e] = (uint64_t)target;
    }
    if (a.mapping && lane < Q) {  // digits of the index, queue 0 most significant
      uint64_t rest = idx;
      for (int q = Q - 1; q > lane; --q) rest /= D;
      a.mapping[e * Q + lane] = (uint8_t)(rest % D);
    }
  };

  int par = 0;
#ifdef MCL_TRACE
  if (lane == 0 && gw < 4096 * 4) {
    unsigned int smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    g_mcl_bsm[gw] = smid;
    for (int u = 0; u < 8; ++u) g_mcl_btrace[gw][u][0] = 0;
  }
#endif
  for (uint64_t i = 0;; ++i) {
    const uint64_t e = unit_epoch(i);
    if (e >= a.E) break;
    const bool whole = i < n_whole;
    MCL_BTRACE(i, 0);
    // ---- a1: C = K + X, range check, bound UB = sum_q max_d C (decides 32-bit loads) ----
    bool bad = false;
    if (lane < QD) {
      bad |= (k0 >= kEntryLimit) | (x0 >= kEntryLimit);
      C64[lane] = k0 + x0;
    }
    if (lane + 32 < QD) {
      bad |= (k1 >= kEntryLimit) | (x1 >= kEntryLimit);
      C64[lane + 32] = k1 + x1;
    }
    const uint64_t en = unit_epoch(i + 1);
    if (en < a.E) prefetch(en);  // travels while this epoch is searched
    __syncwarp();
    uint64_t row = 0;
    if (lane < Q) {
#pragma unroll
      for (int d = 0; d < D; ++d) row = max(row, C64[lane * D + d]);
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) row += __shfl_xor_sync(0xffffffffu, row, off);
    // 32-bit loads need UB < 2^32 - 1: every makespan then stays below the all-ones
    // "no candidate" value the lanes start from (UB = 2^32 - 1 takes the 64-bit rerun)
    const bool anybad = __any_sync(0xffffffffu, bad);
    const bool skip = anybad || row >= 0xffffffffull;
    if (skip && lane == 0 && (whole || wib == 0)) raise_flag(a.flags, anybad ? kFlagRange : kFlagNeedU64);

    uint64_t key = ~0ull;
    if (!skip) {
      // ---- tables: composed costs (u32) and the inner queues' sums ----
      if (lane < QD) Cs[lane] = (T)C64[lane];
      if (lane + 32 < QD) Cs[lane + 32] = (T)C64[lane + 32];
      if (lane < D) {
        const T A = (T)C64[(Q - 3) * D + lane], B = (T)C64[(Q - 2) * D + lane], Cc = (T)C64[(Q - 1) * D + lane];
        in[0 * D + lane] = A;
        in[1 * D + lane] = B;
        in[2 * D + lane] = Cc;
        in[3 * D + lane] = A + B;
        in[4 * D + lane] = A + Cc;
        in[5 * D + lane] = B + Cc;
        in[6 * D + lane] = A + B + Cc;
        in[7 * D + lane] = (T)C64[(Q - 4) * D + lane];
      }
      for (int t = lane; t < kVN; t += 32) {
        const int q = t / (D * D), x = (t / D) % D, d = t % D;
        V[t] = (d == x) ? (T)C64[q * D + x] : T(0);
      }
      __syncwarp();
      MCL_BTRACE(i, 1);
      // ---- a2-a5: each lane walks its share in increasing order, first strict minimum ----
      T best = ~T(0);
      uint32_t best_sb = 0xffffffffu;
      if (whole) {  // lane l: chunks l, l + 32, ... (D super-blocks each)
        for (uint32_t c = lane; c < kChunks; c += 32) {
          T base2[D];
          chunk_base(c, base2);
          for (int y = 0; y < D; ++y) {
            const T* row = V + ((Q - 5) * D + y) * D;
            T base[D];
#pragma unroll
            for (int d = 0; d < D; ++d) base[d] = add_f(base2[d], row[d], one);
            const T gs = superblock_eval<T, D>(base, in, c4, one);
            if (gs < best) {
              best = gs;
              best_sb = c * D + (uint32_t)y;
            }
          }
        }
      } else {  // warp wib of the CTA: super-blocks [s0, s1), lane l: s0 + l, s0 + l + 32, ...
        const uint32_t s0 = kSb * (uint32_t)wib / kBatchWarps, s1 = kSb * (uint32_t)(wib + 1) / kBatchWarps;
        for (uint32_t sb = s0 + lane; sb < s1; sb += 32) {
          T base[D];
          sb_base(sb, base);
          const T gs = superblock_eval<T, D>(base, in, c4, one);
          if (gs < best) {
            best = gs;
            best_sb = sb;
          }
        }
      }
      key = warp_key(best, best_sb);
      MCL_BTRACE(i, 2);
    }
    if (whole) {
      if (!skip) finish(e, key);
      MCL_BTRACE(i, 3);
      continue;
    }
    // a split epoch: the CTA's warps merge their keys in shared memory; warp 0 finishes
    if (lane == 0) s_key[par][wib] = key;
    __syncthreads();
    if (wib == 0 && !skip) {
      uint64_t k = s_key[par][0];
#pragma unroll
      for (int w = 1; w < kBatchWarps; ++w) k = min(k, s_key[par][w]);
      finish(e, k);
    }
    par ^= 1;  // the next split epoch writes the other buffer (one barrier in between)
    MCL_BTRACE(i, 3);
  }
}

// ---------------------------------------------------------------------------------------
// SM-pooled form (default for batches): one CTA of 16 warps per SM shares its epochs at
// sub-epoch granularity. Why: with a warp per epoch the SMSP's oldest-first warp scheduler
// starves the younger warps, so the four warps of an SMSP finish their (equal) work at
// ~35 / 47 / 60 / 74 us and the last ~15 us run one warp per SMSP at ~64-81 % ALU
// (SS7, profiles/r02/batch_study.md). Here a favoured warp simply claims more
// work: the CTA's epochs (blockIdx.x, + gridDim.x, ...: a static, monotone ordinal -> epoch
// map, no global atomics) are cut into PARTS of 32 * kSbLane super-blocks, and the 16 warps
// claim (ordinal, part) pairs from one shared counter. Each epoch's tables (inner sums and
// one-hot outer rows, built once per epoch by the warp that claimed part 0 of the epoch
// kPoolAhead ordinals earlier) live in a ring of kPoolSlots shared-memory slots; a part's
// warp key (makespan << 32 | super-block) is merged by a shared 64-bit atomicMin, and the
// warp completing an epoch's last part re-scans the winning super-block, writes the
// outputs and frees the slot. The lexicographic minimum over parts is the epoch's lowest
// super-block holding the minimum (every lane walks its super-blocks in increasing order
// with strict <), so the result is the same as the warp-per-epoch kernel's.
#ifndef MCL_BATCH_POOL
#define MCL_BATCH_POOL 1  // 0: warp-per-epoch kernel for every batch (A/B builds)
#endif
namespace {
constexpr int kPoolWarps = 16;
#ifndef MCL_POOL_SLOTS
#define MCL_POOL_SLOTS 32
#endif
constexpr int kPoolSlots = MCL_POOL_SLOTS;  // ring of per-epoch table slots
#ifndef MCL_POOL_AHEAD
#define MCL_POOL_AHEAD 12
#endif
constexpr int kPoolAhead = MCL_POOL_AHEAD;  // epochs prepared ahead of the claims
#ifndef MCL_POOL_ZERO_COPY
#define MCL_POOL_ZERO_COPY 0  // 1: the pooled form also for pinned host inputs read in place
#endif
#ifndef MCL_POOL_SBL
#define MCL_POOL_SBL 2u  // super-blocks per lane in one part (when it divides D)
#endif
// CTA-scope acquire/release fence for the shared-memory hand-offs between warps (lighter
// than __threadfence_block's sequentially consistent MEMBAR.SC.CTA)
__device__ __forceinline__ void fence_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }
#ifndef MCL_POOL_ACQREL
#define MCL_POOL_ACQREL 1  // release stores / acquire loads / acq_rel atomics instead of fences
#endif
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void st_release_cta(int* p, int v) {
  asm volatile("st.release.cta.shared.b32 [%0], %1;" ::"r"(smem_addr(p)), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_acquire_cta(const int* p) {
  int v;
  asm volatile("ld.acquire.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(smem_addr(p)) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t atom_add_acq_rel_cta(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.cta.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(smem_addr(p)), "r"(v) : "memory");
  return old;
}
#ifndef MCL_POOL_TAIL
#define MCL_POOL_TAIL 1  // last ordinals of each CTA cut into single-super-block parts
#endif
constexpr int kPoolTail = MCL_POOL_TAIL;
#ifndef MCL_POOL_MIN_PER_SM
#define MCL_POOL_MIN_PER_SM 2
#endif
constexpr int kPoolMinPerSm = MCL_POOL_MIN_PER_SM;  // smaller batches: warp per epoch
}  // namespace

template <int Q, int D>
__global__ void __launch_bounds__(32 * kPoolWarps, 1) search_pool_kernel(BatchArgs a) {
  using T = uint32_t;
  constexpr int QD = Q * D;
  constexpr uint32_t kChunks = (uint32_t)IPow<D, Q - 5>::v;
  constexpr uint32_t kSb = kChunks * D;                       // super-blocks per epoch
  constexpr uint32_t kSbLane = (D % MCL_POOL_SBL == 0) ? MCL_POOL_SBL : 1u;  // super-blocks per lane and part
  constexpr uint32_t kPartSb = 32u * kSbLane;
  constexpr uint32_t kParts = (kSb + kPartSb - 1) / kPartSb;  // parts per epoch
  constexpr uint32_t kParts1 = (kSb + 31u) / 32u;             // the same, one super-block per lane
  constexpr int kVN = (Q - 4) * D * D;
  static_assert(QD <= 64, "two cost entries per lane");
  static_assert(D * D <= 32, "finish: one lane per (x, i) pair of a super-block");
  static_assert(D % kSbLane == 0, "a lane's super-blocks share one chunk");
  struct Slot {
    uint64_t C64[QD];
    T in[8 * D];
    T V[kVN];
  };
  __shared__ __align__(16) Slot s_slot[kPoolSlots];
  __shared__ unsigned long long s_key[kPoolSlots];
  __shared__ uint32_t s_cnt[kPoolSlots];
  __shared__ int s_ready[kPoolSlots];  // ordinal whose tables the slot holds
  __shared__ int s_done[kPoolSlots];   // last ordinal finished in the slot
  __shared__ uint32_t s_skip[kPoolSlots];
  __shared__ uint32_t s_next;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t one = a.one;
  const uint64_t G = gridDim.x, b = blockIdx.x;
#ifdef MCL_TRACE
  // per CTA: entry, first part claimed with its tables ready, first failed claim, last exit
  __shared__ uint32_t s_exit, s_first;
  if (threadIdx.x == 0 && b < 1024) {
    s_exit = 0;
    s_first = 0;
    g_mcl_ptrace[b][0] = btrace_ns();
  }
#endif
  const uint32_t n_ord = a.E > b ? (uint32_t)((a.E - b + G - 1) / G) : 0u;
  const uint32_t n_big = n_ord > (uint32_t)kPoolTail ? n_ord - (uint32_t)kPoolTail : 0u;
  const uint32_t t_big = n_big * kParts;
  const uint32_t total = t_big + (n_ord - n_big) * kParts1;
  if (threadIdx.x < kPoolSlots) {
    s_key[threadIdx.x] = ~0ull;
    s_cnt[threadIdx.x] = 0;
    s_ready[threadIdx.x] = -1;
    s_done[threadIdx.x] = (int)threadIdx.x - kPoolSlots;
  }
  if (threadIdx.x == 0) s_next = 0;
  __syncthreads();

  // ---- a1 + tables of ordinal n, by one whole warp ----
  auto prepare = [&](uint32_t n) {
    const int si = (int)(n % kPoolSlots);
    Slot& S = s_slot[si];
    const uint64_t e = b + (uint64_t)n * G;
    const uint64_t* Ke = a.K + e * QD;
    const uint64_t* Xe = a.X + e * QD;
    uint64_t k0 = 0, x0 = 0, k1 = 0, x1 = 0;
    if (lane < QD) { k0 = Ke[lane]; x0 = Xe[lane]; }
    if (lane + 32 < QD) { k1 = Ke[lane + 32]; x1 = Xe[lane + 32]; }
    if (lane == 0) {  // the slot's previous occupant (ordinal n - kPoolSlots) is finished
#if MCL_POOL_ACQREL
      while (ld_acquire_cta(&s_done[si]) != (int)n - kPoolSlots) __nanosleep(64);
#else
      while (*(volatile int*)&s_done[si] != (int)n - kPoolSlots) __nanosleep(64);
#endif
    }
    __syncwarp();
    bool bad = false;
    if (lane < QD) {
      bad |= (k0 >= kEntryLimit) | (x0 >= kEntryLimit);
      S.C64[lane] = k0 + x0;
    }
    if (lane + 32 < QD) {
      bad |= (k1 >= kEntryLimit) | (x1 >= kEntryLimit);
      S.C64[lane + 32] = k1 + x1;
    }
    __syncwarp();
    uint64_t row = 0;
    if (lane < Q) {
#pragma unroll
      for (int d = 0; d < D; ++d) row = max(row, S.C64[lane * D + d]);
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) row += __shfl_xor_sync(0xffffffffu, row, off);
    const bool anybad = __any_sync(0xffffffffu, bad);
    const bool skip = anybad || row >= 0xffffffffull;  // 32-bit loads need UB < 2^32 - 1
    if (skip && lane == 0) raise_flag(a.flags, anybad ? kFlagRange : kFlagNeedU64);
    if (!skip) {
      if (lane < D) {
        const T A = (T)S.C64[(Q - 3) * D + lane], B = (T)S.C64[(Q - 2) * D + lane],
                Cc = (T)S.C64[(Q - 1) * D + lane];
        S.in[0 * D + lane] = A;
        S.in[1 * D + lane] = B;
        S.in[2 * D + lane] = Cc;
        S.in[3 * D + lane] = A + B;
        S.in[4 * D + lane] = A + Cc;
        S.in[5 * D + lane] = B + Cc;
        S.in[6 * D + lane] = A + B + Cc;
        S.in[7 * D + lane] = (T)S.C64[(Q - 4) * D + lane];
      }
      for (int t = lane; t < kVN; t += 32) {
        const int q = t / (D * D), x = (t / D) % D, d = t % D;
        S.V[t] = (d == x) ? (T)S.C64[q * D + x] : T(0);
      }
    }
    if (lane == 0) s_skip[si] = skip ? 1u : 0u;
    __syncwarp();
#if MCL_POOL_ACQREL
    if (lane == 0) st_release_cta(&s_ready[si], (int)n);
#else
    fence_cta();
    if (lane == 0) *(volatile int*)&s_ready[si] = (int)n;
#endif
  };

  auto chunk_base = [&](const T* V, uint32_t c, T (&bv)[D]) {
#pragma unroll
    for (int d = 0; d < D; ++d) bv[d] = 0;
#pragma unroll
    for (int q = Q - 6; q >= 0; --q) {
      const uint32_t dq = c % D;
      c /= D;
      const T* r = V + (q * D + dq) * D;
#pragma unroll
      for (int d = 0; d < D; ++d) bv[d] = add_f(bv[d], r[d], one);
    }
  };

  // the lowest leaf of the winning super-block and the outputs (as search_batch_kernel)
  auto finish = [&](const Slot& S, uint64_t e, uint64_t key) {
    const T* in = S.in;
    const T* c4 = in + 7 * D;
    const T target = (T)(key >> 32);
    const uint32_t sb = (uint32_t)key;
    T base[D];
    {
      T b2[D];
      chunk_base(S.V, sb / D, b2);
      const T* r = S.V + ((Q - 5) * D + sb % D) * D;
#pragma unroll
      for (int d = 0; d < D; ++d) base[d] = add_f(b2[d], r[d], one);
    }
    const uint32_t x = (uint32_t)lane / D, i = (uint32_t)lane % D;
    T PB[D], PC[D];
    T Mp = 0;
#pragma unroll
    for (int d = 0; d < D; ++d) {
      T v = base[d];
      if (x == (uint32_t)d) v += c4[d];
      if (i == (uint32_t)d) v += in[0 * D + d];
      Mp = max2(Mp, v);
      PB[d] = v + in[1 * D + d];
      PC[d] = v + in[2 * D + d];
    }
    uint32_t hit = 0xffffffffu;
#pragma unroll
    for (int j = D - 1; j >= 0; --j)
#pragma unroll
      for (int k = D - 1; k >= 0; --k) {
        const T v = (j == k) ? max2(Mp, PB[j] + in[2 * D + j]) : max3(Mp, PB[j], PC[k]);
        if (v == target) hit = (uint32_t)(j * D + k);
      }
    const uint32_t m = __ballot_sync(0xffffffffu, lane < D * D && hit != 0xffffffffu);
    uint64_t idx = kNone;
    if (m) {
      const int src = __ffs(m) - 1;
      const uint32_t t = __shfl_sync(0xffffffffu, hit, src);
      idx = (uint64_t)sb * (uint64_t)(D * D * D * D) + (uint64_t)src * (D * D) + t;
    }
    if (lane == 0) {
      a.index[e] = idx;
      a.makespan[e] = (uint64_t)target;
    }
    if (a.mapping && lane < Q) {  // D^Q < 2^32 for every pooled shape: 32-bit digits,
      uint32_t rest = (uint32_t)idx;  // predicated constant divisions (no divergent loop)
#pragma unroll
      for (int q = Q - 1; q > 0; --q)
        if (q > lane) rest /= D;
      a.mapping[e * Q + lane] = (uint8_t)(rest % D);
    }
  };

  if (wib < kPoolAhead && (uint32_t)wib < n_ord) prepare((uint32_t)wib);
  for (;;) {
    uint32_t t = 0;
    if (lane == 0) t = atomicAdd(&s_next, 1u);
    t = __shfl_sync(0xffffffffu, t, 0);
    if (t >= total) {
#ifdef MCL_TRACE
      if (lane == 0 && b < 1024) {
        if (t == total) g_mcl_ptrace[b][2] = btrace_ns();
        if (atomicAdd(&s_exit, 1u) == kPoolWarps - 1) g_mcl_ptrace[b][3] = btrace_ns();
      }
#endif
      break;
    }
    // (ordinal, part, super-blocks per lane): the last kPoolTail ordinals in single-super-
    // block parts, so the warps' last parts end closer together
    uint32_t n, p, sbl, parts;
    if (t < t_big) {
      n = t / kParts;
      p = t % kParts;
      sbl = kSbLane;
      parts = kParts;
    } else {
      n = n_big + (t - t_big) / kParts1;
      p = (t - t_big) % kParts1;
      sbl = 1;
      parts = kParts1;
    }
    const int si = (int)(n % kPoolSlots);
    if (p == 0 && n + kPoolAhead < n_ord) prepare(n + kPoolAhead);
#if MCL_POOL_ACQREL
    if (lane == 0) {
      while (ld_acquire_cta(&s_ready[si]) != (int)n) __nanosleep(32);
    }
    __syncwarp();
#else
    if (lane == 0) {
      while (*(volatile int*)&s_ready[si] != (int)n) __nanosleep(32);
    }
    __syncwarp();
    fence_cta();
#endif
#ifdef MCL_TRACE
    if (lane == 0 && b < 1024 && atomicExch(&s_first, 1u) == 0) g_mcl_ptrace[b][1] = btrace_ns();
#endif
    const bool skip = *(volatile uint32_t*)&s_skip[si] != 0;
    const Slot& S = s_slot[si];
    if (!skip) {
      const T* in = S.in;
      const T* c4 = in + 7 * D;
      T best = ~T(0);
      uint32_t best_sb = 0xffffffffu;
      const uint32_t sb0 = (p * 32u + (uint32_t)lane) * sbl;
      // a lane's super-blocks sb0 .. sb0 + n - 1 (n divides D: one chunk), compile-time n
      auto walk = [&](auto nsb) {
        constexpr uint32_t n_sb = decltype(nsb)::value;
        T base2[D];
        chunk_base(S.V, sb0 / D, base2);
        // at most two super-block bodies in the code (four thrash the instruction cache)
#pragma unroll 2
        for (uint32_t j = 0; j < n_sb; ++j) {
          const uint32_t sb = sb0 + j;
          const T* r = S.V + ((Q - 5) * D + sb % D) * D;
          T base[D];
#pragma unroll
          for (int d = 0; d < D; ++d) base[d] = add_f(base2[d], r[d], one);
          const T gs = superblock_eval<T, D>(base, in, c4, one);
          if (gs < best) {
            best = gs;
            best_sb = sb;
          }
        }
      };
      if (sb0 < kSb) {
        if (kSbLane > 1 && sbl == kSbLane) walk(std::integral_constant<uint32_t, kSbLane>{});
        else walk(std::integral_constant<uint32_t, 1u>{});
      }
      const uint32_t g = __reduce_min_sync(0xffffffffu, (uint32_t)best);
      const uint32_t bsb = __reduce_min_sync(0xffffffffu, (uint32_t)best == g ? best_sb : 0xffffffffu);
      if (lane == 0) atomicMin(&s_key[si], ((unsigned long long)g << 32) | bsb);
    }
    uint32_t c = 0;
#if MCL_POOL_ACQREL
    if (lane == 0) c = atom_add_acq_rel_cta(&s_cnt[si], 1u);  // releases this part's key
    c = __shfl_sync(0xffffffffu, c, 0);
    if (c == parts - 1) {  // this warp completed the epoch (lane 0 acquired every part's key)
      __syncwarp();
#else
    if (lane == 0) {
      fence_cta();
      c = atomicAdd(&s_cnt[si], 1u);
    }
    c = __shfl_sync(0xffffffffu, c, 0);
    if (c == parts - 1) {  // this warp completed the epoch
      fence_cta();
#endif
      const uint64_t key = *(volatile unsigned long long*)&s_key[si];
      if (!skip) finish(S, b + (uint64_t)n * G, key);
      __syncwarp();
      if (lane == 0) {
        s_key[si] = ~0ull;
        s_cnt[si] = 0;
#if MCL_POOL_ACQREL
        st_release_cta(&s_done[si], (int)n);
#else
        fence_cta();
        *(volatile int*)&s_done[si] = (int)n;
#endif
      }
    }
  }
}

#ifdef MCL_TRACE
}  // namespace mcl
extern "C" int mcl_btrace_read(unsigned long long* out, unsigned int* sm, int nwarps) {
  cudaError_t e = cudaMemcpyFromSymbol(out, mcl::g_mcl_btrace, (size_t)nwarps * 8 * 4 * 8);
  if (e == cudaSuccess) e = cudaMemcpyFromSymbol(sm, mcl::g_mcl_bsm, (size_t)nwarps * 4);
  return (int)e;
}
extern "C" int mcl_ptrace_read(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, mcl::g_mcl_ptrace, sizeof(mcl::g_mcl_ptrace));
}
namespace mcl {
#endif

namespace {
template <int Q, int D>
cudaError_t launch_batch_t(const BatchArgs& a, int num_sms, cudaStream_t st, int* grid_out, bool* pooled) {
  *pooled = false;
  // MCL_POOL_MIN_PER_SM (environment, tests / sanitizer runs): the smallest batch, in
  // epochs per SM, that takes the pooled form (a huge value keeps the warp-per-epoch form)
  static const int min_per_sm = env_int("MCL_POOL_MIN_PER_SM", kPoolMinPerSm, 1, 1 << 30);
  if (MCL_BATCH_POOL && (MCL_POOL_ZERO_COPY || !a.host_inputs) && a.E >= (uint64_t)num_sms * min_per_sm) {
    // one 16-warp CTA per SM, epochs blockIdx.x + n * gridDim.x
    search_pool_kernel<Q, D><<<(unsigned)num_sms, 32 * kPoolWarps, 0, st>>>(a);
    *grid_out = num_sms;
    *pooled = true;
    return cudaGetLastError();
  }
  auto k = search_batch_kernel<Q, D>;
  static std::atomic<int> occ[64];
  int dev = 0;
  cudaGetDevice(&dev);
  int per_sm = occ[dev & 63].load(std::memory_order_relaxed);
  if (per_sm == 0) {
    cudaError_t err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, 32 * kBatchWarps, 0);
    if (err != cudaSuccess) return err;
    if (per_sm < 1) per_sm = 1;
    occ[dev & 63].store(per_sm, std::memory_order_relaxed);
  }
  // one resident wave of warps; whole waves of epochs take one warp each, the epochs of
  // the last partial wave one CTA each (its warps split the super-blocks)
  // (measured, scripts/archive/batch_waves.py: splitting pays after at least one whole wave; a
  // batch below one wave runs one warp per epoch)
  const uint64_t ctas = (uint64_t)num_sms * per_sm;
  BatchArgs b = a;
  b.e_full = a.E / (ctas * kBatchWarps) * (ctas * kBatchWarps);
  uint64_t grid = ctas;
  if (b.e_full == 0) {
    b.e_full = a.E;
    grid = std::min<uint64_t>(ctas, (a.E + kBatchWarps - 1) / kBatchWarps);
  }
  k<<<(unsigned)grid, 32 * kBatchWarps, 0, st>>>(b);
  *grid_out = (int)grid;
  return cudaGetLastError();
}
}  // namespace

// Shapes with a warp-per-epoch instantiation: >= 32 chunks per epoch (every lane busy),
// at most 2^26 mappings per epoch (a warp-sized epoch), QD <= 64.
bool batch_supported(uint32_t Q, uint32_t D) {
  switch (Q * 100 + D) {
    case 803: case 903: case 1003: case 1103:  // D = 3: 3^(Q-5) >= 27 ... lanes mostly busy
    case 804: case 904: case 1004: case 1104:
    case 805: case 905:
      return true;
    default:
      return false;
  }
}

cudaError_t launch_batch(const BatchArgs& a, int num_sms, cudaStream_t st, int* grid_out, bool* pooled) {
  switch (a.Q * 100 + a.D) {
    case 803: return launch_batch_t<8, 3>(a, num_sms, st, grid_out, pooled);
    case 903: return launch_batch_t<9, 3>(a, num_sms, st, grid_out, pooled);
    case 1003: return launch_batch_t<10, 3>(a, num_sms, st, grid_out, pooled);
    case 1103: return launch_batch_t<11, 3>(a, num_sms, st, grid_out, pooled);
    case 804: return launch_batch_t<8, 4>(a, num_sms, st, grid_out, pooled);
    case 904: return launch_batch_t<9, 4>(a, num_sms, st, grid_out, pooled);
    case 1004: return launch_batch_t<10, 4>(a, num_sms, st, grid_out, pooled);
    case 1104: return launch_batch_t<11, 4>(a, num_sms, st, grid_out, pooled);
    case 805: return launch_batch_t<8, 5>(a, num_sms, st, grid_out, pooled);
    case 905: return launch_batch_t<9, 5>(a, num_sms, st, grid_out, pooled);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mcl
