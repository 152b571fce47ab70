// search_mixed.cu -- constrained exhaustive search over the FEASIBLE mappings only: a true
// mixed-radix enumeration (reading R11).
//
// The paper's runtime maps only the SCHED_AUTO queues of the ready pool; a SCHED_OFF queue
// "will be statically mapped to the chosen device" and a
// queue may be restricted to the devices its data fits. Here every queue q has an eligible
// device set S_q (mask bits below D; 0 = all D devices), r_q = |S_q| digits:
//   * r_q == 1 (pinned): the queue is removed from the enumeration -- its cost is added to
//     its device's base load and its digit is a constant of the mapping index (radix 1);
//   * the remaining queues keep their order; the OUTER ones (all but the last three, the
//     inner block queues) enumerate only their eligible devices: digit t of queue q selects
//     device S_q[t] (ascending), through one-hot load vectors V[p][t] in shared memory;
//   * the three inner queues (and, for D <= 5, the super-block queue before them) keep the
//     register-blocked leaf table of blocked_core.cuh over all D devices with their
//     ineligible entries at INF (> every feasible makespan), so masked inner queues cost
//     D / r_q extra leaves each (SS7).
// Because every S_q is ascending and the pinned digits are constants, the map from the
// reduced mixed-radix index to the full index m = sum_q d_q D^(Q-1-q) is strictly
// increasing: the first strict minimum in reduced order is the LOWEST FULL INDEX among the
// feasible optima (the tie rule of mcl_map_queues_constrained), and contiguous reduced ranges
// (threads, CTAs, ranks) keep the lexicographic (makespan, full index) merges exact.
//
// Work per epoch: nb = prod over the outer reduced queues of r_q blocks of D^3 leaves, i.e.
// D^3 (or D^4) x the feasible outer space: time proportional to the feasible mappings
// (times the inner INF factor), not to D^Q. Every feasible mapping's makespan is still
// formed explicitly in a register (one max per leaf).
#include "blocked_core.cuh"
#include "peer.cuh"

namespace mcl {

namespace {

// Reduced problem of one epoch (shared memory, built by one warp).
struct MixedTab {
  uint32_t Qr;               // reduced queues incl. virtual padding (>= 3)
  uint32_t O;                // outer reduced queues = Qr - 3
  uint64_t nb;               // blocks of D^3 leaves = prod_{p < O} radix[p]
  uint64_t pin_idx;          // sum over pinned queues of d_q * D^(Q-1-q)
  uint8_t radix[kMaxQueues];
  uint32_t rmul[kMaxQueues];             // ceil(2^20 / radix[p]): division of indices < 2^16
  uint8_t dev[kMaxQueues][kMaxDevices];  // digit -> device of reduced queue p
  uint64_t w[kMaxQueues];                // D^(Q-1-q) of reduced queue p (0 = virtual)
  int8_t orig[kMaxQueues];               // original queue of reduced queue p (-1 = virtual)
};

// q = x / radix[p] and x - q * radix[p]. Block indices of the warp kernel (I = 32 bits) are
// below 2^16 and radices at most 16, so q = (x * ceil(2^20 / r)) >> 20 exactly (the error
// x * (m r - 2^20) / (r 2^20) < 2^16 * 16 / (r 2^20) <= 1 / r); 64-bit indices divide.
template <typename I>
__device__ __forceinline__ I div_radix(I x, const MixedTab& mt, int p, uint32_t* rem) {
  const uint32_t r = mt.radix[p];
  I q;
  if constexpr (sizeof(I) == 4) q = (I)(((uint64_t)x * mt.rmul[p]) >> 20);
  else q = x / r;
  *rem = (uint32_t)(x - q * r);
  return q;
}

// Decode reduced block `blk` into its outer digits (radix[p], p = O-1 fastest) and return
// the prefix load vector base0 + sum_p V[p][t_p]; optionally the full-index part of the
// outer digits.
template <typename T, int D, typename I = uint64_t>
__device__ __forceinline__ void mixed_prefix(T (&P)[D], I blk, const MixedTab& mt,
                                             const T* __restrict__ V, const T* __restrict__ B0,
                                             uint32_t one, uint64_t* full_part = nullptr) {
#pragma unroll
  for (int d = 0; d < D; ++d) P[d] = B0[d];
  uint64_t f = 0;
  for (int p = (int)mt.O - 1; p >= 0; --p) {
    uint32_t t;
    blk = div_radix<I>(blk, mt, p, &t);
    f += (uint64_t)mt.dev[p][t] * mt.w[p];
    const T* v = V + ((size_t)p * D + t) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) P[d] = add_f(P[d], v[d], one);
  }
  if (full_part) *full_part = f;
}

// Full mapping index of leaf `leaf` (inner digits i, j, k over D) of reduced block `blk`.
template <int D, typename I = uint64_t>
__device__ __forceinline__ uint64_t mixed_full_index(I blk, uint32_t leaf, const MixedTab& mt) {
  uint64_t f = mt.pin_idx;
  for (int p = (int)mt.O - 1; p >= 0; --p) {
    uint32_t t;
    blk = div_radix<I>(blk, mt, p, &t);
    f += (uint64_t)mt.dev[p][t] * mt.w[p];
  }
  const uint32_t i = leaf / (D * D), j = (leaf / D) % D, k = leaf % D;
  return f + i * mt.w[mt.O] + j * mt.w[mt.O + 1] + k * mt.w[mt.O + 2];
}

// The reduced problem of one epoch, built by ONE WARP (lane q handles queue q, Q <= 32):
// pinned queues (one eligible device) add their cost to that device's base load s_base and
// a constant digit to pin_idx; the others keep their order with their eligible devices
// ascending; virtual zero-cost queues pad the problem to >= 3 reduced queues; for D <= 5
// the super-block queue keeps all D devices (INF entries). *s_ubr = a bound of every leaf
// the kernels form (decides 32- vs 64-bit loads).
template <typename T, int D>
__device__ __forceinline__ void mixed_build(MixedTab& mt, const uint64_t* C64, uint32_t Q,
                                            const uint16_t* elig_e, uint64_t* s_base, uint64_t inf,
                                            uint64_t* s_ubr) {
  const uint32_t lane = threadIdx.x & 31, full = (1u << D) - 1u;
  const bool act = lane < Q;
  uint32_t m = full;
  if (act && elig_e && elig_e[lane] != 0) m = (uint32_t)elig_e[lane] & full;
  const bool pinned = act && __popc(m) == 1;
  uint64_t wq = 1;  // D^(Q-1-q) <= 2^48 (D^Q <= 2^48 is checked on the host)
  for (uint32_t t = lane + 1; t < Q; ++t) wq *= D;
  const uint32_t freeb = __ballot_sync(0xffffffffu, act && !pinned);
  const uint32_t n = __popc(freeb);
  uint64_t pin = 0, rm = 0;
  if (pinned) {  // its cost joins the device's base load; its digit is a constant (radix 1)
    const uint32_t d = __ffs(m) - 1;
    atomicAdd(reinterpret_cast<unsigned long long*>(&s_base[d]), (unsigned long long)C64[lane * D + d]);
    pin = (uint64_t)d * wq;
  } else if (act) {  // reduced queue p keeps its order among the unpinned queues
    const uint32_t p = __popc(freeb & ((1u << lane) - 1u));
    mt.orig[p] = (int8_t)lane;
    mt.w[p] = wq;
    uint32_t r = 0;
    for (uint32_t d = 0; d < D; ++d) {
      if ((m >> d) & 1u) mt.dev[p][r++] = (uint8_t)d;
      rm = max(rm, C64[lane * D + d]);  // INF entries included: a bound of every leaf
    }
    mt.radix[p] = (uint8_t)r;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    pin += __shfl_xor_sync(0xffffffffu, pin, off);
    rm += __shfl_xor_sync(0xffffffffu, rm, off);
  }
  __syncwarp();
  if (lane == 0) {
    uint32_t nn = n;
    for (; nn < 3; ++nn) {  // virtual inner queues: zero cost on device 0 only, weight 0
      mt.orig[nn] = -1;
      mt.w[nn] = 0;
      mt.radix[nn] = 1;
      mt.dev[nn][0] = 0;
      rm += inf;
    }
    mt.Qr = nn;
    mt.O = nn - 3;
    // the super-block queue (outer position O-1, D <= 5) keeps all D devices (INF entries)
    if (sizeof(T) == 4 && D <= kSuperMaxD && mt.O >= 1) {
      mt.radix[mt.O - 1] = D;
      for (uint32_t d = 0; d < D; ++d) mt.dev[mt.O - 1][d] = (uint8_t)d;
    }
    uint64_t nb = 1;
    for (uint32_t p = 0; p < mt.O; ++p) {
      nb *= mt.radix[p];
      mt.rmul[p] = ((1u << 20) + mt.radix[p] - 1u) / mt.radix[p];
    }
    mt.nb = nb;
    mt.pin_idx = pin;
    // bound of every leaf the kernel forms: max base' + sum of the reduced rows' maxima
    uint64_t bm = 0;
    for (uint32_t d = 0; d < D; ++d) bm = max(bm, s_base[d]);
    *s_ubr = bm + rm;
  }
  __syncwarp();
}

// Inner sums of the last three reduced queues (in[8][D]), the one-hot outer vectors
// V[O][D][D] and the base loads (base0[D]) of the reduced problem, threads t0, t0 + stride, ...
template <typename T, int D>
__device__ __forceinline__ void mixed_tables(const MixedTab& mt, const uint64_t* C64, uint64_t inf,
                                             const uint64_t* s_base, T* in, T* V, T* base0, int t0,
                                             int stride) {
  const uint32_t O = mt.O;
  auto cost = [&](uint32_t p, uint32_t d) -> uint64_t {  // reduced queue p on device d
    const int q = mt.orig[p];
    return q >= 0 ? C64[q * D + d] : (d == 0 ? 0ull : inf);
  };
  for (int t = t0; t < D; t += stride) {
    const uint64_t A = cost(O, t), B = cost(O + 1, t), Cc = cost(O + 2, t);
    in[0 * D + t] = (T)A;
    in[1 * D + t] = (T)B;
    in[2 * D + t] = (T)Cc;
    in[3 * D + t] = (T)(A + B);
    in[4 * D + t] = (T)(A + Cc);
    in[5 * D + t] = (T)(B + Cc);
    in[6 * D + t] = (T)(A + B + Cc);
    in[7 * D + t] = (O >= 1) ? (T)cost(O - 1, t) : (T)0;
    base0[t] = (T)s_base[t];
  }
  for (int t = t0; t < (int)O * D * D; t += stride) {
    const int p = t / (D * D), x = (t / D) % D, d = t % D;
    T v = 0;
    if (x < mt.radix[p]) {
      const uint32_t dv = mt.dev[p][x];
      if ((uint32_t)d == dv) v = (T)cost(p, dv);
    }
    V[t] = v;
  }
}

// Score reduced blocks [b0, b0 + nleft) for one thread (mixed-radix odometer over the outer
// digits, digit O-1 fastest; for D <= 5 it has radix D and whole runs of D blocks are scored
// as one super-block), keeping the first strict minimum.
// I: the block index type (32 bits when the caller knows nb < 2^32: the digit decode then
// divides in 32 bits).
template <typename T, int D, typename I = uint64_t>
__device__ __forceinline__ void walk_mixed(const MixedTab& mt, const T* __restrict__ in,
                                           const T* __restrict__ V, const T* __restrict__ B0,
                                           uint8_t* dig, int nthr, int tid, uint32_t one, I b0,
                                           I nleft, T& best, I& best_blk,
                                           uint32_t& best_span) {
  constexpr bool kSuper = (sizeof(T) == 4 && D <= kSuperMaxD);
  if (!nleft) return;
  const int O = (int)mt.O;
  if (O == 0) {  // one block: the prefix is the base loads
    T P[D];
    load_vec<T, D>(P, B0);
    const T g = block_eval<T, D>(P, in, one);
    if (g < best) {
      best = g;
      best_blk = 0;
      best_span = 1;
    }
    return;
  }
  const T* Vx = V + (size_t)(O - 1) * D * D;
  const T* c4 = in + 7 * D;
  const uint32_t rx = mt.radix[O - 1];
  uint32_t x;
  I hi = div_radix<I>(b0, mt, O - 1, &x);
  T base[D];
  load_vec<T, D>(base, B0);
  for (int p = O - 2; p >= 0; --p) {
    uint32_t t;
    hi = div_radix<I>(hi, mt, p, &t);
    dig[p * nthr + tid] = (uint8_t)t;
    const T* v = V + ((size_t)p * D + t) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) base[d] = add_f(base[d], v[d], one);
  }
  I blk = b0;
  while (true) {
    if (kSuper && x == 0 && nleft >= (I)D) {  // rx == D on the super-block path
      const T gs = superblock_eval<T, D>(base, in, c4, one);
      if (gs < best) {
        best = gs;
        best_blk = blk;
        best_span = D;
      }
      x = D;
      nleft -= D;
      blk += D;
    }
    for (; x < rx && nleft; ++x, --nleft, ++blk) {
      T P[D], vx[D];
      load_vec<T, D>(vx, Vx + x * D);
#pragma unroll
      for (int d = 0; d < D; ++d) P[d] = add_f(base[d], vx[d], one);
      const T g = block_eval<T, D>(P, in, one);
      if (g < best) {
        best = g;
        best_blk = blk;
        best_span = 1;
      }
    }
    if (!nleft) break;
    x = 0;
    for (int p = O - 2; p >= 0; --p) {  // odometer over the mixed-radix outer digits
      const uint32_t old = dig[p * nthr + tid];
      const uint32_t nw = (old + 1 == mt.radix[p]) ? 0u : old + 1;
      dig[p * nthr + tid] = (uint8_t)nw;
      const T* vo = V + ((size_t)p * D + old) * D;
      const T* vn = V + ((size_t)p * D + nw) * D;
#pragma unroll
      for (int d = 0; d < D; ++d) base[d] = base[d] - vo[d] + vn[d];
      if (nw != 0) break;
    }
  }
}

// Lowest full index in reduced blocks [bb, bb + span) whose makespan equals `target`
// (known to exist); all 32 lanes call it.
template <typename T, int D, typename I = uint64_t>
__device__ __forceinline__ uint64_t mixed_span_first_warp(I bb, uint32_t span, const MixedTab& mt,
                                                          const T* __restrict__ V, const T* __restrict__ B0,
                                                          const T* __restrict__ in, T target, uint32_t one) {
  for (uint32_t t = 0; t < span; ++t) {
    T P[D];
    mixed_prefix<T, D, I>(P, (I)(bb + t), mt, V, B0, one);
    const uint32_t leaf = block_first_warp<T, D>(P, in, target);
    if (leaf != 0xffffffffu) return mixed_full_index<D, I>((I)(bb + t), leaf, mt);
  }
  return kNone;
}

}  // namespace

template <typename T, int D>
__global__ void __launch_bounds__(256, (sizeof(T) == 4 && D <= 5) ? 2 : 1) search_mixed_kernel(BlockedArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q;
  const int nthr = blockDim.x, tid = threadIdx.x;
  // layout: C64[Q*D] u64 | in[8*D] T | V[(Q-3)*D*D] T | red[32] Cand | dig[(Q-4)*nthr] u8
  // (the same sizes as the blocked kernel: the reduced problem has at most Q queues)
  uint64_t* C64 = reinterpret_cast<uint64_t*>(smem_raw);
  T* in = reinterpret_cast<T*>(C64 + Q * D);
  T* V = in + 8 * D;
  Cand* red = reinterpret_cast<Cand*>(reinterpret_cast<unsigned char*>(smem_raw) + a.off_red);
  uint8_t* dig = reinterpret_cast<uint8_t*>(smem_raw) + a.off_dig;
  __shared__ MixedTab mt;
  __shared__ uint32_t s_status;
  __shared__ uint64_t s_ub, s_feas;
  __shared__ uint64_t s_ubr;  // bound of the reduced problem (decides u32 vs u64)
  __shared__ uint64_t s_base[D];
  __shared__ __align__(16) T base0[D];
  __shared__ uint64_t s_gmin;
  __shared__ uint32_t s_winner;
  __shared__ Cand s_cand;
  __shared__ bool s_last;
  const uint32_t one = a.one;

  const uint64_t ncta = a.e_full + (a.E - a.e_full) * a.tail_cpe;
  bool abandoned = false;
  for (uint64_t cta = blockIdx.x; cta < ncta; cta += gridDim.x) {
    uint64_t e;
    uint32_t part, parts;
    if (cta < a.e_full) {
      e = cta;
      part = 0;
      parts = 1;
    } else {
      const uint64_t t = cta - a.e_full;
      e = a.e_full + t / a.tail_cpe;
      part = (uint32_t)(t % a.tail_cpe);
      parts = a.tail_cpe;
    }
    // ---- a1: C = K + X, range check; base loads, INF masking, the bound UB ----
    __syncthreads();
    if (tid == 0) { s_status = 0; s_ub = 0; }
    __syncthreads();
    const uint64_t* Ke = a.K + e * Q * D;
    const uint64_t* Xe = a.X + e * Q * D;
    for (uint32_t t = tid; t < Q * D; t += nthr) {
      const uint64_t k = Ke[t], x = Xe[t];
      if (k >= kEntryLimit || x >= kEntryLimit) s_status = kFlagRange;
      C64[t] = k + x;
    }
    __syncthreads();
    const uint16_t* elig_e = a.elig ? a.elig + e * Q : nullptr;
    if (tid < 32) {
      const uint64_t ub = epoch_prologue(C64, Q, D, a.base ? a.base + e * D : nullptr, elig_e, s_base,
                                         &s_status, &s_feas);
      if (tid == 0) s_ub = ub;
    }
    __syncthreads();
    if (s_status) {
      if (tid == 0 && part == 0) raise_flag(a.flags, s_status);
      abandoned = true;
      continue;
    }
    // INF of an ineligible entry: above every feasible makespan (epoch_prologue put
    // UB_f + 1 into the masked entries; without masks the bound UB itself)
    const uint64_t inf = (s_feas != kNone ? s_feas : s_ub) + 1;
    // ---- the reduced problem (one warp: lane q handles queue q, Q <= 32) ----
    if (tid < 32) mixed_build<T, D>(mt, C64, Q, elig_e, s_base, inf, &s_ubr);
    __syncthreads();
    if (sizeof(T) == 4 && s_ubr >= 0xffffffffull) {  // UB < 2^32 - 1 for 32-bit loads
      if (tid == 0 && part == 0) raise_flag(a.flags, kFlagNeedU64);
      abandoned = true;
      continue;
    }
    // ---- tables: inner sums of the last three reduced queues, one-hot outer vectors ----
    mixed_tables<T, D>(mt, C64, inf, s_base, in, V, base0, tid, nthr);
    __syncthreads();

    // ---- this thread's contiguous range of the rank's share of the reduced blocks ----
    const uint64_t nb = mt.nb;
    uint64_t rlo = 0, rhi = nb;
    if (a.world > 1) {  // contiguous shards of the reduced (feasible-order) block space
      rlo = (uint64_t)(((unsigned __int128)nb * (uint64_t)a.rank) / (uint64_t)a.world);
      rhi = (uint64_t)(((unsigned __int128)nb * (uint64_t)(a.rank + 1)) / (uint64_t)a.world);
    }
    const uint64_t nb_rank = rhi - rlo;
    const uint64_t T_all = (uint64_t)parts * nthr;
    const uint64_t gt = (uint64_t)part * nthr + tid;
    const uint64_t per = nb_rank / T_all, rem = nb_rank % T_all;
    const uint64_t b0 = rlo + gt * per + (gt < rem ? gt : rem);
    const uint64_t nleft = per + (gt < rem ? 1 : 0);

    T best = ~T(0);
    uint64_t best_blk = kNone;
    uint32_t best_span = 1;
    walk_mixed<T, D>(mt, in, V, base0, dig, nthr, tid, one, b0, nleft, best, best_blk, best_span);

    // ---- a5: the lowest thread holding the CTA minimum re-scans its best span ----
    {
      const uint64_t bv = (best_blk != kNone) ? (uint64_t)best : kNone;
      uint64_t wmin = bv;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) wmin = min(wmin, __shfl_xor_sync(0xffffffffu, wmin, off));
      __syncthreads();
      if ((tid & 31) == 0) red[tid >> 5].ms = wmin;
      if (tid == 0) s_winner = 0xffffffffu;
      __syncthreads();
      if (tid == 0) {
        uint64_t g = kNone;
        for (int w = 0; w < (nthr + 31) / 32; ++w) g = min(g, red[w].ms);
        s_gmin = g;
        s_cand = Cand{kNone, kNone};
      }
      __syncthreads();
      if (bv != kNone && bv == s_gmin) atomicMin(&s_winner, (uint32_t)tid);
      __syncthreads();
      const uint32_t win = s_winner;
      if (win != 0xffffffffu && (uint32_t)(tid >> 5) == (win >> 5)) {
        const int wl = (int)(win & 31);
        const uint64_t bb = __shfl_sync(0xffffffffu, best_blk, wl);
        const uint32_t span = __shfl_sync(0xffffffffu, best_span, wl);
        const T bt = __shfl_sync(0xffffffffu, best, wl);
        const uint64_t idx = mixed_span_first_warp<T, D>(bb, span, mt, V, base0, in, bt, one);
        if ((uint32_t)tid == win) s_cand = Cand{(uint64_t)bt, idx};
      }
      __syncthreads();
    }
    Cand c = s_cand;
    if (parts == 1) {
      if (tid == 0) write_epoch(a.out, e, Q, D, a.ibits, c, a.flags, s_feas);
      continue;
    }
    Cand* slots = a.scratch + (e - a.e_full) * parts;
    if (tid == 0) {
      slots[part] = c;
      __threadfence();
      const uint32_t prev = atomicAdd(&a.done[e], 1u);
      s_last = (prev == parts - 1);
    }
    __syncthreads();
    if (s_last) {
      __threadfence();
      Cand r{kNone, kNone};
      for (uint32_t t = tid; t < parts; t += nthr) {
        const volatile uint64_t* o = reinterpret_cast<const volatile uint64_t*>(&slots[t]);
        r = cand_min(r, Cand{o[0], o[1]});
      }
      r = block_min(r, red);
      if (tid == 0) {
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags, s_feas);
        a.done[e] = 0;
      }
    }
  }
  if (a.peer.world) peer_finish(a.peer, a.out, a.E, Q, D, a.ibits, a.flags, abandoned);
}

// ---------------------------------------------------------------------------------------
// Batches of constrained epochs: one WARP per epoch (the CTA-per-epoch kernel above spends
// most of a small epoch in CTA barriers and its winner logic; at 25 % pinned + 25 % masked
// queues of cfg2 an epoch has only ~3,700 feasible mappings). The warp builds the reduced
// problem and its tables in its own shared memory, its lanes walk contiguous ranges of the
// reduced blocks (walk_mixed), the lowest lane holding the minimum re-scans its span with
// the whole warp (mixed_span_first_warp) and lane 0 writes the epoch. Only 32-bit loads: an
// epoch whose reduced bound needs 64 bits raises kFlagNeedU64 and the host reruns the call
// on the 64-bit CTA kernel. Single GPU (no shards).
constexpr int kMixedWarps = 4;  // warps per CTA, each its own epochs

__host__ __device__ inline size_t mixed_warp_smem_bytes(uint32_t Q, uint32_t D) {
  // per warp: C64[Q*D] u64 | in[8*D] u32 | V[(Q-3)*D*D] u32 | dig[(Q-3)*32] u8, 16-aligned
  const size_t per = ((size_t)Q * D * 8 + 8 * D * 4 + (size_t)(Q >= 3 ? Q - 3 : 0) * D * D * 4 +
                      (size_t)(Q >= 3 ? Q - 3 : 1) * 32 + 15) / 16 * 16;
  return per * kMixedWarps;
}

template <int D>
__global__ void __launch_bounds__(32 * kMixedWarps, D <= 5 ? 4 : 2) search_mixed_warp_kernel(BlockedArgs a) {
  using T = uint32_t;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const size_t per = mixed_warp_smem_bytes(Q, D) / kMixedWarps;
  unsigned char* mine = smem_raw + per * wib;
  uint64_t* C64 = reinterpret_cast<uint64_t*>(mine);
  T* in = reinterpret_cast<T*>(C64 + Q * D);
  T* V = in + 8 * D;
  uint8_t* dig = reinterpret_cast<uint8_t*>(V + (size_t)(Q >= 3 ? Q - 3 : 0) * D * D);
  __shared__ MixedTab s_mt[kMixedWarps];
  __shared__ uint64_t s_base_w[kMixedWarps][D];
  __shared__ __align__(16) T s_base0[kMixedWarps][D];
  __shared__ uint32_t s_status_w[kMixedWarps];
  __shared__ uint64_t s_feas_w[kMixedWarps], s_ubr_w[kMixedWarps];
  MixedTab& mt = s_mt[wib];
  uint64_t* s_base = s_base_w[wib];
  T* base0 = s_base0[wib];
  const uint32_t one = a.one;
  const uint64_t nwarps = (uint64_t)gridDim.x * kMixedWarps;
  for (uint64_t e = (uint64_t)blockIdx.x * kMixedWarps + wib; e < a.E; e += nwarps) {
    // ---- a1: C = K + X, range check; base loads, INF masking (epoch_prologue) ----
    if (lane == 0) s_status_w[wib] = 0;
    __syncwarp();
    const uint64_t* Ke = a.K + e * Q * D;
    const uint64_t* Xe = a.X + e * Q * D;
    bool bad = false;
    for (uint32_t t = lane; t < Q * D; t += 32) {
      const uint64_t k = Ke[t], x = Xe[t];
      bad |= (k >= kEntryLimit) | (x >= kEntryLimit);
      C64[t] = k + x;
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) s_status_w[wib] = kFlagRange;
    __syncwarp();
    const uint16_t* elig_e = a.elig ? a.elig + e * Q : nullptr;
    const uint64_t ub = epoch_prologue(C64, Q, D, a.base ? a.base + e * D : nullptr, elig_e, s_base,
                                       &s_status_w[wib], &s_feas_w[wib]);
    const uint32_t status = s_status_w[wib];
    if (status) {
      if (lane == 0) raise_flag(a.flags, status);
      continue;
    }
    const uint64_t feas = s_feas_w[wib];
    const uint64_t inf = (feas != kNone ? feas : ub) + 1;
    // ---- the reduced problem and its tables (this warp alone) ----
    mixed_build<T, D>(mt, C64, Q, elig_e, s_base, inf, &s_ubr_w[wib]);
    if (s_ubr_w[wib] >= 0xffffffffull) {  // UB < 2^32 - 1 for 32-bit loads
      if (lane == 0) raise_flag(a.flags, kFlagNeedU64);
      continue;
    }
    mixed_tables<T, D>(mt, C64, inf, s_base, in, V, base0, lane, 32);
    __syncwarp();
    // ---- a2-a5: lane l walks a contiguous range of the reduced blocks ----
    const uint32_t nb = (uint32_t)mt.nb;  // <= 2^16 (host condition)
    const uint32_t pl = nb / 32, rem = nb % 32;
    const uint32_t b0 = (uint32_t)lane * pl + ((uint32_t)lane < rem ? (uint32_t)lane : rem);
    const uint32_t nleft = pl + ((uint32_t)lane < rem ? 1u : 0u);
    T best = ~T(0);
    uint32_t best_blk = 0xffffffffu;
    uint32_t best_span = 1;
    walk_mixed<T, D, uint32_t>(mt, in, V, base0, dig, 32, lane, one, b0, nleft, best, best_blk, best_span);
    // lexicographic (makespan, lane): lanes own increasing block ranges, so the lowest lane
    // holding the minimum holds the lowest reduced (= full) index of it
    uint64_t key = best_blk != 0xffffffffu ? ((uint64_t)best << 32) | (uint32_t)lane : kNone;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) key = min(key, __shfl_xor_sync(0xffffffffu, key, off));
    Cand c{kNone, kNone};
    if (key != kNone) {
      const int wl = (int)(key & 31u);
      const uint32_t bb = __shfl_sync(0xffffffffu, best_blk, wl);
      const uint32_t span = __shfl_sync(0xffffffffu, best_span, wl);
      const T bt = (T)(key >> 32);
      c = Cand{(uint64_t)bt, mixed_span_first_warp<T, D, uint32_t>(bb, span, mt, V, base0, in, bt, one)};
    }
    // a7: outputs, digits of the index in parallel (queue q on lane q, D a constant)
    if (c.ms != kNone && c.ms > feas) c = Cand{kNone, kNone};
    if (lane == 0) {
      a.out.index[e] = c.idx;
      a.out.makespan[e] = c.ms;
    }
    if (a.out.mapping && (uint32_t)lane < Q) {
      uint64_t rest = c.idx;
      for (uint32_t q = Q - 1; q > (uint32_t)lane; --q) rest /= D;
      a.out.mapping[e * Q + lane] = (c.idx == kNone) ? 0xFF : (uint8_t)(rest % D);
    }
    __syncwarp();  // the tables are rebuilt for the next epoch
  }
}

namespace {
template <typename T, int D>
cudaError_t launch_mixed_t(const BlockedArgs& a, dim3 grid, int threads, size_t smem, cudaStream_t st) {
  auto k = search_mixed_kernel<T, D>;
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  k<<<grid, threads, smem, st>>>(a);
  return cudaGetLastError();
}

template <typename T, int D>
int mixed_occ_t(int threads, size_t smem) {
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, search_mixed_kernel<T, D>, threads, smem) != cudaSuccess)
    return 1;
  return n < 1 ? 1 : n;
}
}  // namespace

int mixed_ctas_per_sm(uint32_t D, bool wide, int threads, size_t smem) {
  switch (D) {
#define MCL_MOCC(DD) \
  case DD: return wide ? mixed_occ_t<uint64_t, DD>(threads, smem) : mixed_occ_t<uint32_t, DD>(threads, smem);
    MCL_MOCC(2) MCL_MOCC(3) MCL_MOCC(4) MCL_MOCC(5) MCL_MOCC(6) MCL_MOCC(7) MCL_MOCC(8)
#undef MCL_MOCC
    default: return 1;
  }
}

cudaError_t launch_mixed(const BlockedArgs& a, bool wide, dim3 grid, int threads, size_t smem,
                         cudaStream_t st) {
  switch (a.D) {
#define MCL_MCASE(DD)                                                        \
  case DD:                                                                   \
    return wide ? launch_mixed_t<uint64_t, DD>(a, grid, threads, smem, st)   \
                : launch_mixed_t<uint32_t, DD>(a, grid, threads, smem, st);
    MCL_MCASE(2) MCL_MCASE(3) MCL_MCASE(4) MCL_MCASE(5) MCL_MCASE(6) MCL_MCASE(7) MCL_MCASE(8)
#undef MCL_MCASE
    default: return cudaErrorInvalidValue;
  }
}

namespace {
template <int D>
cudaError_t launch_mixed_warp_t(const BlockedArgs& a, int num_sms, cudaStream_t st, int* grid_out) {
  auto k = search_mixed_warp_kernel<D>;
  const size_t smem = mixed_warp_smem_bytes(a.Q, D);
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, 32 * kMixedWarps, smem);
  if (err != cudaSuccess) return err;
  per_sm = per_sm < 1 ? 1 : per_sm;
  uint64_t grid = (uint64_t)num_sms * per_sm;
  const uint64_t need = (a.E + kMixedWarps - 1) / kMixedWarps;
  if (grid > need) grid = need;
  k<<<(unsigned)grid, 32 * kMixedWarps, smem, st>>>(a);
  *grid_out = (int)grid;
  return cudaGetLastError();
}
}  // namespace

cudaError_t launch_mixed_warp(const BlockedArgs& a, int num_sms, cudaStream_t st, int* grid_out) {
  switch (a.D) {
#define MCL_MWCASE(DD) \
  case DD: return launch_mixed_warp_t<DD>(a, num_sms, st, grid_out);
    MCL_MWCASE(2) MCL_MWCASE(3) MCL_MWCASE(4) MCL_MWCASE(5) MCL_MWCASE(6) MCL_MWCASE(7) MCL_MWCASE(8)
#undef MCL_MWCASE
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mcl
