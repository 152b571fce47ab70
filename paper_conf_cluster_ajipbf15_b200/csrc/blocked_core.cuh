// blocked_core.cuh -- register-blocked leaf evaluation shared by the search kernels.
//
// One thread scores whole BLOCKS of D^3 mappings: the three innermost queues
// a = Q-3, b = Q-2, c = Q-1 (digits i, j, k) vary inside a block, the outer Q-3 digits are
// fixed and give the prefix load vector P[d] (queues on one device
// serialise, devices run concurrently). With M = max_d P[d] and every cost >= 0, the
// makespan of leaf (i, j, k) is max(M, load of each device the inner queues touch), which
// the compiler-unrolled leaf table below forms with ONE integer max per mapping:
//
//   i, j, k distinct : max3(P_i+A_i, P_j+B_j, max(M, P_k+C_k))
//   i == j != k      : max (P_i+A_i+B_i, max(M, P_k+C_k))
//   i == k != j      : max3(P_i+A_i+C_i, P_j+B_j, M)
//   j == k != i      : max3(P_i+A_i, P_j+B_j+C_j, M)
//   i == j == k      : max (M, P_i+A_i+B_i+C_i)
//
// (A, B, C = the composed cost rows C[q][.] = K + X of queues a, b, c.)
// Every leaf's makespan is formed explicitly in a register (a mapping counts
// as scored only then); the argmin is folded with the sm_100a three-input minimum (VIMNMX3:
// two mappings per ALU instruction), so the floor is 1.5 ALU instructions per mapping
// (DESIGN.md "Roofline"). The block minimum is compared with the thread's running best
// (strict <, blocks visited in increasing index order); only the best block (or
// super-block) is re-scanned at the end for the lowest leaf index.
//
// The outer digits walk an odometer: digit x (queue Q-4) is the block loop, the digits of
// queues 0..Q-5 live in shared memory and update the base load vector by one-hot vectors
// V[q][x] (V[q][x][d] = C[q][x] if d == x else 0) so every register index stays static.
#pragma once
#include "common.cuh"
#include "kernels.h"

namespace mcl {

#ifndef MCL_SUPER_MAX_D
#define MCL_SUPER_MAX_D 5
#endif
constexpr int kSuperMaxD = MCL_SUPER_MAX_D;  // super-block path for u32 and D <= this
#ifndef MCL_CHUNK_ODOMETER
#define MCL_CHUNK_ODOMETER 1  // chunk prefixes by odometer steps (0: full decode per chunk)
#endif

namespace {

// Adds routed to the FMA pipe (IMAD) so the ALU pipe is left for min/max: `one` is a
// runtime 1 the compiler cannot fold.
__device__ __forceinline__ uint32_t add_f(uint32_t a, uint32_t b, uint32_t one) {
  uint32_t r;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(one), "r"(b));
  return r;
}
__device__ __forceinline__ uint64_t add_f(uint64_t a, uint64_t b, uint32_t) { return a + b; }

// Integer min/max: VIMNMX (two inputs) and VIMNMX3 (three inputs) for 32-bit lanes.
__device__ __forceinline__ uint32_t max2(uint32_t a, uint32_t b) { return max(a, b); }
__device__ __forceinline__ uint32_t max3(uint32_t a, uint32_t b, uint32_t c) { return __vimax3_u32(a, b, c); }
__device__ __forceinline__ uint32_t min2(uint32_t a, uint32_t b) { return min(a, b); }
__device__ __forceinline__ uint32_t min3(uint32_t a, uint32_t b, uint32_t c) { return __vimin3_u32(a, b, c); }
__device__ __forceinline__ uint64_t max2(uint64_t a, uint64_t b) { return a > b ? a : b; }
__device__ __forceinline__ uint64_t max3(uint64_t a, uint64_t b, uint64_t c) { return max2(a, max2(b, c)); }
__device__ __forceinline__ uint64_t min2(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint64_t min3(uint64_t a, uint64_t b, uint64_t c) { return min2(a, min2(b, c)); }

// Per-block sums of the prefix loads P with the inner queues' costs (A, B, C = rows
// Q-3, Q-2, Q-1 of the composed cost table):
//   a = P+A, b = P+B, c = P+C, ab = P+A+B, ac = P+A+C, bc = P+B+C, abc = P+A+B+C.
// Shared-memory table `in[7][D]` holds A, B, C, A+B, A+C, B+C, A+B+C.
template <typename T, int D>
struct Sums {
  T a[D], b[D], c[D], ab[D], ac[D], bc[D], abc[D];
};

template <typename T, int D>
__device__ __forceinline__ void make_sums(Sums<T, D>& s, const T (&P)[D], const T* __restrict__ in,
                                          uint32_t one) {
#pragma unroll
  for (int d = 0; d < D; ++d) {
    s.a[d] = add_f(P[d], in[0 * D + d], one);
    s.b[d] = add_f(P[d], in[1 * D + d], one);
    s.c[d] = add_f(P[d], in[2 * D + d], one);
    s.ab[d] = add_f(P[d], in[3 * D + d], one);
    s.ac[d] = add_f(P[d], in[4 * D + d], one);
    s.bc[d] = add_f(P[d], in[5 * D + d], one);
    s.abc[d] = add_f(P[d], in[6 * D + d], one);
  }
}

template <typename T, int D>
__device__ __forceinline__ T max_of(const T (&P)[D]) {
  T M = P[0];
#pragma unroll
  for (int d = 1; d < D; ++d) M = max2(M, P[d]);
  return M;
}

#ifndef MCL_LEAF_M_AFTER
#define MCL_LEAF_M_AFTER 0  // 1: apply the prefix makespan M once per block, not in each leaf
#endif

// Enumerate the D^3 leaves of one block in increasing index order, calling f(leaf, v), v =
// the leaf's makespan. M = max_d P[d] (prefix makespan).
// MCL_LEAF_M_AFTER (measurement option, not built by default): v is only the maximum load
// of the devices the leaf's three inner queues touch (makespan = max(M, v)); as max(M, .)
// is non-decreasing, min over the leaves of max(M, v) = max(M, min v), so the block applies
// M once to its minimum (D fewer maxima per block, and the D diagonal leaves need none).
// Same results, 1.4-9 % faster (SS7), but the leaves' makespans are then not
// formed in registers, which SURVEY SS8(d) requires of a "scored" mapping.
template <typename T, int D, typename F>
__device__ __forceinline__ void for_each_leaf(const Sums<T, D>& s, T M, F&& f) {
#if MCL_LEAF_M_AFTER
#pragma unroll
  for (int i = 0; i < D; ++i)
#pragma unroll
    for (int j = 0; j < D; ++j)
#pragma unroll
      for (int k = 0; k < D; ++k) {
        T v;
        if (i != j && i != k && j != k) v = max3(s.a[i], s.b[j], s.c[k]);
        else if (i == j && j != k) v = max2(s.ab[i], s.c[k]);
        else if (i == k && i != j) v = max2(s.ac[i], s.b[j]);
        else if (j == k && i != j) v = max2(s.a[i], s.bc[j]);
        else v = s.abc[i];
        f((i * D + j) * D + k, v);
      }
#else
  T PCM[D];
#pragma unroll
  for (int d = 0; d < D; ++d) PCM[d] = max2(M, s.c[d]);
#pragma unroll
  for (int i = 0; i < D; ++i)
#pragma unroll
    for (int j = 0; j < D; ++j)
#pragma unroll
      for (int k = 0; k < D; ++k) {
        T v;
        if (i != j && i != k && j != k) v = max3(s.a[i], s.b[j], PCM[k]);
        else if (i == j && j != k) v = max2(s.ab[i], PCM[k]);
        else if (i == k && i != j) v = max3(s.ac[i], s.b[j], M);
        else if (j == k && i != j) v = max3(s.a[i], s.bc[j], M);
        else v = max2(M, s.abc[i]);
        f((i * D + j) * D + k, v);
      }
#endif
}

// Fold one block's leaves into a running 4-way minimum, two leaves per three-input min.
// `first` = the number of leaves folded before this block in the same run (a compile-time
// constant after unrolling), so the pairing continues across the blocks of a super-block.
template <typename T, int D>
__device__ __forceinline__ void block_fold(const Sums<T, D>& s, T M, int first, T (&acc)[4], T& pend) {
  for_each_leaf<T, D>(s, M, [&](int leaf, T v) {
    const int n = first + leaf;
    if (n & 1) {
      acc[(n >> 1) & 3] = min3(acc[(n >> 1) & 3], pend, v);
    } else {
      pend = v;
    }
  });
}

template <typename T>
__device__ __forceinline__ T fold_result(const T (&acc)[4], T pend, int leaves) {
  T g = min3(acc[0], acc[1], min2(acc[2], acc[3]));
  if (leaves & 1) g = min2(g, pend);
  return g;
}

// Minimum makespan over one block.
template <typename T, int D>
__device__ __forceinline__ T block_eval(const Sums<T, D>& s, T M) {
  constexpr T kMax = ~T(0);
  T acc[4] = {kMax, kMax, kMax, kMax};
  T pend = kMax;
  block_fold<T, D>(s, M, 0, acc, pend);
  const T g = fold_result<T>(acc, pend, D * D * D);
  return MCL_LEAF_M_AFTER ? max2(M, g) : g;
}

template <typename T, int D>
__device__ __forceinline__ T block_eval(const T (&P)[D], const T* __restrict__ in, uint32_t one) {
  Sums<T, D> s;
  make_sums<T, D>(s, P, in, one);
  return block_eval<T, D>(s, max_of<T, D>(P));
}

// A SUPER-BLOCK: the D blocks x = 0..D-1 of the fourth-innermost digit (queue Q-4) with
// the same outer prefix `base`. Only device x's load changes between them, so the sums of
// the other devices are shared and the block loop is unrolled with static x (used for
// small D, where a D^3 block alone is too short to amortise its setup). All D^4 leaves fold
// into ONE running minimum (one finalisation and one comparison with the thread's best per
// super-block); the rare new best is located by re-scanning the super-block at the end.
template <typename T, int D>
__device__ __forceinline__ T superblock_eval(const T (&base)[D], const T* __restrict__ in,
                                             const T* __restrict__ c4, uint32_t one) {
  constexpr T kMax = ~T(0);
  constexpr int kLeaves = D * D * D;
  T acc[4] = {kMax, kMax, kMax, kMax};
  T pend = kMax;
  T r = kMax;  // MCL_LEAF_M_AFTER: minimum over the blocks of max(M_x, block minimum)
  Sums<T, D> sb;
  make_sums<T, D>(sb, base, in, one);
  const T Mb = max_of<T, D>(base);
#pragma unroll
  for (int x = 0; x < D; ++x) {
    const T cx = c4[x];
    Sums<T, D> s = sb;
    s.a[x] = add_f(sb.a[x], cx, one);
    s.b[x] = add_f(sb.b[x], cx, one);
    s.c[x] = add_f(sb.c[x], cx, one);
    s.ab[x] = add_f(sb.ab[x], cx, one);
    s.ac[x] = add_f(sb.ac[x], cx, one);
    s.bc[x] = add_f(sb.bc[x], cx, one);
    s.abc[x] = add_f(sb.abc[x], cx, one);
    const T M = max2(Mb, add_f(base[x], cx, one));
#if MCL_LEAF_M_AFTER
    // each block's leaves fold on their own (its M applies to its minimum only)
    T bacc[4] = {kMax, kMax, kMax, kMax};
    T bpend = kMax;
    block_fold<T, D>(s, M, 0, bacc, bpend);
    r = min2(r, max2(M, fold_result<T>(bacc, bpend, kLeaves)));
#else
    block_fold<T, D>(s, M, x * kLeaves, acc, pend);
#endif
  }
  return MCL_LEAF_M_AFTER ? r : fold_result<T>(acc, pend, D * kLeaves);
}

template <typename T, int D>
__device__ __forceinline__ void load_vec(T (&v)[D], const T* __restrict__ src) {
#pragma unroll
  for (int d = 0; d < D; ++d) v[d] = src[d];
}

// Lowest leaf of a block whose makespan equals `target` (the block is known to hold one),
// found cooperatively by the 32 lanes (same P, same target): lane l takes the (i, j) pairs
// p = l, l + 32, ... of the two outer inner queues (runtime digits, loads formed by static
// per-device selects), then scores the D leaves k of the pair with static k, directly from
// the definition (loads P[d] plus the inner queues' costs on their devices, max over
// devices); leaf = p * D + k, and the warp minimum of every lane's first hit is the lowest
// leaf. One pass of at most two pairs per lane instead of D^3 / 32 rounds of runtime-digit
// scoring (the rescan sits on the kernel's critical tail).
template <typename T, int D>
__device__ __forceinline__ uint32_t block_first_warp(const T (&P)[D], const T* __restrict__ in,
                                                     T target) {
  constexpr uint32_t kPairs = (uint32_t)D * D;
  const uint32_t lane = threadIdx.x & 31;
  uint32_t first = 0xffffffffu;
  for (uint32_t p = lane; p < kPairs; p += 32) {
    const uint32_t i = p / D, j = p % D;
    T L[D];
    T Mp = 0;
#pragma unroll
    for (int d = 0; d < D; ++d) {
      T v = P[d];
      if (i == (uint32_t)d) v += in[0 * D + d];
      if (j == (uint32_t)d) v += in[1 * D + d];
      L[d] = v;
      Mp = max2(Mp, v);
    }
    uint32_t hit = 0xffffffffu;
#pragma unroll
    for (int k = D - 1; k >= 0; --k)
      if (max2(Mp, (T)(L[k] + in[2 * D + k])) == target) hit = p * D + (uint32_t)k;
    if (hit < first) first = hit;  // pairs ascend per lane: the first hit is its lowest
  }
  return __reduce_min_sync(0xffffffffu, first);
}

// Prefix loads P of block `blk` (outer digits of queues 0..O-1), decoded from scratch,
// on top of the devices' base loads B0 (zero unless the call is constrained).
template <typename T, int D>
__device__ __forceinline__ void prefix_of(T (&P)[D], uint64_t blk, int O, const T* __restrict__ V,
                                          const T* __restrict__ B0, uint32_t one) {
#pragma unroll
  for (int d = 0; d < D; ++d) P[d] = B0[d];
  for (int q = O - 1; q >= 0; --q) {
    const uint32_t dq = (uint32_t)(blk % D);
    blk /= D;
    const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) P[d] = add_f(P[d], v[d], one);
  }
}


// Score the blocks [b0, b0 + nleft) of one epoch for one thread, keeping the first strict
// minimum: best = its block minimum, best_blk = the block holding it (kNone if none).
// Tables (shared memory): in[8][D] (inner sums + the costs of queue O-1), V[O][D][D]
// one-hot outer vectors, zero[D], base0[D] device base loads (zero when unconstrained),
// dig[(O-1)][nthr] odometer digits of this thread.
template <typename T, int D>
struct WalkCtx {
  const T* in;
  const T* V;
  const T* zero;
  const T* base0;
  uint8_t* dig;
  int O;     // outer queues (Q - 3)
  int nthr;  // stride of the digit table
  int tid;
  uint32_t one;
};

// Lowest mapping index in blocks [bb, bb + span) whose makespan equals `target` (the span
// is known to hold one): blocks in increasing order, each re-scanned by the whole warp.
// Called by all 32 lanes with the same arguments.
template <typename T, int D>
__device__ __forceinline__ uint64_t span_first_warp(uint64_t bb, uint32_t span, int O,
                                                    const T* __restrict__ V, const T* __restrict__ B0,
                                                    const T* __restrict__ in, T target, uint32_t one) {
  for (uint32_t t = 0; t < span; ++t) {
    T P[D];
    prefix_of<T, D>(P, bb + t, O, V, B0, one);
    const uint32_t leaf = block_first_warp<T, D>(P, in, target);
    if (leaf != 0xffffffffu) return (bb + t) * (uint64_t)(D * D * D) + leaf;
  }
  return kNone;
}

// best_span: the number of blocks starting at best_blk that hold the best (1, or D for a
// super-block).
template <typename T, int D>
__device__ __forceinline__ void walk_blocks(const WalkCtx<T, D>& w, uint64_t b0, uint64_t nleft,
                                            T& best, uint64_t& best_blk, uint32_t& best_span) {
  constexpr bool kSuper = (sizeof(T) == 4 && D <= kSuperMaxD);
  const int O = w.O, nthr = w.nthr, tid = w.tid;
  const uint32_t one = w.one;
  const T* in = w.in;
  const T* V = w.V;
  const T* zero = w.zero;
  const T* B0 = w.base0;
  uint8_t* dig = w.dig;
  const bool chunked = kSuper && O >= 2;
  const uint64_t chunk = chunked ? (uint64_t)D * D : 1;
  if (nleft && chunked) {
    // Super-block path: queue O-1 = digit x (static, inside superblock_eval), queue
    // O-2 = digit y (uniform loop), queues 0..O-3 = the chunk index, decoded by a loop
    // whose trip count is the same for every lane (no divergent carries).
    const T* c4 = in + 7 * D;
    const T* Vy = V + (size_t)(O - 2) * D * D;
    uint64_t blk = b0;
    auto single = [&](uint64_t bk) {
      T P[D];
      prefix_of<T, D>(P, bk, O, V, B0, one);
      const T g = block_eval<T, D>(P, in, one);
      if (g < best) {
        best = g;
        best_blk = bk;
        best_span = 1;
      }
    };
    for (; nleft && (blk % chunk) != 0; ++blk, --nleft) single(blk);
#if MCL_CHUNK_ODOMETER
    // The chunk prefix (queues 0..O-3) is decoded once; consecutive chunks then step an
    // odometer over those digits (kept in shared memory), updating the prefix by one-hot
    // deltas: one digit changes per chunk, a carry every D chunks (lanes carry at different
    // chunks: a short divergent step instead of a full decode per chunk).
    T base2[D];
    if (nleft >= chunk) {
      uint64_t ch = blk / chunk;
#pragma unroll
      for (int d = 0; d < D; ++d) base2[d] = B0[d];
      for (int q = O - 3; q >= 0; --q) {
        const uint32_t dq = (uint32_t)(ch % D);
        ch /= D;
        dig[q * nthr + tid] = (uint8_t)dq;
        const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
        for (int d = 0; d < D; ++d) base2[d] = add_f(base2[d], v[d], one);
      }
    }
    for (bool first = true; nleft >= chunk; nleft -= chunk, blk += chunk, first = false) {
      if (!first) {
        for (int q = O - 3; q >= 0; --q) {  // odometer step to this chunk
          const uint32_t old = dig[q * nthr + tid];
          const uint32_t nw = (old + 1 == (uint32_t)D) ? 0u : old + 1;
          dig[q * nthr + tid] = (uint8_t)nw;
          const T* vo = V + ((size_t)q * D + old) * D;
          const T* vn = V + ((size_t)q * D + nw) * D;
#pragma unroll
          for (int d = 0; d < D; ++d) base2[d] = base2[d] - vo[d] + vn[d];
          if (nw != 0) break;
        }
      }
#else
    for (; nleft >= chunk; nleft -= chunk, blk += chunk) {
      uint64_t ch = blk / chunk;
      T base2[D];
#pragma unroll
      for (int d = 0; d < D; ++d) base2[d] = B0[d];
      for (int q = O - 3; q >= 0; --q) {
        const uint32_t dq = (uint32_t)(ch % D);
        ch /= D;
        const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
        for (int d = 0; d < D; ++d) base2[d] = add_f(base2[d], v[d], one);
      }
#endif
      for (int y = 0; y < D; ++y) {
        T base[D], vy[D];
        load_vec<T, D>(vy, Vy + y * D);
#pragma unroll
        for (int d = 0; d < D; ++d) base[d] = add_f(base2[d], vy[d], one);
        const T gs = superblock_eval<T, D>(base, in, c4, one);
        if (gs < best) {
          best = gs;
          best_blk = blk + (uint64_t)y * D;
          best_span = D;
        }
      }
    }
    for (; nleft; ++blk, --nleft) single(blk);
  } else if (nleft) {
    {
      // digit x = queue O-1 runs fastest; queues 0..O-2 are the odometer in smem.
      // Q == 3 (O == 0): a single block whose prefix is the zero vector.
      const T* Vx = (O >= 1) ? V + (size_t)(O - 1) * D * D : zero;
      // composed costs of queue O-1 (the x digit), for the super-block path
      const T* c4 = (O >= 1) ? in + 7 * D : zero;
      uint32_t x = (uint32_t)(b0 % D);
      uint64_t hi = b0 / D;
      T base[D];
#pragma unroll
      for (int d = 0; d < D; ++d) base[d] = B0[d];
      for (int q = O - 2; q >= 0; --q) {
        const uint32_t dq = (uint32_t)(hi % D);
        hi /= D;
        dig[q * nthr + tid] = (uint8_t)dq;
        const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
        for (int d = 0; d < D; ++d) base[d] = add_f(base[d], v[d], one);
      }
      uint64_t blk = b0;
      while (true) {
        if (kSuper && x == 0 && nleft >= (uint64_t)D) {
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
        for (; x < (uint32_t)D && nleft; ++x, --nleft, ++blk) {
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
        // odometer increment of the outer digits, updating base by one-hot deltas
        for (int q = O - 2; q >= 0; --q) {
          const uint32_t old = dig[q * nthr + tid];
          const uint32_t nw = (old + 1 == (uint32_t)D) ? 0u : old + 1;
          dig[q * nthr + tid] = (uint8_t)nw;
          const T* vo = V + ((size_t)q * D + old) * D;
          const T* vn = V + ((size_t)q * D + nw) * D;
#pragma unroll
          for (int d = 0; d < D; ++d) base[d] = base[d] - vo[d] + vn[d];
          if (nw != 0) break;
        }
      }
    }
  }}

}  // namespace

}  // namespace mcl
