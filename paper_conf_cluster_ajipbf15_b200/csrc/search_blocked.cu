// search_blocked.cu -- the register-blocked exhaustive mapper search.
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
// Every leaf's makespan is formed explicitly in a register; the argmin is folded with the
// sm_100a three-input minimum (VIMNMX3: two mappings per ALU instruction), so the floor is
// 1.5 ALU instructions per mapping. The block minimum is compared
// with the thread's running best (strict <, blocks visited in increasing index order);
// only the single best block is re-scanned at the end to recover the lowest leaf index.
//
// The outer digits walk an odometer: digit x (queue Q-4) is the block loop, the digits of
// queues 0..Q-5 live in shared memory and update the base load vector by one-hot vectors
// V[q][x] (V[q][x][d] = C[q][x] if d == x else 0) so every register index stays static.
#include "common.cuh"
#include "kernels.h"

namespace mcl {

#ifndef MCL_SUPER_MAX_D
#define MCL_SUPER_MAX_D 5
#endif
constexpr int kSuperMaxD = MCL_SUPER_MAX_D;  // super-block path for u32 and D <= this

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

// Enumerate the D^3 leaves of one block in increasing index order, calling f(leaf, ms).
// M = max_d P[d] (prefix makespan).
template <typename T, int D, typename F>
__device__ __forceinline__ void for_each_leaf(const Sums<T, D>& s, T M, F&& f) {
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
}

// Minimum makespan over one block, folded two leaves per three-input min.
template <typename T, int D>
__device__ __forceinline__ T block_eval(const Sums<T, D>& s, T M) {
  constexpr T kMax = ~T(0);
  T acc[4] = {kMax, kMax, kMax, kMax};
  T pend = kMax;
  for_each_leaf<T, D>(s, M, [&](int leaf, T v) {
    if (leaf & 1) {
      acc[(leaf >> 1) & 3] = min3(acc[(leaf >> 1) & 3], pend, v);
    } else {
      pend = v;
    }
  });
  constexpr int kLeaves = D * D * D;
  T g = min3(acc[0], acc[1], min2(acc[2], acc[3]));
  if (kLeaves & 1) g = min2(g, pend);
  return g;
}

template <typename T, int D>
__device__ __forceinline__ T block_eval(const T (&P)[D], const T* __restrict__ in, uint32_t one) {
  Sums<T, D> s;
  make_sums<T, D>(s, P, in, one);
  return block_eval<T, D>(s, max_of<T, D>(P));
}

// Lowest leaf of the block whose makespan equals `target` (the block is known to hold one).
template <typename T, int D>
__device__ __forceinline__ uint32_t block_first(const T (&P)[D], const T* __restrict__ in,
                                                uint32_t one, T target) {
  Sums<T, D> s;
  make_sums<T, D>(s, P, in, one);
  uint32_t first = 0xffffffffu;
  for_each_leaf<T, D>(s, max_of<T, D>(P), [&](int leaf, T v) {
    first = (v == target && first == 0xffffffffu) ? (uint32_t)leaf : first;
  });
  return first;
}

// A SUPER-BLOCK: the D blocks x = 0..D-1 of the fourth-innermost digit (queue Q-4) with
// the same outer prefix `base`. Only device x's load changes between them, so the sums of
// the other devices are shared and the block loop is unrolled with static x (used for
// small D, where a D^3 block alone is too short to amortise its setup).
template <typename T, int D>
__device__ __forceinline__ void superblock_eval(const T (&base)[D], const T* __restrict__ in,
                                                const T* __restrict__ c4, uint32_t one, T (&g)[D]) {
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
    g[x] = block_eval<T, D>(s, M);
  }
}

template <typename T, int D>
__device__ __forceinline__ void load_vec(T (&v)[D], const T* __restrict__ src) {
#pragma unroll
  for (int d = 0; d < D; ++d) v[d] = src[d];
}

// Prefix loads P of block `blk` (outer digits of queues 0..O-1), decoded from scratch.
template <typename T, int D>
__device__ __forceinline__ void prefix_of(T (&P)[D], uint64_t blk, int O, const T* __restrict__ V,
                                          uint32_t one) {
#pragma unroll
  for (int d = 0; d < D; ++d) P[d] = 0;
  for (int q = O - 1; q >= 0; --q) {
    const uint32_t dq = (uint32_t)(blk % D);
    blk /= D;
    const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) P[d] = add_f(P[d], v[d], one);
  }
}

}  // namespace

// Kernel: gridDim.x = CTAs per epoch (cpe), gridDim.y = epochs handled concurrently.
template <typename T, int D>
__global__ void __launch_bounds__(256, (sizeof(T) == 4 && D <= 5) ? 2 : 1)
    search_blocked_kernel(BlockedArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q;
  const int O = (int)Q - 3;  // outer queues (>= 0)
  const int nthr = blockDim.x, tid = threadIdx.x;
  // layout: C64[Q*D] u64 | in[8*D] T | V[O*D*D] T | red[32] Cand | dig[(O-1)*nthr] u8
  // (in[0..7) = inner sums, in[7] = composed costs of queue Q-4)
  uint64_t* C64 = reinterpret_cast<uint64_t*>(smem_raw);
  T* in = reinterpret_cast<T*>(C64 + Q * D);
  T* V = in + 8 * D;
  Cand* red = reinterpret_cast<Cand*>(
      reinterpret_cast<unsigned char*>(smem_raw) + a.off_red);
  uint8_t* dig = reinterpret_cast<uint8_t*>(smem_raw) + a.off_dig;
  __shared__ __align__(16) T zero[D];
  if (threadIdx.x < D) zero[threadIdx.x] = 0;
  __shared__ int s_bad;
  __shared__ uint64_t s_ub;
  constexpr bool kSuper = (sizeof(T) == 4 && D <= kSuperMaxD);

  for (uint64_t e = blockIdx.y; e < a.E; e += gridDim.y) {
    // ---- a1: cost composition C = K + X, range check, bound UB = sum_q max_d C ----
    __syncthreads();  // the previous epoch's tables are no longer read
    if (tid == 0) { s_bad = 0; s_ub = 0; }
    __syncthreads();
    const uint64_t* Ke = a.K + e * Q * D;
    const uint64_t* Xe = a.X + e * Q * D;
    for (uint32_t t = tid; t < Q * D; t += nthr) {
      const uint64_t k = Ke[t], x = Xe[t];
      if (k >= kEntryLimit || x >= kEntryLimit) s_bad = 1;
      C64[t] = k + x;
    }
    __syncthreads();
    if (s_bad) {
      if (tid == 0 && blockIdx.x == 0) raise_flag(a.flags, kFlagRange);
      continue;
    }
    if (tid < 32) {  // one warp: per-queue row max, then the sum over queues
      uint64_t part = 0;
      for (uint32_t q = tid; q < Q; q += 32) {
        uint64_t m = 0;
        for (int d = 0; d < D; ++d) m = max2(m, C64[q * D + d]);
        part += m;
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) part += __shfl_xor_sync(0xffffffffu, part, off);
      if (tid == 0) s_ub = part;
    }
    __syncthreads();
    if (sizeof(T) == 4 && s_ub >= (1ull << 32)) {
      if (tid == 0 && blockIdx.x == 0) raise_flag(a.flags, kFlagNeedU64);
      continue;
    }
    // ---- tables: inner sums and one-hot outer vectors ----
    for (int t = tid; t < D; t += nthr) {
      const uint64_t A = C64[(Q - 3) * D + t], B = C64[(Q - 2) * D + t], Cc = C64[(Q - 1) * D + t];
      in[0 * D + t] = (T)A;
      in[1 * D + t] = (T)B;
      in[2 * D + t] = (T)Cc;
      in[3 * D + t] = (T)(A + B);
      in[4 * D + t] = (T)(A + Cc);
      in[5 * D + t] = (T)(B + Cc);
      in[6 * D + t] = (T)(A + B + Cc);
    }
    for (int t = tid; t < D; t += nthr) in[7 * D + t] = (O >= 1) ? (T)C64[(O - 1) * D + t] : (T)0;
    for (int t = tid; t < O * D * D; t += nthr) {
      const int q = t / (D * D), x = (t / D) % D, d = t % D;
      V[t] = (d == x) ? (T)C64[q * D + x] : (T)0;
    }
    __syncthreads();

    // ---- a2-a5: this thread's contiguous block range inside the rank's range ----
    // Split points are aligned to whole CHUNKS (D^2 blocks on the super-block path) so the
    // lanes of a warp walk chunks in lock-step; only the rank's two ends can be ragged.
    const uint64_t nb_rank = a.rhi - a.rlo;
    const uint64_t T_all = (uint64_t)gridDim.x * nthr;
    const uint64_t gt = (uint64_t)blockIdx.x * nthr + tid;
    const bool chunked = kSuper && O >= 2;
    const uint64_t chunk = chunked ? (uint64_t)D * D : 1;
    auto split = [&](uint64_t t) -> uint64_t {
      if (t == 0) return a.rlo;
      if (t >= T_all) return a.rhi;
      const uint64_t per = nb_rank / T_all, rem = nb_rank % T_all;
      uint64_t s = a.rlo + t * per + (t < rem ? t : rem);
      s = s / chunk * chunk;
      return s < a.rlo ? a.rlo : (s > a.rhi ? a.rhi : s);
    };
    const uint64_t b0 = split(gt);
    uint64_t nleft = split(gt + 1) - b0;

    T best = ~T(0);
    uint64_t best_blk = kNone;
    const uint32_t one = a.one;
    if (nleft && chunked) {
      // Super-block path: queue O-1 = digit x (static, inside superblock_eval), queue
      // O-2 = digit y (uniform loop), queues 0..O-3 = the chunk index, decoded by a loop
      // whose trip count is the same for every lane (no divergent carries).
      const T* c4 = in + 7 * D;
      const T* Vy = V + (size_t)(O - 2) * D * D;
      uint64_t blk = b0;
      auto single = [&](uint64_t bk) {
        T P[D];
        prefix_of<T, D>(P, bk, O, V, one);
        const T g = block_eval<T, D>(P, in, one);
        if (g < best) {
          best = g;
          best_blk = bk;
        }
      };
      for (; nleft && (blk % chunk) != 0; ++blk, --nleft) single(blk);
      for (; nleft >= chunk; nleft -= chunk, blk += chunk) {
        uint64_t ch = blk / chunk;
        T base2[D];
#pragma unroll
        for (int d = 0; d < D; ++d) base2[d] = 0;
        for (int q = O - 3; q >= 0; --q) {
          const uint32_t dq = (uint32_t)(ch % D);
          ch /= D;
          const T* v = V + ((size_t)q * D + dq) * D;
#pragma unroll
          for (int d = 0; d < D; ++d) base2[d] = add_f(base2[d], v[d], one);
        }
        for (int y = 0; y < D; ++y) {
          T base[D], vy[D];
          load_vec<T, D>(vy, Vy + y * D);
#pragma unroll
          for (int d = 0; d < D; ++d) base[d] = add_f(base2[d], vy[d], one);
          T g[D];
          superblock_eval<T, D>(base, in, c4, one, g);
          T gs = g[0];
#pragma unroll
          for (int t = 1; t < D; ++t) gs = min2(gs, g[t]);
          if (gs < best) {  // rare: locate the first block holding the new minimum
            best = gs;
            const uint64_t bb = blk + (uint64_t)y * D;
#pragma unroll
            for (int t = D - 1; t >= 0; --t)
              if (g[t] == gs) best_blk = bb + t;
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
        for (int d = 0; d < D; ++d) base[d] = 0;
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
            T g[D];
            superblock_eval<T, D>(base, in, c4, one, g);
            T gs = g[0];
#pragma unroll
            for (int t = 1; t < D; ++t) gs = min2(gs, g[t]);
            if (gs < best) {  // rare: locate the first block holding the new minimum
              best = gs;
#pragma unroll
              for (int t = D - 1; t >= 0; --t)
                if (g[t] == gs) best_blk = blk + t;
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
    }
    // ---- a5: lowest index inside the best block, then warp / CTA / epoch argmin ----
    // Thread ranges ascend with the thread id, so the CTA's lowest-index optimum belongs to
    // the LOWEST thread whose best equals the CTA minimum; only that thread re-scans its
    // best block (one block per CTA instead of one per thread).
    __shared__ uint64_t s_gmin;
    __shared__ uint32_t s_winner;
    __shared__ Cand s_cand;
    {
      const uint64_t bv = (best_blk != kNone) ? (uint64_t)best : kNone;
      uint64_t wmin = bv;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) wmin = min(wmin, __shfl_xor_sync(0xffffffffu, wmin, off));
      __syncthreads();  // `red` may still be read by a previous epoch's reduction
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
      if ((uint32_t)tid == s_winner) {
        T P[D];
        prefix_of<T, D>(P, best_blk, O, V, one);
        const uint32_t leaf = block_first<T, D>(P, in, one, best);
        s_cand = Cand{(uint64_t)best, best_blk * (uint64_t)(D * D * D) + leaf};
      }
      __syncthreads();
    }
    Cand c = s_cand;
    if (gridDim.x == 1) {
      if (tid == 0) write_epoch(a.out, e, Q, D, a.ibits, c, a.flags);
      continue;
    }
    __shared__ bool s_last;
    if (tid == 0) {
      a.scratch[e * gridDim.x + blockIdx.x] = c;
      __threadfence();
      const uint32_t prev = atomicAdd(&a.done[e], 1u);
      s_last = (prev == gridDim.x - 1);
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
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags);
        a.done[e] = 0;  // self-reset for the next call
      }
    }
  }
}

template <typename T, int D>
static cudaError_t launch_blocked_t(const BlockedArgs& a, dim3 grid, int threads, size_t smem,
                                   cudaStream_t st) {
  auto k = search_blocked_kernel<T, D>;
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  k<<<grid, threads, smem, st>>>(a);
  return cudaGetLastError();
}

size_t blocked_smem_bytes(uint32_t Q, uint32_t D, bool wide, int threads, size_t* off_red,
                          size_t* off_dig) {
  const size_t tsz = wide ? 8 : 4;
  const int O = (int)Q - 3;
  size_t off = (size_t)Q * D * 8 + 8 * D * tsz + (size_t)(O > 0 ? O : 0) * D * D * tsz;
  off = (off + 15) & ~size_t(15);
  *off_red = off;
  off += 32 * sizeof(Cand);
  *off_dig = off;
  off += (size_t)(O > 1 ? O - 1 : 0) * threads;
  return (off + 15) & ~size_t(15);
}

namespace {
template <typename T, int D>
int occ_t(int threads, size_t smem) {
  // cache the last (threads, smem) query: the launch path asks the same question every call
  static std::atomic<uint64_t> last{0};
  const uint64_t key = ((uint64_t)threads << 40) | ((uint64_t)smem << 8);
  const uint64_t hit = last.load(std::memory_order_relaxed);
  if (hit && (hit & ~0xffull) == key) return (int)(hit & 0xff);
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, search_blocked_kernel<T, D>, threads, smem) !=
      cudaSuccess)
    return 1;
  n = n < 1 ? 1 : (n > 255 ? 255 : n);
  last.store(key | (uint64_t)n, std::memory_order_relaxed);
  return n;
}
}  // namespace

int blocked_ctas_per_sm(uint32_t D, bool wide, int threads, size_t smem) {
#ifdef MCL_ONLY_D
  if (D != MCL_ONLY_D) return 1;
  return wide ? occ_t<uint64_t, MCL_ONLY_D>(threads, smem) : occ_t<uint32_t, MCL_ONLY_D>(threads, smem);
#else
  switch (D) {
    case 2: return wide ? occ_t<uint64_t, 2>(threads, smem) : occ_t<uint32_t, 2>(threads, smem);
    case 3: return wide ? occ_t<uint64_t, 3>(threads, smem) : occ_t<uint32_t, 3>(threads, smem);
    case 4: return wide ? occ_t<uint64_t, 4>(threads, smem) : occ_t<uint32_t, 4>(threads, smem);
    case 5: return wide ? occ_t<uint64_t, 5>(threads, smem) : occ_t<uint32_t, 5>(threads, smem);
    case 6: return wide ? occ_t<uint64_t, 6>(threads, smem) : occ_t<uint32_t, 6>(threads, smem);
    case 7: return wide ? occ_t<uint64_t, 7>(threads, smem) : occ_t<uint32_t, 7>(threads, smem);
    case 8: return wide ? occ_t<uint64_t, 8>(threads, smem) : occ_t<uint32_t, 8>(threads, smem);
    default: return 1;
  }
#endif
}

bool blocked_supported(uint32_t Q, uint32_t D) { return Q >= 3 && D >= 2 && D <= kBlockedMaxD; }

cudaError_t launch_blocked(const BlockedArgs& a, bool wide, dim3 grid, int threads, size_t smem,
                           cudaStream_t st) {
#ifdef MCL_ONLY_D
#define MCL_CASE(DD)                                                                  \
  case DD:                                                                            \
    if (DD != MCL_ONLY_D) return cudaErrorInvalidValue;                               \
    return wide ? launch_blocked_t<uint64_t, DD % MCL_ONLY_D == 0 ? DD : MCL_ONLY_D>(a, grid, threads, smem, st) \
                : launch_blocked_t<uint32_t, DD % MCL_ONLY_D == 0 ? DD : MCL_ONLY_D>(a, grid, threads, smem, st);
#else
#define MCL_CASE(DD)                                                                  \
  case DD:                                                                            \
    return wide ? launch_blocked_t<uint64_t, DD>(a, grid, threads, smem, st)          \
                : launch_blocked_t<uint32_t, DD>(a, grid, threads, smem, st);
#endif
  switch (a.D) {
    MCL_CASE(2)
    MCL_CASE(3)
    MCL_CASE(4)
    MCL_CASE(5)
    MCL_CASE(6)
    MCL_CASE(7)
    MCL_CASE(8)
    default:
      return cudaErrorInvalidValue;
  }
#undef MCL_CASE
}

}  // namespace mcl
