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
#include "blocked_core.cuh"
#include "peer.cuh"

namespace mcl {

#ifdef MCL_TRACE
// Measurement build only (scripts/build_variant.py ... -DMCL_TRACE): per CTA, %globaltimer
// and clock64 at the kernel start, after the tables, after every thread's walk, and at the
// end -- to split the per-launch fixed cost into ramp, prologue, walk and reduction.
__device__ unsigned long long g_mcl_trace[4096][8];
__device__ __forceinline__ unsigned long long trace_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define MCL_TRACE_AT(slot)                                                                 \
  do {                                                                                     \
    if (threadIdx.x == 0 && blockIdx.x < 4096) {                                           \
      g_mcl_trace[blockIdx.x][2 * (slot)] = trace_ns();                                    \
      g_mcl_trace[blockIdx.x][2 * (slot) + 1] = (unsigned long long)clock64();             \
    }                                                                                      \
  } while (0)
#else
#define MCL_TRACE_AT(slot) \
  do {                     \
  } while (0)
#endif

// Kernel work layout over a 1-D grid of CTAs: the first e_full epochs get one CTA each; the
// remaining E - e_full epochs (the "tail") get tail_cpe CTAs each, so the last wave of a
// batch runs split epochs instead of idling (wave quantisation), and a single large epoch
// (e_full = 0) spreads over every CTA. The grid strides over this CTA index space.
// kLean: the register budget of one CTA per SM for the u32 D = 5 kernel, whose two-CTA
// build spills (56 bytes of stack); chosen for single-epoch searches (measured: 12 x 5 one
// epoch 63 -> 50 us), while batched calls keep two CTAs per SM for their grid shapes.
template <typename T, int D, bool kLean = false>
__global__ void __launch_bounds__(256, (sizeof(T) == 4 && D <= 5 && !kLean) ? 2 : 1)
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
  __shared__ uint32_t s_status;
  __shared__ uint64_t s_ub;
  __shared__ uint64_t s_feas;  // feasible bound of a constrained epoch (else kNone)
  __shared__ uint64_t s_base[D];
  __shared__ __align__(16) T base0[D];  // base loads in the search's arithmetic type
  constexpr bool kSuper = (sizeof(T) == 4 && D <= kSuperMaxD);

  const uint64_t ncta = a.e_full + (a.E - a.e_full) * a.tail_cpe;
  bool abandoned = false;  // an epoch skipped on an input error / for the 64-bit rerun
  MCL_TRACE_AT(0);
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
    // ---- a1: cost composition C = K + X, range check, bound UB = sum_q max_d C ----
    __syncthreads();  // the previous epoch's tables are no longer read
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
    if (tid < 32) {  // one warp: base loads, eligibility masking, the bound UB
      const uint64_t ub = epoch_prologue(C64, Q, D, a.base ? a.base + e * D : nullptr,
                                         a.elig ? a.elig + e * Q : nullptr, s_base, &s_status,
                                         &s_feas);
      if (tid == 0) s_ub = ub;
    }
    __syncthreads();
    if (s_status) {
      if (tid == 0 && part == 0) raise_flag(a.flags, s_status);
      abandoned = true;
      continue;
    }
    // 32-bit loads need UB < 2^32 - 1: every makespan then stays below the all-ones
    // "no candidate" value the running minima start from (UB = 2^32 - 1 takes the 64-bit
    // rerun; with UB = 2^32 - 1 an optimum equal to it would never pass the strict <)
    if (sizeof(T) == 4 && s_ub >= 0xffffffffull) {
      if (tid == 0 && part == 0) raise_flag(a.flags, kFlagNeedU64);
      abandoned = true;
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
    for (int t = tid; t < D; t += nthr) base0[t] = (T)s_base[t];
    for (int t = tid; t < O * D * D; t += nthr) {
      const int q = t / (D * D), x = (t / D) % D, d = t % D;
      V[t] = (d == x) ? (T)C64[q * D + x] : (T)0;
    }
    __syncthreads();

    MCL_TRACE_AT(1);
    // ---- a2-a5: this thread's contiguous block range inside the rank's range ----
    // Split points are aligned to whole CHUNKS (D^2 blocks on the super-block path) so the
    // lanes of a warp walk chunks in lock-step; only the rank's two ends can be ragged.
    const uint64_t nb_rank = a.rhi - a.rlo;
    const uint64_t T_all = (uint64_t)parts * nthr;
    const uint64_t gt = (uint64_t)part * nthr + tid;
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
    uint32_t best_span = 1;
    const uint32_t one = a.one;
    const WalkCtx<T, D> wctx{in, V, zero, base0, dig, O, nthr, tid, one};
    walk_blocks<T, D>(wctx, b0, nleft, best, best_blk, best_span);
    // ---- a5: lowest index inside the best block, then warp / CTA / epoch argmin ----
    // Every block belongs to one thread and a thread's span [best_blk, best_blk + span)
    // holds its first minimum, so among the threads whose best equals the CTA minimum the
    // one with the LOWEST best_blk owns the CTA's lowest-index optimum; only that thread's
    // warp re-scans its best block (one block per CTA instead of one per thread).
    __shared__ uint64_t s_gmin;
    __shared__ unsigned long long s_winblk;
    __shared__ uint32_t s_winner;
    __shared__ Cand s_cand;
    {
      const uint64_t bv = (best_blk != kNone) ? (uint64_t)best : kNone;
      uint64_t wmin = bv;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) wmin = min(wmin, __shfl_xor_sync(0xffffffffu, wmin, off));
      __syncthreads();  // `red` may still be read by a previous epoch's reduction
      MCL_TRACE_AT(2);
      if ((tid & 31) == 0) red[tid >> 5].ms = wmin;
      if (tid == 0) {
        s_winner = 0xffffffffu;
        s_winblk = ~0ull;
      }
      __syncthreads();
      if (tid == 0) {
        uint64_t g = kNone;
        for (int w = 0; w < (nthr + 31) / 32; ++w) g = min(g, red[w].ms);
        s_gmin = g;
        s_cand = Cand{kNone, kNone};
      }
      __syncthreads();
      const bool holder = bv != kNone && bv == s_gmin;
      if (holder) atomicMin(&s_winblk, (unsigned long long)best_blk);
      __syncthreads();
      if (holder && best_blk == s_winblk) s_winner = (uint32_t)tid;
      __syncthreads();
      const uint32_t win = s_winner;
      if (win != 0xffffffffu && (uint32_t)(tid >> 5) == (win >> 5)) {  // the winner's warp
        const int wl = (int)(win & 31);
        const uint64_t bb = __shfl_sync(0xffffffffu, best_blk, wl);
        const uint32_t span = __shfl_sync(0xffffffffu, best_span, wl);
        const T bt = __shfl_sync(0xffffffffu, best, wl);
        const uint64_t idx = span_first_warp<T, D>(bb, span, O, V, base0, in, bt, one);
        if ((uint32_t)tid == win) s_cand = Cand{(uint64_t)bt, idx};
      }
      __syncthreads();
    }
    Cand c = s_cand;
    if (parts == 1) {
      if (tid == 0) write_epoch(a.out, e, Q, D, a.ibits, c, a.flags, s_feas);
      continue;
    }
    // a split epoch. When (makespan, index) packs into one u64 (UB < 2^(64 - ibits); every
    // CTA of the epoch sees the same UB), the CTAs fold their candidates into one per-epoch
    // key with atomicMin and the last CTA only decodes it (the lexicographic minimum is the
    // minimum key); otherwise per-CTA candidates go to scratch and the last CTA reduces them.
    __shared__ bool s_last;
    const bool packed = a.keyslot && a.ibits > 0 && a.ibits < 64 && (s_ub >> (64 - a.ibits)) == 0;
    Cand* slots = a.scratch + (e - a.e_full) * parts;
    if (tid == 0) {
      if (packed) {
        if (c.ms != kNone)
          atomicMin(reinterpret_cast<unsigned long long*>(a.keyslot + e),
                    (unsigned long long)((c.ms << a.ibits) | c.idx));
      } else {
        slots[part] = c;
      }
      __threadfence();
      const uint32_t prev = atomicAdd(&a.done[e], 1u);
      s_last = (prev == parts - 1);
    }
    __syncthreads();
    if (s_last && packed) {
      if (tid == 0) {
        __threadfence();
        // read and reset the key in one atomic (all-ones = no candidate / the next call's start)
        const uint64_t key = atomicExch(reinterpret_cast<unsigned long long*>(a.keyslot + e), ~0ull);
        const Cand r = (key == kNone) ? Cand{kNone, kNone}
                                      : Cand{key >> a.ibits, key & ((1ull << a.ibits) - 1)};
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags, s_feas);
        a.done[e] = 0;
      }
    } else if (s_last) {
      __threadfence();
      Cand r{kNone, kNone};
      for (uint32_t t = tid; t < parts; t += nthr) {
        const volatile uint64_t* o = reinterpret_cast<const volatile uint64_t*>(&slots[t]);
        r = cand_min(r, Cand{o[0], o[1]});
      }
      r = block_min(r, red);
      if (tid == 0) {
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags, s_feas);
        a.done[e] = 0;  // self-reset for the next call
      }
    }
  }
  MCL_TRACE_AT(3);
  // fused cross-GPU exchange (NEXT-2): the last CTA reduces over every rank and decodes
  if (a.peer.world) peer_finish(a.peer, a.out, a.E, Q, D, a.ibits, a.flags, abandoned);
}

#ifdef MCL_TRACE
}  // namespace mcl
extern "C" int mcl_trace_read(unsigned long long* out, int n) {
  return (int)cudaMemcpyFromSymbol(out, mcl::g_mcl_trace, (size_t)n * 8 * sizeof(unsigned long long));
}
namespace mcl {
#endif

template <typename T, int D, bool L = false>
static cudaError_t launch_blocked_t(const BlockedArgs& a, dim3 grid, int threads, size_t smem,
                                   cudaStream_t st) {
  auto k = search_blocked_kernel<T, D, L>;
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
template <typename T, int D, bool L = false>
int occ_t(int threads, size_t smem) {
  // cache the last (threads, smem) query: the launch path asks the same question every call
  static std::atomic<uint64_t> last{0};
  const uint64_t key = ((uint64_t)threads << 40) | ((uint64_t)smem << 8);
  const uint64_t hit = last.load(std::memory_order_relaxed);
  if (hit && (hit & ~0xffull) == key) return (int)(hit & 0xff);
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, search_blocked_kernel<T, D, L>, threads, smem) !=
      cudaSuccess)
    return 1;
  n = n < 1 ? 1 : (n > 255 ? 255 : n);
  last.store(key | (uint64_t)n, std::memory_order_relaxed);
  return n;
}
}  // namespace

int blocked_ctas_per_sm(uint32_t D, bool wide, int threads, size_t smem, bool lean) {
#ifndef MCL_ONLY_D
  if (lean && !wide && D == 5) return occ_t<uint32_t, 5, true>(threads, smem);
#endif
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

bool blocked_lean_built(uint32_t D, bool wide) {
#ifndef MCL_ONLY_D
  return !wide && D == 5;
#else
  (void)D;
  (void)wide;
  return false;  // variant builds for one D compile no lean instantiation
#endif
}

cudaError_t launch_blocked(const BlockedArgs& a, bool wide, dim3 grid, int threads, size_t smem,
                           cudaStream_t st, bool lean) {
#ifndef MCL_ONLY_D
  if (lean && !wide && a.D == 5) return launch_blocked_t<uint32_t, 5, true>(a, grid, threads, smem, st);
#endif
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
