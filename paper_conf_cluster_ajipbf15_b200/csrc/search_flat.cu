// search_flat.cu -- batched epochs over a FLATTENED (epoch, block) work space (SURVEY SS8(a)
// a8: the mapper runs once per scheduling epoch).
//
// With one CTA per epoch, E equal-sized epochs quantise into ceil(E / resident CTAs) waves
// (cfg2: 10^4 epochs over 2368 resident warps = 4.2 -> 5 waves, 16 % idle). Here a
// persistent grid of one-warp CTAs cuts the E x nb blocks into equal contiguous segments
// (chunk-aligned so lanes stay in lock-step); a segment crosses epoch boundaries, so a warp
// scores one or more epoch PIECES. Per piece the warp builds the epoch's tables in shared
// memory, every lane walks its sub-range with the register-blocked leaf evaluation of
// blocked_core.cuh, the warp argmin's winner re-scans its best block, and the piece's
// candidate is merged into the epoch's packed key (makespan << index_bits | index) with one
// atomicMin -- lexicographic because the key packs (makespan, index). The warp that
// completes an epoch's block count decodes the key, writes the outputs and resets the
// epoch's key and counter for the next call.
#include "blocked_core.cuh"

namespace mcl {

template <typename T, int D>
__global__ void __launch_bounds__(32, (D <= 5) ? 16 : 8) search_flat_kernel(FlatArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q;
  const int O = (int)Q - 3;
  const int lane = threadIdx.x;
  // layout: C64[Q*D] u64 | in[8*D] T | V[O*D*D] T | dig[(O-1)*32] u8
  uint64_t* C64 = reinterpret_cast<uint64_t*>(smem_raw);
  T* in = reinterpret_cast<T*>(C64 + Q * D);
  T* V = in + 8 * D;
  uint8_t* dig = reinterpret_cast<uint8_t*>(V + (size_t)(O > 0 ? O : 0) * D * D);
  __shared__ __align__(16) T zero[D];
  if (lane < D) zero[lane] = 0;
  constexpr bool kSuper = (sizeof(T) == 4 && D <= kSuperMaxD);
  const uint64_t chunk = (kSuper && O >= 2) ? (uint64_t)D * D : 1;
  const uint64_t nb = a.nb;

  // this warp's chunk-aligned segment of the flattened [0, E * nb) block space
  const uint64_t W = a.E * nb;
  const uint64_t nw = gridDim.x, w = blockIdx.x;
  auto split = [&](uint64_t t) -> uint64_t {
    if (t >= nw) return W;
    const uint64_t per = W / nw, rem = W % nw;
    // align to 32 chunks (one per lane) where an epoch holds that many, so every piece
    // keeps all lanes busy; otherwise to single chunks
    const uint64_t unit = (nb % (32 * chunk) == 0) ? 32 * chunk : chunk;
    return (t * per + (t < rem ? t : rem)) / unit * unit;
  };
  uint64_t f = split(w);
  const uint64_t fend = split(w + 1);
  const WalkCtx<T, D> wctx{in, V, zero, zero, dig, O, 32, lane, a.one};  // no base loads

  while (f < fend) {
    const uint64_t e = f / nb;
    const uint64_t b_lo = f % nb;
    const uint64_t len = (nb - b_lo < fend - f) ? nb - b_lo : fend - f;
    f += len;
    // ---- a1: tables of epoch e (composition, range check, 32-bit bound) ----
    __syncwarp();
    const uint64_t* Ke = a.K + e * Q * D;
    const uint64_t* Xe = a.X + e * Q * D;
    bool bad = false;
    for (uint32_t t = lane; t < Q * D; t += 32) {
      const uint64_t k = Ke[t], x = Xe[t];
      bad |= (k >= kEntryLimit) | (x >= kEntryLimit);
      C64[t] = k + x;
    }
    __syncwarp();
    if (__any_sync(0xffffffffu, bad)) {
      if (lane == 0) raise_flag(a.flags, kFlagRange);
      continue;
    }
    uint64_t part = 0;
    for (uint32_t q = lane; q < Q; q += 32) {
      uint64_t m = 0;
      for (int d = 0; d < D; ++d) m = max2(m, C64[q * D + d]);
      part += m;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) part += __shfl_xor_sync(0xffffffffu, part, off);
    // UB < 2^32 - 1 keeps every makespan below the all-ones start of the running minima
    if (sizeof(T) == 4 && part >= 0xffffffffull) {
      if (lane == 0) raise_flag(a.flags, kFlagNeedU64);
      continue;
    }
    for (int t = lane; t < D; t += 32) {
      const uint64_t A = C64[(Q - 3) * D + t], B = C64[(Q - 2) * D + t], Cc = C64[(Q - 1) * D + t];
      in[0 * D + t] = (T)A;
      in[1 * D + t] = (T)B;
      in[2 * D + t] = (T)Cc;
      in[3 * D + t] = (T)(A + B);
      in[4 * D + t] = (T)(A + Cc);
      in[5 * D + t] = (T)(B + Cc);
      in[6 * D + t] = (T)(A + B + Cc);
      in[7 * D + t] = (O >= 1) ? (T)C64[(O - 1) * D + t] : (T)0;
    }
    for (int t = lane; t < O * D * D; t += 32) {
      const int q = t / (D * D), x = (t / D) % D, d = t % D;
      V[t] = (d == x) ? (T)C64[q * D + x] : (T)0;
    }
    __syncwarp();

    // ---- a2-a4: each lane walks a chunk-aligned sub-range of the piece ----
    const uint64_t nc = (len + chunk - 1) / chunk;
    const uint64_t c_lo = nc * lane / 32, c_hi = nc * (lane + 1) / 32;
    const uint64_t s0 = b_lo + c_lo * chunk;
    const uint64_t s1 = (b_lo + c_hi * chunk < b_lo + len) ? b_lo + c_hi * chunk : b_lo + len;
    T best = ~T(0);
    uint64_t best_blk = kNone;
    uint32_t best_span = 1;
    if (s1 > s0) walk_blocks<T, D>(wctx, s0, s1 - s0, best, best_blk, best_span);

    // ---- a5: warp argmin; lanes ascend with the index, so the lowest lane holding the
    // minimum owns the piece's lowest-index optimum and alone re-scans its best block ----
    const uint64_t bv = (best_blk != kNone) ? (uint64_t)best : kNone;
    uint64_t wmin = bv;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) wmin = min(wmin, __shfl_xor_sync(0xffffffffu, wmin, off));
    const uint32_t holders = __ballot_sync(0xffffffffu, bv != kNone && bv == wmin);
    if (!holders) continue;
    const int wl = __ffs(holders) - 1;
    const uint64_t bb = __shfl_sync(0xffffffffu, best_blk, wl);
    const uint32_t span = __shfl_sync(0xffffffffu, best_span, wl);
    const uint64_t idx = span_first_warp<T, D>(bb, span, O, V, zero, in, (T)wmin, a.one);
    if (lane == wl) {
      atomicMin((unsigned long long*)&a.keys[e], (unsigned long long)((bv << a.ibits) | idx));
      __threadfence();
      // the warp that completes the epoch's block count publishes its result
      const uint64_t before = atomicAdd((unsigned long long*)&a.done_blocks[e], (unsigned long long)len);
      if (before + len == nb) {
        __threadfence();
        const uint64_t key = atomicMax((unsigned long long*)&a.keys[e], 0ull);  // coherent read
        const uint64_t mask = (a.ibits >= 64) ? ~0ull : ((1ull << a.ibits) - 1);
        const Cand c{key >> a.ibits, key & mask};
        a.out.index[e] = c.idx;
        a.out.makespan[e] = c.ms;
        if (a.out.mapping) {
          uint64_t rest = c.idx;
          for (int q = (int)Q - 1; q >= 0; --q) {
            a.out.mapping[e * Q + (uint64_t)q] = (uint8_t)(rest % D);
            rest /= D;
          }
        }
        a.keys[e] = kNone;  // self-reset for the next call
        a.done_blocks[e] = 0;
      }
    }
  }
}

size_t flat_smem_bytes(uint32_t Q, uint32_t D) {
  const int O = (int)Q - 3;
  size_t b = (size_t)Q * D * 8 + 8 * D * 4 + (size_t)(O > 0 ? O : 0) * D * D * 4 +
             (size_t)(O > 1 ? O - 1 : 0) * 32;
  return (b + 15) & ~size_t(15);
}

bool flat_supported(uint32_t Q, uint32_t D, int ibits) {
  return Q >= 3 && D >= 2 && D <= kBlockedMaxD && ibits <= 32;
}

namespace {
template <int D>
cudaError_t launch_flat_t(const FlatArgs& a, int num_sms, cudaStream_t st, int* grid_out) {
  auto k = search_flat_kernel<uint32_t, D>;
  const size_t smem = flat_smem_bytes(a.Q, D);
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(k, smem, cache);
  if (err != cudaSuccess) return err;
  static std::atomic<uint64_t> last{0};  // cached (smem << 8 | CTAs per SM)
  int per_sm = 0;
  const uint64_t hit = last.load(std::memory_order_relaxed);
  if (hit && (hit >> 8) == smem) {
    per_sm = (int)(hit & 0xff);
  } else {
    err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, 32, smem);
    if (err != cudaSuccess) return err;
    per_sm = per_sm < 1 ? 1 : (per_sm > 255 ? 255 : per_sm);
    last.store(((uint64_t)smem << 8) | (uint64_t)per_sm, std::memory_order_relaxed);
  }
  // no more warps than there are chunks of work
  uint64_t grid = (uint64_t)num_sms * per_sm;
  const uint64_t work = a.E * a.nb;
  if (grid > work) grid = work;
  k<<<(unsigned)grid, 32, smem, st>>>(a);
  *grid_out = (int)grid;
  return cudaGetLastError();
}
}  // namespace

cudaError_t launch_flat(const FlatArgs& a, int num_sms, cudaStream_t st, int* grid_out) {
  switch (a.D) {
    case 2: return launch_flat_t<2>(a, num_sms, st, grid_out);
    case 3: return launch_flat_t<3>(a, num_sms, st, grid_out);
    case 4: return launch_flat_t<4>(a, num_sms, st, grid_out);
    case 5: return launch_flat_t<5>(a, num_sms, st, grid_out);
    case 6: return launch_flat_t<6>(a, num_sms, st, grid_out);
    case 7: return launch_flat_t<7>(a, num_sms, st, grid_out);
    case 8: return launch_flat_t<8>(a, num_sms, st, grid_out);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace mcl
