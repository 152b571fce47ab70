// search_bnb.cu -- exact search with pruning: the same lowest-index
// minimum-makespan mapping as the exhaustive kernels, reached by a
// parallel depth-first branch and bound instead of scoring every mapping. Its metric is
// time-to-solution, not mappings/s.
//
// The queue digits are assigned in index order (queue 0 first). A node at depth t holds
// the device loads L of queues 0..t-1 (on top of the base loads) and stands for the index
// range [lo, lo + D^(Q-t)). Three valid lower bounds on every completion's makespan:
//   max_d L_d                         (loads only grow),
//   Mx[t] = max_{q >= t} min_d C[q][d]  (every remaining queue runs somewhere),
//   ceil((sum_d L_d + S[t]) / D), S[t] = sum_{q >= t} min_d C[q][d]  (total work spread
//   perfectly) -- minima over each queue's eligible devices in constrained calls.
// A child is pruned when (LB, lo) >= the best (makespan, index) held so far, by this thread
// or by any thread of the epoch (shared as one packed key (ms << index_bits | index) through
// a global atomicMin; when the makespan cannot fit beside the index, only the makespan is
// shared and the global test becomes LB > ms): no mapping below it can beat what is already
// held, ties included. The lowest-index optimum m* is therefore never pruned (every node
// above it has (LB, lo) <= (ms*, m*)), and the final lexicographic reduction over all
// threads returns it.
//
// Work: the subtrees at depth k (D^k of them, about two per thread) are handed out in
// increasing index order by a per-epoch atomic counter. Every thread starts from the same
// incumbent: the greedy mapping (queue by queue onto the device with the least new load)
// improved by single-queue moves while they lower the makespan. Loads and digits live in
// per-thread local arrays (runtime device ids).
#include "common.cuh"
#include "kernels.h"

namespace mcl {

namespace {

struct Best {
  uint64_t ms, idx;
};

__device__ __forceinline__ bool lex_less(uint64_t a_ms, uint64_t a_idx, uint64_t b_ms, uint64_t b_idx) {
  return a_ms < b_ms || (a_ms == b_ms && a_idx < b_idx);
}

}  // namespace

__global__ void __launch_bounds__(128) search_bnb_kernel(BnbArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t Q = a.Q, D = a.D;
  const int nthr = blockDim.x, tid = threadIdx.x;
  // layout: C64[Q*D] | S[Q+1] | Mx[Q+1] | powD[Q+1] | red[32] Cand | elig[Q] u32
  uint64_t* C64 = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* S = C64 + Q * D;
  uint64_t* Mx = S + (Q + 1);
  uint64_t* powD = Mx + (Q + 1);
  Cand* red = reinterpret_cast<Cand*>(powD + (Q + 1));
  uint32_t* emask = reinterpret_cast<uint32_t*>(red + 32);
  __shared__ uint32_t s_status;
  __shared__ uint64_t s_base[kMaxDevices];
  __shared__ uint64_t s_feas, s_ub;
  __shared__ uint64_t s_start_ms, s_start_idx;
  __shared__ bool s_last;

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
    const uint16_t* elig_e = a.elig ? a.elig + e * Q : nullptr;
    if (tid < 32) {
      // base loads, range and feasibility checks (the INF masking it also applies is unused
      // here: the DFS skips ineligible devices outright, a true mixed-radix search)
      const uint64_t ub = epoch_prologue(C64, Q, D, a.base ? a.base + e * D : nullptr, elig_e,
                                         s_base, &s_status, &s_feas);
      if (tid == 0) s_ub = ub;
    }
    __syncthreads();
    if (s_status) {
      if (tid == 0 && blockIdx.x == 0) raise_flag(a.flags, s_status);
      continue;
    }
    if (tid == 0) {
      // eligible masks, suffix bounds S / Mx over each queue's eligible minimum, D powers
      for (uint32_t q = 0; q < Q; ++q) {
        const uint32_t m = elig_e ? (uint32_t)elig_e[q] : 0u;
        emask[q] = (m == 0) ? ((1u << D) - 1u) : (m & ((1u << D) - 1u));
      }
      S[Q] = 0;
      Mx[Q] = 0;
      for (int q = (int)Q - 1; q >= 0; --q) {
        uint64_t mn = kNone;
        for (uint32_t d = 0; d < D; ++d)
          if ((emask[q] >> d) & 1u) mn = min(mn, C64[q * D + d]);
        S[q] = S[q + 1] + mn;
        Mx[q] = max(Mx[q + 1], mn);
      }
      powD[0] = 1;
      for (uint32_t i = 1; i <= Q; ++i) powD[i] = powD[i - 1] * D;
      // starting incumbent: greedy (queue by queue onto the device with the least new
      // load), then single-queue moves while they lower the makespan
      uint64_t L[kMaxDevices];
      uint32_t g[kMaxQueues];
      for (uint32_t d = 0; d < D; ++d) L[d] = s_base[d];
      for (uint32_t q = 0; q < Q; ++q) {
        uint32_t bd = 0;
        uint64_t bv = kNone;
        for (uint32_t d = 0; d < D; ++d)
          if (((emask[q] >> d) & 1u) && L[d] + C64[q * D + d] < bv) {
            bv = L[d] + C64[q * D + d];
            bd = d;
          }
        L[bd] = bv;
        g[q] = bd;
      }
      for (int pass = 0; pass < 8; ++pass) {
        bool moved = false;
        for (uint32_t q = 0; q < Q; ++q) {
          uint64_t ms = 0;
          for (uint32_t d = 0; d < D; ++d) ms = max(ms, L[d]);
          const uint32_t from = g[q];
          for (uint32_t d = 0; d < D; ++d) {
            if (d == from || !((emask[q] >> d) & 1u)) continue;
            uint64_t nms = 0;
            for (uint32_t x = 0; x < D; ++x) {
              uint64_t lx = L[x];
              if (x == from) lx -= C64[q * D + from];
              if (x == d) lx += C64[q * D + d];
              nms = max(nms, lx);
            }
            if (nms < ms) {
              L[from] -= C64[q * D + from];
              L[d] += C64[q * D + d];
              g[q] = d;
              moved = true;
              break;
            }
          }
        }
        if (!moved) break;
      }
      uint64_t gms = 0, gidx = 0;
      for (uint32_t d = 0; d < D; ++d) gms = max(gms, L[d]);
      for (uint32_t q = 0; q < Q; ++q) gidx = gidx * D + g[q];
      s_start_ms = gms;
      s_start_idx = gidx;
    }
    __syncthreads();

    // The epoch's best so far, shared by every thread through one global word: the packed
    // key (makespan << index_bits | index) when every feasible makespan fits beside the
    // index, else the makespan alone (then ties at the bound are not pruned globally).
    const uint64_t feas_bound = elig_e ? s_feas : s_ub;
    const bool packed = (a.ibits == 0) || (feas_bound < (1ull << (64 - a.ibits)));
    const uint64_t imask = (a.ibits >= 64) ? ~0ull : ((1ull << a.ibits) - 1);
    auto pack = [&](uint64_t ms, uint64_t idx) { return packed ? ((ms << a.ibits) | idx) : ms; };
    volatile uint64_t* ginc = a.inc + e;
    uint64_t g_ms, g_idx;  // cached global incumbent (g_idx = kNone in makespan-only mode)
    auto refresh = [&]() {
      const uint64_t v = *ginc;
      const uint64_t ms = packed ? (v == kNone ? kNone : v >> a.ibits) : v;
      const uint64_t idx = packed ? (v == kNone ? kNone : v & imask) : kNone;
      if (lex_less(ms, idx, g_ms, g_idx)) {
        g_ms = ms;
        g_idx = idx;
      }
    };
    Best best{s_start_ms, s_start_idx};
    g_ms = best.ms;
    g_idx = packed ? best.idx : kNone;
    if (tid == 0) atomicMin((unsigned long long*)ginc, (unsigned long long)pack(best.ms, best.idx));
    refresh();
    // prune a node with bound lb covering indices >= lo: nothing below it can beat the
    // thread's own best or the shared one (makespan-only mode: strictly larger bounds only)
    auto prunable = [&](uint64_t lb, uint64_t lo) {
      if (!lex_less(lb, lo, best.ms, best.idx)) return true;
      return packed ? !lex_less(lb, lo, g_ms, g_idx) : (lb > g_ms);
    };
    auto leaf = [&](uint64_t ms, uint64_t idx) {
      if (lex_less(ms, idx, best.ms, best.idx)) {
        best = Best{ms, idx};
        if (lex_less(ms, packed ? idx : kNone, g_ms, g_idx)) {
          g_ms = ms;
          g_idx = packed ? idx : kNone;
          atomicMin((unsigned long long*)ginc, (unsigned long long)pack(ms, idx));
        }
      }
    };

    // ---- parallel DFS over the depth-k subtrees of this epoch ----
    const uint32_t k = a.k < Q ? a.k : Q;
    const uint64_t nsub = powD[k];
    uint64_t nodes = 0;
    uint64_t L[kMaxDevices];
    uint32_t dig[kMaxQueues];
    uint32_t cur[kMaxQueues + 1];
    uint64_t mxs[kMaxQueues + 1], sums[kMaxQueues + 1], pidx[kMaxQueues + 1];
    while (true) {
      const uint64_t s = atomicAdd((unsigned long long*)&a.next[e], 1ull);
      if (s >= nsub) break;
      refresh();
      // subtree root: the k digits of s (queue 0 most significant)
      for (uint32_t d = 0; d < D; ++d) L[d] = s_base[d];
      bool ok = true;
      uint64_t rest = s;
      for (int q = (int)k - 1; q >= 0; --q) {
        dig[q] = (uint32_t)(rest % D);
        rest /= D;
        if (!((emask[q] >> dig[q]) & 1u)) ok = false;
      }
      if (!ok) continue;
      uint64_t mx = 0, sum = 0;
      for (uint32_t q = 0; q < k; ++q) L[dig[q]] += C64[q * D + dig[q]];
      for (uint32_t d = 0; d < D; ++d) {
        mx = max(mx, L[d]);
        sum += L[d];
      }
      ++nodes;
      if (k == Q) {  // the subtree is a single mapping
        leaf(mx, s);
        continue;
      }
      if (prunable(max(max(mx, Mx[k]), (sum + S[k] + D - 1) / D), s * powD[Q - k])) continue;
      uint32_t t = k;
      mxs[t] = mx;
      sums[t] = sum;
      pidx[t] = s;
      cur[t] = 0;
      while (true) {
        // next eligible device for queue t
        uint32_t d = cur[t];
        while (d < D && !((emask[t] >> d) & 1u)) ++d;
        if (d >= D) {  // exhausted: back up one level and undo its assignment
          if (t == k) break;
          --t;
          L[dig[t]] -= C64[t * D + dig[t]];
          cur[t] = dig[t] + 1;
          continue;
        }
        cur[t] = d + 1;
        ++nodes;
        const uint64_t c = C64[t * D + d];
        const uint64_t nl = L[d] + c;
        const uint64_t nmx = max(mxs[t], nl);
        const uint64_t nsum = sums[t] + c;
        const uint64_t np = pidx[t] * D + d;
        if (t + 1 == Q) {  // a leaf: a complete mapping
          leaf(nmx, np);
          continue;
        }
        if ((nodes & 63) == 0) refresh();
        const uint64_t lb = max(max(nmx, Mx[t + 1]), (nsum + S[t + 1] + D - 1) / D);
        if (prunable(lb, np * powD[Q - t - 1])) continue;  // prune the child
        L[d] = nl;
        dig[t] = d;
        ++t;
        mxs[t] = nmx;
        sums[t] = nsum;
        pidx[t] = np;
        cur[t] = 0;
      }
    }
    if (a.nodes) atomicAdd((unsigned long long*)a.nodes, (unsigned long long)nodes);

    // ---- lexicographic (makespan, index) reduction: thread -> CTA -> epoch ----
    Cand c = block_min(Cand{best.ms, best.idx}, red);
    if (gridDim.x == 1) {
      if (tid == 0) {
        write_epoch(a.out, e, Q, D, a.ibits, c, a.flags);
        a.next[e] = 0;
        a.inc[e] = kNone;
      }
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
        write_epoch(a.out, e, Q, D, a.ibits, r, a.flags);
        a.done[e] = 0;  // self-reset for the next call
        a.next[e] = 0;
        a.inc[e] = kNone;
      }
    }
  }
}

size_t bnb_smem_bytes(uint32_t Q, uint32_t D) {
  size_t b = (size_t)Q * D * 8 + 3 * (size_t)(Q + 1) * 8 + 32 * sizeof(Cand) + (size_t)Q * 4;
  return (b + 15) & ~size_t(15);
}

cudaError_t launch_bnb(const BnbArgs& a, dim3 grid, int threads, cudaStream_t st) {
  const size_t smem = bnb_smem_bytes(a.Q, a.D);
  static SmemAttrCache cache;
  cudaError_t err = ensure_smem(search_bnb_kernel, smem, cache);
  if (err != cudaSuccess) return err;
  search_bnb_kernel<<<grid, threads, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace mcl
