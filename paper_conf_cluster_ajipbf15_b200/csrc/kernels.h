// kernels.h -- internal launch interface between the C-ABI host code (mcl.cpp) and the
// sm_100a kernels. Not part of the public ABI (that is include/mcl.h).
#pragma once
#include <atomic>
#include <cstddef>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

namespace mcl {

// Status bits written by kernels into the handle's host-mapped status word; mcl.cpp turns
// them into an mcl_status_t after the stream sync.
enum : uint32_t {
  kFlagRange = 1u,       // some cost entry or base load >= 2^48
  kFlagNeedU64 = 2u,     // some epoch's bound sum_q max_d C >= 2^32 - 1: rerun with 64-bit loads
  kFlagNoPack = 4u,      // makespan does not fit beside the index in one u64 key (NCCL path)
  kFlagInfeasible = 8u,  // constrained call: some queue has no eligible device below D
  kFlagBadMapping = 16u, // scoring call: a mapping names a device >= D
  kFlagBadModel = 32u,   // cost model: bad kernel id / source / offsets / curve
  kFlagPeerTimeout = 64u,  // fused exchange: some rank did not signal in time
  kFlagTwoStep = 128u,     // fused exchange ran the two-step reduction (informational)
  kFlagBadHint = 256u,     // static policy: a queue hint names a class >= num_classes
};

// Fused cross-GPU exchange (peer.cuh). Slab of each rank, in u64 words:
// [0] signal counter (every rank adds 1 per round), [1] rounds completed, [2] capacity (cap),
// [3, 8) unused,
// [8, 8 + cap) region 0, [8 + cap, 8 + 2 cap) region 1 (round R uses region R % 2).
constexpr uint64_t kPeerHeaderWords = 8;
struct PeerArgs {
  int world;               // 0 = exchange off
  uint64_t* const* slabs;  // [world] every rank's slab, mapped into this process (device array)
  uint64_t* mine;          // this rank's slab
  uint64_t cap;            // epochs per region
  uint32_t* kdone;         // [2]: CTAs of the kernel that finished, "some CTA abandoned its
                           // search" (input error / 64-bit rerun); zero on entry, self-resetting
  uint64_t* gms;           // [cap] scratch: global makespans of the two-step reduction
  uint64_t timeout_ns;
};

// Lexicographic (makespan, mapping index) candidate; see common.cuh.
struct Cand {
  uint64_t ms;
  uint64_t idx;
};

// Outputs of one launch, per epoch.
struct EpochOut {
  uint64_t* index;      // [E]
  uint64_t* makespan;   // [E]
  uint8_t* mapping;     // [E][Q] or nullptr
  uint64_t* key;        // [E] packed key for the cross-GPU reduce, or nullptr (single GPU)
  uint64_t* pair;       // [E][2] (ms, idx) for the two-step cross-GPU reduce, or nullptr
};

constexpr int kBlockedMaxD = 8;  // register-blocked kernel instantiated for D = 2..8

// Per-kernel, per-device cache of the dynamic shared-memory attribute already granted, so
// the hot launch path does not re-issue cudaFuncSetAttribute every call.
struct SmemAttrCache {
  std::atomic<size_t> granted[64];
  SmemAttrCache() {
    for (auto& g : granted) g.store(0);
  }
};

template <typename F>
cudaError_t ensure_smem(F* kernel, size_t smem, SmemAttrCache& cache) {
  int dev = 0;
  cudaGetDevice(&dev);
  std::atomic<size_t>& g = cache.granted[dev & 63];
  if (g.load(std::memory_order_relaxed) >= smem + 1) return cudaSuccess;
  // always set it: the default 48 KB cap also counts the kernel's static shared memory
  cudaError_t err = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err == cudaSuccess) g.store(smem + 1, std::memory_order_relaxed);
  return err;
}

// Integer tuning knob from the environment (read once by the caller), clamped to [lo, hi].
inline int env_int(const char* name, int dflt, int lo, int hi) {
  const char* v = getenv(name);
  if (!v || !*v) return dflt;
  const int x = atoi(v);
  return x < lo ? lo : (x > hi ? hi : x);
}

// Register-blocked search (search_blocked.cu).
struct BlockedArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  uint64_t rlo, rhi;  // this rank's block range [rlo, rhi), blocks of D^3 mappings
  uint64_t e_full;    // epochs 0..e_full-1 get one CTA each
  uint32_t tail_cpe;  // CTAs of each remaining epoch (1-D grid over the CTA index space)
  Cand* scratch;      // [E - e_full][tail_cpe] (split epochs only)
  uint32_t* done;     // [E], zero on entry, self-resetting
  EpochOut out;
  int ibits;
  volatile uint32_t* flags;
  uint32_t one;
  size_t off_red, off_dig;
  const uint64_t* base;  // [E][D] pre-existing device loads, or nullptr (constrained variant)
  const uint16_t* elig;  // [E][Q] eligible-device masks (0 = any), or nullptr
  PeerArgs peer;         // fused cross-GPU exchange (out.key / out.pair set), or world = 0
  int rank, world;       // mixed-radix kernel: shard of the reduced block space (world <= 1: all)
  uint64_t* keyslot;     // [E] packed (makespan, index) keys of split epochs: all ones on
                         // entry, self-resetting; nullptr = merge through scratch only
};

// ceil(log2(N)): bits of the packed key's index field (N >= 1).
inline int index_bits_host(uint64_t N) {
  int b = 0;
  while (b < 64 && ((N - 1) >> b)) ++b;
  return b;
}

bool blocked_supported(uint32_t Q, uint32_t D);
// whether launch_blocked(..., lean = true) runs a separate one-CTA-per-SM build for (D, wide)
bool blocked_lean_built(uint32_t D, bool wide);
// lean: the one-CTA-per-SM register budget where one exists (u32, D = 5; single epochs)
int blocked_ctas_per_sm(uint32_t D, bool wide, int threads, size_t smem, bool lean = false);
size_t blocked_smem_bytes(uint32_t Q, uint32_t D, bool wide, int threads, size_t* off_red,
                          size_t* off_dig);
// one-thread kernel spinning for `ns` nanoseconds of %globaltimer (timing aid, probe.cu)
cudaError_t launch_hold(uint64_t ns, cudaStream_t st);
cudaError_t probe_launch_floor(int sms, cudaStream_t st, int reps, double* empty_us, double* events_us);
cudaError_t launch_blocked(const BlockedArgs& a, bool wide, dim3 grid, int threads, size_t smem,
                           cudaStream_t st, bool lean = false);

// Constrained search over the feasible mappings only (search_mixed.cu, NEXT-3): pinned
// queues folded into the base loads, mixed-radix outer digits; same arguments and shared
// memory layout as the blocked kernel (rlo / rhi unused: the shard is a.rank / a.world of
// each epoch's reduced block space).
int mixed_ctas_per_sm(uint32_t D, bool wide, int threads, size_t smem);
// Batches of constrained epochs, one warp per epoch (u32 loads only; kFlagNeedU64 -> the
// 64-bit CTA kernel). grid_out: CTAs of kMixedWarps warps.
cudaError_t launch_mixed_warp(const BlockedArgs& a, int num_sms, cudaStream_t st, int* grid_out);
cudaError_t launch_mixed(const BlockedArgs& a, bool wide, dim3 grid, int threads, size_t smem,
                         cudaStream_t st);

// Batched epochs over a flattened (epoch, block) space (search_flat.cu): u32 loads, whole
// index space per epoch (no sharding), packed keys (index bits <= 32).
struct FlatArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  uint64_t nb;            // blocks of D^3 mappings per epoch
  int ibits;
  uint64_t* keys;         // [E], all ones on entry, self-resetting
  uint64_t* done_blocks;  // [E], zero on entry, self-resetting
  EpochOut out;
  volatile uint32_t* flags;
  uint32_t one;
};
bool flat_supported(uint32_t Q, uint32_t D, int ibits);
size_t flat_smem_bytes(uint32_t Q, uint32_t D);
cudaError_t launch_flat(const FlatArgs& a, int num_sms, cudaStream_t st, int* grid_out);

// Generic search (search_generic.cu): any Q <= 32, D <= 16, 64-bit loads.
struct GenericArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  uint64_t rlo, rhi;  // this rank's range in ROWS of D mappings (last digit varies in a row)
  Cand* scratch;
  uint32_t* done;
  EpochOut out;
  int ibits;
  volatile uint32_t* flags;
  const uint64_t* base;  // [E][D] or nullptr (constrained variant)
  const uint16_t* elig;  // [E][Q] or nullptr
  PeerArgs peer;         // as BlockedArgs::peer
};
size_t generic_smem_bytes(uint32_t Q, uint32_t D, int threads);

// Exact search with pruning (search_bnb.cu, NEXT-4): parallel depth-first branch and bound.
struct BnbArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  const uint64_t* base;  // [E][D] or nullptr
  const uint16_t* elig;  // [E][Q] or nullptr
  uint32_t k;            // subtree depth handed out by the per-epoch counter
  uint64_t* next;        // [E] subtree counters, zero on entry, self-resetting
  uint64_t* inc;         // [E] best (packed key or makespan) so far, all ones on entry, self-resetting
  uint64_t* nodes;       // nodes visited (accumulated), or nullptr
  Cand* scratch;         // [E][cpe]
  uint32_t* done;        // [E]
  EpochOut out;
  int ibits;
  volatile uint32_t* flags;
};
size_t bnb_smem_bytes(uint32_t Q, uint32_t D);
cudaError_t launch_bnb(const BnbArgs& a, dim3 grid, int threads, cudaStream_t st);

// Cost-table construction (costs.cu, NEXT-1).
struct CostArgs {
  uint32_t D;
  uint64_t EQ;                // epochs x queues
  uint32_t num_kernels;
  const uint64_t* profile;    // [num_kernels][D]
  const uint64_t* offsets;    // [EQ + 1]
  const uint32_t* ids;        // [nnz]
  uint64_t nnz;
  const uint64_t* bytes;      // [EQ]
  const int32_t* source;      // [EQ]
  const uint16_t* cached;     // [EQ] or nullptr
  uint32_t M;
  const uint64_t* sizes;      // [M]
  uint32_t S;                 // host sockets (>= 1)
  const uint8_t* host_socket; // [EQ] or nullptr (socket 0)
  const double* h2d;          // [S][D][M]
  const double* d2h;          // [S][D][M]
  uint32_t host_shared;
  uint64_t* K;                // [EQ][D] out
  uint64_t* X;                // [EQ][D] out
  volatile uint32_t* flags;
};
cudaError_t launch_build_costs(const CostArgs& a, int num_sms, cudaStream_t st);

// Scoring of given mappings (score.cu): makespan[e] of mapping[e][.] with optional base
// loads; a device id >= D raises kFlagBadMapping.
cudaError_t launch_score(uint32_t Q, uint32_t D, uint64_t E, const uint64_t* K, const uint64_t* X,
                         const uint64_t* base, const uint8_t* mapping, uint64_t* makespan,
                         volatile uint32_t* flags, cudaStream_t st);
cudaError_t launch_generic(const GenericArgs& a, dim3 grid, int threads, size_t smem,
                           cudaStream_t st);
// Static hint-based mappings (score.cu, SCHED_AUTO_STATIC): per (epoch, queue) the eligible
// device with the lowest device-profile cost of the queue's class.
cudaError_t launch_static_map(uint32_t Q, uint32_t D, uint64_t E, const uint8_t* hints,
                              uint32_t num_classes, const uint64_t* score, const uint16_t* elig,
                              uint8_t* mapping, volatile uint32_t* flags, cudaStream_t st);

// Batched search, one warp per epoch, compile-time (Q, D) (search_batch.cu): u32 loads,
// unconstrained, single GPU, shapes with >= ~32 chunks of D^2 blocks per epoch.
struct BatchArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  uint64_t* index;
  uint64_t* makespan;
  uint8_t* mapping;
  volatile uint32_t* flags;
  uint32_t one;
  uint64_t e_full;    // set by launch_batch: epochs searched by one warp (whole waves)
  bool host_inputs;   // K / X are pinned host memory read in place (zero-copy): the
                      // warp-per-epoch form, whose per-warp prefetch hides PCIe latency
};
bool batch_supported(uint32_t Q, uint32_t D);
// *pooled = true when the SM-pooled form ran (one 16-warp CTA per SM, sub-epoch parts)
cudaError_t launch_batch(const BatchArgs& a, int num_sms, cudaStream_t st, int* grid_out, bool* pooled);

// Small batched search (search_small.cu): one thread per epoch, tiles staged in shared
// memory by cp.async.bulk (TMA bulk copy). Instantiated for a few (Q, D) shapes.
struct SmallArgs {
  uint32_t Q, D;
  uint64_t E;
  const uint64_t* K;
  const uint64_t* X;
  uint64_t* index;
  uint64_t* makespan;
  uint8_t* mapping;
  volatile uint32_t* flags;
};
bool small_supported(uint32_t Q, uint32_t D);
cudaError_t launch_small(const SmallArgs& a, int num_sms, cudaStream_t st, int* grid_out,
                         int* threads_out);

// Multi-GPU epilogues (reduce.cu).
cudaError_t launch_decode_key(const uint64_t* key, uint64_t E, uint32_t Q, uint32_t D, int ibits,
                              uint64_t* index, uint64_t* makespan, uint8_t* mapping,
                              volatile uint32_t* flags, cudaStream_t st);
cudaError_t launch_pair_candidates(const uint64_t* pair, const uint64_t* gms, uint64_t E,
                                   uint64_t* cand, cudaStream_t st);
cudaError_t launch_decode_pair(const uint64_t* gms, const uint64_t* gidx, uint64_t E, uint32_t Q,
                               uint32_t D, uint64_t* index, uint64_t* makespan, uint8_t* mapping,
                               cudaStream_t st);
cudaError_t launch_extract_ms(const uint64_t* pair, uint64_t E, uint64_t* ms, cudaStream_t st);

// Resident mapper (resident.cu): one warp serving decisions from a mailbox in pinned,
// device-mapped host memory. Control words each on their own 64-byte line; the data
// arrays follow the header in the same allocation (ResidentArgs holds their device aliases).
struct ResidentBox {
  uint64_t req;          // host -> device, written after the inputs: request number (bits
                         // 0-31) | epochs (bits 32-47) | stop (bit 63)
  uint32_t pad0[14];
  uint32_t done_seq;     // (unused: every result record carries its request's tag)
  uint32_t status;       // (unused)
  uint32_t alive;        // 1 while the warp runs
  uint32_t exit_reason;  // 1 stop, 2 idle timeout
  uint32_t pad1[2];
  uint64_t trace[5];     // -DMCL_RESIDENT_TRACE builds: %globaltimer at request seen, inputs
                         // read, scored, results published
  uint32_t pad2[16];
};
static_assert(sizeof(ResidentBox) == 192, "three 64-byte lines");
constexpr uint32_t kResidentMaxMappings = 8192;  // D^Q per epoch (13 index bits: the paper's
                                                 // largest decision, FT's 8 queues x 3 devices = 6561)
constexpr uint32_t kResidentMaxQ = 16, kResidentMaxD = 16;
// Result record of one epoch, three u64 words each written whole by one store (single-copy
// atomic at system scope), each tagged with the request number so the host accepts a
// record only when all three words are this request's -- no fence before a done flag:
//   w0 = seq << 32 | status << 16 | index (< 4096)
//   w1 = (seq mod 2^11) << 53 | makespan (< 2^53)
//   w2 = seq << 32 | digits (queue q's device in bits [q*b, q*b + b), b = bits of D - 1)
constexpr int kResidentRecWords = 3;
struct ResidentArgs {
  ResidentBox* box;           // device alias of the mailbox
  const uint64_t* K;          // [cap][Q][D] device aliases of the mailbox arrays
  const uint64_t* X;
  uint64_t* rec;              // [cap][3] result records
  uint32_t Q, D, N, cap;
  uint32_t seq0;              // request number already served when the warp starts
  uint64_t idle_ns;
};
cudaError_t launch_resident(const ResidentArgs& a, cudaStream_t st);

// ALU throughput probe (probe.cu), SURVEY N7.
cudaError_t probe_alu(int op, int sms, cudaStream_t st, double* lane_ops_per_s,
                      double* lane_ops_per_clk_sm, double* eff_mhz);

}  // namespace mcl
