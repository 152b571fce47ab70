// mcl.cpp -- host side of libmcl.so: the C ABI of include/mcl.h and include/mcl_ext.h.
//
// Validation, pointer classification (device buffers are used in place, host buffers are
// staged through handle-owned device memory), kernel selection, the shard range of this
// rank, the cross-GPU all-reduce (NCCL resolved at run time with dlopen, so the library
// has no link-time NCCL dependency and reuses the copy torch already loaded), and the
// status word the kernels raise (host-mapped pinned memory, read after the stream sync).
//
// There is no CPU fallback: every mapping is scored by the CUDA kernels in this library;
// without a usable CUDA device mcl_mapper_create fails with MCL_E_CUDA.
#include <dlfcn.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <cuda_runtime.h>
#include <nccl.h>

#include "../../include/mcl.h"
#include "../../include/mcl_ext.h"
#include "kernels.h"

namespace {

using mcl::Cand;

// ---------------------------------------------------------------- NCCL (dlopen) -------
struct NcclApi {
  bool ok = false;
  std::string err;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
  ncclResult_t (*CommUserRank)(const ncclComm_t, int*) = nullptr;
};

NcclApi load_nccl() {
  NcclApi api;
  void* lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // torch's copy, if loaded
  if (!lib) lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!lib) lib = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!lib) {
    const char* e = dlerror();
    api.err = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
    return api;
  }
#define MCL_SYM(field, name)                                                   \
  api.field = reinterpret_cast<decltype(api.field)>(dlsym(lib, name));         \
  if (!api.field) {                                                            \
    api.err = std::string("libnccl is missing ") + name;                       \
    return api;                                                                \
  }
  MCL_SYM(AllReduce, "ncclAllReduce")
  MCL_SYM(GetErrorString, "ncclGetErrorString")
  MCL_SYM(GetUniqueId, "ncclGetUniqueId")
  MCL_SYM(CommInitRank, "ncclCommInitRank")
  MCL_SYM(CommDestroy, "ncclCommDestroy")
  MCL_SYM(CommCount, "ncclCommCount")
  MCL_SYM(CommUserRank, "ncclCommUserRank")
#undef MCL_SYM
  api.ok = true;
  return api;
}

NcclApi& nccl() {
  static NcclApi api = load_nccl();
  return api;
}

thread_local std::string g_create_err;

// ---------------------------------------------------------------- device buffers ------
struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t bytes, bool zero = false) {
    if (bytes <= cap) return cudaSuccess;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    size_t want = std::max<size_t>(bytes, 256);
    cudaError_t e = cudaMalloc(&p, want);
    if (e != cudaSuccess) return e;
    cap = want;
    if (zero) return fill(0);
    return cudaSuccess;
  }
  // Fill the whole buffer before any later launch can read it: the memset runs on the
  // legacy stream, which a non-blocking stream (the handle's, or torch's) does not wait
  // for, so the device is synchronised here (buffers grow rarely; not on the hot path).
  cudaError_t fill(int byte) {
    cudaError_t e = cudaMemset(p, byte, cap);
    if (e != cudaSuccess) return e;
    return cudaDeviceSynchronize();
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
};

// mcl_map_queues_pruned scores small index spaces exhaustively (measured crossover)
constexpr uint64_t kPrunedMinMappings = 1ull << 24;

bool mul_overflow_pow(uint32_t D, uint32_t Q, uint64_t limit, uint64_t* out) {
  uint64_t n = 1;
  for (uint32_t q = 0; q < Q; ++q) {
    if (n > limit / D) return true;
    n *= D;
  }
  *out = n;
  return false;
}

}  // namespace

struct mcl_mapper {
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  ncclComm_t comm = nullptr;
  int rank = 0, world = 1;
  int num_sms = 148;
  DevBuf scratch;          // Cand per (epoch, CTA) when an epoch spans several CTAs
  DevBuf keyslot;          // packed-key merge slot per epoch (all ones between calls)
  DevBuf done;             // uint32 per epoch, zero between calls
  DevBuf key, pair, gms, cand;
  DevBuf flat_keys, flat_done;  // flattened batched kernel: per-epoch key / block count
  DevBuf bnb_next, bnb_inc, bnb_nodes;  // pruned search: subtree counters, incumbents, nodes
  DevBuf model_buf[10], cost_k, cost_x;  // cost-table construction: staged model, built K / X
  DevBuf in_k, in_x, in_base, in_elig, out_idx, out_ms, out_map;  // staging for host pointers
  // fused peer exchange (NEXT-2): own slab, kernel CTA counter, two-step scratch, and the
  // device array of every rank's slab address (peers' slabs opened through CUDA IPC)
  DevBuf peer_slab, peer_kdone, peer_gms, peer_ptrs;
  std::vector<void*> peer_opened;
  uint64_t peer_cap = 0;
  uint64_t peer_timeout_ns = 0;
  bool peer_ready = false;
  bool peer_configured = false;  // slabs were imported (cleared only by a new export)
  uint32_t* flags_host = nullptr;               // host-mapped status word
  uint32_t* flags_dev = nullptr;
  int timing = 0;               // 0 off, 1 search kernel, 2 search kernel + whole call
  uint32_t hold_us = 0;         // timing aid: spin kernel ahead of the start event
  bool timing_pending = false;  // events recorded, elapsed times not read yet
  int force_path = 0;
  int pipeline_chunks = 0;      // 0 auto, 1 off, n forced (mcl_set_pipeline_chunks)
  bool async_call = false;      // pipelined chunk: enqueue only (the wrapper syncs, reads flags)
  bool zero_copy = false;       // this call may use pinned host buffers in place (small call)
  // pipelined staging: pipe[0] host->device copies, pipe[1] the searches (one stream, so
  // chunk kernels never run concurrently and share the handle's scratch safely), pipe[2]
  // device->host copies; pipe_ev = start + per-stream join, chunk_ev = per-chunk hand-offs
  cudaStream_t pipe[3] = {nullptr, nullptr, nullptr};
  cudaEvent_t pipe_ev[4] = {nullptr, nullptr, nullptr, nullptr};
  std::vector<cudaEvent_t> chunk_ev;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  int64_t info[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  std::string last_err;
  // resident mapper (mcl_resident_*): mailbox in pinned, mapped host memory, the warp's
  // own stream, its launch arguments (device aliases) and the last request number
  unsigned char* res_mem = nullptr;
  cudaStream_t res_stream = nullptr;
  mcl::ResidentArgs res_args{};
  uint32_t res_seq = 0;
  bool res_started = false;
};

namespace {

mcl_status_t cuda_fail(mcl_mapper* h, cudaError_t e, const char* what) {
  std::string msg = std::string(what) + ": " + cudaGetErrorString(e);
  if (h) h->last_err = msg; else g_create_err = msg;
  return (e == cudaErrorMemoryAllocation) ? MCL_E_NOMEM : MCL_E_CUDA;
}

mcl_status_t nccl_fail(mcl_mapper* h, ncclResult_t r, const char* what) {
  h->last_err = std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "?");
  return MCL_E_NCCL;
}

#define MCL_CUDA(h, expr, what)                      \
  do {                                               \
    cudaError_t _e = (expr);                         \
    if (_e != cudaSuccess) return cuda_fail(h, _e, what); \
  } while (0)

// Is `p` usable in place by kernels on h->device? *dptr receives the address kernels use.
// Pinned (page-locked, mapped) host memory is used in place -- zero-copy over PCIe -- when
// the call is small (h->zero_copy, set per call by map_impl): one launch that reads its
// few hundred bytes of inputs and writes its outputs over the bus instead of 2 H2D + 3 D2H
// copies, each a separate runtime call (cfg1 host-buffer call 36 -> ~16 us). Larger pinned
// batches and pageable memory are staged (pipelined copy engines beat PCIe zero-copy there).
mcl_status_t classify(mcl_mapper* h, const void* p, bool* on_device, const void** dptr = nullptr,
                      bool* in_place_host = nullptr) {
  if (in_place_host) *in_place_host = false;
  cudaPointerAttributes at;
  cudaError_t e = cudaPointerGetAttributes(&at, p);
  if (e != cudaSuccess) {  // CUDA >= 11 reports unregistered host memory as success
    cudaGetLastError();
    h->last_err = std::string("cannot classify a buffer pointer: ") + cudaGetErrorString(e);
    return MCL_E_INVAL;
  }
  if (dptr) *dptr = p;
  if (at.type == cudaMemoryTypeDevice) {
    if (at.device != h->device) {
      h->last_err = "device pointer belongs to another CUDA device";
      return MCL_E_INVAL;
    }
    *on_device = true;
  } else if (at.type == cudaMemoryTypeManaged) {
    *on_device = true;
  } else if (at.type == cudaMemoryTypeHost && h->zero_copy && at.devicePointer) {
    *on_device = true;  // pinned host memory, small call: zero-copy
    if (dptr) *dptr = at.devicePointer;
    if (in_place_host) *in_place_host = true;
  } else {
    *on_device = false;  // pageable or (large call) pinned host memory: staged
  }
  return MCL_OK;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

// Shard [0, units) of every epoch into `world` contiguous ranges; this rank's range.
void shard(uint64_t units, int rank, int world, uint64_t* lo, uint64_t* hi) {
  if (world <= 1) {
    *lo = 0;
    *hi = units;
    return;
  }
  // exact floor(r * units / world) without overflow (units <= 2^48, world <= 2^15)
  *lo = (uint64_t)(((__uint128_t)units * rank) / world);
  *hi = (uint64_t)(((__uint128_t)units * (rank + 1)) / world);
}

// CTAs per epoch and threads per CTA for `units` work units per epoch in this rank.
void size_grid(mcl_mapper* h, uint64_t E, uint64_t units, int ctas_per_sm, int threads,
               dim3* grid) {
  const uint64_t slots = (uint64_t)h->num_sms * std::max(1, ctas_per_sm);
  uint64_t cpe = 1;
  if (E < slots) {
    cpe = (slots + E - 1) / E;
    const uint64_t useful = std::max<uint64_t>(1, (units + threads - 1) / threads);
    cpe = std::min(cpe, useful);
    if (cpe > 65535) cpe = 65535;
  }
  grid->x = (unsigned)cpe;
  grid->y = (unsigned)std::min<uint64_t>(E, 65535);
  grid->z = 1;
}

}  // namespace

extern "C" {

const char* mcl_version(void) { return "mcl 0.1 sm_100a"; }

const char* mcl_status_string(mcl_status_t s) {
  switch (s) {
    case MCL_OK: return "MCL_OK: success";
    case MCL_E_INVAL: return "MCL_E_INVAL: invalid argument";
    case MCL_E_RANGE: return "MCL_E_RANGE: D^Q > 2^48 or a cost entry >= 2^48";
    case MCL_E_CUDA: return "MCL_E_CUDA: CUDA runtime error";
    case MCL_E_NCCL: return "MCL_E_NCCL: NCCL error";
    case MCL_E_NOMEM: return "MCL_E_NOMEM: out of memory";
  }
  return "unknown mcl status";
}

const char* mcl_last_error_string(const mcl_mapper_t* h) {
  return h ? h->last_err.c_str() : g_create_err.c_str();
}

mcl_status_t mcl_mapper_create(const mcl_config_t* cfg, mcl_mapper_t** out) {
  g_create_err.clear();
  if (!cfg || !out) return MCL_E_INVAL;
  *out = nullptr;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaGetDeviceCount");
  if (cfg->device < 0 || cfg->device >= ndev) {
    g_create_err = "device ordinal out of range";
    return MCL_E_INVAL;
  }
  const int world = cfg->world <= 0 ? 1 : cfg->world;
  if (cfg->rank < 0 || cfg->rank >= world || world > 32768) {
    g_create_err = "rank/world out of range";
    return MCL_E_INVAL;
  }
  if (cfg->nccl_comm) {
    if (!nccl().ok) {
      g_create_err = nccl().err;
      return MCL_E_NCCL;
    }
    int n = 0, r = 0;
    if (nccl().CommCount((ncclComm_t)cfg->nccl_comm, &n) != ncclSuccess ||
        nccl().CommUserRank((ncclComm_t)cfg->nccl_comm, &r) != ncclSuccess) {
      g_create_err = "invalid NCCL communicator";
      return MCL_E_NCCL;
    }
    if (n != world || r != cfg->rank) {
      g_create_err = "rank/world do not match the NCCL communicator";
      return MCL_E_INVAL;
    }
  }
  DeviceGuard g(cfg->device);
  mcl_mapper* h = new mcl_mapper();
  h->device = cfg->device;
  h->comm = (ncclComm_t)cfg->nccl_comm;
  h->rank = cfg->rank;
  h->world = world;
  auto fail = [&](cudaError_t err, const char* what) {
    mcl_status_t s = cuda_fail(nullptr, err, what);
    mcl_mapper_destroy(h);
    return s;
  };
  e = cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, h->device);
  if (e != cudaSuccess) return fail(e, "cudaDeviceGetAttribute");
  if (cfg->stream) {
    h->stream = (cudaStream_t)cfg->stream;
  } else {
    e = cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) return fail(e, "cudaStreamCreate");
    h->own_stream = true;
  }
  e = cudaHostAlloc((void**)&h->flags_host, 64, cudaHostAllocMapped);
  if (e != cudaSuccess) return fail(e, "cudaHostAlloc(flags)");
  std::memset(h->flags_host, 0, 64);
  e = cudaHostGetDevicePointer((void**)&h->flags_dev, h->flags_host, 0);
  if (e != cudaSuccess) return fail(e, "cudaHostGetDevicePointer");
  for (auto& ev : h->ev) {
    e = cudaEventCreate(&ev);
    if (e != cudaSuccess) return fail(e, "cudaEventCreate");
  }
  e = h->done.ensure(4096 * sizeof(uint32_t), true);
  if (e != cudaSuccess) return fail(e, "cudaMalloc(done)");
  *out = h;
  return MCL_OK;
}

void mcl_mapper_destroy(mcl_mapper_t* h) {
  if (!h) return;
  mcl_resident_stop(h);
  {
    DeviceGuard g(h->device);
    if (h->stream) cudaStreamSynchronize(h->stream);
    for (void* p : h->peer_opened) cudaIpcCloseMemHandle(p);
    for (DevBuf* b : {&h->peer_slab, &h->peer_kdone, &h->peer_gms, &h->peer_ptrs}) b->release();
    for (DevBuf* b : {&h->scratch, &h->keyslot, &h->done, &h->key, &h->pair, &h->gms, &h->cand, &h->flat_keys,
                      &h->flat_done, &h->bnb_next, &h->bnb_inc, &h->bnb_nodes, &h->in_k,
                      &h->in_base, &h->in_elig,
                      &h->in_x, &h->out_idx, &h->out_ms, &h->out_map, &h->cost_k, &h->cost_x})
      b->release();
    for (DevBuf& b : h->model_buf) b.release();
    if (h->flags_host) cudaFreeHost(h->flags_host);
    for (auto& ev : h->ev)
      if (ev) cudaEventDestroy(ev);
    for (cudaStream_t& ps : h->pipe)
      if (ps) cudaStreamSynchronize(ps), cudaStreamDestroy(ps);
    for (cudaEvent_t& pe : h->pipe_ev)
      if (pe) cudaEventDestroy(pe);
    for (cudaEvent_t& ce : h->chunk_ev) cudaEventDestroy(ce);
    if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  }
  delete h;
}

mcl_status_t mcl_last_launch_info(const mcl_mapper_t* h, int64_t info[8]) {
  if (!h || !info) return MCL_E_INVAL;
  for (int i = 0; i < 8; ++i) info[i] = h->info[i];
  return MCL_OK;
}

mcl_status_t mcl_set_timing_hold(mcl_mapper_t* h, uint32_t hold_us) {
  if (!h || hold_us > 1000000u) return MCL_E_INVAL;
  h->hold_us = hold_us;
  return MCL_OK;
}

mcl_status_t mcl_set_timing(mcl_mapper_t* h, int enable) {
  if (!h) return MCL_E_INVAL;
  if (enable < 0 || enable > 2) return MCL_E_INVAL;
  h->timing = enable;
  h->timing_pending = false;
  return MCL_OK;
}

mcl_status_t mcl_set_pipeline_chunks(mcl_mapper_t* h, int chunks) {
  if (!h || chunks < 0) return MCL_E_INVAL;
  h->pipeline_chunks = chunks;
  return MCL_OK;
}

mcl_status_t mcl_force_path(mcl_mapper_t* h, int path) {
  if (!h || path < 0 || path > 9) return MCL_E_INVAL;
  h->force_path = path;
  return MCL_OK;
}

mcl_status_t mcl_last_kernel_time(const mcl_mapper_t* h, float* kernel_ms, float* call_ms) {
  if (!h) return MCL_E_INVAL;
  float k = 0.f, c = 0.f;
  if (h->timing_pending) {  // the call synchronised its stream, so the events are complete
    DeviceGuard g(h->device);
    if (cudaEventElapsedTime(&k, h->ev[0], h->ev[1]) != cudaSuccess) k = 0.f;
    if (h->timing >= 2 && cudaEventElapsedTime(&c, h->ev[2], h->ev[3]) != cudaSuccess) c = 0.f;
    cudaGetLastError();
  }
  if (kernel_ms) *kernel_ms = k;
  if (call_ms) *call_ms = c;
  return MCL_OK;
}

}  // extern "C"

namespace {

// Stage a host buffer of `bytes` into `buf` (device pointers are used in place).
mcl_status_t stage_in(mcl_mapper* h, DevBuf& buf, const void* src, size_t bytes, bool on_device,
                      const void** out, const void* dsrc = nullptr) {
  if (on_device) {
    *out = dsrc ? dsrc : src;
    return MCL_OK;
  }
  MCL_CUDA(h, buf.ensure(bytes), "cudaMalloc(staging)");
  MCL_CUDA(h, cudaMemcpyAsync(buf.p, src, bytes, cudaMemcpyHostToDevice, h->stream), "H2D");
  *out = buf.p;
  return MCL_OK;
}

// Classify a caller buffer, then stage it in (`src` may be NULL: *out = NULL).
mcl_status_t classify_stage_in(mcl_mapper* h, DevBuf& buf, const void* src, size_t bytes,
                               const void** out, bool* in_place_host = nullptr) {
  *out = nullptr;
  if (in_place_host) *in_place_host = false;
  if (!src) return MCL_OK;
  bool on = false;
  const void* d = nullptr;
  mcl_status_t st = classify(h, src, &on, &d, in_place_host);
  if (st != MCL_OK) return st;
  return stage_in(h, buf, src, bytes, on, out, d);
}

// Argument checks shared by the entry points: Q in [1, 32], D in [1, 16], and an epoch
// count whose [E][Q][D] tables stay addressable. With `N`, also *N = D^Q <= 2^48
// (MCL_E_RANGE otherwise).
mcl_status_t check_shape(mcl_mapper* h, uint32_t Q, uint32_t D, uint64_t epochs, uint64_t* N) {
  if (Q == 0 || D == 0 || Q > MCL_MAX_QUEUES || D > MCL_MAX_DEVICES) {
    h->last_err = "Q must be in [1, 32] and D in [1, 16]";
    return MCL_E_INVAL;
  }
  if (N && mul_overflow_pow(D, Q, 1ull << MCL_MAX_INDEX_BITS, N)) {
    h->last_err = "D^Q exceeds 2^48";
    return MCL_E_RANGE;
  }
  if (epochs > (1ull << 40) / ((uint64_t)Q * D)) {
    h->last_err = "epochs too large";
    return MCL_E_INVAL;
  }
  return MCL_OK;
}

// Result buffers of a search call: device pointers are written in place, host pointers
// through handle-owned device buffers that copy_outputs_back returns to the caller.
struct Outputs {
  uint64_t* idx = nullptr;  // where the kernels write
  uint64_t* ms = nullptr;
  uint8_t* map = nullptr;
  uint64_t* user_idx = nullptr;  // the caller's buffers
  uint64_t* user_ms = nullptr;
  uint8_t* user_map = nullptr;
};

mcl_status_t stage_outputs(mcl_mapper* h, uint64_t epochs, uint32_t Q, uint64_t* index,
                           uint8_t* mapping, uint64_t* makespan, Outputs* o) {
  o->user_idx = index;
  o->user_ms = makespan;
  o->user_map = mapping;
  bool di = true, dm = true, dmap = true;
  const void *pi = index, *pm = makespan, *pmap = mapping;
  mcl_status_t st;
  if (index && (st = classify(h, index, &di, &pi)) != MCL_OK) return st;
  if ((st = classify(h, makespan, &dm, &pm)) != MCL_OK) return st;
  if (mapping && (st = classify(h, mapping, &dmap, &pmap)) != MCL_OK) return st;
  o->idx = (uint64_t*)pi;
  o->ms = (uint64_t*)pm;
  o->map = (uint8_t*)pmap;
  if (!di) {
    MCL_CUDA(h, h->out_idx.ensure(epochs * 8), "cudaMalloc(staging)");
    o->idx = (uint64_t*)h->out_idx.p;
  }
  if (!dm) {
    MCL_CUDA(h, h->out_ms.ensure(epochs * 8), "cudaMalloc(staging)");
    o->ms = (uint64_t*)h->out_ms.p;
  }
  if (!dmap) {
    MCL_CUDA(h, h->out_map.ensure(epochs * Q), "cudaMalloc(staging)");
    o->map = (uint8_t*)h->out_map.p;
  }
  return MCL_OK;
}

// Enqueue the device-to-host copies of staged outputs (the caller syncs the stream).
mcl_status_t copy_outputs_back(mcl_mapper* h, uint64_t epochs, uint32_t Q, const Outputs& o) {
  cudaStream_t s = h->stream;
  if (o.idx != o.user_idx)
    MCL_CUDA(h, cudaMemcpyAsync(o.user_idx, o.idx, epochs * 8, cudaMemcpyDeviceToHost, s), "D2H");
  if (o.ms != o.user_ms)
    MCL_CUDA(h, cudaMemcpyAsync(o.user_ms, o.ms, epochs * 8, cudaMemcpyDeviceToHost, s), "D2H");
  if (o.map != o.user_map)
    MCL_CUDA(h, cudaMemcpyAsync(o.user_map, o.map, epochs * Q, cudaMemcpyDeviceToHost, s), "D2H");
  return MCL_OK;
}

// The status word the kernels raised (read after the stream sync) as an mcl_status_t.
// kFlagNeedU64 and kFlagNoPack are handled by the search itself, not reported.
mcl_status_t status_from_flags(mcl_mapper* h) {
  const uint32_t flags = *(volatile uint32_t*)h->flags_host;
  if (flags & mcl::kFlagBadModel) {
    h->last_err = "invalid cost model (kernel id, source, offsets, sizes or bandwidths)";
    return MCL_E_INVAL;
  }
  if (flags & mcl::kFlagBadMapping) {
    h->last_err = "a mapping names a device >= D";
    return MCL_E_INVAL;
  }
  if (flags & mcl::kFlagRange) {
    h->last_err = "a cost entry, built cost or base load is >= 2^48";
    return MCL_E_RANGE;
  }
  if (flags & mcl::kFlagBadHint) {
    h->last_err = "a queue hint names a class >= num_classes";
    return MCL_E_INVAL;
  }
  if (flags & mcl::kFlagInfeasible) {
    h->last_err = "a queue has no eligible device below D";
    return MCL_E_INVAL;
  }
  if (flags & mcl::kFlagPeerTimeout) {
    h->last_err = "peer exchange timed out (a rank did not make the same call); exchange disabled";
    return MCL_E_NCCL;
  }
  return MCL_OK;
}

void clear_flags(mcl_mapper* h) { *(volatile uint32_t*)h->flags_host = 0; }

// start event of a timed launch; with a hold the stream is kept busy until the launch is
// enqueued, so the events bracket device execution only (mcl_set_timing_hold)
cudaError_t record_start(mcl_mapper* h, cudaStream_t s) {
  if (h->hold_us) {
    const cudaError_t e = mcl::launch_hold((uint64_t)h->hold_us * 1000u, s);
    if (e != cudaSuccess) return e;
  }
  return cudaEventRecord(h->ev[0], s);
}

mcl_status_t map_impl(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                      const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                      const uint64_t* base_load, const uint16_t* eligible,
                      uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan);

// Chunks of a pipelined host-resident call: at least 1.5 MB of K + X per chunk, at most 4
// (each chunk costs ~15-20 us of host enqueue and a kernel ramp; measured,
// scripts/pipeline_study.py: 8 x 4 x 10^4 epochs 0.214 -> 0.186 ms with 2-4 chunks, 2 x 3 x
// 10^6 epochs 2.10 -> 1.90 ms with 4, worse again at 16), each at least one wave of the
// warp-per-epoch kernel (16 epochs per SM) so no chunk runs a partly empty GPU; 1 = no
// pipelining. A forced count (mcl_set_pipeline_chunks) is taken as is.
uint64_t pipeline_chunk_count(const mcl_mapper* h, uint32_t Q, uint32_t D, uint64_t epochs) {
  if (h->pipeline_chunks > 1) return std::min<uint64_t>((uint64_t)h->pipeline_chunks, epochs);
  const uint64_t bytes = 2 * epochs * Q * D * sizeof(uint64_t);
  uint64_t nc = std::min<uint64_t>(4, bytes / (3u << 19));
  nc = std::min<uint64_t>(nc, epochs / ((uint64_t)h->num_sms * 16));
  return std::max<uint64_t>(nc, 1);
}

// Chunk boundaries of a pipelined call: with three or more chunks the first and the last
// are half as large as the others, so the search starts after a short first copy and only a
// short search remains after the last copy (the middle chunks' searches overlap the copies).
uint64_t chunk_edge(uint64_t epochs, uint64_t nc, uint64_t c) {
  if (c >= nc) return epochs;
  if (nc < 3) return epochs * c / nc;
  // weights 1/2, 1, ..., 1, 1/2: cumulative weight of chunks [0, c) is c - 1/2 (c >= 1)
  const uint64_t twice = c == 0 ? 0 : 2 * c - 1;  // in halves, of 2 * (nc - 1) halves
  return (uint64_t)(((__uint128_t)epochs * twice) / (2 * (nc - 1)));
}

// Pipelined staging: chunk c's host->device copies go to pipe[0], its search to pipe[1]
// (after the copy, through an event) and its device->host copies to pipe[2] (after the
// search), so the copies of one chunk overlap the search of another while the searches run
// one after another (they share the handle's scratch: split-epoch slots and done counters).
// The handle's stream is joined at the end. Each search is an ordinary call on device
// pointers into the staging buffers, enqueued without a sync (async_call); the flags of all
// chunks are read once at the end. *plain = true: some epoch's bound needs 64-bit loads
// (every chunk ran the 32-bit kernels), so the caller reruns the whole call unpipelined.
mcl_status_t map_pipelined(mcl_mapper* h, uint32_t Q, uint32_t D, uint64_t epochs, uint64_t nc,
                           const uint64_t* Kh, const uint64_t* Xh, uint64_t* idx_h, uint8_t* map_h,
                           uint64_t* ms_h, bool* plain) {
  *plain = false;
  const size_t row = (size_t)Q * D;
  MCL_CUDA(h, h->in_k.ensure(epochs * row * 8), "cudaMalloc(staging)");
  MCL_CUDA(h, h->in_x.ensure(epochs * row * 8), "cudaMalloc(staging)");
  MCL_CUDA(h, h->out_idx.ensure(epochs * 8), "cudaMalloc(staging)");
  MCL_CUDA(h, h->out_ms.ensure(epochs * 8), "cudaMalloc(staging)");
  if (map_h) MCL_CUDA(h, h->out_map.ensure(epochs * Q), "cudaMalloc(staging)");
  for (cudaStream_t& ps : h->pipe)
    if (!ps) MCL_CUDA(h, cudaStreamCreateWithFlags(&ps, cudaStreamNonBlocking), "cudaStreamCreate(pipe)");
  for (cudaEvent_t& pe : h->pipe_ev)
    if (!pe) MCL_CUDA(h, cudaEventCreateWithFlags(&pe, cudaEventDisableTiming), "cudaEventCreate(pipe)");
  while (h->chunk_ev.size() < 2 * nc) {
    cudaEvent_t ce;
    MCL_CUDA(h, cudaEventCreateWithFlags(&ce, cudaEventDisableTiming), "cudaEventCreate(chunk)");
    h->chunk_ev.push_back(ce);
  }
  uint64_t* Kd = (uint64_t*)h->in_k.p;
  uint64_t* Xd = (uint64_t*)h->in_x.p;
  uint64_t* Id = (uint64_t*)h->out_idx.p;
  uint64_t* Md = (uint64_t*)h->out_ms.p;
  uint8_t* Pd = map_h ? (uint8_t*)h->out_map.p : nullptr;
  const cudaStream_t s0 = h->stream, sin = h->pipe[0], sk = h->pipe[1], sout = h->pipe[2];
  const int timing = h->timing;
  clear_flags(h);
  if (timing >= 2) MCL_CUDA(h, cudaEventRecord(h->ev[2], s0), "cudaEventRecord");
  MCL_CUDA(h, cudaEventRecord(h->pipe_ev[0], s0), "cudaEventRecord(pipe)");
  for (int i = 0; i < 3; ++i)
    MCL_CUDA(h, cudaStreamWaitEvent(h->pipe[i], h->pipe_ev[0], 0), "cudaStreamWaitEvent(pipe)");
  mcl_status_t st = MCL_OK;
  int64_t launches = 0;
  h->timing = 0;  // the chunks' own events are not recorded; the span is (below)
  bool started = false;  // ev[0] goes before the first non-empty chunk's search
  for (uint64_t c = 0; c < nc && st == MCL_OK; ++c) {
    const uint64_t lo = chunk_edge(epochs, nc, c), hi = chunk_edge(epochs, nc, c + 1), ec = hi - lo;
    if (ec == 0) continue;
    cudaEvent_t in_done = h->chunk_ev[2 * c], k_done = h->chunk_ev[2 * c + 1];
    cudaError_t e = cudaMemcpyAsync(Kd + lo * row, Kh + lo * row, ec * row * 8, cudaMemcpyHostToDevice, sin);
    if (e == cudaSuccess) e = cudaMemcpyAsync(Xd + lo * row, Xh + lo * row, ec * row * 8, cudaMemcpyHostToDevice, sin);
    if (e == cudaSuccess) e = cudaEventRecord(in_done, sin);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(sk, in_done, 0);
    if (e == cudaSuccess && timing && !started) e = cudaEventRecord(h->ev[0], sk);
    started = true;
    if (e != cudaSuccess) {
      st = cuda_fail(h, e, "pipelined H2D");
      break;
    }
    h->stream = sk;
    h->async_call = true;
    st = map_impl(h, Q, D, ec, Kd + lo * row, Xd + lo * row, nullptr, nullptr, Id + lo,
                  Pd ? Pd + lo * Q : nullptr, Md + lo);
    h->async_call = false;
    h->stream = s0;
    if (st != MCL_OK) break;
    launches += h->info[1];
    if (timing && c == nc - 1) e = cudaEventRecord(h->ev[1], sk);
    if (e == cudaSuccess) e = cudaEventRecord(k_done, sk);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(sout, k_done, 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(idx_h + lo, Id + lo, ec * 8, cudaMemcpyDeviceToHost, sout);
    if (e == cudaSuccess) e = cudaMemcpyAsync(ms_h + lo, Md + lo, ec * 8, cudaMemcpyDeviceToHost, sout);
    if (e == cudaSuccess && map_h) e = cudaMemcpyAsync(map_h + lo * Q, Pd + lo * Q, ec * Q, cudaMemcpyDeviceToHost, sout);
    if (e != cudaSuccess) st = cuda_fail(h, e, "pipelined D2H");
  }
  h->timing = timing;
  // join the pipe streams into the handle's stream, then wait for everything
  for (int i = 0; i < 3; ++i) {
    cudaEventRecord(h->pipe_ev[1 + i], h->pipe[i]);
    cudaStreamWaitEvent(s0, h->pipe_ev[1 + i], 0);
  }
  if (timing >= 2) cudaEventRecord(h->ev[3], s0);
  const cudaError_t se = cudaStreamSynchronize(s0);
  if (st != MCL_OK) return st;
  MCL_CUDA(h, se, "pipelined call");
  if ((st = status_from_flags(h)) != MCL_OK) return st;
  if (*(volatile uint32_t*)h->flags_host & mcl::kFlagNeedU64) {
    *plain = true;
    return MCL_OK;
  }
  h->info[1] = launches;
  h->info[7] = (int64_t)nc;
  h->timing_pending = timing > 0;
  return MCL_OK;
}

mcl_status_t map_impl(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                      const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                      const uint64_t* base_load, const uint16_t* eligible,
                      uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  uint64_t N = 0;
  mcl_status_t st = check_shape(h, Q, D, epochs, &N);
  if (st != MCL_OK || epochs == 0) return st;
  if (!cost_kernel || !cost_xfer || !mapping_index || !makespan) {
    h->last_err = "NULL required pointer";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  // Pinned host buffers are used in place (zero-copy, see classify) by small calls, and by
  // the warp-per-epoch batch kernel, which loads each epoch's costs one epoch ahead -- its
  // PCIe reads then overlap the search (cfg2 from pinned buffers: 0.142 ms zero-copy vs
  // 0.183 ms with pipelined staging; cfg3's thread-per-epoch kernel is PCIe-bound either
  // way, 1.94 vs 1.91 ms, and keeps the pipeline; profiles/r02/e2e_study.jsonl).
  static const int kZeroCopyMax = mcl::env_int("MCL_ZERO_COPY_MAX", 64 << 10, 0, 1 << 30);
  const bool batch_path = !base_load && !eligible && h->comm == nullptr && !h->peer_ready &&
                          h->world <= 1 && mcl::batch_supported(Q, D) &&
                          epochs >= (uint64_t)h->num_sms * 4 && (h->force_path == 0 || h->force_path == 7);
  h->zero_copy = !h->async_call && h->pipeline_chunks <= 1 &&  // a forced pipeline is staged
                 (batch_path ||
                  (uint64_t)epochs * ((uint64_t)Q * D * 16 + 16 + Q + (base_load ? D * 8 : 0) +
                                      (eligible ? Q * 2 : 0)) <= (uint64_t)kZeroCopyMax);
  struct ZeroCopyReset {  // the flag holds for this call only
    mcl_mapper* h;
    ~ZeroCopyReset() { h->zero_copy = false; }
  } zc_reset{h};
  // With a communicator or imported peer slabs the call is collective (a 1-rank
  // communicator / slab set exercises the same exchange on a single GPU). The fused peer
  // exchange (NEXT-2) takes precedence over NCCL for the calls its slabs can hold.
  const bool fused = h->peer_ready && epochs <= h->peer_cap;
  const bool use_nccl = !fused && h->comm != nullptr;
  const bool multi = fused || use_nccl;
  // A handle whose ranks exchange through peer slabs must never fall back to a sub-range
  // search silently: without the exchange (a call above max_epochs, or the exchange
  // disabled by a timeout) and without a communicator, this rank's shard-local argmin is
  // not the global result.
  if (h->peer_configured && h->world > 1 && !multi) {
    if (!h->peer_ready) {
      h->last_err = "peer exchange disabled by an earlier timeout and no NCCL communicator";
      return MCL_E_NCCL;
    }
    h->last_err = "epochs exceed the peer exchange's max_epochs and the handle has no NCCL communicator";
    return MCL_E_INVAL;
  }

  // ---- host-resident batch: pipelined staging (chunks of H2D / search / D2H) ----
  if (!multi && !base_load && !eligible && h->pipeline_chunks != 1 && !h->async_call && epochs > 1) {
    bool dk = true, dx = true, di = true, dm = true, dmap = false;
    if ((st = classify(h, cost_kernel, &dk)) != MCL_OK) return st;
    if ((st = classify(h, cost_xfer, &dx)) != MCL_OK) return st;
    if ((st = classify(h, mapping_index, &di)) != MCL_OK) return st;
    if ((st = classify(h, makespan, &dm)) != MCL_OK) return st;
    if (mapping && (st = classify(h, mapping, &dmap)) != MCL_OK) return st;
    if (!dk && !dx && !di && !dm && !dmap) {
      const uint64_t nc = pipeline_chunk_count(h, Q, D, epochs);
      if (nc > 1) {
        bool plain = false;
        st = map_pipelined(h, Q, D, epochs, nc, cost_kernel, cost_xfer, mapping_index, mapping,
                           makespan, &plain);
        if (!plain) return st;  // else a bound needs 64-bit loads: the unpipelined call below
      }
    }
  }
  h->info[7] = 0;

  // ---- where do the buffers live? host buffers are staged through device memory ----
  cudaStream_t s = h->stream;
  if (h->timing >= 2) MCL_CUDA(h, cudaEventRecord(h->ev[2], s), "cudaEventRecord");
  const size_t in_bytes = (size_t)epochs * Q * D * sizeof(uint64_t);
  const void *Kp, *Xp, *Bp, *Ep;
  bool k_host = false, x_host = false;  // pinned host inputs read in place (zero-copy)
  if ((st = classify_stage_in(h, h->in_k, cost_kernel, in_bytes, &Kp, &k_host)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_x, cost_xfer, in_bytes, &Xp, &x_host)) != MCL_OK) return st;
  // constrained variant: base loads [E][D] and eligible masks [E][Q] (either may be NULL)
  if ((st = classify_stage_in(h, h->in_base, base_load, epochs * D * 8, &Bp)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_elig, eligible, epochs * Q * 2, &Ep)) != MCL_OK) return st;
  const uint64_t* K = (const uint64_t*)Kp;
  const uint64_t* X = (const uint64_t*)Xp;
  const uint64_t* Bd = (const uint64_t*)Bp;
  const uint16_t* Ed = (const uint16_t*)Ep;
  const bool constrained = base_load || eligible;
  Outputs o;
  if ((st = stage_outputs(h, epochs, Q, mapping_index, mapping, makespan, &o)) != MCL_OK) return st;
  uint64_t* o_idx = o.idx;
  uint64_t* o_ms = o.ms;
  uint8_t* o_map = o.map;

  const int ibits = mcl::index_bits_host(N);
  mcl::EpochOut out{o_idx, o_ms, o_map, nullptr, nullptr};
  if (multi) {
    MCL_CUDA(h, h->key.ensure(epochs * 8), "cudaMalloc(key)");
    MCL_CUDA(h, h->pair.ensure(epochs * 16), "cudaMalloc(pair)");
    out.key = (uint64_t*)h->key.p;
    out.pair = (uint64_t*)h->pair.p;
  }
  mcl::PeerArgs peer{};  // world = 0: exchange off
  if (fused) {
    peer.world = h->world;
    peer.slabs = (uint64_t* const*)h->peer_ptrs.p;
    peer.mine = (uint64_t*)h->peer_slab.p;
    peer.cap = h->peer_cap;
    peer.kdone = (uint32_t*)h->peer_kdone.p;
    peer.gms = (uint64_t*)h->peer_gms.p;
    peer.timeout_ns = h->peer_timeout_ns;
  }
  MCL_CUDA(h, h->done.ensure(epochs * sizeof(uint32_t), true), "cudaMalloc(done)");

  // ---- choose the kernel ----
  const bool shard_mode = h->world > 1;  // NCCL collective or single-GPU shard test
  // the small and flattened kernels take no constraints; the blocked and generic ones do
  int path;
  // warp-per-epoch kernel: batches of at least one epoch per resident CTA (4 per SM)
  const bool batch_ok = !shard_mode && !multi && !constrained && mcl::batch_supported(Q, D);
  // eligible-device masks: the mixed-radix kernel enumerates the feasible mappings only
  const bool mixed_ok = eligible != nullptr && mcl::blocked_supported(Q, D);
  // batches of small constrained epochs: one warp per epoch (at most 2^16 reduced blocks of
  // D^3 leaves per epoch, one resident wave of CTAs filled)
  const bool mixed_warp_ok = mixed_ok && !shard_mode && !multi && N / ((uint64_t)D * D * D) <= (1ull << 16);
  if (!shard_mode && !multi && !constrained && mcl::small_supported(Q, D)) path = 4;
  else if (batch_ok && epochs >= (uint64_t)h->num_sms * 4) path = 7;
  else if (mixed_warp_ok && epochs >= (uint64_t)h->num_sms * 4) path = 11;
  else if (mixed_ok) path = 9;
  else if (mcl::blocked_supported(Q, D)) path = 1;
  else path = 3;
  if (h->force_path && h->force_path != 6) {  // 6 only affects mcl_map_queues_pruned
    const int f = h->force_path;
    const bool ok = (f == 3) || ((f == 1 || f == 2) && mcl::blocked_supported(Q, D)) ||
                    (f == 8 && mixed_ok) || (f == 9 && mixed_warp_ok) ||
                    (f == 7 && batch_ok) ||
                    (f == 5 && epochs > 1 && !shard_mode && !multi && !constrained &&
                     mcl::flat_supported(Q, D, mcl::index_bits_host(N))) ||
                    (f == 4 && !shard_mode && !multi && !constrained && mcl::small_supported(Q, D));
    if (!ok) {
      h->last_err = "forced kernel path does not support this shape / sharding";
      return MCL_E_INVAL;
    }
    // 5 = the flattened form of the blocked u32 kernel; 8 / 9 = the mixed-radix CTA / warp
    // kernels (paths 9 / 11)
    path = (f == 5) ? 1 : (f == 8 ? 9 : (f == 9 ? 11 : f));
  }

  int nlaunch = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    if (!h->async_call) clear_flags(h);
    nlaunch = 0;
    dim3 grid(1, 1, 1);
    int threads = 0;
    bool lean_ran = false;  // the one-CTA-per-SM build of the blocked kernel (reported as path 8)
    bool pool_ran = false;  // the SM-pooled batch kernel (reported as path 12)
    if (h->timing) MCL_CUDA(h, record_start(h, s), "cudaEventRecord(start)");
    if (path == 7) {
      mcl::BatchArgs a{Q, D, epochs, K, X, o_idx, o_ms, o_map, h->flags_dev, 1u, 0, k_host || x_host};
      int gx = 0;
      MCL_CUDA(h, mcl::launch_batch(a, h->num_sms, s, &gx, &pool_ran), "search_batch launch");
      grid.x = gx;
      threads = pool_ran ? 512 : 128;
    } else if (path == 4) {
      mcl::SmallArgs a{Q, D, epochs, K, X, o_idx, o_ms, o_map, h->flags_dev};
      int gx = 0;
      MCL_CUDA(h, mcl::launch_small(a, h->num_sms, s, &gx, &threads), "search_small launch");
      grid.x = gx;
    } else if (path == 1 && epochs > 1 && !shard_mode && !multi &&
               h->force_path == 5 &&
               mcl::flat_supported(Q, D, ibits)) {
      // batched epochs, whole index space: flattened (epoch, block) work distribution
      mcl::FlatArgs a{};
      a.Q = Q; a.D = D; a.E = epochs; a.K = K; a.X = X;
      a.nb = N / ((uint64_t)D * D * D);
      a.ibits = ibits; a.out = out; a.flags = h->flags_dev; a.one = 1;
      if (h->flat_keys.cap < epochs * 8) {
        MCL_CUDA(h, h->flat_keys.ensure(epochs * 8), "cudaMalloc(keys)");
        MCL_CUDA(h, h->flat_keys.fill(0xff), "cudaMemset(keys)");
      }
      MCL_CUDA(h, h->flat_done.ensure(epochs * 8, true), "cudaMalloc(done_blocks)");
      a.keys = (uint64_t*)h->flat_keys.p;
      a.done_blocks = (uint64_t*)h->flat_done.p;
      int gx = 0;
      MCL_CUDA(h, mcl::launch_flat(a, h->num_sms, s, &gx), "search_flat launch");
      grid.x = gx;
      threads = 32;
      path = 5;
    } else if (path == 11) {
      mcl::BlockedArgs a{};
      a.Q = Q; a.D = D; a.E = epochs; a.K = K; a.X = X;
      a.out = out; a.ibits = ibits; a.flags = h->flags_dev; a.one = 1;
      a.base = Bd; a.elig = Ed;
      a.world = 1;
      int gx = 0;
      MCL_CUDA(h, mcl::launch_mixed_warp(a, h->num_sms, s, &gx), "search_mixed_warp launch");
      grid.x = gx;
      threads = 128;
    } else if (path == 9 || path == 10) {
      // constrained: mixed-radix search of the feasible mappings (search_mixed.cu); the
      // shard is taken per epoch on the device from the reduced block count
      const bool wide = (path == 10);
      threads = 256;
      const uint64_t units = N / ((uint64_t)D * D * D);  // upper bound of the reduced blocks
      if (epochs > 1)
        while (threads > 32 && units / (uint64_t)std::max(1, h->world) / threads < 32) threads >>= 1;
      mcl::BlockedArgs a{};
      a.Q = Q; a.D = D; a.E = epochs; a.K = K; a.X = X; a.rlo = 0; a.rhi = 0;
      a.out = out; a.ibits = ibits; a.flags = h->flags_dev; a.one = 1;
      a.base = Bd; a.elig = Ed; a.peer = peer;
      a.rank = shard_mode ? h->rank : 0;
      a.world = shard_mode ? h->world : 1;
      const size_t smem = mcl::blocked_smem_bytes(Q, D, wide, threads, &a.off_red, &a.off_dig);
      const int occ = mcl::mixed_ctas_per_sm(D, wide, threads, smem);
      const uint64_t slots = (uint64_t)h->num_sms * std::max(1, occ);
      uint64_t e_full = 0, tail_cpe = 1;
      if (epochs >= slots) {
        e_full = epochs / slots * slots;
        const uint64_t rem = epochs - e_full;
        const uint64_t max_cpe = std::max<uint64_t>(1, units / (uint64_t)threads);
        tail_cpe = rem ? std::max<uint64_t>(1, std::min(slots / rem, max_cpe)) : 1;
      } else {
        tail_cpe = (slots + epochs - 1) / epochs;
        tail_cpe = std::min<uint64_t>(tail_cpe, std::max<uint64_t>(1, (units + threads - 1) / threads));
      }
      tail_cpe = std::min<uint64_t>(tail_cpe, 65535);
      a.e_full = e_full;
      a.tail_cpe = (uint32_t)tail_cpe;
      const uint64_t ncta = e_full + (epochs - e_full) * tail_cpe;
      grid = dim3((unsigned)std::min<uint64_t>(ncta, 0x7fffffffu), 1, 1);
      if (tail_cpe > 1) {
        MCL_CUDA(h, h->scratch.ensure((size_t)(epochs - e_full) * tail_cpe * sizeof(Cand)),
                 "cudaMalloc(scratch)");
        a.scratch = (Cand*)h->scratch.p;
      }
      a.done = (uint32_t*)h->done.p;
      MCL_CUDA(h, mcl::launch_mixed(a, wide, grid, threads, smem, s), "search_mixed launch");
    } else if (path == 1 || path == 2) {
      const bool wide = (path == 2);
      const uint64_t nb = N / ((uint64_t)D * D * D);
      uint64_t lo, hi;
      shard(nb, h->rank, h->world, &lo, &hi);
      threads = 256;
      if (epochs > 1) {
        // batched epochs: smaller CTAs so every thread still walks >= kMinBlocks blocks
        static const uint64_t kMinBlocks = [] {
          const char* v = getenv("MCL_BATCH_MIN_BLOCKS");  // tuning knob (default 32)
          return (uint64_t)((v && atoi(v) > 0) ? atoi(v) : 32);
        }();
        const uint64_t per_epoch = hi - lo;
        while (threads > 32 && per_epoch / threads < kMinBlocks) threads >>= 1;
      }
      mcl::BlockedArgs a{};
      a.Q = Q; a.D = D; a.E = epochs; a.K = K; a.X = X; a.rlo = lo; a.rhi = hi;
      a.out = out; a.ibits = ibits; a.flags = h->flags_dev; a.one = 1;
      a.base = Bd; a.elig = Ed; a.peer = peer;
      const size_t smem = mcl::blocked_smem_bytes(Q, D, wide, threads, &a.off_red, &a.off_dig);
      const bool lean = epochs == 1;  // single epochs: the spill-free one-CTA D = 5 build
      const int occ = mcl::blocked_ctas_per_sm(D, wide, threads, smem, lean);
      // Work layout (1-D grid): whole waves of epochs get one CTA each; the epochs of the
      // last, partial wave are split over several CTAs so that wave is filled; a batch
      // smaller than one wave spreads every epoch over the resident CTAs.
      const uint64_t slots = (uint64_t)h->num_sms * std::max(1, occ);
      const uint64_t units = hi - lo;
      const uint64_t chunk = (D <= 5 && Q >= 5 && !wide) ? (uint64_t)D * D : 1;
      uint64_t e_full = 0, tail_cpe = 1;
      if (epochs >= slots) {
        e_full = epochs / slots * slots;
        const uint64_t rem = epochs - e_full;
        // split only as far as every thread keeps at least one chunk
        const uint64_t max_cpe = std::max<uint64_t>(1, units / ((uint64_t)threads * chunk));
        tail_cpe = rem ? std::max<uint64_t>(1, std::min(slots / rem, max_cpe)) : 1;
      } else {
        tail_cpe = (slots + epochs - 1) / epochs;
        tail_cpe = std::min<uint64_t>(tail_cpe, std::max<uint64_t>(1, (units + threads - 1) / threads));
      }
      tail_cpe = std::min<uint64_t>(tail_cpe, 65535);
      a.e_full = e_full;
      a.tail_cpe = (uint32_t)tail_cpe;
      const uint64_t ncta = e_full + (epochs - e_full) * tail_cpe;
      grid = dim3((unsigned)std::min<uint64_t>(ncta, 0x7fffffffu), 1, 1);
      if (tail_cpe > 1) {
        MCL_CUDA(h, h->scratch.ensure((size_t)(epochs - e_full) * tail_cpe * sizeof(Cand)),
                 "cudaMalloc(scratch)");
        a.scratch = (Cand*)h->scratch.p;
        if (h->keyslot.cap < epochs * 8) {  // per-epoch packed keys, all ones between calls
          MCL_CUDA(h, h->keyslot.ensure(epochs * 8), "cudaMalloc(keyslot)");
          MCL_CUDA(h, h->keyslot.fill(0xff), "cudaMemset(keyslot)");
        }
        a.keyslot = (uint64_t*)h->keyslot.p;
      }
      a.done = (uint32_t*)h->done.p;
      MCL_CUDA(h, mcl::launch_blocked(a, wide, grid, threads, smem, s, lean), "search_blocked launch");
      lean_ran = lean && mcl::blocked_lean_built(D, wide);
    } else {
      const uint64_t rows = N / D;
      uint64_t lo, hi;
      shard(rows, h->rank, h->world, &lo, &hi);
      threads = 128;
      if (epochs > 1) {
        while (threads > 32 && (hi - lo) / threads < 16) threads >>= 1;
      }
      mcl::GenericArgs a{};
      a.Q = Q; a.D = D; a.E = epochs; a.K = K; a.X = X; a.rlo = lo; a.rhi = hi;
      a.out = out; a.ibits = ibits; a.flags = h->flags_dev;
      a.base = Bd; a.elig = Ed; a.peer = peer;
      const size_t smem = mcl::generic_smem_bytes(Q, D, threads);
      size_grid(h, epochs, hi - lo, 8, threads, &grid);
      if (grid.x > 1) {
        MCL_CUDA(h, h->scratch.ensure((size_t)epochs * grid.x * sizeof(Cand)), "cudaMalloc(scratch)");
        a.scratch = (Cand*)h->scratch.p;
      }
      a.done = (uint32_t*)h->done.p;
      MCL_CUDA(h, mcl::launch_generic(a, grid, threads, smem, s), "search_generic launch");
    }
    ++nlaunch;
    if (h->timing) MCL_CUDA(h, cudaEventRecord(h->ev[1], s), "cudaEventRecord");
    h->info[0] = lean_ran ? 8 : (pool_ran ? 12 : path);
    h->info[2] = (int64_t)grid.x * grid.y;
    h->info[3] = threads;
    h->info[4] = 0;
    h->info[5] = ibits;
    h->info[6] = 0;
    h->info[7] = 0;

    if (use_nccl) {
      ncclResult_t r = nccl().AllReduce(out.key, out.key, epochs, ncclUint64, ncclMin, h->comm, s);
      if (r != ncclSuccess) return nccl_fail(h, r, "ncclAllReduce(key)");
      MCL_CUDA(h, mcl::launch_decode_key(out.key, epochs, Q, D, ibits, o_idx, o_ms, o_map, h->flags_dev, s), "decode launch");
      nlaunch += 1;
      h->info[4] = 1;
    }
    if (h->async_call) {  // a pipelined chunk: the wrapper syncs and reads the flags
      h->info[1] = nlaunch;
      return MCL_OK;
    }
    MCL_CUDA(h, cudaStreamSynchronize(s), "search kernel");
    const uint32_t flags = *(volatile uint32_t*)h->flags_host;
    if (flags & mcl::kFlagPeerTimeout) h->peer_ready = false;  // the slabs' rounds diverged
    if ((st = status_from_flags(h)) != MCL_OK) return st;
    if (fused) {
      h->info[4] = 2;
      h->info[6] = (flags & mcl::kFlagTwoStep) ? 1 : 0;
    }
    if (flags & mcl::kFlagNeedU64) {  // some epoch's bound needs 64-bit loads: rerun the wide kernel
      if (path != 1 && path != 5 && path != 7 && path != 9 && path != 11) {
        h->last_err = "internal: 64-bit request from a 64-bit kernel";
        return MCL_E_CUDA;
      }
      path = (path == 9 || path == 11) ? 10 : 2;
      continue;
    }
    if (use_nccl && (flags & mcl::kFlagNoPack)) {  // key does not pack: two-step lexicographic all-reduce
      uint64_t* gms;
      uint64_t* cand;
      MCL_CUDA(h, h->gms.ensure(epochs * 8), "cudaMalloc(gms)");
      MCL_CUDA(h, h->cand.ensure(epochs * 8), "cudaMalloc(cand)");
      gms = (uint64_t*)h->gms.p;
      cand = (uint64_t*)h->cand.p;
      MCL_CUDA(h, mcl::launch_extract_ms(out.pair, epochs, gms, s), "extract launch");
      ncclResult_t r = nccl().AllReduce(gms, gms, epochs, ncclUint64, ncclMin, h->comm, s);
      if (r != ncclSuccess) return nccl_fail(h, r, "ncclAllReduce(ms)");
      MCL_CUDA(h, mcl::launch_pair_candidates(out.pair, gms, epochs, cand, s), "cand launch");
      r = nccl().AllReduce(cand, cand, epochs, ncclUint64, ncclMin, h->comm, s);
      if (r != ncclSuccess) return nccl_fail(h, r, "ncclAllReduce(idx)");
      MCL_CUDA(h, mcl::launch_decode_pair(gms, cand, epochs, Q, D, o_idx, o_ms, o_map, s), "decode launch");
      nlaunch += 3;
      h->info[6] = 1;
      MCL_CUDA(h, cudaStreamSynchronize(s), "two-step reduce");
    }
    break;
  }
  h->info[1] = nlaunch;

  // ---- results back to host buffers ----
  const bool staged = o.idx != o.user_idx || o.ms != o.user_ms || o.map != o.user_map;
  if ((st = copy_outputs_back(h, epochs, Q, o)) != MCL_OK) return st;
  if (h->timing >= 2) MCL_CUDA(h, cudaEventRecord(h->ev[3], s), "cudaEventRecord");
  // the stream is already idle unless copies or the call-end event were enqueued
  if (staged || h->timing >= 2) MCL_CUDA(h, cudaStreamSynchronize(s), "D2H");
  h->timing_pending = h->timing > 0;  // elapsed times are read lazily (mcl_last_kernel_time)
  return MCL_OK;
}

}  // namespace

extern "C" {

mcl_status_t mcl_map_queues(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                            const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                            uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan) {
  return map_impl(h, Q, D, epochs, cost_kernel, cost_xfer, nullptr, nullptr, mapping_index,
                  mapping, makespan);
}

mcl_status_t mcl_map_queues_constrained(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                        const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                        const mcl_constraints_t* constraints,
                                        uint64_t* mapping_index, uint8_t* mapping,
                                        uint64_t* makespan) {
  return map_impl(h, Q, D, epochs, cost_kernel, cost_xfer,
                  constraints ? constraints->base_load : nullptr,
                  constraints ? constraints->eligible : nullptr, mapping_index, mapping, makespan);
}

mcl_status_t mcl_peer_export(mcl_mapper_t* h, uint64_t max_epochs, uint8_t handle_out[64]) {
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "CUDA IPC handles are 64 bytes");
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  if (!handle_out || max_epochs == 0 || max_epochs > (1ull << 20)) {
    h->last_err = "max_epochs must be in [1, 2^20]";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  MCL_CUDA(h, cudaStreamSynchronize(h->stream), "cudaStreamSynchronize");
  for (void* p : h->peer_opened) cudaIpcCloseMemHandle(p);  // a new slab voids any import
  h->peer_opened.clear();
  h->peer_ready = false;
  h->peer_configured = false;
  h->peer_slab.release();  // a fresh allocation: the handle names exactly this slab
  const size_t words = mcl::kPeerHeaderWords + 2 * max_epochs;
  MCL_CUDA(h, h->peer_slab.ensure(words * 8), "cudaMalloc(peer slab)");
  MCL_CUDA(h, cudaMemset(h->peer_slab.p, 0xff, words * 8), "cudaMemset(peer slab)");  // regions = none
  const uint64_t header[mcl::kPeerHeaderWords] = {0, 0, max_epochs, 0, 0, 0, 0, 0};
  MCL_CUDA(h, cudaMemcpy(h->peer_slab.p, header, sizeof(header), cudaMemcpyHostToDevice), "H2D(slab)");
  MCL_CUDA(h, h->peer_kdone.ensure(8), "cudaMalloc(peer)");
  MCL_CUDA(h, cudaMemset(h->peer_kdone.p, 0, 8), "cudaMemset(peer)");
  MCL_CUDA(h, h->peer_gms.ensure(max_epochs * 8), "cudaMalloc(peer)");
  cudaIpcMemHandle_t ipc;
  MCL_CUDA(h, cudaIpcGetMemHandle(&ipc, h->peer_slab.p), "cudaIpcGetMemHandle");
  MCL_CUDA(h, cudaDeviceSynchronize(), "cudaDeviceSynchronize");  // memsets ran on the legacy stream
  std::memcpy(handle_out, &ipc, sizeof(ipc));
  h->peer_cap = max_epochs;
  return MCL_OK;
}

mcl_status_t mcl_peer_import(mcl_mapper_t* h, const uint8_t* handles, uint32_t timeout_ms) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  if (!handles) {
    h->last_err = "NULL handles";
    return MCL_E_INVAL;
  }
  if (!h->peer_slab.p || h->peer_cap == 0) {
    h->last_err = "mcl_peer_export must come first";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  for (void* p : h->peer_opened) cudaIpcCloseMemHandle(p);
  h->peer_opened.clear();
  h->peer_ready = false;
  std::vector<uint64_t*> ptrs((size_t)h->world);
  for (int r = 0; r < h->world; ++r) {
    if (r == h->rank) {
      ptrs[r] = (uint64_t*)h->peer_slab.p;
      continue;
    }
    cudaIpcMemHandle_t ipc;
    std::memcpy(&ipc, handles + 64 * (size_t)r, sizeof(ipc));
    void* p = nullptr;
    MCL_CUDA(h, cudaIpcOpenMemHandle(&p, ipc, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
    h->peer_opened.push_back(p);
    ptrs[r] = (uint64_t*)p;
    uint64_t cap = 0;
    MCL_CUDA(h, cudaMemcpy(&cap, (uint64_t*)p + 2, 8, cudaMemcpyDeviceToHost), "D2H(peer slab)");
    if (cap != h->peer_cap) {
      h->last_err = "ranks exported slabs of different max_epochs";
      return MCL_E_INVAL;
    }
  }
  MCL_CUDA(h, h->peer_ptrs.ensure((size_t)h->world * 8), "cudaMalloc(peer)");
  MCL_CUDA(h, cudaMemcpy(h->peer_ptrs.p, ptrs.data(), (size_t)h->world * 8, cudaMemcpyHostToDevice),
           "H2D(peer)");
  h->peer_timeout_ns = (uint64_t)(timeout_ms ? timeout_ms : 30000) * 1000000ull;
  h->peer_ready = true;
  h->peer_configured = true;
  return MCL_OK;
}

mcl_status_t mcl_map_queues_pruned(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                   const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                   const mcl_constraints_t* constraints, uint64_t* mapping_index,
                                   uint8_t* mapping, uint64_t* makespan) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  uint64_t N = 0;
  mcl_status_t st = check_shape(h, Q, D, epochs, &N);
  if (st != MCL_OK || epochs == 0) return st;
  if (!cost_kernel || !cost_xfer || !mapping_index || !makespan) {
    h->last_err = "NULL required pointer";
    return MCL_E_INVAL;
  }
  const uint64_t* base_load = constraints ? constraints->base_load : nullptr;
  const uint16_t* eligible = constraints ? constraints->eligible : nullptr;
  // Small index spaces: scoring every mapping is cheaper than a tree search (same result).
  if (N < kPrunedMinMappings && h->comm == nullptr && h->world <= 1 && h->force_path != 6)
    return map_impl(h, Q, D, epochs, cost_kernel, cost_xfer, base_load, eligible, mapping_index,
                    mapping, makespan);
  DeviceGuard g(h->device);
  cudaStream_t s = h->stream;
  if (h->timing >= 2) MCL_CUDA(h, cudaEventRecord(h->ev[2], s), "cudaEventRecord");
  const size_t in_bytes = (size_t)epochs * Q * D * 8;
  const void *K, *X, *B, *El;
  if ((st = classify_stage_in(h, h->in_k, cost_kernel, in_bytes, &K)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_x, cost_xfer, in_bytes, &X)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_base, base_load, epochs * D * 8, &B)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_elig, eligible, epochs * Q * 2, &El)) != MCL_OK) return st;
  Outputs o;
  if ((st = stage_outputs(h, epochs, Q, mapping_index, mapping, makespan, &o)) != MCL_OK) return st;
  // per-epoch subtree counters (zero) and incumbents (all ones), self-resetting
  if (h->bnb_next.cap < epochs * 8) {
    MCL_CUDA(h, h->bnb_next.ensure(epochs * 8, true), "cudaMalloc(bnb)");
    MCL_CUDA(h, h->bnb_inc.ensure(epochs * 8), "cudaMalloc(bnb)");
    MCL_CUDA(h, h->bnb_inc.fill(0xff), "cudaMemset(bnb)");
  }
  MCL_CUDA(h, h->bnb_nodes.ensure(8, true), "cudaMalloc(bnb)");
  MCL_CUDA(h, cudaMemsetAsync(h->bnb_nodes.p, 0, 8, s), "cudaMemset(bnb)");
  MCL_CUDA(h, h->done.ensure(epochs * sizeof(uint32_t), true), "cudaMalloc(done)");

  // one CTA per SM shares an epoch's search when there are few epochs; the shared
  // incumbent prunes so much that wider grids mostly add subtree-root checks
  const int threads = 128;
  const uint64_t slots = (uint64_t)h->num_sms;
  uint64_t cpe = epochs >= slots ? 1 : (slots + epochs - 1) / epochs;
  if (cpe > (N + threads - 1) / threads) cpe = std::max<uint64_t>(1, (N + threads - 1) / threads);
  if (cpe > 65535) cpe = 65535;
  dim3 grid((unsigned)cpe, (unsigned)std::min<uint64_t>(epochs, 65535), 1);
  // subtree depth: about two subtrees per thread of an epoch
  uint32_t k = 0;
  uint64_t nsub = 1;
  while (k < Q && nsub < 2ull * threads * cpe) {
    nsub *= D;
    ++k;
  }
  if (D == 1) k = Q;
  mcl::BnbArgs a{};
  a.Q = Q; a.D = D; a.E = epochs; a.K = (const uint64_t*)K; a.X = (const uint64_t*)X;
  a.base = (const uint64_t*)B; a.elig = (const uint16_t*)El; a.k = k;
  a.next = (uint64_t*)h->bnb_next.p; a.inc = (uint64_t*)h->bnb_inc.p;
  a.nodes = (uint64_t*)h->bnb_nodes.p; a.done = (uint32_t*)h->done.p;
  a.out = mcl::EpochOut{o.idx, o.ms, o.map, nullptr, nullptr};
  a.ibits = mcl::index_bits_host(N); a.flags = h->flags_dev;
  if (grid.x > 1) {
    MCL_CUDA(h, h->scratch.ensure((size_t)epochs * grid.x * sizeof(Cand)), "cudaMalloc(scratch)");
    a.scratch = (Cand*)h->scratch.p;
  }
  clear_flags(h);
  if (h->timing) MCL_CUDA(h, record_start(h, s), "cudaEventRecord(start)");
  MCL_CUDA(h, mcl::launch_bnb(a, grid, threads, s), "search_bnb launch");
  if (h->timing) MCL_CUDA(h, cudaEventRecord(h->ev[1], s), "cudaEventRecord");
  uint64_t nodes = 0;
  MCL_CUDA(h, cudaMemcpyAsync(&nodes, h->bnb_nodes.p, 8, cudaMemcpyDeviceToHost, s), "D2H");
  MCL_CUDA(h, cudaStreamSynchronize(s), "search_bnb");
  if ((st = status_from_flags(h)) != MCL_OK) return st;
  h->info[0] = 6;
  h->info[1] = 1;
  h->info[2] = (int64_t)grid.x * grid.y;
  h->info[3] = threads;
  h->info[4] = 0;
  h->info[5] = a.ibits;
  h->info[6] = 0;
  h->info[7] = (int64_t)nodes;
  if ((st = copy_outputs_back(h, epochs, Q, o)) != MCL_OK) return st;
  if (h->timing >= 2) MCL_CUDA(h, cudaEventRecord(h->ev[3], s), "cudaEventRecord");
  MCL_CUDA(h, cudaStreamSynchronize(s), "D2H");
  h->timing_pending = h->timing > 0;
  return MCL_OK;
}

}  // extern "C"

namespace {

// Build K and X into device buffers Kd, Xd (each [E][Q][D]); stages host model arrays.
mcl_status_t build_costs_dev(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                             const mcl_cost_model_t* m, uint64_t* Kd, uint64_t* Xd) {
  if (!m || !m->kernel_profile || !m->offsets || !m->bytes || !m->source || !m->sizes ||
      !m->h2d_bw || !m->d2h_bw || (m->num_invocations && !m->kernel_ids) ||
      m->num_sizes == 0 || m->num_sizes > 64 || m->num_kernels == 0 || m->num_sockets > 8) {
    h->last_err = "invalid cost model (NULL array, num_sizes outside 1..64, num_sockets > 8 or no kernels)";
    return MCL_E_INVAL;
  }
  const uint64_t EQ = epochs * Q;
  const uint32_t M = m->num_sizes;
  const uint32_t S = m->num_sockets ? m->num_sockets : 1;
  struct Arr {
    const void* src;
    size_t bytes;
    DevBuf* buf;
    const void* dev;
  } arrs[10] = {
      {m->kernel_profile, (size_t)m->num_kernels * D * 8, &h->model_buf[0], nullptr},
      {m->offsets, (size_t)(EQ + 1) * 8, &h->model_buf[1], nullptr},
      {m->kernel_ids, (size_t)m->num_invocations * 4, &h->model_buf[2], nullptr},
      {m->bytes, (size_t)EQ * 8, &h->model_buf[3], nullptr},
      {m->source, (size_t)EQ * 4, &h->model_buf[4], nullptr},
      {m->cached, (size_t)EQ * 2, &h->model_buf[5], nullptr},
      {m->sizes, (size_t)M * 8, &h->model_buf[6], nullptr},
      {m->h2d_bw, (size_t)S * D * M * 8, &h->model_buf[7], nullptr},
      {m->d2h_bw, (size_t)S * D * M * 8, &h->model_buf[8], nullptr},
      {m->host_socket, (size_t)EQ, &h->model_buf[9], nullptr},
  };
  mcl_status_t st;
  for (auto& a : arrs) {
    if (a.bytes == 0) continue;
    if ((st = classify_stage_in(h, *a.buf, a.src, a.bytes, &a.dev)) != MCL_OK) return st;
  }
  mcl::CostArgs c{};
  c.D = D; c.EQ = EQ; c.num_kernels = m->num_kernels;
  c.profile = (const uint64_t*)arrs[0].dev; c.offsets = (const uint64_t*)arrs[1].dev;
  c.ids = (const uint32_t*)arrs[2].dev; c.nnz = m->num_invocations;
  c.bytes = (const uint64_t*)arrs[3].dev; c.source = (const int32_t*)arrs[4].dev;
  c.cached = (const uint16_t*)arrs[5].dev; c.M = M; c.sizes = (const uint64_t*)arrs[6].dev;
  c.h2d = (const double*)arrs[7].dev; c.d2h = (const double*)arrs[8].dev;
  c.S = S; c.host_socket = (const uint8_t*)arrs[9].dev;
  c.host_shared = m->host_shared; c.K = Kd; c.X = Xd; c.flags = h->flags_dev;
  MCL_CUDA(h, mcl::launch_build_costs(c, h->num_sms, h->stream), "build_costs launch");
  return MCL_OK;
}

}  // namespace

extern "C" {

mcl_status_t mcl_build_costs(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                             const mcl_cost_model_t* model, uint64_t* cost_kernel,
                             uint64_t* cost_xfer) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  mcl_status_t st = check_shape(h, Q, D, epochs, nullptr);
  if (st != MCL_OK || epochs == 0) return st;
  if (!cost_kernel || !cost_xfer) {
    h->last_err = "NULL output";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  bool dk, dx;
  if ((st = classify(h, cost_kernel, &dk)) != MCL_OK) return st;
  if ((st = classify(h, cost_xfer, &dx)) != MCL_OK) return st;
  const size_t out_bytes = (size_t)epochs * Q * D * 8;
  uint64_t* Kd = cost_kernel;
  uint64_t* Xd = cost_xfer;
  if (!dk) {
    MCL_CUDA(h, h->cost_k.ensure(out_bytes), "cudaMalloc(costs)");
    Kd = (uint64_t*)h->cost_k.p;
  }
  if (!dx) {
    MCL_CUDA(h, h->cost_x.ensure(out_bytes), "cudaMalloc(costs)");
    Xd = (uint64_t*)h->cost_x.p;
  }
  clear_flags(h);
  if (h->timing) MCL_CUDA(h, record_start(h, h->stream), "cudaEventRecord(start)");
  if ((st = build_costs_dev(h, Q, D, epochs, model, Kd, Xd)) != MCL_OK) return st;
  if (h->timing) MCL_CUDA(h, cudaEventRecord(h->ev[1], h->stream), "cudaEventRecord");
  if (!dk) MCL_CUDA(h, cudaMemcpyAsync(cost_kernel, Kd, out_bytes, cudaMemcpyDeviceToHost, h->stream), "D2H");
  if (!dx) MCL_CUDA(h, cudaMemcpyAsync(cost_xfer, Xd, out_bytes, cudaMemcpyDeviceToHost, h->stream), "D2H");
  MCL_CUDA(h, cudaStreamSynchronize(h->stream), "build_costs");
  h->timing_pending = h->timing > 0;
  return status_from_flags(h);
}

mcl_status_t mcl_map_from_profiles(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                   const mcl_cost_model_t* model,
                                   const mcl_constraints_t* constraints,
                                   uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  mcl_status_t st = check_shape(h, Q, D, epochs, nullptr);
  if (st != MCL_OK || epochs == 0) return st;
  DeviceGuard g(h->device);
  const size_t bytes = (size_t)epochs * Q * D * 8;
  MCL_CUDA(h, h->cost_k.ensure(bytes), "cudaMalloc(costs)");
  MCL_CUDA(h, h->cost_x.ensure(bytes), "cudaMalloc(costs)");
  clear_flags(h);
  st = build_costs_dev(h, Q, D, epochs, model, (uint64_t*)h->cost_k.p, (uint64_t*)h->cost_x.p);
  if (st != MCL_OK) return st;
  // the search's own flag checks follow; model errors must be reported first
  MCL_CUDA(h, cudaStreamSynchronize(h->stream), "build_costs");
  if ((st = status_from_flags(h)) != MCL_OK) return st;
  return map_impl(h, Q, D, epochs, (const uint64_t*)h->cost_k.p, (const uint64_t*)h->cost_x.p,
                  constraints ? constraints->base_load : nullptr,
                  constraints ? constraints->eligible : nullptr, mapping_index, mapping, makespan);
}

mcl_status_t mcl_score_mappings(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                const uint64_t* base_load, const uint8_t* mappings,
                                uint64_t* makespan) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  mcl_status_t st = check_shape(h, Q, D, epochs, nullptr);
  if (st != MCL_OK || epochs == 0) return st;
  if (!cost_kernel || !cost_xfer || !mappings || !makespan) {
    h->last_err = "NULL required pointer";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  const void *K, *X, *B, *M;
  const size_t in_bytes = (size_t)epochs * Q * D * 8;
  if ((st = classify_stage_in(h, h->in_k, cost_kernel, in_bytes, &K)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_x, cost_xfer, in_bytes, &X)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_base, base_load, epochs * D * 8, &B)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_elig, mappings, epochs * Q, &M)) != MCL_OK) return st;
  Outputs o;
  if ((st = stage_outputs(h, epochs, Q, nullptr, nullptr, makespan, &o)) != MCL_OK) return st;
  clear_flags(h);
  MCL_CUDA(h, mcl::launch_score(Q, D, epochs, (const uint64_t*)K, (const uint64_t*)X,
                                (const uint64_t*)B, (const uint8_t*)M, o.ms, h->flags_dev, h->stream),
           "score launch");
  if ((st = copy_outputs_back(h, epochs, Q, o)) != MCL_OK) return st;
  MCL_CUDA(h, cudaStreamSynchronize(h->stream), "score kernel");
  return status_from_flags(h);
}

mcl_status_t mcl_static_mappings(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                 const uint8_t* hints, uint32_t num_classes,
                                 const uint64_t* device_score, const uint16_t* eligible,
                                 uint8_t* mappings) {
  if (!h) return MCL_E_INVAL;
  h->last_err.clear();
  mcl_status_t st = check_shape(h, Q, D, epochs, nullptr);
  if (st != MCL_OK || epochs == 0) return st;
  if (!hints || !device_score || !mappings || num_classes == 0 || num_classes > MCL_MAX_DEVICES) {
    h->last_err = "NULL required pointer or num_classes outside 1..16";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  const void *Hd, *Sd, *Ed;
  if ((st = classify_stage_in(h, h->in_k, hints, epochs * Q, &Hd)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_x, device_score, (size_t)num_classes * D * 8, &Sd)) != MCL_OK) return st;
  if ((st = classify_stage_in(h, h->in_elig, eligible, epochs * Q * 2, &Ed)) != MCL_OK) return st;
  bool on = true;
  if ((st = classify(h, mappings, &on)) != MCL_OK) return st;
  uint8_t* Md = mappings;
  if (!on) {
    MCL_CUDA(h, h->out_map.ensure(epochs * Q), "cudaMalloc(staging)");
    Md = (uint8_t*)h->out_map.p;
  }
  clear_flags(h);
  MCL_CUDA(h, mcl::launch_static_map(Q, D, epochs, (const uint8_t*)Hd, num_classes, (const uint64_t*)Sd,
                                     (const uint16_t*)Ed, Md, h->flags_dev, h->stream),
           "static_map launch");
  if (!on) MCL_CUDA(h, cudaMemcpyAsync(mappings, Md, epochs * Q, cudaMemcpyDeviceToHost, h->stream), "D2H");
  MCL_CUDA(h, cudaStreamSynchronize(h->stream), "static_map kernel");
  return status_from_flags(h);
}

}  // extern "C"

extern "C" {

mcl_status_t mcl_probe_int_rate(int device, int op, double* lane_ops_per_s,
                                double* lane_ops_per_clk_sm, double* eff_mhz) {
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return MCL_E_INVAL;
  DeviceGuard g(device);
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess)
    return MCL_E_CUDA;
  double r = 0, c = 0, m = 0;
  cudaError_t e = mcl::probe_alu(op, sms, nullptr, &r, &c, &m);
  if (e == cudaErrorInvalidValue) return MCL_E_INVAL;
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "probe");
  if (lane_ops_per_s) *lane_ops_per_s = r;
  if (lane_ops_per_clk_sm) *lane_ops_per_clk_sm = c;
  if (eff_mhz) *eff_mhz = m;
  return MCL_OK;
}

mcl_status_t mcl_probe_launch_floor(int device, int reps, double* empty_kernel_us, double* events_only_us) {
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev || reps < 1)
    return MCL_E_INVAL;
  DeviceGuard g(device);
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess)
    return MCL_E_CUDA;
  double k = 0, e = 0;
  cudaError_t err = mcl::probe_launch_floor(sms, nullptr, reps, &k, &e);
  if (err != cudaSuccess) return cuda_fail(nullptr, err, "launch floor probe");
  if (empty_kernel_us) *empty_kernel_us = k;
  if (events_only_us) *events_only_us = e;
  return MCL_OK;
}

mcl_status_t mcl_device_sms(int device, int* sms) {
  if (!sms) return MCL_E_INVAL;
  cudaError_t e = cudaDeviceGetAttribute(sms, cudaDevAttrMultiProcessorCount, device);
  return e == cudaSuccess ? MCL_OK : cuda_fail(nullptr, e, "cudaDeviceGetAttribute");
}

mcl_status_t mcl_comm_unique_id(uint8_t id_out[128]) {
  if (!id_out) return MCL_E_INVAL;
  if (!nccl().ok) {
    g_create_err = nccl().err;
    return MCL_E_NCCL;
  }
  ncclUniqueId id;
  if (nccl().GetUniqueId(&id) != ncclSuccess) return MCL_E_NCCL;
  std::memcpy(id_out, &id, sizeof(id));
  return MCL_OK;
}

mcl_status_t mcl_comm_init(int device, int world, int rank, const uint8_t id[128], void** comm_out) {
  if (!id || !comm_out || world < 1 || rank < 0 || rank >= world) return MCL_E_INVAL;
  if (!nccl().ok) {
    g_create_err = nccl().err;
    return MCL_E_NCCL;
  }
  DeviceGuard g(device);
  ncclUniqueId uid;
  std::memcpy(&uid, id, sizeof(uid));
  ncclComm_t c = nullptr;
  ncclResult_t r = nccl().CommInitRank(&c, world, uid, rank);
  if (r != ncclSuccess) {
    g_create_err = std::string("ncclCommInitRank: ") + nccl().GetErrorString(r);
    return MCL_E_NCCL;
  }
  *comm_out = c;
  return MCL_OK;
}

mcl_status_t mcl_comm_destroy(void* comm) {
  if (!comm) return MCL_OK;
  if (!nccl().ok) return MCL_E_NCCL;
  return nccl().CommDestroy((ncclComm_t)comm) == ncclSuccess ? MCL_OK : MCL_E_NCCL;
}

}  // extern "C"

// ---------------------------------------------------------------- resident mapper ------
namespace {

mcl::ResidentBox* res_box(mcl_mapper* h) { return reinterpret_cast<mcl::ResidentBox*>(h->res_mem); }

// (Re)launch the resident warp; it serves the requests numbered after seq0. `alive` is set
// here, before the launch, so 0 is only ever seen after a warp has exited.
mcl_status_t resident_launch(mcl_mapper* h, uint32_t seq0) {
  mcl::ResidentBox* box = res_box(h);
  // no stop bit; the number of the last request (a relaunch for a pending request passes
  // seq0 = its number - 1, so the new warp serves it)
  __atomic_store_n(&box->req, __atomic_load_n(&box->req, __ATOMIC_RELAXED) & ~(1ull << 63), __ATOMIC_RELEASE);
  __atomic_store_n(&box->alive, 1u, __ATOMIC_RELEASE);  // the warp clears it when it exits
  h->res_args.seq0 = seq0;
  MCL_CUDA(h, mcl::launch_resident(h->res_args, h->res_stream), "resident launch");
  return MCL_OK;
}

}  // namespace

extern "C" {

mcl_status_t mcl_resident_start(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint32_t max_epochs,
                                uint32_t idle_ms) {
  if (!h) return MCL_E_INVAL;
  if (h->res_started) {
    h->last_err = "resident mapper already started on this handle";
    return MCL_E_INVAL;
  }
  uint64_t N = 0;
  if (Q < 1 || D < 1 || Q > mcl::kResidentMaxQ || D > mcl::kResidentMaxD || max_epochs < 1 ||
      max_epochs > 64 || mul_overflow_pow(D, Q, mcl::kResidentMaxMappings, &N)) {
    h->last_err = "resident mapper: needs D^Q <= 8192, Q <= 16, D <= 16, 1 <= max_epochs <= 64";
    return MCL_E_INVAL;
  }
  DeviceGuard g(h->device);
  const size_t qd = (size_t)max_epochs * Q * D;
  const size_t off_k = sizeof(mcl::ResidentBox), off_x = off_k + qd * 8, off_r = off_x + qd * 8,
               bytes = off_r + (size_t)max_epochs * mcl::kResidentRecWords * 8;
  if (cudaHostAlloc((void**)&h->res_mem, bytes, cudaHostAllocMapped) != cudaSuccess) {
    cudaGetLastError();
    h->res_mem = nullptr;
    h->last_err = "cudaHostAlloc(resident mailbox) failed";
    return MCL_E_NOMEM;
  }
  std::memset(h->res_mem, 0, bytes);
  unsigned char* dev = nullptr;
  cudaError_t e = cudaHostGetDevicePointer((void**)&dev, h->res_mem, 0);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->res_stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) {
    cudaFreeHost(h->res_mem);
    h->res_mem = nullptr;
    return cuda_fail(h, e, "resident mailbox / stream");
  }
  mcl::ResidentArgs& a = h->res_args;
  a.box = reinterpret_cast<mcl::ResidentBox*>(dev);
  a.K = reinterpret_cast<const uint64_t*>(dev + off_k);
  a.X = reinterpret_cast<const uint64_t*>(dev + off_x);
  a.rec = reinterpret_cast<uint64_t*>(dev + off_r);
  a.Q = Q;
  a.D = D;
  a.N = (uint32_t)N;
  a.cap = max_epochs;
  a.idle_ns = (uint64_t)(idle_ms ? idle_ms : 100) * 1000000ull;
  h->res_seq = 0;
  h->res_started = true;
  const mcl_status_t st = resident_launch(h, 0);
  if (st != MCL_OK) mcl_resident_stop(h);
  return st;
}

mcl_status_t mcl_resident_map(mcl_mapper_t* h, uint64_t epochs, const uint64_t* cost_kernel,
                              const uint64_t* cost_xfer, uint64_t* mapping_index,
                              uint8_t* mapping, uint64_t* makespan) {
  if (!h) return MCL_E_INVAL;
  if (!h->res_started) {
    h->last_err = "resident mapper not started (mcl_resident_start)";
    return MCL_E_INVAL;
  }
  if (epochs == 0) return MCL_OK;
  mcl::ResidentArgs& a = h->res_args;
  if (epochs > a.cap || !cost_kernel || !cost_xfer || !mapping_index || !makespan) {
    h->last_err = "resident mapper: epochs above max_epochs or a NULL buffer";
    return MCL_E_INVAL;
  }
  for (const void* p : {(const void*)cost_kernel, (const void*)cost_xfer, (const void*)mapping_index,
                        (const void*)makespan, (const void*)mapping}) {
    if (!p) continue;
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
      cudaGetLastError();
      h->last_err = "resident mapper: cannot classify a buffer pointer";
      return MCL_E_INVAL;
    }
    if (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged) {
      h->last_err = "resident mapper: buffers must be host memory";
      return MCL_E_INVAL;
    }
  }
  mcl::ResidentBox* box = res_box(h);
  if (!__atomic_load_n(&box->alive, __ATOMIC_ACQUIRE)) {  // idle exit: relaunch
    DeviceGuard g(h->device);
    const cudaError_t e = cudaStreamQuery(h->res_stream);  // the exited kernel is gone
    if (e != cudaSuccess && e != cudaErrorNotReady) return cuda_fail(h, e, "resident kernel");
    cudaGetLastError();
    const mcl_status_t st = resident_launch(h, h->res_seq);
    if (st != MCL_OK) return st;
  }
  const size_t qd = (size_t)epochs * a.Q * a.D;
  unsigned char* base = h->res_mem;
  const size_t off_k = sizeof(mcl::ResidentBox), off_x = off_k + (size_t)a.cap * a.Q * a.D * 8,
               off_r = off_x + (size_t)a.cap * a.Q * a.D * 8;
  std::memcpy(base + off_k, cost_kernel, qd * 8);
  std::memcpy(base + off_x, cost_xfer, qd * 8);
  const uint32_t seq = ++h->res_seq;
  // inputs before the request word (x86 stores are ordered; release for the compiler)
  __atomic_store_n(&box->req, ((uint64_t)epochs << 32) | seq, __ATOMIC_RELEASE);
  // The answer: one three-word record per epoch, each word tagged with this request's
  // number (kernels.h, ResidentArgs); a failed request answers with its status in epoch 0.
  const uint64_t* rec = reinterpret_cast<const uint64_t*>(base + off_r);
  auto ready = [&](uint64_t e) {
    const uint64_t w0 = __atomic_load_n(rec + 3 * e, __ATOMIC_ACQUIRE);
    const uint64_t w1 = __atomic_load_n(rec + 3 * e + 1, __ATOMIC_ACQUIRE);
    const uint64_t w2 = __atomic_load_n(rec + 3 * e + 2, __ATOMIC_ACQUIRE);
    return (uint32_t)(w0 >> 32) == seq && (w1 >> 53) == (seq & 0x7ffu) && (uint32_t)(w2 >> 32) == seq;
  };
  auto answered = [&]() {
    if (!ready(0)) return false;
    if ((__atomic_load_n(rec, __ATOMIC_RELAXED) >> 16) & 0xffffu) return true;  // an error
    for (uint64_t e = 1; e < epochs; ++e)
      if (!ready(e)) return false;
    return true;
  };
  const auto t0 = std::chrono::steady_clock::now();
  for (uint32_t spin = 1;; ++spin) {
    if (answered()) break;
    if ((spin & 1023u) == 0) {
      const bool dead = !__atomic_load_n(&box->alive, __ATOMIC_ACQUIRE);
      if (dead || std::chrono::steady_clock::now() - t0 > std::chrono::seconds(2)) {
        if (dead && answered()) break;
        DeviceGuard g(h->device);
        const cudaError_t e = cudaStreamQuery(h->res_stream);
        h->last_err = dead ? "resident warp exited before answering"
                           : "resident warp did not answer within 2 s";
        if (e != cudaSuccess && e != cudaErrorNotReady) return cuda_fail(h, e, "resident kernel");
        if (!dead) return MCL_E_CUDA;
        // it exited idle between the alive check and the request: a new warp serves it
        const mcl_status_t st = resident_launch(h, seq - 1);
        if (st != MCL_OK) return st;
      }
    }
  }
  const uint32_t status = (uint32_t)(rec[0] >> 16) & 0xffffu;
  if (status & mcl::kFlagRange) {
    h->last_err = "a cost entry >= 2^48";
    return MCL_E_RANGE;
  }
  if (status) {
    h->last_err = "resident mapper: bad request";
    return MCL_E_INVAL;
  }
  const uint32_t b = a.D <= 1 ? 0u : 32u - (uint32_t)__builtin_clz(a.D - 1);
  const uint32_t dmask = (1u << b) - 1u;
  for (uint64_t e = 0; e < epochs; ++e) {
    mapping_index[e] = rec[3 * e] & 0xffffu;
    makespan[e] = rec[3 * e + 1] & ((1ull << 53) - 1);
    if (mapping) {  // the kernel's digits, unpacked into one byte per queue
      const uint32_t packed = (uint32_t)rec[3 * e + 2];
      for (uint32_t q = 0; q < a.Q; ++q) mapping[e * a.Q + q] = (uint8_t)((packed >> (q * b)) & dmask);
    }
  }
  return MCL_OK;
}

#ifdef MCL_RESIDENT_TRACE
// measurement builds only: the resident warp's timestamps of its last request
int mcl_resident_trace(mcl_mapper_t* h, uint64_t out[4]) {
  if (!h || !h->res_mem) return -1;
  for (int i = 0; i < 4; ++i) out[i] = __atomic_load_n(&res_box(h)->trace[i], __ATOMIC_RELAXED);
  return 0;
}
#endif

mcl_status_t mcl_resident_stop(mcl_mapper_t* h) {
  if (!h) return MCL_E_INVAL;
  if (!h->res_mem) return MCL_OK;
  DeviceGuard g(h->device);
  mcl::ResidentBox* box = res_box(h);
  __atomic_store_n(&box->req, __atomic_load_n(&box->req, __ATOMIC_RELAXED) | (1ull << 63), __ATOMIC_RELEASE);
  cudaError_t e = cudaSuccess;
  if (h->res_stream) {
    e = cudaStreamSynchronize(h->res_stream);
    cudaStreamDestroy(h->res_stream);
    h->res_stream = nullptr;
  }
  cudaFreeHost(h->res_mem);
  h->res_mem = nullptr;
  h->res_started = false;
  if (e != cudaSuccess) return cuda_fail(h, e, "resident kernel");
  return MCL_OK;
}

}  // extern "C"
