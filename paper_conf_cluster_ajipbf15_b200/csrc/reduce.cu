// reduce.cu -- epilogues of the cross-GPU argmin over NCCL.
//
// Each rank's search kernel leaves, per epoch, a packed key (makespan << index_bits | index)
// and the raw (makespan, index) pair. After ncclAllReduce(MIN) on the keys every rank holds
// the global lexicographic minimum; these kernels turn it back into the public outputs.
// When no rank's makespan fits beside the index (the reduced key is kNone), the two-step
// path is used instead: all-reduce MIN of the makespans, then all-reduce MIN of the
// indices of the ranks whose local makespan equals the global one. (The fused peer
// exchange, peer.cuh, does the same inside the search kernel.)
#include "common.cuh"
#include "kernels.h"

namespace mcl {

namespace {

__global__ void decode_key_kernel(const uint64_t* __restrict__ key, uint64_t E, uint32_t Q,
                                  uint32_t D, int ibits, uint64_t* index, uint64_t* makespan,
                                  uint8_t* mapping, volatile uint32_t* flags) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E;
       e += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = key[e];
    // no rank's candidate fitted the packed key (see write_epoch): the same on every rank
    if (k == kNone) raise_flag(flags, kFlagNoPack);
    const uint64_t mask = (ibits >= 64) ? ~0ull : ((1ull << ibits) - 1);
    const uint64_t ms = (ibits == 0) ? k : (ibits >= 64 ? 0 : (k >> ibits));
    write_result(index, makespan, mapping, e, Q, D, k & mask, ms);
  }
}

__global__ void extract_ms_kernel(const uint64_t* __restrict__ pair, uint64_t E, uint64_t* ms) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E;
       e += (uint64_t)gridDim.x * blockDim.x)
    ms[e] = pair[2 * e];
}

__global__ void pair_candidates_kernel(const uint64_t* __restrict__ pair,
                                       const uint64_t* __restrict__ gms, uint64_t E,
                                       uint64_t* cand) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E;
       e += (uint64_t)gridDim.x * blockDim.x)
    cand[e] = (pair[2 * e] == gms[e]) ? pair[2 * e + 1] : kNone;
}

__global__ void decode_pair_kernel(const uint64_t* __restrict__ gms,
                                   const uint64_t* __restrict__ gidx, uint64_t E, uint32_t Q,
                                   uint32_t D, uint64_t* index, uint64_t* makespan,
                                   uint8_t* mapping) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E;
       e += (uint64_t)gridDim.x * blockDim.x)
    write_result(index, makespan, mapping, e, Q, D, gidx[e], gms[e]);
}

unsigned grid_for(uint64_t E) {
  uint64_t g = (E + 255) / 256;
  return (unsigned)(g > 4096 ? 4096 : (g == 0 ? 1 : g));
}

}  // namespace

cudaError_t launch_decode_key(const uint64_t* key, uint64_t E, uint32_t Q, uint32_t D, int ibits,
                              uint64_t* index, uint64_t* makespan, uint8_t* mapping,
                              volatile uint32_t* flags, cudaStream_t st) {
  decode_key_kernel<<<grid_for(E), 256, 0, st>>>(key, E, Q, D, ibits, index, makespan, mapping,
                                                 flags);
  return cudaGetLastError();
}

cudaError_t launch_extract_ms(const uint64_t* pair, uint64_t E, uint64_t* ms, cudaStream_t st) {
  extract_ms_kernel<<<grid_for(E), 256, 0, st>>>(pair, E, ms);
  return cudaGetLastError();
}

cudaError_t launch_pair_candidates(const uint64_t* pair, const uint64_t* gms, uint64_t E,
                                   uint64_t* cand, cudaStream_t st) {
  pair_candidates_kernel<<<grid_for(E), 256, 0, st>>>(pair, gms, E, cand);
  return cudaGetLastError();
}

cudaError_t launch_decode_pair(const uint64_t* gms, const uint64_t* gidx, uint64_t E, uint32_t Q,
                               uint32_t D, uint64_t* index, uint64_t* makespan, uint8_t* mapping,
                               cudaStream_t st) {
  decode_pair_kernel<<<grid_for(E), 256, 0, st>>>(gms, gidx, E, Q, D, index, makespan, mapping);
  return cudaGetLastError();
}

}  // namespace mcl
