// peer_tail_bench.cu -- cost of the pieces of the fused exchange's kernel tail (peer.cuh)
// on one GPU, world = 1: a 148 x 256 kernel that does no search, only the tail variant.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ptb scripts/peer_tail_bench.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t gns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint64_t ld_acq_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_rlx_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t atom_acq_rel_gpu(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}

// variant: 0 empty, 1 count, 2 count + fence.sys, 3 count + round (red, fence, red, poll w/
// nanosleep), 4 = 3 without nanosleep, 5 = 3 with atom (returning) signal, 6 = 3 with relaxed
// poll + acquire fence, 7 count + globaltimer only
__global__ void tail(int variant, uint32_t* kdone, uint64_t* slab, uint64_t* out, uint64_t R) {
  __shared__ bool last;
  if (variant == 0) return;
  __syncthreads();
  if (threadIdx.x == 0) last = atom_acq_rel_gpu(kdone, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!last) return;
  if (threadIdx.x == 0) *kdone = 0;
  if (variant == 1) return;
  if (variant == 2) {
    if (threadIdx.x == 0) asm volatile("fence.acq_rel.sys;" ::: "memory");
    return;
  }
  if (variant == 7) {
    if (threadIdx.x == 0) out[0] = gns();
    return;
  }
  if (threadIdx.x == 0) asm volatile("red.relaxed.sys.global.min.u64 [%0], %1;" ::"l"(slab + 8), "l"(R) : "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    if (variant == 5) {
      atomicAdd_system(reinterpret_cast<unsigned long long*>(slab), 1ull);
    } else {
      asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(slab), "l"(1ull) : "memory");
    }
    const uint64_t t0 = gns();
    uint64_t spins = 0;
    if (variant == 6) {
      while (ld_rlx_sys(slab) < R + 1) ++spins;
      asm volatile("fence.acq_rel.sys;" ::: "memory");
    } else {
      while (ld_acq_sys(slab) < R + 1) {
        ++spins;
        if (variant == 3 || variant == 5) __nanosleep(64);
      }
    }
    out[0] = gns() - t0;
    out[1] += spins;
  }
}

int main() {
  uint32_t* kdone;
  uint64_t *slab, *out;
  cudaMalloc(&kdone, 8);
  cudaMalloc(&slab, 1024);
  cudaMalloc(&out, 64);
  cudaMemset(kdone, 0, 8);
  cudaMemset(slab, 0, 1024);
  cudaMemset(out, 0, 64);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  uint64_t R = 0;
  const char* names[] = {"empty", "count", "count+fence.sys", "round(nanosleep)", "round(spin)",
                         "round(atom signal)", "round(relaxed poll)", "count+globaltimer"};
  for (int v = 0; v < 8; ++v) {
    const int n = 2000;
    for (int i = 0; i < 50; ++i) tail<<<148, 256>>>(v, kdone, slab, out, R++ * (v >= 3 && v != 7));
    cudaMemset(out, 0, 64);
    cudaDeviceSynchronize();
    cudaEventRecord(a);
    for (int i = 0; i < n; ++i) tail<<<148, 256>>>(v, kdone, slab, out, (v >= 3 && v != 7) ? R++ : 0);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    uint64_t h[2];
    cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
    // reset the slab counter between variants so R tracks it
    cudaMemset(slab, 0, 1024);
    R = 0;
    printf("%-22s %8.3f us/launch  last wait %llu ns  spins/launch %.2f\n", names[v], 1e3 * ms / n,
           (unsigned long long)(v >= 3 && v != 7 ? h[0] : 0), (double)h[1] / n);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
