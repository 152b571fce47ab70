// Event-timed duration of near-empty kernels (measurement only): what a launch costs on
// this platform when timed like bench.py times the search kernels (a 200 us spin kernel
// first, so the events bracket device execution, not host launch latency).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 launch_floor.cu -o /tmp/launch_floor
#include <cstdio>
#include <cuda_runtime.h>

__global__ void spin(long long ns) {
  long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > ns) break;
  }
}
__global__ void empty(int* p) {
  if (p && threadIdx.x == 1023) *p = 1;
}
template <int SMEM>
__global__ void with_smem(int* p) {
  __shared__ int s[SMEM / 4];
  s[threadIdx.x % (SMEM / 4)] = threadIdx.x;
  __syncthreads();
  if (p && s[(threadIdx.x + 1) % (SMEM / 4)] == -1) *p = 1;
}

template <typename F>
float timeit(F launch) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float tot = 0;
  const int n = 50;
  for (int i = 0; i < n + 5; ++i) {
    spin<<<1, 1>>>(200000);
    cudaEventRecord(a);
    launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (i >= 5) tot += ms;
  }
  return tot / n * 1e3f;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  printf("{\"events_only_us\": %.2f, ", timeit([] {}));
  printf("\"empty_1x32_us\": %.2f, ", timeit([] { empty<<<1, 32>>>(nullptr); }));
  printf("\"empty_%dx512_us\": %.2f, ", sms, timeit([&] { empty<<<sms, 512>>>(nullptr); }));
  printf("\"empty_%dx128_us\": %.2f, ", 4 * sms, timeit([&] { empty<<<4 * sms, 128>>>(nullptr); }));
  printf("\"smem12k_%dx512_us\": %.2f}\n", sms, timeit([&] { with_smem<12288><<<sms, 512>>>(nullptr); }));
  return 0;
}
