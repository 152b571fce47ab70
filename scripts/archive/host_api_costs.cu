// host_api_costs.cu -- host-side cost of the CUDA runtime calls one synchronous
// mcl_map_queues makes (scripts/host_overhead.py measures the whole call).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/hac scripts/host_api_costs.cu -lcuda
#include <chrono>
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>

__global__ void tiny(int* p) {
  if (threadIdx.x == 0 && p) p[0] = 1;
}

template <typename F>
double per_call_us(F f, int n = 20000) {
  for (int i = 0; i < 200; ++i) f();
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) f();
  auto t1 = std::chrono::steady_clock::now();
  return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}

int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  int* d;
  cudaMalloc(&d, 1024);
  int* hp;
  cudaHostAlloc((void**)&hp, 64, cudaHostAllocMapped);
  cudaEvent_t ev, ev_nt;
  cudaEventCreate(&ev);
  cudaEventCreateWithFlags(&ev_nt, cudaEventDisableTiming);
  cudaPointerAttributes at;
  int dev = 0;
  printf("cudaGetDevice            %.3f us\n", per_call_us([&] { cudaGetDevice(&dev); }));
  printf("cudaPointerGetAttributes %.3f us\n", per_call_us([&] { cudaPointerGetAttributes(&at, d); }));
  printf("cudaEventRecord (timing) %.3f us\n", per_call_us([&] { cudaEventRecord(ev, s); }));
  printf("cudaEventRecord (no tim) %.3f us\n", per_call_us([&] { cudaEventRecord(ev_nt, s); }));
  printf("launch (async)           %.3f us\n", per_call_us([&] { tiny<<<1, 32, 0, s>>>(d); }));
  cudaStreamSynchronize(s);
  printf("launch + streamSync      %.3f us\n", per_call_us([&] {
           tiny<<<1, 32, 0, s>>>(d);
           cudaStreamSynchronize(s);
         }));
  printf("launch + 2 events + sync %.3f us\n", per_call_us([&] {
           cudaEventRecord(ev, s);
           tiny<<<1, 32, 0, s>>>(d);
           cudaEventRecord(ev, s);
           cudaStreamSynchronize(s);
         }));
  printf("launch + poll mapped flag %.3f us\n", per_call_us([&] {
           *(volatile int*)hp = 0;
           tiny<<<1, 32, 0, s>>>(hp);
           while (*(volatile int*)hp == 0) {
           }
         }));
  printf("launch + cudaStreamQuery spin %.3f us\n", per_call_us([&] {
           tiny<<<1, 32, 0, s>>>(d);
           while (cudaStreamQuery(s) == cudaErrorNotReady) {
           }
         }));
  unsigned int* hv;
  cudaHostAlloc((void**)&hv, 64, cudaHostAllocMapped);
  unsigned int* dv;
  cudaHostGetDevicePointer((void**)&dv, hv, 0);
  CUstream cs = (CUstream)s;
  unsigned int seq = 0;
  printf("launch + cuStreamWriteValue32 + poll %.3f us\n", per_call_us([&] {
           tiny<<<1, 32, 0, s>>>(d);
           ++seq;
           cuStreamWriteValue32(cs, (CUdeviceptr)dv, seq, 0);
           while (*(volatile unsigned int*)hv != seq) {
           }
         }));
  cudaStreamSynchronize(s);
  printf("cuStreamWriteValue32 enqueue alone %.3f us\n", per_call_us([&] {
           cuStreamWriteValue32(cs, (CUdeviceptr)dv, ++seq, 0);
         }));
  cudaStreamSynchronize(s);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
