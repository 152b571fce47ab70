// Host cost of cudaPointerGetAttributes on pageable / pinned / device pointers (measurement).
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
int main() {
  void* pg = malloc(4096);
  void* pn = nullptr;
  void* dv = nullptr;
  cudaHostAlloc(&pn, 4096, cudaHostAllocMapped);
  cudaMalloc(&dv, 4096);
  const char* names[3] = {"pageable", "pinned", "device"};
  void* ps[3] = {pg, pn, dv};
  for (int k = 0; k < 3; ++k) {
    cudaPointerAttributes at;
    for (int i = 0; i < 1000; ++i) cudaPointerGetAttributes(&at, ps[k]);
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < 100000; ++i) cudaPointerGetAttributes(&at, ps[k]);
    double us = std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count() / 100000;
    printf("{\"measure\": \"cudaPointerGetAttributes\", \"pointer\": \"%s\", \"us\": %.4f}\n", names[k], us);
  }
  return 0;
}
