// Cost of growing a memory pool: cudaMallocFromPoolAsync of doubling sizes.
#include <cstdio>
#include <chrono>
#include <cuda_runtime.h>
int main() {
  cudaFree(0);
  cudaMemPool_t pool; cudaMemPoolProps props{}; props.allocType = cudaMemAllocationTypePinned;
  props.location.type = cudaMemLocationTypeDevice; props.location.id = 0;
  cudaMemPoolCreate(&pool, &props);
  unsigned long long thr = ~0ull; cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  cudaStream_t s; cudaStreamCreate(&s);
  void* prev = nullptr;
  for (size_t sz = 8ull << 20; sz <= (16ull << 30); sz *= 2) {
    auto t0 = std::chrono::steady_clock::now();
    void* p; cudaError_t e = cudaMallocFromPoolAsync(&p, sz, pool, s);
    cudaMemsetAsync(p, 0xFF, sz, s);
    cudaStreamSynchronize(s);
    auto t1 = std::chrono::steady_clock::now();
    if (prev) cudaFreeAsync(prev, s);
    prev = p;
    double ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
    printf("alloc+memset %8.1f MB: %8.2f ms (%s)  -> %.1f GB/s\n", sz / 1048576.0, ms, cudaGetErrorString(e), sz / ms / 1e6);
  }
  // second round: the pool is warm
  cudaStreamSynchronize(s);
  for (size_t sz = 1ull << 30; sz <= (8ull << 30); sz *= 2) {
    auto t0 = std::chrono::steady_clock::now();
    void* p; cudaMallocFromPoolAsync(&p, sz, pool, s); cudaMemsetAsync(p, 0xFF, sz, s); cudaStreamSynchronize(s);
    auto t1 = std::chrono::steady_clock::now();
    cudaFreeAsync(p, s); cudaStreamSynchronize(s);
    printf("warm %8.1f MB: %8.2f ms\n", sz / 1048576.0, std::chrono::duration<double, std::milli>(t1 - t0).count());
  }
  // plain cudaMalloc for comparison
  for (size_t sz = 1ull << 30; sz <= (8ull << 30); sz *= 2) {
    auto t0 = std::chrono::steady_clock::now();
    void* p; cudaMalloc(&p, sz); cudaMemset(p, 0xFF, sz); cudaDeviceSynchronize();
    auto t1 = std::chrono::steady_clock::now();
    cudaFree(p);
    printf("cudaMalloc %8.1f MB: %8.2f ms\n", sz / 1048576.0, std::chrono::duration<double, std::milli>(t1 - t0).count());
  }
  return 0;
}
