// Random 64-bit atomics: rate vs buffer size (L2-resident vs HBM).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ uint64_t hidx(uint64_t i, uint64_t seed, uint64_t n) {
  uint64_t h = (i + seed) * 0x9E3779B97F4A7C15ull; h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
  return __umul64hi(h, n);
}
template <int V>
__global__ void k(u64* buf, uint64_t n8, uint64_t nops, u64* sink) {
  u64 acc = 0;
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < nops; i += (uint64_t)gridDim.x * 256) {
    u64* p = buf + hidx(i, 7, n8);
    if (V == 0) acc ^= atomicCAS(p, 0x1234ull, i);         // CAS (fails mostly)
    if (V == 1) acc ^= atomicExch(p, i);
    if (V == 2) { u64 x; asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(x) : "l"(p)); acc ^= x; }
    if (V == 3) atomicAdd(p, 1ull);                        // RED (no return)
    if (V == 4) { asm volatile("st.global.u64 [%0], %1;" :: "l"(p), "l"(i)); }
  }
  if (acc == 0x123) *sink = acc;
}
template <int V> float run(u64* buf, uint64_t n8, uint64_t nops, u64* sink) {
  unsigned grid = (unsigned)((nops + 255) / 256);
  for (int r = 0; r < 2; r++) k<V><<<grid, 256>>>(buf, n8, nops, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); k<V><<<grid, 256>>>(buf, n8, nops, sink); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms;
}
int main() {
  size_t big = 1ull << 31; u64* buf; u64* sink;
  cudaMalloc(&buf, big); cudaMemset(buf, 0, big); cudaMalloc(&sink, 8);
  const char* names[] = {"CAS", "EXCH", "LD.cg", "RED.add", "ST"};
  uint64_t nops = 1ull << 27;
  for (size_t mb : {16ul, 32ul, 64ul, 1024ul, 2048ul}) {
    uint64_t n8 = (mb << 20) / 8;
    float ms[5] = {run<0>(buf, n8, nops, sink), run<1>(buf, n8, nops, sink), run<2>(buf, n8, nops, sink),
                   run<3>(buf, n8, nops, sink), run<4>(buf, n8, nops, sink)};
    printf("buf %5zu MB:", mb);
    for (int v = 0; v < 5; v++) printf("  %s %6.1f G/s", names[v], nops / ms[v] / 1e6);
    printf("\n");
  }
  return 0;
}
