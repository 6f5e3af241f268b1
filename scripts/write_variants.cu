// Random writes: does a 32-byte sector write cost more than a full 64/128-byte one?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ uint64_t hidx(uint64_t i, uint64_t seed, uint64_t n) {
  uint64_t h = (i + seed) * 0x9E3779B97F4A7C15ull; h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
  return __umul64hi(h, n);
}
// V: 0 = 1 lane writes 32B at a random 64B bucket; 1 = 2 lanes write 64B bucket; 2 = 4 lanes write 128B;
//    3 = 2 lanes read 64B bucket then lane 0 writes 32B (upsert-like RMW); 4 = read 64B then both lanes write 64B
//    5 = 2 lanes read 64B then lane0 does atomicCAS on 8B; 6 = read 64B only (reference)
template <int V>
__global__ void w(u64* __restrict__ buf, uint64_t units64, uint64_t nops, u64* sink) {
  const unsigned lane = threadIdx.x & 31;
  const int G = (V == 0) ? 1 : (V == 2 ? 4 : 2);
  u64 acc = 0;
  for (uint64_t i = (blockIdx.x * 256ull + threadIdx.x) / G; i < nops; i += (uint64_t)gridDim.x * 256 / G) {
    const unsigned sub = lane % G;
    u64* p = buf + hidx(i, 1, (V == 2) ? units64 / 2 : units64) * ((V == 2) ? 16 : 8) + 4 * sub;
    u64 a = i, b = i + 1, c = i + 2, d = i + 3;
    if (V == 3 || V == 4 || V == 5 || V == 6)
      asm volatile("ld.global.cg.L2::64B.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p) : "memory");
    if (V == 0 || V == 1 || V == 2 || V == 4 || (V == 3 && sub == 0))
      asm volatile("st.global.v4.u64 [%0], {%1,%2,%3,%4};" :: "l"(p), "l"(a+1),"l"(b),"l"(c),"l"(d) : "memory");
    if (V == 5 && sub == 0) acc ^= atomicCAS((u64*)p, a, a + 1);
    acc ^= a ^ d;
  }
  if (acc == 0x123) *sink = acc;
}
template <int V> float run(u64* buf, uint64_t units64, uint64_t nops, u64* sink) {
  const int G = (V == 0) ? 1 : (V == 2 ? 4 : 2);
  unsigned grid = (unsigned)((nops * G + 255) / 256);
  for (int r = 0; r < 2; r++) w<V><<<grid, 256>>>(buf, units64, nops, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); w<V><<<grid, 256>>>(buf, units64, nops, sink); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms;
}
int main() {
  size_t bytes = 1263225856; u64* buf; u64* sink;
  cudaMalloc(&buf, bytes); cudaMemset(buf, 1, bytes); cudaMalloc(&sink, 8);
  uint64_t units64 = bytes / 64, nops = 1ull << 27;
  const char* names[] = {"write 32B (1 lane)", "write 64B (2 lanes)", "write 128B (4 lanes)", "read 64B + write 32B",
                         "read 64B + write 64B", "read 64B + CAS 8B", "read 64B only"};
  float ms[7];
  ms[0]=run<0>(buf,units64,nops,sink); ms[1]=run<1>(buf,units64,nops,sink); ms[2]=run<2>(buf,units64,nops,sink);
  ms[3]=run<3>(buf,units64,nops,sink); ms[4]=run<4>(buf,units64,nops,sink); ms[5]=run<5>(buf,units64,nops,sink);
  ms[6]=run<6>(buf,units64,nops,sink);
  for (int v = 0; v < 7; v++) printf("%-24s %8.3f ms  %7.2f G ops/s\n", names[v], ms[v], nops / ms[v] / 1e6);
  cudaError_t e = cudaGetLastError(); printf("err: %s\n", cudaGetErrorString(e));
  return 0;
}
