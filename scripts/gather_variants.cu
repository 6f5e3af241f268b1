// Random 32-byte gather: which load flavour fetches only one sector from HBM?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ uint64_t hidx(uint64_t i, uint64_t seed, uint64_t n) {
  uint64_t h = (i + seed) * 0x9E3779B97F4A7C15ull; h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
  return __umul64hi(h, n);
}
template <int V>
__global__ void g(const u64* __restrict__ buf, uint64_t units, uint64_t nreads, u64* sink) {
  u64 acc = 0;
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < nreads; i += (uint64_t)gridDim.x * 256) {
    const u64* p = buf + hidx(i, 1, units) * 4;
    u64 a=0,b=0,c=0,d=0;
    if (V == 0) asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p));
    if (V == 1) { asm volatile("ld.global.nc.v2.u64 {%0,%1}, [%2];" : "=l"(a),"=l"(b) : "l"(p));
                  asm volatile("ld.global.nc.v2.u64 {%0,%1}, [%2];" : "=l"(c),"=l"(d) : "l"(p+2)); }
    if (V == 2) { asm volatile("ld.global.cg.v2.u64 {%0,%1}, [%2];" : "=l"(a),"=l"(b) : "l"(p));
                  asm volatile("ld.global.cg.v2.u64 {%0,%1}, [%2];" : "=l"(c),"=l"(d) : "l"(p+2)); }
    if (V == 3) asm volatile("ld.global.cg.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p));
    if (V == 4) asm volatile("ld.global.nc.v2.u64 {%0,%1}, [%2];" : "=l"(a),"=l"(b) : "l"(p));
    if (V == 5) asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(a) : "l"(p));
    if (V == 6) asm volatile("ld.global.nc.L2::64B.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p));
    if (V == 7) asm volatile("ld.global.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p));
    if (V == 8) asm volatile("ld.relaxed.gpu.global.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(p));
    if (V == 9) asm volatile("ld.global.cs.v2.u64 {%0,%1}, [%2];" : "=l"(a),"=l"(b) : "l"(p));
    if (V >= 12) {   // G lanes cooperate on one G*32-byte region: one instruction, one line (or two)
      constexpr int G = (V == 12) ? 4 : (V == 13 ? 2 : 8);
      const unsigned lane = threadIdx.x & 31;
      const uint64_t r = hidx((i / G), 1, units / G);      // same region for the G lanes
      const u64* q = buf + r * (4 * G) + 4 * (lane % G);
      asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(a),"=l"(b),"=l"(c),"=l"(d) : "l"(q));
    } else if (V >= 10) {   // 128 B (V=10) or 256 B (V=11) aligned region, all sectors read
      const u64* q = buf + (hidx(i, 1, units / (V == 10 ? 4 : 8))) * (V == 10 ? 16 : 32);
      #pragma unroll
      for (int j = 0; j < (V == 10 ? 4 : 8); j++) {
        u64 e,f,g2,h;
        asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(e),"=l"(f),"=l"(g2),"=l"(h) : "l"(q + 4*j));
        a ^= e ^ f ^ g2 ^ h;
      }
    }
    acc ^= a ^ b ^ c ^ d;
  }
  if (acc == 0x123) *sink = acc;
}
template <int V> float run(const u64* buf, uint64_t units, uint64_t nreads, u64* sink) {
  unsigned grid = (unsigned)((nreads + 255) / 256);
  for (int w = 0; w < 2; w++) g<V><<<grid, 256>>>(buf, units, nreads, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); g<V><<<grid, 256>>>(buf, units, nreads, sink); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms;
}
int main(int argc, char** argv) {
  size_t bytes = 1263225728; u64* buf; u64* sink;
  cudaMalloc(&buf, bytes); cudaMemset(buf, 1, bytes); cudaMalloc(&sink, 8);
  uint64_t units = bytes / 32, nreads = 1ull << 28;
  if (argc > 1) { size_t g = atoi(argv[1]); cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, g); }
  size_t lim; cudaDeviceGetLimit(&lim, cudaLimitMaxL2FetchGranularity); printf("L2 fetch granularity limit %zu\n", lim);
  const char* names[] = {"nc.v4.u64(256b)", "nc.v2.u64x2", "cg.v2.u64x2", "cg.v4.u64", "nc.v2.u64(16B)", "nc.u64(8B)", "nc.L2::64B.v4", "v4.u64 plain", "relaxed.gpu.v4", "cs.v2.u64(16B)", "128B region", "256B region", "4 lanes/128B", "2 lanes/64B", "8 lanes/256B"};
  float ms[15];
  ms[0]=run<0>(buf,units,nreads,sink); ms[1]=run<1>(buf,units,nreads,sink); ms[2]=run<2>(buf,units,nreads,sink);
  ms[3]=run<3>(buf,units,nreads,sink); ms[4]=run<4>(buf,units,nreads,sink); ms[5]=run<5>(buf,units,nreads,sink);
  ms[6]=run<6>(buf,units,nreads,sink); ms[7]=run<7>(buf,units,nreads,sink); ms[8]=run<8>(buf,units,nreads,sink);
  ms[9]=run<9>(buf,units,nreads,sink); ms[10]=run<10>(buf,units,nreads,sink); ms[11]=run<11>(buf,units,nreads,sink);
  ms[12]=run<12>(buf,units,nreads,sink); ms[13]=run<13>(buf,units,nreads,sink); ms[14]=run<14>(buf,units,nreads,sink);
  for (int v = 0; v < 15; v++) printf("%-18s %8.3f ms  %7.2f G thread-reads/s  %7.2f G regions/s\n", names[v], ms[v], nreads / ms[v] / 1e6, nreads / ms[v] / 1e6 / (v==12?4:(v==13?2:(v==14?8:1))));
  return 0;
}
