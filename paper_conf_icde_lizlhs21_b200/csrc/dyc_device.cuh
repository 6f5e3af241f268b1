// dyc_device.cuh — device-side building blocks of the DyCuckoo hot path (sm_100a).
//
// Layout in HBM: subtable t is one array of n_t buckets; a bucket
// is B packed 64-bit slots {key: low 32 bits, value: high 32 bits}; an all-ones
// word is EMPTY (reading Q25/Q26).  B = 4 makes a bucket exactly one 32-byte
// DRAM/L2 sector, read by ONE 256-bit load (LDG.E.ENL2.256), so a probe of the
// two-layer scheme (§V-A) costs one sector.
//
// Hash specification (implemented independently of oracle/):
//   x_s(k)  = ((a_s * k mod p) + b_s) mod p,  p = 2^32 - 5     (Q1)
//   pair(k) : q = x_0(k) mod d(d-1); t1 = q div (d-1); r = q mod (d-1);
//             t2 = r + (r >= t1)                                (Q2)
//   bucket_t(k) = x_{t+1}(k) mod n_t
//   shard(k)    = x_{d+1}(k) mod G
// Here "mod p" folds with 2^32 = 5 (mod p) and "mod n" is Lemire's exact
// fastmod; both are bit-identical to the plain definitions for 32-bit inputs.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace dyc {

constexpr uint32_t kMaxD = 16;
constexpr uint64_t kP = 4294967291ull;
constexpr uint32_t kEmptyKey = 0xFFFFFFFFu;
constexpr unsigned long long kEmptySlot = 0xFFFFFFFFFFFFFFFFull;
constexpr unsigned kFull = 0xFFFFFFFFu;

// Per-launch view of the table (passed by value as a kernel parameter).
struct SubView {
    unsigned long long* slots;   // n * B slots
    uint64_t magic;              // fastmod magic for n
    uint32_t n;                  // buckets
    uint32_t pad;
};

struct TableView {
    SubView sub[kMaxD];
    uint32_t a[kMaxD + 2];
    uint32_t b[kMaxD + 2];
    uint32_t d;
    uint32_t d2;                 // d*(d-1)
    uint64_t magic_d2;           // fastmod magic for d2
    uint32_t dm1;                // d-1
    uint32_t recip_dm1;          // ceil(2^16/(d-1)): q div (d-1) = (q*recip)>>16 for q < 2^8
    uint32_t max_hops;
    // bit t set <=> subtable t satisfies the first-choice-full invariant (FFI,
    // DESIGN.md §5): every stored key whose FIRST choice is t but which lives in
    // its second-choice subtable has a FULL bucket h_t(k).  Then a key absent
    // from a non-full first-choice bucket of such a t is absent from the table,
    // and the second probe can be skipped.  Maintained by the host (dyc_api.cu).
    uint32_t clean;
    // measurement only (dyc_probe_count_enable): {ops, second probes} per kernel
    // kind (find, upsert, delete); nullptr in normal operation
    unsigned long long* probe;
    // the paper's balancing rule (DYC_PLACE_PAPER_WEIGHTED):
    // w[t] = n_t / max(C(m_t, 2), 1) per subtable, a snapshot taken at
    // the start of the batch; nullptr = two-choice first-fit (reading Q3)
    const float* wsel;
    // homeless pairs of lazily settled insert batches (dyc_kernels.cuh
    // stash_find) and their count (a device counter)
    unsigned long long* stash;
    const unsigned long long* stash_n;
};

// Shared-memory copy of the per-subtable fields, indexed by a lane-varying t.
struct SmemView {
    SubView sub[kMaxD];
    uint32_t a[kMaxD + 2];
    uint32_t b[kMaxD + 2];
    float w[kMaxD];              // TableView::wsel copied (0 when first-fit)
    uint32_t weighted;
};

__device__ __forceinline__ void load_view(const TableView& tv, SmemView& s) {
    const uint32_t i = threadIdx.x;
    if (i < tv.d) {
        s.sub[i] = tv.sub[i];
        s.w[i] = tv.wsel ? tv.wsel[i] : 0.f;
    }
    if (i < tv.d + 2) { s.a[i] = tv.a[i]; s.b[i] = tv.b[i]; }
    if (i == 0) s.weighted = tv.wsel != nullptr;
    __syncthreads();
}

// ---------------------------------------------------------------- arithmetic
// x mod p for any 64-bit x, p = 2^32 - 5.
__device__ __forceinline__ uint32_t mod_p(uint64_t x) {
    uint64_t r = (x >> 32) * 5ull + (x & 0xFFFFFFFFull);   // < 6 * 2^32
    r = (r >> 32) * 5ull + (r & 0xFFFFFFFFull);            // <= 2^32 + 24
    if (r >= kP) r -= kP;
    return (uint32_t)r;
}

// x_s(k) = ((a k mod p) + b) mod p.
__device__ __forceinline__ uint32_t hx(uint32_t a, uint32_t b, uint32_t k) {
    uint64_t s = (uint64_t)mod_p((uint64_t)a * k) + b;      // < 2p
    if (s >= kP) s -= kP;
    return (uint32_t)s;
}

// Lemire fastmod: x mod n, exact for 32-bit x and n >= 1 (magic = floor((2^64-1)/n)+1).
__device__ __forceinline__ uint32_t fastmod(uint32_t x, uint64_t magic, uint32_t n) {
    return (uint32_t)__umul64hi(magic * (uint64_t)x, (uint64_t)n);
}

struct Pair { uint32_t t1, t2; };

__device__ __forceinline__ Pair pair_of(const TableView& tv, uint32_t k) {
    uint32_t q = fastmod(hx(tv.a[0], tv.b[0], k), tv.magic_d2, tv.d2);
    uint32_t f = (q * tv.recip_dm1) >> 16;
    uint32_t r = q - f * tv.dm1;
    return Pair{f, r + (r >= f ? 1u : 0u)};
}

// The paper's initial table choice (also after an upsize P:L384): a new
// pair goes to table i of its pair with probability proportional to
// n_i / C(m_i, 2).  The uniform draw is a hash of the key (counter-based, so a
// key's choice is fixed within a batch).  Returns true for the second table.
__device__ __forceinline__ bool weighted_second(const SmemView& s, uint32_t t1, uint32_t t2, uint32_t k) {
    const float w1 = s.w[t1], w2 = s.w[t2];
    uint32_t x = k ^ 0x2545F491u;
    x ^= x >> 16; x *= 0x7FEB352Du; x ^= x >> 15; x *= 0x846CA68Bu; x ^= x >> 16;
    const float u = (float)(x >> 8) * (1.0f / 16777216.0f);
    return u * (w1 + w2) >= w1;
}

__device__ __forceinline__ uint32_t bucket_of(const SmemView& s, uint32_t t, uint32_t k) {
    return fastmod(hx(s.a[t + 1], s.b[t + 1], k), s.sub[t].magic, s.sub[t].n);
}

__device__ __forceinline__ unsigned long long* bucket_ptr(const SmemView& s, uint32_t t, uint32_t b, int B) {
    return s.sub[t].slots + (uint64_t)b * B;
}

__device__ __forceinline__ uint32_t key_of(unsigned long long e) { return (uint32_t)e; }
__device__ __forceinline__ uint32_t val_of(unsigned long long e) { return (uint32_t)(e >> 32); }
__device__ __forceinline__ unsigned long long make_kv(uint32_t k, uint32_t v) {
    return (unsigned long long)k | ((unsigned long long)v << 32);
}

// ---------------------------------------------------------------- loads/stores
// Each lane reads 4 slots (32 bytes) of its group's bucket with ONE 256-bit load
// (LDG.E.ENL2.256).  The L2 prefetch-size qualifier is matched to the bucket:
// without it a miss pulls a whole 128-byte line from HBM (measured: 3.7-3.9
// DRAM sectors per 32- or 64-byte random request), so 64-byte buckets ask for
// .L2::64B and halve the HBM bytes per probe.
template <int B> struct Pf;                      // L2 prefetch size per bucket width
template <> struct Pf<4>  { static constexpr const char* q = ".L2::64B"; };
template <> struct Pf<8>  { static constexpr const char* q = ".L2::64B"; };
template <> struct Pf<16> { static constexpr const char* q = ".L2::128B"; };
template <> struct Pf<32> { static constexpr const char* q = ".L2::256B"; };

#define DYC_LD4(NAME, COP, PF)                                                                   \
    __device__ __forceinline__ void NAME(const unsigned long long* p, unsigned long long* s) {    \
        asm volatile("ld.global" COP PF ".v4.u64 {%0,%1,%2,%3}, [%4];"                            \
                     : "=l"(s[0]), "=l"(s[1]), "=l"(s[2]), "=l"(s[3]) : "l"(p) : "memory");       \
    }                                                                                            \
    __device__ __forceinline__ void NAME##_pred(const unsigned long long* p, unsigned long long* s, \
                                                bool pred) {                                     \
        asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %5, 0;\n\t"                          \
                     "@q ld.global" COP PF ".v4.u64 {%0,%1,%2,%3}, [%4];\n\t}"                  \
                     : "+l"(s[0]), "+l"(s[1]), "+l"(s[2]), "+l"(s[3])                             \
                     : "l"(p), "r"((unsigned)pred) : "memory");                                  \
    }

// read-only probes (find): non-coherent path, no L1 allocation (no reuse)
DYC_LD4(ld4_nc_64, ".nc.L1::no_allocate", ".L2::64B")
DYC_LD4(ld4_nc_128, ".nc.L1::no_allocate", ".L2::128B")
DYC_LD4(ld4_nc_256, ".nc.L1::no_allocate", ".L2::256B")
// probes in kernels that mutate the table: served by L2 (coherent)
DYC_LD4(ld4_cg_64, ".cg", ".L2::64B")
DYC_LD4(ld4_cg_128, ".cg", ".L2::128B")
DYC_LD4(ld4_cg_256, ".cg", ".L2::256B")
#undef DYC_LD4

template <int B>
__device__ __forceinline__ void probe_nc(const unsigned long long* p, unsigned long long* s) {
    if (B <= 8) ld4_nc_64(p, s); else if (B == 16) ld4_nc_128(p, s); else ld4_nc_256(p, s);
}
template <int B>
__device__ __forceinline__ void probe_nc_pred(const unsigned long long* p, unsigned long long* s, bool q) {
    if (B <= 8) ld4_nc_64_pred(p, s, q); else if (B == 16) ld4_nc_128_pred(p, s, q); else ld4_nc_256_pred(p, s, q);
}
template <int B>
__device__ __forceinline__ void probe_cg(const unsigned long long* p, unsigned long long* s) {
    if (B <= 8) ld4_cg_64(p, s); else if (B == 16) ld4_cg_128(p, s); else ld4_cg_256(p, s);
}
template <int B>
__device__ __forceinline__ void probe_cg_pred(const unsigned long long* p, unsigned long long* s, bool q) {
    if (B <= 8) ld4_cg_64_pred(p, s, q); else if (B == 16) ld4_cg_128_pred(p, s, q); else ld4_cg_256_pred(p, s, q);
}

// plain 256-bit streaming read (measurement kernels)
__device__ __forceinline__ void ld4_nc(const unsigned long long* p, unsigned long long* s) {
    asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];"
                 : "=l"(s[0]), "=l"(s[1]), "=l"(s[2]), "=l"(s[3]) : "l"(p));
}

// Value of key k in a 4-slot snapshot (branch-free select chain).
template <int B>
__device__ __forceinline__ bool lookup_slot(const unsigned long long (&s)[B], uint32_t k, uint32_t& v) {
    bool f = false;
#pragma unroll
    for (int j = 0; j < B; j++) {
        const bool h = key_of(s[j]) == k;
        v = h ? val_of(s[j]) : v;
        f |= h;
    }
    return f;
}

template <int B>
__device__ __forceinline__ int match_slot(const unsigned long long (&s)[B], uint32_t k) {
    int hit = -1;
#pragma unroll
    for (int j = B - 1; j >= 0; --j)
        if (key_of(s[j]) == k) hit = j;
    return hit;
}

// Slot atomics on global memory (ATOMG, no generic-address check).
__device__ __forceinline__ unsigned long long cas_slot(unsigned long long* p, unsigned long long cmp,
                                                       unsigned long long v) {
    unsigned long long old;
    asm volatile("atom.global.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "l"(p), "l"(cmp), "l"(v) : "memory");
    return old;
}
// Predicated CAS (no branch around it, so several can be in flight at once);
// returns `dflt` when pred is false.
__device__ __forceinline__ unsigned long long cas_slot_pred(unsigned long long* p, unsigned long long cmp,
                                                            unsigned long long v, bool pred,
                                                            unsigned long long dflt) {
    unsigned long long old = dflt;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %4, 0;\n\t"
                 "@q atom.global.cas.b64 %0, [%1], %2, %3;\n\t}"
                 : "+l"(old) : "l"(p), "l"(cmp), "l"(v), "r"((unsigned)pred) : "memory");
    return old;
}
__device__ __forceinline__ unsigned long long exch_slot(unsigned long long* p, unsigned long long v) {
    unsigned long long old;
    asm volatile("atom.global.exch.b64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ void st_u64_cg(unsigned long long* p, unsigned long long v) {
    asm volatile("st.global.cg.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Warp-aggregated append: every lane of the (converged) warp calls it; lanes with
// pred write `v` to list[cursor++].  One atomic per warp.
__device__ __forceinline__ void warp_append(bool pred, unsigned long long v, unsigned long long* list,
                                            unsigned long long* counter) {
    const unsigned m = __ballot_sync(kFull, pred);
    if (m == 0) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(m) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(counter, (unsigned long long)__popc(m));
    base = __shfl_sync(kFull, base, leader);
    if (pred) list[base + __popc(m & lanemask_lt())] = v;
}

// Block-wide sum of a per-thread counter, one atomicAdd per block.
template <int NT>
__device__ __forceinline__ void block_add(unsigned long long* dst, unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    __shared__ unsigned long long red[NT / 32];
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) red[w] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long s = 0;
#pragma unroll
        for (int i = 0; i < NT / 32; i++) s += red[i];
        if (s) atomicAdd(dst, s);
    }
    __syncthreads();
}

}  // namespace dyc
