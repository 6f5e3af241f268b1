// dyw_kernels.cuh — sm_100a kernels of the WIDE-key DyCuckoo variant (SURVEY
// §8(f) NEXT-3): 64-bit keys, values of W 64-bit words ("Suppose
// the keys are 8-bytes, a bucket can then accommodate 16 KV pairs ... we lock
// the entire bucket exclusively for a warp to perform insertion/deletion").
//
// Two layouts, three placement modes (include/dycuckoo_wide.h):
//   SEP  (paper layout): a bucket is 16 keys = one 128-byte line;
//        the W-word values live in a separate array at the same slot index, so
//        a find that misses or a delete never touches them.  Insertion takes a
//        per-bucket lock (atomicCAS 0->1, release atomicExch -> 0):
//          VOTER   — Alg. 1 as printed: one op per thread; the
//                    warp elects a leader with ballot, the leader try-locks its
//                    bucket, the warp inspects it cooperatively; a failed lock
//                    makes the warp re-vote (reading Q30: lanes that failed
//                    this round are skipped until every active lane has tried).
//          GROUPED — the sm_100a redesign: every lane drives its own op and
//                    try-locks its own bucket in the same round (32 lock round
//                    trips in flight per warp instead of one); lanes whose
//                    buckets coincide are grouped with __match_any_sync so
//                    only one of them asks for the lock; the lock holder scans
//                    the 128-byte bucket alone (four 32-byte loads).
//   PACK (LOCKFREE, W = 1): a slot is one 16-byte {key, value} word pair and a
//        bucket 8 slots = 128 bytes; Blackwell's 128-bit atomics
//        (ATOMG.E.CAS.128 / EXCH.128) move a whole pair at once, so placement
//        needs no lock at all — the same CAS-into-EMPTY / exchange-with-victim
//        scheme as the 32-bit table (dyc_kernels.cuh).
//
// Find and delete are lock-free in every mode, one lane group per
// op: G = B lanes each reading one slot, so one probe = one 128-byte line.
#pragma once
#include "dyc_device.cuh"

namespace dyw {

using dyc::kFull;
using dyc::kMaxD;
using dyc::fastmod;
using dyc::mod_p;
using dyc::lanemask_lt;
using u64 = unsigned long long;

constexpr int kThreads = 256;
constexpr u64 kE = 0xFFFFFFFFFFFFFFFFull;     // EMPTY key (reserved) and empty value word
enum Layout : int { SEP = 0, PACK = 1 };
template <int L> struct Lay;
template <> struct Lay<SEP>  { static constexpr int B = 16; };
template <> struct Lay<PACK> { static constexpr int B = 8; };

enum Ctr : int {
    W_PENDING = 0, W_INSERTED = 1, W_UPDATED = 2, W_FAIL = 3, W_EVICT = 4, W_REMOVED = 5,
    W_RESIDUAL = 6, W_DUMP = 7, W_LOCKFAIL = 8, W_RES_TOTAL = 9, W_COUNT0 = 16, W_N = 32
};

struct WSub {
    u64* keys;          // SEP: n*16 keys; PACK: n*8 {key, value} pairs (2 words each)
    u64* vals;          // SEP: n*16*W value words; PACK: unused
    uint32_t* locks;    // SEP: one lock word per bucket; PACK: unused
    uint64_t magic;
    uint32_t n;
    uint32_t pad;
};

struct WView {
    WSub sub[kMaxD];
    uint32_t a[kMaxD + 2], b[kMaxD + 2], c[kMaxD + 2];
    uint32_t d, d2;
    uint64_t magic_d2;
    uint32_t dm1, max_hops;
};

struct WSmem {
    WSub sub[kMaxD];
    uint32_t a[kMaxD + 2], b[kMaxD + 2], c[kMaxD + 2];
};

__device__ __forceinline__ void load_wview(const WView& tv, WSmem& s) {
    const uint32_t i = threadIdx.x;
    if (i < tv.d) s.sub[i] = tv.sub[i];
    if (i < tv.d + 2) { s.a[i] = tv.a[i]; s.b[i] = tv.b[i]; s.c[i] = tv.c[i]; }
    __syncthreads();
}

// Reading Q33: x_s(k) = (c_s*hi(k) + a_s*lo(k) + b_s) mod p (the 32-bit x_s when hi = 0).
__device__ __forceinline__ uint32_t hxw(uint32_t a, uint32_t b, uint32_t c, u64 k) {
    const uint64_t x = (uint64_t)mod_p((uint64_t)c * (uint32_t)(k >> 32)) + mod_p((uint64_t)a * (uint32_t)k) + b;
    return mod_p(x);
}

struct WPair { uint32_t t1, t2; };

__device__ __forceinline__ WPair wpair(const WView& tv, u64 k) {
    const uint32_t q = fastmod(hxw(tv.a[0], tv.b[0], tv.c[0], k), tv.magic_d2, tv.d2);
    const uint32_t f = q / tv.dm1;
    const uint32_t r = q - f * tv.dm1;
    return WPair{f, r + (r >= f ? 1u : 0u)};
}

__device__ __forceinline__ uint32_t wbucket(const WSmem& s, uint32_t t, u64 k) {
    return fastmod(hxw(s.a[t + 1], s.b[t + 1], s.c[t + 1], k), s.sub[t].magic, s.sub[t].n);
}

__device__ __forceinline__ uint32_t wpartner(const WView& tv, u64 k, uint32_t t) {
    const WPair p = wpair(tv, k);
    return t == p.t1 ? p.t2 : p.t1;
}

__device__ __forceinline__ uint32_t mix64(u64 x) {
    x ^= x >> 33; x *= 0xFF51AFD7ED558CCDull; x ^= x >> 33;
    return (uint32_t)x;
}

// ------------------------------------------------------------------ memory ops
__device__ __forceinline__ u64 ld_key_nc(const u64* p) {
    u64 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::128B.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ u64 ld_cg(const u64* p) {
    u64 v;
    asm volatile("ld.global.cg.L2::128B.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void ld_pair_nc(const u64* p, u64& k, u64& v) {
    asm volatile("ld.global.nc.L1::no_allocate.L2::128B.v2.u64 {%0,%1}, [%2];" : "=l"(k), "=l"(v) : "l"(p));
}
__device__ __forceinline__ void ld_pair_cg(const u64* p, u64& k, u64& v) {
    asm volatile("ld.global.cg.L2::128B.v2.u64 {%0,%1}, [%2];" : "=l"(k), "=l"(v) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_cg(u64* p, u64 v) {
    asm volatile("st.global.cg.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_pair(u64* p, u64 k, u64 v) {
    asm volatile("st.global.cg.v2.u64 [%0], {%1,%2};" :: "l"(p), "l"(k), "l"(v) : "memory");
}
// 128-bit atomics on a {key, value} pair (Blackwell: ATOMG.E.CAS.128 / EXCH.128)
__device__ __forceinline__ void cas128(u64* p, u64 ck, u64 cv, u64 nk, u64 nv, u64& ok, u64& ov) {
    asm volatile("{\n\t.reg .b128 d, c, n;\n\t"
                 "mov.b128 c, {%2, %3};\n\tmov.b128 n, {%4, %5};\n\t"
                 "atom.global.cas.b128 d, [%6], c, n;\n\t"
                 "mov.b128 {%0, %1}, d;\n\t}"
                 : "=l"(ok), "=l"(ov) : "l"(ck), "l"(cv), "l"(nk), "l"(nv), "l"(p) : "memory");
}
__device__ __forceinline__ void exch128(u64* p, u64 nk, u64 nv, u64& ok, u64& ov) {
    asm volatile("{\n\t.reg .b128 d, n;\n\t"
                 "mov.b128 n, {%2, %3};\n\t"
                 "atom.global.exch.b128 d, [%4], n;\n\t"
                 "mov.b128 {%0, %1}, d;\n\t}"
                 : "=l"(ok), "=l"(ov) : "l"(nk), "l"(nv), "l"(p) : "memory");
}

template <int W>
__device__ __forceinline__ void ld_vals(const u64* p, u64 (&v)[W], bool nc) {
    if (W == 1) {
        v[0] = nc ? ld_key_nc(p) : ld_cg(p);
    } else if (W == 2) {
        if (nc) asm volatile("ld.global.nc.L1::no_allocate.v2.u64 {%0,%1}, [%2];" : "=l"(v[0]), "=l"(v[1]) : "l"(p));
        else asm volatile("ld.global.cg.v2.u64 {%0,%1}, [%2];" : "=l"(v[0]), "=l"(v[1]) : "l"(p) : "memory");
    } else {
#pragma unroll
        for (int w = 0; w < W; w += 4) {
            if (nc)
                asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];"
                             : "=l"(v[w]), "=l"(v[w + 1]), "=l"(v[w + 2]), "=l"(v[w + 3]) : "l"(p + w));
            else
                asm volatile("ld.global.cg.v4.u64 {%0,%1,%2,%3}, [%4];"
                             : "=l"(v[w]), "=l"(v[w + 1]), "=l"(v[w + 2]), "=l"(v[w + 3]) : "l"(p + w) : "memory");
        }
    }
}

template <int W>
__device__ __forceinline__ void st_vals(u64* p, const u64 (&v)[W]) {
    if (W == 1) {
        st_cg(p, v[0]);
    } else if (W == 2) {
        asm volatile("st.global.cg.v2.u64 [%0], {%1,%2};" :: "l"(p), "l"(v[0]), "l"(v[1]) : "memory");
    } else {
#pragma unroll
        for (int w = 0; w < W; w += 4)
            asm volatile("st.global.cg.v4.u64 [%0], {%1,%2,%3,%4};"
                         :: "l"(p + w), "l"(v[w]), "l"(v[w + 1]), "l"(v[w + 2]), "l"(v[w + 3]) : "memory");
    }
}

// A list of (key, W-word value) records: pending inserts, failures, residuals.
struct KVList {
    u64* keys;
    u64* vals;
};

// Group-aggregated append: lanes with pred (at most one per group in callers)
// write a record.  One atomic per warp.
template <int W>
__device__ __forceinline__ void kv_append(bool pred, u64 k, const u64 (&v)[W], KVList l, u64* counter) {
    const unsigned m = __ballot_sync(kFull, pred);
    if (m == 0) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(m) - 1;
    u64 base = 0;
    if (lane == leader) base = atomicAdd(counter, (u64)__popc(m));
    base = __shfl_sync(kFull, base, leader);
    if (pred) {
        const u64 at = base + __popc(m & lanemask_lt());
        l.keys[at] = k;
#pragma unroll
        for (int w = 0; w < W; w++) l.vals[at * W + w] = v[w];
    }
}

// Block-aggregated append of up to R records per thread: ONE global atomic per
// block per call (a single list cursor hit by every warp serializes at the L2
// atomic unit; measured ~1 G atomics/s).  Every thread of the block must call it.
template <int W, int R>
__device__ __forceinline__ void block_append(const bool (&pred)[R], const u64 (&k)[R], const u64 (&v)[R][W],
                                             KVList l, u64* counter) {
    __shared__ unsigned s_cnt;
    __shared__ u64 s_base;
    const unsigned lane = threadIdx.x & 31;
    unsigned c = 0;
#pragma unroll
    for (int r = 0; r < R; r++) c += pred[r] ? 1u : 0u;
    unsigned inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(kFull, inc, o);
        if (lane >= (unsigned)o) inc += y;
    }
    const unsigned wtot = __shfl_sync(kFull, inc, 31);
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    unsigned woff = 0;
    if (lane == 31 && wtot) woff = atomicAdd(&s_cnt, wtot);
    woff = __shfl_sync(kFull, woff, 31);
    __syncthreads();
    if (threadIdx.x == 0) s_base = s_cnt ? atomicAdd(counter, (u64)s_cnt) : 0ull;
    __syncthreads();
    u64 at = s_base + woff + (inc - c);
#pragma unroll
    for (int r = 0; r < R; r++) {
        if (pred[r]) {
            l.keys[at] = k[r];
#pragma unroll
            for (int q = 0; q < W; q++) l.vals[at * W + q] = v[r][q];
            at++;
        }
    }
}

template <int NT>
__device__ __forceinline__ void wblock_add(u64* dst, u64 v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    __shared__ u64 red[NT / 32];
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) red[w] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        u64 s = 0;
#pragma unroll
        for (int i = 0; i < NT / 32; i++) s += red[i];
        if (s) atomicAdd(dst, s);
    }
    __syncthreads();
}

// Lane group of G = B lanes; lane `sub` holds slot `sub` of the group's bucket.
template <int G>
struct WGrp {
    unsigned lane, sub, base, gmask;
    __device__ __forceinline__ WGrp() {
        lane = threadIdx.x & 31;
        sub = lane & (G - 1);
        base = lane - sub;
        gmask = (G == 32) ? kFull : (((1u << G) - 1u) << base);
    }
    __device__ __forceinline__ unsigned ballot(bool p) const { return (__ballot_sync(kFull, p) & gmask) >> base; }
    __device__ __forceinline__ u64 bcast(u64 v, unsigned src) const { return __shfl_sync(kFull, v, base + src); }
};

__device__ __forceinline__ unsigned lowest(unsigned bits) { return bits ? (unsigned)(__ffs(bits) - 1) : 0u; }

// One slot of a bucket as seen by its lane: key and (PACK) value.
template <int L>
__device__ __forceinline__ void probe_slot(const WSmem& sv, uint32_t t, uint32_t b, unsigned s, bool nc, bool pred,
                                           u64& k, u64& v) {
    constexpr int B = Lay<L>::B;
    k = kE;
    v = kE;
    if (!pred) return;
    if (L == SEP) {
        const u64* p = sv.sub[t].keys + (uint64_t)b * B + s;
        k = nc ? ld_key_nc(p) : ld_cg(p);
    } else {
        const u64* p = sv.sub[t].keys + ((uint64_t)b * B + s) * 2;
        if (nc) ld_pair_nc(p, k, v); else ld_pair_cg(p, k, v);
    }
}

// Both probes of U ops of a lane group, all loads of a round issued together
// (memory-level parallelism: the kernels are bound by random line requests).
// Per op: the hit (group-relative lane mask, table, bucket; PACK: the value
// word the hit lane read) and, for the upsert, the EMPTY masks of both buckets.
template <int L, int U>
struct Probe2 {
    u64 k[U];
    bool act[U];
    WPair p[U];
    uint32_t b1[U], b2[U];
    unsigned hb[U], em1[U], em2[U];
    uint32_t ht[U], hbk[U];
    u64 hv[U];

    template <int G>
    __device__ __forceinline__ void run(const WView& tv, const WSmem& sv, const WGrp<G>& g, const u64* keys,
                                        uint64_t n, uint64_t base, unsigned grp, bool nc) {
        constexpr int QPW = 32 / G;
        static_assert(U <= G, "one hashing lane per op");
        // the three hashes of op u are computed once, by lane u of the group, and
        // broadcast (computing them on all G lanes made the kernels ALU-bound)
        u64 mk = kE;
        uint32_t mt = 0, m1 = 0, m2 = 0;
        if (g.sub < (unsigned)U) {
            const uint64_t i = base + (uint64_t)g.sub * QPW + grp;
            mk = i < n ? __ldg(keys + i) : kE;
            const WPair mp = wpair(tv, mk);
            mt = mp.t1 | (mp.t2 << 16);
            m1 = wbucket(sv, mp.t1, mk);
            m2 = wbucket(sv, mp.t2, mk);
        }
        u64 sk[U], sval[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            k[u] = g.bcast(mk, u);
            const uint32_t tt = __shfl_sync(kFull, mt, g.base + u);
            p[u] = WPair{tt & 0xFFFFu, tt >> 16};
            b1[u] = __shfl_sync(kFull, m1, g.base + u);
            b2[u] = __shfl_sync(kFull, m2, g.base + u);
            act[u] = k[u] != kE;
            probe_slot<L>(sv, p[u].t1, b1[u], g.sub, nc, act[u], sk[u], sval[u]);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            hb[u] = g.ballot(act[u] && sk[u] == k[u]);
            em1[u] = g.ballot(act[u] && sk[u] == kE);
            ht[u] = p[u].t1;
            hbk[u] = b1[u];
            hv[u] = sval[u];
        }
#pragma unroll
        for (int u = 0; u < U; u++) probe_slot<L>(sv, p[u].t2, b2[u], g.sub, nc, act[u] && !hb[u], sk[u], sval[u]);
#pragma unroll
        for (int u = 0; u < U; u++) {
            const bool need = act[u] && !hb[u];
            const unsigned h2 = g.ballot(need && sk[u] == k[u]);
            em2[u] = g.ballot(need && sk[u] == kE);
            if (need && h2) {
                hb[u] = h2;
                ht[u] = p[u].t2;
                hbk[u] = b2[u];
                hv[u] = sval[u];
            }
        }
    }
};

// ------------------------------------------------------------------ find (S3)
template <int L, int W, int U>
__global__ void __launch_bounds__(kThreads) k_wfind(WView tv, const u64* __restrict__ keys, u64* __restrict__ out,
                                                    uint8_t* __restrict__ found, uint64_t n) {
    constexpr int G = Lay<L>::B, QPW = 32 / G;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const WGrp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    for (uint64_t base = w * QPW * U; base < n; base += nwarps * QPW * U) {
        Probe2<L, U> pr;
        pr.run(tv, sv, g, keys, n, base, grp, true);
        u64 v[U][W];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const bool mine = pr.hb[u] && g.sub == lowest(pr.hb[u]);
#pragma unroll
            for (int q = 0; q < W; q++) v[u][q] = kE;
            if (L == SEP) {
                if (mine) ld_vals<W>(sv.sub[pr.ht[u]].vals + ((uint64_t)pr.hbk[u] * G + g.sub) * W, v[u], true);
            } else {
                v[u][0] = pr.hv[u];
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint64_t i = base + (uint64_t)u * QPW + grp;
            if (i >= n) continue;
            const bool hit = pr.hb[u] != 0;
            const bool writer = hit ? g.sub == lowest(pr.hb[u]) : g.sub == 0;
            if (writer) {
                if (out) {
#pragma unroll
                    for (int q = 0; q < W; q++) out[i * W + q] = hit ? v[u][q] : kE;
                }
                if (found) found[i] = hit ? 1 : 0;
            }
        }
    }
}

// --------------------------------------------------- insert phase 1 (S5)
// Probe both candidate buckets; an existing key gets its value words replaced
// in place (Alg. 1, status UPDATED; no lock is needed: keys never
// move during this kernel and keys in a batch are distinct).  A new key
// (status INSERTED) is, with FUSE (PACK only), CAS-ed into a free slot of its
// first-fit bucket; otherwise it is appended to `pending` for placement.
template <int L, int W, bool FUSE, int U>
__global__ void __launch_bounds__(kThreads) k_wupsert(WView tv, const u64* __restrict__ keys,
                                                      const u64* __restrict__ vals, uint8_t* __restrict__ status,
                                                      uint64_t n, KVList pending, u64* __restrict__ ctr) {
    constexpr int G = Lay<L>::B, QPW = 32 / G;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const WGrp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    u64 n_ins = 0, n_upd = 0;
    constexpr uint64_t per_block = (uint64_t)(kThreads / 32) * QPW * U;
    (void)w;
    (void)nwarps;
    for (uint64_t bbase = (uint64_t)blockIdx.x * per_block; bbase < n; bbase += (uint64_t)gridDim.x * per_block) {
        const uint64_t base = bbase + (uint64_t)(threadIdx.x >> 5) * QPW * U;   // block-uniform trip count
        Probe2<L, U> pr;
        pr.run(tv, sv, g, keys, n, base, grp, false);
        u64 v[U][W];
        bool isnew[U], placed[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint64_t i = base + (uint64_t)u * QPW + grp;
#pragma unroll
            for (int q = 0; q < W; q++) v[u][q] = pr.act[u] ? __ldg(vals + i * W + q) : 0ull;
            if (pr.hb[u] && g.sub == lowest(pr.hb[u])) {
                if (L == SEP) st_vals<W>(sv.sub[pr.ht[u]].vals + ((uint64_t)pr.hbk[u] * G + g.sub) * W, v[u]);
                else st_cg(sv.sub[pr.ht[u]].keys + ((uint64_t)pr.hbk[u] * G + g.sub) * 2 + 1, v[u][0]);
            }
            isnew[u] = pr.act[u] && !pr.hb[u];
            placed[u] = false;
        }
        if (FUSE && L == PACK) {
            // first-fit CAS128 into the free pairs of t1, then t2; every round the
            // U ops of the group each issue one CAS, so their round trips overlap
#pragma unroll
            for (int h = 0; h < 2; h++) {
                unsigned e[U];
#pragma unroll
                for (int u = 0; u < U; u++) e[u] = isnew[u] ? (h ? pr.em2[u] : pr.em1[u]) : 0u;
                for (;;) {
                    unsigned cand[U];
                    bool any = false;
#pragma unroll
                    for (int u = 0; u < U; u++) {
                        cand[u] = g.ballot(!placed[u] && e[u] != 0);
                        any |= cand[u] != 0;
                    }
                    if (!__any_sync(kFull, any)) break;
                    bool ok[U];
#pragma unroll
                    for (int u = 0; u < U; u++) {
                        ok[u] = false;
                        if (cand[u] && g.sub == lowest(e[u])) {
                            const uint32_t t = h ? pr.p[u].t2 : pr.p[u].t1;
                            const uint32_t bb = h ? pr.b2[u] : pr.b1[u];
                            u64 ok_, ov_;
                            cas128(sv.sub[t].keys + ((uint64_t)bb * G + g.sub) * 2, kE, kE, pr.k[u], v[u][0], ok_, ov_);
                            ok[u] = ok_ == kE && ov_ == kE;
                        }
                    }
#pragma unroll
                    for (int u = 0; u < U; u++) {
                        const unsigned okb = g.ballot(ok[u]);
                        if (cand[u]) {
                            if (okb) placed[u] = true;
                            else e[u] &= ~(1u << lowest(e[u]));
                        }
                    }
                }
            }
        }
        const bool lead = g.sub == 0;
        bool app[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint64_t i = base + (uint64_t)u * QPW + grp;
            if (lead && i < n && status) status[i] = pr.act[u] ? (pr.hb[u] ? 2 : 1) : 0;
            app[u] = lead && isnew[u] && !placed[u];
            n_ins += lead && isnew[u];
            n_upd += lead && pr.act[u] && pr.hb[u];
        }
        block_append<W, U>(app, pr.k, v, pending, ctr + W_PENDING);
    }
    wblock_add<kThreads>(ctr + W_INSERTED, n_ins);
    wblock_add<kThreads>(ctr + W_UPDATED, n_upd);
}

// ----------------------------------------------- insert phase 2: VOTER (SEP)
// Algorithm 1 over the records list[0 .. cnt): one record per
// thread; per round the warp elects a leader among its active lanes (ballot),
// the leader try-locks its target bucket (atomicCAS 0 -> 1), the warp reads the
// bucket (lane s: key s) and the leader writes its pair into the first EMPTY
// slot, or — after both first-fit tries (reading Q3) — swaps it with a
// pseudo-random victim (Q5) and carries the victim to the other table of ITS
// pair.  Unlock is atomicExch -> 0 after a fence.  A failed lock makes
// the warp re-vote among the lanes that have not failed this round (Q30).
template <int W>
__global__ void __launch_bounds__(kThreads) k_wplace_voter(WView tv, KVList src, const u64* count_ptr,
                                                           uint64_t count_host, KVList fail, u64* __restrict__ ctr) {
    constexpr int B = 16;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const unsigned lane = threadIdx.x & 31;
    const uint64_t cnt = count_ptr ? *(volatile const u64*)count_ptr : count_host;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t wid = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    u64 ev = 0, lockfail = 0;
    for (uint64_t base = wid * 32; base < cnt; base += nwarps * 32) {
        const uint64_t i = base + lane;
        bool active = i < cnt;
        u64 k = active ? src.keys[i] : kE;
        u64 v[W];
#pragma unroll
        for (int q = 0; q < W; q++) v[q] = active ? src.vals[i * W + q] : 0ull;
        WPair p0 = wpair(tv, k);
        uint32_t t = p0.t1, hop = 0;
        int phase = 0;                                 // 0/1 first-fit t1/t2, 2 evicting
        unsigned tried = 0;
        for (;;) {
            const unsigned act = __ballot_sync(kFull, active);
            if (!act) break;
            unsigned cand = act & ~tried;
            if (!cand) { tried = 0; cand = act; }
            const unsigned l = __ffs(cand) - 1;
            const u64 lk = __shfl_sync(kFull, k, l);
            const uint32_t lt = __shfl_sync(kFull, t, l);
            const int lph = __shfl_sync(kFull, phase, l);
            const uint32_t lhop = __shfl_sync(kFull, hop, l);
            const uint32_t b = wbucket(sv, lt, lk);
            uint32_t* lock = sv.sub[lt].locks + b;
            int ok = 0;
            if (lane == l) ok = atomicCAS(lock, 0u, 1u) == 0u;
            ok = __shfl_sync(kFull, ok, l);
            if (!ok) {
                tried |= 1u << l;
                lockfail += lane == l;
                continue;
            }
            __threadfence();
            u64* kp = sv.sub[lt].keys + (uint64_t)b * B;
            u64* vp = sv.sub[lt].vals + (uint64_t)b * B * W;
            const u64 sk = lane < B ? ld_cg(kp + lane) : 0ull;
            const unsigned em = __ballot_sync(kFull, lane < B && sk == kE);
            const unsigned vs = (mix64(lk ^ ((u64)lhop * 0x9E3779B97F4A7C15ull)) >> 8) & (B - 1);
            const u64 victim_k = __shfl_sync(kFull, sk, vs);
            if (lane == l) {
                if (em) {                                           // Alg. 1
                    const unsigned s = __ffs(em) - 1;
                    st_vals<W>(vp + (uint64_t)s * W, v);
                    st_cg(kp + s, k);
                    active = false;
                } else if (lph < 2) {                               // first-fit t2, then start evicting
                    if (lph == 0) { phase = 1; t = p0.t2; }
                    else { phase = 2; hop = 0; t = (mix64(k) & 1u) ? p0.t2 : p0.t1; }
                } else {                                            // Alg. 1: swap with a victim
                    u64 ov[W];
                    ld_vals<W>(vp + (uint64_t)vs * W, ov, false);
                    st_vals<W>(vp + (uint64_t)vs * W, v);
                    st_cg(kp + vs, k);
                    k = victim_k;
#pragma unroll
                    for (int q = 0; q < W; q++) v[q] = ov[q];
                    ev++;
                    hop++;
                    p0 = wpair(tv, k);
                    t = (lt == p0.t1) ? p0.t2 : p0.t1;
                    if (hop >= tv.max_hops) {                       // failure list
                        const u64 at = atomicAdd(ctr + W_FAIL, 1ull);
                        fail.keys[at] = k;
#pragma unroll
                        for (int q = 0; q < W; q++) fail.vals[at * W + q] = v[q];
                        active = false;
                    }
                }
                __threadfence();
                atomicExch(lock, 0u);
            }
        }
    }
    wblock_add<kThreads>(ctr + W_EVICT, ev);
    wblock_add<kThreads>(ctr + W_LOCKFAIL, lockfail);
}

// --------------------------------------------- insert phase 2: GROUPED (SEP)
// Every lane drives its own record and, each round, try-locks its own target
// bucket; lanes of a warp that target the same bucket are grouped with
// __match_any_sync and only the lowest asks (the others would fail anyway).
// The holder scans the bucket alone (4 x 32-byte loads of the 128-byte line).
// Warps pull new records into idle lanes from their own range of the list.
template <int W>
__global__ void __launch_bounds__(kThreads) k_wplace_grouped(WView tv, KVList src, const u64* count_ptr,
                                                             uint64_t count_host, KVList fail,
                                                             u64* __restrict__ ctr) {
    constexpr int B = 16;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const unsigned lane = threadIdx.x & 31;
    const uint64_t cnt = count_ptr ? *(volatile const u64*)count_ptr : count_host;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t wid = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const uint64_t per = (cnt + nwarps - 1) / nwarps;
    uint64_t next = wid * per;
    const uint64_t end = min(cnt, next + per);
    u64 ev = 0, lockfail = 0;
    bool active = false;
    u64 k = kE, v[W];
#pragma unroll
    for (int q = 0; q < W; q++) v[q] = 0;
    WPair p0{0, 0};
    uint32_t t = 0, hop = 0;
    int phase = 0;
    for (;;) {
        const unsigned idle = __ballot_sync(kFull, !active);
        const uint64_t mine = next + __popc(idle & lanemask_lt());
        next += __popc(idle);
        if (!active && mine < end) {
            k = src.keys[mine];
#pragma unroll
            for (int q = 0; q < W; q++) v[q] = src.vals[mine * W + q];
            p0 = wpair(tv, k);
            t = p0.t1;
            phase = 0;
            hop = 0;
            active = true;
        }
        if (!__any_sync(kFull, active)) break;
        const uint32_t b = active ? wbucket(sv, t, k) : 0u;
        const u64 tag = active ? (((u64)t << 32) | b) : (~0ull - lane);
        const unsigned peers = __match_any_sync(kFull, tag);
        const bool rep = active && lane == (unsigned)(__ffs(peers) - 1);
        uint32_t* lock = sv.sub[t].locks + b;
        bool got = false;
        if (rep) {
            got = atomicCAS(lock, 0u, 1u) == 0u;
            lockfail += !got;
        }
        if (got) {
            __threadfence();
            u64* kp = sv.sub[t].keys + (uint64_t)b * B;
            u64* vp = sv.sub[t].vals + (uint64_t)b * B * W;
            u64 s[B];
#pragma unroll
            for (int q = 0; q < B; q += 4)
                asm volatile("ld.global.cg.v4.u64 {%0,%1,%2,%3}, [%4];"
                             : "=l"(s[q]), "=l"(s[q + 1]), "=l"(s[q + 2]), "=l"(s[q + 3]) : "l"(kp + q) : "memory");
            int free_s = -1;
#pragma unroll
            for (int q = B - 1; q >= 0; --q)
                if (s[q] == kE) free_s = q;
            if (free_s >= 0) {
                st_vals<W>(vp + (uint64_t)free_s * W, v);
                st_cg(kp + free_s, k);
                active = false;
            } else if (phase < 2) {
                if (phase == 0) { phase = 1; t = p0.t2; }
                else { phase = 2; hop = 0; t = (mix64(k) & 1u) ? p0.t2 : p0.t1; }
            } else {
                const unsigned vs = (mix64(k ^ ((u64)hop * 0x9E3779B97F4A7C15ull)) >> 8) & (B - 1);
                u64 vk = kE;
#pragma unroll
                for (int q = 0; q < B; q++) vk = (q == (int)vs) ? s[q] : vk;
                u64 ov[W];
                ld_vals<W>(vp + (uint64_t)vs * W, ov, false);
                st_vals<W>(vp + (uint64_t)vs * W, v);
                st_cg(kp + vs, k);
                const uint32_t lt = t;
                k = vk;
#pragma unroll
                for (int q = 0; q < W; q++) v[q] = ov[q];
                ev++;
                hop++;
                p0 = wpair(tv, k);
                t = (lt == p0.t1) ? p0.t2 : p0.t1;
                if (hop >= tv.max_hops) {
                    const u64 at = atomicAdd(ctr + W_FAIL, 1ull);
                    fail.keys[at] = k;
#pragma unroll
                    for (int q = 0; q < W; q++) fail.vals[at * W + q] = v[q];
                    active = false;
                }
            }
            __threadfence();
            atomicExch(lock, 0u);
        }
    }
    wblock_add<kThreads>(ctr + W_EVICT, ev);
    wblock_add<kThreads>(ctr + W_LOCKFAIL, lockfail);
}

// ------------------------------------------- insert phase 2: LOCKFREE (PACK)
// One lane group (8 lanes, one 16-byte slot each) per record: first-fit CAS128
// into an EMPTY pair of t1 then t2, then an eviction chain of EXCH128 on a
// pseudo-random victim, carrying the victim to the other table of its pair.
// Every pair is held by exactly one slot or one group at any time.
__global__ void __launch_bounds__(kThreads) k_wplace_lockfree(WView tv, KVList src, const u64* count_ptr,
                                                              uint64_t count_host, KVList fail,
                                                              u64* __restrict__ ctr) {
    constexpr int G = 8, QPW = 32 / G;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const WGrp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t cnt = count_ptr ? *(volatile const u64*)count_ptr : count_host;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t wid = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    u64 ev = 0;
    for (uint64_t base = wid * QPW; base < cnt; base += nwarps * QPW) {
        const uint64_t i = base + grp;
        bool done = i >= cnt;
        u64 k = done ? kE : src.keys[i];
        u64 v = done ? 0ull : src.vals[i];
        WPair p = wpair(tv, k);
        uint32_t t = p.t1;
        int phase = 0;
        uint32_t hop = 0;
        for (;;) {
            if (!__any_sync(kFull, !done)) break;
            const uint32_t b = wbucket(sv, t, k);
            u64* bp = sv.sub[t].keys + (uint64_t)b * G * 2;
            u64 sk, sv_;
            probe_slot<PACK>(sv, t, b, g.sub, false, !done, sk, sv_);
            unsigned e = g.ballot(!done && sk == kE);
            bool placed = false;
            for (;;) {                                       // first-fit CAS into the free pairs
                const unsigned cand = g.ballot(!done && !placed && e != 0);
                if (!__any_sync(kFull, cand != 0)) break;
                bool ok = false;
                if (cand && g.sub == lowest(e)) {
                    u64 ok_, ov_;
                    cas128(bp + 2 * g.sub, kE, kE, k, v, ok_, ov_);
                    ok = ok_ == kE && ov_ == kE;
                }
                const unsigned okb = g.ballot(ok);
                if (cand) {
                    if (okb) placed = true;
                    else e &= ~(1u << lowest(e));
                }
            }
            const bool evict = !done && !placed && phase == 2;
            const unsigned vs = (mix64(k ^ ((u64)hop * 0x9E3779B97F4A7C15ull)) >> 8) & (G - 1);
            u64 ok_ = kE, ov_ = kE;
            if (evict && g.sub == vs) exch128(bp + 2 * vs, k, v, ok_, ov_);
            ok_ = g.bcast(ok_, vs);
            ov_ = g.bcast(ov_, vs);
            if (!done) {
                if (placed) {
                    done = true;
                } else if (phase < 2) {
                    if (phase == 0) { phase = 1; t = p.t2; }
                    else { phase = 2; hop = 0; t = (mix64(k) & 1u) ? p.t2 : p.t1; }
                } else {
                    ev += g.sub == 0;
                    hop++;
                    if (ok_ == kE) {
                        done = true;
                    } else {
                        const uint32_t lt = t;
                        k = ok_;
                        v = ov_;
                        p = wpair(tv, k);
                        t = (lt == p.t1) ? p.t2 : p.t1;
                        if (hop >= tv.max_hops) {
                            if (g.sub == 0) {
                                const u64 at = atomicAdd(ctr + W_FAIL, 1ull);
                                fail.keys[at] = k;
                                fail.vals[at] = v;
                            }
                            done = true;
                        }
                    }
                }
            }
        }
    }
    wblock_add<kThreads>(ctr + W_EVICT, ev);
}

// ------------------------------------------------------------------ delete (S4)
// Lock-free in every mode ("does not require locking"): the lane holding
// the key overwrites it with EMPTY (PACK: the whole pair).
template <int L, int W, int U>
__global__ void __launch_bounds__(kThreads) k_wdelete(WView tv, const u64* __restrict__ keys, u64* __restrict__ old,
                                                      uint8_t* __restrict__ status, uint64_t n, u64* __restrict__ ctr) {
    constexpr int G = Lay<L>::B, QPW = 32 / G;
    __shared__ WSmem sv;
    load_wview(tv, sv);
    const WGrp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    u64 removed = 0;
    for (uint64_t base = w * QPW * U; base < n; base += nwarps * QPW * U) {
        Probe2<L, U> pr;
        pr.run(tv, sv, g, keys, n, base, grp, false);
        u64 v[U][W];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const bool mine = pr.hb[u] && g.sub == lowest(pr.hb[u]);
#pragma unroll
            for (int q = 0; q < W; q++) v[u][q] = kE;
            if (mine) {
                if (L == SEP) {
                    if (old) ld_vals<W>(sv.sub[pr.ht[u]].vals + ((uint64_t)pr.hbk[u] * G + g.sub) * W, v[u], false);
                    st_cg(sv.sub[pr.ht[u]].keys + (uint64_t)pr.hbk[u] * G + g.sub, kE);
                } else {
                    v[u][0] = pr.hv[u];
                    st_pair(sv.sub[pr.ht[u]].keys + ((uint64_t)pr.hbk[u] * G + g.sub) * 2, kE, kE);
                }
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint64_t i = base + (uint64_t)u * QPW + grp;
            if (i >= n) continue;
            const bool hit = pr.hb[u] != 0;
            const bool writer = hit ? g.sub == lowest(pr.hb[u]) : g.sub == 0;
            if (writer) {
                if (old) {
#pragma unroll
                    for (int q = 0; q < W; q++) old[i * W + q] = hit ? v[u][q] : kE;
                }
                if (status) status[i] = hit ? 1 : 0;
                removed += hit;
            }
        }
    }
    wblock_add<kThreads>(ctr + W_REMOVED, removed);
}

// ------------------------------------------------------------ upsize (S8)
// One lane per old slot; the B lanes of a bucket rank the entries that stay in
// b and those that move to b + n_old; no conflicts, no locks.
template <int L, int W>
__global__ void __launch_bounds__(kThreads) k_wupsize(WSub o, WSub nw, uint32_t n_old, uint32_t a, uint32_t b,
                                                      uint32_t c) {
    constexpr int B = Lay<L>::B;
    const uint64_t total = (uint64_t)n_old * B;
    const unsigned lane = threadIdx.x & 31;
    const unsigned gmask = ((1u << B) - 1u) << (lane & ~(unsigned)(B - 1));
    const unsigned lt = lanemask_lt() & gmask;
    for (uint64_t base = (uint64_t)blockIdx.x * kThreads; base < total; base += (uint64_t)gridDim.x * kThreads) {
        const uint64_t gi = base + threadIdx.x;
        const bool valid = gi < total;
        u64 k = kE, pv = kE;
        if (valid) {
            if (L == SEP) k = __ldcs(o.keys + gi);
            else { k = __ldcs(o.keys + 2 * gi); pv = __ldcs(o.keys + 2 * gi + 1); }
        }
        const uint32_t bucket = (uint32_t)(gi / B), s = (uint32_t)(gi % B);
        const bool occ = k != kE;
        const bool hi = occ && fastmod(hxw(a, b, c, k), nw.magic, nw.n) != bucket;
        const unsigned hb = __ballot_sync(kFull, occ && hi) & gmask;
        const unsigned lb = __ballot_sync(kFull, occ && !hi) & gmask;
        if (valid) {
            const uint64_t lo_base = (uint64_t)bucket * B, hi_base = ((uint64_t)bucket + n_old) * B;
            if (occ) {
                const uint64_t dst = (hi ? hi_base : lo_base) + __popc((hi ? hb : lb) & lt);
                if (L == SEP) {
                    nw.keys[dst] = k;
#pragma unroll
                    for (int q = 0; q < W; q++) nw.vals[dst * W + q] = __ldcs(o.vals + gi * W + q);
                } else {
                    nw.keys[2 * dst] = k;
                    nw.keys[2 * dst + 1] = pv;
                }
            }
            if (s >= (uint32_t)__popc(lb)) {
                if (L == SEP) nw.keys[lo_base + s] = kE;
                else { nw.keys[2 * (lo_base + s)] = kE; nw.keys[2 * (lo_base + s) + 1] = kE; }
            }
            if (s >= (uint32_t)__popc(hb)) {
                if (L == SEP) nw.keys[hi_base + s] = kE;
                else { nw.keys[2 * (hi_base + s)] = kE; nw.keys[2 * (hi_base + s) + 1] = kE; }
            }
        }
    }
}

// ----------------------------------------------------------- downsize (S9)
// One lane per slot of the halved table: b' takes old b' then old b'+h in slot
// order, keeps the first B (Q18), the rest become residuals.
template <int L, int W>
__global__ void __launch_bounds__(kThreads) k_wdownsize(WSub o, WSub nw, uint32_t h, KVList residual,
                                                        u64* __restrict__ ctr) {
    constexpr int B = Lay<L>::B;
    const uint64_t total = (uint64_t)h * B;
    const unsigned lane = threadIdx.x & 31;
    const unsigned gmask = ((1u << B) - 1u) << (lane & ~(unsigned)(B - 1));
    const unsigned lt = lanemask_lt() & gmask;
    for (uint64_t base = (uint64_t)blockIdx.x * kThreads; base < total; base += (uint64_t)gridDim.x * kThreads) {
        const uint64_t gi = base + threadIdx.x;
        const bool valid = gi < total;
        u64 k1 = kE, k2 = kE, p1 = kE, p2 = kE;
        if (valid) {
            if (L == SEP) { k1 = __ldcs(o.keys + gi); k2 = __ldcs(o.keys + gi + total); }
            else {
                k1 = __ldcs(o.keys + 2 * gi); p1 = __ldcs(o.keys + 2 * gi + 1);
                k2 = __ldcs(o.keys + 2 * (gi + total)); p2 = __ldcs(o.keys + 2 * (gi + total) + 1);
            }
        }
        const bool o1 = k1 != kE, o2 = k2 != kE;
        const unsigned m1 = __ballot_sync(kFull, o1) & gmask, m2 = __ballot_sync(kFull, o2) & gmask;
        const uint32_t c1 = __popc(m1), ctot = c1 + __popc(m2);
        const uint32_t r1 = __popc(m1 & lt), r2 = c1 + __popc(m2 & lt);
        const uint64_t bb = (gi / B) * B;
        const uint32_t s = (uint32_t)(gi % B);
        bool res = false;
        u64 rv[W];
#pragma unroll
        for (int q = 0; q < W; q++) rv[q] = 0;
        if (valid) {
            if (o1) {
                if (L == SEP) {
                    nw.keys[bb + r1] = k1;
#pragma unroll
                    for (int q = 0; q < W; q++) nw.vals[(bb + r1) * W + q] = __ldcs(o.vals + gi * W + q);
                } else { nw.keys[2 * (bb + r1)] = k1; nw.keys[2 * (bb + r1) + 1] = p1; }
            }
            if (o2) {
                if (L == SEP) {
#pragma unroll
                    for (int q = 0; q < W; q++) rv[q] = __ldcs(o.vals + (gi + total) * W + q);
                } else {
                    rv[0] = p2;
                }
                if (r2 < (uint32_t)B) {
                    if (L == SEP) {
                        nw.keys[bb + r2] = k2;
#pragma unroll
                        for (int q = 0; q < W; q++) nw.vals[(bb + r2) * W + q] = rv[q];
                    } else { nw.keys[2 * (bb + r2)] = k2; nw.keys[2 * (bb + r2) + 1] = p2; }
                } else {
                    res = true;
                }
            }
            if (s >= ctot) {
                if (L == SEP) nw.keys[bb + s] = kE;
                else { nw.keys[2 * (bb + s)] = kE; nw.keys[2 * (bb + s) + 1] = kE; }
            }
        }
        const unsigned rm = __ballot_sync(kFull, res);
        if (rm && lane == (unsigned)(__ffs(rm) - 1)) atomicAdd(ctr + W_RES_TOTAL, (u64)__popc(rm));
        kv_append<W>(res, k2, rv, residual, ctr + W_RESIDUAL);
    }
}

// ------------------------------------------------------- stats / dump (S10)
template <int L>
__global__ void __launch_bounds__(kThreads) k_wcount(WSub s, u64* __restrict__ cnt_out) {
    constexpr int B = Lay<L>::B;
    const uint64_t total = (uint64_t)s.n * B;
    u64 c = 0;
    for (uint64_t gi = (uint64_t)blockIdx.x * kThreads + threadIdx.x; gi < total; gi += (uint64_t)gridDim.x * kThreads)
        c += (L == SEP ? s.keys[gi] : s.keys[2 * gi]) != kE;
    wblock_add<kThreads>(cnt_out, c);
}

template <int L, int W>
__global__ void __launch_bounds__(kThreads) k_wdump(WSub s, uint32_t t, u64* __restrict__ keys, u64* __restrict__ vals,
                                                    uint32_t* __restrict__ tab, u64* __restrict__ bkt, uint64_t cap,
                                                    u64* __restrict__ cursor) {
    constexpr int B = Lay<L>::B;
    const uint64_t total = (uint64_t)s.n * B;
    for (uint64_t gi = (uint64_t)blockIdx.x * kThreads + threadIdx.x; gi < total;
         gi += (uint64_t)gridDim.x * kThreads) {
        const u64 k = L == SEP ? s.keys[gi] : s.keys[2 * gi];
        if (k == kE) continue;
        const u64 at = atomicAdd(cursor, 1ull);
        if (at >= cap) continue;
        keys[at] = k;
        if (L == SEP) {
#pragma unroll
            for (int q = 0; q < W; q++) vals[at * W + q] = s.vals[gi * W + q];
        } else {
            vals[at] = s.keys[2 * gi + 1];
        }
        tab[at] = t;
        bkt[at] = gi / B;
    }
}

__global__ void k_whash_probe(WView tv, const u64* __restrict__ keys, uint64_t n, uint32_t* __restrict__ x,
                              uint32_t* __restrict__ pr) {
    const uint32_t ns = tv.d + 2;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const u64 k = keys[i];
        for (uint32_t s = 0; s < ns; s++) x[i * ns + s] = hxw(tv.a[s], tv.b[s], tv.c[s], k);
        const WPair p = wpair(tv, k);
        pr[2 * i] = p.t1;
        pr[2 * i + 1] = p.t2;
    }
}

}  // namespace dyw
