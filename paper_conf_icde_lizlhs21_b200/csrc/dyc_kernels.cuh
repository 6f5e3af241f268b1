// dyc_kernels.cuh — the sm_100a kernels of the DyCuckoo hot path.
//
// Rows of SURVEY.md §8(a) and the kernel implementing each:
//   S2+S3 find ............. k_find      (<= 2 probes)
//   S2+S5 insert phase 1 ... k_upsert    (Alg. 1 L536-539 upsert; FUSE: first-fit CAS)
//   S7    insert phase 2 ... k_place     (eviction chains; failure list P:L737)
//   S4    delete ........... k_delete    (no lock)
//   S8    upsize ........... k_upsize    (bucket b -> b or b+|h|)
//   S9    downsize ......... k_downsize  (merge b, b+|h|/2; residuals)
//   S10   stats / dump ..... k_count, k_dump
//   S11   routing .......... k_route_count, k_route_scatter, k_route_unpermute
// The paper's voter/lock mechanism (Alg. 1) was designed around
// Pascal's slow contended atomics; here a key-value pair is one 64-bit word, so
// lock-free atomicCAS (into an EMPTY slot) and atomicExch (eviction) on the slot
// itself replace the bucket lock.
#pragma once
#include "dyc_device.cuh"

namespace dyc {

constexpr int kThreads = 256;
// minimum resident blocks per SM requested from ptxas (register budget) per kernel family
#ifndef DYC_FIND_MINB
#define DYC_FIND_MINB 3
#endif
#ifndef DYC_UPSERT_MINB
#define DYC_UPSERT_MINB 1
#endif
#ifndef DYC_DELETE_MINB
#define DYC_DELETE_MINB 1
#endif
#ifndef DYC_PLACE_MINB
#define DYC_PLACE_MINB 1
#endif
#ifndef DYC_UPSERT_U
#define DYC_UPSERT_U 4
#endif
#ifndef DYC_DELETE_U
#define DYC_DELETE_U 2
#endif
#ifndef DYC_UPSERT_SPEC
#define DYC_UPSERT_SPEC 0
#endif
#ifndef DYC_FIND_ILP
#define DYC_FIND_ILP 4
#endif
#ifndef DYC_FIND_ORDER
#define DYC_FIND_ORDER 0
#endif

// Device counters.  [0, C_ACC0) are per batch (zeroed when a batch starts);
// [C_ACC0, C_COUNT0) accumulate across batches until the host reads them back
// (read_ctr applies them to its live count and statistics, then zeroes them),
// so a batch that does not need an exact count can return without a host wait.
enum CounterIdx : int {
    C_PENDING = 0,    // new keys handed to k_place
    C_INSERTED = 1,   // ops with status INSERTED
    C_UPDATED = 2,    // ops with status UPDATED
    C_FAIL = 3,       // homeless pairs appended by k_place (synchronous settling)
    C_RESIDUAL = 4,   // downsize residuals
    C_DUMP = 5,       // dump cursor
    C_SECOND = 6,     // keys in their second-choice subtable (stats)
    C_RES_TOTAL = 7,  // residuals over several downsizes of one alpha loop
    C_DEFER = 8,      // ops on a subtable locked by a resize in flight (NEXT-1)
    C_ACC0 = 11,
    C_STASH = 11,     // pairs in the stash (homeless after a lazily settled batch)
    C_REMOVED = 12,   // delete hits
    C_EVICT = 13,     // eviction hops
    C_ADDED = 14,     // INSERTED statuses (live-count increments)
    C_PEND_ACC = 15,  // new keys handed to k_place (statistics)
    C_COUNT0 = 16,    // per-subtable live counts [16, 32)
    C_N = 32
};

// ------------------------------------------------------------- lane groups
// G = B/4 lanes cooperate on one bucket: lane `sub` of the group holds slots
// [4*sub, 4*sub+4) of it (one 256-bit load), so one warp-wide load instruction
// probes 32/G buckets and a 128-byte bucket (B = 16) costs ONE line request.
// Measured on B200: ~53 G random line requests/s whether a
// request carries 32 or 128 bytes, so wide buckets read cooperatively are free
// bytes that cut second-table probes (φ) and evictions.  This is the warp-
// cooperative bucket scan of the paper with
// __ballot_sync deciding the hit lane.
template <int G>
struct Grp {
    unsigned lane, sub, base, gmask;
    __device__ __forceinline__ Grp() {
        lane = threadIdx.x & 31;
        sub = lane & (G - 1);
        base = lane - sub;
        gmask = (G == 32) ? kFull : (((1u << G) - 1u) << base);
    }
    // group-local ballot: bit s <=> lane `s` of this group voted true
    __device__ __forceinline__ unsigned ballot(bool p) const { return (__ballot_sync(kFull, p) & gmask) >> base; }
    __device__ __forceinline__ unsigned long long bcast(unsigned long long v, unsigned src) const {
        return __shfl_sync(kFull, v, base + src);
    }
    __device__ __forceinline__ uint32_t bcast32(uint32_t v, unsigned src) const {
        return __shfl_sync(kFull, v, base + src);
    }
};

__device__ __forceinline__ unsigned first_lane(unsigned bits) { return bits ? (unsigned)(__ffs(bits) - 1) : 0u; }

__device__ __forceinline__ uint32_t mix32(uint32_t x) {
    x ^= x >> 16; x *= 0x7FEB352Du; x ^= x >> 15; x *= 0x846CA68Bu; x ^= x >> 16;
    return x;
}

// First-fit CAS of kv into an EMPTY slot of the bucket whose group snapshot is s
// (slot order).  Called by every lane of the warp (ballots); `want` is uniform
// within a group.  A failed CAS means another key took that slot: try the next.
template <int G>
__device__ __forceinline__ bool coop_cas_empty(const Grp<G>& g, unsigned long long* bp,
                                               const unsigned long long (&s)[4], bool want,
                                               unsigned long long kv) {
    unsigned emask = 0;
#pragma unroll
    for (int j = 0; j < 4; j++)
        if (s[j] == kEmptySlot) emask |= 1u << j;
    bool placed = false;
    for (;;) {
        const unsigned cand = g.ballot(want && !placed && emask != 0);
        if (!__any_sync(kFull, cand != 0)) break;
        const unsigned owner = first_lane(cand);
        bool ok = false;
        if (cand && g.sub == owner) {
            const unsigned j = __ffs(emask) - 1;
            ok = cas_slot(bp + 4 * g.sub + j, kEmptySlot, kv) == kEmptySlot;
            emask &= ~(1u << j);
        }
        ok = __shfl_sync(kFull, ok, g.base + owner);
        if (cand && ok) placed = true;
    }
    return placed;
}

__device__ __forceinline__ unsigned empty_mask(const unsigned long long (&s)[4]) {
    unsigned m = 0;
#pragma unroll
    for (int j = 0; j < 4; j++)
        if (s[j] == kEmptySlot) m |= 1u << j;
    return m;
}

// ------------------------------------------------------------------- stash
// Pairs that an insert batch could not place within L_max hops wait in
// the stash until the host's next read-back settles them (retry, then
// failure-triggered upsizes, Q17); until then they are live keys of the map, so
// find, the existence check of insert and delete look there after both
// candidate buckets missed (the stash is empty in normal operation: one load of
// its count per thread).  Returns the stash index of k, or -1.  The group's
// lead lane scans; the result is broadcast.
template <int G>
__device__ __forceinline__ int64_t stash_find(const Grp<G>& g, const TableView& tv, uint64_t sn, uint32_t k, bool want) {
    int64_t at = -1;
    if (g.sub == 0 && want && k != kEmptyKey)
        for (uint64_t j = 0; j < sn; j++)
            if (key_of(*(volatile unsigned long long*)(tv.stash + j)) == k) { at = (int64_t)j; break; }
    return (int64_t)__shfl_sync(kFull, (unsigned long long)at, g.base);
}

__device__ __forceinline__ uint64_t stash_count(const TableView& tv) {
    return tv.stash_n ? *(volatile const unsigned long long*)tv.stash_n : 0ull;
}

// ----------------------------------------------------------------- find (S3)
// ILP queries per group; all first probes are issued back to back, then the
// second probes (predicated, only after a first-probe miss: <= 2 lookups).
// A miss in a non-full first-choice bucket of a subtable that holds the
// first-choice-full invariant (TableView::clean) is final: no second probe.
// The stash check stays a run-time one here (a null count pointer when the
// host knows the stash is empty): measured 3.87 vs 4.29 ms at C2 against a
// compile-time variant without it, from instruction scheduling alone
// (profiles/r2_variants.md).
// S1 (staged batches, dyc_staged.cuh): every key is known to be absent from its
// first-choice bucket (the staged pass read it); only the second one is probed.
template <int B, int ILP, bool S1 = false>
__global__ void __launch_bounds__(kThreads, DYC_FIND_MINB) k_find(TableView tv, const uint32_t* __restrict__ keys,
                                                   uint32_t* __restrict__ vals, uint8_t* __restrict__ found,
                                                   uint64_t n, const unsigned long long* __restrict__ n_dev = nullptr,
                                                   const uint32_t* __restrict__ idx = nullptr) {
    // S1: op i (keys[i]) is entry i of a staged batch's need list; its results go to [idx[i]]
    constexpr int G = B / 4, QPW = 32 / G;
    __shared__ SmemView sv;
    load_view(tv, sv);
    if (n_dev) n = min(n, (uint64_t)*n_dev);     // op count known on the device only (mixed batches)
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t wtile = (uint64_t)QPW * ILP;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const uint64_t sn = stash_count(tv);
    unsigned long long n_ops = 0, n_p2 = 0;
    for (uint64_t base = w * wtile; base < n; base += nwarps * wtile) {
        uint32_t k[ILP], v[ILP];
        bool f[ILP], c1[ILP];
        const unsigned long long* p2[ILP];
        unsigned long long s[ILP][4];
#pragma unroll
        for (int j = 0; j < ILP; j++) {
            const uint64_t i = base + (uint64_t)j * QPW + grp;
            k[j] = i < n ? __ldg(keys + i) : kEmptyKey;
        }
#pragma unroll
        for (int j = 0; j < ILP; j++) {
            const Pair p = pair_of(tv, k[j]);
            c1[j] = (tv.clean >> p.t1) & 1u;
#if DYC_FIND_ORDER == 2
            probe_nc<B>(bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k[j]), B) + 4 * g.sub, s[j]);
            asm volatile("" ::: "memory");
            p2[j] = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k[j]), B) + 4 * g.sub;
#else
            p2[j] = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k[j]), B) + 4 * g.sub;
            if (S1) {
#pragma unroll
                for (int q = 0; q < 4; q++) s[j][q] = kEmptySlot;
            } else {
                probe_nc<B>(bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k[j]), B) + 4 * g.sub, s[j]);
            }
#if DYC_FIND_ORDER == 1
            asm volatile("" ::: "memory");   // issue this probe before the next query's view reads
#endif
#endif
        }
        bool need2[ILP];
#pragma unroll
        for (int j = 0; j < ILP; j++) {
            uint32_t lv = 0;
            const bool lh = lookup_slot<4>(s[j], k[j], lv) && k[j] != kEmptyKey;
            const unsigned hb = g.ballot(lh);
            const unsigned eb = g.ballot(empty_mask(s[j]) != 0);
            f[j] = hb != 0;
            v[j] = g.bcast32(lv, first_lane(hb));
            need2[j] = !f[j] && k[j] != kEmptyKey && (S1 || !(c1[j] && eb != 0));
            n_ops += g.sub == 0 && k[j] != kEmptyKey;
            n_p2 += g.sub == 0 && need2[j];
        }
#pragma unroll
        for (int j = 0; j < ILP; j++) probe_nc_pred<B>(p2[j], s[j], need2[j]);
#pragma unroll
        for (int j = 0; j < ILP; j++) {
            uint32_t lv = 0;
            const bool lh = need2[j] && lookup_slot<4>(s[j], k[j], lv);
            const unsigned hb = g.ballot(lh);
            const uint32_t v2 = g.bcast32(lv, first_lane(hb));
            if (hb) { f[j] = true; v[j] = v2; }
            if (sn) {
                const int64_t at = stash_find(g, tv, sn, k[j], !f[j]);
                if (at >= 0) { f[j] = true; v[j] = val_of(tv.stash[at]); }
            }
            const uint64_t i = base + (uint64_t)j * QPW + grp;
            if (g.sub == 0 && i < n) {
                const uint64_t o = S1 ? (uint64_t)__ldg(idx + i) : i;
                vals[o] = f[j] ? v[j] : kEmptyKey;
                if (found) found[o] = f[j] ? 1 : 0;
            }
        }
    }
    if (tv.probe) {
        block_add<kThreads>(tv.probe + 0, n_ops);
        block_add<kThreads>(tv.probe + 1, n_p2);
    }
}

// ------------------------------------------------------- placement (S7 core)
// Cuckoo placement of a pair known to be absent, by one lane group.  First-fit
// over the ordered pair (reading Q3); then an eviction chain: exchange with a
// pseudo-random victim slot (Q5) and carry the victim to the OTHER table of ITS
// pair.  Every pair is held by exactly one group or one slot at
// any time (atomicExch), so nothing is lost or duplicated.  After max_hops hops
// (Q6) the carried pair is returned as homeless.  Returns true when placed;
// groups that enter with done == true only take part in the ballots.
template <int B>
__device__ __forceinline__ bool coop_place(const Grp<B / 4>& g, const TableView& tv, const SmemView& sv,
                                           unsigned long long& kv, bool done, bool first_fit, uint32_t& ev) {
    uint32_t k = key_of(kv);
    const Pair p = pair_of(tv, k);
    unsigned long long s[4] = {kEmptySlot, kEmptySlot, kEmptySlot, kEmptySlot};
    if (first_fit) {
        unsigned long long* b1 = bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k), B);
        probe_cg_pred<B>(b1 + 4 * g.sub, s, !done);
        done |= coop_cas_empty(g, b1, s, !done, kv);
        unsigned long long* b2 = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k), B);
        probe_cg_pred<B>(b2 + 4 * g.sub, s, !done);
        done |= coop_cas_empty(g, b2, s, !done, kv);
    }
    uint32_t t = (mix32(k) & 1u) ? p.t2 : p.t1;
    for (uint32_t hop = 0; hop < tv.max_hops; hop++) {
        if (!__any_sync(kFull, !done)) break;
        unsigned long long* bp = bucket_ptr(sv, t, bucket_of(sv, t, k), B);
        if (hop > 0) {
            probe_cg_pred<B>(bp + 4 * g.sub, s, !done);
            done |= coop_cas_empty(g, bp, s, !done, kv);
        }
        const uint32_t victim = (mix32(k ^ (hop * 0x9E3779B9u)) >> 8) & (B - 1);
        const unsigned owner = victim >> 2;
        unsigned long long old = kEmptySlot;
        if (!done && g.sub == owner) old = exch_slot(bp + victim, kv);
        old = g.bcast(old, owner);
        if (!done) {
            ev += (g.sub == 0);
            if (old == kEmptySlot) {
                done = true;
            } else {
                kv = old;
                k = key_of(kv);
                const Pair q = pair_of(tv, k);
                t = (t == q.t1) ? q.t2 : q.t1;
            }
        }
    }
    return done;
}

// First-fit CAS for U independent ops of a group at once: each round, every op
// that still has a candidate EMPTY slot issues one CAS (all U in flight
// together), so the atomic round trips of different ops overlap.
template <int G, int U>
__device__ __forceinline__ void coop_cas_multi(const Grp<G>& g, unsigned long long* const (&bp)[U],
                                               unsigned (&em)[U], const bool (&want)[U],
                                               const unsigned long long (&kv)[U], bool (&placed)[U]) {
    for (;;) {
        unsigned cand[U];
        bool any = false;
#pragma unroll
        for (int u = 0; u < U; u++) {
            cand[u] = g.ballot(want[u] && !placed[u] && em[u] != 0);
            any |= cand[u] != 0;
        }
        if (!__any_sync(kFull, any)) break;
        unsigned long long old[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            old[u] = 0;
            if (cand[u] && g.sub == first_lane(cand[u])) {
                const unsigned j = __ffs(em[u]) - 1;
                old[u] = cas_slot(bp[u] + 4 * g.sub + j, kEmptySlot, kv[u]);
                em[u] &= ~(1u << j);
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const unsigned long long o = g.bcast(old[u], first_lane(cand[u]));
            if (cand[u] && o == kEmptySlot) placed[u] = true;
        }
    }
}

// ------------------------------------------------------ insert phase 1 (S5)
// Upsert: probe t1's bucket, then t2's; an existing key gets its value replaced
// (Alg. 1, status UPDATED).  A new key (status INSERTED) is, with FUSE,
// CAS-ed into a free slot of its first-fit bucket right away; otherwise (or if
// both candidate buckets are full) it is appended to `pending` for k_place.
// Keys never move during this kernel (no evictions), so the existence check is
// exact; FUSE is only used when no upsize can be needed ((m+n) <= beta*N).
// Each group carries U ops whose probes are issued together (memory-level
// parallelism: the kernel is bound by random line requests).
//
// LK (resize under live traffic, NEXT-1): subtable `locked` is
// being resized by a concurrent kernel, so its (old, read-only) buffer may be
// probed but not written.  An existing key found there keeps status UPDATED but
// its new value is appended to `defer` (applied by k_apply after the resize is
// committed); a new key may only take a free slot of its OTHER candidate bucket,
// else it is pending (placed after the commit).
// W: the paper-weighted placement mode (compile time); STASH as in k_find.
// S1 as in k_find: the first-choice bucket is known not to hold the key and
// not to be a placement candidate (staged batches send a key here when its
// first-choice bucket was full); only the second bucket is probed.
template <int B, bool FUSE, int U, bool LK = false, bool W = false, bool STASH = false, bool S1 = false>
__global__ void __launch_bounds__(kThreads, DYC_UPSERT_MINB) k_upsert(TableView tv, const uint32_t* __restrict__ keys,
                                                     const uint32_t* __restrict__ vals,
                                                     uint8_t* __restrict__ status, uint64_t n,
                                                     unsigned long long* __restrict__ pending,
                                                     unsigned long long* __restrict__ ctr,
                                                     uint32_t locked = 0xFFFFFFFFu,
                                                     unsigned long long* __restrict__ defer = nullptr,
                                                     const unsigned long long* __restrict__ n_dev = nullptr,
                                                     const uint32_t* __restrict__ idx = nullptr) {
    // S1: op i ((keys, vals)[i]) is entry i of a staged batch's need list; its status goes to status[idx[i]]
    constexpr int G = B / 4, QPW = 32 / G;
    __shared__ SmemView sv;
    load_view(tv, sv);
    if (n_dev) n = min(n, (uint64_t)*n_dev);     // op count known on the device only (mixed batches)
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const uint64_t sn = STASH ? stash_count(tv) : 0ull;
    unsigned long long n_ins = 0, n_upd = 0, n_ops = 0, n_p2 = 0;
    for (uint64_t base = w * (QPW * U); base < n; base += nwarps * (QPW * U)) {
        // per op only the match position and the free-slot mask of each bucket
        // are kept, not the 4-slot snapshots (register budget -> more ops in flight)
        uint64_t i[U];
        uint32_t k[U];
        unsigned long long kv[U];
        unsigned long long* b1[U];
        unsigned long long* b2[U];
        unsigned h1[U], h2[U], em1[U], em2[U];
        bool need2[U], isnew[U], placed[U];
        int j1[U], j2[U];
        bool lk1[U], lk2[U];
        bool ch2[U];                     // paper-weighted mode: the new key's table is t2
#if DYC_UPSERT_SPEC
        // speculative: both candidate buckets are read together (one round trip);
        // the t2 read is wasted only for keys found in t1 (updates)
        {
            unsigned long long s1[U][4], s2[U][4];
#pragma unroll
            for (int u = 0; u < U; u++) {
                i[u] = base + (uint64_t)u * QPW + grp;
                const bool valid = i[u] < n;
                k[u] = valid ? __ldg(keys + i[u]) : kEmptyKey;
                kv[u] = make_kv(k[u], valid ? __ldg(vals + i[u]) : 0u);
                const Pair p = pair_of(tv, k[u]);
                lk1[u] = LK && p.t1 == locked;
                lk2[u] = LK && p.t2 == locked;
                ch2[u] = W && weighted_second(sv, p.t1, p.t2, k[u]);
                b1[u] = bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k[u]), B);
                b2[u] = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k[u]), B);
                probe_cg<B>(b1[u] + 4 * g.sub, s1[u]);
#pragma unroll
                for (int q = 0; q < 4; q++) s2[u][q] = kEmptySlot;
                probe_cg_pred<B>(b2[u] + 4 * g.sub, s2[u], k[u] != kEmptyKey);
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
                const bool active = k[u] != kEmptyKey;
                j1[u] = match_slot<4>(s1[u], k[u]);
                em1[u] = lk1[u] ? 0u : empty_mask(s1[u]);
                h1[u] = g.ballot(active && j1[u] >= 0);
                need2[u] = active && h1[u] == 0;
                j2[u] = need2[u] ? match_slot<4>(s2[u], k[u]) : -1;
                em2[u] = (lk2[u] || !need2[u]) ? 0u : empty_mask(s2[u]);
            }
        }
#else
        {
            unsigned long long s1[U][4];
            bool c1[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                i[u] = base + (uint64_t)u * QPW + grp;
                const bool valid = i[u] < n;
                k[u] = valid ? __ldg(keys + i[u]) : kEmptyKey;
                kv[u] = make_kv(k[u], valid ? __ldg(vals + i[u]) : 0u);
                const Pair p = pair_of(tv, k[u]);
                lk1[u] = LK && p.t1 == locked;
                lk2[u] = LK && p.t2 == locked;
                ch2[u] = W && weighted_second(sv, p.t1, p.t2, k[u]);
                c1[u] = ((tv.clean >> p.t1) & 1u) && !lk1[u];
                b1[u] = bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k[u]), B);
                b2[u] = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k[u]), B);
                if (S1) {
#pragma unroll
                    for (int q = 0; q < 4; q++) s1[u][q] = kEmptySlot;
                } else {
                    probe_cg<B>(b1[u] + 4 * g.sub, s1[u]);
                }
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
                const bool active = k[u] != kEmptyKey;
                j1[u] = match_slot<4>(s1[u], k[u]);
                const unsigned e = empty_mask(s1[u]);
                em1[u] = (S1 || lk1[u]) ? 0u : e;
                h1[u] = g.ballot(active && j1[u] >= 0);
                // first-choice-full invariant: absent from a non-full first-choice
                // bucket of a clean subtable => absent from the table (no t2 probe)
                const unsigned eb = g.ballot(e != 0);   // every lane votes (no short circuit)
                const bool skip = c1[u] && eb != 0;
                need2[u] = active && h1[u] == 0 && (S1 || !skip);
                n_ops += g.sub == 0 && active;
                n_p2 += g.sub == 0 && need2[u];
            }
        }
        {
            unsigned long long s2[U][4];
#pragma unroll
            for (int u = 0; u < U; u++) {
#pragma unroll
                for (int q = 0; q < 4; q++) s2[u][q] = kEmptySlot;
                probe_cg_pred<B>(b2[u] + 4 * g.sub, s2[u], need2[u]);
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
                j2[u] = match_slot<4>(s2[u], k[u]);
                em2[u] = (lk2[u] || !need2[u]) ? 0u : empty_mask(s2[u]);
            }
        }
#endif
#pragma unroll
        for (int u = 0; u < U; u++) {
            h2[u] = g.ballot(need2[u] && j2[u] >= 0);
            if (h1[u] && !lk1[u] && g.sub == first_lane(h1[u])) st_u64_cg(b1[u] + 4 * g.sub + j1[u], kv[u]);
            if (h2[u] && !lk2[u] && g.sub == first_lane(h2[u])) st_u64_cg(b2[u] + 4 * g.sub + j2[u], kv[u]);
            if (LK) warp_append(g.sub == 0 && ((h1[u] && lk1[u]) || (h2[u] && lk2[u])), kv[u], defer, ctr + C_DEFER);
            isnew[u] = k[u] != kEmptyKey && h1[u] == 0 && h2[u] == 0;
            placed[u] = false;
            if (sn) {                       // a stashed pair is present: update it in place
                const int64_t at = stash_find(g, tv, sn, k[u], isnew[u]);
                if (at >= 0) {
                    if (g.sub == 0) st_u64_cg(tv.stash + at, kv[u]);
                    isnew[u] = false;
                    h1[u] |= 1u;            // status UPDATED below
                }
            }
        }
        if (FUSE) {
            // paper-weighted mode: only the chosen table's bucket is a candidate
            // (P:L361); a full one sends the key to k_place, which evicts there
            if (W) {
#pragma unroll
                for (int u = 0; u < U; u++) {
                    if (ch2[u]) em1[u] = 0;
                    else em2[u] = 0;
                }
            }
            coop_cas_multi<G, U>(g, b1, em1, isnew, kv, placed);
            coop_cas_multi<G, U>(g, b2, em2, isnew, kv, placed);
        }
        const bool lead = g.sub == 0;
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint8_t st = k[u] == kEmptyKey ? 0 : ((h1[u] | h2[u]) ? 2 : 1);
            if (lead && i[u] < n && status) status[S1 ? (uint64_t)__ldg(idx + i[u]) : i[u]] = st;
            warp_append(lead && isnew[u] && !placed[u], kv[u], pending, ctr + C_PENDING);
            n_ins += lead && st == 1;
            n_upd += lead && st == 2;
        }
    }
    block_add<kThreads>(ctr + C_INSERTED, n_ins);
    block_add<kThreads>(ctr + C_UPDATED, n_upd);
    if (tv.probe) {
        block_add<kThreads>(tv.probe + 2, n_ops);
        block_add<kThreads>(tv.probe + 3, n_p2);
    }
}

// ------------------------------------------------------ insert phase 2 (S7)
// Persistent kernel over list[0 .. *count) (count read on the device, so no host
// round trip is needed between phase 1 and phase 2).  Each warp owns a
// contiguous range of the list; its lane groups pull the next key from that
// range as soon as their current chain ends, so a long eviction chain does not
// hold the other groups of the warp idle.  Per group a small state machine:
//   phase 0/1 : first-fit probe of t1 / t2 (reading Q3; skipped when
//               first_fit = false, i.e. the upsert already found t1 full),
//   phase 2   : eviction hops: probe for a free slot (after the first hop), else
//               exchange a pseudo-random victim (Q5) and carry it to the other
//               table of ITS pair; after max_hops (Q6) the
//               carried pair goes to the failure list.
template <int B, bool W = false>
__global__ void __launch_bounds__(kThreads, DYC_PLACE_MINB) k_place(TableView tv, const unsigned long long* __restrict__ list,
                                                    const unsigned long long* count_ptr, uint64_t count_host,
                                                    unsigned long long* __restrict__ fail_list,
                                                    unsigned long long* __restrict__ ctr, bool first_fit,
                                                    unsigned long long* __restrict__ fail_cursor = nullptr,
                                                    bool lazy_counts = false) {
    constexpr int G = B / 4;
    __shared__ SmemView sv;
    load_view(tv, sv);
    const Grp<G> g;
    const uint64_t cnt = count_ptr ? *(volatile const unsigned long long*)count_ptr : count_host;
    // the placement of a lazily settled insert batch also moves the batch's
    // counts into the accumulators (k_upsert has finished: stream order)
    if (lazy_counts && blockIdx.x == 0 && threadIdx.x == 0) {
        atomicAdd(ctr + C_PEND_ACC, (unsigned long long)cnt);
        atomicAdd(ctr + C_ADDED, *(volatile const unsigned long long*)(ctr + C_INSERTED));
    }
    unsigned long long* const fcur = fail_cursor ? fail_cursor : ctr + C_FAIL;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const uint64_t per = (cnt + nwarps - 1) / nwarps;
    uint64_t next = w * per;
    const uint64_t end = min(cnt, next + per);
    unsigned long long kv = kEmptySlot;
    uint32_t k = 0, t = 0, hop = 0, ev = 0;
    int phase = -1;                       // -1 idle, 0/1 first-fit t1/t2, 2 evicting
    for (;;) {
        // refill idle groups from the warp's range (one ballot, no atomics)
        const bool idle = phase < 0;
        const unsigned want = __ballot_sync(kFull, idle && g.sub == 0);   // one bit per idle group leader
        const uint64_t mine = next + __popc(want & ((1u << g.base) - 1u)); // idle leaders before this group
        next += __popc(want);
        if (idle && mine < end && key_of(list[mine]) != kEmptyKey) {   // (a stash tombstone is skipped)
            kv = list[mine];
            k = key_of(kv);
            const Pair p = pair_of(tv, k);
            phase = first_fit ? 0 : 2;
            // without first-fit, hop 0 evicts from t1 without a probe: k_upsert
            // saw that bucket full; its t2 bucket may be unread (first-choice-full
            // shortcut) and evicting from a non-full bucket would break the
            // invariant for the victim.  Paper-weighted mode: the chosen table
            // plays t1's part (probed once, then evicted from).
            t = (W && weighted_second(sv, p.t1, p.t2, k)) ? p.t2 : p.t1;
            hop = 0;
        }
        if (!__any_sync(kFull, phase >= 0)) break;
        const bool act = phase >= 0;
        unsigned long long* bp = bucket_ptr(sv, t, bucket_of(sv, t, k), B);
        const bool try_free = act && (phase < 2 || hop > 0);
        unsigned long long s[4] = {kEmptySlot, kEmptySlot, kEmptySlot, kEmptySlot};
        probe_cg_pred<B>(bp + 4 * g.sub, s, try_free);
        unsigned em[1] = {try_free ? empty_mask(s) : 0u};
        unsigned long long* const bpa[1] = {bp};
        const bool want1[1] = {try_free};
        const unsigned long long kva[1] = {kv};
        bool placed[1] = {false};
        coop_cas_multi<G, 1>(g, bpa, em, want1, kva, placed);
        const bool evict = act && !placed[0] && phase == 2;
        const uint32_t victim = (mix32(k ^ (hop * 0x9E3779B9u)) >> 8) & (B - 1);
        const unsigned owner = victim >> 2;
        unsigned long long old = kEmptySlot;
        if (evict && g.sub == owner) old = exch_slot(bp + victim, kv);
        old = g.bcast(old, owner);
        bool fail = false;
        if (act && placed[0]) {
            phase = -1;
        } else if (act && phase < 2) {
            const Pair p = pair_of(tv, k);
            if (W) { phase = 2; hop = 0; }                   // evict from the chosen table
            else if (phase == 0) { phase = 1; t = p.t2; }
            else { phase = 2; hop = 0; t = (mix32(k) & 1u) ? p.t2 : p.t1; }
        } else if (evict) {
            ev += (g.sub == 0);
            hop++;
            if (old == kEmptySlot) {
                phase = -1;
            } else {
                kv = old;
                k = key_of(kv);
                const Pair q = pair_of(tv, k);
                t = (t == q.t1) ? q.t2 : q.t1;
                if (hop >= tv.max_hops) { fail = true; phase = -1; }
            }
        }
        warp_append(g.sub == 0 && fail, kv, fail_list, fcur);
    }
    block_add<kThreads>(ctr + C_EVICT, ev);
}

// Reinsert every live slot of a detached buffer through the insert path (the
// resize baselines of P:L736 and P:L809).
template <int B>
__global__ void __launch_bounds__(kThreads) k_reinsert(TableView tv, const unsigned long long* __restrict__ slots,
                                                       uint64_t nslots, unsigned long long* __restrict__ fail_list,
                                                       unsigned long long* __restrict__ ctr) {
    constexpr int G = B / 4, QPW = 32 / G;
    __shared__ SmemView sv;
    load_view(tv, sv);
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    uint32_t ev = 0;
    for (uint64_t base = w * QPW; base < nslots; base += nwarps * QPW) {
        const uint64_t i = base + grp;
        unsigned long long kv = i < nslots ? slots[i] : kEmptySlot;
        const bool done = coop_place<B>(g, tv, sv, kv, kv == kEmptySlot, true, ev);
        warp_append(g.sub == 0 && !done, kv, fail_list, ctr + C_FAIL);
    }
    block_add<kThreads>(ctr + C_EVICT, ev);
}

// ------------------------------------------------------------- delete (S4)
// Probe t1 then t2; the lane holding the key overwrites its slot with EMPTY (no
// lock: keys in a batch are distinct).  U ops per group in flight.
// LK: a key found in the `locked` subtable (being resized concurrently) is
// reported DELETED with its old value, and its removal is appended to `defer`
// (applied by k_apply after the resize is committed).
// S1 as in k_find (staged batches): the key is known absent from its first-choice bucket.
template <int B, int U, bool LK = false, bool STASH = false, bool S1 = false>
__global__ void __launch_bounds__(kThreads, DYC_DELETE_MINB) k_delete(TableView tv, const uint32_t* __restrict__ keys,
                                                     uint32_t* __restrict__ old_vals,
                                                     uint8_t* __restrict__ status, uint64_t n,
                                                     unsigned long long* __restrict__ ctr,
                                                     uint32_t locked = 0xFFFFFFFFu,
                                                     unsigned long long* __restrict__ defer = nullptr,
                                                     const unsigned long long* __restrict__ n_dev = nullptr,
                                                     const uint32_t* __restrict__ idx = nullptr) {
    // S1: op i (keys[i]) is entry i of a staged batch's need list; its results go to [idx[i]]
    constexpr int G = B / 4, QPW = 32 / G;
    __shared__ SmemView sv;
    load_view(tv, sv);
    if (n_dev) n = min(n, (uint64_t)*n_dev);     // op count known on the device only (mixed batches)
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    const uint64_t sn = STASH ? stash_count(tv) : 0ull;
    unsigned long long removed = 0, n_ops = 0, n_p2 = 0;
    for (uint64_t base = w * (QPW * U); base < n; base += nwarps * (QPW * U)) {
        uint64_t i[U];
        uint32_t k[U];
        unsigned long long s1[U][4], s2[U][4];
        unsigned long long* b1[U];
        unsigned long long* b2[U];
        unsigned h1[U];
        bool need2[U], lk1[U], lk2[U];
        int j1[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            i[u] = base + (uint64_t)u * QPW + grp;
            k[u] = i[u] < n ? __ldg(keys + i[u]) : kEmptyKey;
            const Pair p = pair_of(tv, k[u]);
            lk1[u] = LK && p.t1 == locked;
            lk2[u] = LK && p.t2 == locked;
            b1[u] = bucket_ptr(sv, p.t1, bucket_of(sv, p.t1, k[u]), B);
            b2[u] = bucket_ptr(sv, p.t2, bucket_of(sv, p.t2, k[u]), B);
            if (S1) {
#pragma unroll
                for (int q = 0; q < 4; q++) s1[u][q] = kEmptySlot;
            } else {
                probe_cg<B>(b1[u] + 4 * g.sub, s1[u]);
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const bool active = k[u] != kEmptyKey;
            j1[u] = active ? match_slot<4>(s1[u], k[u]) : -1;
            h1[u] = g.ballot(j1[u] >= 0);
            // no first-choice-full shortcut here (unlike k_find / k_upsert): the
            // deletes of this same batch make buckets non-full while it runs
            need2[u] = active && h1[u] == 0;
            n_ops += g.sub == 0 && active;
            n_p2 += g.sub == 0 && need2[u];
#pragma unroll
            for (int q = 0; q < 4; q++) s2[u][q] = kEmptySlot;
            probe_cg_pred<B>(b2[u] + 4 * g.sub, s2[u], need2[u]);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            uint32_t lv1 = 0, lv2 = 0;
            lookup_slot<4>(s1[u], k[u], lv1);
            lookup_slot<4>(s2[u], k[u], lv2);
            const int j2 = need2[u] ? match_slot<4>(s2[u], k[u]) : -1;
            const unsigned h2 = g.ballot(j2 >= 0);
            if (h1[u] && !lk1[u] && g.sub == first_lane(h1[u])) st_u64_cg(b1[u] + 4 * g.sub + j1[u], kEmptySlot);
            if (h2 && !lk2[u] && g.sub == first_lane(h2)) st_u64_cg(b2[u] + 4 * g.sub + j2, kEmptySlot);
            if (LK) warp_append(g.sub == 0 && ((h1[u] && lk1[u]) || (h2 && lk2[u])), make_kv(k[u], 0u), defer, ctr + C_DEFER);
            const uint32_t o1 = g.bcast32(lv1, first_lane(h1[u]));
            const uint32_t o2 = g.bcast32(lv2, first_lane(h2));
            bool hit = (h1[u] | h2) != 0;
            uint32_t ov = h1[u] ? o1 : (h2 ? o2 : kEmptyKey);
            if (sn) {                       // a stashed pair: remove it from the stash
                const int64_t at = stash_find(g, tv, sn, k[u], !hit && k[u] != kEmptyKey);
                if (at >= 0) {
                    ov = val_of(tv.stash[at]);
                    if (g.sub == 0) st_u64_cg(tv.stash + at, kEmptySlot);
                    hit = true;
                }
            }
            if (g.sub == 0 && i[u] < n) {
                const uint64_t o = S1 ? (uint64_t)__ldg(idx + i[u]) : i[u];
                if (old_vals) old_vals[o] = ov;
                if (status) status[o] = hit ? 1 : 0;
            }
            removed += (g.sub == 0 && hit);
        }
    }
    block_add<kThreads>(ctr + C_REMOVED, removed);
    if (tv.probe) {
        block_add<kThreads>(tv.probe + 4, n_ops);
        block_add<kThreads>(tv.probe + 5, n_p2);
    }
}

// Applies the deferred ops of a batch that ran while a subtable was locked by a
// resize (NEXT-1), once the resize is committed: each listed key is present in
// one of its two candidate buckets; `del` removes it, otherwise its value is
// replaced by the listed one.  One lane group per entry.
template <int B>
__global__ void __launch_bounds__(kThreads) k_apply(TableView tv, const unsigned long long* __restrict__ list,
                                                    const unsigned long long* __restrict__ count_ptr, bool del) {
    constexpr int G = B / 4, QPW = 32 / G;
    __shared__ SmemView sv;
    load_view(tv, sv);
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t cnt = *count_ptr;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    for (uint64_t base = w * QPW; base < cnt; base += nwarps * QPW) {
        const uint64_t i = base + grp;
        const unsigned long long kv = i < cnt ? list[i] : kEmptySlot;
        const uint32_t k = key_of(kv);
        const Pair p = pair_of(tv, k);
        const unsigned long long new_e = del ? kEmptySlot : kv;
#pragma unroll
        for (int h = 0; h < 2; h++) {
            unsigned long long* bp = bucket_ptr(sv, h ? p.t2 : p.t1, bucket_of(sv, h ? p.t2 : p.t1, k), B);
            unsigned long long s[4];
            probe_cg<B>(bp + 4 * g.sub, s);
            const int j = k != kEmptyKey ? match_slot<4>(s, k) : -1;
            const unsigned hb = g.ballot(j >= 0);
            if (hb && g.sub == first_lane(hb)) st_u64_cg(bp + 4 * g.sub + j, new_e);
        }
    }
}

// ------------------------------------------------------------- upsize (S8)
// One lane per old slot; the B lanes of a bucket rank their entries with a
// ballot (the warp-cooperative bucket pass of P:L379-380).  New bucket b gets the
// entries that stay, b+n_old the ones that move; unused slots are written EMPTY,
// so the new buffer needs no memset.  Streams: read 8 B, write 16 B per old slot.
// Streaming layout: each thread loads kResU slots up front (bytes in flight for
// HBM), the two new buckets are assembled in a per-warp shared-memory tile, and
// lane s then writes slot s of both, so every store instruction of a warp covers
// 256 contiguous bytes.
#ifndef DYC_RES_U_UP
#define DYC_RES_U_UP 4
#endif
#ifndef DYC_RES_U_DOWN
#define DYC_RES_U_DOWN 4
#endif
constexpr int kResU = DYC_RES_U_UP;      // slots per thread per pass, upsize
constexpr int kResUD = DYC_RES_U_DOWN;   // new slots per thread per pass, downsize

template <int B>
// In place (DYC_RESIZE_IN_PLACE) old_s == new_s: bucket b is read and written
// by the same B lanes (the ballots order every read of b before its writes),
// and b + n_old is fresh memory no lane reads, so no pointer is __restrict__.
__global__ void __launch_bounds__(kThreads, 8) k_upsize(const unsigned long long* old_s,
                                                     unsigned long long* new_s, uint32_t n_old,
                                                     uint32_t a, uint32_t b, uint64_t magic2, uint32_t n2) {
    static_assert(B <= 32 && (32 % B) == 0, "bucket must divide a warp");
    __shared__ unsigned long long tile[kThreads / 32][2][32];
    const uint64_t total = (uint64_t)n_old * B;
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned gbase = lane & ~(unsigned)(B - 1);
    const unsigned gmask = (B == 32) ? kFull : (((1u << B) - 1u) << gbase);
    const unsigned lt = lanemask_lt() & gmask;
    const unsigned s = lane & (B - 1);
    for (uint64_t base = (uint64_t)blockIdx.x * kThreads * kResU; base < total;
         base += (uint64_t)gridDim.x * kThreads * kResU) {
        unsigned long long e[kResU];
#pragma unroll
        for (int u = 0; u < kResU; u++) {
            const uint64_t g = base + (uint64_t)u * kThreads + threadIdx.x;
            e[u] = g < total ? __ldcs(old_s + g) : kEmptySlot;
        }
#pragma unroll
        for (int u = 0; u < kResU; u++) {
            const uint64_t g = base + (uint64_t)u * kThreads + threadIdx.x;
            const uint32_t bucket = (uint32_t)(g / B);
            const bool occ = key_of(e[u]) != kEmptyKey;
            bool hi = false;
            if (occ) hi = fastmod(hx(a, b, key_of(e[u])), magic2, n2) != bucket;
            const unsigned hb = __ballot_sync(kFull, occ && hi) & gmask;
            const unsigned lb = __ballot_sync(kFull, occ && !hi) & gmask;
            tile[w][0][lane] = kEmptySlot;
            tile[w][1][lane] = kEmptySlot;
            __syncwarp();
            if (occ) tile[w][hi ? 1 : 0][gbase + __popc((hi ? hb : lb) & lt)] = e[u];
            __syncwarp();
            const unsigned long long lo_v = tile[w][0][lane], hi_v = tile[w][1][lane];
            __syncwarp();
            if (g < total) {
                __stcs(new_s + (uint64_t)bucket * B + s, lo_v);
                __stcs(new_s + ((uint64_t)bucket + n_old) * B + s, hi_v);
            }
        }
    }
}

// ----------------------------------------------------------- downsize (S9)
// One lane per slot of the halved table: new bucket b' takes old b' then old
// b'+h in slot order, keeps the first B (reading Q18) and appends the rest to
// the residual list, which k_place then inserts into the pairs' other tables
// (P:L392-393).  Streams: read 16 B, write 8 B per new slot.  Same streaming
// layout as k_upsize (kResU slots per thread, per-warp tile, coalesced stores).
template <int B>
// In place old_s == new_s: new bucket b' is written only by the lanes that read
// old b' and b'+h (after the ballots on them); the upper half is unmapped later.
__global__ void __launch_bounds__(kThreads) k_downsize(const unsigned long long* old_s,
                                                       unsigned long long* new_s, uint32_t h,
                                                       unsigned long long* __restrict__ residual,
                                                       unsigned long long* __restrict__ ctr) {
    static_assert(B <= 32 && (32 % B) == 0, "bucket must divide a warp");
    __shared__ unsigned long long tile[kThreads / 32][32];
    // residuals of one pass are gathered per block and appended with ONE
    // global atomic (a per-warp append put ~0.4M atomics on one counter)
    __shared__ unsigned long long s_res[kThreads * kResUD];
    __shared__ unsigned s_nres;
    __shared__ unsigned long long s_gbase;
    if (threadIdx.x == 0) s_nres = 0;
    __syncthreads();
    const uint64_t total = (uint64_t)h * B;
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned gbase = lane & ~(unsigned)(B - 1);
    const unsigned gmask = (B == 32) ? kFull : (((1u << B) - 1u) << gbase);
    const unsigned lt = lanemask_lt() & gmask;
    unsigned long long nres = 0;
    for (uint64_t base = (uint64_t)blockIdx.x * kThreads * kResUD; base < total;
         base += (uint64_t)gridDim.x * kThreads * kResUD) {
        unsigned long long e1[kResUD], e2[kResUD];
#pragma unroll
        for (int u = 0; u < kResUD; u++) {
            const uint64_t g = base + (uint64_t)u * kThreads + threadIdx.x;
            e1[u] = g < total ? __ldcs(old_s + g) : kEmptySlot;
            e2[u] = g < total ? __ldcs(old_s + g + total) : kEmptySlot;
        }
#pragma unroll
        for (int u = 0; u < kResUD; u++) {
            const uint64_t g = base + (uint64_t)u * kThreads + threadIdx.x;
            const bool o1 = key_of(e1[u]) != kEmptyKey, o2 = key_of(e2[u]) != kEmptyKey;
            const unsigned m1 = __ballot_sync(kFull, o1) & gmask;
            const unsigned m2 = __ballot_sync(kFull, o2) & gmask;
            const uint32_t c1 = __popc(m1);
            const uint32_t r1 = __popc(m1 & lt), r2 = c1 + __popc(m2 & lt);
            tile[w][lane] = kEmptySlot;
            __syncwarp();
            if (o1) tile[w][gbase + r1] = e1[u];                  // r1 < c1 <= B always fits
            const bool res = o2 && r2 >= (uint32_t)B;
            if (o2 && !res) tile[w][gbase + r2] = e2[u];
            __syncwarp();
            const unsigned long long v = tile[w][lane];
            __syncwarp();
            if (g < total) __stcs(new_s + g, v);
            nres += res;
            const unsigned rb = __ballot_sync(kFull, res);
            unsigned wb = 0;
            if (rb && lane == 0) wb = atomicAdd(&s_nres, (unsigned)__popc(rb));
            wb = __shfl_sync(kFull, wb, 0);
            if (res) s_res[wb + __popc(rb & lanemask_lt())] = e2[u];
        }
        __syncthreads();
        const unsigned nb = s_nres;
        if (nb) {
            if (threadIdx.x == 0) s_gbase = atomicAdd(ctr + C_RESIDUAL, (unsigned long long)nb);
            __syncthreads();
            for (unsigned i = threadIdx.x; i < nb; i += kThreads) residual[s_gbase + i] = s_res[i];
        }
        __syncthreads();
        if (threadIdx.x == 0) s_nres = 0;
        __syncthreads();
    }
    block_add<kThreads>(ctr + C_RES_TOTAL, nres);
}

// ---------------------------------------------------------- stats / dump (S10)
// Paper-weighted placement snapshot: w[t] = n_t / max(C(m_t, 2), 1)
// from the live counts k_count left in ctr[C_COUNT0 + t] (n_t in slots; the
// common factor B cancels in the ratio).
__global__ void k_weights(TableView tv, uint32_t B, const unsigned long long* __restrict__ ctr, float* __restrict__ w) {
    const uint32_t t = threadIdx.x;
    if (t >= tv.d) return;
    const double m = (double)ctr[C_COUNT0 + t];
    double c = m * (m - 1.0) / 2.0;
    if (c < 1.0) c = 1.0;
    w[t] = (float)((double)tv.sub[t].n * (double)B / c);
}

template <int B>
__global__ void __launch_bounds__(kThreads) k_count(TableView tv, uint32_t t, unsigned long long* __restrict__ ctr) {
    const unsigned long long* slots = tv.sub[t].slots;
    const uint64_t total = (uint64_t)tv.sub[t].n * B;
    unsigned long long cnt = 0, second = 0;
    for (uint64_t g = (uint64_t)blockIdx.x * kThreads + threadIdx.x; g < total; g += (uint64_t)gridDim.x * kThreads) {
        const unsigned long long e = slots[g];
        if (key_of(e) != kEmptyKey) {
            cnt++;
            if (pair_of(tv, key_of(e)).t2 == t) second++;
        }
    }
    block_add<kThreads>(ctr + C_COUNT0 + t, cnt);
    block_add<kThreads>(ctr + C_SECOND, second);
}

template <int B>
__global__ void __launch_bounds__(kThreads) k_dump(TableView tv, uint32_t t, unsigned long long* __restrict__ kv,
                                                   uint32_t* __restrict__ tab, unsigned long long* __restrict__ bkt,
                                                   uint64_t cap, unsigned long long* __restrict__ ctr) {
    const unsigned long long* slots = tv.sub[t].slots;
    const uint64_t total = (uint64_t)tv.sub[t].n * B;
    for (uint64_t base = (uint64_t)blockIdx.x * kThreads; base < total; base += (uint64_t)gridDim.x * kThreads) {
        const uint64_t g = base + threadIdx.x;
        const unsigned long long e = g < total ? slots[g] : kEmptySlot;
        const bool occ = key_of(e) != kEmptyKey;
        const unsigned m = __ballot_sync(kFull, occ);
        if (!m) continue;
        const int leader = __ffs(m) - 1;
        unsigned long long pos = 0;
        if ((int)(threadIdx.x & 31) == leader) pos = atomicAdd(ctr + C_DUMP, (unsigned long long)__popc(m));
        pos = __shfl_sync(kFull, pos, leader) + __popc(m & lanemask_lt());
        if (occ && pos < cap) {
            kv[pos] = e;
            tab[pos] = t;
            bkt[pos] = g / B;
        }
    }
}

__global__ void k_hash_probe(TableView tv, const uint32_t* __restrict__ keys, uint64_t n, uint32_t* __restrict__ x,
                             uint32_t* __restrict__ pr) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t k = keys[i];
    for (uint32_t s = 0; s < tv.d + 2; s++) x[i * (tv.d + 2) + s] = hx(tv.a[s], tv.b[s], k);
    const Pair p = pair_of(tv, k);
    pr[2 * i] = p.t1;
    pr[2 * i + 1] = p.t2;
}

// --------------------------------------------------------------- routing (S11)
// ------------------------------------------------- grouping by destination
// Used for shard routing (dest = x_{d+1}(k) mod G) and for mixed batches
// (dest = op code).  Block-aggregated: each block bins a tile of kTileItems ops in
// shared memory, reserves its range per destination with ONE global atomic per
// (block, destination), then places its ops; so contention does not grow with
// the batch even when G is 1.
constexpr int kTileItems = 8;

// Warp-aggregated shared-memory counter increment: the lanes of a warp that
// share a destination are grouped with __match_any_sync and their leader adds
// the group's size with ONE atomic; each lane gets its rank inside the
// destination.  (One atomic per lane on a shared counter serialises 32-way
// when every op has the same destination: G = 1, or an op-code split.)
// Every lane of the warp must call it; lanes with valid == false take no slot.
__device__ __forceinline__ unsigned warp_rank_add(unsigned* counters, uint32_t d, bool valid) {
    const uint32_t key = valid ? d : 0xFFFFFFFFu;
    const unsigned peers = __match_any_sync(kFull, key);
    const unsigned leader = __ffs(peers) - 1;
    const unsigned lane = threadIdx.x & 31;
    unsigned b = 0;
    if (valid && lane == leader) b = atomicAdd(&counters[d], (unsigned)__popc(peers));
    b = __shfl_sync(kFull, b, leader);
    return b + __popc(peers & ((1u << lane) - 1u));
}

struct HashDest {
    uint32_t a, b, world;
    uint64_t magic;
    const uint32_t* keys;
    __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return fastmod(hx(a, b, keys[i]), magic, world); }
    __device__ __forceinline__ uint32_t of_key(uint32_t k) const { return fastmod(hx(a, b, k), magic, world); }
};
struct OpDest {
    const uint8_t* ops;
    __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return ops[i] & 3u; }
};

// Pass 1: per-warp shared histograms (32-bit shared atomics, low contention),
// summed per block, one global atomic per (block, destination).
template <class Dest>
__global__ void __launch_bounds__(kThreads) k_group_count(Dest dest, uint64_t n, uint32_t world,
                                                          unsigned long long* __restrict__ counts) {
    extern __shared__ unsigned hist32[];                    // [kThreads/32][world]
    for (uint32_t x = threadIdx.x; x < (kThreads / 32) * world; x += blockDim.x) hist32[x] = 0;
    __syncthreads();
    unsigned* mine = hist32 + (threadIdx.x >> 5) * world;
    constexpr int IT = 4;
    for (uint64_t b0 = (uint64_t)blockIdx.x * kThreads * IT; b0 < n; b0 += (uint64_t)gridDim.x * kThreads * IT) {
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            warp_rank_add(mine, i < n ? dest(i) : 0u, i < n);
        }
    }
    __syncthreads();
    for (uint32_t w = threadIdx.x; w < world; w += blockDim.x) {
        unsigned long long c = 0;
        for (int q = 0; q < kThreads / 32; q++) c += hist32[q * world + w];
        if (c) atomicAdd(&counts[w], c);
    }
}

// Pass 2: each block bins a tile of kTileItems ops per thread in shared memory,
// reserves its range per destination with ONE global atomic per (tile, dest),
// then writes its ops (order inside a (tile, dest) range is unspecified).
template <class Dest>
__global__ void __launch_bounds__(kThreads) k_group_scatter(Dest dest, const uint32_t* __restrict__ keys,
                                                            const uint32_t* __restrict__ vals_in, uint64_t n,
                                                            uint32_t world, unsigned long long* __restrict__ cursor,
                                                            uint32_t* __restrict__ keys_out,
                                                            uint32_t* __restrict__ vals_out,
                                                            uint32_t* __restrict__ pos_out,
                                                            const uint8_t* __restrict__ tags_in = nullptr,
                                                            uint8_t* __restrict__ tags_out = nullptr) {
    extern __shared__ unsigned long long base[];            // per-destination global base of this tile
    unsigned* cnt = (unsigned*)(base + world);              // per-destination count / running rank
    const uint64_t tile = (uint64_t)kThreads * kTileItems;
    for (uint64_t t0 = (uint64_t)blockIdx.x * tile; t0 < n; t0 += (uint64_t)gridDim.x * tile) {
        for (uint32_t w = threadIdx.x; w < world; w += blockDim.x) cnt[w] = 0;
        __syncthreads();
        uint32_t dd[kTileItems], rk[kTileItems];
#pragma unroll
        for (int j = 0; j < kTileItems; j++) {
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            dd[j] = i < n ? dest(i) : 0xFFFFFFFFu;
            rk[j] = warp_rank_add(cnt, dd[j], i < n);           // rank within (tile, dest)
        }
        __syncthreads();
        for (uint32_t w = threadIdx.x; w < world; w += blockDim.x)
            base[w] = cnt[w] ? atomicAdd(&cursor[w], (unsigned long long)cnt[w]) : 0ull;
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kTileItems; j++) {
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            if (dd[j] != 0xFFFFFFFFu) {
                const uint64_t pos = base[dd[j]] + rk[j];
                keys_out[pos] = keys[i];
                if (vals_out) vals_out[pos] = vals_in ? vals_in[i] : 0u;
                if (tags_out) tags_out[pos] = tags_in[i];
                pos_out[i] = (uint32_t)pos;
            }
        }
        __syncthreads();
    }
}

// Fixed region bases for the phases of a mixed batch: op code c's ops go to
// [c*n, (c+1)*n) of the scratch, so every phase's keys start at an address the
// host knows while its count stays on the device (no host wait).
__global__ void k_fixed_bases(unsigned long long* __restrict__ cursor, uint32_t regions, uint64_t n) {
    if (threadIdx.x < regions) cursor[threadIdx.x] = (unsigned long long)threadIdx.x * n;
}

// Exclusive prefix sum of the per-destination counts into the scatter cursors (one block).
__global__ void k_route_offsets(const unsigned long long* __restrict__ counts, uint32_t world,
                                unsigned long long* __restrict__ cursor) {
    if (threadIdx.x == 0) {
        unsigned long long acc = 0;
        for (uint32_t w = 0; w < world; w++) {
            cursor[w] = acc;
            acc += counts[w];
        }
    }
}

__global__ void __launch_bounds__(kThreads) k_route_unpermute(const uint32_t* __restrict__ pos, uint64_t n,
                                                              const uint32_t* __restrict__ rv,
                                                              const uint8_t* __restrict__ rs,
                                                              uint32_t* __restrict__ vals, uint8_t* __restrict__ st) {
    constexpr int IT = 4;                                   // 4 ops per thread, loads in flight together
    for (uint64_t b0 = (uint64_t)blockIdx.x * kThreads * IT; b0 < n; b0 += (uint64_t)gridDim.x * kThreads * IT) {
        uint32_t p[IT], v[IT];
        uint8_t s8[IT];
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            p[j] = i < n ? pos[i] : 0u;
        }
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            v[j] = (i < n && rv && vals) ? rv[p[j]] : 0u;
            s8[j] = (i < n && rs && st) ? rs[p[j]] : 0u;
        }
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            if (i < n) {
                if (rv && vals) vals[i] = v[j];
                if (rs && st) st[i] = s8[j];
            }
        }
    }
}

// ------------------------------------- peer-memory routing (S11, fused path)
// Dispatch and combine written straight into the owners' / requesters' memory
// (NVLink peer pointers from CUDA IPC; local pointers when G shards share one
// GPU).  Replaces route_count + count exchange + route_scatter + all-to-all
// (dispatch) and all-to-all + route_unpermute (combine): the shard hash, the
// reservation of the destination range and the transfer are one kernel, and a
// reply lands at its op's index in the requester's result.
//
// A receive buffer of capacity `cap` is structure-of-arrays, so the owner's
// batch kernels read its keys and values in place:
//   keys u32[cap] @ 0 | vals u32[cap] @ 4cap | meta u64[cap] @ 8cap | tags u8[cap] @ 16cap
// meta = src_index | (uint64)src_rank << 32.
constexpr uint32_t kMaxPeers = 64;
struct PeerPtrs {
    void* p[kMaxPeers];
};
constexpr int kPushItems = 8;                    // ops per thread per tile (tile = 2048 ops)
#ifndef DYC_PUSH_ATOMIC
#define DYC_PUSH_ATOMIC atomicAdd_system
#endif
#ifndef DYC_PUSH_BPS
#define DYC_PUSH_BPS 4                           // resident push blocks per SM (persistent grid)
#endif

// Each block takes a tile of 2048 ops: it hashes them to their shards, ranks
// them per shard in shared memory and stages them there grouped by shard; it
// reserves the tile's range in every destination with ONE system-scope atomic
// on that shard's counter (atomics crossing NVLink scale with tiles, not ops);
// then the staged tile is copied out so that consecutive threads store to
// consecutive addresses of one destination's range (coalesced peer stores).
// Ops past `cap` are not stored (the owner sees count > cap and fails).
__global__ void __launch_bounds__(kThreads) k_route_push(HashDest dest, const uint32_t* __restrict__ vals,
                                                         const uint8_t* __restrict__ tags, uint64_t n,
                                                         uint32_t world, uint32_t src_rank, PeerPtrs recv,
                                                         PeerPtrs recv_count, uint64_t cap) {
    constexpr int T = kThreads * kPushItems;
    __shared__ uint32_t s_key[T], s_val[T], s_idx[T];
    __shared__ uint8_t s_tag[T], s_dst[T];
    __shared__ unsigned cnt[kMaxPeers], off[kMaxPeers + 1];
    __shared__ unsigned long long base[kMaxPeers];
    // the tile's keys, values and op codes are loaded into registers in one go,
    // and the next tile's loads are issued before the current tile is copied
    // out, so each tile exposes at most one memory latency
    uint32_t kk[kPushItems], vv[kPushItems];
    uint8_t tg[kPushItems];
    auto load_tile = [&](uint64_t t0) {
        const unsigned nt = t0 < n ? (unsigned)((n - t0) < (uint64_t)T ? (n - t0) : (uint64_t)T) : 0u;
#pragma unroll
        for (int j = 0; j < kPushItems; j++) {
            const unsigned li = j * kThreads + threadIdx.x;
            const bool ok = li < nt;
            kk[j] = ok ? __ldcs(dest.keys + t0 + li) : 0u;
            vv[j] = (ok && vals) ? __ldcs(vals + t0 + li) : 0u;
            tg[j] = (ok && tags) ? tags[t0 + li] : (uint8_t)0;
        }
    };
    const uint64_t stride = (uint64_t)gridDim.x * T;
    uint64_t t0 = (uint64_t)blockIdx.x * T;
    if (t0 < n) load_tile(t0);
    for (; t0 < n; t0 += stride) {
        const unsigned nt = (unsigned)((n - t0) < (uint64_t)T ? (n - t0) : (uint64_t)T);
        for (uint32_t w = threadIdx.x; w < world; w += blockDim.x) cnt[w] = 0;
        __syncthreads();
        uint32_t dd[kPushItems], rk[kPushItems];
#pragma unroll
        for (int j = 0; j < kPushItems; j++) {
            const unsigned li = j * kThreads + threadIdx.x;
            dd[j] = li < nt ? dest.of_key(kk[j]) : 0xFFFFFFFFu;
            rk[j] = warp_rank_add(cnt, dd[j], li < nt);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned acc = 0;
            for (uint32_t w = 0; w < world; w++) { off[w] = acc; acc += cnt[w]; }
            off[world] = acc;
        }
        for (uint32_t w = threadIdx.x; w < world; w += blockDim.x)
            base[w] = cnt[w] ? DYC_PUSH_ATOMIC((unsigned long long*)recv_count.p[w], (unsigned long long)cnt[w])
                             : 0ull;
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kPushItems; j++) {
            const unsigned li = j * kThreads + threadIdx.x;
            if (li < nt) {
                const unsigned p = off[dd[j]] + rk[j];
                s_key[p] = kk[j];
                s_val[p] = vv[j];
                s_idx[p] = (uint32_t)(t0 + li);
                s_tag[p] = tg[j];
                s_dst[p] = (uint8_t)dd[j];
            }
        }
        __syncthreads();
        if (t0 + stride < n) load_tile(t0 + stride);          // in flight during the copy-out
        for (unsigned p = threadIdx.x; p < nt; p += kThreads) {
            const uint32_t w = s_dst[p];
            const uint64_t g = base[w] + (p - off[w]);
            if (g < cap) {
                char* b = (char*)recv.p[w];
                reinterpret_cast<uint32_t*>(b)[g] = s_key[p];
                if (vals) reinterpret_cast<uint32_t*>(b + 4 * cap)[g] = s_val[p];
                reinterpret_cast<unsigned long long*>(b + 8 * cap)[g] =
                    (unsigned long long)s_idx[p] | ((unsigned long long)src_rank << 32);
                if (tags) reinterpret_cast<uint8_t*>(b + 16 * cap)[g] = s_tag[p];
            }
        }
        __syncthreads();
    }
    __threadfence_system();
}

// Combine: the result of received op j goes to index src_index of its
// requester's result arrays (peer pointers), i.e. straight into request order.
__global__ void __launch_bounds__(kThreads) k_route_reply(const unsigned long long* __restrict__ meta, uint64_t n,
                                                          const uint32_t* __restrict__ rv,
                                                          const uint8_t* __restrict__ rs, PeerPtrs out_vals,
                                                          PeerPtrs out_status) {
    constexpr int IT = 4;
    for (uint64_t b0 = (uint64_t)blockIdx.x * kThreads * IT; b0 < n; b0 += (uint64_t)gridDim.x * kThreads * IT) {
        unsigned long long m[IT];
        uint32_t v[IT];
        uint8_t s8[IT];
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            m[j] = i < n ? meta[i] : 0ull;
            v[j] = (i < n && rv) ? rv[i] : 0u;
            s8[j] = (i < n && rs) ? rs[i] : 0u;
        }
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            if (i < n) {
                const uint32_t src = (uint32_t)(m[j] >> 32), idx = (uint32_t)m[j];
                if (rv) reinterpret_cast<uint32_t*>(out_vals.p[src])[idx] = v[j];
                if (rs) reinterpret_cast<uint8_t*>(out_status.p[src])[idx] = s8[j];
            }
        }
    }
    __threadfence_system();
}

// ------------------------------------------------------ random-gather ceiling
// The probe access pattern with no table logic: reads of one B-slot bucket at
// uniformly random bucket-aligned offsets, by a G = B/4 lane group with the same
// 256-bit loads and L2 prefetch size as k_find.  Its rate is the random-access
// ceiling the probe kernels are compared with.
// WRITE (1, 2 or 3): after its read, each group also writes into the bucket it
// read (the probe-then-write pattern of an insert or delete: one read plus one
// dirty-line write-back per op); the written word depends only on the group's
// own probe.  1: an 8-byte plain store (delete's EMPTY store); 2: an 8-byte
// atomicCAS (insert's claim of a free slot); 3: a full 32-byte sector store.
template <int B, int WRITE = 0>
__global__ void __launch_bounds__(kThreads) k_gather(unsigned long long* __restrict__ buf, uint64_t n_units,
                                                     uint64_t n_reads, uint64_t seed,
                                                     unsigned long long* __restrict__ sink) {
    constexpr int G = B / 4, QPW = 32 / G, ILP = 4;
    const Grp<G> g;
    const unsigned grp = g.lane / G;
    const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
    const uint64_t w = (uint64_t)blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5);
    unsigned long long acc = 0;
    for (uint64_t base = w * QPW * ILP; base < n_reads; base += nwarps * QPW * ILP) {
        unsigned long long s[ILP][4];
        unsigned long long* wp[ILP];
#pragma unroll
        for (int j = 0; j < ILP; j++) {
            const uint64_t i = base + (uint64_t)j * QPW + grp;
            uint64_t h = (i + seed) * 0x9E3779B97F4A7C15ull;
            h ^= h >> 29;
            h *= 0xBF58476D1CE4E5B9ull;
            h ^= h >> 32;
            unsigned long long* p = buf + __umul64hi(h, n_units) * B + 4 * g.sub;
            if (WRITE) {
                probe_cg_pred<B>(p, s[j], i < n_reads);
                wp[j] = i < n_reads ? p : nullptr;
            } else {
                probe_nc_pred<B>(p, s[j], i < n_reads);
            }
        }
#pragma unroll
        for (int j = 0; j < ILP; j++) acc ^= s[j][0] ^ s[j][1] ^ s[j][2] ^ s[j][3];
        if (WRITE) {
#pragma unroll
            for (int j = 0; j < ILP; j++) {
                if (g.sub != 0 || !wp[j]) continue;       // address: the group's own probe only
                if (WRITE == 1) st_u64_cg(wp[j], s[j][0] + 1);
                if (WRITE == 2) acc ^= atomicCAS(wp[j], s[j][0], s[j][0] + 1);
                if (WRITE == 3)
                    asm volatile("st.global.v4.u64 [%0], {%1,%2,%3,%4};" ::"l"(wp[j]), "l"(s[j][0] + 1), "l"(s[j][1]),
                                 "l"(s[j][2]), "l"(s[j][3])
                                 : "memory");
            }
        }
    }
    if (acc == 0x0123456789ABCDEFull) *sink = acc;   // keeps the loads alive
}

}  // namespace dyc
