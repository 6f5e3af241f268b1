// dyc_binned.cuh — region-binned execution of large batches (L2-blocked probes).
//
// The direct kernels (dyc_kernels.cuh) probe buckets in batch order, so a batch
// much larger than L2 costs one random HBM access per probe: about 50-55 G
// accesses/s on B200, whatever the access size (profiles/r1_memory_model.md).
// A batch of n ops over a table of NB buckets touches every bucket n/NB times
// per probe pass (6.8 at config C2).  Binned execution turns that reuse into L2
// hits: the ops are grouped by the REGION of the bucket they probe next (a
// region is 2^rshift consecutive buckets of the concatenated subtables, sized
// to a fraction of the 126 MB L2), and each pass walks the groups in region
// order, so the blocks in flight probe one region at a time.  The pass that
// follows is fed through the same grouping, and the per-op results are grouped
// by op index (2^ishift ops per group, an L2-sized output window) before they
// are written back in request order.
//
// Semantics are those of the direct kernels (the paper's batch model, P:L464;
// keys distinct within a batch, Q9), pass by pass:
//   find   F1 probe h^{t1}  ->  F2 probe h^{t2} for F1 misses (<= 2 lookups)
//   delete the same, the matching slot is overwritten with EMPTY
//   insert I1 probe t1, I2 probe t2: existence over BOTH buckets before any
//          placement (reading Q7), an existing key's value is replaced (Alg. 1
//          L536-539, Q8); then first-fit placement over (t1, t2) (reading Q3):
//          I2 CASes keys whose t1 bucket was full into t2 right away, I3 CASes
//          the others into t1 and passes overflow to I4 (t2); keys with both
//          buckets full go to the eviction kernel k_place.
// Keys never move during I1-I4 (CAS into EMPTY slots only, no eviction), so the
// existence check is exact, as in k_upsert.  Used only when no upsize can be
// needed before placement ((m+n) <= beta*N, the FUSE case of k_upsert) and no
// resize is in flight; everything else takes the direct kernels.
//
// Per-op streams are structure-of-arrays records (key, value, op index) written
// by block-aggregated appends: a block ranks its records per bin in shared
// memory and reserves each bin's range with ONE global atomic, so contention
// does not grow with the batch.  Bin b of a pass occupies [off[b], off[b+1])
// of its record array (capacity from the per-region counts of k_bin_hist) and
// is filled up to cur[b]; positions past cur[b] are skipped.
#pragma once
#include "dyc_kernels.cuh"

namespace dyc {

constexpr uint32_t kMaxBins = 1024;   // regions per bin set; result groups per batch
constexpr int kScatterItems = 8;      // ops per thread per tile in k_bin_scatter
constexpr int kOutItems = 8;          // records per thread in k_bin_out

struct BinCtx {
    uint64_t gbase[kMaxD];   // first global bucket of subtable t (subtables concatenated)
    uint32_t rshift;         // region of a bucket = (gbase[t] + b) >> rshift
    uint32_t R;              // regions
    uint32_t ishift;         // result group of op i = i >> ishift
    uint32_t Rout;           // result groups
};

// Per-block shared copy of the bin context (indexed by a lane-varying t).
struct BinSmem {
    uint64_t gbase[kMaxD];
};

__device__ __forceinline__ void load_bins(const TableView& tv, const BinCtx& bc, BinSmem& bs) {
    if (threadIdx.x < tv.d) bs.gbase[threadIdx.x] = bc.gbase[threadIdx.x];
}

__device__ __forceinline__ uint32_t region_of(const BinSmem& bs, uint32_t rshift, uint32_t t, uint32_t b) {
    return (uint32_t)((bs.gbase[t] + b) >> rshift);
}

// bin j with off[j] <= p < off[j+1] (off has R+1 entries, non-decreasing)
__device__ __forceinline__ uint32_t bin_of_pos(const uint32_t* off, uint32_t R, uint32_t p) {
    uint32_t lo = 0, hi = R;            // invariant: off[lo] <= p < off[hi]
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (off[mid] <= p) lo = mid; else hi = mid;
    }
    return lo;
}

// ------------------------------------------------------------- region counts
// hist[0..R): ops per region of h^{t1}(k); hist[R..2R): per region of h^{t2}(k).
// The reserved key is not counted (its result is written by k_bin_scatter).
__global__ void __launch_bounds__(kThreads) k_bin_hist(TableView tv, BinCtx bc, const uint32_t* __restrict__ keys,
                                                       uint64_t n, uint32_t* __restrict__ hist) {
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t h[];                      // [2R]
    for (uint32_t x = threadIdx.x; x < 2 * bc.R; x += blockDim.x) h[x] = 0;
    load_bins(tv, bc, bs);
    load_view(tv, sv);                                   // (syncs)
    constexpr int IT = 4;
    for (uint64_t b0 = (uint64_t)blockIdx.x * kThreads * IT; b0 < n; b0 += (uint64_t)gridDim.x * kThreads * IT) {
        uint32_t k[IT];
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = b0 + (uint64_t)j * kThreads + threadIdx.x;
            k[j] = i < n ? __ldcs(keys + i) : kEmptyKey;
        }
#pragma unroll
        for (int j = 0; j < IT; j++) {
            if (k[j] == kEmptyKey) continue;
            const Pair p = pair_of(tv, k[j]);
            atomicAdd(&h[region_of(bs, bc.rshift, p.t1, bucket_of(sv, p.t1, k[j]))], 1u);
            atomicAdd(&h[bc.R + region_of(bs, bc.rshift, p.t2, bucket_of(sv, p.t2, k[j]))], 1u);
        }
    }
    __syncthreads();
    for (uint32_t x = threadIdx.x; x < 2 * bc.R; x += blockDim.x)
        if (h[x]) atomicAdd(&hist[x], h[x]);
}

// Block-wide exclusive scan of up to 1024 values (one per thread; blockDim 1024).
__device__ __forceinline__ uint32_t block_excl_scan_1024(uint32_t v, uint32_t* warp_sums) {
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (unsigned)o) x += y;
    }
    if (lane == 31) warp_sums[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t s = warp_sums[lane];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, s, o);
            if (lane >= (unsigned)o) s += y;
        }
        warp_sums[lane] = s;                              // inclusive over warps
    }
    __syncthreads();
    const uint32_t before = w ? warp_sums[w - 1] : 0u;
    __syncthreads();
    return before + x - v;
}

// Offsets of the two bin sets and the initial cursors (one block of 1024 threads):
//   off[0..R]       = exclusive scan of hist[0..R)   (regions of t1)
//   off[R+1..2R+1]  = exclusive scan of hist[R..2R)  (regions of t2)
//   cur[c*R + j]    = off of cursor set c's bins: c = 0, 2 -> t1 offsets; 1, 3 -> t2 offsets
//   rcur[j]         = j << ishift (result group j holds ops [j<<ishift, (j+1)<<ishift))
__global__ void __launch_bounds__(1024) k_bin_offsets(const uint32_t* __restrict__ hist, uint32_t R, uint32_t Rout,
                                                      uint32_t ishift, uint32_t* __restrict__ off,
                                                      uint32_t* __restrict__ cur, uint32_t* __restrict__ rcur) {
    __shared__ uint32_t ws[32];
    const uint32_t j = threadIdx.x;
    for (int s = 0; s < 2; s++) {
        const uint32_t v = j < R ? hist[s * R + j] : 0u;
        const uint32_t e = block_excl_scan_1024(v, ws);
        if (j < R) {
            off[s * (R + 1) + j] = e;
            cur[(0 + s) * R + j] = e;
            cur[(2 + s) * R + j] = e;
        }
        if (j == R - 1) off[s * (R + 1) + R] = e + v;
    }
    if (j < Rout) rcur[j] = j << ishift;
}

// ------------------------------------------------------- grouping by region
// Tile of kThreads*kScatterItems ops: rank per t1-region in shared memory, one
// global atomic per (tile, region), then write (key[, value], op index).  The
// reserved key gets its "absent" result here (value EMPTY, flag 0) and no record.
__global__ void __launch_bounds__(kThreads) k_bin_scatter(TableView tv, BinCtx bc, const uint32_t* __restrict__ keys,
                                                          const uint32_t* __restrict__ vals, uint64_t n,
                                                          uint32_t* __restrict__ cur, uint32_t* __restrict__ ok,
                                                          uint32_t* __restrict__ ov, uint32_t* __restrict__ oi,
                                                          uint32_t* __restrict__ rv_out, uint8_t* __restrict__ rs_out) {
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t cnt[];                    // [R]
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const uint64_t tile = (uint64_t)kThreads * kScatterItems;
    for (uint64_t t0 = (uint64_t)blockIdx.x * tile; t0 < n; t0 += (uint64_t)gridDim.x * tile) {
        for (uint32_t x = threadIdx.x; x < bc.R; x += blockDim.x) cnt[x] = 0;
        __syncthreads();
        uint32_t k[kScatterItems], r[kScatterItems], rk[kScatterItems];
#pragma unroll
        for (int j = 0; j < kScatterItems; j++) {
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            k[j] = i < n ? __ldcs(keys + i) : kEmptyKey;
            r[j] = 0xFFFFFFFFu;
            if (k[j] != kEmptyKey) {
                const Pair p = pair_of(tv, k[j]);
                r[j] = region_of(bs, bc.rshift, p.t1, bucket_of(sv, p.t1, k[j]));
                rk[j] = atomicAdd(&cnt[r[j]], 1u);
            } else if (i < n) {
                if (rv_out) rv_out[i] = kEmptyKey;
                if (rs_out) rs_out[i] = 0;
            }
        }
        __syncthreads();
        for (uint32_t x = threadIdx.x; x < bc.R; x += blockDim.x)
            if (cnt[x]) cnt[x] = atomicAdd(&cur[x], cnt[x]);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < kScatterItems; j++) {
            if (r[j] == 0xFFFFFFFFu) continue;
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            const uint32_t pos = cnt[r[j]] + rk[j];
            ok[pos] = k[j];
            if (ov) ov[pos] = __ldcs(vals + i);
            oi[pos] = (uint32_t)i;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------ probe passes
// Common frame of the probe passes: block b takes the records at positions
// [b*TILE, (b+1)*TILE) of its input (TILE = U ops per lane group), skipping the
// unfilled tail of every bin.  Records are appended to at most two output bin
// sets: "next" (R regions, the next pass) and "res" (Rout result groups).
// Shared memory: [in_off R+1][in_cur R][next counts R][res counts Rout].
struct PassIO {
    const uint32_t* in_off;   // R+1 bin offsets of the input
    const uint32_t* in_cur;   // R fill cursors of the input
    const uint32_t* ik;       // input keys
    const uint32_t* iv;       // input values (insert passes)
    const uint32_t* ii;       // input op indices (nullable in placement passes)
    uint32_t* nk;             // next-pass records
    uint32_t* nv;
    uint32_t* ni;
    uint32_t* ncur;           // next-pass cursors [R]
    uint32_t* res_i;          // result records: op index | flags
    uint32_t* res_v;          // result values (find/delete)
    uint32_t* rcur;           // result cursors [Rout]
};

template <int G, int U>
struct PassFrame {
    uint32_t* s_off;
    uint32_t* s_cur;
    uint32_t* s_next;
    uint32_t* s_res;
    uint32_t R, Rout;
    __device__ __forceinline__ PassFrame(uint32_t* smem, const BinCtx& bc, const PassIO& io) {
        R = bc.R;
        Rout = bc.Rout;
        s_off = smem;
        s_cur = s_off + R + 1;
        s_next = s_cur + R;
        s_res = s_next + R;
        for (uint32_t x = threadIdx.x; x <= R; x += blockDim.x) s_off[x] = io.in_off[x];
        for (uint32_t x = threadIdx.x; x < R; x += blockDim.x) {
            s_cur[x] = io.in_cur[x];
            s_next[x] = 0;
        }
        for (uint32_t x = threadIdx.x; x < Rout; x += blockDim.x) s_res[x] = 0;
    }
    static constexpr uint32_t kGroups = kThreads / G;
    static constexpr uint32_t kTile = kGroups * U;
    // position of op u of this lane group, and whether it holds a record
    __device__ __forceinline__ bool pos(unsigned grp_in_block, int u, uint32_t& p) const {
        const uint64_t q = (uint64_t)blockIdx.x * kTile + (uint64_t)u * kGroups + grp_in_block;
        p = (uint32_t)q;
        if (q >= s_off[R]) return false;
        const uint32_t j = bin_of_pos(s_off, R, p);
        return p < s_cur[j];
    }
    // after ranks were taken (__syncthreads before): one global atomic per non-empty bin
    __device__ __forceinline__ void reserve(const PassIO& io) {
        for (uint32_t x = threadIdx.x; x < R; x += blockDim.x)
            if (s_next[x]) s_next[x] = atomicAdd(&io.ncur[x], s_next[x]);
        for (uint32_t x = threadIdx.x; x < Rout; x += blockDim.x)
            if (s_res[x]) s_res[x] = atomicAdd(&io.rcur[x], s_res[x]);
    }
};

__host__ __device__ constexpr uint32_t pass_smem_words(uint32_t R, uint32_t Rout) { return 3 * R + 1 + Rout; }

// F1/F2 (find) and D1/D2 (delete): probe h^{t1} (SECOND = false) or h^{t2}.
// A hit gives a result record (index | 1<<31, value); DEL also overwrites the
// slot with EMPTY.  A miss in pass 1 becomes a record of the t2
// region bins; a miss in pass 2 is a result record (index, EMPTY).
template <int B, int U, bool DEL, bool SECOND>
__global__ void __launch_bounds__(kThreads) k_bin_fd(TableView tv, BinCtx bc, PassIO io,
                                                     unsigned long long* __restrict__ ctr) {
    constexpr int G = B / 4, QPW = 32 / G;
    using F = PassFrame<G, U>;
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    F fr(smem, bc, io);
    load_bins(tv, bc, bs);
    load_view(tv, sv);                                   // (syncs)
    const Grp<G> g;
    const unsigned gib = (threadIdx.x >> 5) * QPW + g.lane / G;
    uint32_t k[U], idx[U], v[U], bin[U], rank[U];
    bool hit[U], has[U], nxt[U];
    {
        unsigned long long s[U][4];
        unsigned long long* bp[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            uint32_t p;
            has[u] = fr.pos(gib, u, p);
            k[u] = has[u] ? __ldcs(io.ik + p) : kEmptyKey;
            idx[u] = has[u] ? __ldcs(io.ii + p) : 0u;
            const Pair pr = pair_of(tv, k[u]);
            const uint32_t t = SECOND ? pr.t2 : pr.t1;
            const uint32_t b = bucket_of(sv, t, k[u]);
            bp[u] = bucket_ptr(sv, t, b, B);
#pragma unroll
            for (int q = 0; q < 4; q++) s[u][q] = kEmptySlot;
            if (DEL) probe_cg_pred<B>(bp[u] + 4 * g.sub, s[u], has[u]);
            else probe_nc_pred<B>(bp[u] + 4 * g.sub, s[u], has[u]);
            if (!SECOND) {
                const uint32_t b2 = bucket_of(sv, pr.t2, k[u]);
                bin[u] = region_of(bs, bc.rshift, pr.t2, b2);
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            uint32_t lv = 0;
            const int j = has[u] ? match_slot<4>(s[u], k[u]) : -1;
            lookup_slot<4>(s[u], k[u], lv);
            const unsigned hb = g.ballot(j >= 0);
            if (DEL && hb && g.sub == first_lane(hb)) st_u64_cg(bp[u] + 4 * g.sub + j, kEmptySlot);
            v[u] = g.bcast32(lv, first_lane(hb));
            hit[u] = hb != 0;
        }
    }
    unsigned long long removed = 0;
    const bool lead = g.sub == 0;
#pragma unroll
    for (int u = 0; u < U; u++) {
        nxt[u] = !SECOND && has[u] && !hit[u];
        if (!has[u] || !lead) continue;
        if (nxt[u]) {
            rank[u] = atomicAdd(&fr.s_next[bin[u]], 1u);
        } else {
            bin[u] = idx[u] >> bc.ishift;
            rank[u] = atomicAdd(&fr.s_res[bin[u]], 1u);
        }
        removed += DEL && hit[u];
    }
    __syncthreads();
    fr.reserve(io);
    __syncthreads();
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (!has[u] || !lead) continue;
        if (nxt[u]) {
            const uint32_t q = fr.s_next[bin[u]] + rank[u];
            io.nk[q] = k[u];
            io.ni[q] = idx[u];
        } else {
            const uint32_t q = fr.s_res[bin[u]] + rank[u];
            io.res_i[q] = idx[u] | (hit[u] ? 0x80000000u : 0u);
            io.res_v[q] = hit[u] ? v[u] : kEmptyKey;
        }
    }
    if (DEL) block_add<kThreads>(ctr + C_REMOVED, removed);
}

// I1 (t1) / I2 (t2): existence check of an insert over both buckets.  A match
// gets its value replaced in place (Alg. 1) and status UPDATED.  In I1
// a miss goes on to the t2 bins carrying "t1 had a free slot" in bit 31 of its
// index.  In I2 a miss is a new key (status INSERTED): with the flag it goes to
// the t1 placement bins (first-fit prefers t1, Q3), otherwise it is CASed into
// a free slot of t2 now, else it is pending for k_place.
template <int B, int U, bool SECOND>
__global__ void __launch_bounds__(kThreads) k_bin_ins(TableView tv, BinCtx bc, PassIO io,
                                                      unsigned long long* __restrict__ pending,
                                                      unsigned long long* __restrict__ ctr) {
    constexpr int G = B / 4, QPW = 32 / G;
    using F = PassFrame<G, U>;
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    F fr(smem, bc, io);
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const Grp<G> g;
    const unsigned gib = (threadIdx.x >> 5) * QPW + g.lane / G;
    uint32_t k[U], v[U], idx[U], bin[U], rank[U];
    bool has[U], hit[U], fwd[U], placed[U];
    unsigned em[U];
    unsigned long long* bp[U];
    unsigned long long kv[U];
    {
        unsigned long long s[U][4];
#pragma unroll
        for (int u = 0; u < U; u++) {
            uint32_t p;
            has[u] = fr.pos(gib, u, p);
            k[u] = has[u] ? __ldcs(io.ik + p) : kEmptyKey;
            v[u] = has[u] ? __ldcs(io.iv + p) : 0u;
            idx[u] = has[u] ? __ldcs(io.ii + p) : 0u;
            kv[u] = make_kv(k[u], v[u]);
            const Pair pr = pair_of(tv, k[u]);
            const uint32_t t = SECOND ? pr.t2 : pr.t1;
            bp[u] = bucket_ptr(sv, t, bucket_of(sv, t, k[u]), B);
#pragma unroll
            for (int q = 0; q < 4; q++) s[u][q] = kEmptySlot;
            probe_cg_pred<B>(bp[u] + 4 * g.sub, s[u], has[u]);
            const uint32_t tn = SECOND ? pr.t1 : pr.t2;   // bins of the next pass
            bin[u] = region_of(bs, bc.rshift, tn, bucket_of(sv, tn, k[u]));
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const int j = has[u] ? match_slot<4>(s[u], k[u]) : -1;
            const unsigned hb = g.ballot(j >= 0);
            if (hb && g.sub == first_lane(hb)) st_u64_cg(bp[u] + 4 * g.sub + j, kv[u]);
            hit[u] = hb != 0;
            em[u] = empty_mask(s[u]);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const bool anyfree = g.ballot(has[u] && em[u] != 0) != 0;
            if (!SECOND) {
                fwd[u] = has[u] && !hit[u];               // on to I2, flag: t1 had a free slot
                if (fwd[u] && anyfree) idx[u] |= 0x80000000u;
            } else {
                fwd[u] = has[u] && !hit[u] && (idx[u] & 0x80000000u);   // on to I3 (t1 placement)
                idx[u] &= 0x7FFFFFFFu;
            }
            placed[u] = false;
        }
    }
    if (SECOND) {
        bool want[U];
#pragma unroll
        for (int u = 0; u < U; u++) want[u] = has[u] && !hit[u] && !fwd[u];
        coop_cas_multi<G, U>(g, bp, em, want, kv, placed);
#pragma unroll
        for (int u = 0; u < U; u++) warp_append(g.sub == 0 && want[u] && !placed[u], kv[u], pending, ctr + C_PENDING);
    }
    const bool lead = g.sub == 0;
    uint32_t rbin[U], rrank[U];
    unsigned long long n_ins = 0, n_upd = 0;
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (!has[u] || !lead) continue;
        if (fwd[u]) rank[u] = atomicAdd(&fr.s_next[bin[u]], 1u);
        const bool res = hit[u] || SECOND;                // I1 misses get their status in I2
        if (res && io.res_i) {
            rbin[u] = (idx[u] & 0x7FFFFFFFu) >> bc.ishift;
            rrank[u] = atomicAdd(&fr.s_res[rbin[u]], 1u);
        }
        n_upd += hit[u];
        n_ins += SECOND && !hit[u];
    }
    __syncthreads();
    fr.reserve(io);
    __syncthreads();
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (!has[u] || !lead) continue;
        if (fwd[u]) {
            const uint32_t q = fr.s_next[bin[u]] + rank[u];
            io.nk[q] = k[u];
            io.nv[q] = v[u];
            if (!SECOND) io.ni[q] = idx[u];
        }
        if ((hit[u] || SECOND) && io.res_i) {
            const uint32_t q = fr.s_res[rbin[u]] + rrank[u];
            io.res_i[q] = (idx[u] & 0x3FFFFFFFu) | ((hit[u] ? 2u : 1u) << 30);
        }
    }
    block_add<kThreads>(ctr + C_INSERTED, n_ins);
    block_add<kThreads>(ctr + C_UPDATED, n_upd);
}

// I3 (t1) / I4 (t2): first-fit CAS of new keys into a free slot of the bucket
// (fresh probe: earlier passes of this batch may have filled it).  I3 overflow
// goes to the t2 bins (I4), I4 overflow to the pending list (k_place).
template <int B, int U, bool SECOND>
__global__ void __launch_bounds__(kThreads) k_bin_place(TableView tv, BinCtx bc, PassIO io,
                                                        unsigned long long* __restrict__ pending,
                                                        unsigned long long* __restrict__ ctr) {
    constexpr int G = B / 4, QPW = 32 / G;
    using F = PassFrame<G, U>;
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    F fr(smem, bc, io);
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const Grp<G> g;
    const unsigned gib = (threadIdx.x >> 5) * QPW + g.lane / G;
    uint32_t k[U], v[U], bin[U], rank[U];
    bool has[U], placed[U];
    unsigned em[U];
    unsigned long long* bp[U];
    unsigned long long kv[U];
    {
        unsigned long long s[U][4];
#pragma unroll
        for (int u = 0; u < U; u++) {
            uint32_t p;
            has[u] = fr.pos(gib, u, p);
            k[u] = has[u] ? __ldcs(io.ik + p) : kEmptyKey;
            v[u] = has[u] ? __ldcs(io.iv + p) : 0u;
            kv[u] = make_kv(k[u], v[u]);
            const Pair pr = pair_of(tv, k[u]);
            const uint32_t t = SECOND ? pr.t2 : pr.t1;
            bp[u] = bucket_ptr(sv, t, bucket_of(sv, t, k[u]), B);
#pragma unroll
            for (int q = 0; q < 4; q++) s[u][q] = kEmptySlot;
            probe_cg_pred<B>(bp[u] + 4 * g.sub, s[u], has[u]);
            if (!SECOND) bin[u] = region_of(bs, bc.rshift, pr.t2, bucket_of(sv, pr.t2, k[u]));
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            em[u] = has[u] ? empty_mask(s[u]) : 0u;
            placed[u] = false;
        }
    }
    coop_cas_multi<G, U>(g, bp, em, has, kv, placed);
    const bool lead = g.sub == 0;
    if constexpr (SECOND) {
#pragma unroll
        for (int u = 0; u < U; u++) warp_append(lead && has[u] && !placed[u], kv[u], pending, ctr + C_PENDING);
    } else {
#pragma unroll
        for (int u = 0; u < U; u++)
            if (lead && has[u] && !placed[u]) rank[u] = atomicAdd(&fr.s_next[bin[u]], 1u);
        __syncthreads();
        fr.reserve(io);
        __syncthreads();
#pragma unroll
        for (int u = 0; u < U; u++) {
            if (!(lead && has[u] && !placed[u])) continue;
            const uint32_t q = fr.s_next[bin[u]] + rank[u];
            io.nk[q] = k[u];
            io.nv[q] = v[u];
        }
    }
}

// ---------------------------------------------------------- results in order
// Result group j holds the records of ops [j<<ishift, (j+1)<<ishift) up to
// rcur[j]; blocks run in group order, so the scattered writes of one group land
// in an L2-resident window (2^ishift values + flags) and reach HBM as full lines.
//   find/delete (res_v != null): vals[i] = value, flag[i] = bit 31
//   insert      (res_v == null): flag[i] = bits 30..31 (INSERTED / UPDATED)
__global__ void __launch_bounds__(kThreads) k_bin_out(const uint32_t* __restrict__ res_i,
                                                      const uint32_t* __restrict__ res_v,
                                                      const uint32_t* __restrict__ rcur, uint32_t ishift, uint64_t n,
                                                      uint32_t* __restrict__ vals, uint8_t* __restrict__ flag) {
    const uint64_t b0 = (uint64_t)blockIdx.x * kThreads * kOutItems;
    uint32_t ri[kOutItems], rv[kOutItems];
    bool ok[kOutItems];
#pragma unroll
    for (int j = 0; j < kOutItems; j++) {
        const uint64_t p = b0 + (uint64_t)j * kThreads + threadIdx.x;
        ok[j] = p < n && p < __ldg(rcur + (p >> ishift));
        ri[j] = ok[j] ? __ldcs(res_i + p) : 0u;
        rv[j] = (ok[j] && res_v) ? __ldcs(res_v + p) : 0u;
    }
#pragma unroll
    for (int j = 0; j < kOutItems; j++) {
        if (!ok[j]) continue;
        if (res_v) {
            const uint32_t i = ri[j] & 0x7FFFFFFFu;
            if (vals) vals[i] = rv[j];
            if (flag) flag[i] = (uint8_t)(ri[j] >> 31);
        } else if (flag) {
            flag[ri[j] & 0x3FFFFFFFu] = (uint8_t)(ri[j] >> 30);
        }
    }
}

}  // namespace dyc
