// dyc_binned.cuh — region-binned execution of large batches (L2-blocked probes).
//
// The direct kernels (dyc_kernels.cuh) probe buckets in batch order, so a batch
// much larger than L2 costs one random HBM access per probe: about 50-55 G
// accesses/s on B200, whatever the access size (profiles/r1_memory_model.md).
// A batch of n ops over a table of NB buckets touches every bucket n/NB times
// per probe pass (6.8 at config C2).  Binned execution turns that reuse into L2
// hits: the ops are grouped by the REGION of the bucket they probe next (a
// region is 2^rshift consecutive buckets of one subtable, sized to a fraction of
// the 126 MB L2), and each pass walks the groups in region order, so the blocks
// in flight probe one region at a time.  The pass that follows is fed through
// the same grouping, and the per-op results are grouped by op index (2^ishift
// ops per group, an L2-sized output window) before they are written back in
// request order.
//
// Semantics are those of the direct kernels (the paper's batch model, P:L464;
// keys distinct within a batch, Q9), pass by pass:
//   find   F1 probe h^{t1}  ->  F2 probe h^{t2} for F1 misses (<= 2 lookups)
//   delete the same, the matching slot is overwritten with EMPTY
//   insert I1 probe t1: a match is updated in place (Alg. 1, Q8);
//          otherwise the key is placed in a free slot of t1 right away
//          (first-fit prefers t1, Q3) -- tentatively, because the existence
//          check over BOTH buckets (reading Q7) finishes only in
//          I2 probe t2: a match is updated in place and, if I1 placed the key
//          in t1, that copy is removed by the cleanup pass I3 (so a key is
//          never left twice); a new key not placed by I1 takes a free slot of
//          t2, else it goes to the eviction kernel k_place.
// No key moves during I1-I3 (CAS into EMPTY slots, no eviction), so the
// existence check is exact, as in k_upsert.  Used only when no upsize can be
// needed before placement ((m+n) <= beta*N, the FUSE case of k_upsert) and no
// resize is in flight; everything else takes the direct kernels.
//
// Record streams.  A stream is an array of fixed-size records cut into chunks
// of kChunk records.  Bin b owns chunks [base[b], base[b+1]) sized from its
// EXPECTED count (keys hash uniformly: the t1 and t2 of a key are each uniform
// over the d subtables, and its bucket uniform inside the subtable) plus one
// partial chunk per emitting block; a bin that outgrows its range takes chunks
// from a shared overflow pool sized for the worst case, so any key set is
// correct (only its locality degrades).  fill[c] = (bin << 16) | records in
// chunk c (0 = unused).  The binned kernels are persistent (kBinBPS blocks per
// SM); a block keeps, per bin, the chunk it is filling in shared memory and
// takes a new chunk with ONE global atomic when that one is full.  Per tile of
// ops: rank per bin in shared memory, __syncthreads, reserve, __syncthreads,
// write.  Tiles are handed out by a global counter (next tile prefetched), so
// the blocks in flight stay within one region.  Consumers walk the bins' chunks
// in order (= region order), then the used part of the pool.
//
// One lane per op: each lane reads its whole bucket (B/4 loads of 32 bytes) and
// hashes once per pass; the global bucket of the OTHER candidate travels in the
// record (hashed once in k_bin_scatter).
#pragma once
#include "dyc_kernels.cuh"

namespace dyc {

#ifndef DYC_BIN_BPS
#define DYC_BIN_BPS 4
#endif
#ifndef DYC_BIN_U
#define DYC_BIN_U 1
#endif
constexpr uint32_t kMaxBins = 1024;   // regions per bin set; result groups per batch
constexpr uint32_t kChunk = 128;      // records per chunk
constexpr uint32_t kChunkShift = 7;
constexpr int kBinBPS = DYC_BIN_BPS;  // resident blocks per SM of every binned kernel (register budget)
constexpr uint32_t kNone = 0xFFFFFFFFu;
constexpr int kTileCtrs = 16;         // dynamic tile counters, one per binned launch of a batch
constexpr uint32_t kPoolAlign = 8;    // chunks; a multiple of every consumer tile (kThreads*U/kChunk, U <= 4)

struct BinCtx {
    uint64_t gbase[kMaxD];   // first global bucket of subtable t; a multiple of 2^rshift
    uint32_t rshift;         // region of global bucket g = g >> rshift (never spans two subtables)
    uint32_t R;              // regions
    uint32_t ishift;         // result group of op i = i >> ishift (ishift >= kChunkShift)
    uint32_t Rout;           // result groups
    uint32_t P;              // blocks of every binned launch
};

// A binned, chunked record stream (see the header comment).
template <class Rec>
struct Stream {
    Rec* rec;                // chunk c holds positions [c*kChunk, (c+1)*kChunk)
    uint32_t* fill;          // per chunk: (bin << 16) | records
    uint32_t* ctr;           // [nbins + 1]: next free chunk of each bin; [nbins] = next pool chunk
    const uint32_t* base;    // [nbins + 1]: first chunk of each bin; base[nbins] = first pool chunk
    uint32_t nbins;
    uint32_t pool_end;       // chunks allocated for the stream
};

// Expected-count capacity of a bin in chunks (identical on host and device).
__host__ __device__ __forceinline__ uint32_t bin_cap_chunks(uint64_t expect, uint32_t P, uint32_t passes) {
    const uint64_t c = expect + expect / 32 + 1024;
    return (uint32_t)((c + kChunk - 1) >> kChunkShift) + passes * (P + 1);
}

// Records of region r expected in a batch of n ops: n/d keys choose each subtable
// (as t1, and as t2), spread uniformly over its nb_t buckets.
__host__ __device__ __forceinline__ uint64_t region_expect(uint64_t n, uint32_t d, uint64_t nb_t, uint64_t rbuckets) {
    return (n * rbuckets) / ((uint64_t)d * (nb_t ? nb_t : 1));
}

// Per-block shared state common to the binned kernels.
struct BinSmem {
    uint64_t gbase[kMaxD];
    uint8_t t_of_r[kMaxBins];           // subtable of region r
    uint32_t tile, tile2;               // tiles handed to the block (current / next)
};

__device__ __forceinline__ void load_bins(const TableView& tv, const BinCtx& bc, BinSmem& bs) {
    if (threadIdx.x < tv.d) bs.gbase[threadIdx.x] = bc.gbase[threadIdx.x];
    for (uint32_t r = threadIdx.x; r < bc.R; r += blockDim.x) {
        const uint64_t g = (uint64_t)r << bc.rshift;
        uint32_t t = 0;
        for (uint32_t u = 1; u < tv.d; u++)
            if (bc.gbase[u] <= g) t = u;
        bs.t_of_r[r] = (uint8_t)t;
    }
}

// Block-wide exclusive scan of up to 1024 values (one per thread; blockDim 1024).
__device__ __forceinline__ uint32_t block_excl_scan_1024(uint32_t v, uint32_t* warp_sums) {
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
_Pragma("unroll")
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (unsigned)o) x += y;
    }
    if (lane == 31) warp_sums[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t s = warp_sums[lane];
_Pragma("unroll")
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

// Chunk ranges of a region-binned stream (one block of 1024 threads): bin r of
// subtable t gets bin_cap_chunks(expected) chunks, the pool follows.  Also
// resets the cursors.  `passes` = launches appending to the stream.
__global__ void __launch_bounds__(1024) k_bin_init_regions(TableView tv, BinCtx bc, uint64_t n, uint32_t passes,
                                                           uint32_t* __restrict__ base, uint32_t* __restrict__ ctr) {
    __shared__ uint32_t ws[32];
    const uint32_t r = threadIdx.x;
    uint32_t v = 0;
    if (r < bc.R) {
        const uint64_t g0 = (uint64_t)r << bc.rshift;
        uint32_t t = 0;
        for (uint32_t u = 1; u < tv.d; u++)
            if (bc.gbase[u] <= g0) t = u;
        const uint64_t lo = g0 - bc.gbase[t];
        const uint64_t lim = lo + (1ull << bc.rshift), nbt = tv.sub[t].n;
        const uint64_t hi = nbt < lim ? nbt : lim;
        v = bin_cap_chunks(region_expect(n, tv.d, tv.sub[t].n, hi > lo ? hi - lo : 0), bc.P, passes);
    }
    const uint32_t e = block_excl_scan_1024(v, ws);
    if (r < bc.R) base[r] = ctr[r] = e;
    // the pool starts on a tile boundary (consumer tiles never straddle it)
    if (r == bc.R - 1) base[bc.R] = ctr[bc.R] = (e + v + kPoolAlign - 1) / kPoolAlign * kPoolAlign;
}

// Result groups: group j holds exactly min(2^ishift, n - j*2^ishift) records.
__global__ void k_bin_init_results(BinCtx bc, uint32_t passes, uint32_t* __restrict__ base,
                                   uint32_t* __restrict__ ctr, uint32_t* __restrict__ tiles) {
    const uint32_t per = ((1u << bc.ishift) >> kChunkShift) + passes * (bc.P + 1);
    for (uint32_t j = threadIdx.x; j <= bc.Rout; j += blockDim.x) base[j] = ctr[j] = j * per;
    for (uint32_t j = threadIdx.x; j < (uint32_t)kTileCtrs; j += blockDim.x) tiles[j] = 0;
}

// ------------------------------------------------------------------ emitter
// Block-level appends to a Stream.  Shared memory: 6 words per bin: count of
// this tile, current chunk, its fill, and for this tile: base in the current
// chunk, records that fit there, base in new chunks.
template <class Rec>
struct Emitter {
    uint32_t* s;
    uint32_t nb;
    Stream<Rec> st;
    __device__ __forceinline__ Emitter(uint32_t* smem, uint32_t nbins, const Stream<Rec>& stream)
        : s(smem), nb(nbins), st(stream) {}
    __device__ __forceinline__ void init() const {
        for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) {
            s[b] = 0;
            s[nb + b] = kNone;
            s[2 * nb + b] = 0;
        }
    }
    __device__ __forceinline__ uint32_t rank(uint32_t b) const { return atomicAdd(&s[b], 1u); }
    // k consecutive chunks of bin b (from the pool once the bin's range is used up)
    __device__ __forceinline__ uint32_t alloc(uint32_t b, uint32_t k) const {
        const uint32_t first = atomicAdd(&st.ctr[b], k);
        if (first + k <= st.base[b + 1]) return first;
        return atomicAdd(&st.ctr[st.nbins], k);
    }
    // after a __syncthreads: place this tile's records of every bin
    __device__ __forceinline__ void reserve() const {
        for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) {
            const uint32_t c = s[b];
            if (!c) continue;
            uint32_t cur = s[nb + b], f = s[2 * nb + b];
            const uint32_t room = cur == kNone ? 0u : kChunk - f;
            const uint32_t take = min(room, c);
            s[3 * nb + b] = cur * kChunk + f;
            s[4 * nb + b] = take;
            const uint32_t rest = c - take;
            if (rest) {
                const uint32_t k = (rest + kChunk - 1) >> kChunkShift;
                const uint32_t first = alloc(b, k);
                if (cur != kNone) st.fill[cur] = (b << 16) | kChunk;
                for (uint32_t j = 0; j + 1 < k; j++) st.fill[first + j] = (b << 16) | kChunk;
                s[5 * nb + b] = first * kChunk;
                cur = first + k - 1;
                f = rest - (k - 1) * kChunk;
            } else {
                f += c;
            }
            s[nb + b] = cur;
            s[2 * nb + b] = f;
            s[b] = 0;
        }
    }
    __device__ __forceinline__ void put(uint32_t b, uint32_t r, const Rec& v) const {
        const uint32_t take = s[4 * nb + b];
        const uint32_t pos = r < take ? s[3 * nb + b] + r : s[5 * nb + b] + (r - take);
        st.rec[pos] = v;
    }
    // after the last tile and a __syncthreads
    __device__ __forceinline__ void finish() const {
        for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) {
            const uint32_t cur = s[nb + b];
            if (cur != kNone) st.fill[cur] = (b << 16) | s[2 * nb + b];
        }
    }
};

// ---------------------------------------------------------------- consumers
// Tiles of kTileChunks chunks: first the bins' ranges [0, base[nbins]), then
// the used pool [base[nbins], ctr[nbins]).  Tiles are taken from a global
// counter; thread 0 fetches the next tile while the block works on this one.
template <int U>
struct Walker {
    static constexpr uint32_t kTileRecs = kThreads * U;
    static constexpr uint32_t kTileChunks = kTileRecs / kChunk;
    uint32_t area_tiles, pool_first, pool_tiles;
    uint32_t* counter;
    __device__ __forceinline__ uint32_t total() const { return area_tiles + pool_tiles; }
    // first chunk of tile t
    __device__ __forceinline__ uint32_t chunk0(uint32_t t) const {
        return t < area_tiles ? t * kTileChunks : pool_first + (t - area_tiles) * kTileChunks;
    }
};

template <int U, class Rec>
__device__ __forceinline__ Walker<U> make_walker(const Stream<Rec>& in, uint32_t* counter) {
    static_assert((kThreads * U) % kChunk == 0, "tile must be whole chunks");
    Walker<U> w;
    const uint32_t area = in.base[in.nbins];
    const uint32_t used = *(volatile const uint32_t*)(in.ctr + in.nbins);
    w.area_tiles = (area + Walker<U>::kTileChunks - 1) / Walker<U>::kTileChunks;
    w.pool_first = area;
    w.pool_tiles = (used - area + Walker<U>::kTileChunks - 1) / Walker<U>::kTileChunks;
    w.counter = counter;
    return w;
}

// Position of record u of this lane in the tile starting at chunk c0, and
// whether it holds a record (and its bin).
template <int U>
__device__ __forceinline__ bool tile_rec(const uint32_t* __restrict__ fill, uint32_t c0, uint32_t pool_end, int u,
                                         uint32_t& p, uint32_t& bin) {
    const uint32_t off = (uint32_t)u * kThreads + threadIdx.x;
    const uint32_t c = c0 + (off >> kChunkShift);
    p = (c << kChunkShift) + (off & (kChunk - 1));
    if (c >= pool_end) return false;
    const uint32_t fb = __ldg(fill + c);
    bin = fb >> 16;
    return (off & (kChunk - 1)) < (fb & 0xFFFFu);
}

// One lane reads a whole bucket: B/4 loads of 32 bytes.
template <int B, bool NC>
__device__ __forceinline__ void probe_lane(const unsigned long long* bp, unsigned long long (&s)[B], bool pred) {
_Pragma("unroll")
    for (int q = 0; q < B / 4; q++) {
        if (NC) probe_nc_pred<B>(bp + 4 * q, s + 4 * q, pred);
        else probe_cg_pred<B>(bp + 4 * q, s + 4 * q, pred);
    }
}

template <int B>
__device__ __forceinline__ int lane_match(const unsigned long long (&s)[B], uint32_t k) {
    int hit = -1;
_Pragma("unroll")
    for (int j = B - 1; j >= 0; --j)
        if (key_of(s[j]) == k) hit = j;
    return hit;
}

template <int B>
__device__ __forceinline__ uint32_t lane_value(const unsigned long long (&s)[B], int j) {
    uint32_t v = kEmptyKey;
_Pragma("unroll")
    for (int q = 0; q < B; q++)
        if (q == j) v = val_of(s[q]);
    return v;
}

template <int B>
__device__ __forceinline__ uint32_t lane_free_mask(const unsigned long long (&s)[B]) {
    uint32_t m = 0;
_Pragma("unroll")
    for (int j = 0; j < B; j++)
        if (s[j] == kEmptySlot) m |= 1u << j;
    return m;
}

// First-fit CAS of U records into the EMPTY slots of their snapshots, in slot
// order: every round issues the CAS of each still-unplaced record at once (one
// instruction for the warp, whatever slot each lane targets), so a round costs
// one atomic round trip; a failed CAS (another op of this pass took the slot)
// moves on to the next free slot.
template <int U>
__device__ __forceinline__ void lane_cas_multi(unsigned long long* const (&bp)[U], uint32_t (&free)[U],
                                               const bool (&want)[U], const unsigned long long (&kv)[U],
                                               bool (&placed)[U]) {
    bool todo[U];
_Pragma("unroll")
    for (int u = 0; u < U; u++) {
        placed[u] = false;
        todo[u] = want[u] && free[u] != 0;
    }
    for (;;) {
        bool any = false;
_Pragma("unroll")
        for (int u = 0; u < U; u++) any |= todo[u];
        if (!any) break;
        unsigned long long old[U];
        uint32_t j[U];
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            j[u] = todo[u] ? (uint32_t)(__ffs(free[u]) - 1) : 0u;
            old[u] = cas_slot_pred(bp[u] + j[u], kEmptySlot, kv[u], todo[u], 0ull);
        }
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            if (!todo[u]) continue;
            free[u] &= ~(1u << j[u]);
            if (old[u] == kEmptySlot) { placed[u] = true; todo[u] = false; }
            else todo[u] = free[u] != 0;
        }
    }
}

__device__ __forceinline__ uint32_t gbucket(const BinSmem& bs, const SmemView& sv, uint32_t t, uint32_t k) {
    return (uint32_t)(bs.gbase[t] + bucket_of(sv, t, k));
}

// Loads the U records of this lane in the tile at chunk c0 (kNone: none), with
// whether each position holds a record and its bin.  Issued one tile ahead of
// its use (see DYC_BIN_TILE_LOOP), so the stream latency overlaps the probes
// and appends of the tile before.
template <int U>
__device__ __forceinline__ void load_recs(const Stream<uint4>& in, uint32_t c0, uint4 (&r)[U], bool (&has)[U],
                                          uint32_t (&bin)[U]) {
_Pragma("unroll")
    for (int u = 0; u < U; u++) {
        uint32_t p = 0;
        bin[u] = 0;
        has[u] = c0 != kNone && tile_rec<U>(in.fill, c0, in.pool_end, u, p, bin[u]);
        r[u] = has[u] ? __ldcs(in.rec + p) : make_uint4(kEmptyKey, 0, 0, 0);
    }
}

// Hashes a record's bucket in the subtable of its region and issues the probe.
template <int B, bool NC>
__device__ __forceinline__ void probe_rec(const BinSmem& bs, const SmemView& sv, const uint4& r, bool has,
                                          uint32_t bin, uint32_t& cur, unsigned long long*& bp,
                                          unsigned long long (&s)[B]) {
    const uint32_t t = bs.t_of_r[has ? bin : 0];
    const uint32_t b = has ? bucket_of(sv, t, r.x) : 0u;
    cur = (uint32_t)(bs.gbase[t] + b);
    bp = bucket_ptr(sv, t, b, B);
    probe_lane<B, NC>(bp, s, has);
}

// Tile loop of a persistent consumer of stream IN: the body runs for every tile
// with the tile's records prefetched in pr/ph/pb (record, present, bin); the
// records of the next tile are loaded before the body, and thread 0 fetches the
// index of the tile after that, so neither latency sits on the body's chain.
#define DYC_BIN_TILE_LOOP(U_, IN, WK, BS, ...)                                              \
    {                                                                                       \
        if (threadIdx.x == 0) {                                                             \
            (BS).tile = atomicAdd((WK).counter, 1u);                                        \
            (BS).tile2 = atomicAdd((WK).counter, 1u);                                       \
        }                                                                                   \
        __syncthreads();                                                                    \
        uint32_t tile_ = (BS).tile, next_ = (BS).tile2;                                     \
        uint4 pr[U_];                                                                       \
        bool ph[U_];                                                                        \
        uint32_t pb[U_];                                                                    \
        load_recs<U_>(IN, tile_ < (WK).total() ? (WK).chunk0(tile_) : kNone, pr, ph, pb);   \
        while (tile_ < (WK).total()) {                                                      \
            __syncthreads();                                                                \
            uint32_t nn_ = 0;                                                               \
            if (threadIdx.x == 0) nn_ = atomicAdd((WK).counter, 1u);                        \
            uint4 qr[U_];                                                                   \
            bool qh[U_];                                                                    \
            uint32_t qb[U_];                                                                \
            load_recs<U_>(IN, next_ < (WK).total() ? (WK).chunk0(next_) : kNone, qr, qh, qb); \
            __VA_ARGS__                                                                     \
            _Pragma("unroll") for (int u_ = 0; u_ < U_; u_++) {                             \
                pr[u_] = qr[u_];                                                            \
                ph[u_] = qh[u_];                                                            \
                pb[u_] = qb[u_];                                                            \
            }                                                                               \
            if (threadIdx.x == 0) (BS).tile = nn_;                                          \
            __syncthreads();                                                                \
            tile_ = next_;                                                                  \
            next_ = (BS).tile;                                                              \
        }                                                                                   \
    }

// ------------------------------------------------------- grouping by region
// Records {key, value, op index, global bucket of t2} grouped by the t1 region.
// The reserved key gets its "absent" result here (value EMPTY, flag 0).
__global__ void __launch_bounds__(kThreads, kBinBPS) k_bin_scatter(TableView tv, BinCtx bc,
                                                                   const uint32_t* __restrict__ keys,
                                                                   const uint32_t* __restrict__ vals, uint64_t n,
                                                                   Stream<uint4> out, uint32_t* __restrict__ rv_out,
                                                                   uint8_t* __restrict__ rs_out) {
    constexpr int IT = 4;
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    const Emitter<uint4> em(smem, bc.R, out);
    em.init();
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const uint64_t tile = (uint64_t)kThreads * IT;
    for (uint64_t t0 = (uint64_t)blockIdx.x * tile; t0 < n; t0 += (uint64_t)gridDim.x * tile) {
        uint4 r[IT];
        uint32_t bin[IT], rk[IT];
_Pragma("unroll")
        for (int j = 0; j < IT; j++) {
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            r[j].x = i < n ? __ldcs(keys + i) : kEmptyKey;
            r[j].y = (i < n && vals) ? __ldcs(vals + i) : 0u;
            r[j].z = (uint32_t)i;
            r[j].w = 0;
        }
_Pragma("unroll")
        for (int j = 0; j < IT; j++) {
            const uint64_t i = t0 + (uint64_t)j * kThreads + threadIdx.x;
            bin[j] = kNone;
            rk[j] = 0;
            if (r[j].x != kEmptyKey) {
                const Pair p = pair_of(tv, r[j].x);
                bin[j] = gbucket(bs, sv, p.t1, r[j].x) >> bc.rshift;
                r[j].w = gbucket(bs, sv, p.t2, r[j].x);
                rk[j] = em.rank(bin[j]);
            } else if (i < n) {
                if (rv_out) rv_out[i] = kEmptyKey;
                if (rs_out) rs_out[i] = 0;
            }
        }
        __syncthreads();
        em.reserve();
        __syncthreads();
_Pragma("unroll")
        for (int j = 0; j < IT; j++)
            if (bin[j] != kNone) em.put(bin[j], rk[j], r[j]);
    }
    __syncthreads();
    em.finish();
}

// ------------------------------------------------------------ probe passes
// F1/F2 (find) and D1/D2 (delete): probe the bucket of the record's region
// (SECOND = false: h^{t1}, else h^{t2}).  A hit gives a result record {index |
// 1<<31, value}; DEL also overwrites the slot with EMPTY.  A miss
// in pass 1 becomes a record of the t2 region bins; a miss in pass 2 is a
// result record {index, EMPTY}.
template <int B, int U, bool DEL, bool SECOND>
__global__ void __launch_bounds__(kThreads, kBinBPS) k_bin_fd(TableView tv, BinCtx bc, Stream<uint4> in,
                                                              Stream<uint4> next, Stream<uint2> res,
                                                              uint32_t* __restrict__ tiles,
                                                              unsigned long long* __restrict__ ctr) {
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    const uint32_t nbn = SECOND ? 0u : bc.R;
    const Emitter<uint4> en(smem, nbn, next);
    const Emitter<uint2> er(smem + 6 * nbn, bc.Rout, res);
    en.init();
    er.init();
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const Walker<U> wk = make_walker<U>(in, tiles);
    unsigned long long removed = 0;
    DYC_BIN_TILE_LOOP(U, in, wk, bs, {
        uint4 r[U];
        bool has[U], hit[U];
        uint32_t v[U], ob[U], rk[U], cur[U];
        {
            unsigned long long s[U][B];
            unsigned long long* bp[U];
_Pragma("unroll")
            for (int u = 0; u < U; u++) {
                r[u] = pr[u];
                has[u] = ph[u];
                probe_rec<B, !DEL>(bs, sv, r[u], has[u], pb[u], cur[u], bp[u], s[u]);
            }
_Pragma("unroll")
            for (int u = 0; u < U; u++) {
                const int j = has[u] ? lane_match<B>(s[u], r[u].x) : -1;
                hit[u] = j >= 0;
                v[u] = lane_value<B>(s[u], j);
                if (DEL && hit[u]) st_u64_cg(bp[u] + j, kEmptySlot);
                removed += DEL && hit[u];
            }
        }
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            ob[u] = 0;
            rk[u] = 0;
            if (!has[u]) continue;
            if (!SECOND && !hit[u]) {
                ob[u] = r[u].w >> bc.rshift;
                rk[u] = en.rank(ob[u]);
            } else {
                ob[u] = r[u].z >> bc.ishift;
                rk[u] = er.rank(ob[u]);
            }
        }
        __syncthreads();
        en.reserve();
        er.reserve();
        __syncthreads();
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            if (!has[u]) continue;
            if (!SECOND && !hit[u]) en.put(ob[u], rk[u], make_uint4(r[u].x, 0u, r[u].z, cur[u]));
            else er.put(ob[u], rk[u], make_uint2(r[u].z | (hit[u] ? 0x80000000u : 0u), v[u]));
        }
    })
    __syncthreads();
    en.finish();
    er.finish();
    if (DEL) block_add<kThreads>(ctr + C_REMOVED, removed);
}

// I1 (SECOND = false, t1) / I2 (t2) of an insert.  Records: {key, value,
// index | flag, global bucket of the other candidate}; flag (bit 31, I1 -> I2):
// "placed in t1 by I1".  Results: {index | status << 30}.
//   I1: match -> value replaced (UPDATED); else CAS into a free slot of t1
//       (tentative), and on to I2 either way.
//   I2: match -> value replaced (UPDATED); if I1 placed the key in t1 too, a
//       cleanup record {key} goes to the t1 bins.  No match -> INSERTED; if I1
//       did not place it, CAS into a free slot of t2, else pending (k_place).
template <int B, int U, bool SECOND>
__global__ void __launch_bounds__(kThreads, kBinBPS) k_bin_ins(TableView tv, BinCtx bc, Stream<uint4> in,
                                                               Stream<uint4> next, Stream<uint32_t> res,
                                                               unsigned long long* __restrict__ pending,
                                                               uint32_t* __restrict__ tiles,
                                                               unsigned long long* __restrict__ ctr) {
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    extern __shared__ uint32_t smem[];
    const Emitter<uint4> en(smem, bc.R, next);
    const Emitter<uint32_t> er(smem + 6 * bc.R, res.rec ? bc.Rout : 0u, res);
    en.init();
    er.init();
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const Walker<U> wk = make_walker<U>(in, tiles);
    unsigned long long n_ins = 0, n_upd = 0, n_clean = 0;
    DYC_BIN_TILE_LOOP(U, in, wk, bs, {
        uint4 r[U];
        bool has[U], hit[U], fwd[U];
        uint32_t nb_[U], nrk[U], rb[U], rrk[U], cur[U];
        {
            unsigned long long s[U][B];
            unsigned long long* bp[U];
_Pragma("unroll")
            for (int u = 0; u < U; u++) {
                r[u] = pr[u];
                has[u] = ph[u];
                probe_rec<B, false>(bs, sv, r[u], has[u], pb[u], cur[u], bp[u], s[u]);
            }
            unsigned long long kv[U];
            uint32_t fm[U];
            bool want[U], placed[U];
_Pragma("unroll")
            for (int u = 0; u < U; u++) {
                const int j = has[u] ? lane_match<B>(s[u], r[u].x) : -1;
                hit[u] = j >= 0;
                kv[u] = make_kv(r[u].x, r[u].y);
                if (hit[u]) st_u64_cg(bp[u] + j, kv[u]);
                fm[u] = lane_free_mask<B>(s[u]);
                const bool placed1 = SECOND && (r[u].z & 0x80000000u) != 0;
                // I1: tentative t1 placement of every miss; I2: t2 placement of a
                // new key that I1 could not place
                want[u] = has[u] && !hit[u] && !placed1;
            }
            lane_cas_multi<U>(bp, fm, want, kv, placed);
_Pragma("unroll")
            for (int u = 0; u < U; u++) {
                if (!SECOND) {
                    fwd[u] = has[u] && !hit[u];
                    if (placed[u]) r[u].z |= 0x80000000u;
                } else {
                    const bool placed1 = (r[u].z & 0x80000000u) != 0;
                    r[u].z &= 0x7FFFFFFFu;
                    fwd[u] = has[u] && hit[u] && placed1;          // remove the t1 copy
                    if (want[u] && !placed[u]) {
                        const unsigned long long c = atomicAdd(ctr + C_PENDING, 1ull);
                        pending[c] = kv[u];
                    }
                }
            }
        }
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            nb_[u] = nrk[u] = rb[u] = rrk[u] = 0;
            if (!has[u]) continue;
            if (fwd[u]) {
                nb_[u] = r[u].w >> bc.rshift;
                nrk[u] = en.rank(nb_[u]);
            }
            if ((hit[u] || SECOND) && res.rec) {
                rb[u] = (r[u].z & 0x3FFFFFFFu) >> bc.ishift;
                rrk[u] = er.rank(rb[u]);
            }
            n_upd += hit[u];
            n_ins += SECOND && !hit[u];
            n_clean += SECOND && fwd[u];
        }
        __syncthreads();
        en.reserve();
        er.reserve();
        __syncthreads();
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            if (!has[u]) continue;
            if (fwd[u]) en.put(nb_[u], nrk[u], make_uint4(r[u].x, r[u].y, r[u].z, cur[u]));
            if ((hit[u] || SECOND) && res.rec)
                er.put(rb[u], rrk[u], (r[u].z & 0x3FFFFFFFu) | ((hit[u] ? 2u : 1u) << 30));
        }
    })
    __syncthreads();
    en.finish();
    er.finish();
    block_add<kThreads>(ctr + C_INSERTED, n_ins);
    block_add<kThreads>(ctr + C_UPDATED, n_upd);
    if (SECOND) block_add<kThreads>(ctr + C_CLEANUP, n_clean);
}

// I3: removes the copies I1 placed in t1 of keys that I2 found (and updated) in
// t2.  Does nothing unless the C_CLEANUP counter is non-zero.
template <int B, int U>
__global__ void __launch_bounds__(kThreads, kBinBPS) k_bin_cleanup(TableView tv, BinCtx bc, Stream<uint4> in,
                                                                   uint32_t* __restrict__ tiles,
                                                                   const unsigned long long* __restrict__ ctr) {
    if (*(volatile const unsigned long long*)(ctr + C_CLEANUP) == 0) return;
    __shared__ SmemView sv;
    __shared__ BinSmem bs;
    load_bins(tv, bc, bs);
    load_view(tv, sv);
    const Walker<U> wk = make_walker<U>(in, tiles);
    DYC_BIN_TILE_LOOP(U, in, wk, bs, {
        unsigned long long s[U][B];
        unsigned long long* bp[U];
        uint4 r[U];
        bool has[U];
        uint32_t cur[U];
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            r[u] = pr[u];
            has[u] = ph[u];
            probe_rec<B, false>(bs, sv, r[u], has[u], pb[u], cur[u], bp[u], s[u]);
        }
_Pragma("unroll")
        for (int u = 0; u < U; u++) {
            const int j = has[u] ? lane_match<B>(s[u], r[u].x) : -1;
            if (j >= 0) st_u64_cg(bp[u] + j, kEmptySlot);
        }
    })
}

// ---------------------------------------------------------- results in order
// Result group j holds the records of ops [j<<ishift, (j+1)<<ishift); blocks
// walk the chunks in group order, so the scattered writes of one group land in
// an L2-resident window (2^ishift values + flags) and reach HBM as full lines.
//   find/delete (uint2 {index | found<<31, value}): vals[i] = value, flag[i] = found
//   insert      (uint32 {index | status<<30}):      flag[i] = status
template <class Rec>
__global__ void __launch_bounds__(kThreads) k_bin_out(Stream<Rec> res, uint32_t* __restrict__ vals,
                                                      uint8_t* __restrict__ flag) {
    constexpr int IT = 8;
    const uint64_t b0 = (uint64_t)blockIdx.x * kThreads * IT;
    const uint64_t end = (uint64_t)res.base[res.nbins] * kChunk;
    Rec rr[IT];
    bool ok[IT];
_Pragma("unroll")
    for (int j = 0; j < IT; j++) {
        const uint64_t p = b0 + (uint64_t)j * kThreads + threadIdx.x;
        ok[j] = false;
        if (p < end) {
            const uint32_t fb = __ldg(res.fill + (p >> kChunkShift));
            ok[j] = (p & (kChunk - 1)) < (fb & 0xFFFFu);
        }
        if (ok[j]) rr[j] = __ldcs(res.rec + p);
    }
_Pragma("unroll")
    for (int j = 0; j < IT; j++) {
        if (!ok[j]) continue;
        if constexpr (sizeof(Rec) == 8) {
            const uint2 x = *reinterpret_cast<const uint2*>(&rr[j]);
            const uint32_t i = x.x & 0x7FFFFFFFu;
            if (vals) vals[i] = x.y;
            if (flag) flag[i] = (uint8_t)(x.x >> 31);
        } else {
            const uint32_t x = *reinterpret_cast<const uint32_t*>(&rr[j]);
            if (flag) flag[x & 0x3FFFFFFFu] = (uint8_t)(x >> 30);
        }
    }
}

}  // namespace dyc
