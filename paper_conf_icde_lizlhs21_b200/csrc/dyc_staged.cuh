// dyc_staged.cuh — chunk-staged execution of large batches (B = 8).
//
// The probe kernels of dyc_kernels.cuh touch one random bucket per probe; on
// B200 a random HBM request costs the same ~19 ps whether it carries 32 or 128
// bytes, so they run at the random-access wall.  When a batch is
// large next to the table (C2: 6.8 ops per bucket), most buckets are visited
// several times, and the batch can instead be ORDERED by the table chunk its
// first-choice bucket lies in (a chunk = 1024 consecutive buckets of one
// subtable, 64 KB), after which every chunk is read from HBM once, as one
// contiguous TMA bulk copy into shared memory, its ops are applied there with
// shared-memory atomics, and it is written back once (insert / delete).  The
// random traffic becomes streaming traffic; what remains random is the second
// probe of the ops whose first-choice bucket cannot decide them, which run
// through the ordinary kernels afterwards on a compacted list.
//
// Semantics are those of the direct kernels (P:L188-189 map semantics, the
// batch model of P:L464 with distinct keys, Q9): each op's result depends only
// on the table before the batch and on its own key, never on the order of the
// ops inside the batch, so reordering changes where keys land (first-fit slot
// choice), not any result.  The first-choice-full invariant (FFI)
// decides a miss in a non-full first-choice bucket of a clean subtable exactly
// as in k_find / k_upsert; a delete takes the fullness of the bucket as it was
// when its chunk was loaded (deletes of the same batch empty slots).
//
// Passes (one CUDA stream, no host wait; DESIGN.md §5 "Staged batches"):
//   k_st_hist       one hash per op: its global first-choice bucket gb (kept),
//                   and a per-chunk histogram (shared-memory counters)
//   k_st_scan       chunk offsets; level-1 bins (2^s1 chunks each) and the
//                   level-2 tile tables
//   k_st_scatter<1> tile-local counting sort by bin in shared memory, coalesced
//                   runs out; per op its index in the tile's sorted order, per
//                   sorted position the global destination (dmap)
//   k_st_scatter<2> the same inside each bin, by chunk
//   k_st_apply      one CTA per chunk: TMA bulk load, ops in shared memory,
//                   TMA bulk store; undecided ops -> need list (per-warp
//                   shared-memory buffers, one global atomic per 64 entries;
//                   each entry: key, value, chunk-order position)
//   (need list)     k_upsert / k_find / k_delete with the first probe skipped
//                   (S1), results written at the entries' positions
//   k_st_unperm     results back to request order, tile by tile: the tile's
//                   sorted results are gathered through dmap into shared memory,
//                   then every op takes its own (level 2, then level 1)
#pragma once
#include "dyc_kernels.cuh"

namespace dyc {

#ifndef DYC_ST_LOG
#define DYC_ST_LOG 10
#endif
#ifndef DYC_ST_AT
#define DYC_ST_AT 256
#endif
constexpr int kStLog = DYC_ST_LOG;                // buckets per chunk = 1024
constexpr int kStAT = DYC_ST_AT;                  // threads of the apply kernel
constexpr uint32_t kStChunk = 1u << kStLog;
constexpr uint32_t kStSlots = kStChunk * 8;       // B = 8: 64 KB of shared memory
constexpr int kStBins1 = 256;                     // level-1 bins (at most)
#ifndef DYC_ST_TILE
#define DYC_ST_TILE 4096
#endif
#ifndef DYC_ST_T
#define DYC_ST_T 512
#endif
#ifndef DYC_ST_SCATTER_MINB
#define DYC_ST_SCATTER_MINB 3
#endif
#ifndef DYC_ST_APPLY_U
#define DYC_ST_APPLY_U 8
#endif
constexpr int kStTile = DYC_ST_TILE;              // ops per partition tile (<= 65536: 16-bit sorted index)
constexpr int kStT = DYC_ST_T;                    // threads of the scatter / unperm kernels
constexpr int kStPer = kStTile / kStT;            // ops per thread (8)
#ifndef DYC_ST_UT
#define DYC_ST_UT 1024
#endif
constexpr int kStUT = DYC_ST_UT;                  // threads of the unperm kernel
constexpr int kStUPer = kStTile / kStUT;          // positions per thread (unperm)
constexpr int kStMaxS1 = 8;                       // 2^s1 chunks per level-1 bin, <= 256
constexpr uint32_t kStMaxChunks = kStLog >= 10 ? 32768 : 49152;   // k_st_hist: one shared counter per chunk
constexpr int kStHistT = 1024;
#ifndef DYC_ST_HIST_PER
#define DYC_ST_HIST_PER 8
#endif
constexpr int kStHistPer = DYC_ST_HIST_PER;
#ifndef DYC_ST_WUNROLL
#define DYC_ST_WUNROLL 8
#endif
constexpr int kStWU = DYC_ST_WUNROLL;             // unroll of the scatter write-out loop
constexpr int kStApplyU = DYC_ST_APPLY_U;         // ops per lane in flight (apply)
constexpr int kStNeedBuf = 64;                    // per-warp need-list buffer (apply)
constexpr int kStRun = 256;                       // bins (level 1) or chunks of a bin (level 2), at most

struct StagedView {
    uint32_t cbase[kMaxD + 1];   // first chunk of subtable t (prefix of ceil(n_t / kStChunk))
    uint32_t nc;                 // chunks in all
    uint32_t s1;                 // level-1 bin of chunk c = c >> s1
    uint32_t nbins;              // ceil(nc / 2^s1) <= kStBins1
};

// ------------------------------------------------------------ TMA bulk copies
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void st_mbar_init(unsigned long long* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_addr(bar)) : "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// one elected thread: arm the barrier with the byte count and start the copy
__device__ __forceinline__ void st_bulk_load(void* dst, const void* src, uint32_t bytes, unsigned long long* bar) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_addr(bar)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_addr(dst)), "l"(src), "r"(bytes), "r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void st_mbar_wait(unsigned long long* bar, uint32_t parity) {
    uint32_t done = 0;
    for (uint32_t spin = 0;; spin++) {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(smem_addr(bar)), "r"(parity) : "memory");
        if (done) break;
        if (spin > (1u << 26)) __trap();   // a copy that never lands: fail loudly, never hang
    }
}
// one elected thread, after every writer's fence.proxy.async and a barrier
__device__ __forceinline__ void st_bulk_store(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" :: "l"(dst), "r"(smem_addr(src)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// Exclusive block scan of one value per thread (NT threads); *total = the sum.
template <int NT>
__device__ __forceinline__ uint32_t st_block_scan(uint32_t v, uint32_t* warp_sums, uint32_t* total) {
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= (unsigned)o) x += y;
    }
    if (lane == 31) warp_sums[w] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (int i = 0; i < NT / 32; i++) { const uint32_t s = warp_sums[i]; warp_sums[i] = acc; acc += s; }
        *total = acc;
    }
    __syncthreads();
    return x - v + warp_sums[w];
}

// --------------------------------------------------------------- histogram
// Persistent (one CTA per SM): gout[i] = global first-choice bucket of op i,
// gb = cbase[t1] * kStChunk + bucket_t1(k), chunk = gb >> kStLog;
// per-chunk counts in shared memory, one global atomic per chunk per CTA.
__global__ void __launch_bounds__(kStHistT) k_st_hist(TableView tv, StagedView s, const uint32_t* __restrict__ keys,
                                                      uint64_t n, uint32_t* __restrict__ gout,
                                                      uint32_t* __restrict__ chunk_cnt) {
    extern __shared__ uint32_t h[];
    __shared__ SmemView sv;
    __shared__ uint32_t cb[kMaxD + 1];
    for (uint32_t i = threadIdx.x; i < s.nc; i += kStHistT) h[i] = 0;
    if (threadIdx.x <= tv.d) cb[threadIdx.x] = s.cbase[threadIdx.x];
    load_view(tv, sv);
    constexpr uint64_t step = (uint64_t)kStHistT * kStHistPer;
    const uint64_t per = ((n + gridDim.x - 1) / gridDim.x + step - 1) / step * step;
    const uint64_t a = (uint64_t)blockIdx.x * per, z = min(n, a + per);
    for (uint64_t base = a; base < z; base += step) {
        uint32_t kk[kStHistPer];
#pragma unroll
        for (int j = 0; j < kStHistPer; j++) {
            const uint64_t i = base + (uint64_t)j * kStHistT + threadIdx.x;
            kk[j] = i < z ? __ldg(keys + i) : 0u;
        }
#pragma unroll
        for (int j = 0; j < kStHistPer; j++) {
            const uint64_t i = base + (uint64_t)j * kStHistT + threadIdx.x;
            if (i < z) {
                const Pair p = pair_of(tv, kk[j]);
                const uint32_t gb = cb[p.t1] * kStChunk + bucket_of(sv, p.t1, kk[j]);
                gout[i] = gb;
                atomicAdd(&h[gb >> kStLog], 1u);
            }
        }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < s.nc; i += kStHistT)
        if (h[i]) atomicAdd(chunk_cnt + i, h[i]);
}

// Chunk offsets (exclusive scan, one block), their cursors, the level-1 bins
// (offsets, cursors) and the level-2 tiling: bin b owns tiles
// [tile_first[b], tile_first[b+1]) of kStTile ops.
__global__ void __launch_bounds__(1024) k_st_scan(StagedView s, const uint32_t* __restrict__ chunk_cnt,
                                                  uint32_t* __restrict__ chunk_off, uint32_t* __restrict__ cur2,
                                                  uint32_t* __restrict__ bin_off, uint32_t* __restrict__ cur1,
                                                  uint32_t* __restrict__ tile_first, uint32_t* __restrict__ tile_bin,
                                                  uint32_t* __restrict__ tile_lo, uint32_t* __restrict__ tile_hi) {
    __shared__ uint32_t part[1024];
    const uint32_t per = (s.nc + 1023) / 1024;
    const uint32_t a = min(s.nc, threadIdx.x * per), z = min(s.nc, a + per);
    uint32_t sum = 0;
    for (uint32_t i = a; i < z; i++) sum += chunk_cnt[i];
    part[threadIdx.x] = sum;
    __syncthreads();
    for (int o = 1; o < 1024; o <<= 1) {          // Hillis-Steele inclusive scan
        const uint32_t y = threadIdx.x >= (unsigned)o ? part[threadIdx.x - o] : 0u;
        __syncthreads();
        part[threadIdx.x] += y;
        __syncthreads();
    }
    uint32_t acc = part[threadIdx.x] - sum;
    for (uint32_t i = a; i < z; i++) {
        chunk_off[i] = acc;
        cur2[i] = acc;
        acc += chunk_cnt[i];
    }
    if (threadIdx.x == 1023) chunk_off[s.nc] = part[1023];
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tf = 0;
        for (uint32_t b = 0; b < s.nbins; b++) {
            const uint32_t lo = chunk_off[b << s.s1], hi = chunk_off[min(s.nc, (b + 1) << s.s1)];
            bin_off[b] = lo;
            cur1[b] = lo;
            tile_first[b] = tf;
            tf += (hi - lo + kStTile - 1) / kStTile;
        }
        bin_off[s.nbins] = chunk_off[s.nc];
        tile_first[s.nbins] = tf;
    }
    __syncthreads();
    // the level-2 tiling written out once: tile T of bin b covers
    // [bin_off[b] + j*kStTile, min(bin_off[b+1], ... + kStTile)), j = T - tile_first[b]
    for (uint32_t b = threadIdx.x; b < s.nbins; b += 1024) {
        const uint32_t lo = bin_off[b], hi = bin_off[b + 1];
        for (uint32_t T = tile_first[b], j = 0; T < tile_first[b + 1]; T++, j++) {
            tile_bin[T] = b;
            tile_lo[T] = lo + j * kStTile;
            tile_hi[T] = min(hi, lo + (j + 1) * kStTile);
        }
    }
}

// Tile T of the level-1 order (level-2 tiling): its bin and op range (k_st_scan's tables).
__device__ __forceinline__ bool st_tile2(const StagedView& s, const uint32_t* tile_first, const uint32_t* tile_bin,
                                         const uint32_t* tile_lo, const uint32_t* tile_hi, uint32_t T, uint32_t& b,
                                         uint32_t& lo, uint32_t& hi) {
    if (T >= tile_first[s.nbins]) return false;
    b = tile_bin[T];
    lo = tile_lo[T];
    hi = tile_hi[T];
    return true;
}

// ------------------------------------------------------------------ scatter
// One tile of kStTile ops: counting sort by bin in shared memory (ranks from
// shared atomics), one global cursor reservation per (tile, bin), coalesced runs
// out.  LEVEL 1: bins = level-1 bins over the request order; LEVEL 2: the
// chunks of one level-1 bin over that bin's ops.  spos[op] = the op's index in
// the tile's sorted order; dmap[tile start + p] = the global position the
// tile's p-th sorted op went to (what k_st_unperm reads the results back from).
// Level 2 writes the chunk-local bucket (gb & 1023) as 16 bits instead of gb.
template <int LEVEL, bool VALS>
__global__ void __launch_bounds__(kStT, DYC_ST_SCATTER_MINB) k_st_scatter(StagedView s, const uint32_t* __restrict__ kin,
                                                     const uint32_t* __restrict__ vin, const uint32_t* __restrict__ gin,
                                                     uint64_t n, const uint32_t* __restrict__ tile_first,
                                                     const uint32_t* __restrict__ tile_bin,
                                                     const uint32_t* __restrict__ tile_lo,
                                                     const uint32_t* __restrict__ tile_hi, uint32_t* __restrict__ cur,
                                                     uint32_t* __restrict__ kout, uint32_t* __restrict__ vout,
                                                     uint32_t* __restrict__ gout, uint16_t* __restrict__ lbout,
                                                     uint16_t* __restrict__ spos, uint32_t* __restrict__ dmap) {
    extern __shared__ __align__(16) uint32_t sm[];
    uint32_t* sk = sm;                              // [kStTile]
    uint32_t* sg = sm + kStTile;                    // [kStTile]
    uint32_t* svl = sm + 2 * kStTile;               // [kStTile] (VALS)
    uint8_t* sbin = (uint8_t*)(sm + (VALS ? 3 : 2) * kStTile);   // [kStTile]
    __shared__ uint32_t cnt[kStRun], off[kStRun], gbase[kStRun], wsum[kStT / 32], tot;
    __shared__ uint32_t sb, slo, shi, sok;
    uint32_t nb, t0, tn, c0 = 0;
    if (LEVEL == 1) {
        nb = s.nbins;
        t0 = blockIdx.x * kStTile;
        tn = (uint32_t)(n - t0 < (uint64_t)kStTile ? n - t0 : (uint64_t)kStTile);
    } else {
        if (threadIdx.x == 0) {
            uint32_t b = 0, lo = 0, hi = 0;
            sok = st_tile2(s, tile_first, tile_bin, tile_lo, tile_hi, blockIdx.x, b, lo, hi);
            sb = b; slo = lo; shi = hi;
        }
        __syncthreads();
        if (!sok) return;
        nb = 1u << s.s1;
        t0 = slo;
        tn = shi - slo;
        c0 = sb << s.s1;
    }
    if (threadIdx.x < kStRun) cnt[threadIdx.x] = 0;
    __syncthreads();
    // (the bin is recomputed from gg where needed: fewer live registers, three CTAs per SM)
    uint32_t kk[kStPer], vv[kStPer], gg[kStPer], rk[kStPer];
    auto bin_of = [&](uint32_t g) { return LEVEL == 1 ? g >> (kStLog + s.s1) : (g >> kStLog) - c0; };
#pragma unroll
    for (int j = 0; j < kStPer; j++) {
        const uint32_t li = j * kStT + threadIdx.x;
        const bool ok = li < tn;
        kk[j] = ok ? __ldg(kin + t0 + li) : 0u;
        vv[j] = (VALS && ok) ? __ldg(vin + t0 + li) : 0u;
        gg[j] = ok ? __ldg(gin + t0 + li) : 0u;
    }
#pragma unroll
    for (int j = 0; j < kStPer; j++) {
        const uint32_t li = j * kStT + threadIdx.x;
        rk[j] = li < tn ? atomicAdd(&cnt[bin_of(gg[j])], 1u) : 0u;
    }
    __syncthreads();
    const uint32_t c = threadIdx.x < nb ? cnt[threadIdx.x] : 0u;
    const uint32_t ex = st_block_scan<kStT>(c, wsum, &tot);
    if (threadIdx.x < nb) {
        const uint32_t g = c ? atomicAdd(cur + c0 + threadIdx.x, c) : 0u;
        off[threadIdx.x] = ex;
        gbase[threadIdx.x] = g;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kStPer; j++) {
        const uint32_t li = j * kStT + threadIdx.x;
        if (li < tn) {
            const uint32_t b = bin_of(gg[j]);
            const uint32_t p = off[b] + rk[j];
            sk[p] = kk[j];
            sg[p] = gg[j];
            if (VALS) svl[p] = vv[j];
            sbin[p] = (uint8_t)b;
            spos[t0 + li] = (uint16_t)p;
        }
    }
    __syncthreads();
#pragma unroll kStWU
    for (uint32_t p = threadIdx.x; p < tn; p += kStT) {
        const uint32_t b = sbin[p];
        const uint32_t d = gbase[b] + (p - off[b]);
        dmap[t0 + p] = d;
        kout[d] = sk[p];
        if (VALS) vout[d] = svl[p];
        if (LEVEL == 1) gout[d] = sg[p];
        else lbout[d] = (uint16_t)(sg[p] & (kStChunk - 1));
    }
}

// ------------------------------------------------------------------- apply
// One CTA per chunk with at least one op.  OP: 0 insert (upsert, FUSE: first-fit
// into the first-choice bucket), 1 find, 2 delete.  Per op, in shared memory:
//   hit in the first-choice bucket -> decided here (update / value / erase);
//   miss, subtable clean (FFI), bucket non-full (delete: non-full when loaded)
//       -> decided here (insert: CAS into a free slot; when the bucket has
//          filled up meanwhile, the key is absent and its first choice full:
//          the need list places it);
//   otherwise -> need list (index p into the chunk order), run afterwards
//       through the direct kernel with the first probe skipped (S1).
// Insert statuses: 1 INSERTED, 2 UPDATED; delete: 1 DELETED; find: found flag.
template <int OP>
__global__ void __launch_bounds__(kStAT) k_st_apply(TableView tv, StagedView s, const uint32_t* __restrict__ k2,
                                                       const uint32_t* __restrict__ v2, const uint16_t* __restrict__ lb2,
                                                       const uint32_t* __restrict__ chunk_off,
                                                       uint8_t* __restrict__ st2, uint32_t* __restrict__ r2,
                                                       uint32_t* __restrict__ need, uint32_t* __restrict__ need_k,
                                                       uint32_t* __restrict__ need_v,
                                                       unsigned long long* __restrict__ need_cnt,
                                                       unsigned long long* __restrict__ ctr) {
    extern __shared__ __align__(128) unsigned long long tab[];
    __shared__ __align__(8) unsigned long long bar;
    __shared__ uint32_t fullw[kStChunk / 32];
    __shared__ uint32_t nbuf[kStAT / 32][kStNeedBuf];     // need list: chunk-order position,
    __shared__ uint32_t nbufk[kStAT / 32][kStNeedBuf];    // key and (insert) value of each entry
    __shared__ uint32_t nbufv[OP == 0 ? kStAT / 32 : 1][OP == 0 ? kStNeedBuf : 1];
    __shared__ int changed;
    const uint32_t c = blockIdx.x;
    const uint32_t o0 = chunk_off[c], o1 = chunk_off[c + 1];
    if (o0 == o1) return;
    uint32_t t = 0;
    for (uint32_t i = 1; i < tv.d; i++) t = s.cbase[i] <= c ? i : t;
    const uint32_t b0 = (c - s.cbase[t]) << kStLog;
    const SubView sub = tv.sub[t];
    const uint32_t nbk = min(kStChunk, sub.n - b0);
    unsigned long long* gsrc = sub.slots + (uint64_t)b0 * 8;
    const uint32_t bytes = nbk * 64u;
    if (threadIdx.x == 0) {
        st_mbar_init(&bar);
        st_bulk_load(tab, gsrc, bytes, &bar);
        changed = 0;
    }
    if (OP == 2)
        for (uint32_t i = threadIdx.x; i < kStChunk / 32; i += kStAT) fullw[i] = 0;
    __syncthreads();                      // barrier initialized, fullw zeroed
    st_mbar_wait(&bar, 0);
    if (OP == 2) {                        // fullness of every bucket before any erase
        for (uint32_t q = threadIdx.x; q < nbk; q += kStAT) {
            bool full = true;
#pragma unroll
            for (int j = 0; j < 8; j++) full &= tab[q * 8 + ((j + (q >> 1)) & 7u)] != kEmptySlot;   // bank rotation
            if (full) atomicOr(&fullw[q >> 5], 1u << (q & 31));
        }
        __syncthreads();
    }
    const bool clean = (tv.clean >> t) & 1u;
    unsigned long long n_a = 0, n_b = 0;
    bool mod = false;
    const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t ncount = 0;                  // entries in this warp's need buffer (warp-uniform)
    auto flush = [&]() {
        __syncwarp();
        if (ncount) {
            unsigned long long gb = 0;
            if (lane == 0) gb = atomicAdd(need_cnt, (unsigned long long)ncount);
            gb = __shfl_sync(kFull, gb, 0);
            for (uint32_t i = lane; i < ncount; i += 32) {
                need[gb + i] = nbuf[w][i];
                need_k[gb + i] = nbufk[w][i];
                if (OP == 0) need_v[gb + i] = nbufv[w][i];
            }
            ncount = 0;
        }
        __syncwarp();
    };
    constexpr int U = kStApplyU;
    for (uint32_t base = o0 + w * 32 * U; base < o1; base += kStAT * U) {
        uint32_t kk[U], vv[U], ll[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t p = base + u * 32 + lane;
            const bool valid = p < o1;
            kk[u] = valid ? __ldg(k2 + p) : kEmptyKey;
            vv[u] = (OP == 0 && valid) ? __ldg(v2 + p) : 0u;
            ll[u] = valid ? (uint32_t)__ldg(lb2 + p) : 0u;
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t p = base + u * 32 + lane;
            const bool valid = p < o1;
            const uint32_t k = kk[u];
            const bool act = valid && k != kEmptyKey;
            const uint32_t lb = act ? ll[u] : 0u;
            volatile unsigned long long* bk = tab + lb * 8;
            int hit = -1;
            uint32_t hv = 0;
            unsigned emask = 0;
            // The bucket is read as four 16-byte quads.  A 64-byte bucket starts
            // at quad group 0 or 4 of the 8 in a 128-byte bank row, so lanes
            // reading quad q of random buckets would meet in 2 groups; each lane
            // starts at its own rotation instead (all 8 groups in use).
            const uint32_t rot = (lb >> 1) & 3u;
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const uint32_t qq = (q + rot) & 3u;
                unsigned long long e[2];
                asm volatile("ld.shared.v2.u64 {%0,%1}, [%2];" : "=l"(e[0]), "=l"(e[1])
                             : "r"(smem_addr(tab + lb * 8 + qq * 2)) : "memory");
#pragma unroll
                for (int h = 0; h < 2; h++) {
                    const uint32_t jj = qq * 2 + h;
                    if (act && key_of(e[h]) == k) { hit = (int)jj; hv = val_of(e[h]); }
                    if (e[h] == kEmptySlot) emask |= 1u << jj;
                }
            }
            bool to_need = false;
            if (OP == 0) {
                const unsigned long long kv = make_kv(k, vv[u]);
                uint8_t st = 0;
                if (act && hit >= 0) {
                    bk[hit] = kv;
                    st = 2;
                    mod = true;
                    n_b++;
                } else if (act && clean && emask) {
                    bool placed = false;
                    for (;;) {
                        if (!emask) {             // every snapshot slot taken meanwhile: re-read
#pragma unroll
                            for (int j = 0; j < 8; j++)
                                if (bk[j] == kEmptySlot) emask |= 1u << j;
                            if (!emask) break;
                        }
                        const int j = __ffs(emask) - 1;
                        emask &= emask - 1;
                        if (atomicCAS((unsigned long long*)&tab[lb * 8 + j], kEmptySlot, kv) == kEmptySlot) {
                            placed = true;
                            break;
                        }
                    }
                    if (placed) { st = 1; n_a++; mod = true; }
                    else to_need = true;
                } else if (act) {
                    to_need = true;
                }
                if (valid && !to_need) st2[p] = st;
            } else if (OP == 1) {
                if (valid) {
                    if (act && hit >= 0) { st2[p] = 1; r2[p] = hv; }
                    else if (!act || (clean && emask)) { st2[p] = 0; r2[p] = kEmptyKey; }
                    else to_need = true;
                }
            } else {
                if (valid) {
                    const bool was_full = (fullw[lb >> 5] >> (lb & 31)) & 1u;
                    if (act && hit >= 0) {
                        bk[hit] = kEmptySlot;
                        st2[p] = 1;
                        r2[p] = hv;
                        mod = true;
                        n_a++;
                    } else if (!act || (clean && !was_full)) {
                        st2[p] = 0;
                        r2[p] = kEmptyKey;
                    } else {
                        to_need = true;
                    }
                }
            }
            const unsigned m = __ballot_sync(kFull, to_need);
            if (m) {
                if (ncount + __popc(m) > (uint32_t)kStNeedBuf) flush();
                if (to_need) {
                    const uint32_t e = ncount + __popc(m & lanemask_lt());
                    nbuf[w][e] = p;
                    nbufk[w][e] = k;
                    if (OP == 0) nbufv[OP == 0 ? w : 0][OP == 0 ? e : 0] = vv[u];
                }
                ncount += __popc(m);
            }
        }
    }
    flush();
    if (OP == 0) {
        block_add<kStAT>(ctr + C_INSERTED, n_a);
        block_add<kStAT>(ctr + C_UPDATED, n_b);
    } else if (OP == 2) {
        block_add<kStAT>(ctr + C_REMOVED, n_a);
    }
    if (OP != 1) {
        if (mod) changed = 1;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (threadIdx.x == 0 && changed) st_bulk_store(gsrc, tab, bytes);
    }
}

// ------------------------------------------------------------------ results
// Results of one tile back to the order before its scatter: the tile's sorted
// results are gathered through dmap (runs of consecutive positions, so the reads
// coalesce) into shared memory, then op i of the tile takes entry spos[i].
template <int LEVEL>
__global__ void __launch_bounds__(kStUT) k_st_unperm(StagedView s, uint64_t n, const uint32_t* __restrict__ tile_first,
                                                    const uint32_t* __restrict__ tile_bin,
                                                    const uint32_t* __restrict__ tile_lo,
                                                    const uint32_t* __restrict__ tile_hi,
                                                    const uint32_t* __restrict__ dmap, const uint16_t* __restrict__ spos,
                                                    const uint8_t* __restrict__ src_s, const uint32_t* __restrict__ src_r,
                                                    uint8_t* __restrict__ dst_s, uint32_t* __restrict__ dst_r) {
    __shared__ uint32_t sr[kStTile];
    __shared__ uint8_t ss[kStTile];
    uint32_t t0, tn;
    if (LEVEL == 1) {
        t0 = blockIdx.x * kStTile;
        tn = (uint32_t)(n - t0 < (uint64_t)kStTile ? n - t0 : (uint64_t)kStTile);
    } else {
        if (blockIdx.x >= tile_first[s.nbins]) return;
        t0 = tile_lo[blockIdx.x];
        tn = tile_hi[blockIdx.x] - t0;
    }
    uint16_t q[kStUPer];
    uint32_t vr[kStUPer];
    uint8_t vs[kStUPer];
#pragma unroll
    for (int j = 0; j < kStUPer; j++) {
        const uint32_t i = j * kStUT + threadIdx.x;
        const bool ok = i < tn;
        q[j] = ok ? spos[t0 + i] : (uint16_t)0;
        const uint32_t src = ok ? dmap[t0 + i] : 0u;
        vs[j] = (dst_s && ok) ? src_s[src] : (uint8_t)0;
        vr[j] = (dst_r && ok) ? src_r[src] : 0u;
    }
#pragma unroll
    for (int j = 0; j < kStUPer; j++) {
        const uint32_t p = j * kStUT + threadIdx.x;
        if (p < tn) { ss[p] = vs[j]; sr[p] = vr[j]; }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kStUPer; j++) {
        const uint32_t i = j * kStUT + threadIdx.x;
        if (i < tn) {
            if (dst_s) dst_s[t0 + i] = ss[q[j]];
            if (dst_r) dst_r[t0 + i] = sr[q[j]];
        }
    }
}

}  // namespace dyc
