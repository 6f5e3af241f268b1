// dyc_api.cu — host control (resize policy, scratch, counters) and the C ABI of
// libdyc.so (include/dycuckoo.h).
//
// Host policy (readings Q11-Q13, Q17, Q29):
//   insert: upsize the smallest subtable while (m + n_new) > beta*N, place, settle
//           failures (retry, then failure-triggered upsize), then the
//           alpha loop;
//   delete: erase, then halve the largest subtable while m < alpha*N (unless it
//           is odd / a single bucket, or halving would exceed beta; a downsize
//           whose residuals needed a failure upsize ends the loop, Q17b).
// All comparisons are `(double)m <op> bound*(double)N` on the host (Q29).
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include <cuda.h>
#include <cuda_runtime.h>

#include "dycuckoo.h"
#include "dyc_device.cuh"
#include "dyc_kernels.cuh"
#include "dyc_staged.cuh"

using namespace dyc;

namespace {

thread_local std::string g_err;

dyc_status set_err(dyc_status s, const std::string& msg) {
    g_err = msg;
    return s;
}

dyc_status cuda_err(cudaError_t e, const char* what) {
    return set_err(e == cudaErrorMemoryAllocation ? DYC_ERR_OOM : DYC_ERR_CUDA,
                   std::string(what) + ": " + cudaGetErrorString(e));
}

#define CU(x)                                            \
    do {                                                 \
        cudaError_t e_ = (x);                            \
        if (e_ != cudaSuccess) return cuda_err(e_, #x);  \
    } while (0)

#define TRY(x)                          \
    do {                                \
        dyc_status s_ = (x);            \
        if (s_ != DYC_OK) return s_;    \
    } while (0)

uint64_t splitmix64(uint64_t& s) {
    uint64_t z = (s += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t fastmod_magic(uint64_t n) { return n <= 1 ? 0ull : (~0ull / n) + 1ull; }

inline cudaStream_t S(dyc_stream_t s) { return reinterpret_cast<cudaStream_t>(s); }

// ------------------------------------------------------------ virtual memory
// Subtables can live in a reserved virtual address range whose physical
// backing grows and shrinks in place (DYC_RESIZE_IN_PLACE): an upsize maps only
// the new half behind the old buckets and splits there, a
// downsize merges into the lower half and unmaps the upper one.
// The driver entry points are fetched through the runtime, so libdyc.so has no
// link-time libcuda dependency; if any is missing the tables use cudaMalloc.
struct VmmApi {
    bool ok = false;
    CUresult (*reserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
    CUresult (*addr_free)(CUdeviceptr, size_t) = nullptr;
    CUresult (*create)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long) = nullptr;
    CUresult (*release)(CUmemGenericAllocationHandle) = nullptr;
    CUresult (*map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
    CUresult (*unmap)(CUdeviceptr, size_t) = nullptr;
    CUresult (*set_access)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t) = nullptr;
    CUresult (*granularity)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags) = nullptr;
};

VmmApi& vmm_api() {
    static VmmApi v;
    static bool tried = false;
    if (tried) return v;
    tried = true;
    auto get = [](const char* name, void** fn) {
        cudaDriverEntryPointQueryResult q;
        return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
               q == cudaDriverEntryPointSuccess && *fn;
    };
    bool ok = get("cuMemAddressReserve", (void**)&v.reserve) && get("cuMemAddressFree", (void**)&v.addr_free) &&
              get("cuMemCreate", (void**)&v.create) && get("cuMemRelease", (void**)&v.release) &&
              get("cuMemMap", (void**)&v.map) && get("cuMemUnmap", (void**)&v.unmap) &&
              get("cuMemSetAccess", (void**)&v.set_access) &&
              get("cuMemGetAllocationGranularity", (void**)&v.granularity);
    cudaGetLastError();
    v.ok = ok;
    return v;
}

}  // namespace

// The placement kernel of the table's mode (first-fit or paper-weighted).
#define DYC_PLACE_K(BB) (t->weighted ? k_place<BB, true> : k_place<BB, false>)

// Error channel shared with the other translation units (dyc_dist.cu).
void dyc_internal_set_error(const std::string& msg) { g_err = msg; }

struct dyc_table {
    dyc_config cfg{};
    int device = 0;
    int num_sms = 148;
    int place_blocks = 148 * 8;            // persistent grid of k_place
    // device memory: cudaMalloc plus a per-table cache of released buffers
    // (stream-ordered pool growth measured 10-30 GB/s on B200 vs ~1 ms/GB for
    // cudaMalloc; profiles/r1_memory_model.md)
    struct CachedBuf { void* p; uint64_t bytes; cudaEvent_t ev; };
    std::vector<CachedBuf> cache;
    uint64_t cache_bytes = 0;
    std::unordered_map<void*, uint64_t> live;   // pointer -> bytes of live allocations
    unsigned long long* sub[DYC_MAX_D] = {};
    uint64_t nb[DYC_MAX_D] = {};
    // in-place resizing (DYC_RESIZE_IN_PLACE): subtable t lives in a reserved
    // virtual range when vm[t].base != 0; chunks are the physical pieces mapped
    // at its end, in mapping order
    struct Vm {
        CUdeviceptr base = 0;
        size_t reserved = 0, mapped = 0;
        std::vector<std::pair<CUmemGenericAllocationHandle, size_t>> chunks;
    } vm[DYC_MAX_D];
    bool in_place = false;
    size_t vm_gran = 0;
    uint32_t vm_shrink_pending = 0;        // subtables halved in place, upper half still mapped
    uint64_t n_vm_map = 0, n_vm_unmap = 0;
    uint32_t a[DYC_MAX_D + 2] = {}, b[DYC_MAX_D + 2] = {};
    uint64_t m = 0;
    // first-choice-full invariant per subtable (TableView::clean):
    // set for all on create / clear; an upsize of t (split buckets are no longer
    // full) or a live resize of t clears bit t; a batch that removed keys, a
    // reinsert
    // baseline clears all.  Downsizes and placements (first-fit, evictions)
    // preserve it.
    uint32_t clean = 0;
    // m is the live count as of the last counter read-back.  A batch that cannot
    // trigger a resize decision skips its read-back (lazy): its counts wait in
    // the accumulating device counters (C_ADDED, C_REMOVED, ...) until the next
    // read_ctr applies them, and the exact count lies in
    // [m - lazy_del, m + lazy_add] (flush_m before any decision that needs it).
    // lazy_ev marks the last lazy batch on its stream (ev_pending until read).
    bool m_lazy = false;
    uint64_t lazy_del = 0, lazy_add = 0;
    cudaEvent_t lazy_ev = nullptr;
    bool ev_pending = false;
    bool ins_lazy = false;                 // the last insert's per-batch stats are still on the device
    uint64_t ins_n = 0;                    // ops of the insert batch in flight
    // stash (dyc_kernels.cuh stash_find): pairs a lazily settled insert could
    // not place; the next sync_state settles them (retry, failure upsizes)
    unsigned long long* stash = nullptr;
    uint64_t stash_cap = 0;
    uint64_t stash_bound = 0;              // upper bound of its entries since the last settle
    uint64_t del_n = 0;                    // ops of the delete batch in flight
    // placement policy (dyc_config.flags): first-fit (reading Q3) or the
    // paper's weighted rule; the latter keeps d_w, a per-batch
    // snapshot of n_t / C(m_t, 2), and gives up the first-choice-full invariant
    bool weighted = false;
    float* d_w = nullptr;
    bool count_probes = false;             // dyc_probe_count_enable (measurement)
    unsigned long long* d_probe = nullptr; // {ops, second probes} x {find, upsert, delete}
    unsigned long long* list[2] = {nullptr, nullptr};
    uint64_t list_cap = 0;
    unsigned long long* d_ctr = nullptr;   // C_N device counters
    unsigned long long* h_ctr = nullptr;   // pinned mirror
    unsigned long long* h_mix = nullptr;   // pinned: phase sizes of a mixed batch
    // phase sizes of lazily run mixed batches, copied back asynchronously: once
    // a copy has landed (event query, no wait) the bounds that batch added to
    // lazy_add / lazy_del (n each) shrink to its exact sizes, provided no
    // read-back has happened since (sync_epoch)
    struct MixRec { int slot; cudaEvent_t ev; uint64_t epoch, n, ins_bound, del_bound; };
    std::vector<MixRec> mix_recs;
    unsigned long long* h_mix_ring = nullptr;   // pinned [kMixRing][4]
    uint32_t mix_ring_next = 0;
    uint64_t sync_epoch = 0;
    void* stage = nullptr;                 // device staging for the host-buffer entry points
    uint64_t stage_cap = 0;
    cudaStream_t cp_in = nullptr, cp_out = nullptr;   // copy streams of the host-buffer path
    int part_op = 0;                       // 1 insert / 2 delete batch open (dyc_*_begin)
    bool part_fuse = false;
    uint64_t part_left = 0;
    void* mix = nullptr;                   // scratch of dyc_mixed_batch
    uint64_t mix_cap = 0;
    uint64_t n_upsize = 0, n_downsize = 0, n_fail_upsize = 0, n_residual = 0, n_evict = 0, n_place_retry = 0;
    uint64_t n_pending_total = 0;          // new keys handed to k_place by all insert batches
    uint64_t launches = 0;
    uint64_t last_new = 0, last_pending = 0, last_evict = 0;
    cudaStream_t last = nullptr;
    // resize under live traffic (dyc_resize_begin / dyc_resize_commit, NEXT-1):
    // the split / merge kernel of subtable `ti` runs on the caller's resize
    // stream into `nbuf` while batches keep using the old buffer of ti
    // (read-only for them: the LK kernel variants defer any write to ti).
    struct Live {
        bool active = false;
        int dir = 0;
        uint32_t ti = 0;
        unsigned long long* nbuf = nullptr;
        uint64_t nnb = 0;
        unsigned long long* res[2] = {nullptr, nullptr};   // downsize residuals / their failures
        unsigned long long* ctr = nullptr;                  // counters of the resize stream (C_N)
        cudaEvent_t start = nullptr, done = nullptr;
    } rz;
    uint64_t n_live_resize = 0, n_deferred = 0;
    uint64_t n_device_alloc = 0;
    double alloc_ms = 0.0;
    // chunk-staged execution of large batches (dyc_staged.cuh): one scratch
    // buffer, grown on demand; n_staged counts the batches that took the path
    void* stg = nullptr;
    uint64_t stg_cap = 0;
    uint64_t n_staged = 0;
    uint64_t peak_table_bytes = 0;   // high-water mark of the subtables' bytes (cache cap)
    uint64_t n_sync = 0;          // counter read-backs (host waits on the stream)
    double sync_ms = 0.0;
    // per-kernel event profiling (dyc_profile_*)
    bool prof = false;
    struct Rec { int kind; cudaEvent_t a, b; };
    std::vector<Rec> recs;
    std::vector<cudaEvent_t> ev_pool;
    double prof_ms[DYC_PROF_KINDS] = {};
    uint64_t prof_calls[DYC_PROF_KINDS] = {};

    cudaEvent_t ev() {
        if (!ev_pool.empty()) { cudaEvent_t e = ev_pool.back(); ev_pool.pop_back(); return e; }
        cudaEvent_t e = nullptr;
        cudaEventCreate(&e);
        return e;
    }

    uint64_t N() const {
        uint64_t s = 0;
        for (uint32_t t = 0; t < cfg.d; t++) s += nb[t] * cfg.bucket_slots;
        return s;
    }
    // N once the resize in flight (if any) is committed: the size every resize
    // decision is taken against, as if the resize had completed first
    uint64_t N_after() const {
        return rz.active ? N() - nb[rz.ti] * cfg.bucket_slots + rz.nnb * cfg.bucket_slots : N();
    }
    int smallest() const {      // ties -> lowest index (Q12)
        int best = 0;
        for (uint32_t t = 1; t < cfg.d; t++)
            if (nb[t] < nb[best]) best = (int)t;
        return best;
    }
    int largest() const {       // ties -> highest index (Q12)
        int best = (int)cfg.d - 1;
        for (int t = (int)cfg.d - 2; t >= 0; t--)
            if (nb[t] > nb[best]) best = t;
        return best;
    }
    TableView view() const {
        TableView v{};
        for (uint32_t t = 0; t < cfg.d; t++) {
            v.sub[t].slots = sub[t];
            v.sub[t].n = (uint32_t)nb[t];
            v.sub[t].magic = fastmod_magic(nb[t]);
        }
        for (uint32_t s = 0; s < cfg.d + 2; s++) { v.a[s] = a[s]; v.b[s] = b[s]; }
        v.d = cfg.d;
        v.d2 = cfg.d * (cfg.d - 1);
        v.magic_d2 = fastmod_magic(v.d2);
        v.dm1 = cfg.d - 1;
        v.recip_dm1 = (65536u + v.dm1 - 1) / v.dm1;
        v.max_hops = cfg.max_hops;
        v.clean = weighted ? 0u : (rz.active ? (clean & ~(1u << rz.ti)) : clean);
        v.probe = count_probes ? d_probe : nullptr;
        v.wsel = weighted ? d_w : nullptr;
        v.stash = stash;
        v.stash_n = (d_ctr && stash_bound) ? d_ctr + C_STASH : nullptr;   // known empty: no load at all
        return v;
    }
};

namespace {

// Records CUDA events around one launch when profiling is on (measurement only).
struct ProfScope {
    dyc_table* t;
    int kind;
    cudaStream_t st;
    cudaEvent_t a = nullptr;
    ProfScope(dyc_table* t_, int kind_, cudaStream_t st_) : t(t_), kind(kind_), st(st_) {
        t->launches++;
        if (t->prof) { a = t->ev(); cudaEventRecord(a, st); }
    }
    ~ProfScope() {
        if (a) {
            cudaEvent_t b = t->ev();
            cudaEventRecord(b, st);
            t->recs.push_back({kind, a, b});
        }
    }
};

unsigned grid_for(uint64_t work, uint64_t per_block) {
    uint64_t g = (work + per_block - 1) / per_block;
    g = std::max<uint64_t>(1, std::min<uint64_t>(g, 1u << 30));
    return (unsigned)g;
}

// Physical backing of subtable t's virtual range grown to at least `bytes`.
dyc_status vm_grow(dyc_table* t, uint32_t ti, uint64_t bytes) {
    VmmApi& A = vmm_api();
    auto& v = t->vm[ti];
    while (v.mapped < bytes) {
        const size_t sz = (bytes - v.mapped + t->vm_gran - 1) / t->vm_gran * t->vm_gran;
        if (v.mapped + sz > v.reserved) return set_err(DYC_ERR_OOM, "subtable outgrew its reserved address range");
        CUmemAllocationProp prop{};
        prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
        prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        prop.location.id = t->device;
        CUmemGenericAllocationHandle h;
        const auto t0 = std::chrono::steady_clock::now();
        if (A.create(&h, sz, &prop, 0) != CUDA_SUCCESS) return set_err(DYC_ERR_OOM, "cuMemCreate failed");
        if (A.map(v.base + v.mapped, sz, 0, h, 0) != CUDA_SUCCESS) {
            A.release(h);
            return set_err(DYC_ERR_CUDA, "cuMemMap failed");
        }
        CUmemAccessDesc acc{};
        acc.location = prop.location;
        acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        if (A.set_access(v.base + v.mapped, sz, &acc, 1) != CUDA_SUCCESS) {
            A.unmap(v.base + v.mapped, sz);
            A.release(h);
            return set_err(DYC_ERR_CUDA, "cuMemSetAccess failed");
        }
        t->alloc_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        v.chunks.push_back({h, sz});
        v.mapped += sz;
        t->n_vm_map++;
    }
    return DYC_OK;
}

// Unmaps the chunks of subtable t's range that lie wholly at or beyond `keep`
// bytes.  The caller guarantees no enqueued work still touches them.
void vm_shrink(dyc_table* t, uint32_t ti, uint64_t keep) {
    VmmApi& A = vmm_api();
    auto& v = t->vm[ti];
    while (!v.chunks.empty() && v.mapped - v.chunks.back().second >= keep) {
        const auto c = v.chunks.back();
        A.unmap(v.base + v.mapped - c.second, c.second);
        A.release(c.first);
        v.mapped -= c.second;
        v.chunks.pop_back();
        t->n_vm_unmap++;
    }
}

// A fresh virtual range for subtable t with `bytes` mapped (false if virtual
// memory is not available: the caller falls back to cudaMalloc).
bool vm_create(dyc_table* t, uint32_t ti, uint64_t bytes) {
    VmmApi& A = vmm_api();
    if (!t->in_place || !A.ok || t->vm_gran == 0) return false;
    auto& v = t->vm[ti];
    const size_t reserve = (size_t)1 << 38;            // 256 GB of address space: any subtable fits
    if (A.reserve(&v.base, reserve, t->vm_gran, 0, 0) != CUDA_SUCCESS) {
        v.base = 0;
        return false;
    }
    v.reserved = reserve;
    v.mapped = 0;
    if (vm_grow(t, ti, bytes) != DYC_OK) {
        vm_shrink(t, ti, 0);
        A.addr_free(v.base, v.reserved);
        v = dyc_table::Vm();
        cudaGetLastError();
        return false;
    }
    return true;
}

// Releases a virtual range (after the work that used it: synchronizes `st`).
void vm_release_range(dyc_table* t, dyc_table::Vm& v, cudaStream_t st) {
    if (!v.base) return;
    cudaStreamSynchronize(st);
    VmmApi& A = vmm_api();
    for (auto it = v.chunks.rbegin(); it != v.chunks.rend(); ++it) {
        v.mapped -= it->second;
        A.unmap(v.base + v.mapped, it->second);
        A.release(it->first);
        t->n_vm_unmap++;
    }
    A.addr_free(v.base, v.reserved);
    v = dyc_table::Vm();
}

void vm_release(dyc_table* t, uint32_t ti, cudaStream_t st) { vm_release_range(t, t->vm[ti], st); }

// Releases the buffer of subtable ti (virtual range or cached cudaMalloc).
void dev_free(dyc_table* t, void* p, cudaStream_t st);
void free_sub(dyc_table* t, uint32_t ti, cudaStream_t st) {
    if (t->vm[ti].base) vm_release(t, ti, st);
    else dev_free(t, t->sub[ti], st);
    t->sub[ti] = nullptr;
}

void trim_cache(dyc_table* t) {
    for (auto& c : t->cache) {
        cudaFree(c.p);                       // synchronizes the device
        if (c.ev) t->ev_pool.push_back(c.ev);
    }
    t->cache.clear();
    t->cache_bytes = 0;
}

// Allocation: an exact-size buffer released earlier by this table is reused (the
// stream first waits for the work that used it); otherwise cudaMalloc.  On OOM
// the cache is flushed and the allocation retried once.
dyc_status dev_alloc(dyc_table* t, void** p, uint64_t bytes, cudaStream_t st) {
    bytes = std::max<uint64_t>(bytes, 256);
    for (size_t i = 0; i < t->cache.size(); i++) {
        if (t->cache[i].bytes == bytes) {
            dyc_table::CachedBuf c = t->cache[i];
            t->cache.erase(t->cache.begin() + (long)i);
            t->cache_bytes -= c.bytes;
            if (c.ev) {
                cudaStreamWaitEvent(st, c.ev, 0);
                t->ev_pool.push_back(c.ev);
            }
            *p = c.p;
            t->live[c.p] = bytes;
            return DYC_OK;
        }
    }
    const auto t0 = std::chrono::steady_clock::now();
    cudaError_t e = cudaMalloc(p, bytes);
    if (e == cudaErrorMemoryAllocation && !t->cache.empty()) {
        cudaGetLastError();
        trim_cache(t);
        e = cudaMalloc(p, bytes);
    }
    t->n_device_alloc++;
    t->alloc_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if (e != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return set_err(DYC_ERR_OOM, std::string("device allocation of ") + std::to_string(bytes) + " bytes failed: " +
                                        cudaGetErrorString(e));
    }
    t->live[*p] = bytes;
    return DYC_OK;
}

// Release: the buffer goes to the cache, tagged with an event on `st` so that a
// later reuse waits for the work still using it.
void dev_free(dyc_table* t, void* p, cudaStream_t st) {
    if (!p) return;
    auto it = t->live.find(p);
    const uint64_t bytes = it == t->live.end() ? 0 : it->second;
    if (it != t->live.end()) t->live.erase(it);
    cudaEvent_t ev = t->ev();
    cudaEventRecord(ev, st);
    t->cache.push_back({p, bytes, ev});
    t->cache_bytes += bytes;
    // keep up to twice the table's high-water size (+256 MB) cached, not just
    // its current size: a shrink phase would otherwise free (cudaFree syncs the
    // device) exactly the buffers the next growth phase allocates again, and
    // fresh cudaMalloc calls are where the stream configs' run-to-run variance
    // came from (profiles/r1t_c5_variance.md; C3-RE's 9 cudaMalloc calls per
    // pass took 12 ms in r2m and 84 ms in r2n with a cap of one high-water size:
    // a growth phase holds every smaller power-of-two buffer of the subtables
    // in the cache at once).  An allocation that fails flushes the cache and
    // retries; dyc_trim releases it.
    uint64_t cur = 0;
    for (uint32_t i = 0; i < t->cfg.d; i++) cur += t->nb[i] * t->cfg.bucket_slots * 8;
    t->peak_table_bytes = std::max(t->peak_table_bytes, cur);
    const uint64_t cap = (256ull << 20) + 2 * t->peak_table_bytes;
    while (t->cache_bytes > cap && !t->cache.empty()) {      // oldest first
        cudaEventSynchronize(t->cache.front().ev);
        cudaFree(t->cache.front().p);
        t->ev_pool.push_back(t->cache.front().ev);
        t->cache_bytes -= t->cache.front().bytes;
        t->cache.erase(t->cache.begin());
    }
}

dyc_status read_ctr(dyc_table* t, cudaStream_t st) {
    // a lazy batch may have run on another stream: its counts must have landed
    // in the accumulators before the copy and the reset below
    if (t->ev_pending && t->lazy_ev) CU(cudaStreamWaitEvent(st, t->lazy_ev, 0));
    CU(cudaMemcpyAsync(t->h_ctr, t->d_ctr, C_N * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    const auto t0 = std::chrono::steady_clock::now();
    CU(cudaStreamSynchronize(st));
    t->sync_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    t->n_sync++;
    // the stream is idle: the upper halves of subtables merged in place can go
    for (uint32_t i = 0; t->vm_shrink_pending && i < t->cfg.d; i++)
        if (t->vm_shrink_pending & (1u << i)) {
            vm_shrink(t, i, t->nb[i] * t->cfg.bucket_slots * 8);
            t->vm_shrink_pending &= ~(1u << i);
        }
    // every read-back applies what the batches counted since the last one (the
    // lazy ones included): live-count changes, evictions, pending keys
    const unsigned long long* h = t->h_ctr;
    const unsigned long long added = h[C_ADDED], removed = h[C_REMOVED];
    t->m = t->m + added - removed;
    if (removed) t->clean = 0;   // emptied slots break the first-choice-full invariant
    t->n_evict += h[C_EVICT];
    t->n_pending_total += h[C_PEND_ACC];
    if (t->ins_lazy) {
        t->last_new = h[C_INSERTED];
        t->last_pending = h[C_PENDING];
        t->last_evict = h[C_EVICT];
        t->ins_lazy = false;
    }
    if (added | removed | h[C_EVICT] | h[C_PEND_ACC])
        CU(cudaMemsetAsync(t->d_ctr + C_REMOVED, 0, (C_COUNT0 - C_REMOVED) * sizeof(unsigned long long), st));
    t->m_lazy = false;
    t->ev_pending = false;
    t->lazy_del = t->lazy_add = 0;
    t->sync_epoch++;
    return DYC_OK;
}

// zeroes the per-batch counters ([0, C_ACC0) and the per-subtable counts); the
// accumulators and the stash count belong to read_ctr / the stash settling
dyc_status zero_ctr(dyc_table* t, cudaStream_t st) {
    CU(cudaMemsetAsync(t->d_ctr, 0, C_ACC0 * sizeof(unsigned long long), st));
    CU(cudaMemsetAsync(t->d_ctr + C_COUNT0, 0, (C_N - C_COUNT0) * sizeof(unsigned long long), st));
    return DYC_OK;
}

// A lazy batch returns without a host wait: remember its stream position.
dyc_status mark_lazy(dyc_table* t, cudaStream_t st) {
    if (!t->lazy_ev) CU(cudaEventCreateWithFlags(&t->lazy_ev, cudaEventDisableTiming));
    CU(cudaEventRecord(t->lazy_ev, st));
    t->ev_pending = true;
    return DYC_OK;
}

constexpr uint64_t kStashMin = 1ull << 20, kStashMax = 1ull << 26;   // stash entries
constexpr uint32_t kMixRing = 16;                                     // async phase-size copies in flight

dyc_status zero_one(dyc_table* t, int idx, cudaStream_t st) {
    CU(cudaMemsetAsync(t->d_ctr + idx, 0, sizeof(unsigned long long), st));
    return DYC_OK;
}

dyc_status ensure_lists(dyc_table* t, uint64_t n, cudaStream_t st) {
    if (n <= t->list_cap) return DYC_OK;
    uint64_t cap = std::max<uint64_t>(n, 2 * t->list_cap);
    void* l0 = nullptr;
    void* l1 = nullptr;
    TRY(dev_alloc(t, &l0, cap * 8, st));
    dyc_status s = dev_alloc(t, &l1, cap * 8, st);
    if (s != DYC_OK) {
        dev_free(t, l0, st);
        return s;
    }
    dev_free(t, t->list[0], st);
    dev_free(t, t->list[1], st);
    t->list[0] = (unsigned long long*)l0;
    t->list[1] = (unsigned long long*)l1;
    t->list_cap = cap;
    return DYC_OK;
}

// Paper-weighted mode: snapshot w[t] = n_t / C(m_t, 2) from a count
// of every subtable (one streaming pass over the table, in stream order, so it
// sees the state the next placement kernel starts from).
// Stash capacity for `need` entries; live entries are carried over (in stream order).
dyc_status ensure_stash(dyc_table* t, uint64_t need, cudaStream_t st) {
    if (need <= t->stash_cap) return DYC_OK;
    const uint64_t cap = std::max<uint64_t>(need, 2 * t->stash_cap);
    void* p = nullptr;
    TRY(dev_alloc(t, &p, cap * 8, st));
    if (t->stash && t->stash_bound)
        CU(cudaMemcpyAsync(p, t->stash, t->stash_cap * 8, cudaMemcpyDeviceToDevice, st));
    dev_free(t, t->stash, st);
    t->stash = (unsigned long long*)p;
    t->stash_cap = cap;
    return DYC_OK;
}

template <int B>
dyc_status refresh_weights(dyc_table* t, cudaStream_t st) {
    if (!t->weighted) return DYC_OK;
    CU(cudaMemsetAsync(t->d_ctr + C_COUNT0, 0, t->cfg.d * sizeof(unsigned long long), st));
    const TableView tv = t->view();
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        ProfScope ps(t, DYC_PROF_OTHER, st);
        k_count<B><<<grid_for(t->nb[i] * B, kThreads * 8), kThreads, 0, st>>>(tv, i, t->d_ctr);
    }
    {
        ProfScope ps(t, DYC_PROF_OTHER, st);
        k_weights<<<1, 32, 0, st>>>(tv, B, t->d_ctr, t->d_w);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

template <int B>
dyc_status upsize_table(dyc_table* t, uint32_t ti, cudaStream_t st) {
    const uint64_t n_old = t->nb[ti], n_new = 2 * n_old;
    if (n_new > 0xFFFFFFFFull) return set_err(DYC_ERR_OOM, "subtable would exceed 2^32 buckets");
    const uint64_t slots = n_old * B;
    if (t->vm[ti].base) {
        // in place: map the new half behind the old buckets, split there
        t->vm_shrink_pending &= ~(1u << ti);
        TRY(vm_grow(t, ti, n_new * B * 8));
        {
            ProfScope ps(t, DYC_PROF_UPSIZE, st);
            k_upsize<B><<<grid_for(slots, kThreads * kResU), kThreads, 0, st>>>(
                t->sub[ti], t->sub[ti], (uint32_t)n_old, t->a[ti + 1], t->b[ti + 1], fastmod_magic(n_new),
                (uint32_t)n_new);
        }
        CU(cudaGetLastError());
    } else {
        void* p = nullptr;
        TRY(dev_alloc(t, &p, n_new * B * 8, st));
        {
            ProfScope ps(t, DYC_PROF_UPSIZE, st);
            k_upsize<B><<<grid_for(slots, kThreads * kResU), kThreads, 0, st>>>(
                t->sub[ti], (unsigned long long*)p, (uint32_t)n_old, t->a[ti + 1], t->b[ti + 1], fastmod_magic(n_new),
                (uint32_t)n_new);
        }
        CU(cudaGetLastError());
        free_sub(t, ti, st);
        t->sub[ti] = (unsigned long long*)p;
    }
    t->nb[ti] = n_new;
    t->clean &= ~(1u << ti);        // split buckets are no longer full
    return DYC_OK;
}

// Retries the nfail homeless pairs in list[cur]: first a plain retry pass, then
// failure-triggered upsizes (Q17: nothing is ever dropped).
template <int B>
dyc_status settle(dyc_table* t, int cur, uint64_t nfail, cudaStream_t st, unsigned long long* const* lists = nullptr) {
    unsigned long long* const* L = lists ? lists : t->list;
    int round = 0;
    while (nfail > 0) {
        if (round > 0) {
            TRY(upsize_table<B>(t, (uint32_t)t->smallest(), st));
            t->n_fail_upsize++;
        }
        round++;
        t->n_place_retry++;
        TRY(zero_one(t, C_FAIL, st));
        {
            ProfScope ps(t, DYC_PROF_PLACE, st);
            DYC_PLACE_K(B)<<<grid_for(nfail, kThreads / (B / 4)), kThreads, 0, st>>>(t->view(), L[cur], nullptr, nfail,
                                                                              L[1 - cur], t->d_ctr, true, nullptr, false);
        }
        CU(cudaGetLastError());
        TRY(read_ctr(t, st));
        nfail = t->h_ctr[C_FAIL];
        cur = 1 - cur;
        if (round > 64) return set_err(DYC_ERR_INSERT_FAILED, "placement kept failing after 64 upsizes");
    }
    return DYC_OK;
}

// Launches k_place over list[src][0..cnt) (count on the host or in a device
// counter); homeless pairs are appended to list[1-src] at the C_FAIL cursor.
template <int B>
dyc_status launch_place(dyc_table* t, int src, const unsigned long long* d_count, uint64_t h_count, bool first_fit,
                        cudaStream_t st) {
    ProfScope ps(t, DYC_PROF_PLACE, st);
    DYC_PLACE_K(B)<<<t->place_blocks, kThreads, 0, st>>>(t->view(), t->list[src], d_count, h_count, t->list[1 - src],
                                                     t->d_ctr, first_fit, nullptr, false);
    CU(cudaGetLastError());
    return DYC_OK;
}

// Place list[src][0..cnt) and settle failures.
template <int B>
dyc_status place_and_settle(dyc_table* t, int src, const unsigned long long* d_count, uint64_t h_count,
                            bool first_fit, cudaStream_t st) {
    TRY(zero_one(t, C_FAIL, st));
    TRY(launch_place<B>(t, src, d_count, h_count, first_fit, st));
    TRY(read_ctr(t, st));
    return settle<B>(t, 1 - src, t->h_ctr[C_FAIL], st);
}

// Settles the stash (pairs the lazily settled inserts could not place):
// one placement pass over it, then the usual retry / failure-upsize loop (Q17).
template <int B>
dyc_status settle_stash(dyc_table* t, cudaStream_t st) {
    const uint64_t S = t->h_ctr[C_STASH];
    TRY(ensure_lists(t, S, st));
    TRY(zero_one(t, C_FAIL, st));
    {
        ProfScope ps(t, DYC_PROF_PLACE, st);
        DYC_PLACE_K(B)<<<t->place_blocks, kThreads, 0, st>>>(t->view(), t->stash, nullptr, S, t->list[1], t->d_ctr, true, nullptr, false);
    }
    CU(cudaGetLastError());
    TRY(zero_one(t, C_STASH, st));
    t->stash_bound = 0;
    TRY(read_ctr(t, st));
    return settle<B>(t, 1, t->h_ctr[C_FAIL], st);
}

// Exact state: apply every count still on the device and settle the stash.
template <int B>
dyc_status sync_state(dyc_table* t, cudaStream_t st) {
    TRY(read_ctr(t, st));
    if (t->h_ctr[C_STASH]) return settle_stash<B>(t, st);
    t->stash_bound = 0;
    return DYC_OK;
}

template <int B>
dyc_status flush_m(dyc_table* t, cudaStream_t st) {
    return (t->m_lazy || t->ev_pending || t->stash_bound) ? sync_state<B>(t, st) : DYC_OK;
}

// Halves subtable ti: merge kernel, then residual placement into
// the pairs' other tables (a separate kernel, so excluding t is not
// needed for correctness, Q16).  Residual failures are appended to list[1] at
// the C_FAIL cursor and settled by the caller (several downsizes of one alpha
// loop share one host sync).
template <int B>
dyc_status downsize_launch(dyc_table* t, uint32_t ti, cudaStream_t st) {
    const uint64_t n_old = t->nb[ti], h = n_old / 2;
    if (n_old < 2 || (n_old & 1)) return set_err(DYC_ERR_INVALID_ARG, "subtable cannot be halved");
    TRY(zero_one(t, C_RESIDUAL, st));
    if (t->vm[ti].base) {
        // in place: merge into the lower half; the upper half is unmapped at the
        // next host read-back (nothing enqueued after it touches it)
        {
            ProfScope ps(t, DYC_PROF_DOWNSIZE, st);
            k_downsize<B><<<grid_for(h * B, kThreads * kResUD), kThreads, 0, st>>>(t->sub[ti], t->sub[ti], (uint32_t)h,
                                                                           t->list[0], t->d_ctr);
        }
        CU(cudaGetLastError());
        t->vm_shrink_pending |= 1u << ti;
    } else {
        void* p = nullptr;
        TRY(dev_alloc(t, &p, h * B * 8, st));
        {
            ProfScope ps(t, DYC_PROF_DOWNSIZE, st);
            k_downsize<B><<<grid_for(h * B, kThreads * kResUD), kThreads, 0, st>>>(t->sub[ti], (unsigned long long*)p,
                                                                           (uint32_t)h, t->list[0], t->d_ctr);
        }
        CU(cudaGetLastError());
        free_sub(t, ti, st);
        t->sub[ti] = (unsigned long long*)p;
    }
    t->nb[ti] = h;
    TRY(refresh_weights<B>(t, st));
    return launch_place<B>(t, 0, t->d_ctr + C_RESIDUAL, 0, true, st);
}

template <int B>
dyc_status downsize_table(dyc_table* t, uint32_t ti, cudaStream_t st) {
    TRY(ensure_lists(t, (t->nb[ti] / 2) * B, st));
    TRY(zero_one(t, C_FAIL, st));
    TRY(zero_one(t, C_RES_TOTAL, st));
    TRY(downsize_launch<B>(t, ti, st));
    TRY(read_ctr(t, st));
    t->n_residual += t->h_ctr[C_RES_TOTAL];
    return settle<B>(t, 1, t->h_ctr[C_FAIL], st);
}

// Lower bound (Q11-Q13): while m < alpha*N halve the largest
// subtable (unless it is odd / a single bucket, or halving would exceed beta).
// The halvings depend only on m and the sizes, so the whole sequence is planned
// on the host and launched back to back; residual failures of all of them are
// settled once at the end (Q17: retry, then failure-triggered upsizes).
template <int B>
dyc_status enforce_lower(dyc_table* t, cudaStream_t st) {
    TRY(flush_m<B>(t, st));
    uint64_t nb[DYC_MAX_D];
    for (uint32_t i = 0; i < t->cfg.d; i++) nb[i] = t->nb[i];
    std::vector<uint32_t> plan;
    uint64_t res_bound = 0;
    for (;;) {
        uint64_t N = 0;
        for (uint32_t i = 0; i < t->cfg.d; i++) N += nb[i] * B;
        if (!((double)t->m < t->cfg.alpha * (double)N)) break;
        int ti = (int)t->cfg.d - 1;                                   // largest, ties -> highest (Q12)
        for (int i = (int)t->cfg.d - 2; i >= 0; i--)
            if (nb[i] > nb[ti]) ti = i;
        if (nb[ti] < 2 || (nb[ti] & 1)) break;
        const uint64_t N_after = N - (nb[ti] / 2) * B;
        if ((double)t->m > t->cfg.beta * (double)N_after) break;
        plan.push_back((uint32_t)ti);
        res_bound += (nb[ti] / 2) * B;
        nb[ti] /= 2;
    }
    if (plan.empty()) return DYC_OK;
    TRY(ensure_lists(t, std::min<uint64_t>(res_bound, t->m + 1) + 1, st));
    TRY(zero_one(t, C_FAIL, st));
    TRY(zero_one(t, C_RES_TOTAL, st));
    for (uint32_t ti : plan) {
        TRY(downsize_launch<B>(t, ti, st));
        t->n_downsize++;
    }
    TRY(read_ctr(t, st));
    t->n_residual += t->h_ctr[C_RES_TOTAL];
    TRY(settle<B>(t, 1, t->h_ctr[C_FAIL], st));
    return DYC_OK;
}

// ------------------------------------------------ resize under live traffic (NEXT-1)
// Commits the resize in flight: the caller's stream waits for the split/merge
// kernel, the new buffer replaces the old one (released after the batches that
// still read it), and a downsize's residuals are placed into their pairs' other
// tables and settled like any placement failure (Q17).
template <int B>
dyc_status live_commit(dyc_table* t, cudaStream_t st) {
    auto& r = t->rz;
    if (!r.active) return DYC_OK;
    CU(cudaStreamWaitEvent(st, r.done, 0));
    const uint32_t ti = r.ti;
    t->vm_shrink_pending &= ~(1u << ti);
    free_sub(t, ti, st);
    t->sub[ti] = r.nbuf;
    t->nb[ti] = r.nnb;
    r.active = false;
    r.nbuf = nullptr;
    t->n_live_resize++;
    if (r.dir > 0) {
        t->n_upsize++;
        return DYC_OK;
    }
    t->n_downsize++;
    TRY(zero_one(t, C_FAIL, st));
    {
        ProfScope ps(t, DYC_PROF_PLACE, st);
        DYC_PLACE_K(B)<<<t->place_blocks, kThreads, 0, st>>>(t->view(), r.res[0], r.ctr + C_RESIDUAL, 0, r.res[1],
                                                         t->d_ctr, true, nullptr, false);
    }
    CU(cudaGetLastError());
    CU(cudaMemcpyAsync(t->d_ctr + C_RES_TOTAL, r.ctr + C_RES_TOTAL, 8, cudaMemcpyDeviceToDevice, st));
    TRY(read_ctr(t, st));
    t->n_residual += t->h_ctr[C_RES_TOTAL];
    TRY(settle<B>(t, 1, t->h_ctr[C_FAIL], st, r.res));
    dev_free(t, r.res[0], st);
    dev_free(t, r.res[1], st);
    r.res[0] = r.res[1] = nullptr;
    return DYC_OK;
}

// Checks a resize request against the policy's shape rules and
// resolves subtable -1 to the policy's choice.
dyc_status pick_resize(const dyc_table* t, int direction, int subtable, int& ti) {
    ti = subtable;
    if (direction > 0) {
        if (ti < 0) ti = t->smallest();
        if (ti >= (int)t->cfg.d || t->nb[ti] != t->nb[t->smallest()])
            return set_err(DYC_ERR_INVALID_ARG, "only a smallest subtable may be doubled (P:L311-312)");
        if (2 * t->nb[ti] > 0xFFFFFFFFull) return set_err(DYC_ERR_OOM, "subtable would exceed 2^32 buckets");
    } else {
        if (ti < 0) ti = t->largest();
        if (ti >= (int)t->cfg.d || t->nb[ti] != t->nb[t->largest()])
            return set_err(DYC_ERR_INVALID_ARG, "only a largest subtable may be halved (P:L311-312)");
        if (t->nb[ti] < 2 || (t->nb[ti] & 1)) return set_err(DYC_ERR_INVALID_ARG, "subtable cannot be halved");
    }
    return DYC_OK;
}

// Starts the split or merge of one subtable on
// `rs`, after the work already enqueued on `st`, and returns; see dyc_resize_begin.
template <int B>
dyc_status live_begin(dyc_table* t, int direction, int subtable, cudaStream_t st, cudaStream_t rs) {
    auto& r = t->rz;
    if (r.active) return set_err(DYC_ERR_INVALID_ARG, "a resize is already in flight (dyc_resize_commit first)");
    if (t->part_op) return set_err(DYC_ERR_INVALID_ARG, "a batch is open (dyc_*_end first)");
    TRY(flush_m<B>(t, st));
    int ti = -1;
    TRY(pick_resize(t, direction, subtable, ti));
    if (!r.start) CU(cudaEventCreateWithFlags(&r.start, cudaEventDisableTiming));
    if (!r.done) CU(cudaEventCreateWithFlags(&r.done, cudaEventDisableTiming));
    if (!r.ctr) CU(cudaMalloc(&r.ctr, C_N * 8));
    CU(cudaEventRecord(r.start, st));
    CU(cudaStreamWaitEvent(rs, r.start, 0));
    const uint64_t n_old = t->nb[ti];
    const uint64_t nn = direction > 0 ? 2 * n_old : n_old / 2;
    void* p = nullptr;
    TRY(dev_alloc(t, &p, nn * B * 8, rs));
    if (direction > 0) {
        ProfScope ps(t, DYC_PROF_UPSIZE, rs);
        k_upsize<B><<<grid_for(n_old * B, kThreads * kResU), kThreads, 0, rs>>>(t->sub[ti], (unsigned long long*)p,
                                                                        (uint32_t)n_old, t->a[ti + 1], t->b[ti + 1],
                                                                        fastmod_magic(nn), (uint32_t)nn);
    } else {
        void* r0 = nullptr;
        void* r1 = nullptr;
        dyc_status s = dev_alloc(t, &r0, nn * B * 8, rs);
        if (s == DYC_OK) s = dev_alloc(t, &r1, nn * B * 8, rs);
        if (s != DYC_OK) {
            dev_free(t, p, rs);
            dev_free(t, r0, rs);
            return s;
        }
        r.res[0] = (unsigned long long*)r0;
        r.res[1] = (unsigned long long*)r1;
        CU(cudaMemsetAsync(r.ctr, 0, C_N * 8, rs));
        ProfScope ps(t, DYC_PROF_DOWNSIZE, rs);
        k_downsize<B><<<grid_for(nn * B, kThreads * kResUD), kThreads, 0, rs>>>(t->sub[ti], (unsigned long long*)p,
                                                                       (uint32_t)nn, r.res[0], r.ctr);
    }
    CU(cudaGetLastError());
    CU(cudaEventRecord(r.done, rs));
    t->clean &= ~(1u << ti);        // LK batches may bypass ti's (old) buckets
    r.active = true;
    r.dir = direction;
    r.ti = (uint32_t)ti;
    r.nbuf = (unsigned long long*)p;
    r.nnb = nn;
    return DYC_OK;
}

// After a mutating batch: the alpha loop (Q11), taken against the size
// the table has once the resize in flight is committed; it commits first when
// it has to act.
template <int B>
dyc_status policy_lower(dyc_table* t, cudaStream_t st) {
    TRY(flush_m<B>(t, st));
    if (t->rz.active) {
        if (!((double)t->m < t->cfg.alpha * (double)t->N_after())) return DYC_OK;
        TRY(live_commit<B>(t, st));
    }
    return enforce_lower<B>(t, st);
}

template <int B>
dyc_status launch_apply(dyc_table* t, const unsigned long long* list, bool del, uint64_t n, cudaStream_t st) {
    ProfScope ps(t, DYC_PROF_OTHER, st);
    k_apply<B><<<grid_for(n, kThreads / (B / 4)), kThreads, 0, st>>>(t->view(), list, t->d_ctr + C_DEFER, del);
    CU(cudaGetLastError());
    return DYC_OK;
}

// insert = begin (scratch, counters, FUSE decision) + one k_upsert per chunk of
// the batch + end (resize decision, placement, failures, alpha loop).  Splitting
// the upsert into chunks is invisible to the semantics: every chunk only probes,
// updates and CASes into free slots (or queues to the pending list), and all
// placement with evictions happens once, in insert_end.
//
// While a resize is in flight (NEXT-1) a batch that could need an upsize
// ((m+n) > beta*N_after) commits it first; any other runs the LK upsert against
// the old buffer of the locked subtable and commits only if some of its ops
// need that subtable (deferred updates, keys with no free non-locked slot).
template <int B>
dyc_status insert_begin(dyc_table* t, uint64_t n, cudaStream_t st, bool& fuse) {
    // with lazy counts the live count is at most m + lazy_add: below beta with
    // that bound, below beta for sure; otherwise the decision needs the exact m
    const bool lazy = t->m_lazy || t->ev_pending || t->stash_bound;
    if (lazy && (t->rz.active || (double)(t->m + t->lazy_add + n) > t->cfg.beta * (double)t->N()))
        TRY(flush_m<B>(t, st));
    if (t->rz.active && (double)(t->m + n) > t->cfg.beta * (double)t->N_after()) TRY(live_commit<B>(t, st));
    TRY(ensure_lists(t, n, st));
    // stash capacity: a quarter of the table's slots, 1M..64M pairs (lazy
    // inserts run until their summed sizes would exceed it)
    TRY(ensure_stash(t, std::min<uint64_t>(kStashMax, std::max<uint64_t>(kStashMin, t->N() / 4)), st));
    TRY(zero_ctr(t, st));
    TRY(refresh_weights<B>(t, st));
    t->ins_n = n;
    fuse = t->rz.active || (double)(t->m + t->lazy_add + n) <= t->cfg.beta * (double)t->N();
    return DYC_OK;
}

template <int B>
dyc_status insert_chunk(dyc_table* t, const uint32_t* keys, const uint32_t* vals, uint8_t* status, uint64_t n,
                        bool fuse, cudaStream_t st, const unsigned long long* n_dev = nullptr, unsigned max_grid = 0,
                        const uint32_t* skip1_idx = nullptr) {
    constexpr int U = DYC_UPSERT_U;
    unsigned grid = grid_for(n, (uint64_t)(kThreads / (B / 4)) * U);
    if (max_grid) grid = std::min(grid, max_grid);
    {
        ProfScope ps(t, DYC_PROF_UPSERT, st);
        const bool sp = t->stash_bound != 0;
        const unsigned long long* nd = n_dev;
        unsigned long long* pl = t->list[0];
#define DYC_UPSERT_LAUNCH(FU, LKV, DEFER)                                                                      \
    do {                                                                                                      \
        const uint32_t lk = LKV ? t->rz.ti : 0xFFFFFFFFu;                                                     \
        if (t->weighted) {                                                                                    \
            if (sp) k_upsert<B, FU, U, LKV, true, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, pl, t->d_ctr, lk, DEFER, nd); \
            else k_upsert<B, FU, U, LKV, true, false><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, pl, t->d_ctr, lk, DEFER, nd); \
        } else {                                                                                              \
            if (sp) k_upsert<B, FU, U, LKV, false, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, pl, t->d_ctr, lk, DEFER, nd); \
            else k_upsert<B, FU, U, LKV, false, false><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, pl, t->d_ctr, lk, DEFER, nd); \
        }                                                                                                     \
    } while (0)
        if (skip1_idx)   // staged batches: first-choice bucket known full, key known absent from it
            k_upsert<B, true, U, false, false, false, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, pl,
                                                                                     t->d_ctr, 0xFFFFFFFFu, nullptr, nd,
                                                                                     skip1_idx);
        else if (t->rz.active) DYC_UPSERT_LAUNCH(true, true, t->list[1]);
        else if (fuse) DYC_UPSERT_LAUNCH(true, false, nullptr);
        else DYC_UPSERT_LAUNCH(false, false, nullptr);
#undef DYC_UPSERT_LAUNCH
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

template <int B>
dyc_status insert_end(dyc_table* t, bool fuse, cudaStream_t st) {
    if (t->rz.active) {
        TRY(read_ctr(t, st));
        const uint64_t ins = t->h_ctr[C_INSERTED], pend = t->h_ctr[C_PENDING], dfr = t->h_ctr[C_DEFER];
        t->n_deferred += dfr;
        const uint64_t ev0 = t->n_evict;
        if (pend || dfr) {
            TRY(live_commit<B>(t, st));
            if (dfr) TRY(launch_apply<B>(t, t->list[1], false, dfr, st));
            if (pend) TRY(place_and_settle<B>(t, 0, t->d_ctr + C_PENDING, 0, true, st));
        }
        t->m += ins;
        t->last_new = ins;
        t->last_pending = pend;
        t->n_pending_total += pend;
        t->last_evict = t->n_evict - ev0;
        return policy_lower<B>(t, st);
    }
    uint64_t add_bound = t->ins_n;
    if (!fuse) {
        // the resize decision needs n_new before any placement (Q11)
        TRY(read_ctr(t, st));
        const uint64_t n_new = t->h_ctr[C_INSERTED];
        while ((double)(t->m + n_new) > t->cfg.beta * (double)t->N()) {
            TRY(upsize_table<B>(t, (uint32_t)t->smallest(), st));
            t->n_upsize++;
        }
        TRY(refresh_weights<B>(t, st));   // after an upsize the bigger table draws more
        add_bound = n_new;
    }
    // placement of the keys whose candidate buckets were full.  Lazy when the
    // stash can take every key of the batch: pairs still homeless after L_max
    // hops go to the stash, which every later batch consults and the next
    // exact read-back settles (Q17), so the batch ends without a host
    // wait.  Otherwise (a batch larger than the stash) failures are settled
    // here, synchronously.
    const bool lazy_place = t->stash_bound + add_bound <= t->stash_cap;
    if (!lazy_place) TRY(zero_one(t, C_FAIL, st));
    {
        ProfScope ps(t, DYC_PROF_PLACE, st);
        DYC_PLACE_K(B)<<<t->place_blocks, kThreads, 0, st>>>(t->view(), t->list[0], t->d_ctr + C_PENDING, 0,
                                                         lazy_place ? t->stash : t->list[1], t->d_ctr, !fuse,
                                                         t->d_ctr + (lazy_place ? C_STASH : C_FAIL), true);
    }
    CU(cudaGetLastError());
    t->ins_lazy = true;
    t->lazy_add += add_bound;     // the batch's INSERTED count reaches m at the next read-back
    t->m_lazy = true;
    TRY(mark_lazy(t, st));
    if (lazy_place) {
        t->stash_bound += add_bound;
    } else {
        TRY(read_ctr(t, st));
        const bool stash_nonempty = t->h_ctr[C_STASH] != 0;
        TRY(settle<B>(t, 1, t->h_ctr[C_FAIL], st));
        if (stash_nonempty) TRY(sync_state<B>(t, st));
    }
    // the alpha loop cannot fire while a lower bound of m is >= alpha*N
    if (t->m >= t->lazy_del && (double)(t->m - t->lazy_del) >= t->cfg.alpha * (double)t->N()) return DYC_OK;
    return enforce_lower<B>(t, st);
}

template <int B, int OP>
dyc_status staged_run(dyc_table* t, const uint32_t* keys, const uint32_t* vals, uint8_t* out_st, uint32_t* out_r,
                      uint64_t n, cudaStream_t st);
bool staged_ok(const dyc_table* t, uint64_t n, int op);

template <int B>
dyc_status insert_impl(dyc_table* t, const uint32_t* keys, const uint32_t* vals, uint8_t* status, uint64_t n,
                       cudaStream_t st) {
    bool fuse = false;
    TRY(insert_begin<B>(t, n, st, fuse));
    // a large batch that needs no upsize runs chunk-staged (dyc_staged.cuh)
    if (fuse && staged_ok(t, n, 0) && B == 8) TRY((staged_run<B, 0>(t, keys, vals, status, nullptr, n, st)));
    else TRY(insert_chunk<B>(t, keys, vals, status, n, fuse, st));
    return insert_end<B>(t, fuse, st);
}

template <int B>
dyc_status find_impl(dyc_table* t, const uint32_t* keys, uint32_t* vals, uint8_t* found, uint64_t n,
                     cudaStream_t st, const unsigned long long* n_dev = nullptr, unsigned max_grid = 0,
                     const uint32_t* skip1_idx = nullptr) {
    constexpr int ILP = (B <= 16) ? DYC_FIND_ILP : 2;
    constexpr uint64_t per_block = (uint64_t)(kThreads / (B / 4)) * ILP;   // queries per block per pass
    unsigned grid = grid_for(n, per_block);
    if (max_grid) grid = std::min(grid, max_grid);
    {
        ProfScope ps(t, DYC_PROF_FIND, st);
        if (skip1_idx) k_find<B, ILP, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, found, n, n_dev, skip1_idx);
        else k_find<B, ILP><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, found, n, n_dev);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

// delete = prep (counters; with a resize in flight also the deferred list) +
// one k_delete per chunk + end (m, deferred removals, alpha loop).
template <int B>
dyc_status delete_prep(dyc_table* t, uint64_t n, cudaStream_t st) {
    if (t->rz.active) TRY(flush_m<B>(t, st));
    t->del_n = n;
    if (t->rz.active) {
        TRY(ensure_lists(t, n, st));
        TRY(zero_one(t, C_DEFER, st));
    }
    return DYC_OK;
}

template <int B>
dyc_status delete_chunk(dyc_table* t, const uint32_t* keys, uint32_t* vals, uint8_t* status, uint64_t n,
                        cudaStream_t st, const unsigned long long* n_dev = nullptr, unsigned max_grid = 0,
                        const uint32_t* skip1_idx = nullptr) {
    {
        ProfScope ps(t, DYC_PROF_DELETE, st);
        constexpr int U = DYC_DELETE_U;
        unsigned grid = grid_for(n, (uint64_t)(kThreads / (B / 4)) * U);
        if (max_grid) grid = std::min(grid, max_grid);
        const bool sp = t->stash_bound != 0;
        if (skip1_idx) {
            k_delete<B, U, false, false, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->d_ctr,
                                                                         0xFFFFFFFFu, nullptr, n_dev, skip1_idx);
        } else if (t->rz.active) {
            if (sp) k_delete<B, U, true, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->d_ctr, t->rz.ti, t->list[0], n_dev);
            else k_delete<B, U, true, false><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->d_ctr, t->rz.ti, t->list[0], n_dev);
        } else {
            if (sp) k_delete<B, U, false, true><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->d_ctr, 0xFFFFFFFFu, nullptr, n_dev);
            else k_delete<B, U, false, false><<<grid, kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->d_ctr, 0xFFFFFFFFu, nullptr, n_dev);
        }
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

template <int B>
dyc_status delete_end(dyc_table* t, cudaStream_t st) {
    // no resize in flight and a LOWER bound of m after this batch (m minus
    // every removal that may still be pending, this batch's included) is
    // >= alpha*N: the alpha loop cannot fire, so the removals stay on
    // the device until the next read-back (m_lazy).  m itself is then an upper
    // bound, which is what the beta test of the next insert needs.
    const uint64_t pend = t->lazy_del + t->del_n;
    if (!t->rz.active && t->m >= pend && (double)(t->m - pend) >= t->cfg.alpha * (double)t->N()) {
        if (t->del_n) t->clean = 0;
        TRY(mark_lazy(t, st));
        t->lazy_del = pend;
        t->m_lazy = true;
        return DYC_OK;
    }
    TRY(read_ctr(t, st));   // applies the removals to m
    if (t->rz.active && t->h_ctr[C_DEFER]) {
        const uint64_t dfr = t->h_ctr[C_DEFER];
        t->n_deferred += dfr;
        TRY(live_commit<B>(t, st));
        TRY(launch_apply<B>(t, t->list[0], true, dfr, st));
    }
    return policy_lower<B>(t, st);
}

template <int B>
dyc_status delete_impl(dyc_table* t, const uint32_t* keys, uint32_t* vals, uint8_t* status, uint64_t n,
                       cudaStream_t st) {
    TRY(delete_prep<B>(t, n, st));
    if (staged_ok(t, n, 2) && B == 8) TRY((staged_run<B, 2>(t, keys, nullptr, status, vals, n, st)));
    else TRY(delete_chunk<B>(t, keys, vals, status, n, st));
    return delete_end<B>(t, st);
}

template <int B>
dyc_status find_top(dyc_table* t, const uint32_t* keys, uint32_t* vals, uint8_t* found, uint64_t n, cudaStream_t st) {
    if (staged_ok(t, n, 1) && B == 8) return staged_run<B, 1>(t, keys, nullptr, found, vals, n, st);
    return find_impl<B>(t, keys, vals, found, n, st);
}

// ------------------------------------------------------------------ staged path
// Chunk-staged execution of a large batch (dyc_staged.cuh): used
// for B = 8 when the batch has at least as many ops as the table has buckets
// (auto), or always (DYC_STAGED_FORCE) / never (DYC_STAGED_OFF); never with a
// resize in flight, the paper-weighted placement, or a possibly non-empty
// stash (those keep the direct kernels).
constexpr uint64_t kStagedMinOps = 1ull << 20;

StagedView staged_view(const dyc_table* t) {
    StagedView s{};
    uint32_t c = 0;
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        s.cbase[i] = c;
        c += (uint32_t)((t->nb[i] + kStChunk - 1) / kStChunk);
    }
    s.cbase[t->cfg.d] = c;
    s.nc = c;
    uint32_t s1 = 0;
    while (((uint64_t)c + (1ull << s1) - 1) >> s1 > (uint64_t)kStBins1) s1++;
    s.s1 = s1;
    s.nbins = (uint32_t)(((uint64_t)c + (1ull << s1) - 1) >> s1);
    return s;
}

// op: 0 insert, 1 find, 2 delete.  Automatic choice: inserts and deletes only.
// A staged find decides ~68% of a C2 batch in the chunk pass but must still
// probe the second bucket of the rest; measured slower than k_find alone
// (5.4 vs 3.9 ms at C2, profiles/r2_staged.md), so finds stage only when forced.
bool staged_ok(const dyc_table* t, uint64_t n, int op) {
    if (t->cfg.bucket_slots != 8 || t->weighted || t->rz.active || t->stash_bound || n == 0 || n >= (1ull << 31))
        return false;
    if (t->cfg.flags & DYC_STAGED_OFF) return false;
    const StagedView s = staged_view(t);
    if (s.s1 > (uint32_t)kStMaxS1 || s.nc > kStMaxChunks) return false;
    if (t->cfg.flags & DYC_STAGED_FORCE) return true;
    if (op == 1) return false;
    uint64_t buckets = 0;
    for (uint32_t i = 0; i < t->cfg.d; i++) buckets += t->nb[i];
    return n >= kStagedMinOps && n >= buckets;
}

// Scratch of one staged batch of n ops over nc chunks (u32 arrays of n unless noted):
//   g (first-choice buckets; later the need list), k1 v1 g1 (level-1 order),
//   k2 v2 (level-2 = chunk order), lb2 spos1 spos2 [u16 x n], st1 st2 [u8 x n],
//   run1 / roff1 [tiles1 x 256 u32 / 257 u16], run2 / roff2 [tiles2 x ...],
//   chunk_cnt chunk_off cur2 [nc + 1], bin_off cur1 tile_first [kStBins1 + 1],
//   need_cnt [u64].  The need list's keys / values / results reuse k1 / v1
//   (free after the level-2 scatter), its statuses st1.
struct StagedBufs {
    uint32_t *g, *k1, *v1, *g1, *k2, *v2, *dmap1, *dmap2;
    uint16_t *lb2, *spos1, *spos2;
    uint8_t *st1, *st2;
    uint32_t *chunk_cnt, *chunk_off, *cur2, *bin_off, *cur1, *tile_first, *tile_bin, *tile_lo, *tile_hi;
    unsigned long long* need_cnt;
};

dyc_status staged_bufs(dyc_table* t, uint64_t n, uint32_t nc, uint64_t tiles2, cudaStream_t st, StagedBufs& b) {
    auto al = [](uint64_t x) { return (x + 255) & ~255ull; };
    const uint64_t a4 = al(4 * n), a2 = al(2 * n), a1 = al(n);
    const uint64_t tt = al(4ull * (tiles2 + 1));
    const uint64_t sc = al(4ull * (nc + 1)), sb = al(4ull * (kStBins1 + 1));
    const uint64_t bytes = 8 * a4 + 3 * a2 + 2 * a1 + 3 * tt + 3 * sc + 3 * sb + 256;
    if (bytes > t->stg_cap) {
        dev_free(t, t->stg, st);
        t->stg = nullptr;
        t->stg_cap = 0;
        const uint64_t cap = bytes + bytes / 4;
        TRY(dev_alloc(t, &t->stg, cap, st));
        t->stg_cap = cap;
    }
    char* p = (char*)t->stg;
    auto take = [&](uint64_t sz) { char* q = p; p += sz; return q; };
    b.g = (uint32_t*)take(a4); b.k1 = (uint32_t*)take(a4); b.v1 = (uint32_t*)take(a4); b.g1 = (uint32_t*)take(a4);
    b.k2 = (uint32_t*)take(a4); b.v2 = (uint32_t*)take(a4);
    b.lb2 = (uint16_t*)take(a2); b.spos1 = (uint16_t*)take(a2); b.spos2 = (uint16_t*)take(a2);
    b.st1 = (uint8_t*)take(a1); b.st2 = (uint8_t*)take(a1);
    b.dmap1 = (uint32_t*)take(a4); b.dmap2 = (uint32_t*)take(a4);
    b.tile_bin = (uint32_t*)take(tt); b.tile_lo = (uint32_t*)take(tt); b.tile_hi = (uint32_t*)take(tt);
    b.chunk_cnt = (uint32_t*)take(sc); b.chunk_off = (uint32_t*)take(sc); b.cur2 = (uint32_t*)take(sc);
    b.bin_off = (uint32_t*)take(sb); b.cur1 = (uint32_t*)take(sb); b.tile_first = (uint32_t*)take(sb);
    b.need_cnt = (unsigned long long*)take(256);
    return DYC_OK;
}

// OP 0 insert (keys, vals -> out_st), 1 find (keys -> out_r values, out_st found),
// 2 delete (keys -> out_r old values, out_st status).  Outputs are nullable.
template <int B, int OP>
dyc_status staged_run(dyc_table* t, const uint32_t* keys, const uint32_t* vals, uint8_t* out_st, uint32_t* out_r,
                      uint64_t n, cudaStream_t st) {
    constexpr bool VALS = OP == 0;
    const StagedView sv = staged_view(t);
    const uint64_t tiles1 = (n + kStTile - 1) / kStTile;
    const uint64_t tiles2 = tiles1 + sv.nbins;
    StagedBufs b{};
    TRY(staged_bufs(t, n, sv.nc, tiles2, st, b));
    const uint32_t sm_scatter = (VALS ? 3 : 2) * kStTile * 4 + kStTile;
    // opt-in shared-memory sizes, once per device (function attributes are per device context)
    static std::atomic<uint64_t> attr_devices{0};
    const uint64_t dev_bit = 1ull << (t->device & 63);
    if (!(attr_devices.load() & dev_bit)) {
        CU(cudaFuncSetAttribute(k_st_apply<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kStSlots * 8));
        CU(cudaFuncSetAttribute(k_st_apply<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, kStSlots * 8));
        CU(cudaFuncSetAttribute(k_st_apply<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, kStSlots * 8));
        CU(cudaFuncSetAttribute(k_st_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, kStMaxChunks * 4));
        CU(cudaFuncSetAttribute(k_st_scatter<1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * kStTile * 4 + kStTile));
        CU(cudaFuncSetAttribute(k_st_scatter<2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * kStTile * 4 + kStTile));
        CU(cudaFuncSetAttribute(k_st_scatter<1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * kStTile * 4 + kStTile));
        CU(cudaFuncSetAttribute(k_st_scatter<2, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * kStTile * 4 + kStTile));
        attr_devices.fetch_or(dev_bit);
    }
    t->n_staged++;
    const TableView tv = t->view();
    {
        ProfScope ps(t, DYC_PROF_ST_HIST, st);
        CU(cudaMemsetAsync(b.chunk_cnt, 0, 4ull * (sv.nc + 1), st));
        CU(cudaMemsetAsync(b.need_cnt, 0, 8, st));
        const unsigned per_sm = sv.nc * 4 <= 100u * 1024 ? 2u : 1u;    // two CTAs per SM when both counter sets fit
        k_st_hist<<<t->num_sms * per_sm, kStHistT, sv.nc * 4, st>>>(tv, sv, keys, n, b.g, b.chunk_cnt);
        k_st_scan<<<1, 1024, 0, st>>>(sv, b.chunk_cnt, b.chunk_off, b.cur2, b.bin_off, b.cur1, b.tile_first,
                                      b.tile_bin, b.tile_lo, b.tile_hi);
    }
    {
        ProfScope ps(t, DYC_PROF_ST_SCATTER, st);
        k_st_scatter<1, VALS><<<(unsigned)tiles1, kStT, sm_scatter, st>>>(
            sv, keys, vals, b.g, n, b.tile_first, b.tile_bin, b.tile_lo, b.tile_hi, b.cur1, b.k1, b.v1, b.g1, nullptr,
            b.spos1, b.dmap1);
        k_st_scatter<2, VALS><<<(unsigned)tiles2, kStT, sm_scatter, st>>>(
            sv, b.k1, b.v1, b.g1, n, b.tile_first, b.tile_bin, b.tile_lo, b.tile_hi, b.cur2, b.k2, b.v2, nullptr, b.lb2,
            b.spos2, b.dmap2);
    }
    CU(cudaGetLastError());
    // r2 (sorted 32-bit results of find / delete) lives in v2, which those ops do not carry;
    // the need list reuses g (free after the level-1 scatter)
    uint32_t* r2 = OP == 0 ? nullptr : b.v2;
    uint32_t* need = b.g;
    {
        ProfScope ps(t, DYC_PROF_ST_APPLY, st);
        // the need list: positions in g, keys / values in k1 / v1 (free after the level-2 scatter)
        k_st_apply<OP><<<sv.nc, kStAT, kStSlots * 8, st>>>(tv, sv, b.k2, b.v2, b.lb2, b.chunk_off, b.st2, r2, need,
                                                             b.k1, b.v1, b.need_cnt, t->d_ctr);
    }
    CU(cudaGetLastError());
    // the ops their first-choice bucket could not decide (the need list: keys,
    // values and positions in the chunk order) run through the direct kernel
    // with the first probe skipped, writing their results at those positions
    const unsigned gneed = (unsigned)t->num_sms * 8;
    if (OP == 0) TRY(insert_chunk<B>(t, b.k1, b.v1, b.st2, n, true, st, b.need_cnt, gneed, need));
    else if (OP == 1) TRY(find_impl<B>(t, b.k1, r2, b.st2, n, st, b.need_cnt, gneed, need));
    else TRY(delete_chunk<B>(t, b.k1, r2, b.st2, n, st, b.need_cnt, gneed, need));
    {
        ProfScope ps(t, DYC_PROF_ST_UNPERM, st);
        // back to request order: chunk order -> level-1 order (into st1 / v1) -> caller
        uint32_t* r1 = OP == 0 ? nullptr : b.v1;
        k_st_unperm<2><<<(unsigned)tiles2, kStUT, 0, st>>>(sv, n, b.tile_first, b.tile_bin, b.tile_lo, b.tile_hi,
                                                           b.dmap2, b.spos2, b.st2, r2, b.st1, r1);
        if (out_st || out_r)
            k_st_unperm<1><<<(unsigned)tiles1, kStUT, 0, st>>>(sv, n, b.tile_first, b.tile_bin, b.tile_lo, b.tile_hi,
                                                               b.dmap1, b.spos1, b.st1, r1, out_st, out_r);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

// ------------------------------------------------------------------ host-buffer path
// The batch is staged on the device chunk by chunk: H2D of chunk c+1 (copy-in
// stream) overlaps the kernel of chunk c (the caller's stream) and the D2H of
// chunk c-1 (copy-out stream), so PCIe and HBM work concurrently.
constexpr uint64_t kChunk = 1ull << 22;

struct HostPipe {
    dyc_table* t;
    cudaStream_t st;
    std::vector<cudaEvent_t> evs;
    cudaEvent_t ev() { evs.push_back(t->ev()); return evs.back(); }
    ~HostPipe() { for (auto e : evs) t->ev_pool.push_back(e); }
};

dyc_status ensure_stage(dyc_table* t, uint64_t bytes, cudaStream_t st);

dyc_status ensure_copy_streams(dyc_table* t) {
    if (!t->cp_in) CU(cudaStreamCreateWithFlags(&t->cp_in, cudaStreamNonBlocking));
    if (!t->cp_out) CU(cudaStreamCreateWithFlags(&t->cp_out, cudaStreamNonBlocking));
    return DYC_OK;
}

// copy `bytes_per_op` x len of each input from host to the staging slices, make st wait
dyc_status pipe_in(HostPipe& P, void* const* dst, const void* const* src, const uint64_t* esz, int nin,
                   uint64_t off, uint64_t len) {
    dyc_table* t = P.t;
    for (int q = 0; q < nin; q++)
        CU(cudaMemcpyAsync((char*)dst[q] + off * esz[q], (const char*)src[q] + off * esz[q], len * esz[q],
                           cudaMemcpyHostToDevice, t->cp_in));
    cudaEvent_t e = P.ev();
    CU(cudaEventRecord(e, t->cp_in));
    CU(cudaStreamWaitEvent(P.st, e, 0));
    return DYC_OK;
}

dyc_status pipe_out(HostPipe& P, void* const* dst, const void* const* src, const uint64_t* esz, int nout,
                    uint64_t off, uint64_t len) {
    dyc_table* t = P.t;
    cudaEvent_t e = P.ev();
    CU(cudaEventRecord(e, P.st));
    CU(cudaStreamWaitEvent(t->cp_out, e, 0));
    for (int q = 0; q < nout; q++)
        if (dst[q])
            CU(cudaMemcpyAsync((char*)dst[q] + off * esz[q], (const char*)src[q] + off * esz[q], len * esz[q],
                               cudaMemcpyDeviceToHost, t->cp_out));
    return DYC_OK;
}

template <int B>
dyc_status insert_host_impl(dyc_table* t, const uint32_t* hk, const uint32_t* hv, uint8_t* hs, uint64_t n,
                            cudaStream_t st) {
    TRY(ensure_copy_streams(t));
    TRY(ensure_stage(t, n * 9 + 64, st));
    uint32_t* k = (uint32_t*)t->stage;
    uint32_t* v = k + n;
    uint8_t* s = (uint8_t*)(v + n);
    HostPipe P{t, st, {}};
    bool fuse = false;
    TRY(insert_begin<B>(t, n, st, fuse));
    for (uint64_t off = 0; off < n; off += kChunk) {
        const uint64_t len = std::min(kChunk, n - off);
        void* d_in[2] = {k, v};
        const void* h_in[2] = {hk, hv};
        const uint64_t es[2] = {4, 4};
        TRY(pipe_in(P, d_in, h_in, es, 2, off, len));
        TRY(insert_chunk<B>(t, k + off, v + off, hs ? s + off : nullptr, len, fuse, st));
        void* h_out[1] = {hs};
        const void* d_out[1] = {s};
        const uint64_t eo[1] = {1};
        if (hs) TRY(pipe_out(P, h_out, d_out, eo, 1, off, len));
    }
    TRY(insert_end<B>(t, fuse, st));
    CU(cudaStreamSynchronize(t->cp_out));
    CU(cudaStreamSynchronize(st));
    return DYC_OK;
}

template <int B>
dyc_status find_host_impl(dyc_table* t, const uint32_t* hk, uint32_t* hv, uint8_t* hf, uint64_t n, cudaStream_t st) {
    TRY(ensure_copy_streams(t));
    TRY(ensure_stage(t, n * 9 + 64, st));
    uint32_t* k = (uint32_t*)t->stage;
    uint32_t* v = k + n;
    uint8_t* f = (uint8_t*)(v + n);
    HostPipe P{t, st, {}};
    for (uint64_t off = 0; off < n; off += kChunk) {
        const uint64_t len = std::min(kChunk, n - off);
        void* d_in[1] = {k};
        const void* h_in[1] = {hk};
        const uint64_t es[1] = {4};
        TRY(pipe_in(P, d_in, h_in, es, 1, off, len));
        TRY(find_impl<B>(t, k + off, v + off, hf ? f + off : nullptr, len, st));
        void* h_out[2] = {hv, hf};
        const void* d_out[2] = {v, f};
        const uint64_t eo[2] = {4, 1};
        TRY(pipe_out(P, h_out, d_out, eo, 2, off, len));
    }
    CU(cudaStreamSynchronize(t->cp_out));
    CU(cudaStreamSynchronize(st));
    return DYC_OK;
}

template <int B>
dyc_status delete_host_impl(dyc_table* t, const uint32_t* hk, uint32_t* hv, uint8_t* hs, uint64_t n,
                            cudaStream_t st) {
    TRY(ensure_copy_streams(t));
    TRY(ensure_stage(t, n * 9 + 64, st));
    uint32_t* k = (uint32_t*)t->stage;
    uint32_t* v = k + n;
    uint8_t* s = (uint8_t*)(v + n);
    HostPipe P{t, st, {}};
    TRY(delete_prep<B>(t, n, st));
    for (uint64_t off = 0; off < n; off += kChunk) {
        const uint64_t len = std::min(kChunk, n - off);
        void* d_in[1] = {k};
        const void* h_in[1] = {hk};
        const uint64_t es[1] = {4};
        TRY(pipe_in(P, d_in, h_in, es, 1, off, len));
        TRY(delete_chunk<B>(t, k + off, hv ? v + off : nullptr, hs ? s + off : nullptr, len, st));
        void* h_out[2] = {hv, hs};
        const void* d_out[2] = {v, s};
        const uint64_t eo[2] = {4, 1};
        TRY(pipe_out(P, h_out, d_out, eo, 2, off, len));
    }
    TRY(delete_end<B>(t, st));
    CU(cudaStreamSynchronize(t->cp_out));
    CU(cudaStreamSynchronize(st));
    return DYC_OK;
}

// Baselines (measurement only): reinsert one subtable or everything.
template <int B>
dyc_status reinsert_resize(dyc_table* t, int direction, int ti, bool all, cudaStream_t st) {
    const uint32_t d = t->cfg.d;
    unsigned long long* old[DYC_MAX_D] = {};
    dyc_table::Vm old_vm[DYC_MAX_D];
    uint64_t old_nb[DYC_MAX_D] = {};
    bool touched[DYC_MAX_D] = {};
    for (uint32_t i = 0; i < d; i++) touched[i] = all || (int)i == ti;
    uint64_t live_bound = 0;
    for (uint32_t i = 0; i < d; i++) {
        if (!touched[i]) continue;
        const uint64_t nn = direction > 0 ? 2 * t->nb[i] : t->nb[i] / 2;
        if (nn == 0 || nn > 0xFFFFFFFFull) return set_err(DYC_ERR_INVALID_ARG, "bad subtable size");
        void* p = nullptr;
        TRY(dev_alloc(t, &p, nn * B * 8, st));
        CU(cudaMemsetAsync(p, 0xFF, nn * B * 8, st));
        old[i] = t->sub[i];
        old_vm[i] = t->vm[i];
        t->vm[i] = dyc_table::Vm();
        t->vm_shrink_pending &= ~(1u << i);
        old_nb[i] = t->nb[i];
        t->sub[i] = (unsigned long long*)p;
        t->nb[i] = nn;
        live_bound += old_nb[i] * B;
    }
    TRY(ensure_lists(t, live_bound, st));
    TRY(zero_ctr(t, st));
    const TableView tv = t->view();
    for (uint32_t i = 0; i < d; i++) {
        if (!touched[i]) continue;
        const uint64_t ns = old_nb[i] * B;
        ProfScope ps(t, DYC_PROF_REINSERT, st);
        k_reinsert<B><<<grid_for(ns, kThreads / (B / 4)), kThreads, 0, st>>>(tv, old[i], ns, t->list[1], t->d_ctr);
        CU(cudaGetLastError());
    }
    TRY(read_ctr(t, st));
    const uint64_t nfail = t->h_ctr[C_FAIL];
    for (uint32_t i = 0; i < d; i++)
        if (touched[i]) {
            if (old_vm[i].base) vm_release_range(t, old_vm[i], st);
            else dev_free(t, old[i], st);
        }
    if (nfail) TRY(place_and_settle<B>(t, 1, nullptr, nfail, true, st));
    t->clean = 0;
    return DYC_OK;
}

template <int B>
dyc_status resize_impl(dyc_table* t, int direction, int subtable, int method, cudaStream_t st) {
    TRY(live_commit<B>(t, st));
    TRY(flush_m<B>(t, st));
    if (direction == 0) {
        while ((double)t->m > t->cfg.beta * (double)t->N()) {
            TRY(upsize_table<B>(t, (uint32_t)t->smallest(), st));
            t->n_upsize++;
        }
        return enforce_lower<B>(t, st);
    }
    if (method == DYC_RESIZE_REHASH_ALL) {
        TRY(reinsert_resize<B>(t, direction, -1, true, st));
        if (direction > 0) t->n_upsize++; else t->n_downsize++;
        return DYC_OK;
    }
    int ti = -1;
    TRY(pick_resize(t, direction, subtable, ti));
    if (method == DYC_RESIZE_REINSERT_SUBTABLE) {
        TRY(reinsert_resize<B>(t, direction, ti, false, st));
    } else if (direction > 0) {
        TRY(upsize_table<B>(t, (uint32_t)ti, st));
    } else {
        TRY(downsize_table<B>(t, (uint32_t)ti, st));
    }
    if (direction > 0) t->n_upsize++; else t->n_downsize++;
    return DYC_OK;
}

template <int B>
dyc_status stats_impl(dyc_table* t, dyc_stats_t* out, cudaStream_t st) {
    TRY(live_commit<B>(t, st));
    TRY(flush_m<B>(t, st));        // exact counts, empty stash
    TRY(zero_ctr(t, st));
    const TableView tv = t->view();
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        ProfScope ps(t, DYC_PROF_OTHER, st);
        k_count<B><<<grid_for(t->nb[i] * B, kThreads * 8), kThreads, 0, st>>>(tv, i, t->d_ctr);
        CU(cudaGetLastError());
    }
    TRY(read_ctr(t, st));
    std::memset(out, 0, sizeof(*out));
    out->m = t->m;
    out->N = t->N();
    out->d = t->cfg.d;
    out->B = B;
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        out->buckets[i] = t->nb[i];
        out->count[i] = t->h_ctr[C_COUNT0 + i];
    }
    out->fill = out->N ? (double)out->m / (double)out->N : 0.0;
    out->n_upsize = t->n_upsize;
    out->n_downsize = t->n_downsize;
    out->n_fail_upsize = t->n_fail_upsize;
    out->n_residual = t->n_residual;
    out->n_evict = t->n_evict;
    out->n_place_retry = t->n_place_retry;
    out->n_second_table = t->h_ctr[C_SECOND];
    out->bytes_allocated = out->N * 8 + 2 * t->list_cap * 8 + t->stage_cap + C_N * 8;
    out->bytes_cached = t->cache_bytes;
    out->last_insert_new = t->last_new;
    out->last_insert_pending = t->last_pending;
    out->last_insert_evictions = t->last_evict;
    out->n_live_resize = t->n_live_resize;
    out->n_deferred = t->n_deferred;
    out->n_device_alloc = t->n_device_alloc;
    out->alloc_ms = t->alloc_ms;
    out->n_sync = t->n_sync;
    out->sync_ms = t->sync_ms;
    out->n_pending = t->n_pending_total;
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        if (t->vm[i].base) out->vm_subtables++;
        out->vm_mapped_bytes += t->vm[i].mapped;
    }
    out->n_vm_map = t->n_vm_map;
    out->n_vm_unmap = t->n_vm_unmap;
    out->n_staged = t->n_staged;
    return DYC_OK;
}

template <int B>
dyc_status dump_impl(dyc_table* t, uint64_t* h_kv, uint32_t* h_tab, uint64_t* h_bkt, uint64_t cap, uint64_t* n_out,
                     cudaStream_t st) {
    TRY(live_commit<B>(t, st));
    TRY(flush_m<B>(t, st));
    const uint64_t m = t->m;
    void *kv = nullptr, *tb = nullptr, *bk = nullptr;
    TRY(dev_alloc(t, &kv, m * 8, st));
    TRY(dev_alloc(t, &tb, m * 4, st));
    TRY(dev_alloc(t, &bk, m * 8, st));
    TRY(zero_one(t, C_DUMP, st));
    const TableView tv = t->view();
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        ProfScope ps(t, DYC_PROF_OTHER, st);
        k_dump<B><<<grid_for(t->nb[i] * B, kThreads), kThreads, 0, st>>>(
            tv, i, (unsigned long long*)kv, (uint32_t*)tb, (unsigned long long*)bk, m, t->d_ctr);
        CU(cudaGetLastError());
    }
    TRY(read_ctr(t, st));
    const uint64_t cnt = t->h_ctr[C_DUMP];
    const uint64_t ncopy = std::min(std::min(cnt, m), cap);
    if (ncopy) {
        if (h_kv) CU(cudaMemcpyAsync(h_kv, kv, ncopy * 8, cudaMemcpyDeviceToHost, st));
        if (h_tab) CU(cudaMemcpyAsync(h_tab, tb, ncopy * 4, cudaMemcpyDeviceToHost, st));
        if (h_bkt) CU(cudaMemcpyAsync(h_bkt, bk, ncopy * 8, cudaMemcpyDeviceToHost, st));
    }
    dev_free(t, kv, st);
    dev_free(t, tb, st);
    dev_free(t, bk, st);
    CU(cudaStreamSynchronize(st));
    if (n_out) *n_out = cnt;
    if (cnt != m) return set_err(DYC_ERR_CUDA, "dump found " + std::to_string(cnt) + " live slots, expected " +
                                                   std::to_string(m));
    return DYC_OK;
}

// Mixed batch (reading Q10: finds, then inserts, then deletes).  The ops are
// grouped by op code on the device into fixed regions [c*n, (c+1)*n) of the
// scratch; each phase runs on its region with its count read by the kernels on
// the device, so the grouping costs no host wait and each phase waits only
// when its own resize decision needs the exact live count.  Op codes outside
// 0..2 land in region 3 and get status DYC_OP_NONE.
template <int B>
dyc_status mixed_impl(dyc_table* t, const uint8_t* d_ops, const uint32_t* d_keys, const uint32_t* d_values,
                      uint32_t* d_values_out, uint8_t* d_status, uint64_t n, cudaStream_t st) {
    const uint64_t need = n * (4 * 4 + 4 * 4 + 4 * 4 + 4 + 4) + 256;   // k, v, out v (4n each), status (4n), pos
    if (need > t->mix_cap) {
        if (t->mix) dev_free(t, t->mix, st);
        t->mix = nullptr;
        t->mix_cap = 0;
        TRY(dev_alloc(t, &t->mix, need, st));
        t->mix_cap = need;
    }
    unsigned long long* cnt = (unsigned long long*)t->mix;      // [0..4) counts, [4..8) cursors
    uint32_t* k = (uint32_t*)(cnt + 8);
    uint32_t* v = k + 4 * n;
    uint32_t* ov = v + 4 * n;
    uint32_t* pos = ov + 4 * n;
    uint8_t* sts = (uint8_t*)(pos + n);
    CU(cudaMemsetAsync(cnt, 0, 8 * 8, st));
    {
        ProfScope ps(t, DYC_PROF_OTHER, st);
        const OpDest od{d_ops};
        k_group_count<OpDest><<<std::min<unsigned>(grid_for(n, kThreads * 4), t->num_sms * 8), kThreads,
                                (kThreads / 32) * 4 * 4, st>>>(od, n, 4, cnt);
        k_fixed_bases<<<1, 32, 0, st>>>(cnt + 4, 4, n);
        k_group_scatter<OpDest><<<grid_for(n, (uint64_t)kThreads * kTileItems), kThreads, 4 * 12, st>>>(
            od, d_keys, d_values, n, 4, cnt + 4, k, v, pos);
    }
    CU(cudaGetLastError());
    // phase sizes: bounded by n on the host.  When that bound cannot rule out a
    // resize decision of either phase, read the exact sizes back once,
    // together with the counters (the read-back a decision needs anyway)
    // tighten the bounds with the phase sizes of earlier lazy mixed batches
    // whose asynchronous copies have landed (no wait)
    while (!t->mix_recs.empty()) {
        const dyc_table::MixRec r = t->mix_recs.front();
        const cudaError_t q = cudaEventQuery(r.ev);
        if (q == cudaErrorNotReady) break;
        if (q != cudaSuccess) return cuda_err(q, "cudaEventQuery");
        if (r.epoch == t->sync_epoch) {
            const unsigned long long* h = t->h_mix_ring + 4 * r.slot;
            const uint64_t ei = std::min<uint64_t>(h[1], r.ins_bound), ed = std::min<uint64_t>(h[2], r.del_bound);
            t->lazy_add -= std::min(t->lazy_add, r.ins_bound - ei);
            t->lazy_del -= std::min(t->lazy_del, r.del_bound - ed);
        }
        t->ev_pool.push_back(r.ev);
        t->mix_recs.erase(t->mix_recs.begin());
    }
    uint64_t ni = n, nd = n;
    const bool loose_ok = (double)(t->m + t->lazy_add + n) <= t->cfg.beta * (double)t->N() &&
                          t->m >= t->lazy_del + n &&
                          (double)(t->m - t->lazy_del - n) >= t->cfg.alpha * (double)t->N();
    if (!loose_ok && !t->rz.active) {
        CU(cudaMemcpyAsync(t->h_mix, cnt, 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
        TRY(sync_state<B>(t, st));
        ni = t->h_mix[1];
        nd = t->h_mix[2];
    } else if (t->mix_recs.size() < kMixRing) {
        // copy the sizes back in the background; a later batch tightens the
        // bounds this one adds once the copy has landed
        const int slot = (int)(t->mix_ring_next++ % kMixRing);
        CU(cudaMemcpyAsync(t->h_mix_ring + 4 * slot, cnt, 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
        cudaEvent_t ev = t->ev();
        CU(cudaEventRecord(ev, st));
        t->mix_recs.push_back({slot, ev, t->sync_epoch, n, n, n});
    }
    // phase 1: finds observe the table before the batch
    TRY(find_impl<B>(t, k, ov, sts, n, st, cnt + 0));
    // phase 2: inserts (one batch of ni <= n new keys)
    bool fuse = false;
    TRY(insert_begin<B>(t, ni, st, fuse));
    TRY(insert_chunk<B>(t, k + n, v + n, sts + n, n, fuse, st, cnt + 1));
    TRY(insert_end<B>(t, fuse, st));
    CU(cudaMemsetAsync(ov + n, 0xFF, n * 4, st));
    // phase 3: deletes
    TRY(delete_prep<B>(t, nd, st));
    TRY(delete_chunk<B>(t, k + 2 * n, ov + 2 * n, sts + 2 * n, n, st, cnt + 2));
    TRY(delete_end<B>(t, st));
    // region 3: invalid op codes
    CU(cudaMemsetAsync(ov + 3 * n, 0xFF, n * 4, st));
    CU(cudaMemsetAsync(sts + 3 * n, 0, n, st));
    return dyc_route_unpermute(pos, n, d_values_out ? ov : nullptr, d_status ? sts : nullptr, d_values_out, d_status,
                               st);
}

#define DISPATCH_B(t, CALL)                                                        \
    switch ((t)->cfg.bucket_slots) {                                               \
        case 4: { constexpr int B_ = 4; return CALL; }                             \
        case 8: { constexpr int B_ = 8; return CALL; }                             \
        case 16: { constexpr int B_ = 16; return CALL; }                           \
        case 32: { constexpr int B_ = 32; return CALL; }                           \
        default: return set_err(DYC_ERR_INVALID_ARG, "unsupported bucket_slots");  \
    }

dyc_status live_commit_any(dyc_table* t, cudaStream_t st) { DISPATCH_B(t, live_commit<B_>(t, st)); }

dyc_status check_table(const dyc_table* t) {
    if (!t) return set_err(DYC_ERR_INVALID_ARG, "null table");
    return DYC_OK;
}

dyc_status enter(dyc_table* t, dyc_stream_t s) {
    TRY(check_table(t));
    CU(cudaSetDevice(t->device));
    t->last = S(s);
    return DYC_OK;
}

dyc_status ensure_stage(dyc_table* t, uint64_t bytes, cudaStream_t st) {
    if (bytes <= t->stage_cap) return DYC_OK;
    if (t->stage) dev_free(t, t->stage, st);
    t->stage = nullptr;
    t->stage_cap = 0;
    TRY(dev_alloc(t, &t->stage, bytes, st));
    t->stage_cap = bytes;
    return DYC_OK;
}

}  // namespace

// ============================================================================ C ABI
extern "C" {

const char* dyc_last_error(void) { return g_err.c_str(); }
const char* dyc_version(void) { return "dycuckoo-b200 0.1 (sm_100a)"; }

dyc_status dyc_config_default(dyc_config* cfg) {
    if (!cfg) return set_err(DYC_ERR_INVALID_ARG, "null cfg");
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->d = 4;
    cfg->bucket_slots = 8;   // 64-byte buckets read by 2-lane groups
    cfg->alpha = 0.3;
    cfg->beta = 0.85;
    cfg->init_capacity = 4096;
    cfg->seed = 0x5EED0001ull;
    cfg->max_hops = 64;
    cfg->flags = 0;          // in-place resizing is opt-in (measured slower here: DESIGN.md §5)
    return DYC_OK;
}

dyc_status dyc_create_ex(const dyc_config* cfg, dyc_table** out) {
    if (!cfg || !out) return set_err(DYC_ERR_INVALID_ARG, "null argument");
    *out = nullptr;
    const uint32_t d = cfg->d, B = cfg->bucket_slots;
    if (d < 2 || d > DYC_MAX_D) return set_err(DYC_ERR_INVALID_ARG, "d must be in 2..16");
    if (B != 4 && B != 8 && B != 16 && B != 32) return set_err(DYC_ERR_INVALID_ARG, "bucket_slots must be 4, 8, 16 or 32");
    if (!(cfg->alpha > 0.0 && cfg->alpha < cfg->beta && cfg->beta < 1.0))
        return set_err(DYC_ERR_INVALID_ARG, "need 0 < alpha < beta < 1");
    if (cfg->alpha > cfg->beta * (double)d / (double)(d + 1))
        return set_err(DYC_ERR_INVALID_ARG, "need alpha <= beta*d/(d+1) (P:L315-318)");
    if (cfg->max_hops < 1) return set_err(DYC_ERR_INVALID_ARG, "max_hops must be >= 1");
    if (cfg->flags & ~(uint32_t)(DYC_PLACE_PAPER_WEIGHTED | DYC_RESIZE_IN_PLACE | DYC_STAGED_OFF | DYC_STAGED_FORCE))
        return set_err(DYC_ERR_INVALID_ARG, "flags: only DYC_PLACE_PAPER_WEIGHTED | DYC_RESIZE_IN_PLACE | "
                                            "DYC_STAGED_OFF | DYC_STAGED_FORCE are defined");
    if ((cfg->flags & DYC_STAGED_OFF) && (cfg->flags & DYC_STAGED_FORCE))
        return set_err(DYC_ERR_INVALID_ARG, "flags: DYC_STAGED_OFF and DYC_STAGED_FORCE exclude each other");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_err(DYC_ERR_NO_DEVICE, "no CUDA device");
    }
    dyc_table* t = new dyc_table();
    t->cfg = *cfg;
    cudaGetDevice(&t->device);
    cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, t->device);
    // persistent k_place grid: exactly one wave of the instance this table
    // launches (the register count, hence the residency, depends on B)
    int occ = 0;
    switch (cfg->bucket_slots) {
        case 4: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_place<4>, kThreads, 0); break;
        case 8: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_place<8>, kThreads, 0); break;
        case 16: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_place<16>, kThreads, 0); break;
        default: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_place<32>, kThreads, 0); break;
    }
    t->place_blocks = t->num_sms * std::max(1, occ);
    uint64_t st = cfg->seed;
    for (uint32_t s = 0; s < d + 2; s++) {
        t->a[s] = (uint32_t)(1 + splitmix64(st) % (kP - 1));   // a_s in [1, p)
        t->b[s] = (uint32_t)(splitmix64(st) % kP);             // b_s in [0, p)
    }
    uint64_t per = (cfg->init_capacity + (uint64_t)d * B - 1) / ((uint64_t)d * B);   // Q13
    if (per < 1) per = 1;
    if (per > 0xFFFFFFFFull) {
        dyc_destroy(t);
        return set_err(DYC_ERR_INVALID_ARG, "init_capacity too large");
    }
    dyc_status s = DYC_OK;
    t->in_place = (cfg->flags & DYC_RESIZE_IN_PLACE) != 0 && vmm_api().ok;
    if (t->in_place) {
        CUmemAllocationProp prop{};
        prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
        prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        prop.location.id = t->device;
        size_t g = 0;
        if (vmm_api().granularity(&g, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || g == 0)
            t->in_place = false;
        t->vm_gran = g;
    }
    for (uint32_t i = 0; i < d && s == DYC_OK; i++) {
        void* p = nullptr;
        if (vm_create(t, i, per * B * 8)) p = (void*)t->vm[i].base;
        else s = dev_alloc(t, &p, per * B * 8, nullptr);
        if (s == DYC_OK) {
            t->sub[i] = (unsigned long long*)p;
            t->nb[i] = per;
            if (cudaMemsetAsync(p, 0xFF, per * B * 8, nullptr) != cudaSuccess) s = cuda_err(cudaGetLastError(), "memset");
        }
    }
    if (s == DYC_OK && cudaMalloc(&t->d_ctr, C_N * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMalloc");
    // C_REMOVED is only ever zeroed by read_ctr after it applies the count
    if (s == DYC_OK && cudaMemset(t->d_ctr, 0, C_N * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMemset");
    if (s == DYC_OK && cudaMalloc(&t->d_probe, 6 * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMalloc");
    if (s == DYC_OK && cudaMemset(t->d_probe, 0, 6 * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMemset");
    t->weighted = (cfg->flags & DYC_PLACE_PAPER_WEIGHTED) != 0;
    if (s == DYC_OK && cudaMalloc(&t->d_w, DYC_MAX_D * sizeof(float)) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMalloc");
    if (s == DYC_OK && cudaMemset(t->d_w, 0, DYC_MAX_D * sizeof(float)) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMemset");
    t->clean = (1u << d) - 1u;      // an empty table satisfies the invariant
    if (s == DYC_OK && cudaMallocHost(&t->h_ctr, C_N * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMallocHost");
    if (s == DYC_OK && cudaMallocHost(&t->h_mix, 4 * 8) != cudaSuccess) s = cuda_err(cudaGetLastError(), "cudaMallocHost");
    if (s == DYC_OK && cudaMallocHost(&t->h_mix_ring, kMixRing * 4 * 8) != cudaSuccess)
        s = cuda_err(cudaGetLastError(), "cudaMallocHost");
    if (s == DYC_OK && cudaDeviceSynchronize() != cudaSuccess) s = cuda_err(cudaGetLastError(), "create");
    if (s != DYC_OK) {
        dyc_destroy(t);
        return s;
    }
    *out = t;
    return DYC_OK;
}

dyc_status dyc_create(uint32_t d, uint64_t init_capacity, double alpha, double beta, dyc_table** out) {
    dyc_config c;
    dyc_config_default(&c);
    c.d = d;
    c.init_capacity = init_capacity;
    c.alpha = alpha;
    c.beta = beta;
    return dyc_create_ex(&c, out);
}

dyc_status dyc_destroy(dyc_table* t) {
    if (!t) return DYC_OK;
    cudaSetDevice(t->device);
    cudaDeviceSynchronize();
    for (uint32_t i = 0; i < DYC_MAX_D; i++) vm_release(t, i, nullptr);
    for (auto& kv : t->live) cudaFree(kv.first);   // subtables, lists, staging, scratch
    t->live.clear();
    trim_cache(t);
    if (t->d_ctr) cudaFree(t->d_ctr);
    if (t->d_probe) cudaFree(t->d_probe);
    if (t->d_w) cudaFree(t->d_w);
    if (t->rz.ctr) cudaFree(t->rz.ctr);
    if (t->rz.start) cudaEventDestroy(t->rz.start);
    if (t->rz.done) cudaEventDestroy(t->rz.done);
    if (t->lazy_ev) cudaEventDestroy(t->lazy_ev);
    if (t->h_ctr) cudaFreeHost(t->h_ctr);
    if (t->h_mix) cudaFreeHost(t->h_mix);
    if (t->h_mix_ring) cudaFreeHost(t->h_mix_ring);
    for (auto& r : t->mix_recs) cudaEventDestroy(r.ev);
    if (t->cp_in) cudaStreamDestroy(t->cp_in);
    if (t->cp_out) cudaStreamDestroy(t->cp_out);
    cudaDeviceSynchronize();
    for (auto& r : t->recs) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    for (auto e : t->ev_pool) cudaEventDestroy(e);
    delete t;
    return DYC_OK;
}

dyc_status dyc_insert_batch(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_values, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!d_keys || !d_values) return set_err(DYC_ERR_INVALID_ARG, "null keys/values");
    DISPATCH_B(t, insert_impl<B_>(t, d_keys, d_values, d_status, n, S(stream)));
}

dyc_status dyc_insert_begin(dyc_table* t, uint64_t n_total, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op) return set_err(DYC_ERR_INVALID_ARG, "a batch is already open");
    t->part_op = 1;
    t->part_left = n_total;
    bool fuse = false;
    dyc_status s;
    switch (t->cfg.bucket_slots) {
        case 4: s = insert_begin<4>(t, n_total, S(stream), fuse); break;
        case 8: s = insert_begin<8>(t, n_total, S(stream), fuse); break;
        case 16: s = insert_begin<16>(t, n_total, S(stream), fuse); break;
        default: s = insert_begin<32>(t, n_total, S(stream), fuse); break;
    }
    t->part_fuse = fuse;
    if (s != DYC_OK) t->part_op = 0;
    return s;
}

dyc_status dyc_insert_part(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_values, uint8_t* d_status,
                           uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op != 1) return set_err(DYC_ERR_INVALID_ARG, "no insert batch open");
    if (n > t->part_left) return set_err(DYC_ERR_INVALID_ARG, "parts exceed n_total");
    if (n == 0) return DYC_OK;
    t->part_left -= n;
    DISPATCH_B(t, insert_chunk<B_>(t, d_keys, d_values, d_status, n, t->part_fuse, S(stream)));
}

dyc_status dyc_insert_end(dyc_table* t, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op != 1) return set_err(DYC_ERR_INVALID_ARG, "no insert batch open");
    t->part_op = 0;
    DISPATCH_B(t, insert_end<B_>(t, t->part_fuse, S(stream)));
}

dyc_status dyc_delete_begin(dyc_table* t, uint64_t n_total, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op) return set_err(DYC_ERR_INVALID_ARG, "a batch is already open");
    t->part_op = 2;
    t->part_left = n_total;
    DISPATCH_B(t, delete_prep<B_>(t, n_total, S(stream)));
}

dyc_status dyc_delete_part(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out, uint8_t* d_status,
                           uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op != 2) return set_err(DYC_ERR_INVALID_ARG, "no delete batch open");
    if (n > t->part_left) return set_err(DYC_ERR_INVALID_ARG, "parts exceed n_total");
    if (n == 0) return DYC_OK;
    t->part_left -= n;
    DISPATCH_B(t, delete_chunk<B_>(t, d_keys, d_values_out, d_status, n, S(stream)));
}

dyc_status dyc_delete_end(dyc_table* t, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op != 2) return set_err(DYC_ERR_INVALID_ARG, "no delete batch open");
    t->part_op = 0;
    DISPATCH_B(t, delete_end<B_>(t, S(stream)));
}

dyc_status dyc_find_batch(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out, uint8_t* d_found, uint64_t n,
                          dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!d_keys || !d_values_out) return set_err(DYC_ERR_INVALID_ARG, "null keys/values_out");
    DISPATCH_B(t, find_top<B_>(t, d_keys, d_values_out, d_found, n, S(stream)));
}

dyc_status dyc_delete_batch(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!d_keys) return set_err(DYC_ERR_INVALID_ARG, "null keys");
    DISPATCH_B(t, delete_impl<B_>(t, d_keys, d_values_out, d_status, n, S(stream)));
}

dyc_status dyc_mixed_batch(dyc_table* t, const uint8_t* d_ops, const uint32_t* d_keys, const uint32_t* d_values,
                           uint32_t* d_values_out, uint8_t* d_status, uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!d_ops || !d_keys) return set_err(DYC_ERR_INVALID_ARG, "null ops/keys");
    if (n > 0xFFFFFFFFull / 4) return set_err(DYC_ERR_INVALID_ARG, "mixed batch must be < 2^30 ops");
    DISPATCH_B(t, mixed_impl<B_>(t, d_ops, d_keys, d_values, d_values_out, d_status, n, S(stream)));
}

dyc_status dyc_resize_ex(dyc_table* t, int direction, int subtable, int method, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (direction < -1 || direction > 1 || method < 0 || method > 2)
        return set_err(DYC_ERR_INVALID_ARG, "bad direction/method");
    DISPATCH_B(t, resize_impl<B_>(t, direction, subtable, method, S(stream)));
}

dyc_status dyc_resize(dyc_table* t, int direction, int subtable, dyc_stream_t stream) {
    return dyc_resize_ex(t, direction, subtable, DYC_RESIZE_SPLIT, stream);
}

dyc_status dyc_resize_begin(dyc_table* t, int direction, int subtable, dyc_stream_t stream,
                            dyc_stream_t resize_stream) {
    TRY(enter(t, stream));
    if (direction != 1 && direction != -1) return set_err(DYC_ERR_INVALID_ARG, "direction must be +1 or -1");
    DISPATCH_B(t, live_begin<B_>(t, direction, subtable, S(stream), S(resize_stream)));
}

dyc_status dyc_resize_commit(dyc_table* t, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->part_op) return set_err(DYC_ERR_INVALID_ARG, "a batch is open (dyc_*_end first)");
    DISPATCH_B(t, live_commit<B_>(t, S(stream)));
}

dyc_status dyc_resize_query(const dyc_table* t, int* in_flight, int* kernel_done) {
    TRY(check_table(t));
    if (in_flight) *in_flight = t->rz.active ? 1 : 0;
    if (kernel_done) {
        *kernel_done = 1;
        if (t->rz.active) {
            const cudaError_t e = cudaEventQuery(t->rz.done);
            if (e == cudaErrorNotReady) *kernel_done = 0;
            else if (e != cudaSuccess) return cuda_err(e, "cudaEventQuery");
        }
    }
    return DYC_OK;
}

dyc_status dyc_clear(dyc_table* t, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (t->rz.active) TRY(live_commit_any(t, S(stream)));
    for (uint32_t i = 0; i < t->cfg.d; i++)
        CU(cudaMemsetAsync(t->sub[i], 0xFF, t->nb[i] * t->cfg.bucket_slots * 8, S(stream)));
    // the counts still on the device are read (statistics) and the stash is
    // discarded with the rest of the contents
    if (t->m_lazy || t->ev_pending) TRY(read_ctr(t, S(stream)));
    CU(cudaMemsetAsync(t->d_ctr + C_STASH, 0, sizeof(unsigned long long), S(stream)));
    t->stash_bound = 0;
    t->m = 0;
    t->clean = (1u << t->cfg.d) - 1u;
    return DYC_OK;
}

dyc_status dyc_trim(dyc_table* t) {
    TRY(check_table(t));
    CU(cudaSetDevice(t->device));
    if (t->stg) {                     // staged-batch scratch (dyc_staged.cuh)
        dev_free(t, t->stg, t->last);
        t->stg = nullptr;
        t->stg_cap = 0;
    }
    trim_cache(t);
    return DYC_OK;
}

dyc_status dyc_stats(dyc_table* t, dyc_stats_t* out, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (!out) return set_err(DYC_ERR_INVALID_ARG, "null out");
    DISPATCH_B(t, stats_impl<B_>(t, out, S(stream)));
}

dyc_status dyc_shape(const dyc_table* t, uint64_t* buckets, uint64_t* m_lo, uint64_t* m_hi, uint64_t* n_fail_upsize) {
    TRY(check_table(t));
    if (buckets)
        for (uint32_t i = 0; i < t->cfg.d; i++) buckets[i] = t->nb[i];
    if (m_lo) *m_lo = t->m >= t->lazy_del ? t->m - t->lazy_del : 0;
    if (m_hi) *m_hi = t->m + t->lazy_add;
    if (n_fail_upsize) *n_fail_upsize = t->n_fail_upsize;
    return DYC_OK;
}

dyc_status dyc_dump(dyc_table* t, uint64_t* h_kv, uint32_t* h_table, uint64_t* h_bucket, uint64_t cap,
                    uint64_t* n_out, dyc_stream_t stream) {
    TRY(enter(t, stream));
    DISPATCH_B(t, dump_impl<B_>(t, h_kv, h_table, h_bucket, cap, n_out, S(stream)));
}

dyc_status dyc_hash_params(const dyc_table* t, uint64_t* a, uint64_t* b) {
    TRY(check_table(t));
    for (uint32_t s = 0; s < t->cfg.d + 2; s++) {
        if (a) a[s] = t->a[s];
        if (b) b[s] = t->b[s];
    }
    return DYC_OK;
}

dyc_status dyc_hash_probe(dyc_table* t, const uint32_t* d_keys, uint64_t n, uint32_t* d_x, uint32_t* d_pair,
                          dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    {
        ProfScope ps(t, DYC_PROF_OTHER, S(stream));
        k_hash_probe<<<grid_for(n, 128), 128, 0, S(stream)>>>(t->view(), d_keys, n, d_x, d_pair);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_insert_batch_host(dyc_table* t, const uint32_t* h_keys, const uint32_t* h_values, uint8_t* h_status,
                                 uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!h_keys || !h_values) return set_err(DYC_ERR_INVALID_ARG, "null keys/values");
    DISPATCH_B(t, insert_host_impl<B_>(t, h_keys, h_values, h_status, n, S(stream)));
}

dyc_status dyc_find_batch_host(dyc_table* t, const uint32_t* h_keys, uint32_t* h_values_out, uint8_t* h_found,
                               uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!h_keys || !h_values_out) return set_err(DYC_ERR_INVALID_ARG, "null keys/values_out");
    DISPATCH_B(t, find_host_impl<B_>(t, h_keys, h_values_out, h_found, n, S(stream)));
}

dyc_status dyc_delete_batch_host(dyc_table* t, const uint32_t* h_keys, uint32_t* h_values_out, uint8_t* h_status,
                                 uint64_t n, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (n == 0) return DYC_OK;
    if (!h_keys) return set_err(DYC_ERR_INVALID_ARG, "null keys");
    DISPATCH_B(t, delete_host_impl<B_>(t, h_keys, h_values_out, h_status, n, S(stream)));
}

uint64_t dyc_launch_count(const dyc_table* t, int reset) {
    if (!t) return 0;
    uint64_t c = t->launches;
    if (reset) const_cast<dyc_table*>(t)->launches = 0;
    return c;
}

dyc_status dyc_profile_enable(dyc_table* t, int enable) {
    TRY(check_table(t));
    for (auto& r : t->recs) { t->ev_pool.push_back(r.a); t->ev_pool.push_back(r.b); }
    t->recs.clear();
    for (int k = 0; k < DYC_PROF_KINDS; k++) { t->prof_ms[k] = 0; t->prof_calls[k] = 0; }
    t->prof = enable != 0;
    return DYC_OK;
}

dyc_status dyc_probe_count_enable(dyc_table* t, int enable) {
    TRY(check_table(t));
    CU(cudaSetDevice(t->device));
    CU(cudaMemset(t->d_probe, 0, 6 * 8));
    t->count_probes = enable != 0;
    return DYC_OK;
}

dyc_status dyc_probe_count_read(dyc_table* t, uint64_t* out6) {
    TRY(check_table(t));
    if (!out6) return set_err(DYC_ERR_INVALID_ARG, "null out");
    CU(cudaSetDevice(t->device));
    CU(cudaDeviceSynchronize());
    CU(cudaMemcpy(out6, t->d_probe, 6 * 8, cudaMemcpyDeviceToHost));
    CU(cudaMemset(t->d_probe, 0, 6 * 8));
    return DYC_OK;
}

dyc_status dyc_clean_mask(const dyc_table* t, uint32_t* mask) {
    TRY(check_table(t));
    if (!mask) return set_err(DYC_ERR_INVALID_ARG, "null out");
    *mask = t->rz.active ? (t->clean & ~(1u << t->rz.ti)) : t->clean;
    return DYC_OK;
}

dyc_status dyc_profile_read(dyc_table* t, double* ms, uint64_t* calls) {
    TRY(check_table(t));
    for (auto& r : t->recs) {
        CU(cudaEventSynchronize(r.b));
        float x = 0.f;
        CU(cudaEventElapsedTime(&x, r.a, r.b));
        t->prof_ms[r.kind] += x;
        t->prof_calls[r.kind]++;
        t->ev_pool.push_back(r.a);
        t->ev_pool.push_back(r.b);
    }
    t->recs.clear();
    for (int k = 0; k < DYC_PROF_KINDS; k++) {
        if (ms) ms[k] = t->prof_ms[k];
        if (calls) calls[k] = t->prof_calls[k];
    }
    return DYC_OK;
}

dyc_status dyc_route_count(dyc_table* t, const uint32_t* d_keys, uint64_t n, uint32_t world, uint64_t* d_counts,
                           dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (world < 1 || world > 1024) return set_err(DYC_ERR_INVALID_ARG, "world must be 1..1024");
    CU(cudaMemsetAsync(d_counts, 0, world * 8, S(stream)));
    if (n == 0) return DYC_OK;
    const uint32_t sh = t->cfg.d + 1;
    {
        ProfScope ps(t, DYC_PROF_OTHER, S(stream));
        const HashDest hd{t->a[sh], t->b[sh], world, fastmod_magic(world), d_keys};
        k_group_count<HashDest><<<std::min<unsigned>(grid_for(n, kThreads * 4), t->num_sms * 8), kThreads,
                                  (kThreads / 32) * world * 4,
                                  S(stream)>>>(hd, n, world, (unsigned long long*)d_counts);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_route_scatter(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_vals_in,
                             const uint8_t* d_tags_in, uint64_t n, uint32_t world, const uint64_t* d_counts,
                             uint64_t* d_cursor, uint32_t* d_keys_out, uint32_t* d_vals_out, uint8_t* d_tags_out,
                             uint32_t* d_pos, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (world < 1 || world > 1024) return set_err(DYC_ERR_INVALID_ARG, "world must be 1..1024");
    if (n == 0) return DYC_OK;
    if (n > 0xFFFFFFFFull) return set_err(DYC_ERR_INVALID_ARG, "route batch must be < 2^32 ops");
    const uint32_t sh = t->cfg.d + 1;
    {
        ProfScope ps(t, DYC_PROF_OTHER, S(stream));
        k_route_offsets<<<1, 32, 0, S(stream)>>>((const unsigned long long*)d_counts, world,
                                                 (unsigned long long*)d_cursor);
    }
    {
        ProfScope ps(t, DYC_PROF_OTHER, S(stream));
        const HashDest hd{t->a[sh], t->b[sh], world, fastmod_magic(world), d_keys};
        k_group_scatter<HashDest><<<grid_for(n, (uint64_t)kThreads * kTileItems), kThreads, world * 12,
                                    S(stream)>>>(hd, d_keys, d_vals_in, n, world, (unsigned long long*)d_cursor,
                                                 d_keys_out, d_vals_out, d_pos, d_tags_in,
                                                 d_tags_in ? d_tags_out : nullptr);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_route_unpermute(const uint32_t* d_pos, uint64_t n, const uint32_t* d_reply_vals,
                               const uint8_t* d_reply_status, uint32_t* d_vals, uint8_t* d_status,
                               dyc_stream_t stream) {
    if (n == 0) return DYC_OK;
    k_route_unpermute<<<grid_for(n, kThreads * 4), kThreads, 0, S(stream)>>>(d_pos, n, d_reply_vals, d_reply_status,
                                                                        d_vals, d_status);
    CU(cudaGetLastError());
    return DYC_OK;
}

// ---------------------------------------------- peer-memory routing (fused)
dyc_status dyc_ipc_alloc(uint64_t bytes, void** d_ptr) {
    if (!d_ptr || bytes == 0) return set_err(DYC_ERR_INVALID_ARG, "dyc_ipc_alloc: null out pointer or 0 bytes");
    *d_ptr = nullptr;
    cudaError_t e = cudaMalloc(d_ptr, bytes);
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        return set_err(DYC_ERR_OOM, "dyc_ipc_alloc: out of device memory");
    }
    CU(e);
    CU(cudaMemset(*d_ptr, 0, bytes));
    return DYC_OK;
}

dyc_status dyc_ipc_free(void* d_ptr) {
    if (d_ptr) CU(cudaFree(d_ptr));
    return DYC_OK;
}

dyc_status dyc_ipc_get_handle(void* d_ptr, void* handle64) {
    if (!d_ptr || !handle64) return set_err(DYC_ERR_INVALID_ARG, "dyc_ipc_get_handle: null pointer");
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "CUDA IPC handle is 64 bytes");
    cudaIpcMemHandle_t h;
    CU(cudaIpcGetMemHandle(&h, d_ptr));
    memcpy(handle64, &h, 64);
    return DYC_OK;
}

dyc_status dyc_ipc_open(const void* handle64, void** d_ptr) {
    if (!d_ptr || !handle64) return set_err(DYC_ERR_INVALID_ARG, "dyc_ipc_open: null pointer");
    cudaIpcMemHandle_t h;
    memcpy(&h, handle64, 64);
    CU(cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess));
    return DYC_OK;
}

dyc_status dyc_ipc_close(void* d_ptr) {
    if (d_ptr) CU(cudaIpcCloseMemHandle(d_ptr));
    return DYC_OK;
}

dyc_status dyc_route_push(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_vals, const uint8_t* d_tags,
                          uint64_t n, uint32_t world, uint32_t src_rank, void* const* d_recv,
                          uint64_t* const* d_recv_count, uint64_t recv_cap, dyc_stream_t stream) {
    TRY(enter(t, stream));
    if (world < 1 || world > kMaxPeers) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_push: world must be 1..64");
    if (src_rank >= world) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_push: src_rank >= world");
    if (!d_recv || !d_recv_count) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_push: null peer arrays");
    if (n > 0xFFFFFFFFull) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_push: batch must be < 2^32 ops");
    if (n == 0) return DYC_OK;
    PeerPtrs rp{}, cp{};
    for (uint32_t w = 0; w < world; w++) {
        if (!d_recv[w] || !d_recv_count[w]) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_push: null peer pointer");
        rp.p[w] = d_recv[w];
        cp.p[w] = d_recv_count[w];
    }
    const uint32_t sh = t->cfg.d + 1;
    {
        ProfScope ps(t, DYC_PROF_OTHER, S(stream));
        const HashDest hd{t->a[sh], t->b[sh], world, fastmod_magic(world), d_keys};
        k_route_push<<<std::min<unsigned>(grid_for(n, (uint64_t)kThreads * kPushItems), t->num_sms * DYC_PUSH_BPS), kThreads,
                       0, S(stream)>>>(hd, d_vals, d_tags, n, world, src_rank, rp, cp, recv_cap);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_route_reply(const void* d_recv, uint64_t recv_cap, uint64_t n, const uint32_t* d_vals,
                           const uint8_t* d_status, uint32_t world, uint32_t* const* d_out_vals,
                           uint8_t* const* d_out_status, dyc_stream_t stream) {
    if (world < 1 || world > kMaxPeers) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: world must be 1..64");
    if (n == 0) return DYC_OK;
    if (!d_recv) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: null receive buffer");
    if (n > recv_cap) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: n > recv_cap");
    if ((d_vals == nullptr) != (d_out_vals == nullptr) || (d_status == nullptr) != (d_out_status == nullptr))
        return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: a result array and its destinations must both be given");
    PeerPtrs vp{}, sp{};
    for (uint32_t w = 0; w < world; w++) {
        if (d_out_vals) {
            if (!d_out_vals[w]) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: null peer pointer");
            vp.p[w] = d_out_vals[w];
        }
        if (d_out_status) {
            if (!d_out_status[w]) return set_err(DYC_ERR_INVALID_ARG, "dyc_route_reply: null peer pointer");
            sp.p[w] = d_out_status[w];
        }
    }
    const unsigned long long* meta = (const unsigned long long*)((const char*)d_recv + 8 * recv_cap);
    k_route_reply<<<grid_for(n, kThreads * 4), kThreads, 0, S(stream)>>>(meta, n, d_vals, d_status, vp, sp);
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_set_l2_fetch_granularity(uint32_t bytes) {
    if (bytes > 128) return set_err(DYC_ERR_INVALID_ARG, "granularity must be 0..128");
    CU(cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, bytes));
    return DYC_OK;
}

dyc_status dyc_get_l2_fetch_granularity(uint32_t* bytes) {
    size_t v = 0;
    CU(cudaDeviceGetLimit(&v, cudaLimitMaxL2FetchGranularity));
    if (bytes) *bytes = (uint32_t)v;
    return DYC_OK;
}

dyc_status dyc_bench_gather_ex(void* d_buf, uint64_t buf_bytes, uint64_t n_reads, uint32_t bytes_per_read,
                               uint64_t seed, uint32_t flags, uint64_t* d_sink, dyc_stream_t stream) {
    if (bytes_per_read != 32 && bytes_per_read != 64 && bytes_per_read != 128 && bytes_per_read != 256)
        return set_err(DYC_ERR_INVALID_ARG, "bytes_per_read must be 32, 64, 128 or 256");
    if (flags & ~7u) return set_err(DYC_ERR_INVALID_ARG, "flags: DYC_GATHER_WRITE (1) | DYC_GATHER_CAS (2) | DYC_GATHER_SECTOR (4)");
    const int wmode = (flags & 4u) ? 3 : (flags & 2u) ? 2 : (flags & 1u) ? 1 : 0;
    const uint64_t units = buf_bytes / bytes_per_read;
    if (units == 0) return set_err(DYC_ERR_INVALID_ARG, "buffer too small");
    const uint64_t lanes_per_read = bytes_per_read / 32;
    const unsigned grid = grid_for(n_reads * lanes_per_read, (uint64_t)kThreads * 4);
    unsigned long long* buf = (unsigned long long*)d_buf;
    unsigned long long* sink = (unsigned long long*)d_sink;
#define DYC_GATHER(BB)                                                                                    \
    switch (wmode) {                                                                                      \
        case 0: k_gather<BB, 0><<<grid, kThreads, 0, S(stream)>>>(buf, units, n_reads, seed, sink); break; \
        case 1: k_gather<BB, 1><<<grid, kThreads, 0, S(stream)>>>(buf, units, n_reads, seed, sink); break; \
        case 2: k_gather<BB, 2><<<grid, kThreads, 0, S(stream)>>>(buf, units, n_reads, seed, sink); break; \
        default: k_gather<BB, 3><<<grid, kThreads, 0, S(stream)>>>(buf, units, n_reads, seed, sink); break; \
    }
    switch (bytes_per_read) {
        case 32: DYC_GATHER(4); break;
        case 64: DYC_GATHER(8); break;
        case 128: DYC_GATHER(16); break;
        default: DYC_GATHER(32); break;
    }
#undef DYC_GATHER
    CU(cudaGetLastError());
    return DYC_OK;
}

dyc_status dyc_bench_gather(const void* d_buf, uint64_t buf_bytes, uint64_t n_reads, uint32_t bytes_per_read,
                            uint64_t seed, uint64_t* d_sink, dyc_stream_t stream) {
    return dyc_bench_gather_ex(const_cast<void*>(d_buf), buf_bytes, n_reads, bytes_per_read, seed, 0, d_sink,
                               stream);
}

}  // extern "C"

// ---------------------------------------------------------------- wide-key table (NEXT-3)
#include "dyw_api.cuh"
