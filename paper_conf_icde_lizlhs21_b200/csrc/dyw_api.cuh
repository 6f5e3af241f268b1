// dyw_api.cuh — host control and C ABI of the wide-key table (include/dycuckoo_wide.h,
// SURVEY §8(f) NEXT-3).  Included at the end of dyc_api.cu (one translation
// unit: it shares the error helpers).  The policy is the 32-bit table's
// (Q11-Q13, Q17, Q17b, Q29), written for the wide layouts.
#include "dycuckoo_wide.h"
#include "dyw_kernels.cuh"

#ifndef DYW_U
#define DYW_U 4   // ops per lane group in flight in find / upsert / delete
#endif
#ifndef DYW_U_CAS
#define DYW_U_CAS 2   // ... in the LOCKFREE upsert, whose CAS128 rounds lose to more in flight (measured U = 1/2/4)
#endif

struct dyw_table {
    dyw_config cfg{};
    int L = dyw::SEP;     // layout
    int B = 16;           // slots per bucket
    int W = 2;            // value words
    int device = 0, num_sms = 148;
    dyw::u64* keys[DYC_MAX_D] = {};
    dyw::u64* vals[DYC_MAX_D] = {};
    uint32_t* locks[DYC_MAX_D] = {};
    uint64_t nb[DYC_MAX_D] = {};
    uint32_t a[DYC_MAX_D + 2] = {}, b[DYC_MAX_D + 2] = {}, c[DYC_MAX_D + 2] = {};
    uint64_t m = 0;
    dyw::KVList list[2] = {{nullptr, nullptr}, {nullptr, nullptr}};
    uint64_t list_cap = 0;
    dyw::u64* d_ctr = nullptr;
    dyw::u64* h_ctr = nullptr;
    uint64_t n_upsize = 0, n_downsize = 0, n_fail_upsize = 0, n_residual = 0, n_evict = 0, n_lock_fail = 0;
    uint64_t last_new = 0, last_pending = 0, launches = 0;

    uint64_t N() const {
        uint64_t s = 0;
        for (uint32_t t = 0; t < cfg.d; t++) s += nb[t] * B;
        return s;
    }
    int smallest() const {
        int best = 0;
        for (uint32_t t = 1; t < cfg.d; t++)
            if (nb[t] < nb[best]) best = (int)t;
        return best;
    }
    int largest() const {
        int best = (int)cfg.d - 1;
        for (int t = (int)cfg.d - 2; t >= 0; t--)
            if (nb[t] > nb[best]) best = t;
        return best;
    }
    dyw::WSub sub(uint32_t t) const {
        return dyw::WSub{keys[t], vals[t], locks[t], fastmod_magic(nb[t]), (uint32_t)nb[t], 0};
    }
    dyw::WView view() const {
        dyw::WView v{};
        for (uint32_t t = 0; t < cfg.d; t++) v.sub[t] = sub(t);
        for (uint32_t s = 0; s < cfg.d + 2; s++) { v.a[s] = a[s]; v.b[s] = b[s]; v.c[s] = c[s]; }
        v.d = cfg.d;
        v.d2 = cfg.d * (cfg.d - 1);
        v.magic_d2 = fastmod_magic(v.d2);
        v.dm1 = cfg.d - 1;
        v.max_hops = cfg.max_hops;
        return v;
    }
    uint64_t key_words_per_slot() const { return L == dyw::PACK ? 2 : 1; }
};

namespace {

using dyw::u64;

dyc_status w_read_ctr(dyw_table* t, cudaStream_t st) {
    CU(cudaMemcpyAsync(t->h_ctr, t->d_ctr, dyw::W_N * 8, cudaMemcpyDeviceToHost, st));
    CU(cudaStreamSynchronize(st));
    return DYC_OK;
}

dyc_status w_zero(dyw_table* t, int idx, int cnt, cudaStream_t st) {
    CU(cudaMemsetAsync(t->d_ctr + idx, 0, (size_t)cnt * 8, st));
    return DYC_OK;
}

// Allocates one subtable of n buckets (keys EMPTY, locks 0).
dyc_status w_alloc_sub(dyw_table* t, uint64_t n, u64** k, u64** v, uint32_t** l, cudaStream_t st) {
    *k = nullptr; *v = nullptr; *l = nullptr;
    const uint64_t slots = n * t->B;
    CU(cudaMallocAsync((void**)k, slots * t->key_words_per_slot() * 8, st));
    CU(cudaMemsetAsync(*k, 0xFF, slots * t->key_words_per_slot() * 8, st));
    if (t->L == dyw::SEP) {
        CU(cudaMallocAsync((void**)v, slots * t->W * 8, st));
        CU(cudaMallocAsync((void**)l, n * 4, st));
        CU(cudaMemsetAsync(*l, 0, n * 4, st));
    }
    return DYC_OK;
}

void w_free_sub(u64* k, u64* v, uint32_t* l, cudaStream_t st) {
    if (k) cudaFreeAsync(k, st);
    if (v) cudaFreeAsync(v, st);
    if (l) cudaFreeAsync(l, st);
}

dyc_status w_ensure_lists(dyw_table* t, uint64_t n, cudaStream_t st) {
    if (n <= t->list_cap) return DYC_OK;
    const uint64_t cap = std::max<uint64_t>(n, 2 * t->list_cap);
    for (int i = 0; i < 2; i++) {
        if (t->list[i].keys) cudaFreeAsync(t->list[i].keys, st);
        if (t->list[i].vals) cudaFreeAsync(t->list[i].vals, st);
        t->list[i] = {nullptr, nullptr};
    }
    t->list_cap = 0;
    for (int i = 0; i < 2; i++) {
        CU(cudaMallocAsync((void**)&t->list[i].keys, cap * 8, st));
        CU(cudaMallocAsync((void**)&t->list[i].vals, cap * t->W * 8, st));
    }
    t->list_cap = cap;
    return DYC_OK;
}

// Persistent grid of exactly one wave for kernel `k` (its residency depends on
// its register count; a grid past one wave leaves a partial second wave).
template <class K>
unsigned w_one_wave(K k, int sms) {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, dyw::kThreads, 0);
    return (unsigned)(sms * std::max(1, occ));
}

template <int L, int W>
dyc_status w_launch_place(dyw_table* t, const dyw::KVList& src, const u64* d_count, uint64_t h_count,
                          const dyw::KVList& fail, cudaStream_t st) {
    t->launches++;
    if (L == dyw::PACK) {
        if (W == 1) {
            static const unsigned g = w_one_wave(dyw::k_wplace_lockfree, t->num_sms);
            dyw::k_wplace_lockfree<<<g, dyw::kThreads, 0, st>>>(t->view(), src, d_count, h_count, fail, t->d_ctr);
        }
    } else if (t->cfg.mode == DYW_MODE_VOTER) {
        static const unsigned g = w_one_wave(dyw::k_wplace_voter<W>, t->num_sms);
        dyw::k_wplace_voter<W><<<g, dyw::kThreads, 0, st>>>(t->view(), src, d_count, h_count, fail, t->d_ctr);
    } else {
        static const unsigned g = w_one_wave(dyw::k_wplace_grouped<W>, t->num_sms);
        dyw::k_wplace_grouped<W><<<g, dyw::kThreads, 0, st>>>(t->view(), src, d_count, h_count, fail, t->d_ctr);
    }
    CU(cudaGetLastError());
    return DYC_OK;
}

template <int L, int W>
dyc_status w_upsize(dyw_table* t, uint32_t ti, cudaStream_t st) {
    const uint64_t n_old = t->nb[ti], n_new = 2 * n_old;
    if (n_new > 0xFFFFFFFFull) return set_err(DYC_ERR_OOM, "subtable would exceed 2^32 buckets");
    u64 *k, *v;
    uint32_t* l;
    TRY(w_alloc_sub(t, n_new, &k, &v, &l, st));
    dyw::WSub nw{k, v, l, fastmod_magic(n_new), (uint32_t)n_new, 0};
    t->launches++;
    dyw::k_wupsize<L, W><<<grid_for(n_old * dyw::Lay<L>::B, dyw::kThreads), dyw::kThreads, 0, st>>>(
        t->sub(ti), nw, (uint32_t)n_old, t->a[ti + 1], t->b[ti + 1], t->c[ti + 1]);
    CU(cudaGetLastError());
    w_free_sub(t->keys[ti], t->vals[ti], t->locks[ti], st);
    t->keys[ti] = k; t->vals[ti] = v; t->locks[ti] = l;
    t->nb[ti] = n_new;
    return DYC_OK;
}

// Retries nfail homeless records in list[cur]: a plain retry, then
// failure-triggered upsizes (Q17).
template <int L, int W>
dyc_status w_settle(dyw_table* t, int cur, uint64_t nfail, cudaStream_t st) {
    int round = 0;
    while (nfail > 0) {
        if (round > 0) {
            TRY((w_upsize<L, W>(t, (uint32_t)t->smallest(), st)));
            t->n_fail_upsize++;
        }
        round++;
        TRY(w_zero(t, dyw::W_FAIL, 2, st));          // W_FAIL, W_EVICT
        TRY((w_launch_place<L, W>(t, t->list[cur], nullptr, nfail, t->list[1 - cur], st)));
        TRY(w_read_ctr(t, st));
        t->n_evict += t->h_ctr[dyw::W_EVICT];
        t->n_lock_fail += t->h_ctr[dyw::W_LOCKFAIL];
        nfail = t->h_ctr[dyw::W_FAIL];
        cur = 1 - cur;
        if (round > 64) return set_err(DYC_ERR_INSERT_FAILED, "placement kept failing after 64 upsizes");
    }
    return DYC_OK;
}

template <int L, int W>
dyc_status w_downsize(dyw_table* t, uint32_t ti, cudaStream_t st) {
    const uint64_t n_old = t->nb[ti], h = n_old / 2;
    if (n_old < 2 || (n_old & 1)) return set_err(DYC_ERR_INVALID_ARG, "subtable cannot be halved");
    TRY(w_ensure_lists(t, h * dyw::Lay<L>::B + 1, st));
    u64 *k, *v;
    uint32_t* l;
    TRY(w_alloc_sub(t, h, &k, &v, &l, st));
    dyw::WSub nw{k, v, l, fastmod_magic(h), (uint32_t)h, 0};
    TRY(w_zero(t, dyw::W_FAIL, 7, st));               // W_FAIL .. W_RES_TOTAL
    t->launches++;
    dyw::k_wdownsize<L, W><<<grid_for(h * dyw::Lay<L>::B, dyw::kThreads), dyw::kThreads, 0, st>>>(
        t->sub(ti), nw, (uint32_t)h, t->list[0], t->d_ctr);
    CU(cudaGetLastError());
    w_free_sub(t->keys[ti], t->vals[ti], t->locks[ti], st);
    t->keys[ti] = k; t->vals[ti] = v; t->locks[ti] = l;
    t->nb[ti] = h;
    // residuals go to the other table of their pair (separate kernel, Q16)
    TRY((w_launch_place<L, W>(t, t->list[0], t->d_ctr + dyw::W_RESIDUAL, 0, t->list[1], st)));
    TRY(w_read_ctr(t, st));
    t->n_evict += t->h_ctr[dyw::W_EVICT];
    t->n_lock_fail += t->h_ctr[dyw::W_LOCKFAIL];
    t->n_residual += t->h_ctr[dyw::W_RES_TOTAL];
    t->n_downsize++;
    return w_settle<L, W>(t, 1, t->h_ctr[dyw::W_FAIL], st);
}

template <int L, int W>
dyc_status w_enforce_lower(dyw_table* t, cudaStream_t st) {
    for (;;) {
        const uint64_t N = t->N();
        if (!((double)t->m < t->cfg.alpha * (double)N)) break;
        const int ti = t->largest();
        if (t->nb[ti] < 2 || (t->nb[ti] & 1)) break;
        const uint64_t N_after = N - (t->nb[ti] / 2) * t->B;
        if ((double)t->m > t->cfg.beta * (double)N_after) break;
        const uint64_t f0 = t->n_fail_upsize;
        TRY((w_downsize<L, W>(t, (uint32_t)ti, st)));
        if (t->n_fail_upsize != f0) break;            // Q17b
    }
    return DYC_OK;
}

template <int L, int W>
dyc_status w_insert(dyw_table* t, const u64* keys, const u64* vals, uint8_t* status, uint64_t n, cudaStream_t st) {
    TRY(w_ensure_lists(t, n, st));
    TRY(w_zero(t, 0, dyw::W_N, st));
    const bool fuse = L == dyw::PACK && (double)(t->m + n) <= t->cfg.beta * (double)t->N();
    constexpr int QPW = 32 / dyw::Lay<L>::B, U = L == dyw::PACK ? DYW_U_CAS : DYW_U;
    const unsigned grid = grid_for(n, (uint64_t)(dyw::kThreads / 32) * QPW * U);
    t->launches++;
    if constexpr (L == dyw::PACK) {
        if (fuse)
            dyw::k_wupsert<L, W, true, U><<<grid, dyw::kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->list[0],
                                                                          t->d_ctr);
        else
            dyw::k_wupsert<L, W, false, U><<<grid, dyw::kThreads, 0, st>>>(t->view(), keys, vals, status, n,
                                                                           t->list[0], t->d_ctr);
    } else {                                      // lock modes: every new key goes through placement
        dyw::k_wupsert<L, W, false, U><<<grid, dyw::kThreads, 0, st>>>(t->view(), keys, vals, status, n, t->list[0],
                                                                       t->d_ctr);
    }
    CU(cudaGetLastError());
    TRY(w_read_ctr(t, st));
    const uint64_t n_new = t->h_ctr[dyw::W_INSERTED], pend = t->h_ctr[dyw::W_PENDING];
    if (!fuse)
        while ((double)(t->m + n_new) > t->cfg.beta * (double)t->N()) {   // P:L305, Q11
            TRY((w_upsize<L, W>(t, (uint32_t)t->smallest(), st)));
            t->n_upsize++;
        }
    t->last_new = n_new;
    t->last_pending = pend;
    if (pend) {
        TRY(w_zero(t, dyw::W_FAIL, 2, st));
        TRY((w_launch_place<L, W>(t, t->list[0], nullptr, pend, t->list[1], st)));
        TRY(w_read_ctr(t, st));
        t->n_evict += t->h_ctr[dyw::W_EVICT];
        t->n_lock_fail += t->h_ctr[dyw::W_LOCKFAIL];
        TRY((w_settle<L, W>(t, 1, t->h_ctr[dyw::W_FAIL], st)));
    }
    t->m += n_new;
    return w_enforce_lower<L, W>(t, st);
}

template <int L, int W>
dyc_status w_find(dyw_table* t, const u64* keys, u64* out, uint8_t* found, uint64_t n, cudaStream_t st) {
    constexpr int QPW = 32 / dyw::Lay<L>::B, U = DYW_U;
    t->launches++;
    dyw::k_wfind<L, W, U><<<grid_for(n, (uint64_t)(dyw::kThreads / 32) * QPW * U), dyw::kThreads, 0, st>>>(
        t->view(), keys, out, found, n);
    CU(cudaGetLastError());
    return DYC_OK;
}

template <int L, int W>
dyc_status w_delete(dyw_table* t, const u64* keys, u64* out, uint8_t* status, uint64_t n, cudaStream_t st) {
    constexpr int QPW = 32 / dyw::Lay<L>::B, U = DYW_U;
    TRY(w_zero(t, dyw::W_REMOVED, 1, st));
    t->launches++;
    dyw::k_wdelete<L, W, U><<<grid_for(n, (uint64_t)(dyw::kThreads / 32) * QPW * U), dyw::kThreads, 0, st>>>(
        t->view(), keys, out, status, n, t->d_ctr);
    CU(cudaGetLastError());
    TRY(w_read_ctr(t, st));
    t->m -= t->h_ctr[dyw::W_REMOVED];
    return w_enforce_lower<L, W>(t, st);
}

template <int L, int W>
dyc_status w_resize(dyw_table* t, int direction, int subtable, cudaStream_t st) {
    if (direction == 0) {
        while ((double)t->m > t->cfg.beta * (double)t->N()) {
            TRY((w_upsize<L, W>(t, (uint32_t)t->smallest(), st)));
            t->n_upsize++;
        }
        return w_enforce_lower<L, W>(t, st);
    }
    int ti = subtable;
    if (direction > 0) {
        if (ti < 0) ti = t->smallest();
        if (ti >= (int)t->cfg.d || t->nb[ti] != t->nb[t->smallest()])
            return set_err(DYC_ERR_INVALID_ARG, "only a smallest subtable may be doubled (P:L311-312)");
        TRY((w_upsize<L, W>(t, (uint32_t)ti, st)));
        t->n_upsize++;
    } else {
        if (ti < 0) ti = t->largest();
        if (ti >= (int)t->cfg.d || t->nb[ti] != t->nb[t->largest()])
            return set_err(DYC_ERR_INVALID_ARG, "only a largest subtable may be halved (P:L311-312)");
        TRY((w_downsize<L, W>(t, (uint32_t)ti, st)));
    }
    CU(cudaStreamSynchronize(st));
    return DYC_OK;
}

template <int L, int W>
dyc_status w_stats(dyw_table* t, dyw_stats_t* out, cudaStream_t st) {
    TRY(w_zero(t, dyw::W_COUNT0, DYC_MAX_D, st));
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        t->launches++;
        dyw::k_wcount<L><<<grid_for(t->nb[i] * t->B, dyw::kThreads * 8), dyw::kThreads, 0, st>>>(
            t->sub(i), t->d_ctr + dyw::W_COUNT0 + i);
        CU(cudaGetLastError());
    }
    TRY(w_read_ctr(t, st));
    std::memset(out, 0, sizeof(*out));
    out->m = t->m;
    out->N = t->N();
    out->d = t->cfg.d;
    out->B = t->B;
    out->W = t->W;
    out->mode = t->cfg.mode;
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        out->buckets[i] = t->nb[i];
        out->count[i] = t->h_ctr[dyw::W_COUNT0 + i];
    }
    out->fill = out->N ? (double)out->m / (double)out->N : 0.0;
    out->n_upsize = t->n_upsize;
    out->n_downsize = t->n_downsize;
    out->n_fail_upsize = t->n_fail_upsize;
    out->n_residual = t->n_residual;
    out->n_evict = t->n_evict;
    out->n_lock_fail = t->n_lock_fail;
    out->last_insert_new = t->last_new;
    out->last_insert_pending = t->last_pending;
    out->bytes_allocated = out->N * 8 * (t->key_words_per_slot() + (t->L == dyw::SEP ? t->W : 0)) +
                           (t->L == dyw::SEP ? out->N / t->B * 4 : 0) + 2 * t->list_cap * 8 * (1 + t->W);
    return DYC_OK;
}

template <int L, int W>
dyc_status w_dump(dyw_table* t, uint64_t* hk, uint64_t* hv, uint32_t* htab, uint64_t* hbkt, uint64_t cap,
                  uint64_t* n_out, cudaStream_t st) {
    const uint64_t m = std::max<uint64_t>(t->m, 1);
    u64 *k = nullptr, *v = nullptr, *bk = nullptr;
    uint32_t* tb = nullptr;
    CU(cudaMallocAsync((void**)&k, m * 8, st));
    CU(cudaMallocAsync((void**)&v, m * W * 8, st));
    CU(cudaMallocAsync((void**)&tb, m * 4, st));
    CU(cudaMallocAsync((void**)&bk, m * 8, st));
    TRY(w_zero(t, dyw::W_DUMP, 1, st));
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        t->launches++;
        dyw::k_wdump<L, W><<<grid_for(t->nb[i] * t->B, dyw::kThreads), dyw::kThreads, 0, st>>>(
            t->sub(i), i, k, v, tb, bk, m, t->d_ctr + dyw::W_DUMP);
        CU(cudaGetLastError());
    }
    TRY(w_read_ctr(t, st));
    const uint64_t cnt = t->h_ctr[dyw::W_DUMP];
    const uint64_t nc = std::min(std::min(cnt, t->m), cap);
    if (nc) {
        if (hk) CU(cudaMemcpyAsync(hk, k, nc * 8, cudaMemcpyDeviceToHost, st));
        if (hv) CU(cudaMemcpyAsync(hv, v, nc * W * 8, cudaMemcpyDeviceToHost, st));
        if (htab) CU(cudaMemcpyAsync(htab, tb, nc * 4, cudaMemcpyDeviceToHost, st));
        if (hbkt) CU(cudaMemcpyAsync(hbkt, bk, nc * 8, cudaMemcpyDeviceToHost, st));
    }
    cudaFreeAsync(k, st);
    cudaFreeAsync(v, st);
    cudaFreeAsync(tb, st);
    cudaFreeAsync(bk, st);
    CU(cudaStreamSynchronize(st));
    if (n_out) *n_out = cnt;
    if (cnt != t->m)
        return set_err(DYC_ERR_CUDA, "dump found " + std::to_string(cnt) + " live slots, expected " + std::to_string(t->m));
    return DYC_OK;
}

#define DISPATCH_WIDE(t, CALL)                                                                  \
    do {                                                                                        \
        if ((t)->L == dyw::PACK) { constexpr int L_ = dyw::PACK, W_ = 1; return CALL; }         \
        switch ((t)->W) {                                                                       \
            case 1: { constexpr int L_ = dyw::SEP, W_ = 1; return CALL; }                       \
            case 2: { constexpr int L_ = dyw::SEP, W_ = 2; return CALL; }                       \
            default: { constexpr int L_ = dyw::SEP, W_ = 4; return CALL; }                      \
        }                                                                                       \
    } while (0)

dyc_status w_enter(dyw_table* t) {
    if (!t) return set_err(DYC_ERR_INVALID_ARG, "null table");
    CU(cudaSetDevice(t->device));
    return DYC_OK;
}

}  // namespace

extern "C" {

dyc_status dyw_config_default(dyw_config* cfg) {
    if (!cfg) return set_err(DYC_ERR_INVALID_ARG, "null cfg");
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->d = 4;
    cfg->value_words = 2;
    cfg->mode = DYW_MODE_VOTER;
    cfg->max_hops = 64;
    cfg->alpha = 0.3;
    cfg->beta = 0.85;
    cfg->init_capacity = 4096;
    cfg->seed = 0x5EED0001ull;
    return DYC_OK;
}

dyc_status dyw_destroy(dyw_table* t) {
    if (!t) return DYC_OK;
    cudaSetDevice(t->device);
    cudaDeviceSynchronize();
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        if (t->keys[i]) cudaFree(t->keys[i]);
        if (t->vals[i]) cudaFree(t->vals[i]);
        if (t->locks[i]) cudaFree(t->locks[i]);
    }
    for (int i = 0; i < 2; i++) {
        if (t->list[i].keys) cudaFree(t->list[i].keys);
        if (t->list[i].vals) cudaFree(t->list[i].vals);
    }
    if (t->d_ctr) cudaFree(t->d_ctr);
    if (t->h_ctr) cudaFreeHost(t->h_ctr);
    delete t;
    return DYC_OK;
}

dyc_status dyw_create(const dyw_config* cfg, dyw_table** out) {
    if (!cfg || !out) return set_err(DYC_ERR_INVALID_ARG, "null argument");
    *out = nullptr;
    const uint32_t d = cfg->d, W = cfg->value_words;
    if (d < 2 || d > DYC_MAX_D) return set_err(DYC_ERR_INVALID_ARG, "d must be in 2..16");
    if (cfg->mode > DYW_MODE_LOCKFREE) return set_err(DYC_ERR_INVALID_ARG, "unknown mode");
    if (cfg->mode == DYW_MODE_LOCKFREE ? W != 1 : (W != 1 && W != 2 && W != 4))
        return set_err(DYC_ERR_INVALID_ARG, "value_words must be 1, 2 or 4 (LOCKFREE: 1)");
    if (!(cfg->alpha > 0.0 && cfg->alpha < cfg->beta && cfg->beta < 1.0))
        return set_err(DYC_ERR_INVALID_ARG, "need 0 < alpha < beta < 1");
    if (cfg->alpha > cfg->beta * (double)d / (double)(d + 1))
        return set_err(DYC_ERR_INVALID_ARG, "need alpha <= beta*d/(d+1) (P:L315-318)");
    if (cfg->max_hops < 1) return set_err(DYC_ERR_INVALID_ARG, "max_hops must be >= 1");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_err(DYC_ERR_NO_DEVICE, "no CUDA device");
    }
    dyw_table* t = new dyw_table();
    t->cfg = *cfg;
    t->L = cfg->mode == DYW_MODE_LOCKFREE ? dyw::PACK : dyw::SEP;
    t->B = t->L == dyw::PACK ? 8 : 16;
    t->W = (int)W;
    cudaGetDevice(&t->device);
    cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, t->device);
    uint64_t s = cfg->seed;
    for (uint32_t i = 0; i < d + 2; i++) {            // the 32-bit table's draws (Q1) ...
        t->a[i] = (uint32_t)(1 + splitmix64(s) % (kP - 1));
        t->b[i] = (uint32_t)(splitmix64(s) % kP);
    }
    for (uint32_t i = 0; i < d + 2; i++) t->c[i] = (uint32_t)(1 + splitmix64(s) % (kP - 1));   // ... then c_s (Q33)
    uint64_t per = (cfg->init_capacity + (uint64_t)d * t->B - 1) / ((uint64_t)d * t->B);       // Q13
    if (per < 1) per = 1;
    if (per > 0xFFFFFFFFull) {
        delete t;
        return set_err(DYC_ERR_INVALID_ARG, "init_capacity too large");
    }
    dyc_status st = DYC_OK;
    for (uint32_t i = 0; i < d && st == DYC_OK; i++) {
        st = w_alloc_sub(t, per, &t->keys[i], &t->vals[i], &t->locks[i], nullptr);
        t->nb[i] = per;
    }
    if (st == DYC_OK && cudaMalloc(&t->d_ctr, dyw::W_N * 8) != cudaSuccess) st = cuda_err(cudaGetLastError(), "cudaMalloc");
    if (st == DYC_OK && cudaMallocHost(&t->h_ctr, dyw::W_N * 8) != cudaSuccess)
        st = cuda_err(cudaGetLastError(), "cudaMallocHost");
    if (st == DYC_OK && cudaDeviceSynchronize() != cudaSuccess) st = cuda_err(cudaGetLastError(), "create");
    if (st != DYC_OK) {
        dyw_destroy(t);
        return st;
    }
    *out = t;
    return DYC_OK;
}

dyc_status dyw_insert_batch(dyw_table* t, const uint64_t* d_keys, const uint64_t* d_values, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream) {
    TRY(w_enter(t));
    if (n == 0) return DYC_OK;
    if (!d_keys || !d_values) return set_err(DYC_ERR_INVALID_ARG, "null keys/values");
    DISPATCH_WIDE(t, (w_insert<L_, W_>(t, (const u64*)d_keys, (const u64*)d_values, d_status, n, S(stream))));
}

dyc_status dyw_find_batch(dyw_table* t, const uint64_t* d_keys, uint64_t* d_values_out, uint8_t* d_found,
                          uint64_t n, dyc_stream_t stream) {
    TRY(w_enter(t));
    if (n == 0) return DYC_OK;
    if (!d_keys || !d_values_out) return set_err(DYC_ERR_INVALID_ARG, "null keys/values_out");
    DISPATCH_WIDE(t, (w_find<L_, W_>(t, (const u64*)d_keys, (u64*)d_values_out, d_found, n, S(stream))));
}

dyc_status dyw_delete_batch(dyw_table* t, const uint64_t* d_keys, uint64_t* d_values_out, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream) {
    TRY(w_enter(t));
    if (n == 0) return DYC_OK;
    if (!d_keys) return set_err(DYC_ERR_INVALID_ARG, "null keys");
    DISPATCH_WIDE(t, (w_delete<L_, W_>(t, (const u64*)d_keys, (u64*)d_values_out, d_status, n, S(stream))));
}

dyc_status dyw_resize(dyw_table* t, int direction, int subtable, dyc_stream_t stream) {
    TRY(w_enter(t));
    if (direction < -1 || direction > 1) return set_err(DYC_ERR_INVALID_ARG, "bad direction");
    DISPATCH_WIDE(t, (w_resize<L_, W_>(t, direction, subtable, S(stream))));
}

dyc_status dyw_clear(dyw_table* t, dyc_stream_t stream) {
    TRY(w_enter(t));
    for (uint32_t i = 0; i < t->cfg.d; i++) {
        CU(cudaMemsetAsync(t->keys[i], 0xFF, t->nb[i] * t->B * t->key_words_per_slot() * 8, S(stream)));
        if (t->locks[i]) CU(cudaMemsetAsync(t->locks[i], 0, t->nb[i] * 4, S(stream)));
    }
    t->m = 0;
    return DYC_OK;
}

dyc_status dyw_stats(dyw_table* t, dyw_stats_t* out, dyc_stream_t stream) {
    TRY(w_enter(t));
    if (!out) return set_err(DYC_ERR_INVALID_ARG, "null out");
    DISPATCH_WIDE(t, (w_stats<L_, W_>(t, out, S(stream))));
}

dyc_status dyw_dump(dyw_table* t, uint64_t* h_keys, uint64_t* h_values, uint32_t* h_table, uint64_t* h_bucket,
                    uint64_t cap, uint64_t* n_out, dyc_stream_t stream) {
    TRY(w_enter(t));
    DISPATCH_WIDE(t, (w_dump<L_, W_>(t, h_keys, h_values, h_table, h_bucket, cap, n_out, S(stream))));
}

dyc_status dyw_hash_probe(dyw_table* t, const uint64_t* d_keys, uint64_t n, uint32_t* d_x, uint32_t* d_pair,
                          dyc_stream_t stream) {
    TRY(w_enter(t));
    if (n == 0) return DYC_OK;
    t->launches++;
    dyw::k_whash_probe<<<grid_for(n, 256), 256, 0, S(stream)>>>(t->view(), (const u64*)d_keys, n, d_x, d_pair);
    CU(cudaGetLastError());
    return DYC_OK;
}

uint64_t dyw_launch_count(dyw_table* t, int reset) {
    if (!t) return 0;
    const uint64_t n = t->launches;
    if (reset) t->launches = 0;
    return n;
}

}  // extern "C"
