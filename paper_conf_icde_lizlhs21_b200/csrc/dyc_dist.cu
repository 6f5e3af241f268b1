// dyc_dist.cu — hash-partitioned DyCuckoo across processes (one per GPU) and
// local virtual shards, behind the C ABI (include/dycuckoo.h, dyc_dist_*).
//
// SURVEY §8(e) / DESIGN.md §7.  G = world * local_shards shards; key k belongs
// to shard s(k) = x_{d+1}(k) mod G (the (d+1)-th universal hash of P:L271,
// independent of the pair and bucket hashes), held by rank s / local_shards.
// Every shard is a complete DyCuckoo (its own d subtables and [alpha, beta]
// resizing); ops on different keys never interact (P:L464 batch
// model, keys distinct within a batch), so the union of the shards has exactly
// the single-table semantics.
//
// One batch (every rank calls the same op in the same order, n may differ):
//   dyc_route_count + dyc_route_scatter (kernels): group the ops by shard
//   NCCL: exchange the per-shard counts (world * local_shards u64 per rank)
//   host: one read-back of the counts (the only host wait of the routing)
//   NCCL: grouped ncclSend/ncclRecv of keys [values, op codes], one pair per
//         (peer, local shard), received shard-major so that every local shard's
//         ops are contiguous
//   owner: one ordinary batch per local shard (the single-table path, its own
//          resize decisions)
//   NCCL: the replies travel back into the send layout
//   dyc_route_unpermute (kernel): results in request order.
// With world == 1 and no NCCL id nothing is exchanged: the grouped send buffer
// already is the shard-major receive buffer of the local shards.  With an id
// and world == 1 the exchange runs through NCCL to self (tests of that path).
//
// NCCL is loaded with dlopen("libnccl.so.2") at dyc_dist_create time (the copy
// torch has already loaded resolves by soname), so libdyc.so has no link-time
// NCCL dependency and single-GPU users never need it.  Only the handful of NCCL
// entry points used here are declared, with NCCL's own ABI.
#include <dlfcn.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "dycuckoo.h"

void dyc_internal_set_error(const std::string& msg);   // dyc_api.cu (thread-local dyc_last_error)

namespace {

// ------------------------------------------------------------------ NCCL ABI (subset)
typedef struct ncclComm* ncclComm_t;
typedef struct { char internal[DYC_NCCL_UNIQUE_ID_BYTES]; } ncclUniqueId;
typedef int ncclResult_t;          // ncclSuccess = 0
constexpr int kNcclInt8 = 0;       // ncclInt8 / ncclChar: byte transfers

struct Nccl {
    bool ok = false;
    std::string why;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    ncclResult_t (*Send)(const void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*GetVersion)(int*) = nullptr;
};

Nccl& nccl() {
    static Nccl n;
    static bool tried = false;
    if (tried) return n;
    tried = true;
    const char* env = getenv("DYC_NCCL_LIB");
    void* h = dlopen(env && *env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        n.why = std::string("cannot load NCCL (libnccl.so.2): ") + dlerror();
        return n;
    }
#define DYC_SYM(field, name)                                                   \
    n.field = reinterpret_cast<decltype(n.field)>(dlsym(h, name));             \
    if (!n.field) { n.why = std::string("NCCL symbol missing: ") + name; return n; }
    DYC_SYM(GetUniqueId, "ncclGetUniqueId")
    DYC_SYM(CommInitRank, "ncclCommInitRank")
    DYC_SYM(CommDestroy, "ncclCommDestroy")
    DYC_SYM(GroupStart, "ncclGroupStart")
    DYC_SYM(GroupEnd, "ncclGroupEnd")
    DYC_SYM(Send, "ncclSend")
    DYC_SYM(Recv, "ncclRecv")
    DYC_SYM(GetErrorString, "ncclGetErrorString")
    DYC_SYM(GetVersion, "ncclGetVersion")
#undef DYC_SYM
    n.ok = true;
    return n;
}

dyc_status err(dyc_status s, const std::string& msg) {
    dyc_internal_set_error(msg);
    return s;
}

#define DCU(x)                                                                                        \
    do {                                                                                              \
        cudaError_t e_ = (x);                                                                         \
        if (e_ != cudaSuccess)                                                                        \
            return err(e_ == cudaErrorMemoryAllocation ? DYC_ERR_OOM : DYC_ERR_CUDA,                   \
                       std::string(#x) + ": " + cudaGetErrorString(e_));                              \
    } while (0)

#define DNC(x)                                                                                        \
    do {                                                                                              \
        ncclResult_t r_ = (x);                                                                        \
        if (r_ != 0) return err(DYC_ERR_NCCL, std::string(#x) + ": " + nccl().GetErrorString(r_));    \
    } while (0)

#define DTRY(x)                         \
    do {                                \
        dyc_status s_ = (x);            \
        if (s_ != DYC_OK) return s_;    \
    } while (0)

inline cudaStream_t S(dyc_stream_t s) { return reinterpret_cast<cudaStream_t>(s); }

// A growable device buffer (cudaMalloc; regrowth is rare and happens between batches).
struct DBuf {
    void* p = nullptr;
    uint64_t cap = 0;
    dyc_status ensure(uint64_t bytes, cudaStream_t st) {
        if (bytes <= cap) return DYC_OK;
        if (p) {
            DCU(cudaStreamSynchronize(st));
            DCU(cudaFree(p));
            p = nullptr;
            cap = 0;
        }
        bytes = bytes + bytes / 4 + 256;
        DCU(cudaMalloc(&p, bytes));
        cap = bytes;
        return DYC_OK;
    }
    template <class T> T* as(uint64_t byte_off = 0) const { return (T*)((char*)p + byte_off); }
    void release() { if (p) cudaFree(p); p = nullptr; cap = 0; }
};

}  // namespace

struct dyc_dist {
    int rank = 0, world = 1, device = 0;
    uint32_t L = 1;                      // local shards
    uint32_t G = 1;                      // global shards = world * L
    ncclComm_t comm = nullptr;
    bool use_nccl = false;               // world > 1, or an id given with world 1 (self exchange)
    std::vector<dyc_table*> shard;       // local shard l is global shard rank*L + l
    DBuf counts, cursor, rcounts;        // u64[G], u64[G], u64[world*L]
    DBuf sk, sv, st, pos;                // grouped send buffers: keys, values, op codes; pos of op i
    DBuf rk, rv, rt;                     // shard-major receive buffers (world > 1)
    DBuf ov, os;                         // owner results (values, status), shard-major
    DBuf iv, is;                         // results back in the send layout
    unsigned long long* h_cnt = nullptr; // pinned: counts[G] | rcounts[world*L]
    uint64_t last_recv = 0;
    uint64_t n_batches = 0, n_exchanged = 0;
};

namespace {

enum Op { OP_INSERT = 1, OP_FIND = 2, OP_DELETE = 3, OP_MIXED = 4 };

// Send offset of (peer p, local shard l): the grouped send buffer is ordered by
// global shard s = p*L + l, so it is the prefix sum of counts[] up to s.
// Receive offset (shard-major): base[l] + sum_{p' < p} rc[p'][l].
struct Plan {
    std::vector<uint64_t> soff, scnt;    // [G]
    std::vector<uint64_t> roff, rcnt;    // [world*L], indexed p*L + l
    std::vector<uint64_t> base, tot;     // [L]
    uint64_t nrecv = 0;
};

Plan make_plan(const dyc_dist* D, const unsigned long long* cnt, const unsigned long long* rc) {
    Plan P;
    const uint32_t G = D->G, L = D->L, W = (uint32_t)D->world;
    P.soff.resize(G);
    P.scnt.resize(G);
    uint64_t acc = 0;
    for (uint32_t s = 0; s < G; s++) { P.soff[s] = acc; P.scnt[s] = cnt[s]; acc += cnt[s]; }
    P.base.assign(L, 0);
    P.tot.assign(L, 0);
    for (uint32_t l = 0; l < L; l++)
        for (uint32_t p = 0; p < W; p++) P.tot[l] += rc[p * L + l];
    uint64_t b = 0;
    for (uint32_t l = 0; l < L; l++) { P.base[l] = b; b += P.tot[l]; }
    P.nrecv = b;
    P.roff.resize((size_t)W * L);
    P.rcnt.resize((size_t)W * L);
    for (uint32_t l = 0; l < L; l++) {
        uint64_t o = P.base[l];
        for (uint32_t p = 0; p < W; p++) { P.roff[p * L + l] = o; P.rcnt[p * L + l] = rc[p * L + l]; o += rc[p * L + l]; }
    }
    return P;
}

// One grouped exchange of `esz`-byte elements: forward (send layout -> shard-major
// receive layout) or backward (the reverse).
dyc_status exchange(dyc_dist* D, const Plan& P, const void* src, void* dst, uint32_t esz, bool forward, cudaStream_t st) {
    Nccl& N = nccl();
    const uint32_t L = D->L;
    DNC(N.GroupStart());
    for (int p = 0; p < D->world; p++) {
        for (uint32_t l = 0; l < L; l++) {
            const uint64_t s_off = P.soff[(uint32_t)p * L + l], s_cnt = P.scnt[(uint32_t)p * L + l];
            const uint64_t r_off = P.roff[(uint32_t)p * L + l], r_cnt = P.rcnt[(uint32_t)p * L + l];
            // forward: my ops for (p, l) go to p; p's ops for my shard l arrive from p
            // backward: my results for p's ops of shard l go back to p; mine come from p
            if (forward) {
                if (s_cnt) { ncclResult_t r = N.Send((const char*)src + s_off * esz, s_cnt * esz, kNcclInt8, p, D->comm, st);
                             if (r) { N.GroupEnd(); return err(DYC_ERR_NCCL, std::string("ncclSend: ") + N.GetErrorString(r)); } }
                if (r_cnt) { ncclResult_t r = N.Recv((char*)dst + r_off * esz, r_cnt * esz, kNcclInt8, p, D->comm, st);
                             if (r) { N.GroupEnd(); return err(DYC_ERR_NCCL, std::string("ncclRecv: ") + N.GetErrorString(r)); } }
            } else {
                if (r_cnt) { ncclResult_t r = N.Send((const char*)src + r_off * esz, r_cnt * esz, kNcclInt8, p, D->comm, st);
                             if (r) { N.GroupEnd(); return err(DYC_ERR_NCCL, std::string("ncclSend: ") + N.GetErrorString(r)); } }
                if (s_cnt) { ncclResult_t r = N.Recv((char*)dst + s_off * esz, s_cnt * esz, kNcclInt8, p, D->comm, st);
                             if (r) { N.GroupEnd(); return err(DYC_ERR_NCCL, std::string("ncclRecv: ") + N.GetErrorString(r)); } }
            }
        }
    }
    DNC(N.GroupEnd());
    return DYC_OK;
}

dyc_status run_batch(dyc_dist* D, Op op, const uint8_t* d_ops, const uint32_t* d_keys, const uint32_t* d_values,
                     uint32_t* d_values_out, uint8_t* d_status, uint64_t n, cudaStream_t st) {
    DCU(cudaSetDevice(D->device));
    if (n > 0xFFFFFFFFull) return err(DYC_ERR_INVALID_ARG, "dyc_dist: a batch must be < 2^32 ops");
    if (n && !d_keys) return err(DYC_ERR_INVALID_ARG, "dyc_dist: null keys");
    if (n && (op == OP_INSERT || op == OP_MIXED) && !d_values) return err(DYC_ERR_INVALID_ARG, "dyc_dist: null values");
    if (n && op == OP_MIXED && !d_ops) return err(DYC_ERR_INVALID_ARG, "dyc_dist: null op codes");
    if (n && op == OP_FIND && !d_values_out) return err(DYC_ERR_INVALID_ARG, "dyc_dist: null values_out");
    const uint32_t G = D->G, L = D->L, W = (uint32_t)D->world;
    const bool carry_vals = op == OP_INSERT || op == OP_MIXED;
    const bool carry_tags = op == OP_MIXED;
    const bool want_vals = op != OP_INSERT && d_values_out;   // find / delete / mixed return values
    dyc_table* h0 = D->shard[0];                             // all shards share the hash constants
    // 1. group by shard
    DTRY(D->sk.ensure(4 * n + 4, st));
    DTRY(D->pos.ensure(4 * n + 4, st));
    if (carry_vals) DTRY(D->sv.ensure(4 * n + 4, st));
    if (carry_tags) DTRY(D->st.ensure(n + 4, st));
    DTRY(dyc_route_count(h0, d_keys, n, G, D->counts.as<uint64_t>(), st));
    if (n)
        DTRY(dyc_route_scatter(h0, d_keys, carry_vals ? d_values : nullptr, carry_tags ? d_ops : nullptr, n, G,
                               D->counts.as<uint64_t>(), D->cursor.as<uint64_t>(), D->sk.as<uint32_t>(),
                               carry_vals ? D->sv.as<uint32_t>() : nullptr, carry_tags ? D->st.as<uint8_t>() : nullptr,
                               D->pos.as<uint32_t>(), st));
    // 2. counts: mine to every peer, theirs to me
    unsigned long long* hc = D->h_cnt;
    unsigned long long* hr = D->h_cnt + G;
    if (D->use_nccl) {
        Nccl& N = nccl();
        DNC(N.GroupStart());
        for (uint32_t p = 0; p < W; p++) {
            ncclResult_t r = N.Send(D->counts.as<char>(8ull * p * L), 8ull * L, kNcclInt8, (int)p, D->comm, st);
            if (!r) r = N.Recv(D->rcounts.as<char>(8ull * p * L), 8ull * L, kNcclInt8, (int)p, D->comm, st);
            if (r) { N.GroupEnd(); return err(DYC_ERR_NCCL, std::string("count exchange: ") + N.GetErrorString(r)); }
        }
        DNC(N.GroupEnd());
        DCU(cudaMemcpyAsync(hr, D->rcounts.p, 8ull * W * L, cudaMemcpyDeviceToHost, st));
    }
    DCU(cudaMemcpyAsync(hc, D->counts.p, 8ull * G, cudaMemcpyDeviceToHost, st));
    DCU(cudaStreamSynchronize(st));
    if (!D->use_nccl) memcpy(hr, hc, 8ull * G);
    const Plan P = make_plan(D, hc, hr);
    D->last_recv = P.nrecv;
    D->n_batches++;
    // 3. requests: shard-major receive buffers (the send buffer itself when W == 1)
    const uint32_t* rk = D->sk.as<uint32_t>();
    const uint32_t* rv = carry_vals ? D->sv.as<uint32_t>() : nullptr;
    const uint8_t* rt = carry_tags ? D->st.as<uint8_t>() : nullptr;
    const uint64_t R = P.nrecv;
    if (D->use_nccl) {
        DTRY(D->rk.ensure(4 * R + 4, st));
        DTRY(exchange(D, P, D->sk.p, D->rk.p, 4, true, st));
        rk = D->rk.as<uint32_t>();
        if (carry_vals) {
            DTRY(D->rv.ensure(4 * R + 4, st));
            DTRY(exchange(D, P, D->sv.p, D->rv.p, 4, true, st));
            rv = D->rv.as<uint32_t>();
        }
        if (carry_tags) {
            DTRY(D->rt.ensure(R + 4, st));
            DTRY(exchange(D, P, D->st.p, D->rt.p, 1, true, st));
            rt = D->rt.as<uint8_t>();
        }
        D->n_exchanged += R;
    }
    // 4. the owners: one ordinary batch per local shard
    DTRY(D->os.ensure(R + 4, st));
    if (want_vals) DTRY(D->ov.ensure(4 * R + 4, st));
    for (uint32_t l = 0; l < L; l++) {
        const uint64_t b = P.base[l], m = P.tot[l];
        if (m == 0) continue;
        dyc_table* t = D->shard[l];
        uint8_t* so = D->os.as<uint8_t>(b);
        uint32_t* vo = want_vals ? D->ov.as<uint32_t>(4 * b) : nullptr;
        switch (op) {
            case OP_INSERT: DTRY(dyc_insert_batch(t, rk + b, rv + b, so, m, st)); break;
            case OP_FIND: DTRY(dyc_find_batch(t, rk + b, vo, so, m, st)); break;
            case OP_DELETE: DTRY(dyc_delete_batch(t, rk + b, vo, so, m, st)); break;
            case OP_MIXED: DTRY(dyc_mixed_batch(t, rt + b, rk + b, rv + b, vo, so, m, st)); break;
        }
    }
    // 5. replies back into the send layout, then request order
    const uint8_t* is = D->os.as<uint8_t>();
    const uint32_t* iv = want_vals ? D->ov.as<uint32_t>() : nullptr;
    if (D->use_nccl) {
        DTRY(D->is.ensure(n + 4, st));
        DTRY(exchange(D, P, D->os.p, D->is.p, 1, false, st));
        is = D->is.as<uint8_t>();
        if (want_vals) {
            DTRY(D->iv.ensure(4 * n + 4, st));
            DTRY(exchange(D, P, D->ov.p, D->iv.p, 4, false, st));
            iv = D->iv.as<uint32_t>();
        }
    }
    if (n) DTRY(dyc_route_unpermute(D->pos.as<uint32_t>(), n, iv, d_status ? is : nullptr, want_vals ? d_values_out : nullptr,
                                    d_status, st));
    return DYC_OK;
}

dyc_status check_dist(const dyc_dist* D) {
    if (!D) return err(DYC_ERR_INVALID_ARG, "null dyc_dist");
    return DYC_OK;
}

}  // namespace

extern "C" {

dyc_status dyc_dist_get_unique_id(void* id) {
    if (!id) return err(DYC_ERR_INVALID_ARG, "dyc_dist_get_unique_id: null output");
    Nccl& N = nccl();
    if (!N.ok) return err(DYC_ERR_NCCL, N.why);
    ncclUniqueId u;
    DNC(N.GetUniqueId(&u));
    memcpy(id, &u, sizeof(u));
    return DYC_OK;
}

dyc_status dyc_dist_create_ex(const dyc_config* cfg, const void* nccl_unique_id, int rank, int world,
                              uint32_t local_shards, dyc_dist** out) {
    if (!cfg || !out) return err(DYC_ERR_INVALID_ARG, "dyc_dist_create_ex: null argument");
    *out = nullptr;
    if (world < 1 || rank < 0 || rank >= world) return err(DYC_ERR_INVALID_ARG, "dyc_dist_create: need 0 <= rank < world");
    if (local_shards < 1 || (uint64_t)world * local_shards > 1024)
        return err(DYC_ERR_INVALID_ARG, "dyc_dist_create: need 1 <= local_shards and world*local_shards <= 1024");
    if (world > 1 && !nccl_unique_id) return err(DYC_ERR_INVALID_ARG, "dyc_dist_create: world > 1 needs an NCCL unique id");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return err(DYC_ERR_NO_DEVICE, "no CUDA device");
    }
    dyc_dist* D = new dyc_dist();
    D->rank = rank;
    D->world = world;
    D->L = local_shards;
    D->G = (uint32_t)world * local_shards;
    cudaGetDevice(&D->device);
    auto fail = [&](dyc_status s) { dyc_dist_destroy(D); return s; };
    for (uint32_t l = 0; l < D->L; l++) {
        dyc_table* t = nullptr;
        dyc_status s = dyc_create_ex(cfg, &t);     // same seed everywhere: one hash family (Q1)
        if (s != DYC_OK) return fail(s);
        D->shard.push_back(t);
    }
    if (cudaMallocHost(&D->h_cnt, 8ull * 2 * D->G) != cudaSuccess) {
        cudaGetLastError();
        return fail(err(DYC_ERR_OOM, "dyc_dist_create: pinned counters"));
    }
    dyc_status s = D->counts.ensure(8ull * D->G, nullptr);
    if (s == DYC_OK) s = D->cursor.ensure(8ull * D->G, nullptr);
    if (s == DYC_OK) s = D->rcounts.ensure(8ull * D->G, nullptr);
    if (s != DYC_OK) return fail(s);
    D->use_nccl = world > 1 || nccl_unique_id != nullptr;
    if (D->use_nccl) {
        Nccl& N = nccl();
        if (!N.ok) return fail(err(DYC_ERR_NCCL, N.why));
        ncclUniqueId u;
        memcpy(&u, nccl_unique_id, sizeof(u));
        ncclResult_t r = N.CommInitRank(&D->comm, world, u, rank);
        if (r != 0) {
            D->comm = nullptr;
            return fail(err(DYC_ERR_NCCL, std::string("ncclCommInitRank: ") + N.GetErrorString(r)));
        }
    }
    *out = D;
    return DYC_OK;
}

dyc_status dyc_dist_create(uint32_t d, uint64_t init_capacity_per_shard, double alpha, double beta,
                           const void* nccl_unique_id, int rank, int world, dyc_dist** out) {
    dyc_config c;
    dyc_config_default(&c);
    c.d = d;
    c.init_capacity = init_capacity_per_shard;
    c.alpha = alpha;
    c.beta = beta;
    return dyc_dist_create_ex(&c, nccl_unique_id, rank, world, 1, out);
}

dyc_status dyc_dist_destroy(dyc_dist* D) {
    if (!D) return DYC_OK;
    cudaSetDevice(D->device);
    cudaDeviceSynchronize();
    if (D->comm && nccl().ok) nccl().CommDestroy(D->comm);
    for (dyc_table* t : D->shard) dyc_destroy(t);
    for (DBuf* b : {&D->counts, &D->cursor, &D->rcounts, &D->sk, &D->sv, &D->st, &D->pos, &D->rk, &D->rv, &D->rt,
                    &D->ov, &D->os, &D->iv, &D->is})
        b->release();
    if (D->h_cnt) cudaFreeHost(D->h_cnt);
    delete D;
    return DYC_OK;
}

dyc_status dyc_dist_insert_batch(dyc_dist* D, const uint32_t* d_keys, const uint32_t* d_values, uint8_t* d_status,
                                 uint64_t n, dyc_stream_t stream) {
    DTRY(check_dist(D));
    return run_batch(D, OP_INSERT, nullptr, d_keys, d_values, nullptr, d_status, n, S(stream));
}

dyc_status dyc_dist_find_batch(dyc_dist* D, const uint32_t* d_keys, uint32_t* d_values_out, uint8_t* d_found,
                               uint64_t n, dyc_stream_t stream) {
    DTRY(check_dist(D));
    return run_batch(D, OP_FIND, nullptr, d_keys, nullptr, d_values_out, d_found, n, S(stream));
}

dyc_status dyc_dist_delete_batch(dyc_dist* D, const uint32_t* d_keys, uint32_t* d_values_out, uint8_t* d_status,
                                 uint64_t n, dyc_stream_t stream) {
    DTRY(check_dist(D));
    return run_batch(D, OP_DELETE, nullptr, d_keys, nullptr, d_values_out, d_status, n, S(stream));
}

dyc_status dyc_dist_mixed_batch(dyc_dist* D, const uint8_t* d_ops, const uint32_t* d_keys, const uint32_t* d_values,
                                uint32_t* d_values_out, uint8_t* d_status, uint64_t n, dyc_stream_t stream) {
    DTRY(check_dist(D));
    return run_batch(D, OP_MIXED, d_ops, d_keys, d_values, d_values_out, d_status, n, S(stream));
}

dyc_status dyc_dist_info(const dyc_dist* D, int* rank, int* world, uint32_t* local_shards, uint64_t* last_recv) {
    DTRY(check_dist(D));
    if (rank) *rank = D->rank;
    if (world) *world = D->world;
    if (local_shards) *local_shards = D->L;
    if (last_recv) *last_recv = D->last_recv;
    return DYC_OK;
}

dyc_status dyc_dist_shard(const dyc_dist* D, uint32_t local_index, dyc_table** out) {
    DTRY(check_dist(D));
    if (!out || local_index >= D->L) return err(DYC_ERR_INVALID_ARG, "dyc_dist_shard: bad index or null output");
    *out = D->shard[local_index];
    return DYC_OK;
}

}  // extern "C"
