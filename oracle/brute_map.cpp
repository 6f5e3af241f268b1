// brute_map.cpp — the brute-force map of the KV-store semantics:
// std::unordered_map<uint32_t, uint32_t>, single-threaded.  TEST INFRASTRUCTURE
// and CPU BASELINE (ii) of BASELINE.md §3 only: bench.py's cpu_baseline leg
// times it beside the DyCuckoo oracle; nothing on the product path uses it.
// Semantics (readings Q8, Q10, Q25): insert -> 1 inserted / 2 updated and
// M[k] = v; find -> (M[k], 1) or (0xFFFFFFFF, 0); delete -> (old, 1) and erase,
// or (0xFFFFFFFF, 0); key 0xFFFFFFFF is reserved (status 0, no effect); a mixed
// batch runs its finds, then its inserts, then its deletes.
#include <cstdint>
#include <unordered_map>

namespace {
constexpr uint32_t kEmpty = 0xFFFFFFFFu;
struct Map { std::unordered_map<uint32_t, uint32_t> m; };
}

extern "C" {

void* bm_create(uint64_t reserve) {
    Map* M = new Map();
    if (reserve) M->m.reserve(reserve);
    return M;
}

void bm_destroy(void* h) { delete static_cast<Map*>(h); }

uint64_t bm_size(void* h) { return static_cast<Map*>(h)->m.size(); }

void bm_insert_batch(void* h, const uint32_t* keys, const uint32_t* vals, uint8_t* status, uint64_t n) {
    auto& m = static_cast<Map*>(h)->m;
    for (uint64_t i = 0; i < n; i++) {
        if (keys[i] == kEmpty) { if (status) status[i] = 0; continue; }
        auto r = m.insert_or_assign(keys[i], vals[i]);
        if (status) status[i] = r.second ? 1 : 2;
    }
}

void bm_find_batch(void* h, const uint32_t* keys, uint32_t* vals, uint8_t* found, uint64_t n) {
    auto& m = static_cast<Map*>(h)->m;
    for (uint64_t i = 0; i < n; i++) {
        auto it = keys[i] == kEmpty ? m.end() : m.find(keys[i]);
        const bool hit = it != m.end();
        vals[i] = hit ? it->second : kEmpty;
        if (found) found[i] = hit;
    }
}

void bm_delete_batch(void* h, const uint32_t* keys, uint32_t* vals, uint8_t* status, uint64_t n) {
    auto& m = static_cast<Map*>(h)->m;
    for (uint64_t i = 0; i < n; i++) {
        auto it = keys[i] == kEmpty ? m.end() : m.find(keys[i]);
        const bool hit = it != m.end();
        if (vals) vals[i] = hit ? it->second : kEmpty;
        if (status) status[i] = hit;
        if (hit) m.erase(it);
    }
}

void bm_mixed_batch(void* h, const uint8_t* ops, const uint32_t* keys, const uint32_t* vals, uint32_t* vals_out,
                    uint8_t* status, uint64_t n) {
    auto& m = static_cast<Map*>(h)->m;
    for (uint64_t i = 0; i < n; i++)
        if (ops[i] > 2) { vals_out[i] = kEmpty; status[i] = 0; }   // no operation (reading Q10)
    for (int phase = 0; phase < 3; phase++)
        for (uint64_t i = 0; i < n; i++) {
            if (ops[i] != phase) continue;
            if (phase == 0) bm_find_batch(h, keys + i, vals_out + i, status + i, 1);
            else if (phase == 1) { bm_insert_batch(h, keys + i, vals + i, status + i, 1); vals_out[i] = kEmpty; }
            else bm_delete_batch(h, keys + i, vals_out + i, status + i, 1);
        }
    (void)m;
}

}  // extern "C"
