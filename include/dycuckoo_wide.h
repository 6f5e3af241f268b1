/*
 * dycuckoo_wide.h — C ABI of the WIDE-key DyCuckoo table.
 *
 * The same dynamic two-layer cuckoo table as dycuckoo.h (P:L270-273, P:L305-312,
 * P:L374-395), with 8-byte keys and values of W 8-byte words
 * ("Suppose the keys are 8-bytes, a bucket can then accommodate 16
 * KV pairs.  Furthermore, we lock the entire bucket exclusively for a warp to
 * perform insertion/deletion ... we do not limit ourselves to supporting KV
 * pairs with only 64 bits").  Hash: reading Q33 of DESIGN.md,
 *     x_s(k) = (c_s * hi32(k) + a_s * lo32(k) + b_s) mod (2^32 - 5),
 * pair / bucket / shard as in dycuckoo.h; a key below 2^32 hashes exactly as in
 * the 32-bit table.  The key 0xFFFFFFFFFFFFFFFF is reserved (EMPTY): such an op
 * gets status DYC_OP_NONE.  A find miss writes W words of all ones.
 *
 * Placement modes (how concurrent inserts into one bucket are arbitrated):
 *   DYW_MODE_VOTER    Alg. 1 as printed: bucket locks taken by a
 *                     warp-elected leader; the warp inspects the bucket.
 *                     Layout: 16 keys per 128-byte bucket, values in a separate
 *                     array.  W = 1, 2 or 4.
 *   DYW_MODE_GROUPED  same layout and locks; every lane try-locks its own bucket
 *                     each round, same-bucket lanes grouped by __match_any_sync.
 *   DYW_MODE_LOCKFREE no locks: 16-byte {key, value} slots, 8 per 128-byte
 *                     bucket, moved with 128-bit atomicCAS / atomicExch
 *                     (sm_90+/sm_100a).  W = 1 only.
 * Find and delete never lock.
 *
 * Conventions are those of dycuckoo.h: device pointers owned by the caller,
 * stream-ordered calls (insert and delete synchronize `stream` to take resize
 * decisions), keys distinct within a batch, n = 0 is a no-op, errors as
 * dyc_status with a message in dyc_last_error().  Values are row-major: op i's
 * words are values[i*W .. i*W+W).
 */
#ifndef DYCUCKOO_WIDE_H
#define DYCUCKOO_WIDE_H

#include <stdint.h>
#include "dycuckoo.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dyw_table dyw_table;

enum { DYW_MODE_VOTER = 0, DYW_MODE_GROUPED = 1, DYW_MODE_LOCKFREE = 2 };

typedef struct {
    uint32_t d;              /* subtables, 2..DYC_MAX_D                                  */
    uint32_t value_words;    /* W: 1, 2 or 4 (8, 16 or 32-byte values); LOCKFREE: 1     */
    uint32_t mode;           /* DYW_MODE_*                                               */
    uint32_t max_hops;       /* L_max (Q6)                                               */
    double   alpha, beta;    /* fill bounds, as in dycuckoo.h (Q14)                      */
    uint64_t init_capacity;  /* slots (Q13)                                              */
    uint64_t seed;           /* SplitMix64 seed of a_s, b_s, then c_s (Q1, Q33)          */
} dyw_config;

typedef struct {
    uint64_t m, N;
    uint32_t d, B, W, mode;
    uint64_t buckets[DYC_MAX_D];
    uint64_t count[DYC_MAX_D];
    double   fill;
    uint64_t n_upsize, n_downsize, n_fail_upsize, n_residual, n_evict;
    uint64_t n_lock_fail;             /* try-locks that found the bucket locked (lock modes) */
    uint64_t last_insert_new, last_insert_pending;
    uint64_t bytes_allocated;
} dyw_stats_t;

/* Defaults: d=4, W=2, VOTER, L_max=64, alpha=0.3, beta=0.85, init_capacity=4096, seed=0x5EED0001. */
dyc_status dyw_config_default(dyw_config* cfg);
/* DYC_ERR_INVALID_ARG for a bad d / W / mode combination or bounds violating
 * 0 < alpha < beta < 1, alpha <= beta*d/(d+1); DYC_ERR_OOM; DYC_ERR_NO_DEVICE. */
dyc_status dyw_create(const dyw_config* cfg, dyw_table** out);
dyc_status dyw_destroy(dyw_table* t);

/* Upsert (Alg. 1, two-phase reading Q7): d_status[i] = 1 inserted,
 * 2 updated, 0 reserved key (nullable).  Upsizes first while (m+n_new) > beta*N;
 * halves while m < alpha*N afterwards (Q11). */
dyc_status dyw_insert_batch(dyw_table* t, const uint64_t* d_keys, const uint64_t* d_values, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream);
/* d_values_out: n*W words (value or all ones); d_found nullable.  <= 2 probes. */
dyc_status dyw_find_batch(dyw_table* t, const uint64_t* d_keys, uint64_t* d_values_out, uint8_t* d_found,
                          uint64_t n, dyc_stream_t stream);
/* d_values_out (nullable): the removed values; d_status (nullable): 1 removed. */
dyc_status dyw_delete_batch(dyw_table* t, const uint64_t* d_keys, uint64_t* d_values_out, uint8_t* d_status,
                            uint64_t n, dyc_stream_t stream);
/* As dyc_resize: +1 doubles a smallest subtable, -1 halves a largest, 0 enforces [alpha, beta]. */
dyc_status dyw_resize(dyw_table* t, int direction, int subtable, dyc_stream_t stream);
dyc_status dyw_clear(dyw_table* t, dyc_stream_t stream);
dyc_status dyw_stats(dyw_table* t, dyw_stats_t* out, dyc_stream_t stream);
/* Live contents to host arrays (h_values: cap*W words); any pointer but n_out nullable. */
dyc_status dyw_dump(dyw_table* t, uint64_t* h_keys, uint64_t* h_values, uint32_t* h_table, uint64_t* h_bucket,
                    uint64_t cap, uint64_t* n_out, dyc_stream_t stream);
/* Device-side hash of keys for test vectors: d_x[i*(d+2)+s] = x_s(k_i), d_pair[2i..2i+1] = (t1, t2). */
dyc_status dyw_hash_probe(dyw_table* t, const uint64_t* d_keys, uint64_t n, uint32_t* d_x, uint32_t* d_pair,
                          dyc_stream_t stream);
/* Number of kernels this table launched (reset if `reset`). */
uint64_t dyw_launch_count(dyw_table* t, int reset);

#ifdef __cplusplus
}
#endif
#endif
