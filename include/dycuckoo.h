/*
 * dycuckoo.h — C ABI of libdyc.so, the B200-native DyCuckoo hot path.
 *
 * DyCuckoo: "Dynamic Hash Tables on GPUs" (Li, Zhu, Lyu, Huang, Sun, ICDE'21).
 * P:L<n> cites line n of the paper's text with its section; Qn cites
 * a reading of an ambiguous passage, listed in DESIGN.md §4.
 *
 * The table is a two-layer cuckoo hash table: d subtables (§IV-A) of
 * buckets of B slots; a first-layer hash maps every key to an ordered pair of
 * subtables (§V-A), a second-layer universal hash
 * h^t(k) = ((a_t k + b_t) mod p) mod |h^t| to one bucket per subtable,
 * so find and delete probe at most two buckets.  Inserts run bounded
 * cuckoo eviction chains (Alg. 1).  The fill factor
 * θ = Σm_t / Σn_t is kept inside [alpha, beta] by doubling the
 * smallest or halving the largest subtable, one at a time (§IV-B),
 * splitting or merging its buckets.
 *
 * Conventions common to every entry point
 * ---------------------------------------
 * - Keys and values are uint32.  Key 0xFFFFFFFF (DYC_EMPTY_KEY) is reserved to
 *   mark free slots (reading Q25): an op on it gets status DYC_OP_NONE and has
 *   no effect; the batch does not fail.
 * - Every d_* pointer is DEVICE memory on the table's device, owned by the
 *   caller, and must stay valid until the enqueued work completes.  h_* pointers
 *   are HOST memory (pinned gives the best copy speed, pageable works).  The
 *   table owns its subtables, scratch lists and memory pool.
 * - Arrays are dense, element i belongs to op i.  No alignment beyond the
 *   element type is required.
 * - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   Work is stream-ordered.  find never blocks the host.  A mutating batch
 *   waits for `stream` only when a resize decision needs the exact live count
 *   (S6): an insert whose upper bound m + n may exceed beta*N reads the number
 *   of new keys back once before placing them (Q11); a delete, or an
 *   insert, after which a lower bound of m may fall below alpha*N reads the
 *   counts back for the alpha loop.  Otherwise the batch returns without
 *   waiting: its counts stay in accumulating device counters and are applied
 *   at the next read-back (which first waits for an event recorded on the lazy
 *   batch's stream, so another stream may issue it).  Pairs that an insert
 *   could not place within max_hops hops wait in a device stash that find,
 *   insert and delete consult until the next read-back places them, upsizing
 *   on failure (Q17); results are never affected.  Batches on one
 *   table must not overlap in time: issue them on one stream, or order them
 *   across streams with events.
 * - Batches are single-type.  Keys must be distinct within a batch
 *   (precondition, reading Q9); violating it never corrupts the table but the
 *   final value of a duplicated key is unspecified.
 * - n == 0 is a no-op returning DYC_OK.
 * - Errors are returned, never thrown.  dyc_last_error() gives a thread-local
 *   message.  A CUDA error is sticky: DYC_ERR_CUDA.  An out-of-memory during a
 *   resize returns DYC_ERR_OOM and leaves the table consistent (no key lost).
 * - A table belongs to one host thread at a time.
 */
#ifndef DYCUCKOO_H
#define DYCUCKOO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DYC_MAX_D      16u            /* maximum number of subtables d          */
#define DYC_EMPTY_KEY  0xFFFFFFFFu    /* reserved key (free slot), Q25          */
#define DYC_NOT_FOUND  0xFFFFFFFFu    /* value written for a find/delete miss   */

typedef struct dyc_table dyc_table;   /* opaque; owns subtables, scratch, pool  */
typedef void* dyc_stream_t;           /* cudaStream_t                           */

typedef enum {
    DYC_OK = 0,
    DYC_ERR_INVALID_ARG = 1,
    DYC_ERR_OOM = 2,
    DYC_ERR_CUDA = 3,
    DYC_ERR_INSERT_FAILED = 4,        /* a key could not be placed even after upsizing */
    DYC_ERR_NO_DEVICE = 5,
    DYC_ERR_NCCL = 6                  /* NCCL missing or an NCCL call failed (dyc_dist_*) */
} dyc_status;

/* per-op status codes written to uint8 status / found arrays */
enum {
    DYC_OP_NONE = 0,                  /* absent key, or reserved key            */
    DYC_OP_INSERTED = 1,              /* insert of a key that was absent        */
    DYC_OP_UPDATED = 2,               /* insert of a present key: value replaced (Alg. 1) */
    DYC_OP_FOUND = 1,                 /* find hit                               */
    DYC_OP_DELETED = 1                /* delete hit                             */
};

/* Resize methods for dyc_resize_ex (measurement baselines). */
enum {
    DYC_RESIZE_SPLIT = 0,             /* the paper's method: split/merge one subtable */
    DYC_RESIZE_REINSERT_SUBTABLE = 1, /* baseline of P:L809: reinsert the subtable's entries with the insert path */
    DYC_RESIZE_REHASH_ALL = 2         /* MegaKV-style baseline: double/halve every subtable, reinsert all */
};

typedef struct {
    uint32_t d;              /* subtables, 2..DYC_MAX_D (paper default 4)      */
    uint32_t bucket_slots;   /* B: 4, 8 (64-byte bucket, default), 16 or 32 (Q26)     */
    double   alpha, beta;    /* fill bounds, 0 < alpha < beta < 1, alpha <= beta*d/(d+1) (Q14) */
    uint64_t init_capacity;  /* slots; n0 = max(1, ceil(init_capacity/(d*B))) buckets per subtable (Q13) */
    uint64_t seed;           /* SplitMix64 seed of the hash constants a_s, b_s (Q1)  */
    uint32_t max_hops;       /* L_max: eviction hops per attempt before the failure list (Q6) */
    uint32_t flags;          /* DYC_PLACE_PAPER_WEIGHTED: the paper's placement rule instead
                                of two-choice first-fit (reading Q3);
                                DYC_RESIZE_IN_PLACE: subtables resize in place in
                                reserved address ranges (opt-in)                     */
} dyc_config;

/* dyc_config.flags: in-place resizing.  Each subtable lives in its own reserved
 * virtual address range (256 GB of address space) whose physical backing
 * (cuMemCreate/cuMemMap, 2 MB granules) grows and shrinks with it: an upsize
 * maps only the new half behind the old buckets and splits bucket b into b and
 * b + n there; a downsize merges b' and b' + h into b'
 * and the upper half is unmapped at the next host read-back.  No buffer is
 * copied or held twice.  Falls back to cudaMalloc buffers when the driver's
 * virtual-memory API is unavailable; a resize under live traffic
 * (dyc_resize_begin) or a reinsert baseline (dyc_resize_ex methods 1, 2) moves
 * that subtable to a cudaMalloc buffer.  Opt-in: on the measured B200 driver,
 * mapping and unmapping physical memory costs ~28 ms per GB, far more than the
 * cached cudaMalloc buffers of the default path. */
#define DYC_RESIZE_IN_PLACE 2u

/* dyc_config.flags: the paper's balancing rule (SURVEY §8(f)
 * NEXT-4): a new pair goes to table i of its pair with probability
 * proportional to n_i / C(m_i, 2) (a snapshot of the per-subtable counts taken
 * at the start of each insert batch and after each resize of it, one streaming
 * count pass over the table), and evictions start in that table.  Results are
 * identical to first-fit (placement only changes where keys live); find and
 * the insert existence check always probe both buckets in this mode, since the
 * first-choice-full invariant does not hold under it. */
#define DYC_PLACE_PAPER_WEIGHTED 1u

/* dyc_config.flags: chunk-staged execution of large batches (DESIGN.md §5,
 * "Staged batches").  A single insert (needing no upsize) or delete batch of
 * B = 8 whose op count is at least the table's bucket count (and >= 2^20) is
 * ordered on the device by the 64 KB table chunk (1024 buckets) of each op's
 * first-choice bucket; each chunk is then read once with a
 * TMA bulk copy, its ops are applied in shared memory and it is written back
 * once; ops the first-choice bucket cannot decide go through the direct kernels.
 * Results are those of the direct path (each op's result depends only on the
 * table before the batch and its own key, P:L464 with distinct keys, Q9); only
 * where new keys land may differ.  Scratch: ~40 bytes per op, kept by the table
 * until dyc_trim.  Not used with a resize in flight, the paper-weighted
 * placement, a possibly non-empty stash, or the parts / mixed / host-buffer
 * entry points.  DYC_STAGED_OFF disables it; DYC_STAGED_FORCE uses it for every
 * eligible batch whatever its size, finds included (tests; a staged find is
 * slower than dyc_find_batch's direct kernel at C2); neither = automatic. */
#define DYC_STAGED_OFF 4u
#define DYC_STAGED_FORCE 8u

typedef struct {
    uint64_t m;                       /* live keys Σ m_t                          */
    uint64_t N;                       /* slots Σ n_t * B                          */
    uint32_t d, B;
    uint64_t buckets[DYC_MAX_D];      /* |h^t|                                    */
    uint64_t count[DYC_MAX_D];        /* m_t, counted on the device               */
    double   fill;                    /* θ = m / N                       */
    uint64_t n_upsize, n_downsize;    /* policy resizes                  */
    uint64_t n_fail_upsize;           /* upsizes triggered by placement failure */
    uint64_t n_residual;              /* downsize residuals re-placed    */
    uint64_t n_evict;                 /* eviction hops performed                  */
    uint64_t n_place_retry;           /* extra placement passes over failure lists */
    uint64_t n_second_table;          /* live keys stored in their second-choice subtable (φ·m) */
    uint64_t bytes_allocated;         /* device bytes held by subtables + scratch */
    uint64_t last_insert_new;         /* new keys of the last insert batch               */
    uint64_t last_insert_pending;     /* ... of which needed the eviction kernel (k_place) */
    uint64_t last_insert_evictions;   /* eviction hops of the last insert batch          */
    uint64_t bytes_cached;            /* released buffers kept for reuse (dyc_trim frees them) */
    uint64_t n_live_resize;           /* resizes committed through dyc_resize_begin/commit */
    uint64_t n_deferred;              /* ops deferred because their subtable was being resized */
    uint64_t n_device_alloc;          /* cudaMalloc calls (buffers not served by the cache) */
    double   alloc_ms;                /* host milliseconds spent inside those cudaMalloc calls */
    uint64_t n_sync;                  /* counter read-backs: the host waited on the stream (S6) */
    double   sync_ms;                 /* host milliseconds spent in those waits                */
    uint64_t n_pending;               /* new keys handed to the eviction kernel by all insert batches */
    uint64_t vm_subtables;            /* subtables resized in place (DYC_RESIZE_IN_PLACE)          */
    uint64_t vm_mapped_bytes;         /* physical bytes mapped under their address ranges          */
    uint64_t n_vm_map, n_vm_unmap;    /* physical chunks mapped / unmapped so far                  */
    uint64_t n_staged;                /* batches run chunk-staged (DYC_STAGED_*)                   */
} dyc_stats_t;

/* Fills *cfg with the defaults: d=4, B=8, alpha=0.3, beta=0.85 (Table
 * `tbl:parameters`), init_capacity=4096, seed=0x5EED0001, max_hops=64,
 * flags = 0 (first-fit placement, cudaMalloc subtables). */
dyc_status dyc_config_default(dyc_config* cfg);

/* Creates a table on the current CUDA device with the default config except
 * d, init_capacity, alpha, beta.  *out receives the handle.  Errors:
 * DYC_ERR_INVALID_ARG for d outside 2..16 or bounds violating
 * 0 < alpha < beta < 1, alpha <= beta*d/(d+1); DYC_ERR_OOM; DYC_ERR_NO_DEVICE. */
dyc_status dyc_create(uint32_t d, uint64_t init_capacity, double alpha, double beta, dyc_table** out);
dyc_status dyc_create_ex(const dyc_config* cfg, dyc_table** out);

/* Releases all device memory of the table (synchronizes its last stream). */
dyc_status dyc_destroy(dyc_table* t);

/* Batched insert (P:L188-189 insert(k,v); Alg. 1; §V-B "Insert").
 * d_keys[n], d_values[n]: input.  d_status[n] (nullable): DYC_OP_INSERTED,
 * DYC_OP_UPDATED, or DYC_OP_NONE for the reserved key.  Before placing new keys
 * the table upsizes while (m + n_new) > beta*N (Q11); a placement
 * failure triggers further upsizes; afterwards the alpha bound is
 * enforced.  Returns DYC_ERR_OOM / DYC_ERR_INSERT_FAILED if memory runs out
 * (already-placed ops stay applied; the table stays consistent). */
dyc_status dyc_insert_batch(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_values,
                            uint8_t* d_status, uint64_t n, dyc_stream_t stream);

/* One insert batch delivered in parts (e.g. as shards of it arrive over the
 * network): dyc_insert_begin(n_total), then dyc_insert_part() for parts whose
 * sizes sum to at most n_total, then dyc_insert_end().  Equivalent to one
 * dyc_insert_batch over the concatenation of the parts: one resize decision, one
 * alpha check.  The same for deletes.  No other call on the table
 * may come between begin and end. */
dyc_status dyc_insert_begin(dyc_table* t, uint64_t n_total, dyc_stream_t stream);
dyc_status dyc_insert_part(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_values,
                           uint8_t* d_status, uint64_t n, dyc_stream_t stream);
dyc_status dyc_insert_end(dyc_table* t, dyc_stream_t stream);
dyc_status dyc_delete_begin(dyc_table* t, uint64_t n_total, dyc_stream_t stream);
dyc_status dyc_delete_part(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out,
                           uint8_t* d_status, uint64_t n, dyc_stream_t stream);
dyc_status dyc_delete_end(dyc_table* t, dyc_stream_t stream);

/* Batched find (§V-B "Find"): at most two bucket probes per key.
 * d_values_out[n]: the value, or DYC_NOT_FOUND on a miss ("NULL").
 * d_found[n] (nullable): DYC_OP_FOUND or DYC_OP_NONE.  Never synchronizes. */
dyc_status dyc_find_batch(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out,
                          uint8_t* d_found, uint64_t n, dyc_stream_t stream);

/* Batched delete (§V-B "Delete"): erase on match, no locking.
 * d_values_out[n] (nullable): the removed value or DYC_NOT_FOUND.
 * d_status[n] (nullable): DYC_OP_DELETED or DYC_OP_NONE.  Afterwards the table
 * halves its largest subtable while m < alpha*N (Q11-Q13). */
dyc_status dyc_delete_batch(dyc_table* t, const uint32_t* d_keys, uint32_t* d_values_out,
                            uint8_t* d_status, uint64_t n, dyc_stream_t stream);

/* Mixed batch (configs C4/C5): op i is d_ops[i] in {DYC_MIX_FIND, DYC_MIX_INSERT,
 * DYC_MIX_DELETE}.  The paper batches one op type at a time and calls
 * mixed batches ambiguous (commented); reading Q10: keys are distinct
 * across the whole batch and the phases run find -> insert -> delete, so finds
 * observe the table before the batch.  The ops are grouped by type on the
 * device into fixed regions of a scratch buffer and run as three single-type
 * batches whose op counts stay on the device (the kernels read them), so the
 * grouping adds no host wait; the results return in request order:
 * d_values_out[i] (nullable) = found / removed value, DYC_NOT_FOUND on a miss
 * and for inserts; d_status[i] (nullable) = the op's status code; d_values
 * may be NULL (inserts then store 0).  An op code outside 0..2 gets status
 * DYC_OP_NONE and has no effect.  n < 2^30.  Scratch: about 56 bytes per op,
 * owned by the table. */
enum { DYC_MIX_FIND = 0, DYC_MIX_INSERT = 1, DYC_MIX_DELETE = 2 };
dyc_status dyc_mixed_batch(dyc_table* t, const uint8_t* d_ops, const uint32_t* d_keys,
                           const uint32_t* d_values, uint32_t* d_values_out, uint8_t* d_status,
                           uint64_t n, dyc_stream_t stream);

/* Explicit resize of one subtable (§IV-B; kernels P:L374-395).
 * direction +1: double subtable `subtable` (-1 = the smallest, ties lowest index);
 * direction -1: halve it (-1 = the largest, ties highest index; refused if its
 * bucket count is odd or 1); direction 0: enforce [alpha, beta] with the policy.
 * A choice that would leave a subtable more than twice another is
 * DYC_ERR_INVALID_ARG.  dyc_resize_ex selects the method (DYC_RESIZE_*). */
dyc_status dyc_resize(dyc_table* t, int direction, int subtable, dyc_stream_t stream);
dyc_status dyc_resize_ex(dyc_table* t, int direction, int subtable, int method, dyc_stream_t stream);

/* Resize under live traffic ("we do not need
 * to lock all hash tables and only to resize one", "it only locks the
 * subtable being resized and supports concurrent updates for the remaining
 * subtables").
 *
 * dyc_resize_begin enqueues the split (direction +1) or merge
 * (direction -1) of one subtable (-1 = the policy's choice; the
 * same shape rules as dyc_resize) on `resize_stream`, ordered after the work
 * already enqueued on `stream`, and returns without waiting.  The resize is
 * then "in flight" until it is committed:
 *   - find batches run concurrently with it and see every key (they read the
 *     subtable's old buffer, which nothing writes while it is being copied);
 *   - insert and delete batches run against the old buffer too, with the
 *     resized subtable locked: ops that need to write it (an update or delete
 *     of a key stored there, a new key whose other candidate bucket is full) are
 *     deferred; if a batch has any, it commits the resize at its end and then
 *     applies them, so every batch's statuses, values and the table contents
 *     are exactly those of the sequential order "resize, then the batches";
 *   - every resize decision (Q11) is taken against the post-resize
 *     size; one that has to act commits first;
 *   - dyc_resize*, dyc_stats, dyc_dump and dyc_clear commit first.
 * dyc_resize_commit makes `stream` wait for the resize kernel and installs the
 * new buffer (a downsize then places its residuals); it is a no-op
 * when nothing is in flight.  All batches of the window must be issued on one
 * stream (`stream`), or ordered by the caller.  Errors: DYC_ERR_INVALID_ARG if
 * a resize is already in flight, a part batch is open, or the shape rules
 * forbid the resize; DYC_ERR_OOM. */
dyc_status dyc_resize_begin(dyc_table* t, int direction, int subtable, dyc_stream_t stream,
                            dyc_stream_t resize_stream);
dyc_status dyc_resize_commit(dyc_table* t, dyc_stream_t stream);
/* *in_flight = 1 while a resize is uncommitted; *kernel_done = 1 once its
 * kernel has finished on the device (either pointer may be NULL). */
dyc_status dyc_resize_query(const dyc_table* t, int* in_flight, int* kernel_done);

/* Returns the buffers the table keeps for reuse (released subtables after a
 * resize, old scratch) to the device.  Resizing frees a subtable's old buffer
 * into this cache, so up/down cycles do not pay cudaMalloc each time.  The
 * cache holds at most the table's high-water size + 256 MB (oldest buffers are
 * freed first beyond that). */
dyc_status dyc_trim(dyc_table* t);

/* Empties the table without resizing (all slots EMPTY, m = 0). */
dyc_status dyc_clear(dyc_table* t, dyc_stream_t stream);

/* Statistics; counts m_t with a device kernel and synchronizes `stream`. */
dyc_status dyc_stats(dyc_table* t, dyc_stats_t* out, dyc_stream_t stream);

/* Host view of the table's shape, without touching the device (never
 * synchronizes): buckets[d] (nullable) = |h^t| per subtable as the resize
 * policy has left it; batches that skipped their counter read-back (see the
 * stream semantics above) leave the live count known only within
 * [*m_lo, *m_hi] (equal when nothing is pending); *n_fail_upsize = upsizes so
 * far that placement failures triggered.  Any pointer may be NULL.
 * A resize in flight (dyc_resize_begin) is not included. */
dyc_status dyc_shape(const dyc_table* t, uint64_t* buckets, uint64_t* m_lo, uint64_t* m_hi, uint64_t* n_fail_upsize);

/* Copies the live contents to host arrays (tests/diagnostics, not timed).
 * h_kv[i] = key | (uint64)value << 32; h_table[i] / h_bucket[i] (nullable) give
 * the subtable and bucket holding it.  Order is unspecified.  At most `cap`
 * entries are written; *n_out receives the number of live entries.
 * Synchronizes `stream`. */
dyc_status dyc_dump(dyc_table* t, uint64_t* h_kv, uint32_t* h_table, uint64_t* h_bucket,
                    uint64_t cap, uint64_t* n_out, dyc_stream_t stream);

/* Hash constants a_s, b_s for s = 0..d+1 (s=0 first layer, s=1..d subtables,
 * s=d+1 shard), each array of length >= d+2.  For cross-checking the hash
 * specification against test vectors. */
dyc_status dyc_hash_params(const dyc_table* t, uint64_t* a, uint64_t* b);

/* Evaluates the device hash for n keys (test vectors): d_x[n*(d+2)] receives
 * x_s(k) for s = 0..d+1, d_pair[2n] the ordered pair (t1, t2). */
dyc_status dyc_hash_probe(dyc_table* t, const uint32_t* d_keys, uint64_t n, uint32_t* d_x,
                          uint32_t* d_pair, dyc_stream_t stream);

/* Host-buffer variants (the end-to-end path): copy the inputs host->device,
 * run the batch, copy the outputs device->host and synchronize `stream`.
 * Staging buffers are owned by the table. */
dyc_status dyc_insert_batch_host(dyc_table* t, const uint32_t* h_keys, const uint32_t* h_values,
                                 uint8_t* h_status, uint64_t n, dyc_stream_t stream);
dyc_status dyc_find_batch_host(dyc_table* t, const uint32_t* h_keys, uint32_t* h_values_out,
                               uint8_t* h_found, uint64_t n, dyc_stream_t stream);
dyc_status dyc_delete_batch_host(dyc_table* t, const uint32_t* h_keys, uint32_t* h_values_out,
                                 uint8_t* h_status, uint64_t n, dyc_stream_t stream);

/* Kernel launch counter (for the bench's gpu_launches claim): number of kernels
 * this table has launched since creation or the last reset. */
uint64_t dyc_launch_count(const dyc_table* t, int reset);

/* Per-kernel timing with CUDA events recorded on the launching stream around
 * every kernel this table launches (measurement only; off by default).
 * dyc_profile_enable(t, 1) starts a fresh window; dyc_profile_read() waits for
 * the recorded events and reports, for each kernel kind k < DYC_PROF_KINDS,
 * the summed milliseconds ms[k] and launch count calls[k]. */
#define DYC_PROF_KINDS 16
enum {
    DYC_PROF_FIND = 0, DYC_PROF_UPSERT = 1, DYC_PROF_PLACE = 2, DYC_PROF_DELETE = 3,
    DYC_PROF_UPSIZE = 4, DYC_PROF_DOWNSIZE = 5, DYC_PROF_REINSERT = 6, DYC_PROF_OTHER = 7,
    DYC_PROF_ST_HIST = 8,     /* staged batches: first-choice buckets + chunk histogram, scan      */
    DYC_PROF_ST_SCATTER = 9,  /* staged batches: the two ordering passes (by bin, by chunk)        */
    DYC_PROF_ST_APPLY = 10,   /* staged batches: the per-chunk apply kernel                        */
    DYC_PROF_ST_UNPERM = 11   /* staged batches: need-list compaction, results to request order    */
};
dyc_status dyc_profile_enable(dyc_table* t, int enable);
dyc_status dyc_profile_read(dyc_table* t, double* ms, uint64_t* calls);

/* Probe accounting (measurement only; off by default, costs one extra atomic
 * per block).  While enabled, k_find, k_upsert and k_delete count the ops they
 * process and the second-bucket probes they issue.  dyc_probe_count_read
 * synchronizes the device, writes out6[6] = {find ops, find second probes,
 * upsert ops, upsert second probes, delete ops, delete second probes} (host
 * memory) and resets the counts.  The bench derives its algorithmic bytes per
 * op from these instead of from a model. */
dyc_status dyc_probe_count_enable(dyc_table* t, int enable);
dyc_status dyc_probe_count_read(dyc_table* t, uint64_t* out6);

/* The first-choice-full invariant (FFI; not in the paper): bit t
 * of *mask is set while every stored key whose first-choice subtable is t but
 * which lives in its second choice has a FULL bucket in t.  While it holds, a
 * key absent from a non-full first-choice bucket in t is absent from the
 * table, so find and the existence check of insert skip the second probe
 * (still <= 2 probes).  Set for every t by dyc_create / dyc_clear;
 * cleared for t by an upsize or a live resize of t, and for all t by a batch
 * that removed keys or a reinsert baseline (dyc_resize_ex
 * methods 1, 2).  Downsizes and placements preserve it.  Results never depend
 * on it, only the probe count does.  Batches on one table must not overlap in
 * time (one stream, or ordered by events): a delete running concurrently with
 * a find could make a bucket non-full under it. */
dyc_status dyc_clean_mask(const dyc_table* t, uint32_t* mask);

/* ---------------------------------------------------------------------------
 * Hash-partitioned sharding across G GPUs (build component C1).
 * shard(k) = x_{d+1}(k) mod G, independent of the pair and bucket hashes.
 * The exchange itself is an NCCL all-to-all issued by the caller (one process
 * per GPU, torch.distributed); these kernels do the data-parallel parts.
 * ------------------------------------------------------------------------- */

/* Counts ops per destination shard: d_counts[world] (uint64, device) receives
 * the histogram (world in 1..1024).  `t` supplies the hash constants (all ranks use one seed). */
dyc_status dyc_route_count(dyc_table* t, const uint32_t* d_keys, uint64_t n, uint32_t world,
                           uint64_t* d_counts, dyc_stream_t stream);

/* Groups the ops by destination shard: op i goes to position
 * offset[dest] + (rank of i among ops bound to dest) of d_keys_out / d_vals_out,
 * where offset is the exclusive prefix sum of d_counts[world] (the histogram
 * from dyc_route_count, computed on the device here).  d_cursor[world]
 * (uint64, device) is scratch.  d_vals_in and d_vals_out may be NULL
 * (finds/deletes).  d_tags_in / d_tags_out (nullable) carry a uint8 per op (the op
 * code of a mixed batch).  d_pos[i] (uint32) receives op i's position in the send
 * buffer, for dyc_route_unpermute.  Positions within one destination are in
 * unspecified order. */
dyc_status dyc_route_scatter(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_vals_in,
                             const uint8_t* d_tags_in, uint64_t n, uint32_t world, const uint64_t* d_counts,
                             uint64_t* d_cursor, uint32_t* d_keys_out, uint32_t* d_vals_out,
                             uint8_t* d_tags_out, uint32_t* d_pos, dyc_stream_t stream);

/* Gathers replies back into request order: d_vals[i] = d_reply_vals[d_pos[i]],
 * d_status[i] = d_reply_status[d_pos[i]] (either pair may be NULL). */
dyc_status dyc_route_unpermute(const uint32_t* d_pos, uint64_t n, const uint32_t* d_reply_vals,
                               const uint8_t* d_reply_status, uint32_t* d_vals,
                               uint8_t* d_status, dyc_stream_t stream);

/* ---------------------------------------------------------------------------
 * Sharded table: one process per GPU, each
 * owning `local_shards` complete DyCuckoo tables on its current device, G =
 * world * local_shards shards in all.  Key k belongs to shard
 * s = x_{d+1}(k) mod G (the (d+1)-th universal hash of P:L271, independent of
 * the pair and bucket hashes), owned by rank s / local_shards.  Each shard
 * resizes on its own.  The paper is single-GPU (P:L225 calls
 * host/device transfer orthogonal, commented); the batch calls keep its map
 * semantics (insert/find/delete) and batch model: since
 * keys are distinct within a batch and ops on different keys never interact,
 * every per-op result and the union of the shards' contents equal those of one
 * table given the same batches.
 *
 * Every rank calls the same dyc_dist_* batch function in the same order (a
 * collective; n may differ per rank, 0 included).  A batch groups its ops by
 * shard on the device (dyc_route_count/_scatter), exchanges the per-shard
 * counts and then keys [values, op codes] with grouped ncclSend/ncclRecv over
 * NVLink (one host read-back of the counts per batch), runs one ordinary batch
 * per local shard (so each shard takes its own resize decisions), sends the
 * results back and writes them in request order.  With world == 1 and no id
 * no NCCL is used (local virtual shards).  NCCL (libnccl.so.2) is loaded at run time.
 * Pointers, streams, status codes and preconditions are as for the
 * single-table calls; results for op i of the calling rank are written at
 * index i.  Errors: DYC_ERR_NCCL for a failed NCCL call (the table state is
 * then undefined), otherwise as for the single-table calls.
 * ------------------------------------------------------------------------- */
#define DYC_NCCL_UNIQUE_ID_BYTES 128
typedef struct dyc_dist dyc_dist;     /* opaque; owns its local shards, NCCL communicator, buffers */

/* ncclGetUniqueId into id[DYC_NCCL_UNIQUE_ID_BYTES] (host memory).  Rank 0
 * calls it and distributes the bytes to every rank out of band (e.g. a
 * torch.distributed broadcast).  Needs no GPU.  DYC_ERR_NCCL if NCCL cannot
 * be loaded. */
dyc_status dyc_dist_get_unique_id(void* id);

/* Creates this rank's part of a sharded table: local_shards tables with config
 * *cfg (the same on every rank, seed included) on the current device, and for
 * world > 1 an NCCL communicator from nccl_unique_id (NULL allowed when
 * world == 1: then nothing is exchanged; an id with world == 1 creates a
 * one-rank communicator and runs the exchange through NCCL to self).  Collective across the world.  dyc_dist_create uses the default
 * config with d, init_capacity (per shard), alpha, beta, and one local shard.
 * Errors: DYC_ERR_INVALID_ARG (rank outside [0, world), local_shards 0,
 * world*local_shards > 1024, world > 1 without an id, or a bad cfg),
 * DYC_ERR_NO_DEVICE, DYC_ERR_OOM, DYC_ERR_NCCL. */
dyc_status dyc_dist_create(uint32_t d, uint64_t init_capacity_per_shard, double alpha, double beta,
                           const void* nccl_unique_id, int rank, int world, dyc_dist** out);
dyc_status dyc_dist_create_ex(const dyc_config* cfg, const void* nccl_unique_id, int rank, int world,
                              uint32_t local_shards, dyc_dist** out);
/* Destroys the local shards and the communicator (synchronizes the device). */
dyc_status dyc_dist_destroy(dyc_dist* dist);

/* Sharded batches: as dyc_insert_batch / dyc_find_batch / dyc_delete_batch /
 * dyc_mixed_batch for the calling rank's n ops.  Each synchronizes `stream`
 * once for the routing counts (plus what the local shards' own batches do). */
dyc_status dyc_dist_insert_batch(dyc_dist* dist, const uint32_t* d_keys, const uint32_t* d_values,
                                 uint8_t* d_status, uint64_t n, dyc_stream_t stream);
dyc_status dyc_dist_find_batch(dyc_dist* dist, const uint32_t* d_keys, uint32_t* d_values_out,
                               uint8_t* d_found, uint64_t n, dyc_stream_t stream);
dyc_status dyc_dist_delete_batch(dyc_dist* dist, const uint32_t* d_keys, uint32_t* d_values_out,
                                 uint8_t* d_status, uint64_t n, dyc_stream_t stream);
dyc_status dyc_dist_mixed_batch(dyc_dist* dist, const uint8_t* d_ops, const uint32_t* d_keys,
                                const uint32_t* d_values, uint32_t* d_values_out, uint8_t* d_status,
                                uint64_t n, dyc_stream_t stream);
/* rank, world, local shards, and the number of ops this rank's shards executed
 * in the last batch (any pointer may be NULL). */
dyc_status dyc_dist_info(const dyc_dist* dist, int* rank, int* world, uint32_t* local_shards,
                         uint64_t* last_recv);
/* The table of local shard local_index (global shard rank*local_shards +
 * local_index), owned by dist: for dyc_stats / dyc_dump; do not destroy it or
 * run batches on it directly. */
dyc_status dyc_dist_shard(const dyc_dist* dist, uint32_t local_index, dyc_table** out);

/* ---------------------------------------------------------------------------
 * Fused routing over peer memory (S11).  Instead of
 * count -> exchange counts -> scatter -> all-to-all -> ... -> all-to-all ->
 * unpermute, the dispatch kernel hashes each op to its shard, reserves a range
 * in that shard's receive buffer with one system-scope atomic per (tile,
 * shard) and stores the op there directly; the combine kernel stores each
 * result at its op's index in the requester's result arrays.  Peer buffers are
 * plain cudaMalloc allocations shared through CUDA IPC (NVLink peer pointers
 * between GPUs of one node; the same calls work between processes on one GPU).
 * A receive buffer of capacity `cap` ops is structure-of-arrays, so the owner
 * runs its batch on the keys / values / op codes in place:
 *     keys u32[cap] at byte 0, values u32[cap] at 4*cap,
 *     meta u64[cap] at 8*cap (src_index | src_rank << 32), tags u8[cap] at 16*cap
 * (DYC_ROUTE_RECV_BYTES(cap) = 17*cap bytes).  The caller orders the phases
 * across ranks (dispatch on every rank, barrier, owner batch + combine,
 * barrier) and resets its receive counter between batches.
 * ------------------------------------------------------------------------- */
#define DYC_ROUTE_RECV_BYTES(cap) (17ull * (uint64_t)(cap))

/* Device buffer for IPC sharing: cudaMalloc of `bytes`, zero-filled (so a
 * receive counter starts at 0).  Owned by the caller; release with
 * dyc_ipc_free.  Errors: DYC_ERR_INVALID_ARG (bytes 0), DYC_ERR_OOM. */
dyc_status dyc_ipc_alloc(uint64_t bytes, void** d_ptr);
dyc_status dyc_ipc_free(void* d_ptr);
/* 64-byte cudaIpcMemHandle_t of a dyc_ipc_alloc buffer, written to handle64
 * (host); dyc_ipc_open maps a peer's handle (from another process) and returns
 * its device address; dyc_ipc_close unmaps it.  Both act on the current
 * device.  Errors: DYC_ERR_INVALID_ARG (null), DYC_ERR_CUDA. */
dyc_status dyc_ipc_get_handle(void* d_ptr, void* handle64);
dyc_status dyc_ipc_open(const void* handle64, void** d_ptr);
dyc_status dyc_ipc_close(void* d_ptr);

/* Dispatch: op i (d_keys[i], d_vals[i] or 0, d_tags[i] or 0) goes to shard
 * s = x_{d+1}(k) mod world (same hash as dyc_route_count): at position
 * g = atomicAdd_system(d_recv_count[s], ...) of receive buffer d_recv[s]
 * (layout above) it stores keys[g] = key, values[g] (if d_vals), meta[g] =
 * i | src_rank << 32, tags[g] (if d_tags).  d_recv and d_recv_count are HOST
 * arrays of `world` device pointers (peer or local): d_recv[s] holds recv_cap
 * ops, *d_recv_count[s] is a uint64 counter in shard s's memory.  Ops past
 * recv_cap are dropped; the owner detects *count > recv_cap and must treat the
 * batch as failed.  Order within a shard's buffer is unspecified.  d_vals,
 * d_tags nullable.  world 1..64, src_rank < world, n < 2^32; else
 * DYC_ERR_INVALID_ARG.  `t` supplies the hash constants (all ranks use one seed). */
dyc_status dyc_route_push(dyc_table* t, const uint32_t* d_keys, const uint32_t* d_vals, const uint8_t* d_tags,
                          uint64_t n, uint32_t world, uint32_t src_rank, void* const* d_recv,
                          uint64_t* const* d_recv_count, uint64_t recv_cap, dyc_stream_t stream);

/* Combine: for received op j < n of the local buffer d_recv (capacity
 * recv_cap, layout above) with meta[j] = i | r << 32, stores d_vals[j] into
 * d_out_vals[r][i] and d_status[j] into d_out_status[r][i].  d_out_vals /
 * d_out_status are HOST arrays of `world` device pointers (the requesters'
 * result arrays, peer or local); each pair (d_vals, d_out_vals), (d_status,
 * d_out_status) is both NULL or both given.  n <= recv_cap. */
dyc_status dyc_route_reply(const void* d_recv, uint64_t recv_cap, uint64_t n, const uint32_t* d_vals,
                           const uint8_t* d_status, uint32_t world, uint32_t* const* d_out_vals,
                           uint8_t* const* d_out_status, dyc_stream_t stream);

/* ---------------------------------------------------------------------------
 * Measurement helpers (bench.py; not part of the method).
 * ------------------------------------------------------------------------- */

/* Random-access ceiling: `n_reads` reads of one bucket of `bytes_per_read`
 * (32/64/128/256) bytes at uniformly random aligned offsets of d_buf[buf_bytes],
 * with the probe kernels' access pattern (bytes_per_read/32 lanes, one 256-bit
 * load each, same L2 prefetch size), XOR-reduced into *d_sink.  Bounds what
 * the probe kernels can reach. */
dyc_status dyc_bench_gather(const void* d_buf, uint64_t buf_bytes, uint64_t n_reads,
                            uint32_t bytes_per_read, uint64_t seed, uint64_t* d_sink,
                            dyc_stream_t stream);

/* dyc_bench_gather with flags: DYC_GATHER_WRITE (1) makes every read followed
 * by an 8-byte store into the bucket just read (the probe-then-write pattern of
 * delete: one random read plus one dirty-line write-back per op);
 * DYC_GATHER_CAS (2) makes it an 8-byte atomicCAS instead (insert's claim of a
 * free slot) and DYC_GATHER_SECTOR (4) a full 32-byte sector store (when
 * several are set the highest wins).  The written word depends only on the
 * group's own read.  d_buf is overwritten.  Errors: DYC_ERR_INVALID_ARG for
 * other flag bits or sizes as in dyc_bench_gather. */
#define DYC_GATHER_WRITE 1u
#define DYC_GATHER_CAS 2u
#define DYC_GATHER_SECTOR 4u
dyc_status dyc_bench_gather_ex(void* d_buf, uint64_t buf_bytes, uint64_t n_reads, uint32_t bytes_per_read,
                               uint64_t seed, uint32_t flags, uint64_t* d_sink, dyc_stream_t stream);

/* Device-wide L2 fetch granularity (cudaLimitMaxL2FetchGranularity, bytes in
 * 0..128, a hint) for the current device: how much the L2 pulls from HBM on a
 * sector miss.  Random 32-byte bucket probes want 32. */
dyc_status dyc_set_l2_fetch_granularity(uint32_t bytes);
dyc_status dyc_get_l2_fetch_granularity(uint32_t* bytes);

/* Thread-local message for the last error returned on this thread. */
const char* dyc_last_error(void);

/* Library version string. */
const char* dyc_version(void);

#ifdef __cplusplus
}
#endif

#endif /* DYCUCKOO_H */
