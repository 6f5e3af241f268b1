/*
 * dyc_oracle.c — sequential CPU DyCuckoo oracle.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / `--impl reference` leg may load, link or execute this file.  It
 * shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_icde_lizlhs21_b200/csrc); the two meet only through the seeded
 * inputs of paper_conf_icde_lizlhs21_b200/workload.py and through the hash
 * *specification* written down in DESIGN.md §2 (each side implements it on its
 * own; test vectors cross-check them).
 *
 * It is a plain, slow, obviously-sequential rendering of the method in
 * PAPER.md ("Dynamic Hash Tables on GPUs", Li et al., ICDE'21).  P:L<n> is a
 * line of PAPER.md; Qn is a reading listed in DESIGN.md §4.
 *
 *   map semantics  insert/find/delete ........... P:L188-189 (§II-A)
 *   d subtables, fill factor θ = Σm_i / Σn_i ..... P:L194-196 (§II-A)
 *   universal hash h^i(k)=((a_i k+b_i) mod p) mod |h^i|   P:L270-273 (§IV-A)
 *   resize: double smallest / halve largest ...... P:L305-312 (§IV-B)
 *   upsize split b -> {b, b+|h^i|} ............... P:L374-382 (§IV-D)
 *   downsize merge + residuals (exclude t) ........ P:L387-395 (§IV-D)
 *   two-layer: pair of tables, ≤2 lookups ........ P:L440-441 (§V-A)
 *   eviction goes to the partner of the victim ... P:L443-445 (Example 1)
 *   upsert on existing key ........................ Alg. 1
 *   delete erases on match, no lock .............. P:L591-592
 *   failure → resize ............................. P:L737
 *
 * Parity status: the map semantics (statuses, find values, contents) and the
 * resize schedule (subtable sizes after every batch) are pinned by tests
 * (tests/test_oracle_*.py).  Victim choice, slot positions, φ and eviction
 * counts are placement-only and nondeterministic on the GPU: "parity unpinned"
 * for those outputs (they are reported as statistics only).
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define DYO_P        4294967291ULL   /* 2^32 - 5, the largest 32-bit prime (Q1) */
#define DYO_EMPTY    0xFFFFFFFFu     /* reserved key marking a free slot (Q25) */
#define DYO_DMAX     16
#define DYO_OK       0
#define DYO_FAIL     1

enum { DYO_ST_NONE = 0, DYO_ST_INSERTED = 1, DYO_ST_UPDATED = 2 };
enum { DYO_POLICY_FIRST_FIT = 0, DYO_POLICY_PAPER_WEIGHTED = 1 };

typedef struct { uint32_t key, val; } dyo_slot;

typedef struct {
    uint64_t m, N;                      /* live keys, total slots */
    uint32_t d, B;
    uint64_t buckets[DYO_DMAX];         /* |h^t| */
    uint64_t count[DYO_DMAX];           /* m_t   */
    uint64_t n_upsize, n_downsize, n_fail_upsize, n_residual, n_evict;
    uint64_t max_probes, n_second_table; /* probes per find/delete (I7), keys in 2nd choice */
    uint64_t invariant_errors;
} dyo_stats_t;

typedef struct dyo_table {
    uint32_t d, B, L_max, policy;
    double alpha, beta;
    uint64_t a[DYO_DMAX + 2], b[DYO_DMAX + 2];  /* s=0 pair, s=1..d tables, s=d+1 shard */
    uint64_t n[DYO_DMAX];                        /* buckets per subtable */
    uint64_t m_t[DYO_DMAX];
    dyo_slot *tab[DYO_DMAX];
    uint64_t rng;                                /* victim-choice RNG state */
    uint64_t n_upsize, n_downsize, n_fail_upsize, n_residual, n_evict, max_probes;
    uint64_t invariant_errors;
    char last_error[256];
} dyo_table;

/* ---------------------------------------------------------------- hashing */

/* SplitMix64 (Steele, Lea, Flood 2014): the counter-based generator both sides
 * implement independently to draw a_s, b_s from the user seed (Q1). */
static uint64_t splitmix64(uint64_t *state)
{
    uint64_t z = (*state += 0x9E3779B97F4A7C15ULL);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* x_s(k) = ((a_s * k mod p) + b_s) mod p — the universal hash of P:L271 before
 * its final "mod |h^i|".  a_s < p < 2^32 and k < 2^32, so a_s*k < 2^64 is exact. */
static uint64_t hash_x(const dyo_table *T, uint32_t s, uint32_t k)
{
    uint64_t ak = (T->a[s] * (uint64_t)k) % DYO_P;
    return (ak + T->b[s]) % DYO_P;
}

/* First layer: the ordered pair (t1, t2), t1 != t2, of candidate
 * subtables.  Reading Q2: q = x_0(k) mod d(d-1); t1 = q div (d-1); t2 is the
 * (q mod (d-1))-th of the other d-1 tables.  t1 is tried first. */
static void pair_of(const dyo_table *T, uint32_t k, uint32_t *t1, uint32_t *t2)
{
    uint64_t q = hash_x(T, 0, k) % ((uint64_t)T->d * (T->d - 1));
    uint32_t first = (uint32_t)(q / (T->d - 1));
    uint32_t r = (uint32_t)(q % (T->d - 1));
    *t1 = first;
    *t2 = (r < first) ? r : r + 1;
}

/* Second layer: bucket of k in subtable t, h^t(k) = x_{t+1}(k) mod |h^t|. */
static uint64_t bucket_of(const dyo_table *T, uint32_t t, uint32_t k)
{
    return hash_x(T, t + 1, k) % T->n[t];
}

/* The other table of k's pair, given one of them ("(k',v') is hashed to
 * the pair (h_i,h_t) ... we insert (k',v') to h_t"). */
static uint32_t partner_of(const dyo_table *T, uint32_t k, uint32_t t)
{
    uint32_t t1, t2;
    pair_of(T, k, &t1, &t2);
    return (t == t1) ? t2 : t1;
}

static dyo_slot *bucket_ptr(const dyo_table *T, uint32_t t, uint64_t b)
{
    return T->tab[t] + b * T->B;
}

static uint64_t total_slots(const dyo_table *T)
{
    uint64_t N = 0;
    for (uint32_t t = 0; t < T->d; t++) N += T->n[t] * T->B;
    return N;
}

static uint64_t total_keys(const dyo_table *T)
{
    uint64_t m = 0;
    for (uint32_t t = 0; t < T->d; t++) m += T->m_t[t];
    return m;
}

static void set_error(dyo_table *T, const char *msg)
{
    T->invariant_errors++;
    snprintf(T->last_error, sizeof T->last_error, "%s", msg);
}

/* ---------------------------------------------------------------- lookup */

/* Find the slot holding k among the two candidate buckets (at most two lookups,
 * P:L145; reading Q21: only the two candidates are scanned). */
static dyo_slot *lookup(dyo_table *T, uint32_t k, uint32_t *probes)
{
    uint32_t t1, t2;
    pair_of(T, k, &t1, &t2);
    uint32_t cand[2] = { t1, t2 };
    *probes = 0;
    for (int c = 0; c < 2; c++) {
        dyo_slot *bk = bucket_ptr(T, cand[c], bucket_of(T, cand[c], k));
        (*probes)++;
        for (uint32_t s = 0; s < T->B; s++)
            if (bk[s].key == k) return &bk[s];
    }
    return NULL;
}

static int bucket_store_if_free(dyo_table *T, uint32_t t, dyo_slot kv)
{
    dyo_slot *bk = bucket_ptr(T, t, bucket_of(T, t, kv.key));
    for (uint32_t s = 0; s < T->B; s++) {
        if (bk[s].key == DYO_EMPTY) {
            bk[s] = kv;
            T->m_t[t]++;
            return 1;
        }
    }
    return 0;
}

/* ---------------------------------------------------------------- placement */

/* binom(m,2) guarded to >= 1 (reading Q3 for the paper's weighted rule). */
static double pairs_guarded(uint64_t m)
{
    double c = (double)m * ((double)m - 1.0) / 2.0;
    return c < 1.0 ? 1.0 : c;
}

/* place(kv, exclude, start): cuckoo insertion of a key known to be absent.
 *
 * Initial table (reading Q3): first-fit over the ordered pair (t1 then t2);
 * with DYO_POLICY_PAPER_WEIGHTED the first table is drawn with probability
 * proportional to n_i / binom(m_i, 2).  When both candidate
 * buckets are full the first eviction happens in t1 (Example 1).
 * Each hop: if the bucket has a free slot, store and stop; otherwise swap with
 * a victim slot (pseudo-random, Q5) and continue with the victim in the other
 * table of the VICTIM's pair.  Victims whose partner is
 * `exclude` are never chosen (downsize residuals).  After L_max hops
 * (Q6) the homeless pair is returned through *homeless and DYO_FAIL is
 * returned: the caller must keep it (never dropped, Q17). */
static int place(dyo_table *T, dyo_slot kv, int exclude, int start, dyo_slot *homeless)
{
    dyo_slot cur = kv;
    uint32_t t;
    if (start >= 0) {
        t = (uint32_t)start;
    } else {
        uint32_t t1, t2;
        pair_of(T, cur.key, &t1, &t2);
        if (T->policy == DYO_POLICY_PAPER_WEIGHTED) {
            double w1 = (double)T->n[t1] / pairs_guarded(T->m_t[t1]);
            double w2 = (double)T->n[t2] / pairs_guarded(T->m_t[t2]);
            double u = (double)(splitmix64(&T->rng) >> 11) / 9007199254740992.0;
            t = (u * (w1 + w2) < w1) ? t1 : t2;
        } else {
            if ((int)t1 != exclude && bucket_store_if_free(T, t1, cur)) return DYO_OK;
            if ((int)t2 != exclude && bucket_store_if_free(T, t2, cur)) return DYO_OK;
            t = ((int)t1 != exclude) ? t1 : t2;
        }
    }
    for (uint32_t hop = 0; hop <= T->L_max; hop++) {
        if (bucket_store_if_free(T, t, cur)) return DYO_OK;
        if (hop == T->L_max) break;
        dyo_slot *bk = bucket_ptr(T, t, bucket_of(T, t, cur.key));
        /* candidate victims: slots whose key may legally move to its partner */
        uint32_t legal[64], nl = 0;
        for (uint32_t s = 0; s < T->B; s++)
            if ((int)partner_of(T, bk[s].key, t) != exclude) legal[nl++] = s;
        if (nl == 0) break;
        uint32_t s = legal[splitmix64(&T->rng) % nl];
        dyo_slot victim = bk[s];
        bk[s] = cur;                 /* swap(loc[l*], (k',v')), Alg. 1 */
        cur = victim;
        T->n_evict++;
        t = partner_of(T, cur.key, t);
    }
    /* cur is homeless; it was taken out of table t's accounting if it was a victim */
    *homeless = cur;
    return DYO_FAIL;
}

/* ---------------------------------------------------------------- resizing */

static int smallest_table(const dyo_table *T)
{
    uint32_t best = 0;                          /* ties -> lowest index (Q12) */
    for (uint32_t t = 1; t < T->d; t++)
        if (T->n[t] < T->n[best]) best = t;
    return (int)best;
}

static int largest_table(const dyo_table *T)
{
    uint32_t best = T->d - 1;                   /* ties -> highest index (Q12) */
    for (int t = (int)T->d - 2; t >= 0; t--)
        if (T->n[t] > T->n[best]) best = (uint32_t)t;
    return (int)best;
}

/* Upsize subtable t: |h^t| doubles; an entry of old bucket b goes
 * to b or b+|h^t| (checked: invariant I8).  Returns 0, or -1 on OOM. */
static int upsize_table(dyo_table *T, uint32_t t)
{
    uint64_t n_old = T->n[t], n_new = 2 * n_old;
    dyo_slot *nt = (dyo_slot *)malloc(n_new * T->B * sizeof(dyo_slot));
    if (!nt) return -1;
    for (uint64_t i = 0; i < n_new * T->B; i++) { nt[i].key = DYO_EMPTY; nt[i].val = DYO_EMPTY; }
    uint64_t *fill = (uint64_t *)calloc(n_new, sizeof(uint64_t));
    if (!fill) { free(nt); return -1; }
    uint64_t moved = 0;
    for (uint64_t b = 0; b < n_old; b++) {
        for (uint32_t s = 0; s < T->B; s++) {
            dyo_slot e = T->tab[t][b * T->B + s];
            if (e.key == DYO_EMPTY) continue;
            uint64_t nb = hash_x(T, t + 1, e.key) % n_new;
            if (nb != b && nb != b + n_old) set_error(T, "I8: upsize moved an entry outside {b, b+n}");
            if (fill[nb] >= T->B) { set_error(T, "I8: upsize bucket overflow"); continue; }
            nt[nb * T->B + fill[nb]++] = e;
            moved++;
        }
    }
    if (moved != T->m_t[t]) set_error(T, "I8: upsize did not move exactly m_t entries");
    free(fill);
    free(T->tab[t]);
    T->tab[t] = nt;
    T->n[t] = n_new;
    T->n_upsize++;
    return 0;
}

static int upsize(dyo_table *T)
{
    return upsize_table(T, (uint32_t)smallest_table(T));
}

static void settle_homeless(dyo_table *T, dyo_slot *list, uint64_t cnt);

/* Downsize subtable t: |h^t| halves; new bucket b' receives the
 * entries of old b' then old b'+h; the first B stay (reading Q18), the rest are
 * residuals inserted into the other table of their pair, never into t
 * (P:L392-395).  Residual count is checked against Σ max(0, |b'|+|b'+h|-B) (I9). */
static int downsize_table(dyo_table *T, uint32_t t)
{
    uint64_t n_old = T->n[t], h = n_old / 2;
    if (n_old < 2 || (n_old & 1)) return -1;
    dyo_slot *nt = (dyo_slot *)malloc(h * T->B * sizeof(dyo_slot));
    dyo_slot *res = (dyo_slot *)malloc(2 * h * T->B * sizeof(dyo_slot) + sizeof(dyo_slot));
    if (!nt || !res) { free(nt); free(res); return -1; }
    uint64_t nres = 0, expect_res = 0;
    for (uint64_t bp = 0; bp < h; bp++) {
        uint32_t kept = 0, occupied = 0;
        for (int half = 0; half < 2; half++) {
            uint64_t ob = bp + (half ? h : 0);
            for (uint32_t s = 0; s < T->B; s++) {
                dyo_slot e = T->tab[t][ob * T->B + s];
                if (e.key == DYO_EMPTY) continue;
                occupied++;
                if (hash_x(T, t + 1, e.key) % h != bp) set_error(T, "downsize: entry not hashed to merged bucket");
                if (kept < T->B) nt[bp * T->B + kept++] = e;
                else res[nres++] = e;
            }
        }
        for (uint32_t s = kept; s < T->B; s++) { nt[bp * T->B + s].key = DYO_EMPTY; nt[bp * T->B + s].val = DYO_EMPTY; }
        if (occupied > T->B) expect_res += occupied - T->B;
    }
    if (nres != expect_res) set_error(T, "I9: residual count mismatch");
    free(T->tab[t]);
    T->tab[t] = nt;
    T->n[t] = h;
    T->m_t[t] -= nres;
    T->n_downsize++;
    T->n_residual += nres;
    /* residuals go to the partner table, excluding t */
    dyo_slot *homeless = (dyo_slot *)malloc((nres + 1) * sizeof(dyo_slot));
    uint64_t nh = 0;
    for (uint64_t i = 0; i < nres; i++) {
        dyo_slot hl;
        if (place(T, res[i], (int)t, (int)partner_of(T, res[i].key, t), &hl) != DYO_OK)
            homeless[nh++] = hl;
    }
    free(res);
    /* the downsize is complete: any homeless residual is settled like a failed
     * insert (retry without exclusion, then failure-triggered upsize; Q17) */
    settle_homeless(T, homeless, nh);
    free(homeless);
    return 0;
}

/* Failure path (Q6, Q17): retry each homeless pair; if it
 * fails again, upsize the smallest subtable and retry until it is placed. */
static void settle_homeless(dyo_table *T, dyo_slot *list, uint64_t cnt)
{
    for (uint64_t i = 0; i < cnt; i++) {
        dyo_slot cur = list[i];
        for (;;) {
            dyo_slot hl;
            if (place(T, cur, -1, -1, &hl) == DYO_OK) break;
            cur = hl;
            T->n_fail_upsize++;
            if (upsize(T) != 0) { set_error(T, "out of memory in failure upsize"); return; }
        }
    }
}

/* Lower bound (readings Q11-Q13): while θ < α halve the largest
 * subtable, unless it cannot be halved (odd or a single bucket) or the halving
 * would push θ above β. */
static void enforce_lower(dyo_table *T)
{
    for (;;) {
        uint64_t m = total_keys(T), N = total_slots(T);
        if (!((double)m < T->alpha * (double)N)) break;
        int t = largest_table(T);
        if (T->n[t] < 2 || (T->n[t] & 1)) break;
        uint64_t N_after = N - (T->n[t] / 2) * T->B;
        if ((double)m > T->beta * (double)N_after) break;
        uint64_t fails_before = T->n_fail_upsize;
        downsize_table(T, (uint32_t)t);
        /* reading Q17b: residuals that needed a failure-triggered upsize end the
         * α loop for this batch (otherwise halve/double could cycle forever) */
        if (T->n_fail_upsize != fails_before) break;
    }
}

/* ---------------------------------------------------------------- public API */

dyo_table *dyo_create(uint32_t d, uint32_t B, uint64_t init_capacity, double alpha, double beta,
                      uint64_t seed, uint32_t L_max, uint32_t policy)
{
    if (d < 2 || d > DYO_DMAX || B < 1 || B > 64) return NULL;
    if (!(alpha > 0.0 && alpha < beta && beta < 1.0)) return NULL;
    if (alpha > beta * (double)d / (double)(d + 1)) return NULL;  /* Q14: α ≤ βd/(d+1) */
    dyo_table *T = (dyo_table *)calloc(1, sizeof(dyo_table));
    if (!T) return NULL;
    T->d = d; T->B = B; T->L_max = L_max; T->policy = policy;
    T->alpha = alpha; T->beta = beta;
    uint64_t st = seed;
    for (uint32_t s = 0; s < d + 2; s++) {
        T->a[s] = 1 + splitmix64(&st) % (DYO_P - 1);   /* a_s in [1, p) */
        T->b[s] = splitmix64(&st) % DYO_P;             /* b_s in [0, p) */
    }
    T->rng = seed ^ 0xA5A5A5A5DEADBEEFULL;
    uint64_t per = (init_capacity + (uint64_t)d * B - 1) / ((uint64_t)d * B);  /* Q13 */
    if (per < 1) per = 1;
    for (uint32_t t = 0; t < d; t++) {
        T->n[t] = per;
        T->tab[t] = (dyo_slot *)malloc(per * B * sizeof(dyo_slot));
        if (!T->tab[t]) return NULL;
        for (uint64_t i = 0; i < per * B; i++) { T->tab[t][i].key = DYO_EMPTY; T->tab[t][i].val = DYO_EMPTY; }
    }
    return T;
}

void dyo_destroy(dyo_table *T)
{
    if (!T) return;
    for (uint32_t t = 0; t < T->d; t++) free(T->tab[t]);
    free(T);
}

static int cmp_u32(const void *x, const void *y)
{
    uint32_t a = *(const uint32_t *)x, b = *(const uint32_t *)y;
    return (a > b) - (a < b);
}

/* insert_batch (P:L464 one op type per batch; Alg. 1 semantics; Q7-Q11):
 * n_new = distinct absent keys; upsize while (m + n_new) > β·N; then insert the
 * ops in batch order (upsert or place); settle failures; then the α check. */
void dyo_insert_batch(dyo_table *T, const uint32_t *keys, const uint32_t *vals, uint8_t *status, uint64_t n)
{
    if (n == 0) return;   /* reading Q32: an empty batch is a no-op (no resize check) */
    uint32_t *sorted = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    memcpy(sorted, keys, n * sizeof(uint32_t));
    qsort(sorted, n, sizeof(uint32_t), cmp_u32);
    uint64_t n_new = 0;
    for (uint64_t i = 0; i < n; i++) {
        if (sorted[i] == DYO_EMPTY) continue;
        if (i > 0 && sorted[i] == sorted[i - 1]) continue;
        uint32_t pr;
        if (!lookup(T, sorted[i], &pr)) n_new++;
    }
    free(sorted);
    while ((double)(total_keys(T) + n_new) > T->beta * (double)total_slots(T))
        if (upsize(T) != 0) { set_error(T, "out of memory in upsize"); return; }

    for (uint64_t i = 0; i < n; i++) {
        uint32_t k = keys[i], pr;
        if (k == DYO_EMPTY) { if (status) status[i] = DYO_ST_NONE; continue; }
        dyo_slot *sl = lookup(T, k, &pr);
        if (sl) {                                  /* Alg. 1: key == k' -> overwrite */
            sl->val = vals[i];
            if (status) status[i] = DYO_ST_UPDATED;
            continue;
        }
        dyo_slot kv = { k, vals[i] }, hl;
        /* a failed chain leaves some pair homeless; settle it before the next op
         * so that op's lookup sees every key (no duplicate, no loss; Q17) */
        if (place(T, kv, -1, -1, &hl) != DYO_OK) settle_homeless(T, &hl, 1);
        if (status) status[i] = DYO_ST_INSERTED;
    }
    enforce_lower(T);
}

/* find_batch: value or NULL (reading Q25: 0xFFFFFFFF, found = 0). */
void dyo_find_batch(dyo_table *T, const uint32_t *keys, uint32_t *vals_out, uint8_t *found, uint64_t n)
{
    for (uint64_t i = 0; i < n; i++) {
        uint32_t pr = 0;
        dyo_slot *sl = (keys[i] == DYO_EMPTY) ? NULL : lookup(T, keys[i], &pr);
        if (pr > T->max_probes) T->max_probes = pr;
        if (vals_out) vals_out[i] = sl ? sl->val : DYO_EMPTY;
        if (found) found[i] = sl ? 1 : 0;
    }
}

/* delete_batch: erase on match; then the α check. */
void dyo_delete_batch(dyo_table *T, const uint32_t *keys, uint32_t *old_vals, uint8_t *status, uint64_t n)
{
    if (n == 0) return;   /* reading Q32 */
    for (uint64_t i = 0; i < n; i++) {
        uint32_t pr = 0;
        dyo_slot *sl = (keys[i] == DYO_EMPTY) ? NULL : lookup(T, keys[i], &pr);
        if (pr > T->max_probes) T->max_probes = pr;
        if (old_vals) old_vals[i] = sl ? sl->val : DYO_EMPTY;
        if (status) status[i] = sl ? 1 : 0;
        if (sl) {
            uint32_t t1, t2;
            pair_of(T, keys[i], &t1, &t2);
            /* which table held it: the slot lies inside exactly one table array */
            uint32_t t = (sl >= T->tab[t1] && sl < T->tab[t1] + T->n[t1] * T->B) ? t1 : t2;
            sl->key = DYO_EMPTY;
            sl->val = DYO_EMPTY;
            T->m_t[t]--;
        }
    }
    enforce_lower(T);
}

/* Mixed batch (configs C4/C5).  The paper batches one op type at a time
 * and calls mixed batches ambiguous (commented).  Reading Q10: keys are
 * distinct across the batch; the finds run first (they see the table before the
 * batch), then the inserts, then the deletes, each as a single-type batch in
 * request order.  ops[i]: 0 find, 1 insert, 2 delete.  vals_out[i]: the found /
 * removed value, 0xFFFFFFFF on a miss and for inserts; status[i]: the op's code. */
void dyo_mixed_batch(dyo_table *T, const uint8_t *ops, const uint32_t *keys, const uint32_t *vals,
                     uint32_t *vals_out, uint8_t *status, uint64_t n)
{
    uint64_t *idx = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    uint32_t *k = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    uint32_t *v = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    uint32_t *ov = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    uint8_t *st = (uint8_t *)malloc(n + 1);
    /* an op code outside 0..2 is no operation: status NONE, value NOT_FOUND
       (reading Q10) */
    for (uint64_t i = 0; i < n; i++)
        if (ops[i] > 2) {
            if (vals_out) vals_out[i] = DYO_EMPTY;
            if (status) status[i] = 0;
        }
    for (uint8_t op = 0; op < 3; op++) {
        uint64_t c = 0;
        for (uint64_t i = 0; i < n; i++)
            if (ops[i] == op) { idx[c] = i; k[c] = keys[i]; v[c] = vals ? vals[i] : 0; c++; }
        if (c == 0) continue;
        if (op == 0) dyo_find_batch(T, k, ov, st, c);
        else if (op == 1) { dyo_insert_batch(T, k, v, st, c); for (uint64_t j = 0; j < c; j++) ov[j] = DYO_EMPTY; }
        else dyo_delete_batch(T, k, ov, st, c);
        for (uint64_t j = 0; j < c; j++) {
            if (vals_out) vals_out[idx[j]] = ov[j];
            if (status) status[idx[j]] = st[j];
        }
    }
    free(idx); free(k); free(v); free(ov); free(st);
}

/* Explicit resize (dyc_resize analogue): direction +1 upsizes (the smallest, or
 * `t` if given), -1 downsizes (the largest, or `t`).  A choice that would break
 * "no subtable more than double any other" (I6) is refused (-1). */
int dyo_resize(dyo_table *T, int direction, int t)
{
    if (direction > 0) {
        if (t < 0) t = smallest_table(T);
        if (t >= (int)T->d) return -1;
        if (T->n[t] != T->n[smallest_table(T)]) return -1;   /* only a smallest may double */
        return upsize_table(T, (uint32_t)t);
    }
    if (direction < 0) {
        if (t < 0) t = largest_table(T);
        if (t >= (int)T->d) return -1;
        if (T->n[t] != T->n[largest_table(T)]) return -1;    /* only a largest may halve */
        if (T->n[t] < 2 || (T->n[t] & 1)) return -1;
        return downsize_table(T, (uint32_t)t);
    }
    return 0;
}

void dyo_stats(const dyo_table *T, dyo_stats_t *S)
{
    memset(S, 0, sizeof *S);
    S->d = T->d; S->B = T->B;
    S->m = total_keys(T); S->N = total_slots(T);
    for (uint32_t t = 0; t < T->d; t++) { S->buckets[t] = T->n[t]; S->count[t] = T->m_t[t]; }
    S->n_upsize = T->n_upsize; S->n_downsize = T->n_downsize; S->n_fail_upsize = T->n_fail_upsize;
    S->n_residual = T->n_residual; S->n_evict = T->n_evict; S->max_probes = T->max_probes;
    S->invariant_errors = T->invariant_errors;
    uint64_t second = 0;
    for (uint32_t t = 0; t < T->d; t++)
        for (uint64_t i = 0; i < T->n[t] * T->B; i++) {
            uint32_t k = T->tab[t][i].key, t1, t2;
            if (k == DYO_EMPTY) continue;
            pair_of(T, k, &t1, &t2);
            if (t == t2) second++;
        }
    S->n_second_table = second;
}

/* Contents with positions: kv = key | (uint64)val << 32, table, bucket. */
uint64_t dyo_dump(const dyo_table *T, uint64_t *kv, uint32_t *table, uint64_t *bucket, uint64_t cap)
{
    uint64_t c = 0;
    for (uint32_t t = 0; t < T->d; t++)
        for (uint64_t i = 0; i < T->n[t] * T->B; i++) {
            dyo_slot e = T->tab[t][i];
            if (e.key == DYO_EMPTY) continue;
            if (c < cap) {
                if (kv) kv[c] = (uint64_t)e.key | ((uint64_t)e.val << 32);
                if (table) table[c] = t;
                if (bucket) bucket[c] = i / T->B;
            }
            c++;
        }
    return c;
}

/* Invariants I1, I2, I4, I5 (upper bound), I6 over the oracle's own state.
 * Returns the number of violations; the first message goes to msg. */
uint64_t dyo_check_invariants(dyo_table *T, char *msg, uint64_t msglen)
{
    uint64_t bad = 0, m = 0, N = total_slots(T);
    const char *first = NULL;
    uint64_t nkeys = total_keys(T);
    uint32_t *all = (uint32_t *)malloc((nkeys + 1) * sizeof(uint32_t));
    uint64_t na = 0;
    for (uint32_t t = 0; t < T->d; t++) {
        uint64_t occ = 0;
        for (uint64_t i = 0; i < T->n[t] * T->B; i++) {
            uint32_t k = T->tab[t][i].key, t1, t2;
            if (k == DYO_EMPTY) continue;
            occ++;
            pair_of(T, k, &t1, &t2);
            if (t != t1 && t != t2) { bad++; if (!first) first = "I1: key in a table outside its pair"; }
            if (bucket_of(T, t, k) != i / T->B) { bad++; if (!first) first = "I1: key in the wrong bucket"; }
            if (na <= nkeys) all[na++] = k;
        }
        if (occ != T->m_t[t]) { bad++; if (!first) first = "I4: counter != occupancy"; }
        m += occ;
    }
    qsort(all, na, sizeof(uint32_t), cmp_u32);
    for (uint64_t i = 1; i < na; i++)
        if (all[i] == all[i - 1]) { bad++; if (!first) first = "I2: duplicate key"; }
    free(all);
    if ((double)m > T->beta * (double)N) { bad++; if (!first) first = "I5: fill above beta"; }
    /* the lower bound α is enforced after mutating batches only (a fresh table
     * or a find batch may sit below α); tests check it there */
    uint64_t mn = T->n[0], mx = T->n[0];
    for (uint32_t t = 1; t < T->d; t++) { if (T->n[t] < mn) mn = T->n[t]; if (T->n[t] > mx) mx = T->n[t]; }
    if (mx > 2 * mn) { bad++; if (!first) first = "I6: a subtable more than double another"; }
    if (T->invariant_errors) { bad += T->invariant_errors; if (!first) first = T->last_error; }
    if (msg && msglen) snprintf(msg, msglen, "%s", first ? first : "ok");
    return bad;
}

/* Hash exposure for test vectors and layout checks. */
uint64_t dyo_hash_x(const dyo_table *T, uint32_t s, uint32_t k) { return hash_x(T, s, k); }
void dyo_pair(const dyo_table *T, uint32_t k, uint32_t *t1, uint32_t *t2) { pair_of(T, k, t1, t2); }
uint64_t dyo_bucket(const dyo_table *T, uint32_t t, uint32_t k) { return bucket_of(T, t, k); }
void dyo_hash_params(const dyo_table *T, uint64_t *a, uint64_t *b)
{
    for (uint32_t s = 0; s < T->d + 2; s++) { a[s] = T->a[s]; b[s] = T->b[s]; }
}

/* Check a layout produced elsewhere (the GPU dump) against I1/I2 using this
 * oracle's hash: entry i is key[i] stored in subtable table[i], bucket bucket[i]
 * of a table whose subtables have nb[t] buckets.  Returns the violation count. */
uint64_t dyo_check_layout(const dyo_table *T, const uint64_t *nb, const uint32_t *keys,
                          const uint32_t *table, const uint64_t *bucket, uint64_t count)
{
    uint64_t bad = 0;
    for (uint64_t i = 0; i < count; i++) {
        uint32_t k = keys[i], t1, t2, t = table[i];
        pair_of(T, k, &t1, &t2);
        if (t != t1 && t != t2) { bad++; continue; }
        if (hash_x(T, t + 1, k) % nb[t] != bucket[i]) bad++;
    }
    uint32_t *s = (uint32_t *)malloc((count + 1) * sizeof(uint32_t));
    memcpy(s, keys, count * sizeof(uint32_t));
    qsort(s, count, sizeof(uint32_t), cmp_u32);
    for (uint64_t i = 1; i < count; i++) if (s[i] == s[i - 1]) bad++;
    free(s);
    return bad;
}

/* Test-only hooks for scripted scenarios (Examples 1 and 2): write a pair into
 * a chosen slot / read a slot. */
int dyo_poke(dyo_table *T, uint32_t t, uint64_t b, uint32_t s, uint32_t key, uint32_t val)
{
    if (t >= T->d || b >= T->n[t] || s >= T->B) return -1;
    dyo_slot *sl = &T->tab[t][b * T->B + s];
    if (sl->key == DYO_EMPTY && key != DYO_EMPTY) T->m_t[t]++;
    if (sl->key != DYO_EMPTY && key == DYO_EMPTY) T->m_t[t]--;
    sl->key = key; sl->val = val;
    return 0;
}

uint64_t dyo_peek(const dyo_table *T, uint32_t t, uint64_t b, uint32_t s)
{
    dyo_slot e = T->tab[t][b * T->B + s];
    return (uint64_t)e.key | ((uint64_t)e.val << 32);
}

/* Sequential place() of a single absent pair, exposing the eviction rule for
 * Example 1.  Returns DYO_OK or DYO_FAIL. */
int dyo_place_one(dyo_table *T, uint32_t key, uint32_t val)
{
    dyo_slot kv = { key, val }, hl;
    int r = place(T, kv, -1, -1, &hl);
    if (r != DYO_OK) settle_homeless(T, &hl, 1);
    return r;
}

/* Test-only hook for the negative pins of dyo_check_invariants (I4): shift the
 * per-subtable counter m_t by delta without touching the slots. */
int dyo_debug_adjust_count(dyo_table *T, uint32_t t, int64_t delta)
{
    if (t >= T->d) return -1;
    T->m_t[t] = (uint64_t)((int64_t)T->m_t[t] + delta);
    return 0;
}
