/*
 * dyw_oracle.c — sequential CPU oracle of the WIDE-key DyCuckoo variant
 * (8-byte keys, values wider than 32 bits).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / `--impl reference` leg may load, link or execute this file.  It
 * shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_icde_lizlhs21_b200/csrc); the two meet only through seeded inputs
 * and through the hash *specification* of DESIGN.md §2 / reading Q33, which
 * each side implements on its own (test vectors cross-check them).
 *
 * It is the narrow oracle (dyc_oracle.c) with the key widened to 64 bits and the
 * value to W 64-bit words, as the paper allows ("Suppose the keys
 * are 8-bytes, a bucket can then accommodate 16 KV pairs ... we do not limit
 * ourselves to supporting KV pairs with only 64 bits").  The structure and the
 * policies are the same and cite the same passages:
 *
 *   map semantics insert/find/delete ............. P:L188-189
 *   hash: x_s(k) = (c_s*hi(k) + a_s*lo(k) + b_s) mod p ... P:L270-273, Q1, Q33
 *   resize: double smallest / halve largest ....... P:L305-312, Q11-Q13
 *   upsize split, downsize merge + residuals ...... P:L374-395
 *   two-layer pair, <= 2 lookups .................. P:L440-441, Q2
 *   eviction to the victim's partner .............. P:L443-445
 *   upsert on an existing key ..................... Alg. 1, Q7/Q8
 *   delete erases on match ........................ P:L591-592
 *   failure -> retry -> upsize .................... P:L737, Q17
 *
 * The bucket locks and the voter coordination of Alg. 1 only
 * arbitrate concurrent writers; a sequential program needs neither, so they
 * have no counterpart here.  Placement (slot, table, φ, evictions) is "parity
 * unpinned" exactly as in the narrow oracle.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define DYW_P      4294967291ULL                /* 2^32 - 5 (Q1) */
#define DYW_EMPTY  0xFFFFFFFFFFFFFFFFULL        /* reserved key marking a free slot (Q25, widened) */
#define DYW_DMAX   16
#define DYW_WMAX   4
#define DYW_OK     0
#define DYW_FAIL   1

typedef struct { uint64_t key; uint64_t val[DYW_WMAX]; } dyw_slot;

typedef struct {
    uint64_t m, N;
    uint32_t d, B, W, pad;
    uint64_t buckets[DYW_DMAX];
    uint64_t count[DYW_DMAX];
    uint64_t n_upsize, n_downsize, n_fail_upsize, n_residual, n_evict;
    uint64_t max_probes, invariant_errors;
} dyw_stats_t;

typedef struct {
    uint32_t d, B, W, L_max;
    double alpha, beta;
    uint64_t a[DYW_DMAX + 2], b[DYW_DMAX + 2], c[DYW_DMAX + 2];
    uint64_t n[DYW_DMAX], m_t[DYW_DMAX];
    dyw_slot *tab[DYW_DMAX];
    uint64_t rng;
    uint64_t n_upsize, n_downsize, n_fail_upsize, n_residual, n_evict, max_probes, invariant_errors;
    char last_error[256];
} dyw_table;

/* ---------------------------------------------------------------- hashing */

static uint64_t splitmix64(uint64_t *state)
{
    uint64_t z = (*state += 0x9E3779B97F4A7C15ULL);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* Reading Q33: the universal hash of P:L271 extended to 64-bit keys as the
 * Carter-Wegman vector form over the two 32-bit halves,
 *     x_s(k) = (c_s * hi(k) + a_s * lo(k) + b_s) mod p,
 * so a key below 2^32 hashes exactly as in the 32-bit table. */
static uint64_t hash_x(const dyw_table *T, uint32_t s, uint64_t k)
{
    uint64_t lo = k & 0xFFFFFFFFULL, hi = k >> 32;
    uint64_t x = (T->c[s] * hi) % DYW_P;
    x = (x + (T->a[s] * lo) % DYW_P) % DYW_P;
    return (x + T->b[s]) % DYW_P;
}

static void pair_of(const dyw_table *T, uint64_t k, uint32_t *t1, uint32_t *t2)
{
    uint64_t q = hash_x(T, 0, k) % ((uint64_t)T->d * (T->d - 1));   /* Q2 */
    uint32_t first = (uint32_t)(q / (T->d - 1));
    uint32_t r = (uint32_t)(q % (T->d - 1));
    *t1 = first;
    *t2 = (r < first) ? r : r + 1;
}

static uint64_t bucket_of(const dyw_table *T, uint32_t t, uint64_t k)
{
    return hash_x(T, t + 1, k) % T->n[t];
}

static uint32_t partner_of(const dyw_table *T, uint64_t k, uint32_t t)
{
    uint32_t t1, t2;
    pair_of(T, k, &t1, &t2);
    return (t == t1) ? t2 : t1;
}

static dyw_slot *bucket_ptr(const dyw_table *T, uint32_t t, uint64_t b) { return T->tab[t] + b * T->B; }

static uint64_t total_slots(const dyw_table *T)
{
    uint64_t N = 0;
    for (uint32_t t = 0; t < T->d; t++) N += T->n[t] * T->B;
    return N;
}

static uint64_t total_keys(const dyw_table *T)
{
    uint64_t m = 0;
    for (uint32_t t = 0; t < T->d; t++) m += T->m_t[t];
    return m;
}

static void set_error(dyw_table *T, const char *msg)
{
    T->invariant_errors++;
    snprintf(T->last_error, sizeof T->last_error, "%s", msg);
}

static void clear_slot(dyw_slot *s)
{
    s->key = DYW_EMPTY;
    for (int w = 0; w < DYW_WMAX; w++) s->val[w] = DYW_EMPTY;
}

/* ---------------------------------------------------------------- lookup */

static dyw_slot *lookup(dyw_table *T, uint64_t k, uint32_t *probes)
{
    uint32_t t1, t2;
    pair_of(T, k, &t1, &t2);
    uint32_t cand[2] = { t1, t2 };
    *probes = 0;
    for (int c = 0; c < 2; c++) {
        dyw_slot *bk = bucket_ptr(T, cand[c], bucket_of(T, cand[c], k));
        (*probes)++;
        for (uint32_t s = 0; s < T->B; s++)
            if (bk[s].key == k) return &bk[s];
    }
    return NULL;
}

static int bucket_store_if_free(dyw_table *T, uint32_t t, const dyw_slot *kv)
{
    dyw_slot *bk = bucket_ptr(T, t, bucket_of(T, t, kv->key));
    for (uint32_t s = 0; s < T->B; s++)
        if (bk[s].key == DYW_EMPTY) {
            bk[s] = *kv;
            T->m_t[t]++;
            return 1;
        }
    return 0;
}

/* place(): two-choice first-fit over the ordered pair (Q3), then an eviction
 * chain with a pseudo-random victim (Q5) that moves to the other table of ITS
 * pair, never into `exclude`; after L_max hops (Q6)
 * the carried pair is returned homeless (never dropped, Q17). */
static int place(dyw_table *T, dyw_slot kv, int exclude, int start, dyw_slot *homeless)
{
    dyw_slot cur = kv;
    uint32_t t;
    if (start >= 0) {
        t = (uint32_t)start;
    } else {
        uint32_t t1, t2;
        pair_of(T, cur.key, &t1, &t2);
        if ((int)t1 != exclude && bucket_store_if_free(T, t1, &cur)) return DYW_OK;
        if ((int)t2 != exclude && bucket_store_if_free(T, t2, &cur)) return DYW_OK;
        t = ((int)t1 != exclude) ? t1 : t2;
    }
    for (uint32_t hop = 0; hop <= T->L_max; hop++) {
        if (bucket_store_if_free(T, t, &cur)) return DYW_OK;
        if (hop == T->L_max) break;
        dyw_slot *bk = bucket_ptr(T, t, bucket_of(T, t, cur.key));
        uint32_t legal[64], nl = 0;
        for (uint32_t s = 0; s < T->B; s++)
            if ((int)partner_of(T, bk[s].key, t) != exclude) legal[nl++] = s;
        if (nl == 0) break;
        uint32_t s = legal[splitmix64(&T->rng) % nl];
        dyw_slot victim = bk[s];
        bk[s] = cur;                                   /* swap, Alg. 1 */
        cur = victim;
        T->n_evict++;
        t = partner_of(T, cur.key, t);
    }
    *homeless = cur;
    return DYW_FAIL;
}

/* ---------------------------------------------------------------- resizing */

static int smallest_table(const dyw_table *T)
{
    uint32_t best = 0;
    for (uint32_t t = 1; t < T->d; t++)
        if (T->n[t] < T->n[best]) best = t;
    return (int)best;
}

static int largest_table(const dyw_table *T)
{
    uint32_t best = T->d - 1;
    for (int t = (int)T->d - 2; t >= 0; t--)
        if (T->n[t] > T->n[best]) best = (uint32_t)t;
    return (int)best;
}

static int upsize_table(dyw_table *T, uint32_t t)
{
    uint64_t n_old = T->n[t], n_new = 2 * n_old;
    dyw_slot *nt = (dyw_slot *)malloc(n_new * T->B * sizeof(dyw_slot));
    uint64_t *fill = (uint64_t *)calloc(n_new, sizeof(uint64_t));
    if (!nt || !fill) { free(nt); free(fill); return -1; }
    for (uint64_t i = 0; i < n_new * T->B; i++) clear_slot(&nt[i]);
    uint64_t moved = 0;
    for (uint64_t b = 0; b < n_old; b++)
        for (uint32_t s = 0; s < T->B; s++) {
            dyw_slot e = T->tab[t][b * T->B + s];
            if (e.key == DYW_EMPTY) continue;
            uint64_t nb = hash_x(T, t + 1, e.key) % n_new;
            if (nb != b && nb != b + n_old) set_error(T, "I8: upsize moved an entry outside {b, b+n}");
            if (fill[nb] >= T->B) { set_error(T, "I8: upsize bucket overflow"); continue; }
            nt[nb * T->B + fill[nb]++] = e;
            moved++;
        }
    if (moved != T->m_t[t]) set_error(T, "I8: upsize did not move exactly m_t entries");
    free(fill);
    free(T->tab[t]);
    T->tab[t] = nt;
    T->n[t] = n_new;
    T->n_upsize++;
    return 0;
}

static int upsize(dyw_table *T) { return upsize_table(T, (uint32_t)smallest_table(T)); }

static void settle_homeless(dyw_table *T, dyw_slot *list, uint64_t cnt)
{
    for (uint64_t i = 0; i < cnt; i++) {
        dyw_slot cur = list[i];
        for (;;) {
            dyw_slot hl;
            if (place(T, cur, -1, -1, &hl) == DYW_OK) break;
            cur = hl;
            T->n_fail_upsize++;
            if (upsize(T) != 0) { set_error(T, "out of memory in failure upsize"); return; }
        }
    }
}

static int downsize_table(dyw_table *T, uint32_t t)      /* P:L387-395, Q16, Q18 */
{
    uint64_t n_old = T->n[t], h = n_old / 2;
    if (n_old < 2 || (n_old & 1)) return -1;
    dyw_slot *nt = (dyw_slot *)malloc(h * T->B * sizeof(dyw_slot));
    dyw_slot *res = (dyw_slot *)malloc((2 * h * T->B + 1) * sizeof(dyw_slot));
    if (!nt || !res) { free(nt); free(res); return -1; }
    uint64_t nres = 0, expect_res = 0;
    for (uint64_t bp = 0; bp < h; bp++) {
        uint32_t kept = 0, occupied = 0;
        for (int half = 0; half < 2; half++) {
            uint64_t ob = bp + (half ? h : 0);
            for (uint32_t s = 0; s < T->B; s++) {
                dyw_slot e = T->tab[t][ob * T->B + s];
                if (e.key == DYW_EMPTY) continue;
                occupied++;
                if (hash_x(T, t + 1, e.key) % h != bp) set_error(T, "downsize: entry not hashed to merged bucket");
                if (kept < T->B) nt[bp * T->B + kept++] = e;
                else res[nres++] = e;
            }
        }
        for (uint32_t s = kept; s < T->B; s++) clear_slot(&nt[bp * T->B + s]);
        if (occupied > T->B) expect_res += occupied - T->B;
    }
    if (nres != expect_res) set_error(T, "I9: residual count mismatch");
    free(T->tab[t]);
    T->tab[t] = nt;
    T->n[t] = h;
    T->m_t[t] -= nres;
    T->n_downsize++;
    T->n_residual += nres;
    dyw_slot *homeless = (dyw_slot *)malloc((nres + 1) * sizeof(dyw_slot));
    uint64_t nh = 0;
    for (uint64_t i = 0; i < nres; i++) {
        dyw_slot hl;
        if (place(T, res[i], (int)t, (int)partner_of(T, res[i].key, t), &hl) != DYW_OK) homeless[nh++] = hl;
    }
    free(res);
    settle_homeless(T, homeless, nh);
    free(homeless);
    return 0;
}

static void enforce_lower(dyw_table *T)                  /* P:L305; Q11-Q13, Q17b */
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
        if (T->n_fail_upsize != fails_before) break;
    }
}

/* ---------------------------------------------------------------- public API */

dyw_table *dyw_o_create(uint32_t d, uint32_t B, uint32_t W, uint64_t init_capacity, double alpha, double beta,
                        uint64_t seed, uint32_t L_max)
{
    if (d < 2 || d > DYW_DMAX || B < 1 || B > 64 || W < 1 || W > DYW_WMAX) return NULL;
    if (!(alpha > 0.0 && alpha < beta && beta < 1.0)) return NULL;
    if (alpha > beta * (double)d / (double)(d + 1)) return NULL;          /* Q14 */
    dyw_table *T = (dyw_table *)calloc(1, sizeof(dyw_table));
    if (!T) return NULL;
    T->d = d; T->B = B; T->W = W; T->L_max = L_max;
    T->alpha = alpha; T->beta = beta;
    uint64_t st = seed;
    for (uint32_t s = 0; s < d + 2; s++) {                 /* same draws as the 32-bit table ... */
        T->a[s] = 1 + splitmix64(&st) % (DYW_P - 1);
        T->b[s] = splitmix64(&st) % DYW_P;
    }
    for (uint32_t s = 0; s < d + 2; s++)                   /* ... then the high-half multipliers (Q33) */
        T->c[s] = 1 + splitmix64(&st) % (DYW_P - 1);
    T->rng = seed ^ 0xA5A5A5A5DEADBEEFULL;
    uint64_t per = (init_capacity + (uint64_t)d * B - 1) / ((uint64_t)d * B);   /* Q13 */
    if (per < 1) per = 1;
    for (uint32_t t = 0; t < d; t++) {
        T->n[t] = per;
        T->tab[t] = (dyw_slot *)malloc(per * B * sizeof(dyw_slot));
        if (!T->tab[t]) return NULL;
        for (uint64_t i = 0; i < per * B; i++) clear_slot(&T->tab[t][i]);
    }
    return T;
}

void dyw_o_destroy(dyw_table *T)
{
    if (!T) return;
    for (uint32_t t = 0; t < T->d; t++) free(T->tab[t]);
    free(T);
}

static int cmp_u64(const void *x, const void *y)
{
    uint64_t a = *(const uint64_t *)x, b = *(const uint64_t *)y;
    return (a > b) - (a < b);
}

/* values are row-major: op i's words are vals[i*W .. i*W+W) */
void dyw_o_insert_batch(dyw_table *T, const uint64_t *keys, const uint64_t *vals, uint8_t *status, uint64_t n)
{
    if (n == 0) return;                                                  /* Q32 */
    uint64_t *sorted = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    memcpy(sorted, keys, n * sizeof(uint64_t));
    qsort(sorted, n, sizeof(uint64_t), cmp_u64);
    uint64_t n_new = 0;
    for (uint64_t i = 0; i < n; i++) {
        if (sorted[i] == DYW_EMPTY) continue;
        if (i > 0 && sorted[i] == sorted[i - 1]) continue;
        uint32_t pr;
        if (!lookup(T, sorted[i], &pr)) n_new++;
    }
    free(sorted);
    while ((double)(total_keys(T) + n_new) > T->beta * (double)total_slots(T))   /* Q11 */
        if (upsize(T) != 0) { set_error(T, "out of memory in upsize"); return; }
    for (uint64_t i = 0; i < n; i++) {
        uint64_t k = keys[i];
        uint32_t pr;
        if (k == DYW_EMPTY) { if (status) status[i] = 0; continue; }
        dyw_slot *sl = lookup(T, k, &pr);
        if (sl) {                                                         /* Alg. 1 */
            for (uint32_t w = 0; w < T->W; w++) sl->val[w] = vals[i * T->W + w];
            if (status) status[i] = 2;
            continue;
        }
        dyw_slot kv, hl;
        clear_slot(&kv);
        kv.key = k;
        for (uint32_t w = 0; w < T->W; w++) kv.val[w] = vals[i * T->W + w];
        if (place(T, kv, -1, -1, &hl) != DYW_OK) settle_homeless(T, &hl, 1);
        if (status) status[i] = 1;
    }
    enforce_lower(T);
}

void dyw_o_find_batch(dyw_table *T, const uint64_t *keys, uint64_t *vals_out, uint8_t *found, uint64_t n)
{
    for (uint64_t i = 0; i < n; i++) {
        uint32_t pr = 0;
        dyw_slot *sl = (keys[i] == DYW_EMPTY) ? NULL : lookup(T, keys[i], &pr);
        if (pr > T->max_probes) T->max_probes = pr;
        if (vals_out)
            for (uint32_t w = 0; w < T->W; w++) vals_out[i * T->W + w] = sl ? sl->val[w] : DYW_EMPTY;
        if (found) found[i] = sl ? 1 : 0;
    }
}

void dyw_o_delete_batch(dyw_table *T, const uint64_t *keys, uint64_t *old_vals, uint8_t *status, uint64_t n)
{
    if (n == 0) return;
    for (uint64_t i = 0; i < n; i++) {
        uint32_t pr = 0;
        dyw_slot *sl = (keys[i] == DYW_EMPTY) ? NULL : lookup(T, keys[i], &pr);
        if (pr > T->max_probes) T->max_probes = pr;
        if (old_vals)
            for (uint32_t w = 0; w < T->W; w++) old_vals[i * T->W + w] = sl ? sl->val[w] : DYW_EMPTY;
        if (status) status[i] = sl ? 1 : 0;
        if (sl) {
            uint32_t t1, t2;
            pair_of(T, keys[i], &t1, &t2);
            uint32_t t = (sl >= T->tab[t1] && sl < T->tab[t1] + T->n[t1] * T->B) ? t1 : t2;
            clear_slot(sl);
            T->m_t[t]--;
        }
    }
    enforce_lower(T);
}

int dyw_o_resize(dyw_table *T, int direction, int t)
{
    if (direction > 0) {
        if (t < 0) t = smallest_table(T);
        if (t >= (int)T->d || T->n[t] != T->n[smallest_table(T)]) return -1;
        return upsize_table(T, (uint32_t)t);
    }
    if (direction < 0) {
        if (t < 0) t = largest_table(T);
        if (t >= (int)T->d || T->n[t] != T->n[largest_table(T)]) return -1;
        if (T->n[t] < 2 || (T->n[t] & 1)) return -1;
        return downsize_table(T, (uint32_t)t);
    }
    return 0;
}

void dyw_o_stats(const dyw_table *T, dyw_stats_t *S)
{
    memset(S, 0, sizeof *S);
    S->d = T->d; S->B = T->B; S->W = T->W;
    S->m = total_keys(T); S->N = total_slots(T);
    for (uint32_t t = 0; t < T->d; t++) { S->buckets[t] = T->n[t]; S->count[t] = T->m_t[t]; }
    S->n_upsize = T->n_upsize; S->n_downsize = T->n_downsize; S->n_fail_upsize = T->n_fail_upsize;
    S->n_residual = T->n_residual; S->n_evict = T->n_evict; S->max_probes = T->max_probes;
    S->invariant_errors = T->invariant_errors;
}

/* keys[i], vals[i*W..], table[i], bucket[i] of every live entry (any order). */
uint64_t dyw_o_dump(const dyw_table *T, uint64_t *keys, uint64_t *vals, uint32_t *table, uint64_t *bucket,
                    uint64_t cap)
{
    uint64_t c = 0;
    for (uint32_t t = 0; t < T->d; t++)
        for (uint64_t i = 0; i < T->n[t] * T->B; i++) {
            const dyw_slot *e = &T->tab[t][i];
            if (e->key == DYW_EMPTY) continue;
            if (c < cap) {
                if (keys) keys[c] = e->key;
                if (vals) for (uint32_t w = 0; w < T->W; w++) vals[c * T->W + w] = e->val[w];
                if (table) table[c] = t;
                if (bucket) bucket[c] = i / T->B;
            }
            c++;
        }
    return c;
}

uint64_t dyw_o_check_invariants(dyw_table *T, char *msg, uint64_t msglen)
{
    uint64_t bad = 0, m = 0, N = total_slots(T), nkeys = total_keys(T), na = 0;
    const char *first = NULL;
    uint64_t *all = (uint64_t *)malloc((nkeys + 1) * sizeof(uint64_t));
    for (uint32_t t = 0; t < T->d; t++) {
        uint64_t occ = 0;
        for (uint64_t i = 0; i < T->n[t] * T->B; i++) {
            uint64_t k = T->tab[t][i].key;
            uint32_t t1, t2;
            if (k == DYW_EMPTY) continue;
            occ++;
            pair_of(T, k, &t1, &t2);
            if (t != t1 && t != t2) { bad++; if (!first) first = "I1: key in a table outside its pair"; }
            if (bucket_of(T, t, k) != i / T->B) { bad++; if (!first) first = "I1: key in the wrong bucket"; }
            if (na <= nkeys) all[na++] = k;
        }
        if (occ != T->m_t[t]) { bad++; if (!first) first = "I4: counter != occupancy"; }
        m += occ;
    }
    qsort(all, na, sizeof(uint64_t), cmp_u64);
    for (uint64_t i = 1; i < na; i++)
        if (all[i] == all[i - 1]) { bad++; if (!first) first = "I2: duplicate key"; }
    free(all);
    if ((double)m > T->beta * (double)N) { bad++; if (!first) first = "I5: fill above beta"; }
    uint64_t mn = T->n[0], mx = T->n[0];
    for (uint32_t t = 1; t < T->d; t++) { if (T->n[t] < mn) mn = T->n[t]; if (T->n[t] > mx) mx = T->n[t]; }
    if (mx > 2 * mn) { bad++; if (!first) first = "I6: a subtable more than double another"; }
    if (T->invariant_errors) { bad += T->invariant_errors; if (!first) first = T->last_error; }
    if (msg && msglen) snprintf(msg, msglen, "%s", first ? first : "ok");
    return bad;
}

uint64_t dyw_o_hash_x(const dyw_table *T, uint32_t s, uint64_t k) { return hash_x(T, s, k); }
void dyw_o_pair(const dyw_table *T, uint64_t k, uint32_t *t1, uint32_t *t2) { pair_of(T, k, t1, t2); }
uint64_t dyw_o_bucket(const dyw_table *T, uint32_t t, uint64_t k) { return bucket_of(T, t, k); }
void dyw_o_hash_params(const dyw_table *T, uint64_t *a, uint64_t *b, uint64_t *c)
{
    for (uint32_t s = 0; s < T->d + 2; s++) { a[s] = T->a[s]; b[s] = T->b[s]; c[s] = T->c[s]; }
}

/* I1/I2 of a layout produced elsewhere (the GPU dump), with this oracle's hash. */
uint64_t dyw_o_check_layout(const dyw_table *T, const uint64_t *nb, const uint64_t *keys, const uint32_t *table,
                            const uint64_t *bucket, uint64_t count)
{
    uint64_t bad = 0;
    for (uint64_t i = 0; i < count; i++) {
        uint32_t t1, t2, t = table[i];
        pair_of(T, keys[i], &t1, &t2);
        if (t != t1 && t != t2) { bad++; continue; }
        if (hash_x(T, t + 1, keys[i]) % nb[t] != bucket[i]) bad++;
    }
    uint64_t *s = (uint64_t *)malloc((count + 1) * sizeof(uint64_t));
    memcpy(s, keys, count * sizeof(uint64_t));
    qsort(s, count, sizeof(uint64_t), cmp_u64);
    for (uint64_t i = 1; i < count; i++) if (s[i] == s[i - 1]) bad++;
    free(s);
    return bad;
}
