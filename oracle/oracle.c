/*
 * oracle/oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU equi-join used as the parity authority
 * for the CUDA path in paper_conf_sigmod_paullhl21_b200/csrc.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load it.  It shares no code, header, hash function or constant with
 * the CUDA path.
 *
 * What it computes (the plain definition of the paper's
 * equi-join of two relations R and S, §3 "we
 * specifically focus on equi-joins"; probe semantics P:469-475):
 *
 *   J        = { (k, a, b) : (k, a) in R, (k, b) in S }   (bag semantics, C2)
 *   count    = |J|
 *   checksum = sum over J of (a*C + b) mod 2^64            (reading C3)
 *              C = 2^32 for 4-byte payloads, 0x9E3779B97F4A7C15 for 8-byte
 *   pair_digest = sum over J of a*b mod 2^64               (reading C3b)
 *              bilinear in the pair, so it changes when an S row is paired
 *              with the wrong R row even where count and checksum cannot
 *   triples  = J sorted by unsigned lexicographic (k, a, b)  (reading C17)
 *
 * Algorithm (SURVEY.md §8c "Algorithm"): build a chained hash table over R
 * (T = next_pow2(max(2, 2|R|)) heads, Fibonacci hashing of the key, 8-byte
 * keys folded k ^ (k >> 32) first), then probe it with every S tuple in S
 * order, then sort the emitted triples with qsort.
 *
 * Pins (tests/test_oracle.py): numpy brute-force nested loop on tiny inputs,
 * closed-form counts/checksums of the generated workloads, numpy sort-merge
 * multiplicity sums, hand-worked golden fixture.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint64_t count;
    uint64_t checksum;
    uint64_t n_out;      /* triples written (<= out_cap) */
    uint64_t pair_digest;
    int32_t  overflow;   /* 1 if count > out_cap while materialising */
    int32_t  status;     /* 0 ok, -1 out of memory */
} oracle_result_t;

static const uint64_t FIB = 0x9E3779B97F4A7C15ull;

static unsigned log2_u64(uint64_t t) {
    unsigned l = 0;
    while ((1ull << l) < t) l++;
    return l;
}

static uint64_t table_size(uint64_t nr) {
    uint64_t t = 2;
    while (t < 2 * nr) t <<= 1;
    return t;
}

/* ------------------------------------------------------------------ 4+4 B */
typedef struct { uint32_t k, a, b; } trip32_t;

static int cmp_trip32(const void *x, const void *y) {
    const trip32_t *p = (const trip32_t *)x, *q = (const trip32_t *)y;
    if (p->k != q->k) return p->k < q->k ? -1 : 1;
    if (p->a != q->a) return p->a < q->a ? -1 : 1;
    if (p->b != q->b) return p->b < q->b ? -1 : 1;
    return 0;
}

int oracle_join_k32(const uint32_t *rk, const uint32_t *ra, uint64_t nr,
                    const uint32_t *sk, const uint32_t *sb, uint64_t ns,
                    uint32_t *out_k, uint32_t *out_a, uint32_t *out_b,
                    uint64_t out_cap, oracle_result_t *res)
{
    memset(res, 0, sizeof(*res));
    uint64_t T = table_size(nr);
    unsigned shift = 64 - log2_u64(T);
    int64_t *head = (int64_t *)malloc(T * sizeof(int64_t));
    int64_t *next = (int64_t *)malloc((nr ? nr : 1) * sizeof(int64_t));
    trip32_t *trip = NULL;
    if (out_k && out_cap) trip = (trip32_t *)malloc(out_cap * sizeof(trip32_t));
    if (!head || !next || (out_k && out_cap && !trip)) {
        free(head); free(next); free(trip);
        res->status = -1;
        return -1;
    }
    for (uint64_t h = 0; h < T; h++) head[h] = -1;

    /* build: for i in R order, push i at the front of chain h(k_i) */
    for (uint64_t i = 0; i < nr; i++) {
        uint64_t h = ((uint64_t)rk[i] * FIB) >> shift;
        next[i] = head[h];
        head[h] = (int64_t)i;
    }
    /* probe: for j in S order, walk chain h(k_j), emit every equal key */
    uint64_t count = 0, checksum = 0, n_out = 0, digest = 0;
    for (uint64_t j = 0; j < ns; j++) {
        uint32_t k = sk[j];
        uint64_t h = ((uint64_t)k * FIB) >> shift;
        for (int64_t i = head[h]; i >= 0; i = next[i]) {
            if (rk[i] != k) continue;
            count += 1;
            checksum += ((uint64_t)ra[i] << 32) + (uint64_t)sb[j]; /* a*2^32 + b */
            digest += (uint64_t)ra[i] * (uint64_t)sb[j];            /* a*b */
            if (out_k) {
                if (n_out < out_cap) {
                    trip[n_out].k = k; trip[n_out].a = ra[i]; trip[n_out].b = sb[j];
                    n_out++;
                } else {
                    res->overflow = 1;
                }
            }
        }
    }
    if (out_k && n_out) {
        qsort(trip, n_out, sizeof(trip32_t), cmp_trip32);
        for (uint64_t t = 0; t < n_out; t++) {
            out_k[t] = trip[t].k; out_a[t] = trip[t].a; out_b[t] = trip[t].b;
        }
    }
    res->count = count;
    res->checksum = checksum;
    res->n_out = n_out;
    res->pair_digest = digest;
    free(head); free(next); free(trip);
    return 0;
}

/* ------------------------------------------------------------------ 8+8 B */
typedef struct { uint64_t k, a, b; } trip64_t;

static int cmp_trip64(const void *x, const void *y) {
    const trip64_t *p = (const trip64_t *)x, *q = (const trip64_t *)y;
    if (p->k != q->k) return p->k < q->k ? -1 : 1;
    if (p->a != q->a) return p->a < q->a ? -1 : 1;
    if (p->b != q->b) return p->b < q->b ? -1 : 1;
    return 0;
}

int oracle_join_k64(const uint64_t *rk, const uint64_t *ra, uint64_t nr,
                    const uint64_t *sk, const uint64_t *sb, uint64_t ns,
                    uint64_t *out_k, uint64_t *out_a, uint64_t *out_b,
                    uint64_t out_cap, oracle_result_t *res)
{
    memset(res, 0, sizeof(*res));
    uint64_t T = table_size(nr);
    unsigned shift = 64 - log2_u64(T);
    int64_t *head = (int64_t *)malloc(T * sizeof(int64_t));
    int64_t *next = (int64_t *)malloc((nr ? nr : 1) * sizeof(int64_t));
    trip64_t *trip = NULL;
    if (out_k && out_cap) trip = (trip64_t *)malloc(out_cap * sizeof(trip64_t));
    if (!head || !next || (out_k && out_cap && !trip)) {
        free(head); free(next); free(trip);
        res->status = -1;
        return -1;
    }
    for (uint64_t h = 0; h < T; h++) head[h] = -1;

    for (uint64_t i = 0; i < nr; i++) {
        uint64_t f = rk[i] ^ (rk[i] >> 32);           /* fold 8-byte key */
        uint64_t h = (f * FIB) >> shift;
        next[i] = head[h];
        head[h] = (int64_t)i;
    }
    uint64_t count = 0, checksum = 0, n_out = 0, digest = 0;
    for (uint64_t j = 0; j < ns; j++) {
        uint64_t k = sk[j];
        uint64_t f = k ^ (k >> 32);
        uint64_t h = (f * FIB) >> shift;
        for (int64_t i = head[h]; i >= 0; i = next[i]) {
            if (rk[i] != k) continue;
            count += 1;
            checksum += ra[i] * FIB + sb[j];              /* a*C + b, C = 0x9E37... */
            digest += ra[i] * sb[j];                      /* a*b mod 2^64 */
            if (out_k) {
                if (n_out < out_cap) {
                    trip[n_out].k = k; trip[n_out].a = ra[i]; trip[n_out].b = sb[j];
                    n_out++;
                } else {
                    res->overflow = 1;
                }
            }
        }
    }
    if (out_k && n_out) {
        qsort(trip, n_out, sizeof(trip64_t), cmp_trip64);
        for (uint64_t t = 0; t < n_out; t++) {
            out_k[t] = trip[t].k; out_a[t] = trip[t].a; out_b[t] = trip[t].b;
        }
    }
    res->count = count;
    res->checksum = checksum;
    res->n_out = n_out;
    res->pair_digest = digest;
    free(head); free(next); free(trip);
    return 0;
}
