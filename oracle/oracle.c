/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * oracle for the HYBRID-DBSCAN hot path (Gowanlock et al., IPDPSW 2017).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_ipps_gowanlockrblp17_b200/) shares no code with it and never
 * calls it.
 *
 * Citations are PAPER.md line numbers ("P:n") plus the section / algorithm.
 *
 * What it computes:
 *   (O1) the neighbour predicate  q in N_eps(p)  <=>  dist(p,q) <= eps
 *        (Sec. II-A), evaluated as fl(fl(dx*dx)+fl(dy*dy)) <= fl(eps*eps)
 *        in the input precision with no FMA contraction (reading R1/R2;
 *        the paper never states the precision).  This file MUST be compiled with
 *        -ffp-contract=off; the #error below enforces the matching define.
 *   (O2) the neighbour table T (Sec. III): for every p, the
 *        ascending list of q (0-based) with q in N_eps(p), p itself included
 *        (N_eps(p) = {q in D | dist(p,q) <= eps}).  Brute force over all
 *        n^2 ordered pairs -- the definition itself, no grid.
 *   (O3) DBSCAN on T: Algorithm 1 executed literally over
 *        p = 0..n-1 with its NeighborSearch (lines 9, 18) replaced by a lookup
 *        in T, which is exactly the paper's "modified DBSCAN".
 *        Readings of the garbled pseudo-code (R4-R6): line 21 is NOT
 *        nested inside line 16 (Ester et al. semantics), the final noise set is
 *        D \ clusterSet, and line 24 executes only in the else branch.
 *
 * Parity pins: tests/test_oracle_pins.py (hand-worked lattices, closed forms,
 * sklearn / scipy cross-checks, invariants).  Every function below is pinned.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#ifndef ORACLE_FP_CONTRACT_OFF
#error "oracle.c must be compiled with -ffp-contract=off -DORACLE_FP_CONTRACT_OFF (no FMA in the predicate)"
#endif

/* ------------------------------------------------------------------------ */
/* O1: the neighbour predicate, P:147-148 (dist(p,q) <= eps, inclusive).    */
/* ------------------------------------------------------------------------ */
static int is_neighbor_f64(double xp, double yp, double xq, double yq, double eps2)
{
    double dx = xp - xq;          /* fl(x_p - x_q) */
    double dy = yp - yq;          /* fl(y_p - y_q) */
    double dx2 = dx * dx;         /* fl(dx*dx)     */
    double dy2 = dy * dy;         /* fl(dy*dy)     */
    double d2 = dx2 + dy2;        /* fl(dx2 + dy2) -- no contraction (-ffp-contract=off) */
    return d2 <= eps2;
}

static int is_neighbor_f32(float xp, float yp, float xq, float yq, float eps2)
{
    float dx = xp - xq;
    float dy = yp - yq;
    float dx2 = dx * dx;
    float dy2 = dy * dy;
    float d2 = dx2 + dy2;
    return d2 <= eps2;
}

int oracle_predicate_f64(double xp, double yp, double xq, double yq, double eps)
{
    double eps2 = eps * eps;      /* fl(eps*eps) */
    return is_neighbor_f64(xp, yp, xq, yq, eps2);
}

int oracle_predicate_f32(float xp, float yp, float xq, float yq, float eps)
{
    float eps2 = eps * eps;
    return is_neighbor_f32(xp, yp, xq, yq, eps2);
}

int oracle_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ------------------------------------------------------------------------ */
/* O2: brute-force epsilon join for a list of query rows.                   */
/*                                                                          */
/* rows == NULL means "every row 0..n-1".  Two calls:                        */
/*   oracle_join_count_*: cnt[r] = |N_eps(rows[r])|                          */
/*   oracle_join_fill_*:  nbr[off[r] .. off[r+1]) = N_eps(rows[r]) ascending */
/* xy is interleaved (x0,y0,x1,y1,...), n rows.                             */
/* ------------------------------------------------------------------------ */
#define ROW(r) ((rows) ? rows[(r)] : (int64_t)(r))

void oracle_join_count_f64(const double* xy, int64_t n, double eps,
                           const int64_t* rows, int64_t nrows, uint64_t* cnt)
{
    double eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 64)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        double xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0;
        for (int64_t q = 0; q < n; ++q)
            c += (uint64_t)is_neighbor_f64(xp, yp, xy[2 * q], xy[2 * q + 1], eps2);
        cnt[r] = c;
    }
}

void oracle_join_fill_f64(const double* xy, int64_t n, double eps,
                          const int64_t* rows, int64_t nrows,
                          const uint64_t* off, uint32_t* nbr)
{
    double eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 64)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        double xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t k = off[r];
        for (int64_t q = 0; q < n; ++q)   /* ascending q => ascending list */
            if (is_neighbor_f64(xp, yp, xy[2 * q], xy[2 * q + 1], eps2))
                nbr[k++] = (uint32_t)q;
    }
}

void oracle_join_count_f32(const float* xy, int64_t n, float eps,
                           const int64_t* rows, int64_t nrows, uint64_t* cnt)
{
    float eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 64)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        float xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0;
        for (int64_t q = 0; q < n; ++q)
            c += (uint64_t)is_neighbor_f32(xp, yp, xy[2 * q], xy[2 * q + 1], eps2);
        cnt[r] = c;
    }
}

void oracle_join_fill_f32(const float* xy, int64_t n, float eps,
                          const int64_t* rows, int64_t nrows,
                          const uint64_t* off, uint32_t* nbr)
{
    float eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 64)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        float xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t k = off[r];
        for (int64_t q = 0; q < n; ++q)
            if (is_neighbor_f32(xp, yp, xy[2 * q], xy[2 * q + 1], eps2))
                nbr[k++] = (uint32_t)q;
    }
}

/* Per-row (count, order-independent 64-bit hash) of N_eps(p), streamed so
 * that tables too large to hold twice on the host can still be compared
 * row-for-row.  hash = sum over q in N_eps(p) of mix64(q)
 * (mod 2^64), mix64 = the SplitMix64 finaliser.  Test-only comparison aid,
 * not part of the method. */
static uint64_t mix64(uint64_t x)
{
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

void oracle_join_rowhash_f64(const double* xy, int64_t n, double eps,
                             const int64_t* rows, int64_t nrows,
                             uint64_t* cnt, uint64_t* hash)
{
    double eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 16)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        double xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0, h = 0;
        for (int64_t q = 0; q < n; ++q)
            if (is_neighbor_f64(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) {
                ++c;
                h += mix64((uint64_t)q);
            }
        cnt[r] = c;
        hash[r] = h;
    }
}

void oracle_join_rowhash_f32(const float* xy, int64_t n, float eps,
                             const int64_t* rows, int64_t nrows,
                             uint64_t* cnt, uint64_t* hash)
{
    float eps2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 16)
    for (r = 0; r < nrows; ++r) {
        int64_t p = ROW(r);
        float xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0, h = 0;
        for (int64_t q = 0; q < n; ++q)
            if (is_neighbor_f32(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) {
                ++c;
                h += mix64((uint64_t)q);
            }
        cnt[r] = c;
        hash[r] = h;
    }
}

/* ------------------------------------------------------------------------ */
/* O2, second construction: an x-sorted plane sweep (no cells, no tree).    */
/* The north star asks for the oracle to be checked against "a naive        */
/* R-tree-free scan"; this is that scan ("O2 at scale" (i)).   */
/* Points are ordered by (x, id); for each p the scan walks outwards from p */
/* in both directions and stops at the first q with fl(dx*dx) > fl(eps^2),  */
/* dx = fl(x_q - x_p).  The stop is exact under O1: fl(x_q - x_p) is         */
/* monotone in x_q, so dx*dx only grows along each direction, and           */
/* d2 = fl(dx2 + dy2) >= dx2 because dy2 >= 0 and rounding is monotone.     */
/* Output: per-row (count, sum of mix64(q)) like oracle_join_rowhash_*.     */
/* ------------------------------------------------------------------------ */
typedef struct { double x; int64_t id; } sweep_key;

static int sweep_cmp(const void* a, const void* b)
{
    const sweep_key* u = (const sweep_key*)a;
    const sweep_key* v = (const sweep_key*)b;
    if (u->x < v->x) return -1;
    if (u->x > v->x) return 1;
    return (u->id > v->id) - (u->id < v->id);
}

static sweep_key* sweep_order(const double* xs, int64_t n)
{
    sweep_key* k = (sweep_key*)malloc(sizeof(sweep_key) * (size_t)(n ? n : 1));
    if (!k) return NULL;
    for (int64_t i = 0; i < n; ++i) {
        k[i].x = xs[i];
        k[i].id = i;
    }
    qsort(k, (size_t)n, sizeof(sweep_key), sweep_cmp);
    return k;
}

int oracle_sweep_rowhash_f64(const double* xy, int64_t n, double eps, uint64_t* cnt, uint64_t* hash)
{
    double eps2 = eps * eps;
    double* xs = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    if (!xs) return -1;
    for (int64_t i = 0; i < n; ++i) xs[i] = xy[2 * i];
    sweep_key* ord = sweep_order(xs, n);
    free(xs);
    if (!ord) return -1;
    int64_t i;
#pragma omp parallel for schedule(dynamic, 256)
    for (i = 0; i < n; ++i) {
        int64_t p = ord[i].id;
        double xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0, h = 0;
        for (int64_t j = i; j < n; ++j) {          /* rightwards, including p itself */
            int64_t q = ord[j].id;
            double dx = xy[2 * q] - xp;
            double dx2 = dx * dx;
            if (dx2 > eps2) break;
            if (is_neighbor_f64(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) { ++c; h += mix64((uint64_t)q); }
        }
        for (int64_t j = i - 1; j >= 0; --j) {     /* leftwards */
            int64_t q = ord[j].id;
            double dx = xy[2 * q] - xp;
            double dx2 = dx * dx;
            if (dx2 > eps2) break;
            if (is_neighbor_f64(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) { ++c; h += mix64((uint64_t)q); }
        }
        cnt[p] = c;
        hash[p] = h;
    }
    free(ord);
    return 0;
}

int oracle_sweep_rowhash_f32(const float* xy, int64_t n, float eps, uint64_t* cnt, uint64_t* hash)
{
    float eps2 = eps * eps;
    double* xs = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    if (!xs) return -1;
    for (int64_t i = 0; i < n; ++i) xs[i] = (double)xy[2 * i];   /* exact widening: same order */
    sweep_key* ord = sweep_order(xs, n);
    free(xs);
    if (!ord) return -1;
    int64_t i;
#pragma omp parallel for schedule(dynamic, 256)
    for (i = 0; i < n; ++i) {
        int64_t p = ord[i].id;
        float xp = xy[2 * p], yp = xy[2 * p + 1];
        uint64_t c = 0, h = 0;
        for (int64_t j = i; j < n; ++j) {
            int64_t q = ord[j].id;
            float dx = xy[2 * q] - xp;
            float dx2 = dx * dx;
            if (dx2 > eps2) break;
            if (is_neighbor_f32(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) { ++c; h += mix64((uint64_t)q); }
        }
        for (int64_t j = i - 1; j >= 0; --j) {
            int64_t q = ord[j].id;
            float dx = xy[2 * q] - xp;
            float dx2 = dx * dx;
            if (dx2 > eps2) break;
            if (is_neighbor_f32(xp, yp, xy[2 * q], xy[2 * q + 1], eps2)) { ++c; h += mix64((uint64_t)q); }
        }
        cnt[p] = c;
        hash[p] = h;
    }
    free(ord);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* O3: Algorithm 1 on the neighbour table T.         */
/*                                                                          */
/* T is CSR: N_eps(p) = nbr[off[p] .. off[p+1]).                             */
/* Output: labels[p] = index of the cluster C in the order Alg. 1 line 24   */
/* appends it (0, 1, ...) for p in clusterSet, -1 for noise (R5);           */
/* is_core[p] = (|N_eps(p)| >= minpts); returns |C|.             */
/*                                                                          */
/* The sets of Alg. 1 are plain arrays: visitedSet, clusterSet as flags,    */
/* the working set N as a FIFO array plus an "in N" flag (set semantics).   */
/* ------------------------------------------------------------------------ */
int64_t oracle_dbscan(const uint64_t* off, const uint32_t* nbr, int64_t n,
                      uint64_t minpts, int32_t* labels, uint8_t* is_core)
{
    uint8_t* visited = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1);   /* line 2 */
    uint8_t* in_cluster = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1); /* line 3 */
    uint8_t* in_noise = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1);   /* line 4 */
    uint8_t* in_N = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1);
    /* Every element pushed onto N comes from some N_eps list read once per
     * visited core (lines 9, 18), so off[n] + n bounds the pushes. */
    uint64_t cap = (n > 0 ? off[n] : 0) + (uint64_t)n + 1;
    uint32_t* N = (uint32_t*)malloc(cap * sizeof(uint32_t));
    int64_t n_clusters = 0;                                               /* line 5: C <- {} */
    if (!visited || !in_cluster || !in_noise || !in_N || !N) {
        free(visited); free(in_cluster); free(in_noise); free(in_N); free(N);
        return -1;
    }
    for (int64_t p = 0; p < n; ++p) labels[p] = -1;

    for (int64_t p = 0; p < n; ++p) {                                     /* line 6 */
        if (visited[p]) continue;
        /* line 7: a new cluster C <- {}; its index is n_clusters if kept.  */
        visited[p] = 1;                                                   /* line 8 */
        uint64_t np = off[p + 1] - off[p];                                /* line 9: N <- T[p] */
        if (np < minpts) {                                                /* line 10 */
            in_noise[p] = 1;
            continue;
        }
        int32_t cid = (int32_t)n_clusters;                                /* line 11 (else) */
        labels[p] = cid; in_cluster[p] = 1;                               /* lines 12-13 */
        uint64_t head = 0, tail = 0;
        for (uint64_t k = off[p]; k < off[p + 1]; ++k) {                  /* N <- N_eps(p) */
            uint32_t q = nbr[k];
            if (!in_N[q]) { in_N[q] = 1; N[tail++] = q; }
        }
        while (head < tail) {                                             /* line 14 */
            uint32_t i = N[head++];
            in_N[i] = 0;                                                  /* line 15: N <- N \ i */
            if (!visited[i]) {                                            /* line 16 */
                visited[i] = 1;                                           /* line 17 */
                uint64_t ni = off[i + 1] - off[i];                        /* line 18: N^ <- T[i] */
                if (ni >= minpts) {                                       /* line 19 */
                    for (uint64_t k = off[i]; k < off[i + 1]; ++k) {      /* line 20: N <- N u N^ */
                        uint32_t q = nbr[k];
                        if (!in_N[q]) {
                            if (tail == cap) {  /* cannot happen (bound above); be safe */
                                free(visited); free(in_cluster); free(in_noise); free(in_N); free(N);
                                return -1;
                            }
                            in_N[q] = 1; N[tail++] = q;
                        }
                    }
                }
            }
            if (!in_cluster[i]) {                                         /* line 21 (R4: not nested in 16) */
                labels[i] = cid;                                          /* line 22 */
                in_cluster[i] = 1;                                        /* line 23 */
            }
        }
        ++n_clusters;                                                     /* line 24: C <- C u {C} */
    }
    /* R5: final noise set = D \ clusterSet (labels already -1 there). */
    if (is_core)
        for (int64_t p = 0; p < n; ++p)
            is_core[p] = (uint8_t)((off[p + 1] - off[p]) >= minpts);
    free(visited); free(in_cluster); free(in_noise); free(in_N); free(N);
    return n_clusters;
}
