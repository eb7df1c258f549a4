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

/* The scan reads the points through sorted copies (sx, sy, sid): the same
 * values in the same order as ord[j].id would give, laid out for locality
 * (the arithmetic is unchanged; only the memory layout differs). */
#define SWEEP_BODY(T, IS_NEIGHBOR)                                                  \
    int64_t i;                                                                      \
    _Pragma("omp parallel for schedule(dynamic, 256)")                              \
    for (i = 0; i < n; ++i) {                                                       \
        T xp = sx[i], yp = sy[i];                                                   \
        /* the scan's stop points: first j > i (rightwards) and last j < i         \
         * (leftwards) with fl(dx*dx) > eps2 -- binary searches, exact because    \
         * fl(dx*dx) is monotone along each direction (see above) */              \
        int64_t lo = i + 1, hi = n;                                                 \
        while (lo < hi) {                                                           \
            int64_t m = lo + (hi - lo) / 2;                                         \
            T dx = sx[m] - xp;                                                      \
            if (dx * dx > eps2) hi = m; else lo = m + 1;                            \
        }                                                                           \
        int64_t jend = lo;                                                          \
        lo = 0; hi = i;                                                             \
        while (lo < hi) {                                                           \
            int64_t m = lo + (hi - lo) / 2;                                         \
            T dx = sx[m] - xp;                                                      \
            if (dx * dx > eps2) lo = m + 1; else hi = m;                            \
        }                                                                           \
        int64_t jbeg = lo;                                                          \
        uint64_t c = 0, h = 0;                                                      \
        for (int64_t j = jbeg; j < jend; ++j) {                                     \
            int hit = IS_NEIGHBOR(xp, yp, sx[j], sy[j], eps2);                      \
            c += (uint64_t)hit;                                                     \
            h += hit ? mix64((uint64_t)sid[j]) : 0;                                 \
        }                                                                           \
        cnt[sid[i]] = c;                                                            \
        hash[sid[i]] = h;                                                           \
    }

int oracle_sweep_rowhash_f64(const double* xy, int64_t n, double eps, uint64_t* cnt, uint64_t* hash)
{
    double eps2 = eps * eps;
    double* xs = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    if (!xs) return -1;
    for (int64_t k = 0; k < n; ++k) xs[k] = xy[2 * k];
    sweep_key* ord = sweep_order(xs, n);
    free(xs);
    if (!ord) return -1;
    double* sx = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    double* sy = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    int64_t* sid = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n ? n : 1));
    if (!sx || !sy || !sid) { free(ord); free(sx); free(sy); free(sid); return -1; }
    for (int64_t k = 0; k < n; ++k) {
        sid[k] = ord[k].id;
        sx[k] = xy[2 * ord[k].id];
        sy[k] = xy[2 * ord[k].id + 1];
    }
    free(ord);
    SWEEP_BODY(double, is_neighbor_f64)
    free(sx); free(sy); free(sid);
    return 0;
}

int oracle_sweep_rowhash_f32(const float* xy, int64_t n, float eps, uint64_t* cnt, uint64_t* hash)
{
    float eps2 = eps * eps;
    double* xs = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    if (!xs) return -1;
    for (int64_t k = 0; k < n; ++k) xs[k] = (double)xy[2 * k];   /* exact widening: same order */
    sweep_key* ord = sweep_order(xs, n);
    free(xs);
    if (!ord) return -1;
    float* sx = (float*)malloc(sizeof(float) * (size_t)(n ? n : 1));
    float* sy = (float*)malloc(sizeof(float) * (size_t)(n ? n : 1));
    int64_t* sid = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n ? n : 1));
    if (!sx || !sy || !sid) { free(ord); free(sx); free(sy); free(sid); return -1; }
    for (int64_t k = 0; k < n; ++k) {
        sid[k] = ord[k].id;
        sx[k] = xy[2 * ord[k].id];
        sy[k] = xy[2 * ord[k].id + 1];
    }
    free(ord);
    SWEEP_BODY(float, is_neighbor_f32)
    free(sx); free(sy); free(sid);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* O2, third construction: the plane sweep inside horizontal strips.        */
/* At 50M points (C5) a single x-sorted sweep tests ~5*10^4 points per row; */
/* here the points are cut into strips b_t <= y < b_{t+1} of width about    */
/* 2*eps, each strip sorted by (x, id), and row p scans the x-window of its */
/* own strip and the two adjacent ones exactly as the plane sweep does.     */
/* Exactness: for p in strip s and q in strip >= s+2 (or <= s-2), the real  */
/* |y_q - y_p| exceeds the real width b_{t+1} - b_t of a strip between      */
/* them, so by monotone rounding fl(|y_q - y_p|) >= fl(b_{t+1} - b_t) and   */
/* d2 >= fl(dy*dy) >= fl(fl(b_{t+1} - b_t)^2).  The code checks that this   */
/* last value exceeds eps2 for EVERY strip (else it returns -2), so no      */
/* neighbour is ever outside the three strips.  Per-row output as above.    */
/* ------------------------------------------------------------------------ */
static int strip_cmp(const void* a, const void* b)   /* keys (strip, x, id) */
{
    const double* u = (const double*)a;
    const double* v = (const double*)b;
    if (u[0] < v[0]) return -1;
    if (u[0] > v[0]) return 1;
    if (u[1] < v[1]) return -1;
    if (u[1] > v[1]) return 1;
    return (u[2] > v[2]) - (u[2] < v[2]);
}

static int cmp_u32(const void* a, const void* b)
{
    uint32_t u = *(const uint32_t*)a, v = *(const uint32_t*)b;
    return (u > v) - (u < v);
}

#define DEFINE_STRIPS(T, SUF, IS_NEIGHBOR)                                                     \
typedef struct { int64_t n, ns; T *sx, *sy; int64_t *sid, *sst, *sbeg; } strips_##SUF;        \
static void strips_free_##SUF(strips_##SUF* s)                                                 \
{                                                                                              \
    free(s->sx); free(s->sy); free(s->sid); free(s->sst); free(s->sbeg);                       \
}                                                                                              \
/* 0 = ok, -1 = allocation failed, -2 = a strip is not wider than eps */                      \
static int strips_build_##SUF(const T* xy, int64_t n, T eps, T eps2, strips_##SUF* s)         \
{                                                                                              \
    memset(s, 0, sizeof(*s));                                                                  \
    s->n = n;                                                                                  \
    double ymin = 0, ymax = 0;                                                                 \
    for (int64_t k = 0; k < n; ++k) {                                                          \
        double y = (double)xy[2 * k + 1];                                                      \
        if (k == 0 || y < ymin) ymin = y;                                                      \
        if (k == 0 || y > ymax) ymax = y;                                                      \
    }                                                                                          \
    double H = 2.0 * (double)eps;                                                              \
    if ((ymax - ymin) / H > (double)(1 << 22)) H = (ymax - ymin) / (double)(1 << 22);          \
    int64_t ns = (int64_t)((ymax - ymin) / H) + 2;                                             \
    s->ns = ns;                                                                                \
    T* b = (T*)malloc(sizeof(T) * (size_t)(ns + 1));                                           \
    s->sbeg = (int64_t*)calloc((size_t)(ns + 1), sizeof(int64_t));                             \
    int64_t* sk = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n ? n : 1));                     \
    if (!b || !s->sbeg || !sk) { free(b); free(sk); strips_free_##SUF(s); return -1; }         \
    for (int64_t t = 0; t <= ns; ++t) b[t] = (T)(ymin + (double)t * H);                       \
    b[0] = (T)ymin;                                                                            \
    for (int64_t t = 0; t < ns; ++t) {   /* every strip is wider than eps (header above) */    \
        T wd = b[t + 1] - b[t];                                                                \
        T wd2 = wd * wd;                                                                       \
        if (!(wd2 > eps2)) { free(b); free(sk); strips_free_##SUF(s); return -2; }             \
    }                                                                                          \
    if (!((double)b[ns] > ymax)) { free(b); free(sk); strips_free_##SUF(s); return -2; }       \
    for (int64_t k = 0; k < n; ++k) {   /* strip of k: last t with b[t] <= y */                \
        T y = xy[2 * k + 1];                                                                   \
        int64_t lo = 0, hi = ns;                                                               \
        while (hi - lo > 1) {                                                                  \
            int64_t m = lo + (hi - lo) / 2;                                                    \
            if (b[m] <= y) lo = m; else hi = m;                                                \
        }                                                                                      \
        sk[k] = lo;                                                                            \
        s->sbeg[lo + 1]++;                                                                     \
    }                                                                                          \
    free(b);                                                                                   \
    for (int64_t t = 0; t < ns; ++t) s->sbeg[t + 1] += s->sbeg[t];                             \
    int64_t* cur = (int64_t*)malloc(sizeof(int64_t) * (size_t)(ns + 1));                       \
    double* key = (double*)malloc(sizeof(double) * 3 * (size_t)(n ? n : 1));                  \
    s->sst = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n ? n : 1));                          \
    if (!cur || !key || !s->sst) { free(cur); free(key); free(sk); strips_free_##SUF(s); return -1; } \
    memcpy(cur, s->sbeg, sizeof(int64_t) * (size_t)(ns + 1));                                  \
    for (int64_t k = 0; k < n; ++k) {   /* counting scatter by strip */                        \
        int64_t d = cur[sk[k]]++;                                                              \
        key[3 * d] = (double)sk[k];                                                            \
        key[3 * d + 1] = (double)xy[2 * k];                                                    \
        key[3 * d + 2] = (double)k;                                                            \
        s->sst[d] = sk[k];                                                                     \
    }                                                                                          \
    free(cur); free(sk);                                                                       \
    int64_t t_;                                                                                \
    _Pragma("omp parallel for schedule(dynamic, 16)")                                          \
    for (t_ = 0; t_ < ns; ++t_)   /* each strip by (x, id) */                                  \
        qsort(key + 3 * s->sbeg[t_], (size_t)(s->sbeg[t_ + 1] - s->sbeg[t_]), 3 * sizeof(double), strip_cmp); \
    s->sx = (T*)malloc(sizeof(T) * (size_t)(n ? n : 1));                                       \
    s->sy = (T*)malloc(sizeof(T) * (size_t)(n ? n : 1));                                       \
    s->sid = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n ? n : 1));                          \
    if (!s->sx || !s->sy || !s->sid) { free(key); strips_free_##SUF(s); return -1; }           \
    for (int64_t k = 0; k < n; ++k) {                                                          \
        s->sid[k] = (int64_t)key[3 * k + 2];                                                   \
        s->sx[k] = xy[2 * s->sid[k]];                                                          \
        s->sy[k] = xy[2 * s->sid[k] + 1];                                                      \
    }                                                                                          \
    free(key);                                                                                 \
    return 0;                                                                                  \
}                                                                                              \
/* x-window [*jb, *je) of strip t around xp: the plane sweep's stop points     */             \
/* (exact: fl(x_j - xp) is monotone along the strip's x order)                 */             \
static void strips_window_##SUF(const strips_##SUF* s, int64_t t, T xp, T eps2, int64_t* jb, int64_t* je) \
{                                                                                              \
    int64_t lo = s->sbeg[t], hi = s->sbeg[t + 1];                                              \
    while (lo < hi) {   /* first j not left-outside (dx < 0, dx^2 > eps2) */                   \
        int64_t m = lo + (hi - lo) / 2;                                                        \
        T dx = s->sx[m] - xp;                                                                  \
        if (dx < 0 && dx * dx > eps2) lo = m + 1; else hi = m;                                 \
    }                                                                                          \
    *jb = lo;                                                                                  \
    hi = s->sbeg[t + 1];                                                                       \
    while (lo < hi) {   /* first j right-outside (dx > 0, dx^2 > eps2) */                      \
        int64_t m = lo + (hi - lo) / 2;                                                        \
        T dx = s->sx[m] - xp;                                                                  \
        if (dx > 0 && dx * dx > eps2) hi = m; else lo = m + 1;                                 \
    }                                                                                          \
    *je = lo;                                                                                  \
}                                                                                              \
int oracle_strip_rowhash_##SUF(const T* xy, int64_t n, T eps, uint64_t* cnt, uint64_t* hash)  \
{                                                                                              \
    T eps2 = eps * eps;                                                                        \
    strips_##SUF s;                                                                            \
    int rc = strips_build_##SUF(xy, n, eps, eps2, &s);                                         \
    if (rc) return rc;                                                                         \
    int64_t i;                                                                                 \
    _Pragma("omp parallel for schedule(dynamic, 256)")                                         \
    for (i = 0; i < n; ++i) {                                                                  \
        T xp = s.sx[i], yp = s.sy[i];                                                          \
        uint64_t c = 0, h = 0;                                                                 \
        for (int64_t t = s.sst[i] - 1; t <= s.sst[i] + 1; ++t) {                               \
            if (t < 0 || t >= s.ns) continue;                                                  \
            int64_t jb, je;                                                                    \
            strips_window_##SUF(&s, t, xp, eps2, &jb, &je);                                    \
            for (int64_t j = jb; j < je; ++j) {                                                \
                int hit = IS_NEIGHBOR(xp, yp, s.sx[j], s.sy[j], eps2);                         \
                c += (uint64_t)hit;                                                            \
                h += hit ? mix64((uint64_t)s.sid[j]) : 0;                                      \
            }                                                                                  \
        }                                                                                      \
        cnt[s.sid[i]] = c;                                                                     \
        hash[s.sid[i]] = h;                                                                    \
    }                                                                                          \
    strips_free_##SUF(&s);                                                                     \
    return 0;                                                                                  \
}                                                                                              \
/* O2 as a full CSR table (count then fill, each list ascending): off[n+1]   */               \
/* is filled here; nbr must hold off[n] entries (second call)                */               \
int oracle_strip_join_##SUF(const T* xy, int64_t n, T eps, uint64_t* off, uint32_t* nbr)       \
{                                                                                              \
    T eps2 = eps * eps;                                                                        \
    strips_##SUF s;                                                                            \
    int rc = strips_build_##SUF(xy, n, eps, eps2, &s);                                         \
    if (rc) return rc;                                                                         \
    int64_t i;                                                                                 \
    if (!nbr) {   /* count pass: off[p + 1] = |N_eps(p)|, then the prefix sum */               \
        off[0] = 0;                                                                            \
        _Pragma("omp parallel for schedule(dynamic, 256)")                                     \
        for (i = 0; i < n; ++i) {                                                              \
            T xp = s.sx[i], yp = s.sy[i];                                                      \
            uint64_t c = 0;                                                                    \
            for (int64_t t = s.sst[i] - 1; t <= s.sst[i] + 1; ++t) {                           \
                if (t < 0 || t >= s.ns) continue;                                              \
                int64_t jb, je;                                                                \
                strips_window_##SUF(&s, t, xp, eps2, &jb, &je);                                \
                for (int64_t j = jb; j < je; ++j) c += (uint64_t)IS_NEIGHBOR(xp, yp, s.sx[j], s.sy[j], eps2); \
            }                                                                                  \
            off[s.sid[i] + 1] = c;                                                             \
        }                                                                                      \
        for (int64_t p = 0; p < n; ++p) off[p + 1] += off[p];                                  \
    } else {      /* fill pass: the lists at off[p], sorted ascending */                       \
        _Pragma("omp parallel for schedule(dynamic, 256)")                                     \
        for (i = 0; i < n; ++i) {                                                              \
            T xp = s.sx[i], yp = s.sy[i];                                                      \
            uint32_t* out = nbr + off[s.sid[i]];                                               \
            uint64_t c = 0;                                                                    \
            for (int64_t t = s.sst[i] - 1; t <= s.sst[i] + 1; ++t) {                           \
                if (t < 0 || t >= s.ns) continue;                                              \
                int64_t jb, je;                                                                \
                strips_window_##SUF(&s, t, xp, eps2, &jb, &je);                                \
                for (int64_t j = jb; j < je; ++j)                                              \
                    if (IS_NEIGHBOR(xp, yp, s.sx[j], s.sy[j], eps2)) out[c++] = (uint32_t)s.sid[j]; \
            }                                                                                  \
            qsort(out, (size_t)c, sizeof(uint32_t), cmp_u32);                                  \
        }                                                                                      \
    }                                                                                          \
    strips_free_##SUF(&s);                                                                     \
    return 0;                                                                                  \
}

DEFINE_STRIPS(double, f64, is_neighbor_f64)
DEFINE_STRIPS(float, f32, is_neighbor_f32)

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
