/*
 * gridjoin.c -- CPU comparator, BENCHMARK/TEST INFRASTRUCTURE ONLY.
 *
 * The "single-thread CPU grid-join" the north star asks to time beside the GPU
 * path (CPU baseline 2, and 3 with threads > 1): the same epsilon
 * self-join through an epsilon-grid index, written
 * plainly for one CPU core:
 *   - cell width w = eps_F * (1 + 2^-19), eps_F = eps in the predicate
 *     precision, FP64 cell arithmetic cx = floor((x - xmin) * fl(1/w))
 *     (R9/R10: the paper's width-eps cells, with the
 *     margin that makes floor-based assignment safe);
 *   - points sorted by (row-major cell key, id) with qsort (the paper's
 *     bin-sorted D);
 *   - per query, the three stencil rows y' in {cy-1, cy, cy+1} are each one
 *     contiguous run of the sorted points, found by binary search;
 *   - the predicate of O1 (no FMA: compiled with -ffp-contract=off).
 * Output: the query rows' neighbour lists (CSR, candidate order).
 *
 * It shares no code with the CUDA library (it is never linked into it) nor
 * with oracle/ (it is checked AGAINST the oracle in tests/).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#ifndef GJ_FP_CONTRACT_OFF
#error "gridjoin.c must be compiled with -ffp-contract=off -DGJ_FP_CONTRACT_OFF"
#endif

typedef struct {
    uint64_t key;
    uint32_t id;
} gj_item;

static int gj_cmp(const void* a, const void* b)
{
    const gj_item* u = (const gj_item*)a;
    const gj_item* v = (const gj_item*)b;
    if (u->key != v->key) return u->key < v->key ? -1 : 1;
    return (u->id > v->id) - (u->id < v->id);
}

typedef struct {
    int64_t n;
    double xmin, ymin, inv_w;
    uint64_t nx, ny;
    gj_item* items;      /* n, sorted by (key, id) */
    double* xs;          /* 2n, coordinates in sorted order (widened for f32) */
} gj_grid;

/* first index in [0, n) whose key >= k */
static int64_t gj_lower(const gj_item* it, int64_t n, uint64_t k)
{
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (it[mid].key < k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

static int gj_build(gj_grid* g, const double* xy, int64_t n, double eps_f)
{
    memset(g, 0, sizeof *g);
    g->n = n;
    if (n == 0) return 0;
    double xmin = xy[0], xmax = xy[0], ymin = xy[1], ymax = xy[1];
    for (int64_t i = 1; i < n; ++i) {
        double x = xy[2 * i], y = xy[2 * i + 1];
        if (x < xmin) xmin = x;
        if (x > xmax) xmax = x;
        if (y < ymin) ymin = y;
        if (y > ymax) ymax = y;
    }
    const double w = eps_f * (1.0 + 0x1p-19);
    const double inv_w = 1.0 / w;
    const double ex = (xmax - xmin) * inv_w, ey = (ymax - ymin) * inv_w;
    if (!(ex <= 0x1p30) || !(ey <= 0x1p30)) return -2;
    g->xmin = xmin;
    g->ymin = ymin;
    g->inv_w = inv_w;
    g->nx = (uint64_t)floor(ex) + 1;
    g->ny = (uint64_t)floor(ey) + 1;
    g->items = (gj_item*)malloc(sizeof(gj_item) * (size_t)n);
    g->xs = (double*)malloc(sizeof(double) * 2 * (size_t)n);
    if (!g->items || !g->xs) return -1;
    for (int64_t i = 0; i < n; ++i) {
        double cx = floor((xy[2 * i] - xmin) * inv_w), cy = floor((xy[2 * i + 1] - ymin) * inv_w);
        uint64_t ux = cx < 0 ? 0 : (uint64_t)cx, uy = cy < 0 ? 0 : (uint64_t)cy;
        if (ux > g->nx - 1) ux = g->nx - 1;
        if (uy > g->ny - 1) uy = g->ny - 1;
        g->items[i].key = uy * g->nx + ux;
        g->items[i].id = (uint32_t)i;
    }
    qsort(g->items, (size_t)n, sizeof(gj_item), gj_cmp);
    for (int64_t i = 0; i < n; ++i) {
        g->xs[2 * i] = xy[2 * (int64_t)g->items[i].id];
        g->xs[2 * i + 1] = xy[2 * (int64_t)g->items[i].id + 1];
    }
    return 0;
}

static void gj_free(gj_grid* g)
{
    free(g->items);
    free(g->xs);
}

/* the three stencil-row runs [lo[r], hi[r]) of the sorted points for point (x, y) */
static void gj_spans(const gj_grid* g, double x, double y, int64_t lo[3], int64_t hi[3])
{
    double fx = floor((x - g->xmin) * g->inv_w), fy = floor((y - g->ymin) * g->inv_w);
    uint64_t cx = fx < 0 ? 0 : (uint64_t)fx, cy = fy < 0 ? 0 : (uint64_t)fy;
    if (cx > g->nx - 1) cx = g->nx - 1;
    if (cy > g->ny - 1) cy = g->ny - 1;
    uint64_t x0 = cx ? cx - 1 : 0, x1 = cx + 1 < g->nx ? cx + 1 : cx;
    for (int r = 0; r < 3; ++r) {
        int64_t yy = (int64_t)cy + r - 1;
        if (yy < 0 || (uint64_t)yy >= g->ny) {
            lo[r] = hi[r] = 0;
            continue;
        }
        lo[r] = gj_lower(g->items, g->n, (uint64_t)yy * g->nx + x0);
        hi[r] = gj_lower(g->items, g->n, (uint64_t)yy * g->nx + x1 + 1);
    }
}

#define GJ_ROW(r) ((rows) ? rows[(r)] : (int64_t)(r))

/* Count then fill for the query rows (rows == NULL: all n).  Pass 1 writes
 * cnt[r]; the caller scans it into off[] and calls again with nbr != NULL.
 * The two passes share one grid (built in gj_prepare). */
static void gj_rows_f64(const gj_grid* g, const double* xy, double eps, const int64_t* rows, int64_t nrows,
                        int threads, uint64_t* cnt, const uint64_t* off, uint32_t* nbr)
{
    const double e2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 256) num_threads(threads)
    for (r = 0; r < nrows; ++r) {
        int64_t p = GJ_ROW(r);
        double xp = xy[2 * p], yp = xy[2 * p + 1];
        int64_t lo[3], hi[3];
        gj_spans(g, xp, yp, lo, hi);
        uint64_t c = 0, k = nbr ? off[r] : 0;
        for (int s = 0; s < 3; ++s)
            for (int64_t j = lo[s]; j < hi[s]; ++j) {
                double dx = xp - g->xs[2 * j];
                double dy = yp - g->xs[2 * j + 1];
                double dx2 = dx * dx;
                double dy2 = dy * dy;
                double d2 = dx2 + dy2;
                if (d2 <= e2) {
                    if (nbr) nbr[k++] = g->items[j].id;
                    ++c;
                }
            }
        if (!nbr) cnt[r] = c;
    }
}

static void gj_rows_f32(const gj_grid* g, const float* xy, float eps, const int64_t* rows, int64_t nrows,
                        int threads, uint64_t* cnt, const uint64_t* off, uint32_t* nbr)
{
    const float e2 = eps * eps;
    int64_t r;
#pragma omp parallel for schedule(dynamic, 256) num_threads(threads)
    for (r = 0; r < nrows; ++r) {
        int64_t p = GJ_ROW(r);
        float xp = xy[2 * p], yp = xy[2 * p + 1];
        int64_t lo[3], hi[3];
        gj_spans(g, (double)xp, (double)yp, lo, hi);
        uint64_t c = 0, k = nbr ? off[r] : 0;
        for (int s = 0; s < 3; ++s)
            for (int64_t j = lo[s]; j < hi[s]; ++j) {
                float dx = xp - (float)g->xs[2 * j];
                float dy = yp - (float)g->xs[2 * j + 1];
                float dx2 = dx * dx;
                float dy2 = dy * dy;
                float d2 = dx2 + dy2;
                if (d2 <= e2) {
                    if (nbr) nbr[k++] = g->items[j].id;
                    ++c;
                }
            }
        if (!nbr) cnt[r] = c;
    }
}

/* ---- public entry points (handle = opaque grid) ---------------------------- */
void* gj_prepare(const void* xy, int64_t n, int is_f32, double eps, int* status)
{
    gj_grid* g = (gj_grid*)calloc(1, sizeof(gj_grid));
    if (!g) {
        *status = -1;
        return NULL;
    }
    double* tmp = NULL;
    const double* xyd = (const double*)xy;
    double eps_f = eps;
    if (is_f32) {
        tmp = (double*)malloc(sizeof(double) * 2 * (size_t)(n ? n : 1));
        if (!tmp) {
            free(g);
            *status = -1;
            return NULL;
        }
        for (int64_t i = 0; i < 2 * n; ++i) tmp[i] = (double)((const float*)xy)[i];
        xyd = tmp;
        eps_f = (double)(float)eps;
    }
    *status = gj_build(g, xyd, n, eps_f);
    free(tmp);
    if (*status) {
        gj_free(g);
        free(g);
        return NULL;
    }
    return g;
}

void gj_release(void* h)
{
    if (!h) return;
    gj_free((gj_grid*)h);
    free(h);
}

void gj_count(void* h, const void* xy, int is_f32, double eps, const int64_t* rows, int64_t nrows, int threads,
              uint64_t* cnt)
{
    if (is_f32)
        gj_rows_f32((const gj_grid*)h, (const float*)xy, (float)eps, rows, nrows, threads, cnt, NULL, NULL);
    else
        gj_rows_f64((const gj_grid*)h, (const double*)xy, eps, rows, nrows, threads, cnt, NULL, NULL);
}

void gj_fill(void* h, const void* xy, int is_f32, double eps, const int64_t* rows, int64_t nrows, int threads,
             const uint64_t* off, uint32_t* nbr)
{
    if (is_f32)
        gj_rows_f32((const gj_grid*)h, (const float*)xy, (float)eps, rows, nrows, threads, NULL, off, nbr);
    else
        gj_rows_f64((const gj_grid*)h, (const double*)xy, eps, rows, nrows, threads, NULL, off, nbr);
}
