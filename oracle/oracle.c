/*
 * oracle.c -- CPU oracle for the distance similarity self-join.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant generator with the CUDA path (paper_conf_ipps_galletg19_b200/).
 *
 * What it computes (the plain definition, §II-A):
 *     R(D, eps) = { (i, j) : i != j, s(i, j) <= e2 }
 *     s(i, j)   = fl(...fl(fl(t_0*t_0) + fl(t_1*t_1)) + ... + fl(t_{n-1}*t_{n-1}))
 *     t_d       = fl(p_i[d] - p_j[d]),   e2 = fl(eps*eps)
 * IEEE-754 binary64, round to nearest even, summed in dimension order, no FMA
 * (compiled with -ffp-contract=off; readings c1, c2).  Self pairs are
 * excluded, exact duplicates i != j are kept (reading c3); both orders (i, j) and
 * (j, i) are in R (reading c4, "add both pairs").
 *
 * O1 (brute force, "two nested loops"): evaluates s(i, j) for every
 *    ordered i != j.  Obviously correct; O(N^2).
 * O2 (CPU grid, "cells of length eps ... only its surrounding cells",
 *    up to 3^n cells): cells of side w = eps*(1+2^-20) anchored at the per-dimension
 *    minimum (readings c5, c6), a hash map from the integer cell tuple to the list of
 *    point ids, and a FULL 3^n neighbourhood scan for every query point.  It does not
 *    use any unidirectional pattern, work queue or sort by workload.
 *
 * Parity status: O1 pinned by closed forms / 1-D two-pointer / hand-checked sets
 * (tests/test_oracle.py); O2 pinned against O1 by brute force on small inputs.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORC_OK 0
#define ORC_EINVAL (-1)
#define ORC_ENOMEM (-2)
#define ORC_ECAP (-3)
#define ORC_EGRID (-4)

/* s(i, j) exactly as defined above (dimension order, separate mul and add). */
static inline double sqdist(const double *a, const double *b, int dim) {
    double s = 0.0;
    for (int d = 0; d < dim; ++d) {
        double t = a[d] - b[d];
        double t2 = t * t;
        s = s + t2;
    }
    return s;
}

/* Order-independent multiset hash of the pair set (test tooling, not method arithmetic). */
static inline uint64_t mix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static inline uint64_t pair_key(uint64_t i, uint64_t j) { return (i << 32) | j; }

int orc_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void orc_set_threads(int t) {
#ifdef _OPENMP
    if (t > 0) omp_set_num_threads(t);
#else
    (void)t;
#endif
}

static int check_args(const double *pts, uint64_t n, int dim, double eps) {
    if (!pts && n) return ORC_EINVAL;
    if (dim < 1 || dim > 8) return ORC_EINVAL;
    if (!(eps > 0.0) || !isfinite(eps)) return ORC_EINVAL;
    if (n >= (1ull << 32)) return ORC_EINVAL;
    for (uint64_t k = 0; k < n * (uint64_t)dim; ++k)
        if (!isfinite(pts[k])) return ORC_EINVAL;
    return ORC_OK;
}

/* ------------------------------------------------------------------ O1 ------ */

/* Brute force over all ordered (i, j), i != j.  Counts pairs, and (optionally)
 * accumulates the multiset hash.  */
int orc_bf_count(const double *pts, uint64_t n, int dim, double eps,
                 uint64_t *count, uint64_t *hash) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    const double e2 = eps * eps;
    uint64_t c = 0, h = 0;
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : c, h)
    for (int64_t i = 0; i < (int64_t)n; ++i) {
        const double *pi = pts + (uint64_t)i * dim;
        for (uint64_t j = 0; j < n; ++j) {
            if ((uint64_t)i == j) continue;
            if (sqdist(pi, pts + j * dim, dim) <= e2) {
                ++c;
                h += mix64(pair_key((uint64_t)i, j));
            }
        }
    }
    if (count) *count = c;
    if (hash) *hash = h;
    return ORC_OK;
}

/* Neighbour rows of selected query points, by brute force.
 * rows[nrows]: query ids.  offsets[nrows+1] receives the row starts.
 * cols: NULL for a sizing call, else capacity `cap` entries; each row ascending j. */
int orc_bf_rows(const double *pts, uint64_t n, int dim, double eps,
                const uint32_t *rows, uint64_t nrows,
                uint64_t *offsets, uint32_t *cols, uint64_t cap) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    if (!offsets || (nrows && !rows)) return ORC_EINVAL;
    for (uint64_t r = 0; r < nrows; ++r)
        if (rows[r] >= n) return ORC_EINVAL;
    const double e2 = eps * eps;
    uint64_t *cnt = (uint64_t *)calloc(nrows + 1, sizeof(uint64_t));
    if (!cnt) return ORC_ENOMEM;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t r = 0; r < (int64_t)nrows; ++r) {
        const uint64_t i = rows[r];
        const double *pi = pts + i * dim;
        uint64_t c = 0;
        for (uint64_t j = 0; j < n; ++j)
            if (j != i && sqdist(pi, pts + j * dim, dim) <= e2) ++c;
        cnt[r] = c;
    }
    offsets[0] = 0;
    for (uint64_t r = 0; r < nrows; ++r) offsets[r + 1] = offsets[r] + cnt[r];
    free(cnt);
    if (!cols) return ORC_OK;
    if (offsets[nrows] > cap) return ORC_ECAP;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t r = 0; r < (int64_t)nrows; ++r) {
        const uint64_t i = rows[r];
        const double *pi = pts + i * dim;
        uint64_t o = offsets[r];
        for (uint64_t j = 0; j < n; ++j)
            if (j != i && sqdist(pi, pts + j * dim, dim) <= e2) cols[o++] = (uint32_t)j;
    }
    return ORC_OK;
}

/* All pairs by brute force, canonical (i, j) order.  out: 2*cap uint32 or NULL. */
int orc_bf_pairs(const double *pts, uint64_t n, int dim, double eps,
                 uint32_t *out, uint64_t cap, uint64_t *count) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    uint32_t *rows = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    uint64_t *off = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    if (!rows || !off) { free(rows); free(off); return ORC_ENOMEM; }
    for (uint64_t i = 0; i < n; ++i) rows[i] = (uint32_t)i;
    rc = orc_bf_rows(pts, n, dim, eps, rows, n, off, NULL, 0);
    if (rc) goto done;
    *count = off[n];
    if (!out) goto done;
    if (off[n] > cap) { rc = ORC_ECAP; goto done; }
    {
        uint32_t *cols = (uint32_t *)malloc((off[n] ? off[n] : 1) * sizeof(uint32_t));
        if (!cols) { rc = ORC_ENOMEM; goto done; }
        rc = orc_bf_rows(pts, n, dim, eps, rows, n, off, cols, off[n]);
        if (!rc)
            for (uint64_t i = 0; i < n; ++i)
                for (uint64_t e = off[i]; e < off[i + 1]; ++e) {
                    out[2 * e] = (uint32_t)i;
                    out[2 * e + 1] = cols[e];
                }
        free(cols);
    }
done:
    free(rows);
    free(off);
    return rc;
}

/* ------------------------------------------------------------------ O2 ------ */

typedef struct {
    uint64_t n;
    int dim;
    double e2;
    const double *pts;
    int64_t *coord;     /* n*dim integer cell tuples                     */
    uint64_t ncells;
    uint64_t *cell_first;  /* ncells+1 : start of each cell in `ids`      */
    uint32_t *ids;         /* point ids grouped by cell, ascending inside  */
    int64_t *cell_coord;   /* ncells*dim                                   */
    uint64_t hcap;         /* hash capacity (power of two)                 */
    int64_t *htab;         /* cell index or -1                             */
} grid_t;

static uint64_t tuple_hash(const int64_t *c, int dim) {
    uint64_t h = 0x84222325cbf29ce4ull;
    for (int d = 0; d < dim; ++d) h = mix64(h ^ (uint64_t)c[d]);
    return h;
}

static int64_t grid_find(const grid_t *g, const int64_t *c) {
    uint64_t h = tuple_hash(c, g->dim) & (g->hcap - 1);
    for (;;) {
        int64_t v = g->htab[h];
        if (v < 0) return -1;
        if (memcmp(g->cell_coord + (uint64_t)v * g->dim, c, sizeof(int64_t) * g->dim) == 0) return v;
        h = (h + 1) & (g->hcap - 1);
    }
}

static void grid_free(grid_t *g) {
    free(g->coord); free(g->cell_first); free(g->ids); free(g->cell_coord); free(g->htab);
    memset(g, 0, sizeof(*g));
}

/* Cells of side w = eps*(1+2^-20) from the per-dimension minimum (readings c5, c6):
 * c_d = floor( fl( fl(x_d - min_d) / w ) ).  */
static int grid_build(grid_t *g, const double *pts, uint64_t n, int dim, double eps) {
    memset(g, 0, sizeof(*g));
    g->n = n; g->dim = dim; g->pts = pts; g->e2 = eps * eps;
    const double w = eps * (1.0 + 0x1p-20);
    double mn[8];
    for (int d = 0; d < dim; ++d) {
        mn[d] = INFINITY;
        for (uint64_t i = 0; i < n; ++i) if (pts[i * dim + d] < mn[d]) mn[d] = pts[i * dim + d];
    }
    g->coord = (int64_t *)malloc((n * dim + 1) * sizeof(int64_t));
    if (!g->coord) return ORC_ENOMEM;
    for (uint64_t i = 0; i < n; ++i)
        for (int d = 0; d < dim; ++d) {
            double q = (pts[i * dim + d] - mn[d]) / w;
            if (!(q < 0x1p30)) { grid_free(g); return ORC_EGRID; }  /* rounding argument needs q < 2^30 */
            g->coord[i * dim + d] = (int64_t)floor(q);
        }
    /* hash map tuple -> cell index, first-seen order */
    g->hcap = 16;
    while (g->hcap < 2 * (n + 1)) g->hcap <<= 1;
    g->htab = (int64_t *)malloc(g->hcap * sizeof(int64_t));
    g->cell_coord = (int64_t *)malloc((n * dim + 1) * sizeof(int64_t));
    uint32_t *cell_of = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    uint64_t *cnt = (uint64_t *)calloc(n + 2, sizeof(uint64_t));
    if (!g->htab || !g->cell_coord || !cell_of || !cnt) { free(cell_of); free(cnt); grid_free(g); return ORC_ENOMEM; }
    for (uint64_t h = 0; h < g->hcap; ++h) g->htab[h] = -1;
    uint64_t nc = 0;
    for (uint64_t i = 0; i < n; ++i) {
        const int64_t *c = g->coord + i * dim;
        int64_t v = grid_find(g, c);
        if (v < 0) {
            v = (int64_t)nc++;
            memcpy(g->cell_coord + (uint64_t)v * dim, c, sizeof(int64_t) * dim);
            uint64_t h = tuple_hash(c, dim) & (g->hcap - 1);
            while (g->htab[h] >= 0) h = (h + 1) & (g->hcap - 1);
            g->htab[h] = v;
        }
        cell_of[i] = (uint32_t)v;
        cnt[v + 1]++;
    }
    g->ncells = nc;
    g->cell_first = (uint64_t *)malloc((nc + 1) * sizeof(uint64_t));
    g->ids = (uint32_t *)malloc((n + 1) * sizeof(uint32_t));
    if (!g->cell_first || !g->ids) { free(cell_of); free(cnt); grid_free(g); return ORC_ENOMEM; }
    g->cell_first[0] = 0;
    for (uint64_t v = 0; v < nc; ++v) g->cell_first[v + 1] = g->cell_first[v] + cnt[v + 1];
    for (uint64_t v = 0; v < nc; ++v) cnt[v] = g->cell_first[v];
    for (uint64_t i = 0; i < n; ++i) g->ids[cnt[cell_of[i]]++] = (uint32_t)i;  /* ascending ids */
    free(cell_of);
    free(cnt);
    return ORC_OK;
}

static int cmp_u32(const void *a, const void *b) {
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return (x > y) - (x < y);
}

/* Full 3^dim neighbourhood scan for query i.  If cols != NULL, writes the neighbour
 * ids (unsorted).  Returns the neighbour count; *calcs gets the candidates evaluated. */
static uint64_t grid_query(const grid_t *g, uint64_t i, uint32_t *cols, uint64_t *calcs) {
    const int dim = g->dim;
    const int64_t *ci = g->coord + i * dim;
    const double *pi = g->pts + i * dim;
    int64_t nb[8] = {0};
    int off[8];
    for (int d = 0; d < dim; ++d) off[d] = -1;
    uint64_t c = 0, ev = 0;
    for (;;) {
        for (int d = 0; d < dim; ++d) nb[d] = ci[d] + off[d];
        int64_t v = grid_find(g, nb);
        if (v >= 0) {
            for (uint64_t e = g->cell_first[v]; e < g->cell_first[v + 1]; ++e) {
                uint32_t j = g->ids[e];
                if (j == i) continue;
                ++ev;
                if (sqdist(pi, g->pts + (uint64_t)j * dim, dim) <= g->e2) {
                    if (cols) cols[c] = j;
                    ++c;
                }
            }
        }
        int d = dim - 1;  /* odometer over {-1,0,1}^dim */
        while (d >= 0 && off[d] == 1) { off[d] = -1; --d; }
        if (d < 0) break;
        off[d]++;
    }
    *calcs = ev;
    return c;
}

/* Count, distance-calculation count (full 3^n scan, j != i) and multiset hash. */
int orc_grid_count(const double *pts, uint64_t n, int dim, double eps,
                   uint64_t *count, uint64_t *calcs, uint64_t *hash, uint64_t *ncells) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    grid_t g;
    rc = grid_build(&g, pts, n, dim, eps);
    if (rc) return rc;
    uint64_t c = 0, ev = 0, h = 0;
    int64_t maxrow = 0;
#pragma omp parallel reduction(+ : c, ev, h)
    {
        /* row buffer sized by the largest 3^n neighbourhood is not known up front;
         * grow on demand. */
        uint64_t bcap = 1024;
        uint32_t *buf = (uint32_t *)malloc(bcap * sizeof(uint32_t));
#pragma omp for schedule(dynamic, 256)
        for (int64_t i = 0; i < (int64_t)n; ++i) {
            uint64_t e;
            uint64_t k = grid_query(&g, (uint64_t)i, NULL, &e);
            if (k > bcap) { while (bcap < k) bcap <<= 1; buf = (uint32_t *)realloc(buf, bcap * sizeof(uint32_t)); }
            if (hash) grid_query(&g, (uint64_t)i, buf, &e);
            c += k;
            ev += e;
            if (hash)
                for (uint64_t t = 0; t < k; ++t) h += mix64(pair_key((uint64_t)i, buf[t]));
        }
        free(buf);
    }
    (void)maxrow;
    if (count) *count = c;
    if (calcs) *calcs = ev;
    if (hash) *hash = h;
    if (ncells) *ncells = g.ncells;
    grid_free(&g);
    return ORC_OK;
}

/* Rows of selected queries through the grid (each row ascending). */
int orc_grid_rows(const double *pts, uint64_t n, int dim, double eps,
                  const uint32_t *rows, uint64_t nrows,
                  uint64_t *offsets, uint32_t *cols, uint64_t cap) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    if (!offsets || (nrows && !rows)) return ORC_EINVAL;
    for (uint64_t r = 0; r < nrows; ++r)
        if (rows[r] >= n) return ORC_EINVAL;
    grid_t g;
    rc = grid_build(&g, pts, n, dim, eps);
    if (rc) return rc;
    uint64_t *cnt = (uint64_t *)calloc(nrows + 1, sizeof(uint64_t));
    if (!cnt) { grid_free(&g); return ORC_ENOMEM; }
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < (int64_t)nrows; ++r) {
        uint64_t e;
        cnt[r] = grid_query(&g, rows[r], NULL, &e);
    }
    offsets[0] = 0;
    for (uint64_t r = 0; r < nrows; ++r) offsets[r + 1] = offsets[r] + cnt[r];
    free(cnt);
    if (cols) {
        if (offsets[nrows] > cap) { grid_free(&g); return ORC_ECAP; }
#pragma omp parallel for schedule(dynamic, 64)
        for (int64_t r = 0; r < (int64_t)nrows; ++r) {
            uint64_t e;
            uint32_t *row = cols + offsets[r];
            uint64_t k = grid_query(&g, rows[r], row, &e);
            qsort(row, k, sizeof(uint32_t), cmp_u32);
        }
    }
    grid_free(&g);
    return ORC_OK;
}

/* All pairs through the grid, canonical (i, j) order. out: 2*cap uint32 or NULL. */
int orc_grid_pairs(const double *pts, uint64_t n, int dim, double eps,
                   uint32_t *out, uint64_t cap, uint64_t *count) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    uint32_t *rows = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    uint64_t *off = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    if (!rows || !off) { free(rows); free(off); return ORC_ENOMEM; }
    for (uint64_t i = 0; i < n; ++i) rows[i] = (uint32_t)i;
    rc = orc_grid_rows(pts, n, dim, eps, rows, n, off, NULL, 0);
    if (rc) goto done;
    *count = off[n];
    if (!out) goto done;
    if (off[n] > cap) { rc = ORC_ECAP; goto done; }
    {
        uint32_t *cols = (uint32_t *)malloc((off[n] ? off[n] : 1) * sizeof(uint32_t));
        if (!cols) { rc = ORC_ENOMEM; goto done; }
        rc = orc_grid_rows(pts, n, dim, eps, rows, n, off, cols, off[n]);
        if (!rc)
            for (uint64_t i = 0; i < n; ++i)
                for (uint64_t e = off[i]; e < off[i + 1]; ++e) {
                    out[2 * e] = (uint32_t)i;
                    out[2 * e + 1] = cols[e];
                }
        free(cols);
    }
done:
    free(rows);
    free(off);
    return rc;
}

/* The oracle's grid as (cell tuple, sorted member ids), for checking the GPU index.
 * Sizing call with coords == NULL returns *ncells.  coords: ncells*dim int64,
 * first: ncells+1, ids: n.  Cells in first-seen order. */
int orc_grid_cells(const double *pts, uint64_t n, int dim, double eps,
                   int64_t *coords, uint64_t *first, uint32_t *ids, uint64_t *ncells) {
    int rc = check_args(pts, n, dim, eps);
    if (rc) return rc;
    grid_t g;
    rc = grid_build(&g, pts, n, dim, eps);
    if (rc) return rc;
    *ncells = g.ncells;
    if (coords) {
        memcpy(coords, g.cell_coord, g.ncells * dim * sizeof(int64_t));
        memcpy(first, g.cell_first, (g.ncells + 1) * sizeof(uint64_t));
        memcpy(ids, g.ids, n * sizeof(uint32_t));
    }
    grid_free(&g);
    return ORC_OK;
}

/* A persistent O2 grid (the same grid_build / grid_query as above, built once) for the
 * full-size element-wise comparisons, which walk the queries in blocks of ids and would
 * otherwise rebuild the grid per block.  The caller keeps `pts` alive until
 * orc_grid_delete.  No new arithmetic: only the lifetime of the grid differs. */
void *orc_grid_new(const double *pts, uint64_t n, int dim, double eps, int *rc_out) {
    int rc = check_args(pts, n, dim, eps);
    grid_t *g = NULL;
    if (!rc) {
        g = (grid_t *)malloc(sizeof(grid_t));
        if (!g) rc = ORC_ENOMEM;
        else if ((rc = grid_build(g, pts, n, dim, eps)) != ORC_OK) { free(g); g = NULL; }
    }
    if (rc_out) *rc_out = rc;
    return g;
}

void orc_grid_delete(void *gp) {
    if (!gp) return;
    grid_free((grid_t *)gp);
    free(gp);
}

/* Rows of the queries lo .. hi-1 (each row ascending), offsets[hi-lo+1]; cols NULL for a
 * sizing call.  Rows in query order, so (i, cols) is already canonical (i, j) order. */
int orc_grid_rows_range(void *gp, uint64_t lo, uint64_t hi, uint64_t *offsets, uint32_t *cols, uint64_t cap) {
    const grid_t *g = (const grid_t *)gp;
    if (!g || !offsets || lo > hi || hi > g->n) return ORC_EINVAL;
    const uint64_t nr = hi - lo;
    uint64_t *cnt = (uint64_t *)calloc(nr + 1, sizeof(uint64_t));
    if (!cnt) return ORC_ENOMEM;
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < (int64_t)nr; ++r) {
        uint64_t e;
        cnt[r] = grid_query(g, lo + (uint64_t)r, NULL, &e);
    }
    offsets[0] = 0;
    for (uint64_t r = 0; r < nr; ++r) offsets[r + 1] = offsets[r] + cnt[r];
    free(cnt);
    if (!cols) return ORC_OK;
    if (offsets[nr] > cap) return ORC_ECAP;
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t r = 0; r < (int64_t)nr; ++r) {
        uint64_t e;
        uint32_t *row = cols + offsets[r];
        uint64_t k = grid_query(g, lo + (uint64_t)r, row, &e);
        qsort(row, k, sizeof(uint32_t), cmp_u32);
    }
    return ORC_OK;
}

/* The multiset hash of an explicit pair list (so tests hash GPU output with the same
 * function the oracle uses, without re-implementing it). */
uint64_t orc_hash_pairs(const uint32_t *pairs, uint64_t count) {
    uint64_t h = 0;
#pragma omp parallel for reduction(+ : h) schedule(static)
    for (int64_t e = 0; e < (int64_t)count; ++e)
        h += mix64(pair_key(pairs[2 * e], pairs[2 * e + 1]));
    return h;
}
