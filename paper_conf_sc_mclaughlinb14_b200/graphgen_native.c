/*
 * graphgen_native.c -- fast seeded input generation (shared by the CUDA path's
 * tests/bench and the oracle's tests).  Holds NONE of the method's arithmetic:
 * it only draws random edges and builds a simple CSR (no BFS, no path counts).
 *
 *   gg_rmat_edges : Graph500-style R-MAT edge list (Chakrabarti et al. [11],
 *                   PAPER.md:336) with a counter-based RNG, so every edge is a
 *                   pure function of (seed, edge index) and the draw is parallel.
 *   gg_permutation: seeded Fisher-Yates permutation (vertex relabelling).
 *   gg_csr_build  : drop self-loops, (symmetrise), sort rows, drop duplicates.
 *
 * Plain C99 + pthreads; compiled by graphgen.py / the Makefile with gcc -O2.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t splitmix64(uint64_t x)
{
    x += 0x9E3779B97F4A7C15ULL;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
    return x ^ (x >> 31);
}

/* uniform double in [0, 1) from (seed, counter) */
static inline double u01(uint64_t seed, uint64_t ctr)
{
    return (double)(splitmix64(splitmix64(seed) ^ ctr) >> 11) * (1.0 / 9007199254740992.0);
}

typedef struct {
    int scale;
    double ab, a_norm, c_norm;
    uint64_t seed;
    int64_t lo, hi;
    int64_t *u, *v;
} rmat_job;

static void *rmat_worker(void *arg)
{
    rmat_job *j = (rmat_job *)arg;
    for (int64_t i = j->lo; i < j->hi; i++) {
        int64_t u = 0, v = 0;
        for (int b = 0; b < j->scale; b++) {
            const uint64_t ctr = ((uint64_t)i * (uint64_t)j->scale + (uint64_t)b) << 1;
            const double r1 = u01(j->seed, ctr), r2 = u01(j->seed, ctr | 1);
            const int ii = r1 > j->ab;
            const int jj = r2 > (ii ? j->c_norm : j->a_norm);
            u |= (int64_t)ii << b;
            v |= (int64_t)jj << b;
        }
        j->u[i] = u;
        j->v[i] = v;
    }
    return NULL;
}

static int clamp_threads(int t) { return t < 1 ? 1 : (t > 64 ? 64 : t); }

/* ne edges of an R-MAT graph with 2^scale vertices; probabilities (a, b, c, 1-a-b-c). */
void gg_rmat_edges(int scale, int64_t ne, double a, double b, double c, uint64_t seed,
                   int64_t *u, int64_t *v, int nthreads)
{
    nthreads = clamp_threads(nthreads);
    pthread_t th[64];
    rmat_job jobs[64];
    const double ab = a + b;
    for (int t = 0; t < nthreads; t++) {
        jobs[t].scale = scale;
        jobs[t].ab = ab;
        jobs[t].a_norm = a / ab;
        jobs[t].c_norm = c / (1.0 - ab);
        jobs[t].seed = seed;
        jobs[t].lo = ne * t / nthreads;
        jobs[t].hi = ne * (t + 1) / nthreads;
        jobs[t].u = u;
        jobs[t].v = v;
        pthread_create(&th[t], NULL, rmat_worker, &jobs[t]);
    }
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
}

/* perm[i] = image of i under a seeded Fisher-Yates shuffle of 0..n-1. */
void gg_permutation(int64_t n, uint64_t seed, int64_t *perm)
{
    for (int64_t i = 0; i < n; i++) perm[i] = i;
    for (int64_t i = n - 1; i > 0; i--) {
        const int64_t j = (int64_t)(u01(seed ^ 0x5DEECE66DULL, (uint64_t)i) * (double)(i + 1));
        const int64_t t = perm[i];
        perm[i] = perm[j];
        perm[j] = t;
    }
}

/* ---------------------------------------------------------------- CSR build */

static int cmp_i32(const void *x, const void *y)
{
    const int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    return (a > b) - (a < b);
}

typedef struct {
    int64_t lo, hi;
    const int64_t *ro;
    int32_t *col;
    int64_t *newdeg;
} sort_job;

static void *sort_worker(void *arg)
{
    sort_job *j = (sort_job *)arg;
    for (int64_t r = j->lo; r < j->hi; r++) {
        int32_t *row = j->col + j->ro[r];
        const int64_t d = j->ro[r + 1] - j->ro[r];
        if (d > 1) qsort(row, (size_t)d, sizeof(int32_t), cmp_i32);
        int64_t k = 0;
        for (int64_t e = 0; e < d; e++)
            if (k == 0 || row[e] != row[k - 1]) row[k++] = row[e];
        j->newdeg[r] = k;
    }
    return NULL;
}

/* Build a simple CSR from an edge list.  Self-loops are dropped; undirected edges
 * are stored as both arcs; rows are sorted ascending and deduplicated.
 * ro_out: int64[n+1]; col_out: int32 with capacity (directed ? ne : 2*ne).
 * Returns nnz, or -1 on allocation failure / out-of-range endpoint. */
int64_t gg_csr_build(int64_t n, int64_t ne, const int64_t *u, const int64_t *v, int directed,
                     int64_t *ro_out, int32_t *col_out, int nthreads)
{
    nthreads = clamp_threads(nthreads);
    int64_t *deg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t *ro = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
    int64_t *newdeg = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    const int64_t cap = directed ? ne : 2 * ne;
    int32_t *tmp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(cap > 0 ? cap : 1));
    int64_t rc = -1;
    if (!deg || !fill || !ro || !newdeg || !tmp) goto done;
    for (int64_t i = 0; i < ne; i++) {
        if (u[i] < 0 || u[i] >= n || v[i] < 0 || v[i] >= n) goto done;
        if (u[i] == v[i]) continue;
        deg[u[i]]++;
        if (!directed) deg[v[i]]++;
    }
    ro[0] = 0;
    for (int64_t r = 0; r < n; r++) ro[r + 1] = ro[r] + deg[r];
    for (int64_t r = 0; r < n; r++) fill[r] = ro[r];
    for (int64_t i = 0; i < ne; i++) {
        if (u[i] == v[i]) continue;
        tmp[fill[u[i]]++] = (int32_t)v[i];
        if (!directed) tmp[fill[v[i]]++] = (int32_t)u[i];
    }
    {
        pthread_t th[64];
        sort_job jobs[64];
        for (int t = 0; t < nthreads; t++) {
            jobs[t].lo = n * t / nthreads;
            jobs[t].hi = n * (t + 1) / nthreads;
            jobs[t].ro = ro;
            jobs[t].col = tmp;
            jobs[t].newdeg = newdeg;
            pthread_create(&th[t], NULL, sort_worker, &jobs[t]);
        }
        for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    }
    ro_out[0] = 0;
    for (int64_t r = 0; r < n; r++) {
        ro_out[r + 1] = ro_out[r] + newdeg[r];
        memcpy(col_out + ro_out[r], tmp + ro[r], sizeof(int32_t) * (size_t)newdeg[r]);
    }
    rc = ro_out[n];
done:
    free(deg);
    free(fill);
    free(ro);
    free(newdeg);
    free(tmp);
    return rc;
}
