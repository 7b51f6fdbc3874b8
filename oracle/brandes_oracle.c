/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct serial Brandes betweenness centrality on the
 * CPU, written from the paper (McLaughlin & Bader, SC'14; /root/reference/
 * PAPER.md, cited "P:<line>").  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or helper with the CUDA path in
 * paper_conf_sc_mclaughlinb14_b200/csrc/ and includes nothing from it.
 *
 * What it computes (Eq.1, P:72 halving, Eq.2, Eq.3):
 *   BC(v) = h * sum_{s in S, s != v} delta_s(v),  h = 1/2 if undirected else 1,
 *   delta_s(v) = sum_{w : d(s,w) = d(s,v)+1, (v,w) in E} sigma_sv/sigma_sw (1+delta_s(w)).
 *
 * Variant 1 (oracle_bc / oracle_single_source) follows SURVEY.md §8(c)'s
 * step-by-step algorithm, i.e. the paper's two stages in its notation:
 *   Stage 1 (Alg. 2): BFS by levels in FIFO order, recording the
 *     visit order S and the level offsets `ends`; sigma of each new level
 *     is PULLED over the vertex's (in-)adjacency in CSR order: sigma_sw =
 *     sum over predecessors u of sigma_su (Brandes; the pull replaces Alg. 2's
 *     atomicAdd push so that the summation order is fixed).
 *   Stage 2 (Alg. 3): successor form, for depth = maxdepth-1 .. 1,
 *     dsw = sum_{v in N(w), d[v]=d[w]+1} sw/sigma[v]*(1+delta[v]) evaluated left
 *     to right in CSR order; bc[w] += delta[w] (the BC update Alg. 3 omits,
 *     Eq. 3).
 * Variant 2 (oracle_bc_push) is textbook Brandes 2001 [7]: sigma pushed in FIFO
 * order, predecessor lists, delta pushed to predecessors while popping S.
 *
 * Conventions: d = -1 for unreachable; sigma, delta, bc in fp64 (SURVEY §8(c)
 * #3); directed graphs use out-neighbours for discovery and successors and
 * in-neighbours (the transpose, in ascending source-id order) for the sigma
 * pull (#17); duplicate sources count with multiplicity (#15).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define ORACLE_OK 0
#define ORACLE_EINVAL (-1)
#define ORACLE_ENOMEM (-2)

typedef struct {
    int32_t n;
    const int64_t *ro;   /* out-adjacency (CSR) */
    const int32_t *col;
    const int64_t *iro;  /* in-adjacency (transpose); == ro/col if undirected */
    const int32_t *icol;
    int directed;
} ograph;

typedef struct {
    int32_t *d;
    double *sigma;
    double *delta;
    int32_t *S;      /* visit order, all levels */
    int32_t *ends;   /* level offsets into S: level L = S[ends[L] .. ends[L+1]) */
    int32_t nlevels; /* number of levels = maxdepth + 1 */
    int64_t n_reached, arcs_reached, dag_arcs;
} ostate;

static int state_alloc(ostate *st, int32_t n)
{
    memset(st, 0, sizeof(*st));
    st->d = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    st->sigma = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    st->delta = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    st->S = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    st->ends = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 2));
    if (!st->d || !st->sigma || !st->delta || !st->S || !st->ends) return ORACLE_ENOMEM;
    return ORACLE_OK;
}

static void state_free(ostate *st)
{
    free(st->d); free(st->sigma); free(st->delta); free(st->S); free(st->ends);
}

/* Build the transpose (in-adjacency) of a directed CSR.  Arcs are visited in
 * CSR order (ascending source), so each in-row lists sources ascending. */
static int build_transpose(int32_t n, const int64_t *ro, const int32_t *col,
                           int64_t **iro_out, int32_t **icol_out)
{
    int64_t nnz = ro[n];
    int64_t *iro = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t *icol = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!iro || !icol || !fill) { free(iro); free(icol); free(fill); return ORACLE_ENOMEM; }
    for (int64_t e = 0; e < nnz; e++) iro[col[e] + 1]++;
    for (int32_t v = 0; v < n; v++) iro[v + 1] += iro[v];
    for (int32_t v = 0; v < n; v++) fill[v] = iro[v];
    for (int32_t u = 0; u < n; u++)
        for (int64_t e = ro[u]; e < ro[u + 1]; e++) icol[fill[col[e]]++] = u;
    free(fill);
    *iro_out = iro;
    *icol_out = icol;
    return ORACLE_OK;
}

static int validate(int32_t n, const int64_t *ro, const int32_t *col)
{
    if (n < 0 || !ro) return ORACLE_EINVAL;
    if (ro[0] != 0) return ORACLE_EINVAL;
    for (int32_t v = 0; v < n; v++)
        if (ro[v + 1] < ro[v]) return ORACLE_EINVAL;
    for (int64_t e = 0; e < ro[n]; e++)
        if (col[e] < 0 || col[e] >= n) return ORACLE_EINVAL;
    return ORACLE_OK;
}

/* Alg. 1: d = inf (-1 here), sigma = 0, delta = 0; d[s] = 0, sigma[s] = 1;
 * S = [s]; ends = [0, 1]. */
static void alg1_init(const ograph *g, ostate *st, int32_t s)
{
    for (int32_t v = 0; v < g->n; v++) { st->d[v] = -1; st->sigma[v] = 0.0; st->delta[v] = 0.0; }
    st->d[s] = 0;
    st->sigma[s] = 1.0;
    st->S[0] = s;
    st->ends[0] = 0;
    st->ends[1] = 1;
    st->nlevels = 1;
}

/* Stage 1 (Alg. 2) with sigma pulled in CSR order; Stage 2 (Alg. 3,
 * P:202-227).  Adds delta into bc (un-halved) if bc != NULL. */
static void brandes_pull_one(const ograph *g, ostate *st, int32_t s, double *bc)
{
    alg1_init(g, st, s);
    int32_t S_len = 1;
    int64_t arcs = 0, dag = 0;
    for (;;) {
        int32_t L = st->nlevels - 1;
        int32_t lo = st->ends[L], hi = st->ends[L + 1];
        int32_t next_lo = S_len;
        /* discovery: for v in Q_curr (= level L), w in neighbors(v) */
        for (int32_t i = lo; i < hi; i++) {
            int32_t v = st->S[i];
            arcs += g->ro[v + 1] - g->ro[v];
            for (int64_t e = g->ro[v]; e < g->ro[v + 1]; e++) {
                int32_t w = g->col[e];
                if (st->d[w] < 0) { st->d[w] = L + 1; st->S[S_len++] = w; }
            }
        }
        if (S_len == next_lo) break; /* Q_next_len = 0 (Alg. 2 l.11) */
        /* sigma of the new level by pull: sigma[w] = sum_{u in pred(w)} sigma[u] */
        for (int32_t i = next_lo; i < S_len; i++) {
            int32_t w = st->S[i];
            double acc = 0.0;
            for (int64_t e = g->iro[w]; e < g->iro[w + 1]; e++) {
                int32_t u = g->icol[e];
                if (st->d[u] == st->d[w] - 1) { acc += st->sigma[u]; dag++; }
            }
            st->sigma[w] = acc;
        }
        st->ends[L + 2] = S_len; /* Alg. 2 l.18-19 */
        st->nlevels = L + 2;
    }
    st->n_reached = S_len;
    st->arcs_reached = arcs;
    st->dag_arcs = dag;
    /* Stage 2: depth = maxdepth - 1 down to 1 (Alg. 2 l.12, Alg. 3 l.2). */
    for (int32_t depth = st->nlevels - 2; depth > 0; depth--) {
        for (int32_t i = st->ends[depth]; i < st->ends[depth + 1]; i++) {
            int32_t w = st->S[i];
            double dsw = 0.0;
            double sw = st->sigma[w];
            for (int64_t e = g->ro[w]; e < g->ro[w + 1]; e++) {
                int32_t v = g->col[e];
                if (st->d[v] == st->d[w] + 1) dsw = dsw + sw / st->sigma[v] * (1.0 + st->delta[v]);
            }
            st->delta[w] = dsw;
            if (bc) bc[w] += dsw; /* Eq. 3 */
        }
    }
}

/* Textbook Brandes 2001 [7] (push sigma in FIFO order, predecessor lists). */
static void brandes_push_one(const ograph *g, ostate *st, int64_t *pred_fill,
                             int32_t *pred, int32_t s, double *bc)
{
    alg1_init(g, st, s);
    int32_t head = 0, tail = 1;
    for (int32_t v = 0; v < g->n; v++) pred_fill[v] = g->iro[v];
    while (head < tail) {
        int32_t v = st->S[head++];
        for (int64_t e = g->ro[v]; e < g->ro[v + 1]; e++) {
            int32_t w = g->col[e];
            if (st->d[w] < 0) { st->d[w] = st->d[v] + 1; st->S[tail++] = w; }
            if (st->d[w] == st->d[v] + 1) {
                st->sigma[w] += st->sigma[v];
                pred[pred_fill[w]++] = v;
            }
        }
    }
    for (int32_t i = tail - 1; i >= 0; i--) {
        int32_t w = st->S[i];
        for (int64_t p = g->iro[w]; p < pred_fill[w]; p++) {
            int32_t v = pred[p];
            st->delta[v] += st->sigma[v] / st->sigma[w] * (1.0 + st->delta[w]);
        }
        if (w != s && bc) bc[w] += st->delta[w];
    }
    st->n_reached = tail;
}

/* ------------------------------------------------------------- public entry */

typedef struct {
    const ograph *g;
    const int32_t *sources;
    int64_t lo, hi;
    double *bc;       /* private, n */
    int variant;      /* 0 pull, 1 push */
    int rc;
} job_t;

static void *run_job(void *arg)
{
    job_t *j = (job_t *)arg;
    ostate st;
    j->rc = state_alloc(&st, j->g->n);
    int64_t *pf = NULL;
    int32_t *pred = NULL;
    if (j->rc == ORACLE_OK && j->variant == 1) {
        pf = (int64_t *)malloc(sizeof(int64_t) * (size_t)(j->g->n > 0 ? j->g->n : 1));
        pred = (int32_t *)malloc(sizeof(int32_t) * (size_t)(j->g->ro[j->g->n] > 0 ? j->g->ro[j->g->n] : 1));
        if (!pf || !pred) j->rc = ORACLE_ENOMEM;
    }
    if (j->rc == ORACLE_OK) {
        for (int64_t i = j->lo; i < j->hi; i++) {
            if (j->variant == 0) brandes_pull_one(j->g, &st, j->sources[i], j->bc);
            else brandes_push_one(j->g, &st, pf, pred, j->sources[i], j->bc);
        }
    }
    free(pf); free(pred);
    state_free(&st);
    return NULL;
}

static int make_graph(ograph *g, int32_t n, const int64_t *ro, const int32_t *col,
                      int directed, int64_t **iro, int32_t **icol)
{
    int rc = validate(n, ro, col);
    if (rc) return rc;
    g->n = n; g->ro = ro; g->col = col; g->directed = directed;
    *iro = NULL; *icol = NULL;
    if (directed) {
        rc = build_transpose(n, ro, col, iro, icol);
        if (rc) return rc;
        g->iro = *iro; g->icol = *icol;
    } else {
        g->iro = ro; g->icol = col;
    }
    return ORACLE_OK;
}

static int oracle_bc_impl(int32_t n, const int64_t *ro, const int32_t *col, int directed,
                          const int32_t *sources, int64_t k, double *bc, int nthreads,
                          int variant)
{
    ograph g;
    int64_t *iro; int32_t *icol;
    int rc = make_graph(&g, n, ro, col, directed, &iro, &icol);
    if (rc) return rc;
    int32_t *all = NULL;
    if (!sources) {
        k = n;
        all = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
        if (!all) { free(iro); free(icol); return ORACLE_ENOMEM; }
        for (int32_t v = 0; v < n; v++) all[v] = v;
        sources = all;
    }
    for (int64_t i = 0; i < k; i++)
        if (sources[i] < 0 || sources[i] >= n) { free(all); free(iro); free(icol); return ORACLE_EINVAL; }
    if (nthreads < 1) nthreads = 1;
    if (nthreads > k) nthreads = (int)(k > 0 ? k : 1);
    for (int32_t v = 0; v < n; v++) bc[v] = 0.0;
    job_t *jobs = (job_t *)calloc((size_t)nthreads, sizeof(job_t));
    pthread_t *th = (pthread_t *)calloc((size_t)nthreads, sizeof(pthread_t));
    double *priv = (double *)calloc((size_t)nthreads * (size_t)(n > 0 ? n : 1), sizeof(double));
    if (!jobs || !th || !priv) rc = ORACLE_ENOMEM;
    for (int t = 0; rc == ORACLE_OK && t < nthreads; t++) {
        jobs[t].g = &g; jobs[t].sources = sources; jobs[t].variant = variant;
        jobs[t].lo = k * t / nthreads; jobs[t].hi = k * (t + 1) / nthreads;
        jobs[t].bc = priv + (size_t)t * (size_t)n;
        if (nthreads == 1) run_job(&jobs[t]);
        else pthread_create(&th[t], NULL, run_job, &jobs[t]);
    }
    if (rc == ORACLE_OK && nthreads > 1)
        for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    for (int t = 0; rc == ORACLE_OK && t < nthreads; t++) {
        if (jobs[t].rc) { rc = jobs[t].rc; break; }
        for (int32_t v = 0; v < n; v++) bc[v] += jobs[t].bc[v];
    }
    if (rc == ORACLE_OK && !directed)
        for (int32_t v = 0; v < n; v++) bc[v] *= 0.5;
    free(jobs); free(th); free(priv); free(all); free(iro); free(icol);
    return rc;
}

/* BC over a source list (NULL = all n vertices), variant 1 (pull).  bc is
 * overwritten; undirected scores are halved. */
int oracle_bc(int32_t n, const int64_t *ro, const int32_t *col, int directed,
              const int32_t *sources, int64_t k, double *bc, int nthreads)
{
    return oracle_bc_impl(n, ro, col, directed, sources, k, bc, nthreads, 0);
}

/* Same result by textbook push Brandes (variant 2). */
int oracle_bc_push(int32_t n, const int64_t *ro, const int32_t *col, int directed,
                   const int32_t *sources, int64_t k, double *bc, int nthreads)
{
    return oracle_bc_impl(n, ro, col, directed, sources, k, bc, nthreads, 1);
}

/* Per-source export for parity: d (-1 = unreachable), sigma, delta (variant 1),
 * level sizes (level_sizes[L] = |{v : d[v] = L}|, caller provides n+1 ints),
 * *num_levels = maxdepth+1, counters[3] = {n_reached, sum of out-degrees of
 * reached vertices, DAG arcs}. Any output pointer may be NULL. */
int oracle_single_source(int32_t n, const int64_t *ro, const int32_t *col, int directed,
                         int32_t s, int32_t *d, double *sigma, double *delta,
                         int32_t *level_sizes, int32_t *num_levels, int64_t *counters)
{
    ograph g;
    int64_t *iro; int32_t *icol;
    int rc = make_graph(&g, n, ro, col, directed, &iro, &icol);
    if (rc) return rc;
    if (s < 0 || s >= n) { free(iro); free(icol); return ORACLE_EINVAL; }
    ostate st;
    rc = state_alloc(&st, n);
    if (rc == ORACLE_OK) {
        brandes_pull_one(&g, &st, s, NULL);
        if (d) memcpy(d, st.d, sizeof(int32_t) * (size_t)n);
        if (sigma) memcpy(sigma, st.sigma, sizeof(double) * (size_t)n);
        if (delta) memcpy(delta, st.delta, sizeof(double) * (size_t)n);
        if (level_sizes)
            for (int32_t L = 0; L < st.nlevels; L++) level_sizes[L] = st.ends[L + 1] - st.ends[L];
        if (num_levels) *num_levels = st.nlevels;
        if (counters) { counters[0] = st.n_reached; counters[1] = st.arcs_reached; counters[2] = st.dag_arcs; }
    }
    state_free(&st);
    free(iro); free(icol);
    return rc;
}

/* Same export by the push variant (d, sigma, delta only). */
int oracle_single_source_push(int32_t n, const int64_t *ro, const int32_t *col, int directed,
                              int32_t s, int32_t *d, double *sigma, double *delta)
{
    ograph g;
    int64_t *iro; int32_t *icol;
    int rc = make_graph(&g, n, ro, col, directed, &iro, &icol);
    if (rc) return rc;
    if (s < 0 || s >= n) { free(iro); free(icol); return ORACLE_EINVAL; }
    ostate st;
    rc = state_alloc(&st, n);
    int64_t *pf = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int32_t *pred = (int32_t *)malloc(sizeof(int32_t) * (size_t)(ro[n] > 0 ? ro[n] : 1));
    if (!pf || !pred) rc = ORACLE_ENOMEM;
    if (rc == ORACLE_OK) {
        brandes_push_one(&g, &st, pf, pred, s, NULL);
        if (d) memcpy(d, st.d, sizeof(int32_t) * (size_t)n);
        if (sigma) memcpy(sigma, st.sigma, sizeof(double) * (size_t)n);
        if (delta) memcpy(delta, st.delta, sizeof(double) * (size_t)n);
    }
    free(pf); free(pred);
    state_free(&st);
    free(iro); free(icol);
    return rc;
}
