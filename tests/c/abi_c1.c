/* abi_c1.c -- a plain C caller of libbc.so (include/bc.h), no Python, no torch.
 *
 *   abi_c1 <graph.txt> <expected_bc.txt> [tolerance]
 *
 * graph.txt:  "n nnz directed" then n+1 row offsets then nnz column indices
 * expected:   n doubles (BC written by a committed script that calls only oracle/)
 *
 * The bc_options struct is first filled with garbage bytes (0xFF) so that a field
 * bc_default_options forgot to set would reach bc_set_options as garbage (VERDICT r1
 * boundary bug: group_ctas).  Then: create, set options, compute all sources (exact BC,
 * P:368), compare element-wise with max |got - ref| / max(|ref|, 1) <= tol (DESIGN R12),
 * destroy.  Exit 0 = parity, 1 = mismatch, 2 = API error, 3 = bad input. */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include "bc.h"

static int api(int rc, const char *what) {
    if (rc != BC_OK) {
        fprintf(stderr, "%s failed: %d %s\n", what, rc, bc_last_error());
        exit(2);
    }
    return rc;
}

int main(int argc, char **argv) {
    if (argc < 3) {
        fprintf(stderr, "usage: %s graph.txt expected.txt [tol]\n", argv[0]);
        return 3;
    }
    const double tol = argc > 3 ? atof(argv[3]) : 1e-9;
    FILE *f = fopen(argv[1], "r");
    if (!f) return 3;
    long long n, nnz;
    int directed;
    if (fscanf(f, "%lld %lld %d", &n, &nnz, &directed) != 3) return 3;
    int64_t *ro = malloc(sizeof(int64_t) * (size_t)(n + 1));
    int32_t *col = malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    for (long long i = 0; i <= n; ++i)
        if (fscanf(f, "%lld", (long long *)&ro[i]) != 1) return 3;
    for (long long i = 0; i < nnz; ++i)
        if (fscanf(f, "%d", &col[i]) != 1) return 3;
    fclose(f);
    double *want = malloc(sizeof(double) * (size_t)n), *got = malloc(sizeof(double) * (size_t)n);
    f = fopen(argv[2], "r");
    if (!f) return 3;
    for (long long i = 0; i < n; ++i)
        if (fscanf(f, "%lf", &want[i]) != 1) return 3;
    fclose(f);

    bc_graph *g = NULL;
    api(bc_graph_create((int32_t)n, nnz, ro, col, directed, 0, &g), "bc_graph_create");
    bc_options o;
    memset(&o, 0xFF, sizeof(o));  /* garbage: every field must be set by the library */
    bc_default_options(&o);
    api(bc_set_options(g, &o), "bc_set_options");
    bc_options back;
    api(bc_get_options(g, &back), "bc_get_options");
    if (back.group_ctas != 0 || back.strategy != BC_STRATEGY_SAMPLING || back.alpha != 768) {
        fprintf(stderr, "options did not round-trip\n");
        return 1;
    }
    for (long long i = 0; i < n; ++i) got[i] = -12345.0;  /* OVERWRITTEN, not accumulated */
    api(bc_compute(g, NULL, 0, got), "bc_compute");
    bc_stats st;
    api(bc_get_stats(g, &st), "bc_get_stats");
    double err = 0.0;
    for (long long i = 0; i < n; ++i) {
        const double e = fabs(got[i] - want[i]) / fmax(fabs(want[i]), 1.0);
        if (e > err) err = e;
    }
    /* the sum-of-distances self-check from the kernel's own counters */
    double sum = 0.0;
    for (long long i = 0; i < n; ++i) sum += got[i];
    const double h = directed ? 1.0 : 0.5;
    const double inv = h * (double)(st.dist_sum - st.n_reached + st.sources);
    bc_destroy(g);
    bc_destroy(NULL);
    printf("n=%lld sources=%lld max_rel_err=%.3e sum=%.17g invariant=%.17g\n", n,
           (long long)st.sources, err, sum, inv);
    if (st.sources != n) return 1;
    if (fabs(sum - inv) > 1e-9 * fmax(fabs(inv), 1.0)) return 1;
    return err <= tol ? 0 : 1;
}
