/*
 * bc.h -- C ABI of libbc.so: betweenness centrality on unweighted graphs on one
 * NVIDIA B200 (sm_100a), after McLaughlin & Bader, "Scalable and High
 * Performance Betweenness Centrality on the GPU", SC'14.  Citations "P:<line>"
 * refer to the paper text; "§8(x)" to SURVEY.md.
 *
 * What is computed (Eq. 1, Eq. 2, Eq. 3):
 *     BC(v) = h * sum_{s in sources, s != v} delta_s(v),   h = 1/2 undirected, 1 directed
 * by Brandes' two stages per source: a forward BFS computing distances d and
 * shortest-path counts sigma (Alg. 2), then a backward sweep over the
 * recorded level order accumulating dependencies delta (Alg. 3).  Each
 * BFS level is expanded work-efficiently (WE, queue-based) or
 * edge-parallel (EP, thread per arc), as chosen by the paper's
 * hybrid selector (Alg. 4) or sampling selector (Alg. 5).
 * No (n-1)(n-2) normalisation and no n/k extrapolation for subsets.
 *
 * Numerics: d is exact; sigma, delta and BC are IEEE fp64.  sigma is an exact
 * integer whenever it is below 2^53; above that it is the fp64 sum of its
 * predecessors' sigma (bc_stats.sigma_inexact reports when an order-dependent
 * fp64 sum reached 2^53).  BC is summed over sources with fp64 atomics, so the
 * last bits may vary run to run (|rel err| << 1e-9).
 *
 * Errors: every int-returning call returns BC_OK (0) or a negative BC_E* code;
 * no exception or abort crosses the ABI.  bc_last_error() returns a
 * human-readable message for the calling host thread's last failure.  On error,
 * output buffers have unspecified contents.
 *
 * Threading: a bc_graph is NOT thread-safe; use one handle per host thread.
 * Successive calls on one handle are ordered even across different streams.
 */
#ifndef BC_B200_BC_H
#define BC_B200_BC_H

#include <stdint.h>

#if defined(__GNUC__)
#define BC_API __attribute__((visibility("default")))
#else
#define BC_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

enum {
    BC_OK = 0,
    BC_EINVAL = -1,    /* invalid argument (bad CSR, out-of-range source, NULL pointer) */
    BC_ENOMEM = -2,    /* host or device allocation failed */
    BC_ECUDA = -3,     /* CUDA runtime / launch error (message in bc_last_error) */
    BC_EINTERNAL = -4  /* internal invariant violated */
};

/* Frontier-expansion strategy. */
enum {
    BC_STRATEGY_WE = 0,       /* work-efficient on every level (Alg. 2/3 only, §IV.A)        */
    BC_STRATEGY_EP = 1,       /* edge-parallel on every level (Jia et al. [23])         */
    BC_STRATEGY_HYBRID = 2,   /* Alg. 4: reconsider when |Q_next_len - Q_curr_len| > alpha    */
    BC_STRATEGY_SAMPLING = 3  /* Alg. 5: median max-depth of n_samps WE roots < gamma*log2(n) */
};

/* Execution engine (how sources are scheduled; results are the same up to fp64 rounding). */
enum {
    BC_ENGINE_AUTO = 0,       /* undirected graphs with n >= 2^21 whose launches run every
                                 level work-efficiently (WE strategy, or SAMPLING with an EP
                                 guard above n) use the GROUP engine; a SAMPLING run whose
                                 Alg. 5 decision is EP on such a graph with a skewed degree
                                 distribution (internally relabelled) runs its main phase on
                                 the BATCHED engine; everything else (all graphs below 2^21,
                                 directed graphs) runs on the PER-SOURCE engine.  Measured
                                 choices, DESIGN.md §5d                                      */
    BC_ENGINE_PER_SOURCE = 1, /* one CTA per source (bc_kernel), every level WE or EP as the
                                 strategy chooses                                            */
    BC_ENGINE_BATCHED = 2,    /* undirected graphs: 64 sources per batch, level-synchronous
                                 over the whole GPU, one 64-bit source mask per vertex and
                                 level; every union-frontier row is read once per level for
                                 all 64 sources (work-efficient, queue-driven expansion)    */
    BC_ENGINE_GROUP = 3       /* undirected graphs, work-efficient levels only (WE strategy,
                                 or SAMPLING with an EP guard above n): the CTAs are split
                                 into groups, each group traverses ONE source at a time with
                                 a group barrier per level, so only a few sources' state is
                                 live (L2-resident on large graphs); other launches fall back
                                 to the per-source engine                                   */
};

typedef struct bc_graph bc_graph; /* opaque; owns device copies of the graph and workspace */

typedef struct bc_options {
    int32_t strategy;        /* BC_STRATEGY_*; default BC_STRATEGY_SAMPLING            */
    int32_t alpha;           /* Alg. 4 frontier-change threshold, default 768          */
    int32_t beta;            /* Alg. 4 EP frontier threshold (strict >), default 512   */
    double gamma;            /* Alg. 5 depth factor, default 4                         */
    int32_t n_samps;         /* Alg. 5 sample count, default 512, 1..8192              */
    int32_t ep_min_frontier; /* Alg. 5 guard: EP only if frontier >= this, default 512 */
    int32_t inflight;        /* sources processed concurrently (one CTA each); 0 = auto        */
    int32_t backward_we;     /* 1: backward always WE (Alg. 3); 0 (default): backward level L
                                uses the mode forward level L used (R8)              */
    /* Implementation knobs (do not change results beyond fp64 rounding order): */
    int32_t block_threads;   /* threads per CTA: 0 = auto (128 below 2^17 vertices, else 512;
                                1024 for degree-relabelled graphs with codes in shared memory),
                                128, 256, 512 or 1024                                          */
    int32_t seq_max_deg;     /* rows up to this degree are summed by one thread in CSR order;
                                longer rows cooperatively.  0 = auto (128)                     */
    int32_t level_store;     /* 0 = auto, 1 = exact int32 d in HBM, 2 = 2-bit codes in shared
                                memory (undirected graphs whose codes fit; else EINVAL),
                                3 = 2-bit codes in HBM/L2 (undirected graphs)                  */
    int32_t warp_max_deg;    /* rows up to this degree are expanded by one warp, longer rows
                                by the whole CTA.  0 = auto (8192)                             */
    int32_t l2_persist;      /* 0 = auto, 1 = on, -1 = off: persisting-L2 access-policy window
                                over the CSR arrays during traversal launches (auto: on, except
                                for degree-relabelled graphs with level codes in shared memory) */
    int32_t sort_frontier;   /* 0 = auto, 1 = on, -1 = off: rebuild large BFS levels in vertex
                                order from a per-level bitmap (locality of rows, codes, sigma)  */
    /* Output post-processing (default 0 = exact BC as defined above): */
    int32_t extrapolate;     /* 1: multiply by n/k (k = number of sources): the k-source
                                estimator of total BC ("trivially adjusted for approximation",
                                P:315, refs [3],[9])                                            */
    int32_t normalize;       /* 1: divide by (n-1)(n-2), the normalisation of P:74             */
    int32_t succ_bits;       /* 0 = auto (on with level_store 3), 1 = on, -1 = off: one
                                bit per arc (per source in flight) marks DAG successors
                                during the forward scan (Jia et al.'s O(m) boolean array,
                                P:129); the backward then reads only successor arcs          */
    int32_t engine;          /* BC_ENGINE_*, default BC_ENGINE_AUTO                            */
    int32_t batch_levels;    /* batched engine: BFS levels a batch may have (0 = auto 64, max
                                254); sources of a deeper batch are rerun per source         */
    int32_t hub_chunk;       /* batched engine: minimum arcs per warp range when a BFS level's
                                arcs are cut into equal warp ranges (rows of any length are
                                split across ranges); 0 = auto 64                            */
    int32_t group_ctas;      /* group engine: CTAs per group; 0 = auto (12 CTAs per group on
                                degree-relabelled graphs, else 4 groups; B200 sweeps,
                                DESIGN.md §5d).  bc_default_options sets every field, this
                                one included                                                  */
} bc_options;

typedef struct bc_stats {
    int64_t sources;          /* sources processed by the last compute call                   */
    int64_t levels;           /* forward BFS levels expanded (sum over sources)               */
    int64_t we_levels;        /* ... of which work-efficient                                  */
    int64_t ep_levels;        /* ... of which edge-parallel                                   */
    int64_t n_reached;        /* sum over sources of reached vertices (incl. the source)      */
    int64_t arcs_reached;     /* sum over sources of out-degrees of reached vertices          */
    int64_t dag_arcs;         /* sum over sources of shortest-path DAG arcs (d[w] = d[u] + 1) */
    int64_t arcs_scanned;     /* arcs actually inspected (forward + backward, WE + EP)        */
    int32_t sampling_ep;      /* Alg. 5 decision of the last call: 1 EP, 0 WE, -1 not run     */
    int32_t sampling_median;  /* Alg. 5 median max-depth key, -1 if not run                   */
    int32_t sigma_inexact;    /* 1 if an order-dependent fp64 sigma sum reached 2^53          */
    int32_t inflight;         /* CTAs (sources in flight) used                                */
    int32_t kernel_launches;  /* kernels libbc launched in the last compute call              */
    int32_t bc_kernel_launches; /* ... of which the main traversal kernel (bc_kernel)         */
    double kernel_ms;         /* summed CUDA-event time of the bc_kernel launches             */
    int64_t phase_cycles[4];  /* SM cycles summed over CTAs in forward WE, forward EP,
                                 backward WE, backward EP levels (device trace)               */
    int64_t batches;          /* batches of 64 sources run by the batched engine (0: not run) */
    int64_t batch_overflows;  /* ... of which exceeded batch_levels and were rerun per source */
    int32_t engines;          /* engines the last compute call launched: bit 0 per-source
                                 (bc_kernel), bit 1 batched, bit 2 group (group_kernel)      */
    int32_t pad_;
    int64_t dist_sum;         /* sum over sources s of sum_t d(s,t) over the reached t: with
                                 n_reached and sources it gives the self-check
                                 sum_v BC(v) = h (dist_sum - n_reached + sources) */
    int64_t handovers;        /* Alg. 4 / Alg. 5 runs on the fast work-efficient kernel: sources
                                 whose selector picked an EP level and were therefore re-run
                                 from scratch by the EP-capable kernel (0 if none)             */
    int64_t group_wait_cycles; /* group engine: SM cycles its CTAs spent waiting at the per-level
                                 group barriers after finishing their own share (summed over
                                 CTAs; load-imbalance + barrier latency), 0 on other engines  */
    int32_t group_mode;       /* group engine level passes of the last call: 0 generic row_pass,
                                 1 fast path, 2 thin rows (bc_thin.cuh); -1 not run           */
    int32_t pad2_;
} bc_stats;

/* Copy a CSR graph to `device` and allocate the per-source workspace.
 *   n            vertices, 0 <= n < 2^31 - 2
 *   nnz          arcs; undirected graphs must store both arcs of every edge (P:145 CSR,
 *                SURVEY §8(b)); nnz < 2^31
 *   row_offsets  HOST int64[n+1], row_offsets[0] = 0, row_offsets[n] = nnz, non-decreasing
 *   col_indices  HOST int32[nnz], 0 <= c < n; self-loops are harmless, parallel arcs count
 *                as distinct paths
 *   directed     0 undirected (scores halved), 1 directed
 *   device       CUDA device ordinal
 *   out          receives the handle (NULL on error)
 * The inputs are copied; the caller keeps ownership of its arrays. */
BC_API int bc_graph_create(int32_t n, int64_t nnz, const int64_t *row_offsets,
                    const int32_t *col_indices, int directed, int device, bc_graph **out);

/* BC over a source list, host in / host out (synchronous).
 *   sources      HOST int32[num_sources] (duplicates count with multiplicity), or NULL for
 *                all n vertices = exact BC
 *   num_sources  ignored if sources == NULL; 0 => bc all zero
 *   bc           HOST double[n], OVERWRITTEN with the (halved if undirected) scores
 * Out-of-range source => BC_EINVAL. */
BC_API int bc_compute(bc_graph *g, const int32_t *sources, int64_t num_sources, double *bc);

/* Same, device in / device out, asynchronous on `cuda_stream` (a cudaStream_t; NULL =
 * legacy default stream).  d_sources is DEVICE int32[k] or NULL (all n vertices); d_bc is
 * DEVICE double[n], OVERWRITTEN with the (halved if undirected) scores of these sources.
 * k = 0 with a non-NULL d_sources (never read) => d_bc all zero; NULL always means all n
 * vertices, whatever k says (an empty device tensor must be passed as a non-NULL pointer:
 * the Python binding does so).  Sources are NOT range-checked on the device (caller's
 * responsibility).  Summing the outputs of disjoint source lists gives the BC of their
 * union (multi-GPU) -- unless `extrapolate` is set, which scales each call by its
 * own n/k (apply the estimator once, after the sum, instead: distributed.bc_distributed). */
BC_API int bc_compute_device(bc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc,
                      void *cuda_stream);

/* Debug/parity export for one source s under the current strategy (SAMPLING uses the
 * decision of the last compute call, WE if none).  Host outputs, each may be NULL:
 *   d            int32[n], BFS distance, -1 = unreachable
 *   sigma        double[n], shortest-path counts (0 if unreachable)
 *   delta        double[n], dependency delta_s(v) (0 for s, unreachable and deepest level)
 *   level_modes  uint8[max_levels], mode used to expand forward level L (0 WE, 1 EP)
 *   num_levels   receives maxdepth + 1 */
BC_API int bc_single_source(bc_graph *g, int32_t s, int32_t *d, double *sigma, double *delta,
                     uint8_t *level_modes, int32_t max_levels, int32_t *num_levels);

/* Per-level trace of one source (the paper's Table I / Fig. 3 study,
 * P:231-263), computed exactly like bc_single_source with one CTA:
 *   level_sizes  int32[max_levels]  vertex frontier |{v : d(s,v) = L}| per level L
 *   fwd_cycles   int64[max_levels]  SM cycles spent on forward level L (incl. bookkeeping)
 *   bwd_cycles   int64[max_levels]  SM cycles spent on backward level L (0 for L = 0 and the
 *                                   deepest level, which Alg. 3 does not process)
 *   num_levels   receives maxdepth + 1 (arrays hold min(max_levels, num_levels) entries) */
BC_API int bc_trace_source(bc_graph *g, int32_t s, int32_t *level_sizes, int64_t *fwd_cycles,
                           int64_t *bwd_cycles, int32_t max_levels, int32_t *num_levels);

/* Debug/parity export of the batched engine for one batch of 1..64 sources (undirected
 * graphs): runs exactly the kernel bc_compute uses in batched mode, with per-source
 * outputs.  Host arrays, row b = sources[b], each may be NULL:
 *   d      int32[k][n]   BFS distance from sources[b], -1 = unreachable
 *   sigma  double[k][n]  shortest-path counts (0 if unreachable)
 *   delta  double[k][n]  dependencies (0 for the source, unreachable and deepest vertices)
 * BC_EINVAL for a directed graph, k outside 1..64, an out-of-range source, or a batch
 * deeper than batch_levels. */
BC_API int bc_batch_sources(bc_graph *g, const int32_t *sources, int32_t k, int32_t *d,
                            double *sigma, double *delta);

BC_API void bc_default_options(bc_options *o);
BC_API int bc_set_options(bc_graph *g, const bc_options *o); /* validates; may reallocate workspace */
BC_API int bc_get_options(const bc_graph *g, bc_options *o);
BC_API int bc_get_stats(bc_graph *g, bc_stats *st);          /* of the last compute call (syncs)   */

/* Release device memory; NULL-safe. */
BC_API void bc_destroy(bc_graph *g);

/* Message for the calling thread's last error ("" if none). Never NULL. */
BC_API const char *bc_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* BC_B200_BC_H */
