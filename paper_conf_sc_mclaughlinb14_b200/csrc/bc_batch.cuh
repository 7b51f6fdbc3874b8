// bc_batch.cuh -- multi-source batched engine: 64 sources per batch, level-synchronous
// over the whole GPU (cooperative persistent kernel, one grid barrier per level).
//
// The same per-source Brandes computation as bc_kernel (Alg. 1-3; d, sigma,
// delta of every source are unchanged), scheduled differently: source b of a batch owns
// bit b of a 64-bit mask per vertex and level, F_L[v] = { b : d_b(v) = L }.  A vertex v
// is expanded once per level L at which ANY source of the batch has it (the union of the
// 64 frontiers, Q_L), so each CSR row read serves every source that has v at that level
// (the Kepler design expanded it once per source).  Warp lanes map to
// sources only inside rows long enough to fill a window (hubs); elsewhere lanes = pairs.
//
//   forward level L, u in Q_L, f = F_L[u], for x in N(u) (CSR order):
//     sigma pull (Alg. 2 l.7-8 as a pull, R18): b in f & F_{L-1}[x] -> acc_b += sigma_b(x)
//     discovery  (Alg. 2 l.5-6): b in f & ~(F_{L-1} | F_L | F_{L+1})[x] -> F_{L+1}[x] |= b
//       (undirected: every neighbour of a level-L vertex is on L-1, L or L+1, so these
//        three masks are the whole "visited" test), x enqueued into Q_{L+1} once
//   backward level L (Alg. 3, omega trick): b in f & F_{L+1}[x] -> acc_b += omega_b(x),
//     delta_b(u) = sigma_b(u) * acc_b, omega_b(u) = (1 + delta_b(u)) / sigma_b(u),
//     bc[u] += sum_b delta_b(u)  (Eq. 3)
//
// Arc-parallel accumulation: each level's rows form one arc space [0, A_L) (Q entries
// carry their arc offset, assigned with the entry by one packed 64-bit atomic at enqueue
// time), cut into equal contiguous ranges, one per warp, lanes = arcs whatever the row
// boundaries.  Every (arc, source) pair of the DAG is one lane-parallel gather plus one
// fire-and-forget fp64 reduction into the row's accumulator:
//   forward  sigma_b(u) += sigma_b(x)                 (sigma_b(u) zeroed when (u, b) is discovered)
//   backward acc_b(u)   += 1/sigma_b(x) + acc_b(x)    (= omega_b(x) = (1 + delta_b(x)) / sigma_b(x))
// and delta_b(u) = sigma_b(u) * acc_b(u) is added to bc[u] one level later.  Sums of
// integers below 2^53 are exact in any order, so sigma stays bit-exact there.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace bcdev {
struct DevStats;
}

namespace bcbatch {

constexpr int BW = 64;        // sources per batch (bits of a mask word)
constexpr int MAX_LCAP = 254; // level slabs per vertex = Lcap + 2 <= 256

struct BParams {
    int n;
    const int *__restrict__ ro;   // int32 CSR (internal ids)
    const int *__restrict__ col;
    const int *__restrict__ src;  // COO source of each arc (multi-source EP levels)
    int nnz;
    int ep_guard;                 // a forward level whose union frontier has >= ep_guard vertices
                                  // is expanded edge-parallel (one scan of all arcs for the 64
                                  // sources; 0 = never); only when *ep_flag == 1 if ep_flag is set
    const int *ep_flag;           // Alg. 5 decision (EP run) or nullptr
    const int *sources;           // caller ids; NULL: source = src_base + idx
    const int *perm;              // caller id -> internal id (NULL: identity)
    long long src_base, k;        // this launch's sources: [src_base, src_base + k) of the list
    int Lcap;                     // levels 0..Lcap can be expanded; deeper => overflow
    int LS;                       // Lcap + 2: mask words per vertex (vertex-major F)
    int min_range;                // minimum arcs per warp range
    unsigned long long *F;        // F[v * LS + L] (zero between batches)
    size_t sn;                    // n rounded up to 32 (allocation)
    double *sig;                  // sig[v * 64 + b]: sigma_b(v)
    double *dacc;                 // dacc[v * 64 + b]: sum of omega_b over v's successors
    int *Q;                       // union frontiers, level after level; capacity qcap
    int *qoff;                    // arc offset of each Q entry within its level
    long long qcap;
    unsigned long long *qctr;     // [LS] per level, packed (entries << 40 | arcs)
    unsigned long long *lvor;     // [LS] OR of the level's masks (levels statistic)
    double *bc;                   // BC in internal ids (accumulated with atomics)
    bcdev::DevStats *stats;
    const int *sampled_flag;      // non-NULL: run only if *sampled_flag == 1 (Alg. 5 EP run)
    int *ovf_src;                 // sources of batches that exceeded Lcap (caller ids)
    long long *ovf_n;
    // per-level trace of batch 0 (tools/batch_trace.py), may be NULL:
    // trace[((dir * LS) + L) * 4 + {0 wall cycles (CTA 0), 1 max warp busy cycles,
    //                               2 sum warp busy cycles, 3 arcs}], dir 0 fwd / 1 bwd
    long long *trace;
    // debug export of one launch (<= 64 sources), internal ids, [64][n]; may be NULL
    int *dbg_d;
    double *dbg_sigma, *dbg_delta;
};

// Kernel symbol for a block size (128 or 256 threads); launched cooperatively.
const void *batch_kernel_fn(int nt);

}  // namespace bcbatch
