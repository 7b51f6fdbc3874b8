// bc_kernels.cuh -- sm_100a device code for per-source Brandes BC.
//
// One CTA owns one source at a time ("coarse-grained" root parallelism, P:118,
// P:198) and loops: Alg. 1 init -> forward levels (Alg. 2) in WE or
// EP mode -> backward levels (Alg. 3) -> BC update (Eq. 3) ->
// reset of only the touched vertices.  Sources are pulled from a global atomic
// counter so the grid is persistent (one CTA per workspace slot).
//
// B200 choices:
//  * sigma is PULLED (sigma[w] = sum of sigma over w's level-(L-1) neighbours)
//    when w itself is expanded, fused with w's discovery scan: one CSR row read
//    serves both, no sigma atomics in WE mode, and rows of degree <= SEQ_MAX_DEG
//    are summed by one thread in CSR order = the oracle's order (bit-exact).
//  * the queue is S itself: level L+1 is appended at S[ends[L+1]...], so Alg. 2's
//    Q_next -> Q_curr copy (l.15-17) disappears (§8(a) a4).
//  * rows of degree > SEQ_MAX_DEG are expanded CTA-cooperatively: block scan of
//    their degrees, arcs dealt round-robin to all threads, owner found by binary
//    search in shared memory, warp-segmented reduction of the partial sums.
//  * backward uses omega[v] = (1 + delta[v]) / sigma[v]: one 8-byte gather per
//    DAG arc, delta[w] = sigma[w] * sum(omega of successors).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace bcdev {

constexpr int NT = 256;             // threads per CTA
constexpr int NWARP = NT / 32;
constexpr int SEQ_MAX_DEG = 32;     // rows up to this degree: one thread, CSR order
constexpr int INF = 0x7F7F7F7F;     // "infinity" distance (memset-able byte pattern)
constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr double TWO53 = 9007199254740992.0;

enum : int { MODE_WE = 0, MODE_EP = 1 };
enum : int { LM_WE = 0, LM_EP = 1, LM_HYBRID = 2, LM_SAMPLED = 3 };

struct DevStats {
    unsigned long long sources, levels, we_levels, ep_levels;
    unsigned long long n_reached, arcs_reached, dag_arcs, arcs_scanned;
    int sigma_inexact;
    int sampling_ep;
    int sampling_median;
    int pad;
};

struct KParams {
    int n;
    int nnz;
    const int *__restrict__ ro;    // out-CSR offsets (int32)
    const int *__restrict__ col;   // out-CSR columns
    const int *__restrict__ src;   // COO source of each out-arc (EP)
    const int *__restrict__ iro;   // in-CSR (directed only)
    const int *__restrict__ icol;
    const int *__restrict__ isrc;
    const int *__restrict__ sources;  // NULL: source = src_base + idx
    long long src_base;
    long long k;                      // sources in this launch
    unsigned long long *work_counter;
    // workspace (slot-major)
    int *d;
    double *sigma;
    double *omega;
    int *S;
    int *ends;
    unsigned char *modes;
    size_t stride_n;     // elements per slot for d/sigma/omega/S
    size_t stride_e;     // elements per slot for ends/modes
    double *bc;
    // strategy
    int launch_mode;
    const int *sampled_flag;  // LM_SAMPLED: 1 = EP run
    int alpha, beta, ep_min_frontier;
    int backward_we;
    int *keys;                // sampling phase: keys[idx] = max depth
    DevStats *stats;
    // debug export (single source), may be NULL
    int *dbg_d;
    double *dbg_sigma;
    double *dbg_delta;
    unsigned char *dbg_modes;
    int dbg_max_levels;
    int *dbg_nlevels;
};

struct Smem {
    long long idx;
    int s_len;
    int warp_tot[NWARP + 1];
    int off[NT];
    int beg[NT];
    double acc[NT];
};

struct Slot {
    int *d;
    double *sigma;
    double *omega;
    int *S;
    int *ends;
    unsigned char *modes;
};

struct Counters {
    unsigned long long arcs_reached = 0, dag = 0, scanned = 0;
    int inexact = 0;
};

// ------------------------------------------------------------------ helpers

__device__ __forceinline__ int block_exclusive_scan(int x, int &total, Smem &sm) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) sm.warp_tot[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        int v = lane < NWARP ? sm.warp_tot[lane] : 0;
        int inc = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(FULL, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane < NWARP) sm.warp_tot[lane] = inc - v;
        if (lane == NWARP - 1) sm.warp_tot[NWARP] = inc;
    }
    __syncthreads();
    total = sm.warp_tot[NWARP];
    return incl - x + sm.warp_tot[wid];
}

__device__ __forceinline__ void discover(int *d, int *S, int *s_len, int u, int L1) {
    if (atomicCAS(&d[u], INF, L1) == INF) {
        int pos = atomicAdd(s_len, 1);
        S[pos] = u;
    }
}

// Segmented (by non-decreasing owner) warp sum; returns true for the tail lane of
// each segment, which then holds the segment total in `val`.
__device__ __forceinline__ bool warp_segmented_sum(int owner, double &val) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        double v2 = __shfl_up_sync(FULL, val, o);
        int o2 = __shfl_up_sync(FULL, owner, o);
        if (lane >= o && o2 == owner) val += v2;
    }
    int nxt = __shfl_down_sync(FULL, owner, 1);
    return owner >= 0 && (lane == 31 || nxt != owner);
}

// Generic "row pass" over a contiguous range of S: every vertex v = S[i] has its
// row [rows[v], rows[v+1]) of `cols` inspected; op(u) returns a double
// contribution.  Returns (for the calling thread) the sum for the vertex it owns in
// the CURRENT tile through `body` -- the pass calls finish(v, acc) once per vertex.
template <class Probe, class Op, class Finish>
__device__ __forceinline__ void row_pass(const int *__restrict__ S, int lo, int hi,
                                         const int *__restrict__ rows,
                                         const int *__restrict__ cols, Smem &sm,
                                         Counters &c, Probe probe, Op op, Finish finish) {
    for (int base = lo; base < hi; base += NT) {
        const int i = base + threadIdx.x;
        int v = -1, beg = 0, deg = 0;
        if (i < hi) {
            v = S[i];
            beg = rows[v];
            deg = rows[v + 1] - beg;
        }
        c.scanned += deg;
        const bool big = deg > SEQ_MAX_DEG;
        double acc = 0.0;
        if (v >= 0 && !big) {
            // one thread, CSR order (same summation order as the oracle)
            int a = beg;
            const int e = beg + deg;
            for (; a + 4 <= e; a += 4) {
                const int u0 = cols[a], u1 = cols[a + 1], u2 = cols[a + 2], u3 = cols[a + 3];
                const int k0 = probe(u0), k1 = probe(u1), k2 = probe(u2), k3 = probe(u3);
                acc += op(u0, k0);
                acc += op(u1, k1);
                acc += op(u2, k2);
                acc += op(u3, k3);
            }
            for (; a < e; ++a) {
                const int u = cols[a];
                acc += op(u, probe(u));
            }
        }
        int total;
        const int off = block_exclusive_scan(big ? deg : 0, total, sm);
        if (total > 0) {  // block-uniform
            sm.off[threadIdx.x] = off;
            sm.beg[threadIdx.x] = beg;
            sm.acc[threadIdx.x] = 0.0;
            __syncthreads();
            for (int jb = 0; jb < total; jb += NT) {
                const int j = jb + threadIdx.x;
                int owner = -1;
                double val = 0.0;
                if (j < total) {
                    int lo2 = 0, hi2 = NT - 1;  // last t with off[t] <= j
                    while (lo2 < hi2) {
                        int mid = (lo2 + hi2 + 1) >> 1;
                        if (sm.off[mid] <= j) lo2 = mid; else hi2 = mid - 1;
                    }
                    owner = lo2;
                    const int u = cols[sm.beg[owner] + (j - sm.off[owner])];
                    val = op(u, probe(u));
                }
                if (warp_segmented_sum(owner, val)) atomicAdd(&sm.acc[owner], val);
            }
            __syncthreads();
            if (big) acc = sm.acc[threadIdx.x];
        }
        if (v >= 0) finish(v, acc, big);
    }
}

__device__ __forceinline__ int next_mode(const KParams &p, int mode, int run_ep, int q_curr,
                                         int q_next) {
    switch (p.launch_mode) {
    case LM_WE: return MODE_WE;
    case LM_EP: return MODE_EP;
    case LM_HYBRID: {  // Alg. 4
        int change = q_next > q_curr ? q_next - q_curr : q_curr - q_next;
        if (change > p.alpha) return q_next > p.beta ? MODE_EP : MODE_WE;
        return mode;
    }
    default:  // LM_SAMPLED: Alg. 5 run mode with the P:301 guard
        return (run_ep && q_next >= p.ep_min_frontier) ? MODE_EP : MODE_WE;
    }
}

// ------------------------------------------------------------------ forward

template <bool DIR>
__device__ void forward_we(const KParams &p, const Slot &sl, int L, int lo, int hi, Smem &sm,
                           Counters &c) {
    int *d = sl.d;
    double *sigma = sl.sigma;
    int *S = sl.S;
    const int L1 = L + 1, Lm1 = L - 1;
    if (!DIR) {
        // fused: discovery of level L+1 and sigma pull for level L in one row scan
        auto probe = [&](int u) -> int { return d[u]; };
        auto op = [&](int u, int du) -> double {
            if (du == Lm1) { c.dag++; return sigma[u]; }
            if (du == INF) discover(d, S, &sm.s_len, u, L1);
            return 0.0;
        };
        auto fin = [&](int v, double acc, bool big) {
            if (L > 0) {
                sigma[v] = acc;
                if (big && acc >= TWO53) c.inexact = 1;
            }
        };
        const unsigned long long before = c.scanned;
        row_pass(S, lo, hi, p.ro, p.col, sm, c, probe, op, fin);
        c.arcs_reached += c.scanned - before;
    } else {
        auto probe = [&](int u) -> int { return d[u]; };
        auto op1 = [&](int u, int du) -> double {
            if (du == INF) discover(d, S, &sm.s_len, u, L1);
            return 0.0;
        };
        auto fin1 = [&](int, double, bool) {};
        const unsigned long long before = c.scanned;
        row_pass(S, lo, hi, p.ro, p.col, sm, c, probe, op1, fin1);
        c.arcs_reached += c.scanned - before;
        if (L > 0) {
            auto op2 = [&](int u, int du) -> double {
                if (du == Lm1) { c.dag++; return sigma[u]; }
                return 0.0;
            };
            auto fin2 = [&](int v, double acc, bool big) {
                sigma[v] = acc;
                if (big && acc >= TWO53) c.inexact = 1;
            };
            row_pass(S, lo, hi, p.iro, p.icol, sm, c, probe, op2, fin2);
        }
    }
}

template <bool DIR>
__device__ void forward_ep(const KParams &p, const Slot &sl, int L, int lo, int hi, Smem &sm,
                           Counters &c) {
    int *d = sl.d;
    double *sigma = sl.sigma;
    int *S = sl.S;
    const int L1 = L + 1, Lm1 = L - 1;
    // Sum of degrees of the frontier (for the TEPS byte model only).
    for (int i = lo + threadIdx.x; i < hi; i += NT) {
        int v = S[i];
        c.arcs_reached += (unsigned long long)(p.ro[v + 1] - p.ro[v]);
    }
    // Thread per arc over ALL arcs (Jia et al. EP).
    for (int a = threadIdx.x; a < p.nnz; a += NT) {
        int x = p.src[a];
        if (d[x] != L) continue;
        int y = p.col[a];
        int dy = d[y];
        if (dy == INF) {
            discover(d, S, &sm.s_len, y, L1);
        } else if (!DIR && dy == Lm1) {
            double s = sigma[y];
            double old = atomicAdd(&sigma[x], s);
            c.dag++;
            if (old + s >= TWO53) c.inexact = 1;
        }
    }
    c.scanned += (unsigned long long)p.nnz;
    if (DIR && L > 0) {
        for (int a = threadIdx.x; a < p.nnz; a += NT) {
            int x = p.isrc[a];
            if (d[x] != L) continue;
            int y = p.icol[a];
            if (d[y] == Lm1) {
                double s = sigma[y];
                double old = atomicAdd(&sigma[x], s);
                c.dag++;
                if (old + s >= TWO53) c.inexact = 1;
            }
        }
        c.scanned += (unsigned long long)p.nnz;
    }
}

// ------------------------------------------------------------------ backward

__device__ __forceinline__ void finish_dependency(const KParams &p, const Slot &sl, int w,
                                                  double acc) {
    const double sw = sl.sigma[w];
    const double delta = sw * acc;                 // delta[w] = sum sw/sigma[v] (1+delta[v])
    sl.omega[w] = (1.0 + delta) / sw;
    if (delta != 0.0) atomicAdd(&p.bc[w], delta);  // Eq. 3
    if (p.dbg_delta) p.dbg_delta[w] = delta;
}

__device__ void backward_we(const KParams &p, const Slot &sl, int L, int lo, int hi, Smem &sm,
                            Counters &c) {
    const int *d = sl.d;
    const double *omega = sl.omega;
    const int L1 = L + 1;
    auto probe = [&](int v) -> int { return d[v]; };
    auto op = [&](int v, int dv) -> double { return dv == L1 ? omega[v] : 0.0; };
    auto fin = [&](int w, double acc, bool) { finish_dependency(p, sl, w, acc); };
    row_pass(sl.S, lo, hi, p.ro, p.col, sm, c, probe, op, fin);
}

__device__ void backward_ep(const KParams &p, const Slot &sl, int L, int lo, int hi, Smem &sm,
                            Counters &c) {
    const int *d = sl.d;
    double *omega = sl.omega;
    const int L1 = L + 1;
    for (int a = threadIdx.x; a < p.nnz; a += NT) {
        int x = p.src[a];
        if (d[x] != L) continue;
        int y = p.col[a];
        if (d[y] == L1) atomicAdd(&omega[x], omega[y]);  // omega[x] == 0 until finished
    }
    c.scanned += (unsigned long long)p.nnz;
    __syncthreads();
    for (int i = lo + threadIdx.x; i < hi; i += NT) {
        int w = sl.S[i];
        finish_dependency(p, sl, w, omega[w]);
    }
}

// ------------------------------------------------------------------ kernel

template <bool DIR>
__global__ void __launch_bounds__(NT) bc_kernel(KParams p) {
    __shared__ Smem sm;
    const size_t slot = blockIdx.x;
    Slot sl;
    sl.d = p.d + slot * p.stride_n;
    sl.sigma = p.sigma + slot * p.stride_n;
    sl.omega = p.omega + slot * p.stride_n;
    sl.S = p.S + slot * p.stride_n;
    sl.ends = p.ends + slot * p.stride_e;
    sl.modes = p.modes + slot * p.stride_e;

    Counters c;
    unsigned long long n_src = 0, n_lv = 0, n_we = 0, n_ep = 0, n_reached = 0;
    const int run_ep = (p.launch_mode == LM_SAMPLED && p.sampled_flag) ? *p.sampled_flag : 0;

    for (;;) {
        if (threadIdx.x == 0) sm.idx = (long long)atomicAdd(p.work_counter, 1ULL);
        __syncthreads();
        const long long idx = sm.idx;
        if (idx >= p.k) break;
        const int s = p.sources ? p.sources[p.src_base + idx] : (int)(p.src_base + idx);
        // Alg. 1; all other entries are already d=INF, sigma=omega=0.
        if (threadIdx.x == 0) {
            sl.d[s] = 0;
            sl.sigma[s] = 1.0;
            sl.S[0] = s;
            sl.ends[0] = 0;
            sl.ends[1] = 1;
            sm.s_len = 1;
        }
        __syncthreads();

        int L = 0, lo = 0, hi = 1;
        int mode = next_mode(p, MODE_WE, run_ep, 0, 1);  // level 0: frontier = {s}
        if (p.launch_mode == LM_HYBRID) mode = MODE_WE;  // Alg. 4 starts WE
        for (;;) {
            if (mode == MODE_WE) forward_we<DIR>(p, sl, L, lo, hi, sm, c);
            else forward_ep<DIR>(p, sl, L, lo, hi, sm, c);
            __syncthreads();
            const int nhi = sm.s_len;
            if (threadIdx.x == 0) {
                sl.modes[L] = (unsigned char)mode;
                sl.ends[L + 2] = nhi;
            }
            if (mode == MODE_WE) n_we++; else n_ep++;
            n_lv++;
            __syncthreads();  // s_len is appended to again by the next level
            if (nhi == hi) break;  // Q_next_len == 0 (Alg. 2 l.11)
            mode = next_mode(p, mode, run_ep, hi - lo, nhi - hi);
            lo = hi;
            hi = nhi;
            ++L;
        }
        const int maxdepth = L;
        const int S_len = hi;
        if (p.keys && threadIdx.x == 0) p.keys[idx] = maxdepth;

        // Stage 2 (Alg. 3).  Deepest level: delta = 0, omega = 1/sigma.
        if (maxdepth >= 1)
            for (int i = lo + threadIdx.x; i < hi; i += NT) {
                int v = sl.S[i];
                sl.omega[v] = 1.0 / sl.sigma[v];
            }
        __syncthreads();
        for (int Lb = maxdepth - 1; Lb >= 1; --Lb) {
            const int blo = sl.ends[Lb], bhi = sl.ends[Lb + 1];
            const int bmode = p.backward_we ? MODE_WE : (int)sl.modes[Lb];
            if (bmode == MODE_WE) backward_we(p, sl, Lb, blo, bhi, sm, c);
            else backward_ep(p, sl, Lb, blo, bhi, sm, c);
            __syncthreads();
        }

        // Debug export, then reset only the touched vertices.
        for (int i = threadIdx.x; i < S_len; i += NT) {
            int v = sl.S[i];
            if (p.dbg_d) {
                p.dbg_d[v] = sl.d[v];
                p.dbg_sigma[v] = sl.sigma[v];
            }
            sl.d[v] = INF;
            sl.sigma[v] = 0.0;
            sl.omega[v] = 0.0;
        }
        if (p.dbg_modes && threadIdx.x == 0) {
            for (int l = 0; l <= maxdepth && l < p.dbg_max_levels; ++l) p.dbg_modes[l] = sl.modes[l];
            *p.dbg_nlevels = maxdepth + 1;
        }
        n_src++;
        n_reached += (unsigned long long)S_len;
        __syncthreads();
    }

    // Statistics: per-thread counters -> warp sums -> global atomics.
    unsigned long long ar = c.arcs_reached, dg = c.dag, sc = c.scanned;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        ar += __shfl_down_sync(FULL, ar, o);
        dg += __shfl_down_sync(FULL, dg, o);
        sc += __shfl_down_sync(FULL, sc, o);
    }
    int inex = __any_sync(FULL, c.inexact);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&p.stats->dag_arcs, dg);
        atomicAdd(&p.stats->arcs_scanned, sc);
        atomicAdd(&p.stats->arcs_reached, ar);
        if (inex) atomicOr(&p.stats->sigma_inexact, 1);
    }
    if (threadIdx.x == 0) {
        atomicAdd(&p.stats->sources, n_src);
        atomicAdd(&p.stats->levels, n_lv);
        atomicAdd(&p.stats->we_levels, n_we);
        atomicAdd(&p.stats->ep_levels, n_ep);
        atomicAdd(&p.stats->n_reached, n_reached);
    }
}

// Alg. 5 decision: sort keys ascending, median = keys[nk/2],
// EP iff median < gamma*log2(n).  One CTA, bitonic sort in shared memory.
__global__ void __launch_bounds__(1024) sampling_decide_kernel(const int *keys, int nk,
                                                               double thresh, int *flag,
                                                               DevStats *st) {
    extern __shared__ int sk[];
    int P = 1;
    while (P < nk) P <<= 1;
    for (int i = threadIdx.x; i < P; i += blockDim.x) sk[i] = i < nk ? keys[i] : 0x7FFFFFFF;
    __syncthreads();
    for (int size = 2; size <= P; size <<= 1) {
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int i = threadIdx.x; i < P; i += blockDim.x) {
                int j = i ^ stride;
                if (j > i) {
                    bool up = (i & size) == 0;
                    int a = sk[i], b = sk[j];
                    if ((a > b) == up) { sk[i] = b; sk[j] = a; }
                }
            }
            __syncthreads();
        }
    }
    if (threadIdx.x == 0) {
        int med = sk[nk / 2];
        int ep = (double)med < thresh ? 1 : 0;
        *flag = ep;
        st->sampling_ep = ep;
        st->sampling_median = med;
    }
}

__global__ void build_src_kernel(const int *__restrict__ ro, int n, int nnz, int *__restrict__ src) {
    for (long long a = blockIdx.x * (long long)blockDim.x + threadIdx.x; a < nnz;
         a += (long long)gridDim.x * blockDim.x) {
        int lo = 0, hi = n - 1;  // last v with ro[v] <= a
        while (lo < hi) {
            int mid = (lo + hi + 1) >> 1;
            if (ro[mid] <= a) lo = mid; else hi = mid - 1;
        }
        src[a] = lo;
    }
}

__global__ void scale_kernel(double *bc, int n, double f) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        bc[i] *= f;
}

}  // namespace bcdev
