// bc_batch.cu -- the multi-source batched engine (design in bc_batch.cuh).
//
// One cooperative persistent kernel; all CTAs work on one batch of 64 sources at a time
// and meet at a grid barrier after every level.  Inside a level every warp owns an equal
// contiguous range of the level's arc space (merge-path style), so rows of any degree --
// hubs included -- are spread evenly and no warp is a long pole.
#define BC_INSTANCE_TU
#include "bc_kernels.cuh"
#include "bc_batch.cuh"

#include <cooperative_groups.h>

namespace cg = cooperative_groups;

namespace bcbatch {

using bcdev::DevStats;
using bcdev::FULL;
using bcdev::TWO53;

constexpr unsigned long long CNT_ONE = 1ull << 40;  // packed level counter: entries << 40 | arcs
constexpr unsigned long long ARC_MASK = CNT_ONE - 1;
constexpr int BIG = 0x7FFFFFFF;

// sigma / acc layout: vertex-major, entry (b, v) at v * 64 + b (the pairs of one vertex
// share sectors: measured 2x faster on c4 than source-major b * sn + v)
__device__ __forceinline__ size_t sidx(const BParams &, int b, int v) { return (size_t)v * BW + (size_t)b; }

struct Cnt {  // per-lane counters of one batch (32-bit: a batch is ~10^8 events per warp at most)
    unsigned reached = 0, ar = 0, dag = 0, sc = 0;
    unsigned long long dsum = 0;  // sum of d_b(u) over the (u, b) pairs this lane counted
    int inexact = 0;
};

__device__ __forceinline__ unsigned long long shfl64(unsigned long long v, int src) {
    return __shfl_sync(FULL, v, src);
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

// Rows r0 .. r0+31 of the current level, lane j holding row r0 + j.
struct Rows {
    int r0;
    int u;                 // vertex
    unsigned long long f;  // its source mask at this level
    int cbeg;              // CSR position of level arc a of this row = a + cbeg
    int start, nxt;        // the row's arcs [start, nxt) in the level's arc space
};

__device__ __forceinline__ void load_rows(const BParams &p, Rows &R, int r0, int qlo, int qn, int A, int L) {
    const int r = r0 + (threadIdx.x & 31);
    R.r0 = r0;
    if (r < qn) {
        R.u = __ldcg(&p.Q[qlo + r]);
        R.start = __ldcg(&p.qoff[qlo + r]);
        R.nxt = r + 1 < qn ? __ldcg(&p.qoff[qlo + r + 1]) : A;
        R.f = __ldcg(&p.F[(size_t)R.u * p.LS + L]);
        R.cbeg = __ldg(&p.ro[R.u]) - R.start;
    } else {
        R.u = 0;
        R.start = R.nxt = BIG;
        R.f = 0ull;
        R.cbeg = 0;
    }
}

// Largest r in [0, qn) with qoff[qlo + r] <= a (32-ary search by the whole warp).
__device__ __forceinline__ int find_row(const BParams &p, int qlo, int qn, int a) {
    const int lane = threadIdx.x & 31;
    int lo = 0, hi = qn;
    while (hi - lo > 32) {
        const int step = (hi - lo + 31) >> 5;
        const int q = lo + lane * step;
        const int v = q < hi ? __ldcg(&p.qoff[qlo + q]) : BIG;
        const int c = __popc(__ballot_sync(FULL, v <= a));
        lo += (c - 1) * step;
        hi = min(hi, lo + step);
    }
    const int q = lo + lane;
    const int v = q < hi ? __ldcg(&p.qoff[qlo + q]) : BIG;
    return lo + __popc(__ballot_sync(FULL, v <= a)) - 1;
}

struct Level {
    int L, qlo, qn, A, qlo_next;
    int per;  // arcs per warp range
};

// Window inside one long row (lanes = sources): the row's pairs are dense (a hub at its
// usual level), so each arc's gathers are two coalesced warp loads, summed in arc order
// in registers and reduced once per window -- per-pair reductions would all hit the same
// 64 accumulators.  Four arcs' gathers are issued before they are added.
template <bool FWD>
__device__ __forceinline__ void gather_row_window(const BParams &p, int x, unsigned long long m, int u) {
    constexpr int U = FWD ? 8 : 4;  // arcs per round: 2U (fwd) / 4U (bwd) loads in flight per lane
    const int lane = threadIdx.x & 31;
    double acc0 = 0.0, acc1 = 0.0;
    unsigned sel = __ballot_sync(FULL, m != 0ull);
    while (sel) {
        double s0[U], s1[U], a0[U], a1[U];
        bool h0[U], h1[U];
#pragma unroll
        for (int t = 0; t < U; ++t) {  // all loads of the round first ...
            const int j = sel ? __ffs(sel) - 1 : -1;
            sel &= sel - 1u;
            const int xj = __shfl_sync(FULL, x, j < 0 ? 0 : j);
            const unsigned long long mj = shfl64(m, j < 0 ? 0 : j);
            h0[t] = j >= 0 && ((mj >> lane) & 1ull);
            h1[t] = j >= 0 && ((mj >> (lane + 32)) & 1ull);
            const size_t r0 = sidx(p, lane, xj), r1 = sidx(p, lane + 32, xj);
            s0[t] = h0[t] ? __ldca(p.sig + r0) : 1.0;
            s1[t] = h1[t] ? __ldca(p.sig + r1) : 1.0;
            if (!FWD) {
                a0[t] = h0[t] ? __ldca(p.dacc + r0) : 0.0;
                a1[t] = h1[t] ? __ldca(p.dacc + r1) : 0.0;
            }
        }
#pragma unroll
        for (int t = 0; t < U; ++t) {  // ... then the arithmetic, in arc order
            if (FWD) {
                acc0 += h0[t] ? s0[t] : 0.0;
                acc1 += h1[t] ? s1[t] : 0.0;
            } else {  // omega_b(x) = 1 / sigma_b(x) + acc_b(x)
                acc0 += h0[t] ? 1.0 / s0[t] + a0[t] : 0.0;
                acc1 += h1[t] ? 1.0 / s1[t] + a1[t] : 0.0;
            }
        }
    }
    double *tgt = FWD ? p.sig : p.dacc;
    if (acc0 != 0.0) atomicAdd(tgt + sidx(p, lane, u), acc0);
    if (acc1 != 0.0) atomicAdd(tgt + sidx(p, lane + 32, u), acc1);
}

// Window spanning several rows (lanes = arcs): the window's (arc, source) pairs are
// compacted into a per-warp list in shared memory and dealt out evenly, U pairs per
// lane in flight: gathers first, then fire-and-forget fp64 reductions into the row's
// accumulator (sums of integers < 2^53 are exact in any order).
template <bool FWD>
__device__ __forceinline__ void accumulate_pairs(const BParams &p, uint16_t *lst, int x, int u,
                                                 unsigned long long m) {
    constexpr int U = FWD ? 6 : 4;
    const int lane = threadIdx.x & 31;
    const int c = __popcll(m);
    int incl = c;
#pragma unroll
    for (int s = 1; s < 32; s <<= 1) {
        const int y = __shfl_up_sync(FULL, incl, s);
        if (lane >= s) incl += y;
    }
    const int P = __shfl_sync(FULL, incl, 31);
    int k = incl - c;
    while (m) {
        const int b = __ffsll((long long)m) - 1;
        m &= m - 1ull;
        lst[k++] = (uint16_t)((lane << 6) | b);
    }
    __syncwarp();
    for (int k0 = 0; k0 < P; k0 += 32 * U) {
        int bb[U], uu[U];
        double sv[U], av[U];
#pragma unroll
        for (int t = 0; t < U; ++t) {
            const int kk = k0 + t * 32 + lane;
            const int e = kk < P ? lst[kk] : -1;
            const int j = e < 0 ? 0 : e >> 6;
            const int xj = __shfl_sync(FULL, x, j);
            uu[t] = __shfl_sync(FULL, u, j);
            bb[t] = e < 0 ? -1 : (e & 63);
            const size_t r = sidx(p, bb[t] < 0 ? 0 : bb[t], xj);
            sv[t] = bb[t] >= 0 ? __ldca(p.sig + r) : 1.0;
            if (!FWD) av[t] = bb[t] >= 0 ? __ldca(p.dacc + r) : 0.0;
        }
#pragma unroll
        for (int t = 0; t < U; ++t)
            if (bb[t] >= 0)  // RED.ADD.F64 (result unused)
                atomicAdd((FWD ? p.sig : p.dacc) + sidx(p, bb[t], uu[t]), FWD ? sv[t] : 1.0 / sv[t] + av[t]);
    }
    __syncwarp();
}

// ---- one warp's range [a_lo, a_hi) of level L's arc space
//
// Software-pipelined: the rows of window i+1 are fetched in two stages (Q / offsets,
// then mask / CSR start) behind window i's column, mask, discovery and gather loads,
// and the enqueue reservation of window i is consumed only after its gathers are
// issued, so a window costs about four dependent memory round trips.

struct RowStage {  // stage 1 of a row fetch (lane j: row r0 + j)
    int r0, u, start, nxt;
};

__device__ __forceinline__ void rows_stage1(const BParams &p, RowStage &S, int r0, int qlo, int qn, int A) {
    const int r = r0 + (threadIdx.x & 31);
    S.r0 = r0;
    if (r < qn) {
        S.u = __ldcg(&p.Q[qlo + r]);
        S.start = __ldcg(&p.qoff[qlo + r]);
        S.nxt = r + 1 < qn ? __ldcg(&p.qoff[qlo + r + 1]) : A;
    } else {
        S.u = -1;
        S.start = S.nxt = BIG;
    }
}

__device__ __forceinline__ void rows_stage2(const BParams &p, Rows &R, const RowStage &S, int L) {
    R.r0 = S.r0;
    R.u = S.u < 0 ? 0 : S.u;
    R.start = S.start;
    R.nxt = S.nxt;
    if (S.u >= 0) {
        R.f = __ldcg(&p.F[(size_t)S.u * p.LS + L]);
        R.cbeg = __ldg(&p.ro[S.u]) - S.start;
    } else {
        R.f = 0ull;
        R.cbeg = 0;
    }
}

template <bool FWD>
__device__ __forceinline__ void process_range(const BParams &p, const Level &lv, int a_lo, int a_hi, Cnt &c,
                                              unsigned long long &wor, uint16_t *lst, long long *tprof) {
    const int lane = threadIdx.x & 31;
    const int L = lv.L;
    const int LS = p.LS;
    const long long tr0 = clock64();
    int rb = find_row(p, lv.qlo, lv.qn, a_lo);  // row containing arc `base`
    Rows R;
    RowStage S;
    rows_stage1(p, S, rb, lv.qlo, lv.qn, lv.A);
    rows_stage2(p, R, S, L);
    for (int base = a_lo; base < a_hi; base += 32) {
        // rows ending inside the window: bit k <=> some cached row ends at arc base + k
        const int rel = R.nxt - base;
        const unsigned M = __reduce_or_sync(FULL, (rel >= 1 && rel <= 31) ? (1u << rel) : 0u);
        const bool end32 = __any_sync(FULL, rel == 32);
        const unsigned below = lane == 31 ? FULL : ((2u << lane) - 1u);
        const int o = __popc(M & below);  // lane's row, relative to rb
        const int a = base + lane;
        const bool ok = a < a_hi;
        const unsigned long long f = shfl64(R.f, o);
        const int cb = __shfl_sync(FULL, R.cbeg, o);
        const int u = __shfl_sync(FULL, R.u, o);
        const int rs = __shfl_sync(FULL, R.start, o), re = __shfl_sync(FULL, R.nxt, o);
        const int x = ok ? __ldg(&p.col[a + cb]) : 0;                 // trip 1
        const int rb_next = rb + __popc(M) + (end32 ? 1 : 0);         // row containing arc base + 32
        const bool more = base + 32 < a_hi;
        const bool newrows = more && rb_next != rb;
        if (newrows) rows_stage1(p, S, rb_next, lv.qlo, lv.qn, lv.A);  // behind trip 1
        unsigned long long m;  // sources whose accumulator for u takes a term from x
        unsigned nb = 0u;
        int dv = 0, incl = 0;
        unsigned long long resv = 0ull;
        if (FWD) {
            unsigned long long fp = 0ull, fc = 0ull, fn = 0ull;
            unsigned long long *Fx = p.F + (size_t)x * LS + L;
            if (ok) {                                                  // trip 2
                if (L > 0) fp = __ldca(Fx - 1);  // levels L-1, L: fixed during this level
                fc = __ldca(Fx);
                fn = __ldcg(Fx + 1);             // level L+1: being built (atomics, L2)
            }
            m = f & fp;
            const unsigned long long dm = ok ? (f & ~(fp | fc | fn)) : 0ull;
            bool fresh = false;
            if (dm) {                                                  // trip 3
                dv = __ldg(&p.ro[x + 1]) - __ldg(&p.ro[x]);            // (degree, in the same trip)
                const unsigned long long old = atomicOr(Fx + 1, dm);
                fresh = old == 0ull;  // the first discoverer enqueues x
                unsigned long long nw = dm & ~old;  // (x, b) pairs this lane discovered
                while (nw) {
                    const int b = __ffsll((long long)nw) - 1;
                    nw &= nw - 1ull;
                    p.sig[sidx(p, b, x)] = 0.0;
                    p.dacc[sidx(p, b, x)] = 0.0;
                }
            }
            nb = __ballot_sync(FULL, fresh);
            if (nb) {  // reserve Q entries + arcs; the result is consumed after the gathers
                if (!fresh) dv = 0;
                incl = dv;
#pragma unroll
                for (int s = 1; s < 32; s <<= 1) {
                    const int y = __shfl_up_sync(FULL, incl, s);
                    if (lane >= s) incl += y;
                }
                const int tot = __shfl_sync(FULL, incl, 31);
                if (lane == 0)
                    resv = atomicAdd(&p.qctr[L + 1], ((unsigned long long)__popc(nb) << 40) | (unsigned long long)tot);
            }
            c.dag += (unsigned)__popcll(m);
            if (ok && a == rs) {  // first arc of the row: per-row statistics
                c.reached += (unsigned)__popcll(f);
                c.dsum += (unsigned long long)L * (unsigned long long)__popcll(f);
                c.ar += (unsigned)__popcll(f) * (unsigned)(re - rs);
                wor |= f;
            }
        } else {
            m = ok ? (f & __ldca(p.F + (size_t)x * LS + L + 1)) : 0ull;  // trip 2
        }
        if (newrows) rows_stage2(p, R, S, L);  // next window's rows (stage 1 has long arrived)
        // one dense row (a hub at its usual level): lanes = sources, register sums;
        // otherwise lanes = pairs.  `u_row` is the window's row when M == 0.
        const int npairs = __reduce_add_sync(FULL, (unsigned)__popcll(m));
        const long long tg = clock64();
        const bool rowwin = M == 0u && npairs > 96;
        if (rowwin) gather_row_window<FWD>(p, x, m, u);   // trip 4
        else if (npairs) accumulate_pairs<FWD>(p, lst, x, u, m);
        if (tprof && lane == 0) {
            tprof[rowwin ? 0 : 1] += clock64() - tg;
            tprof[rowwin ? 2 : 3] += 1;
            tprof[4] += npairs;
        }
        if (FWD && nb) {
            resv = shfl64(resv, 0);
            if ((nb >> lane) & 1u) {
                const int pos = lv.qlo_next + (int)(resv >> 40) + __popc(nb & ((1u << lane) - 1u));
                p.Q[pos] = x;
                p.qoff[pos] = (int)(resv & ARC_MASK) + incl - dv;
            }
        }
        if (lane == 0) c.sc += (unsigned)min(32, a_hi - base);
        rb = rb_next;
    }
    if (tprof && lane == 0) tprof[5] += clock64() - tr0;
}

// ---- one warp's range [a_lo, a_hi) of ALL arcs: a multi-source edge-parallel forward level
// (Jia et al.'s EP, P:96 / P:112, with one arc scan serving every source of the batch).  The
// row of arc a is src[a]; a 32-arc window whose rows hold no frontier vertex of any source
// costs two coalesced loads.  Per arc the same work as process_range<true>: the sigma pull
// of the row's sources from x = col[a], the discovery of x for the sources that reach it
// first, x enqueued into Q_{L+1} once (the backward and later WE levels run on the queues).
__device__ __forceinline__ void process_range_ep(const BParams &p, const Level &lv, int a_lo, int a_hi, Cnt &c,
                                                 unsigned long long &wor, uint16_t *lst) {
    const int lane = threadIdx.x & 31;
    const int L = lv.L;
    const int LS = p.LS;
    for (int base = a_lo; base < a_hi; base += 32) {
        const int a = base + lane;
        const bool ok = a < a_hi;
        if (lane == 0) c.sc += (unsigned)min(32, a_hi - base);
        const int u = ok ? __ldg(&p.src[a]) : 0;
        const unsigned long long f = ok ? __ldcg(&p.F[(size_t)u * LS + L]) : 0ull;
        if (!__any_sync(FULL, f != 0ull)) continue;
        const int x = f ? __ldg(&p.col[a]) : 0;
        unsigned long long fp = 0ull, fc = 0ull, fn = 0ull;
        unsigned long long *Fx = p.F + (size_t)x * LS + L;
        if (f) {
            if (L > 0) fp = __ldca(Fx - 1);
            fc = __ldca(Fx);
            fn = __ldcg(Fx + 1);
        }
        const unsigned long long m = f & fp;
        const unsigned long long dm = f & ~(fp | fc | fn);
        bool fresh = false;
        int dv = 0, incl = 0;
        unsigned long long resv = 0ull;
        if (dm) {
            dv = __ldg(&p.ro[x + 1]) - __ldg(&p.ro[x]);
            const unsigned long long old = atomicOr(Fx + 1, dm);
            fresh = old == 0ull;
            unsigned long long nw = dm & ~old;
            while (nw) {
                const int b = __ffsll((long long)nw) - 1;
                nw &= nw - 1ull;
                p.sig[sidx(p, b, x)] = 0.0;
                p.dacc[sidx(p, b, x)] = 0.0;
            }
        }
        const unsigned nb = __ballot_sync(FULL, fresh);
        if (nb) {
            if (!fresh) dv = 0;
            incl = dv;
#pragma unroll
            for (int s = 1; s < 32; s <<= 1) {
                const int y = __shfl_up_sync(FULL, incl, s);
                if (lane >= s) incl += y;
            }
            const int tot = __shfl_sync(FULL, incl, 31);
            if (lane == 0)
                resv = atomicAdd(&p.qctr[L + 1], ((unsigned long long)__popc(nb) << 40) | (unsigned long long)tot);
        }
        c.dag += (unsigned)__popcll(m);
        if (f) {  // first arc of a frontier row: per-row statistics
            const int rs = __ldg(&p.ro[u]);
            if (a == rs) {
                const unsigned nf = (unsigned)__popcll(f);
                c.reached += nf;
                c.ar += nf * (unsigned)(__ldg(&p.ro[u + 1]) - rs);
                c.dsum += (unsigned long long)L * nf;
                wor |= f;
            }
        }
        const int npairs = __reduce_add_sync(FULL, (unsigned)__popcll(m));
        int same = 0;
        __match_all_sync(FULL, u, &same);
        if (same && npairs > 96 && __all_sync(FULL, ok)) gather_row_window<true>(p, x, m, u);
        else if (npairs) accumulate_pairs<true>(p, lst, x, u, m);
        if (nb) {
            resv = shfl64(resv, 0);
            if ((nb >> lane) & 1u) {
                const int pos = lv.qlo_next + (int)(resv >> 40) + __popc(nb & ((1u << lane) - 1u));
                p.Q[pos] = x;
                p.qoff[pos] = (int)(resv & ARC_MASK) + incl - dv;
            }
        }
    }
}

// delta_b(u) = sigma_b(u) * acc_b(u) for every pair of level L (complete after the
// barrier that ended backward level L), summed over b into bc[u] (Eq. 3).
// Thread per (entry, source): 64 consecutive threads share one Q entry.
template <int NT>
__device__ __forceinline__ void delta_pass(const BParams &p, int L, int qlo, int qn, Cnt &c) {
    const int gtid = blockIdx.x * NT + threadIdx.x, GT = gridDim.x * NT;
    const long long np = (long long)qn * BW;
    for (long long t0 = (long long)gtid - (threadIdx.x & 31); t0 < np; t0 += GT) {  // warp-uniform trip count
        const long long t = t0 + (threadIdx.x & 31);
        double d = 0.0;
        int u = -1;
        if (t < np) {
            u = __ldcg(&p.Q[qlo + (int)(t >> 6)]);
            const int b = (int)(t & 63);
            if ((__ldcg(&p.F[(size_t)u * p.LS + L]) >> b) & 1ull) {
                const double su = __ldcg(p.sig + sidx(p, b, u));
                if (su >= TWO53) c.inexact = 1;  // order-dependent sum of >= 3 terms possible
                d = su * __ldcg(p.dacc + sidx(p, b, u));
                if (p.dbg_delta) p.dbg_delta[(size_t)b * p.n + u] = d;
            }
        }
        d = warp_sum(d);  // the 32 lanes share u (64 pairs per entry = 2 warps)
        if ((threadIdx.x & 31) == 0 && u >= 0 && d != 0.0) atomicAdd(&p.bc[u], d);
    }
}

__device__ __forceinline__ void trace_level(const BParams &p, int dir, int L, int A, long long t0, bool active) {
    if ((threadIdx.x & 31) != 0 || !active) return;
    long long *t = p.trace + ((size_t)dir * p.LS + L) * 12;
    const long long dt = clock64() - t0;
    atomicMax(&t[1], dt);
    atomicAdd((unsigned long long *)&t[2], (unsigned long long)dt);
    if (threadIdx.x == 0 && blockIdx.x == 0) t[3] = A;
}

// trace slots 4.. of a level: cycles in row windows, in pair lists, their counts, pairs,
// cycles in the whole range
__device__ __forceinline__ void trace_flush(const BParams &p, int dir, int L, long long *tp) {
    if ((threadIdx.x & 31) != 0) return;
    long long *t = p.trace + ((size_t)dir * p.LS + L) * 12 + 4;
    for (int i = 0; i < 6; ++i)
        if (tp[i]) atomicAdd((unsigned long long *)&t[i], (unsigned long long)tp[i]);
}

template <int NT>
__global__ void __launch_bounds__(NT, 768 / NT) batch_kernel(BParams p) {
    if (p.sampled_flag && __ldcg(p.sampled_flag) == 0) return;  // Alg. 5 chose WE: bc_kernel runs
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_qlo[MAX_LCAP + 4];  // Q offset of each level
    __shared__ int s_A[MAX_LCAP + 4];    // arcs of each level
    __shared__ unsigned char s_ep[MAX_LCAP + 4];  // forward level L ran edge-parallel
    const int run_ep = p.ep_flag ? __ldcg(p.ep_flag) : 1;
    __shared__ long long s_ovf;
    __shared__ uint16_t s_lst[NT / 32][32 * BW];  // per-warp (arc, source) pair lists
    uint16_t *lst = s_lst[threadIdx.x >> 5];
    const int lane = threadIdx.x & 31;
    const int gtid = blockIdx.x * NT + threadIdx.x, GT = gridDim.x * NT;
    const int gw = gtid >> 5, GW = GT >> 5;
    const int LS = p.LS;
    __shared__ unsigned long long s_cnt[NT / 32][5];  // per-warp totals over completed batches
    __shared__ int s_inexact;
    if (lane == 0)
        for (int i = 0; i < 5; ++i) s_cnt[threadIdx.x >> 5][i] = 0ull;
    if (threadIdx.x == 0) s_inexact = 0;
    const long long nbatch = (p.k + BW - 1) / BW;

    for (long long bt = 0; bt < nbatch; ++bt) {
        const long long b0 = bt * BW;
        const int nb = (int)min((long long)BW, p.k - b0);
        Cnt cb;  // this batch's counters, kept only if it completes (no overflow)
        unsigned long long wor = 0ull;
        // ---- Alg. 1 for the batch: d_b(s_b) = 0, sigma_b(s_b) = 1
        if (threadIdx.x == 0) s_qlo[0] = 0;
        if (gtid < nb) {
            const int b = gtid;
            int s = p.sources ? p.sources[p.src_base + b0 + b] : (int)(p.src_base + b0 + b);
            if (p.perm) s = p.perm[s];
            p.sig[sidx(p, b, s)] = 1.0;
            if (p.dbg_d) {
                p.dbg_d[(size_t)b * p.n + s] = 0;
                p.dbg_sigma[(size_t)b * p.n + s] = 1.0;
            }
            const int deg = p.ro[s + 1] - p.ro[s];
            // isolated sources have no arcs: bit set, never expanded (every Q row has deg >= 1)
            if (atomicOr(&p.F[(size_t)s * LS], 1ull << b) == 0ull && deg > 0) {
                const unsigned long long old = atomicAdd(&p.qctr[0], CNT_ONE | (unsigned long long)deg);
                p.Q[(int)(old >> 40)] = s;
                p.qoff[(int)(old >> 40)] = (int)(old & ARC_MASK);
            }
            if (deg == 0) {  // its BFS is level 0 alone
                cb.reached += 1;
                atomicOr(&p.lvor[0], 1ull << b);
            }
        }
        grid.sync();

        // ---- forward (Alg. 2), one level per grid barrier
        Level lv;
        lv.L = 0;
        lv.qlo = 0;
        bool ovf = false;
        for (;;) {
            const unsigned long long qc = __ldcg(&p.qctr[lv.L]);
            lv.qn = (int)(qc >> 40);
            lv.A = (int)(qc & ARC_MASK);
            lv.qlo_next = lv.qlo + lv.qn;
            lv.per = max(p.min_range, (lv.A + GW - 1) / GW);
            if (threadIdx.x == 0) {
                s_qlo[lv.L + 1] = lv.qlo_next;
                s_A[lv.L] = lv.A;
            }
            // multi-source EP level: the union frontier is large enough (Alg. 5 guard)
            const bool ep = run_ep && p.ep_guard > 0 && lv.qn >= p.ep_guard;
            if (threadIdx.x == 0) s_ep[lv.L] = ep ? 1 : 0;
            const int nact = lv.A > 0 ? (lv.A + lv.per - 1) / lv.per : 0;
            const long long t0 = clock64();
            long long tp[6] = {0, 0, 0, 0, 0, 0};
            long long *tpp = (p.trace && bt == 0) ? tp : nullptr;
            if (ep) {
                const int per = max(p.min_range, (p.nnz + GW - 1) / GW);
                if (gw * (long long)per < p.nnz) process_range_ep(p, lv, gw * per, min(p.nnz, (gw + 1) * per), cb, wor, lst);
            } else if (gw < nact) {
                process_range<true>(p, lv, gw * lv.per, min(lv.A, (gw + 1) * lv.per), cb, wor, lst, tpp);
            }
            if (tpp) trace_flush(p, 0, lv.L, tp);
            if (p.trace && bt == 0) trace_level(p, 0, lv.L, lv.A, t0, gw < nact);
            {
                const unsigned lo32 = __reduce_or_sync(FULL, (unsigned)wor);
                const unsigned hi32 = __reduce_or_sync(FULL, (unsigned)(wor >> 32));
                const unsigned long long w64 = ((unsigned long long)hi32 << 32) | lo32;
                if (lane == 0 && w64) atomicOr(&p.lvor[lv.L], w64);
            }
            wor = 0ull;
            grid.sync();
            if (p.trace && bt == 0 && gtid == 0) atomicAdd((unsigned long long *)&p.trace[lv.L * 12], (unsigned long long)(clock64() - t0));
            const int qn1 = (int)(__ldcg(&p.qctr[lv.L + 1]) >> 40);
            if (qn1 == 0) break;  // Q_next_len == 0 (Alg. 2 l.11)
            if (lv.L + 1 > p.Lcap) {
                ovf = true;
                break;
            }
            lv.qlo = lv.qlo_next;
            ++lv.L;
        }
        const int Lmax = lv.L;
        const int Ltop = ovf ? Lmax + 1 : Lmax;  // deepest level holding Q entries
        if (threadIdx.x == 0) s_qlo[Lmax + 2] = s_qlo[Lmax + 1] + (int)(__ldcg(&p.qctr[Lmax + 1]) >> 40);
        __syncthreads();

        if (!ovf) {
            // ---- backward (Alg. 3), deepest level first.  The deepest level's pairs have
            // no successors: acc = 0 (zeroed at discovery), delta = 0, omega = 1 / sigma.
            for (int Lb = Lmax - 1; Lb >= 1; --Lb) {
                Level bl;
                bl.L = Lb;
                bl.qlo = s_qlo[Lb];
                bl.qn = s_qlo[Lb + 1] - bl.qlo;
                bl.A = s_A[Lb];
                bl.qlo_next = s_qlo[Lb + 1];
                bl.per = max(p.min_range, (bl.A + GW - 1) / GW);
                const int nact = bl.A > 0 ? (bl.A + bl.per - 1) / bl.per : 0;
                const long long t0 = clock64();
                long long tp[6] = {0, 0, 0, 0, 0, 0};
                long long *tpp = (p.trace && bt == 0) ? tp : nullptr;
                if (gw < nact) process_range<false>(p, bl, gw * bl.per, min(bl.A, (gw + 1) * bl.per), cb, wor, lst, tpp);
                if (tpp) trace_flush(p, 1, Lb, tp);
                // level Lb + 1 is complete since the last barrier: its deltas into bc
                if (Lb + 1 < Lmax) delta_pass<NT>(p, Lb + 1, s_qlo[Lb + 1], s_qlo[Lb + 2] - s_qlo[Lb + 1], cb);
                if (p.trace && bt == 0) trace_level(p, 1, Lb, bl.A, t0, gw < nact);
                grid.sync();
                if (p.trace && bt == 0 && gtid == 0) atomicAdd((unsigned long long *)&p.trace[((LS + Lb) * 12)], (unsigned long long)(clock64() - t0));
            }
            if (Lmax >= 2) delta_pass<NT>(p, 1, s_qlo[1], s_qlo[2] - s_qlo[1], cb);
            if (p.dbg_d) {  // debug export: d and sigma of every pair
                for (int l = 1; l <= Lmax; ++l) {
                    const long long np = (long long)(s_qlo[l + 1] - s_qlo[l]) * BW;
                    for (long long t = gtid; t < np; t += GT) {
                        const int u = __ldcg(&p.Q[s_qlo[l] + (int)(t >> 6)]);
                        const int b = (int)(t & 63);
                        if ((__ldcg(&p.F[(size_t)u * LS + l]) >> b) & 1ull) {
                            p.dbg_d[(size_t)b * p.n + u] = l;
                            p.dbg_sigma[(size_t)b * p.n + u] = __ldcg(p.sig + sidx(p, b, u));
                        }
                    }
                }
            }
            grid.sync();
        } else if (blockIdx.x == 0) {
            // more than Lcap + 1 levels: this batch's sources go to the per-source kernel
            if (threadIdx.x == 0) s_ovf = (long long)atomicAdd((unsigned long long *)p.ovf_n, (unsigned long long)nb);
            __syncthreads();
            for (int b = threadIdx.x; b < nb; b += NT)
                p.ovf_src[s_ovf + b] = p.sources ? p.sources[p.src_base + b0 + b] : (int)(p.src_base + b0 + b);
        }

        // ---- reset for the next batch: masks of every Q entry and of the sources, counters
        for (int l = 1; l <= Ltop; ++l)
            for (int i = s_qlo[l] + gtid; i < s_qlo[l + 1]; i += GT) p.F[(size_t)__ldcg(&p.Q[i]) * LS + l] = 0ull;
        if (gtid < nb) {
            int s = p.sources ? p.sources[p.src_base + b0 + gtid] : (int)(p.src_base + b0 + gtid);
            if (p.perm) s = p.perm[s];
            p.F[(size_t)s * LS] = 0ull;
        }
        if (blockIdx.x == 0) {
            for (int l = threadIdx.x; l <= Ltop + 1 && l < LS; l += NT) p.qctr[l] = 0ull;
            if (threadIdx.x < 32) {
                unsigned long long lvs = 0, lve = 0;
                for (int l = threadIdx.x; l <= Ltop && l < LS; l += 32) {
                    const unsigned long long pc = (unsigned long long)__popcll(__ldcg(&p.lvor[l]));
                    lvs += pc;
                    if (s_ep[l]) lve += pc;
                    p.lvor[l] = 0ull;
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    lvs += __shfl_xor_sync(FULL, lvs, o);
                    lve += __shfl_xor_sync(FULL, lve, o);
                }
                if (threadIdx.x == 0) {
                    if (!ovf) {
                        atomicAdd(&p.stats->levels, lvs);
                        atomicAdd(&p.stats->we_levels, lvs - lve);
                        atomicAdd(&p.stats->ep_levels, lve);
                        atomicAdd(&p.stats->sources, (unsigned long long)nb);
                    } else {
                        atomicAdd(&p.stats->batch_overflows, 1ull);
                    }
                    atomicAdd(&p.stats->batches, 1ull);
                }
            }
        }
        if (!ovf) {  // overflowed batches are counted by the per-source rerun
            unsigned long long v[5] = {cb.reached, cb.ar, cb.dag, cb.sc, cb.dsum};
#pragma unroll
            for (int i = 0; i < 5; ++i) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v[i] += __shfl_xor_sync(FULL, v[i], o);
                if (lane == 0) s_cnt[threadIdx.x >> 5][i] += v[i];
            }
        }
        if (cb.inexact) s_inexact = 1;
        grid.sync();
    }

    // per-warp flush of the byte-model counters
    __syncthreads();
    if (lane == 0) {
        const unsigned long long *v = s_cnt[threadIdx.x >> 5];
        if (v[0]) atomicAdd(&p.stats->n_reached, v[0]);
        if (v[1]) atomicAdd(&p.stats->arcs_reached, v[1]);
        if (v[2]) atomicAdd(&p.stats->dag_arcs, v[2]);
        if (v[3]) atomicAdd(&p.stats->arcs_scanned, v[3]);
        if (v[4]) atomicAdd(&p.stats->dist_sum, v[4]);
    }
    if (threadIdx.x == 0 && s_inexact) atomicOr(&p.stats->sigma_inexact, 1);
}

const void *batch_kernel_fn(int nt) {
    return nt == 128 ? (const void *)batch_kernel<128> : (const void *)batch_kernel<256>;
}

}  // namespace bcbatch
