// bc_batch.cu -- the multi-source batched engine (design in bc_batch.cuh).
//
// One cooperative persistent kernel; all CTAs work on one batch of 64 sources at a time
// and meet at a grid barrier after every level.  Work inside a level is pulled from
// global counters (16 frontier vertices, or one hub chunk, per grab) by whole warps.
#define BC_INSTANCE_TU
#include "bc_kernels.cuh"
#include "bc_batch.cuh"

#include <cooperative_groups.h>

namespace cg = cooperative_groups;

namespace bcbatch {

using bcdev::DevStats;
using bcdev::FULL;
using bcdev::TWO53;

constexpr int GRAB = 16;                          // frontier vertices per warp grab
constexpr unsigned long long CNT_ONE = 1ull << 40; // packed hub counter: count << 40 | chunks
constexpr unsigned long long CH_MASK = CNT_ONE - 1;

struct Cnt {
    unsigned long long reached = 0, ar = 0, dag = 0, sc = 0;
    int inexact = 0;
};

__device__ __forceinline__ unsigned long long shfl64(unsigned long long v, int src) {
    return __shfl_sync(FULL, v, src);
}

// Append hub vertex x (deg > CH) to the hub list of level `lvl` (entries start at hlo).
__device__ __forceinline__ void hub_push(const BParams &p, int lvl, int hlo, int x, int deg) {
    const unsigned long long nch = (unsigned long long)((deg + p.CH - 1) / p.CH);
    const unsigned long long old = atomicAdd(&p.hcnt[lvl], CNT_ONE | nch);
    const int pos = hlo + (int)(old >> 40);
    p.hv[pos] = x;
    p.hb[pos] = (int)(old & CH_MASK);
}

// Sum over the arcs j (in ascending lane order = CSR order) of the current 32-arc
// group whose mask bit of this lane's source is set: acc0 += val[x_j*64 + lane],
// acc1 += val[x_j*64 + 32 + lane].  Four arcs' gathers are issued before they are
// added; skipped slots add +0.0, which leaves the sums bit-identical.
__device__ __forceinline__ void gather_group(const double *__restrict__ val, int x, unsigned long long m,
                                             int lane, double &acc0, double &acc1) {
    unsigned sel = __ballot_sync(FULL, m != 0ull);
    while (sel) {
        int j[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            j[t] = sel ? __ffs(sel) - 1 : -1;
            sel &= sel - 1u;  // sel == 0 stays 0
        }
        double g0[4], g1[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int jj = j[t] < 0 ? 0 : j[t];
            const int xj = __shfl_sync(FULL, x, jj);
            const unsigned long long mj = j[t] < 0 ? 0ull : shfl64(m, jj);
            const double *row = val + (size_t)xj * BW;
            g0[t] = (mj >> lane) & 1ull ? __ldcg(row + lane) : 0.0;
            g1[t] = (mj >> (lane + 32)) & 1ull ? __ldcg(row + 32 + lane) : 0.0;
        }
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            acc0 += g0[t];
            acc1 += g1[t];
        }
    }
}

// Forward scan of arcs [a0, a1) of a level-L vertex with source mask f (one warp).
template <bool PULL>
__device__ __forceinline__ void fwd_seg(const BParams &p, int L, unsigned long long f, int a0, int a1,
                                        int qlo_next, int hlo_next, double &acc0, double &acc1, Cnt &c) {
    const int lane = threadIdx.x & 31;
    const int LS = p.LS;
    for (int base = a0; base < a1; base += 32) {
        const int a = base + lane;
        const bool ok = a < a1;
        const int x = ok ? __ldg(&p.col[a]) : 0;
        unsigned long long fp = 0ull, fc = 0ull, fn = 0ull;
        unsigned long long *Fx = p.F + (size_t)x * LS + L;
        if (ok) {
            if (PULL) fp = __ldcg(Fx - 1);
            fc = __ldcg(Fx);
            fn = __ldcg(Fx + 1);
        }
        const unsigned long long pm = f & fp;
        const unsigned long long dm = ok ? (f & ~(fp | fc | fn)) : 0ull;
        bool fresh = false;
        if (dm) fresh = atomicOr(Fx + 1, dm) == 0ull;  // first discoverer enqueues x
        const unsigned nb = __ballot_sync(FULL, fresh);
        if (nb) {
            const int leader = __ffs(nb) - 1;
            int qb = 0;
            if (lane == leader) qb = atomicAdd(&p.qcnt[L + 1], __popc(nb));
            qb = __shfl_sync(FULL, qb, leader);
            if (fresh) {
                p.Q[qlo_next + qb + __popc(nb & ((1u << lane) - 1u))] = x;
                const int deg = __ldg(&p.ro[x + 1]) - __ldg(&p.ro[x]);
                if (deg > p.CH) hub_push(p, L + 1, hlo_next, x, deg);
            }
        }
        if (PULL) {
            c.dag += (unsigned long long)__popcll(pm);
            gather_group(p.sig, x, pm, lane, acc0, acc1);
        }
    }
}

// Backward scan of arcs [a0, a1) of a level-L vertex: omega of successors (F_{L+1}).
__device__ __forceinline__ void bwd_seg(const BParams &p, int L, unsigned long long f, int a0, int a1,
                                        double &acc0, double &acc1) {
    const int lane = threadIdx.x & 31;
    for (int base = a0; base < a1; base += 32) {
        const int a = base + lane;
        const bool ok = a < a1;
        const int x = ok ? __ldg(&p.col[a]) : 0;
        const unsigned long long fs = ok ? __ldcg(p.F + (size_t)x * p.LS + L + 1) : 0ull;
        gather_group(p.sig, x, f & fs, lane, acc0, acc1);
    }
}

// Alg. 3 l.8 with the omega trick for the lane's two sources of vertex u (mask f),
// then Eq. 3: returns the lane's share of sum_b delta_b(u).
__device__ __forceinline__ double finish_pair(const BParams &p, int u, unsigned long long f, double acc0,
                                              double acc1) {
    const int lane = threadIdx.x & 31;
    double bs = 0.0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int b = lane + 32 * h;
        if ((f >> b) & 1ull) {
            double *e = p.sig + (size_t)u * BW + b;
            const double su = __ldcg(e);
            const double delta = su * (h ? acc1 : acc0);
            *e = (1.0 + delta) / su;
            bs += delta;
            if (p.dbg_delta) p.dbg_delta[(size_t)b * p.n + u] = delta;
        }
    }
    return bs;
}

__device__ __forceinline__ void store_sigma(const BParams &p, int u, int L, unsigned long long f, double acc0,
                                            double acc1) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int b = lane + 32 * h;
        if ((f >> b) & 1ull) {
            const double s = h ? acc1 : acc0;
            p.sig[(size_t)u * BW + b] = s;
            if (p.dbg_d) {
                p.dbg_d[(size_t)b * p.n + u] = L;
                p.dbg_sigma[(size_t)b * p.n + u] = s;
            }
        }
    }
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

// Hub entry holding chunk ci of a level: the last entry in [hlo, hlo + hn) whose first
// chunk index is <= ci (first-chunk indices grow with the entry index).
__device__ __forceinline__ int hub_find(const BParams &p, int hlo, int hn, int ci) {
    int lo = 0, hi = hn - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (__ldcg(&p.hb[hlo + mid]) <= ci) lo = mid;
        else hi = mid - 1;
    }
    return hlo + lo;
}

template <int NT>
__global__ void __launch_bounds__(NT, 1024 / NT) batch_kernel(BParams p) {
    if (p.sampled_flag && __ldcg(p.sampled_flag) == 0) return;  // Alg. 5 chose WE: bc_kernel runs
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_qlo[MAX_LCAP + 4];   // Q offset of each level
    __shared__ int s_hlo[MAX_LCAP + 4];   // hub-entry offset of each level
    __shared__ int s_hch[MAX_LCAP + 4];   // hub chunks of each level
    __shared__ int s_ovf;
    const int lane = threadIdx.x & 31;
    const int gtid = blockIdx.x * NT + threadIdx.x, GT = gridDim.x * NT;
    const int LS = p.LS;
    int *grab_f = p.grab, *hgrab_f = p.grab + LS, *grab_b = p.grab + 2 * LS, *hgrab_b = p.grab + 3 * LS;
    Cnt c;
    const long long nbatch = (p.k + BW - 1) / BW;

    for (long long bt = 0; bt < nbatch; ++bt) {
        const long long b0 = bt * BW;
        const int nb = (int)min((long long)BW, p.k - b0);
        Cnt cb;  // this batch's counters, kept only if it completes (no overflow)
        // ---- Alg. 1 for the batch: d_b(s_b) = 0, sigma_b(s_b) = 1
        if (threadIdx.x == 0) {
            s_qlo[0] = 0;
            s_hlo[0] = 0;
        }
        if (gtid < nb) {
            const int b = gtid;
            int s = p.sources ? p.sources[p.src_base + b0 + b] : (int)(p.src_base + b0 + b);
            if (p.perm) s = p.perm[s];
            p.sig[(size_t)s * BW + b] = 1.0;
            if (p.dbg_d) {
                p.dbg_d[(size_t)b * p.n + s] = 0;
                p.dbg_sigma[(size_t)b * p.n + s] = 1.0;
            }
            if (atomicOr(&p.F[(size_t)s * LS], 1ull << b) == 0ull) {
                p.Q[atomicAdd(&p.qcnt[0], 1)] = s;
                const int deg = p.ro[s + 1] - p.ro[s];
                if (deg > p.CH) hub_push(p, 0, 0, s, deg);
            }
        }
        grid.sync();

        // ---- forward (Alg. 2), one level per grid barrier
        int L = 0, qlo = 0, hlo = 0;
        bool ovf = false;
        for (;;) {
            const int qn = __ldcg(&p.qcnt[L]);
            const unsigned long long hc = __ldcg(&p.hcnt[L]);
            const int hn = (int)(hc >> 40), hch = (int)(hc & CH_MASK);
            const int qlo_next = qlo + qn, hlo_next = hlo + hn;
            if (threadIdx.x == 0) {
                s_qlo[L + 1] = qlo_next;
                s_hlo[L + 1] = hlo_next;
                s_hch[L] = hch;
            }
            unsigned long long wor = 0ull;
            // hub chunks first (the long poles), then whole rows
            for (;;) {
                int ci = 0;
                if (lane == 0) ci = atomicAdd(&hgrab_f[L], 1);
                ci = __shfl_sync(FULL, ci, 0);
                if (ci >= hch) break;
                int pos = 0;
                if (lane == 0) pos = hub_find(p, hlo, hn, ci);
                pos = __shfl_sync(FULL, pos, 0);
                const int h = __ldcg(&p.hv[pos]);
                const int chunk = ci - __ldcg(&p.hb[pos]);
                const int rb = __ldg(&p.ro[h]), re = __ldg(&p.ro[h + 1]);
                const int a0 = rb + chunk * p.CH, a1 = min(re, a0 + p.CH);
                const unsigned long long f = __ldcg(&p.F[(size_t)h * LS + L]);
                double acc0 = 0.0, acc1 = 0.0;
                if (L > 0) {
                    fwd_seg<true>(p, L, f, a0, a1, qlo_next, hlo_next, acc0, acc1, cb);
                    double *ha = p.hacc + (size_t)pos * BW;
                    if (((f >> lane) & 1ull) && acc0 != 0.0) atomicAdd(ha + lane, acc0);
                    if (((f >> (lane + 32)) & 1ull) && acc1 != 0.0) atomicAdd(ha + 32 + lane, acc1);
                } else {
                    fwd_seg<false>(p, L, f, a0, a1, qlo_next, hlo_next, acc0, acc1, cb);
                }
                if (lane == 0) {
                    cb.sc += (unsigned long long)(a1 - a0);
                    if (chunk == 0) {
                        cb.reached += (unsigned long long)__popcll(f);
                        cb.ar += (unsigned long long)__popcll(f) * (unsigned long long)(re - rb);
                        wor |= f;
                    }
                }
            }
            for (;;) {
                int i0 = 0;
                if (lane == 0) i0 = atomicAdd(&grab_f[L], GRAB);
                i0 = __shfl_sync(FULL, i0, 0);
                if (i0 >= qn) break;
                const int cnt = min(GRAB, qn - i0);
                int my_u = 0, my_b = 0, my_e = 0;
                unsigned long long my_f = 0ull;
                if (lane < cnt) {
                    my_u = __ldcg(&p.Q[qlo + i0 + lane]);
                    my_b = __ldg(&p.ro[my_u]);
                    my_e = __ldg(&p.ro[my_u + 1]);
                    my_f = __ldcg(&p.F[(size_t)my_u * LS + L]);
                }
                for (int j = 0; j < cnt; ++j) {
                    const int u = __shfl_sync(FULL, my_u, j);
                    const int rb = __shfl_sync(FULL, my_b, j), re = __shfl_sync(FULL, my_e, j);
                    if (re - rb > p.CH) continue;  // hub: done by chunks
                    const unsigned long long f = shfl64(my_f, j);
                    double acc0 = 0.0, acc1 = 0.0;
                    if (L > 0) {
                        fwd_seg<true>(p, L, f, rb, re, qlo_next, hlo_next, acc0, acc1, cb);
                        store_sigma(p, u, L, f, acc0, acc1);
                    } else {
                        fwd_seg<false>(p, L, f, rb, re, qlo_next, hlo_next, acc0, acc1, cb);
                    }
                    if (lane == 0) {
                        cb.sc += (unsigned long long)(re - rb);
                        cb.reached += (unsigned long long)__popcll(f);
                        cb.ar += (unsigned long long)__popcll(f) * (unsigned long long)(re - rb);
                        wor |= f;
                    }
                }
            }
            if (lane == 0 && wor) atomicOr(&p.lvor[L], wor);
            grid.sync();
            if (hn > 0 && L > 0) {  // hub sigma = sum of its chunks' partial pulls
                for (int e = gtid >> 5; e < hn; e += GT >> 5) {
                    const int pos = hlo + e;
                    const int h = __ldcg(&p.hv[pos]);
                    const unsigned long long f = __ldcg(&p.F[(size_t)h * LS + L]);
                    double *ha = p.hacc + (size_t)pos * BW;
                    const double v0 = __ldcg(ha + lane), v1 = __ldcg(ha + 32 + lane);
                    ha[lane] = 0.0;
                    ha[32 + lane] = 0.0;
                    if ((((f >> lane) & 1ull) && v0 >= TWO53) || (((f >> (lane + 32)) & 1ull) && v1 >= TWO53))
                        cb.inexact = 1;  // chunk partials were summed in arrival order
                    store_sigma(p, h, L, f, v0, v1);
                }
                grid.sync();
            }
            const int qn1 = __ldcg(&p.qcnt[L + 1]);
            if (qn1 == 0) break;                    // Q_next_len == 0 (Alg. 2 l.11)
            if (L + 1 > p.Lcap) { ovf = true; break; }
            qlo = qlo_next;
            hlo = hlo_next;
            ++L;
        }
        const int Ltop = ovf ? L + 1 : L;  // deepest level holding Q entries
        if (threadIdx.x == 0) {
            const int qn1 = __ldcg(&p.qcnt[L + 1]);
            const unsigned long long hc1 = __ldcg(&p.hcnt[L + 1]);
            s_qlo[L + 2] = s_qlo[L + 1] + qn1;
            s_hlo[L + 2] = s_hlo[L + 1] + (int)(hc1 >> 40);
            s_ovf = 0;
        }
        __syncthreads();

        // ---- backward (Alg. 3), deepest level first
        if (!ovf) {
            for (int Lb = L; Lb >= 1; --Lb) {
                const bool scan = Lb < L;  // the deepest level has no successors: delta = 0
                const int bqlo = s_qlo[Lb], bqn = s_qlo[Lb + 1] - s_qlo[Lb];
                const int bhlo = s_hlo[Lb], bhn = s_hlo[Lb + 1] - s_hlo[Lb], bhch = s_hch[Lb];
                if (scan && bhn > 0) {
                    for (;;) {
                        int ci = 0;
                        if (lane == 0) ci = atomicAdd(&hgrab_b[Lb], 1);
                        ci = __shfl_sync(FULL, ci, 0);
                        if (ci >= bhch) break;
                        int pos = 0;
                        if (lane == 0) pos = hub_find(p, bhlo, bhn, ci);
                        pos = __shfl_sync(FULL, pos, 0);
                        const int h = __ldcg(&p.hv[pos]);
                        const int chunk = ci - __ldcg(&p.hb[pos]);
                        const int rb = __ldg(&p.ro[h]), re = __ldg(&p.ro[h + 1]);
                        const int a0 = rb + chunk * p.CH, a1 = min(re, a0 + p.CH);
                        const unsigned long long f = __ldcg(&p.F[(size_t)h * LS + Lb]);
                        double acc0 = 0.0, acc1 = 0.0;
                        bwd_seg(p, Lb, f, a0, a1, acc0, acc1);
                        double *ha = p.hacc + (size_t)pos * BW;
                        if (((f >> lane) & 1ull) && acc0 != 0.0) atomicAdd(ha + lane, acc0);
                        if (((f >> (lane + 32)) & 1ull) && acc1 != 0.0) atomicAdd(ha + 32 + lane, acc1);
                        if (lane == 0) cb.sc += (unsigned long long)(a1 - a0);
                    }
                }
                for (;;) {
                    int i0 = 0;
                    if (lane == 0) i0 = atomicAdd(&grab_b[Lb], GRAB);
                    i0 = __shfl_sync(FULL, i0, 0);
                    if (i0 >= bqn) break;
                    const int cnt = min(GRAB, bqn - i0);
                    int my_u = 0, my_b = 0, my_e = 0;
                    unsigned long long my_f = 0ull;
                    if (lane < cnt) {
                        my_u = __ldcg(&p.Q[bqlo + i0 + lane]);
                        my_b = __ldg(&p.ro[my_u]);
                        my_e = __ldg(&p.ro[my_u + 1]);
                        my_f = __ldcg(&p.F[(size_t)my_u * LS + Lb]);
                    }
                    for (int j = 0; j < cnt; ++j) {
                        const int u = __shfl_sync(FULL, my_u, j);
                        const int rb = __shfl_sync(FULL, my_b, j), re = __shfl_sync(FULL, my_e, j);
                        if (scan && re - rb > p.CH) continue;  // hub: done by chunks
                        const unsigned long long f = shfl64(my_f, j);
                        double acc0 = 0.0, acc1 = 0.0;
                        if (scan) {
                            bwd_seg(p, Lb, f, rb, re, acc0, acc1);
                            if (lane == 0) cb.sc += (unsigned long long)(re - rb);
                        }
                        const double bs = warp_sum(finish_pair(p, u, f, acc0, acc1));
                        if (lane == 0 && bs != 0.0) atomicAdd(&p.bc[u], bs);
                    }
                }
                grid.sync();
                if (scan && bhn > 0) {
                    for (int e = gtid >> 5; e < bhn; e += GT >> 5) {
                        const int pos = bhlo + e;
                        const int h = __ldcg(&p.hv[pos]);
                        const unsigned long long f = __ldcg(&p.F[(size_t)h * LS + Lb]);
                        double *ha = p.hacc + (size_t)pos * BW;
                        const double v0 = __ldcg(ha + lane), v1 = __ldcg(ha + 32 + lane);
                        ha[lane] = 0.0;
                        ha[32 + lane] = 0.0;
                        const double bs = warp_sum(finish_pair(p, h, f, v0, v1));
                        if (lane == 0 && bs != 0.0) atomicAdd(&p.bc[h], bs);
                    }
                    grid.sync();
                }
            }
        } else if (blockIdx.x == 0) {
            // more than Lcap + 1 levels: this batch's sources go to the per-source kernel
            if (threadIdx.x == 0) s_ovf = (int)atomicAdd((unsigned long long *)p.ovf_n, (unsigned long long)nb);
            __syncthreads();
            for (int b = threadIdx.x; b < nb; b += NT)
                p.ovf_src[s_ovf + b] = p.sources ? p.sources[p.src_base + b0 + b] : (int)(p.src_base + b0 + b);
        }

        // ---- reset for the next batch: masks of every Q entry, level counters
        for (int l = 0; l <= Ltop; ++l)
            for (int i = s_qlo[l] + gtid; i < s_qlo[l + 1]; i += GT) p.F[(size_t)__ldcg(&p.Q[i]) * LS + l] = 0ull;
        if (blockIdx.x == 0) {
            for (int l = threadIdx.x; l <= Ltop + 1 && l < LS; l += NT) {
                p.qcnt[l] = 0;
                p.hcnt[l] = 0ull;
                grab_f[l] = hgrab_f[l] = grab_b[l] = hgrab_b[l] = 0;
            }
            if (threadIdx.x < 32) {
                unsigned long long lv = 0;
                for (int l = threadIdx.x; l <= Ltop && l < LS; l += 32) {
                    lv += (unsigned long long)__popcll(__ldcg(&p.lvor[l]));
                    p.lvor[l] = 0ull;
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) lv += __shfl_xor_sync(FULL, lv, o);
                if (threadIdx.x == 0) {
                    if (!ovf) {
                        atomicAdd(&p.stats->levels, lv);
                        atomicAdd(&p.stats->we_levels, lv);
                        atomicAdd(&p.stats->sources, (unsigned long long)nb);
                    } else {
                        atomicAdd(&p.stats->batch_overflows, 1ull);
                    }
                    atomicAdd(&p.stats->batches, 1ull);
                }
            }
        }
        if (!ovf) {
            c.reached += cb.reached;
            c.ar += cb.ar;
            c.dag += cb.dag;
            c.sc += cb.sc;
        }
        c.inexact |= cb.inexact;
        grid.sync();
    }

    // per-warp flush of the byte-model counters; overflowed batches are
    // counted by the per-source kernel that reruns them
    unsigned long long r = c.reached, a = c.ar, d = c.dag, s = c.sc;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        r += __shfl_xor_sync(FULL, r, o);
        a += __shfl_xor_sync(FULL, a, o);
        d += __shfl_xor_sync(FULL, d, o);
        s += __shfl_xor_sync(FULL, s, o);
    }
    const int inex = __any_sync(FULL, c.inexact);
    if (lane == 0) {
        if (r) atomicAdd(&p.stats->n_reached, r);
        if (a) atomicAdd(&p.stats->arcs_reached, a);
        if (d) atomicAdd(&p.stats->dag_arcs, d);
        if (s) atomicAdd(&p.stats->arcs_scanned, s);
        if (inex) atomicOr(&p.stats->sigma_inexact, 1);
    }
}

const void *batch_kernel_fn(int nt) {
    return nt == 128 ? (const void *)batch_kernel<128>
           : nt == 512 ? (const void *)batch_kernel<512>
                       : (const void *)batch_kernel<256>;
}

}  // namespace bcbatch
