// bc_thin.cuh -- thin-row level passes of the group engine (DESIGN.md §5c'): the same
// forward (Alg. 2 l.3-8 as a pull) and backward (Alg. 3 l.5-9 with the omega
// trick; Eq. 3) as forward_we / backward_we, for large graphs whose rows
// are short and even (no hubs: c5ws, the Watts-Strogatz small world, degree ~10).
//
// Each row is taken by VW lanes (default 1: one row per lane); every lane runs U independent
// col -> code -> sigma chains per iteration (arcs t, t + VW, ..., t + (U-1) VW of its slice),
// the iteration count is warp-uniform, and the S entries / row bounds of the lane's next
// chunk are loaded while the current chunk is expanded.  Against the generic row_pass
// (aligned quads, 3-4 sequential probe -> gather rounds per row, SIMT efficiency 0.67,
// spills at the 64-register cap) this measured 1503 -> 1416 ms per 2,048 c5ws sources on
// B200; virtual warps of 2/4/8 lanes per row (Hong et al.) keep fewer rows in flight and
// were slower (profiles/r02/ab/thin_rows.txt).  With VW > 1 the per-row sum is reduced over
// the VW lanes (a different order of additions: sigma sums of integers below 2^53 are exact
// in any order, omega sums are checked at 1e-9).  Rows longer than THIN_MAX are queued and
// expanded by a whole warp each afterwards.
//
// Level codes are the group engine's global 2-bit codes (GlobalCodes: 0 unvisited,
// 1 + L mod 3), read through L1 (invalidated at every group barrier).  Discoveries are
// idempotent ORs of the code and of the level bitmap (the group compacts level L+1 from
// it); the forward marks the DAG successor arcs in the successor bitmap (one 64-bit window
// per thin row, two REDs), the backward visits only those arcs.
#pragma once

namespace bcdev {

// lanes per row (VW) and arcs in flight per lane (U), forward / backward
#ifndef BC_THIN_VWF
#define BC_THIN_VWF 1
#endif
#ifndef BC_THIN_UF
#define BC_THIN_UF 4
#endif
#ifndef BC_THIN_VWB
#define BC_THIN_VWB 1
#endif
#ifndef BC_THIN_UB
#define BC_THIN_UB 4
#endif
constexpr int THIN_MAX = bcgroup::THIN_MAX_ROW;  // longer rows: one warp each

struct ThinLevel {
    const int *__restrict__ ro;
    const int *__restrict__ col;
    const uint32_t *__restrict__ sbr;  // successor bits (backward reads)
    uint32_t *codes;  // 2-bit codes, this group
    uint32_t *nb;     // forward: bitmap of level L+1
    uint32_t *sb;     // successor bits over CSR positions (nullptr = off)
    double *sig;      // sigma (forward) / sigma-then-omega (backward)
    int kmatch;       // forward: key(L-1) (predecessors); backward: key(L+1) (successors)
    int knew;         // forward: key(L+1)
};

__device__ __forceinline__ int gcode(const uint32_t *codes, int u) {
    const uint32_t wd = __ldca(&codes[(unsigned)u >> 4]);  // L1: invalidated at every barrier
    return (int)(__funnelshift_r(wd, wd, (unsigned)u << 1) & 3u);
}

// Forward arcs a0 + j * stride (j < U; a0 already includes the lane's offset in its row) of a
// row ending at e (stride = VW, or 32 for a wide row).  Adds the pull sum to acc, counts the
// DAG (predecessor) arcs, and returns the warp ballot of successor arcs of slot j in succm[j].
template <int U>
__device__ __forceinline__ void thin_fwd_step(const ThinLevel &t, int a0, int e, int stride, double &acc,
                                              unsigned &dag, unsigned (&succm)[U]) {
    int u[U];
    bool ok[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
        const int a = a0 + j * stride;
        ok[j] = a < e;
        u[j] = ok[j] ? ld_col(t.col + a) : 0;
    }
    int k[U];
#pragma unroll
    for (int j = 0; j < U; ++j) k[j] = gcode(t.codes, u[j]);
    double g[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
        const bool pg = ok[j] && k[j] == t.kmatch;
        g[j] = ldca_if(t.sig + u[j], pg);
        dag += (unsigned)pg;
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {
        const bool un = ok[j] && k[j] == 0;
        red_or_global_if(&t.codes[(unsigned)u[j] >> 4], (uint32_t)t.knew << (((unsigned)u[j] << 1) & 30u), un);
        red_or_global_if(&t.nb[(unsigned)u[j] >> 5], 1u << (u[j] & 31), un);
    }
#pragma unroll
    for (int j = 0; j < U; ++j) succm[j] = __ballot_sync(FULL, ok[j] && (k[j] == 0 || k[j] == t.knew));
#pragma unroll
    for (int j = 0; j < U; ++j) acc += g[j];
}

template <int U>
__device__ __forceinline__ double thin_bwd_step(const ThinLevel &t, int a0, int e, int stride, uint64_t win,
                                                int wbase) {
    int u[U];
    bool s[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
        const int a = a0 + j * stride;
        s[j] = a < e && ((win >> (a - wbase)) & 1ull);
        u[j] = s[j] ? ld_col(t.col + a) : 0;
    }
    double g[U];
#pragma unroll
    for (int j = 0; j < U; ++j) g[j] = ldca_if(t.sig + u[j], s[j]);
    double acc = 0.0;
#pragma unroll
    for (int j = 0; j < U; ++j) acc += g[j];
    return acc;
}

// Successor bits of arcs [a, a + 32) (a whole warp's 32 consecutive arcs), or a window.
__device__ __forceinline__ uint64_t sb_pair(const uint32_t *sb, int w0, bool two) {
    uint64_t w = __ldcg(&sb[w0]);
    if (two) w |= (uint64_t)__ldcg(&sb[w0 + 1]) << 32;
    return w;
}

// One forward (FWD) or backward level over S[lo, hi) of this CTA (warps sm.gw0 + wid of
// sm.gwn sharing the pass).  Forward finish: sigma[v] = sum (L > 0).  Backward finish:
// finish_dependency (omega in place, bc += delta).  Ends with a CTA barrier.
#ifndef BC_THIN_NOINLINE
#define BC_THIN_NOINLINE 0
#endif
#if BC_THIN_NOINLINE
#define BC_THIN_INL __noinline__
#else
#define BC_THIN_INL __forceinline__
#endif
template <int NT, bool FWD, int VW = FWD ? BC_THIN_VWF : BC_THIN_VWB, int U = FWD ? BC_THIN_UF : BC_THIN_UB>
__device__ BC_THIN_INL void thin_pass(const KParams &p, const ThinLevel &t, const int *__restrict__ S, int lo,
                                          int hi, int L, int *bigq, Smem<NT> &sm, Counters &c) {
    constexpr int RPW = 32 / VW;
    constexpr unsigned VMASK = VW == 32 ? FULL : (1u << VW) - 1u;
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int sub = lane & (VW - 1), grp = lane / VW;
    const bool bits = t.sb != nullptr;
    unsigned dag = 0;
    // this warp's chunks of RPW rows: chunk k starts at lo + (gw0 + wid + k gwn) RPW
    const int step = sm.gwn * RPW;
    const int sbase = lo + (sm.gw0 + wid) * RPW;
    auto chunk = [&](int k) -> int { return sbase + k * step; };
    // software pipeline over the chunks: the row bounds of chunk k+1 and the vertex of chunk
    // k+2 are loaded while chunk k is expanded
    int v_n = -1, beg_n = 0, end_n = 0, v_nn = -1;
    {
        const int i0 = chunk(0) + grp, i1 = chunk(1) + grp;
        if (i0 < hi) {
            v_n = S[i0];
            beg_n = t.ro[v_n];
            end_n = t.ro[v_n + 1];
        }
        if (i1 < hi) v_nn = S[i1];
    }
    for (int k = 0; chunk(k) < hi; ++k) {
        int v = v_n, beg = beg_n, end = end_n;
        v_n = v_nn;
        beg_n = end_n = 0;
        if (v_n >= 0) {
            beg_n = t.ro[v_n];
            end_n = t.ro[v_n + 1];
        }
        const int i2 = chunk(k + 2) + grp;
        v_nn = i2 < hi ? S[i2] : -1;
        double sw = 0.0;
        const bool thin = v >= 0 && end - beg <= THIN_MAX;
        if (!thin) {  // wide row: queued for a whole warp
            if (sub == 0 && v >= 0) bigq[atomicAdd(&sm.nbig, 1)] = v;
            end = beg;
        } else if (sub == 0) {
            c.scanned += end - beg;
            if (FWD) c.arcs_reached += end - beg;
            if (!FWD && v >= 0) sw = __ldcg(&t.sig[v]);  // sigma[v], issued early
        }
        const int wbase = (beg >> 5) << 5;  // the row's <= 64-arc successor window
        const int nit = (end - beg + VW * U - 1) / (VW * U);
        const int maxit = (int)__reduce_max_sync(FULL, (unsigned)nit);
        double acc = 0.0;
        if (FWD) {
            uint64_t win = 0;
            for (int it = 0; it < maxit; ++it) {
                const int a0 = beg + it * VW * U;
                unsigned sm_[U];
                thin_fwd_step<U>(t, a0 + sub, end, VW, acc, dag, sm_);
                if (bits) {
#pragma unroll
                    for (int j = 0; j < U; ++j) {
                        const uint64_t slice = (sm_[j] >> (grp * VW)) & VMASK;
                        const int off = a0 + j * VW - wbase;
                        if (off < 64) win |= slice << off;  // bits past the row's end are 0
                    }
                }
            }
            if (bits && sub == 0) {
                red_or_global_if(&t.sb[wbase >> 5], (uint32_t)win, (uint32_t)win != 0u);
                red_or_global_if(&t.sb[(wbase >> 5) + 1], (uint32_t)(win >> 32), (win >> 32) != 0ull);
            }
        } else {
            if (VW == 1 && BC_SUCC_EXTRACT) {  // the row's successors, four at a time
                acc = succ_sum(t.sbr, t.col, t.sig, beg, end);
            } else {
                const uint64_t win = end > beg ? sb_pair(t.sbr, wbase >> 5, end > wbase + 32) : 0ull;
                for (int it = 0; it < maxit; ++it) {
                    const int a0 = beg + it * VW * U;
                    acc += thin_bwd_step<U>(t, a0 + sub, end, VW, win, wbase);
                }
            }
        }
#pragma unroll
        for (int o = VW / 2; o > 0; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
        if (sub == 0 && thin) {
            if (FWD) {
                if (L > 0) {
                    t.sig[v] = acc;
                    if (acc >= TWO53) c.inexact = 1;
                }
            } else {
                finish_dependency(p, sw, t.sig, v, acc);
            }
        }
    }
    // wide rows (degree > THIN_MAX): one warp per row, 32 U arcs in flight
    if (__syncthreads_or(sm.nbig > 0)) {
        const int nb = sm.nbig;
        for (int r = wid; r < nb; r += NW) {
            const int v = __ldcg(&bigq[r]);
            const int b = t.ro[v], e = t.ro[v + 1];
            double acc = 0.0, sw = 0.0;
            if (lane == 0) {
                c.scanned += e - b;
                if (FWD) c.arcs_reached += e - b;
            }
            if (!FWD) sw = __ldcg(&t.sig[v]);
            for (int a0 = b; a0 < e; a0 += 32 * U) {
                if (FWD) {
                    unsigned sm_[U];
                    thin_fwd_step<U>(t, a0 + lane, e, 32, acc, dag, sm_);
                    if (bits && lane == 0) {
#pragma unroll
                        for (int j = 0; j < U; ++j) {
                            const int A = a0 + 32 * j, sh = A & 31;
                            const unsigned m = sm_[j];
                            red_or_global_if(&t.sb[A >> 5], m << sh, m != 0u);
                            red_or_global_if(&t.sb[(A >> 5) + 1], sh ? m >> (32 - sh) : 0u, sh != 0 && (m >> (32 - sh)) != 0u);
                        }
                    }
                } else {
                    // successor bits of this lane's arcs a0 + lane + 32 j
#pragma unroll
                    for (int j = 0; j < U; ++j) {
                        const int a = a0 + lane + 32 * j;
                        const bool s = a < e && ((__ldcg(&t.sbr[a >> 5]) >> (a & 31)) & 1u);
                        const int u = s ? ld_col(t.col + a) : 0;
                        acc += ldca_if(t.sig + u, s);
                    }
                }
            }
            acc = warp_sum(acc);
            if (lane == 0) {
                if (FWD) {
                    if (L > 0) {
                        t.sig[v] = acc;
                        if (acc >= TWO53) c.inexact = 1;
                    }
                } else {
                    finish_dependency(p, sw, t.sig, v, acc);
                }
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) sm.nbig = 0;
    }
    if (FWD) c.dag += dag;
    __syncthreads();
}

}  // namespace bcdev
