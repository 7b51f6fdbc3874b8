// bc_fast.cuh -- the work-efficient fast path for undirected graphs with 2-bit level codes:
//  * G = false: codes in shared memory, bc_kernel<false, SmemCodes, NT, false, false> (every
//    work-efficient launch on n <= ~2^18, i.e. c1..c4);
//  * G = true: codes in global memory (L1-cached reads), the group engine (bc_group.cu, c5),
//    with idempotent discovery marks and the successor bitmap over arcs.
//
// Same arithmetic, same order and same outputs as the generic row_pass / forward_we /
// backward_we (Alg. 2 l.3-8 as a pull; Alg. 3 l.5-9; Eq. 3),
// written for fewer issued instructions per arc (ncu r01: 2.07 warp instructions and ~56
// thread instructions per scanned arc, issue-bound at 61 %):
//  * the probe of a 2-bit code is one LDS + one funnel rotate (the rotate amount 2u mod 32
//    is taken from u << 1 by the hardware's mod-32 wrap) + one AND;
//  * sigma / omega gathers are PREDICATED loads (no select, no branch);
//  * one-thread rows run a warp-uniform quad loop (trip count = the chunk's longest row),
//    so claims are gated by one warp vote per quad and issued as predicated shared atomics
//    (a per-lane trip count with per-slot claims was measured 4 % slower on c4);
//  * discoveries are appended to S with one shared atomic per warp and arc slot (and marked
//    in the sorted-frontier bitmap when the level is likely to be large);
//  * DAG arcs are counted per quad from the gather predicates.
// One-thread rows still sum in CSR order (= the oracle's order, DESIGN R4).
#pragma once

namespace bcdev {

__device__ __forceinline__ int code_at(const uint32_t *sw, int u) {
    const uint32_t wd = sw[(unsigned)u >> 4];
    return (int)(__funnelshift_r(wd, wd, (unsigned)u << 1) & 3u);  // rotate by 2(u mod 16)
}

// v = c ? *p : 0.0, as a predicated ld.global.ca (L1-cached; see ld_sig).
__device__ __forceinline__ double ldca_if(const double *p, bool c) {
    double v;
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\tmov.f64 %0, 0d0000000000000000;\n\t"
        "@q ld.global.ca.f64 %0, [%1];\n\t}"
        : "=d"(v)
        : "l"(p), "r"((unsigned)c));
    return v;
}

// old word if c (atomic OR into shared memory), else 0.
__device__ __forceinline__ uint32_t atom_or_shared_if(uint32_t *addr, uint32_t val, bool c) {
    uint32_t old = 0u;
    const unsigned a = (unsigned)__cvta_generic_to_shared(addr);
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q atom.shared.or.b32 %0, [%1], %2;\n\t}"
        : "+r"(old)
        : "r"(a), "r"(val), "r"((unsigned)c)
        : "memory");
    return old;
}

// Per-level context of the fast path.
struct FastLevel {
    uint32_t *sw;      // 2-bit codes (shared memory if !G, global memory if G)
    uint32_t *gnb;     // non-null: discoveries go to this level bitmap ONLY (no S append); the
                       // kernel rebuilds level L+1 from it in vertex order (sorted frontiers)
    uint32_t *sb;      // G: successor bits over CSR positions (nullptr = off; Jia et al.'s O(m)
                       // boolean array): the forward marks the DAG successor arcs, the
                       // backward visits only them (no code probe, columns only for them)
    double *sig;       // sigma (forward) / sigma-then-omega (backward), this slot
    int *Snext;        // S + hi: where level L+1 is appended (queue mode)
    int *cnt;          // &sm.cnt[L % 3]
    int kmatch;        // forward: key(L-1) (predecessors); backward: key(L+1) (successors)
    int knew;          // forward: key(L+1), the code a discovery sets (as a 2-bit value)
};



template <bool G>
__device__ __forceinline__ int fcode(const FastLevel &f, int u) {
    if (!G) return code_at(f.sw, u);
    const uint32_t wd = __ldca(&f.sw[(unsigned)u >> 4]);  // L1: invalidated at every level start
    return (int)(__funnelshift_r(wd, wd, (unsigned)u << 1) & 3u);
}

__device__ __forceinline__ void red_or_global_if(uint32_t *addr, uint32_t val, bool c) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.global.or.b32 [%0], %1;\n\t}"
                 :
                 : "l"(addr), "r"(val), "r"((unsigned)c)
                 : "memory");
}

// Claims of up to four neighbours (forward only), warp-uniform call.
//  !G: predicated shared atomics on the code words; winners are marked in the level bitmap
//      (large levels: the kernel rebuilds level L+1 from it in vertex order) or appended to
//      S with ONE warp scan and ONE shared atomic for all four slots.
//   G: no winner election: every claimer ORs the code and the level bitmap (idempotent,
//      fire-and-forget); the group engine compacts level L+1 from the bitmap.
template <bool G>
__device__ __forceinline__ void fast_claims(const FastLevel &f, const int (&u)[4], const bool (&un)[4]) {
    if (G) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            red_or_global_if(&f.sw[(unsigned)u[j] >> 4], (uint32_t)f.knew << (((unsigned)u[j] << 1) & 30u), un[j]);
            red_or_global_if(&f.gnb[(unsigned)u[j] >> 5], 1u << (u[j] & 31), un[j]);
        }
        return;
    }
    bool won[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const unsigned sh = ((unsigned)u[j] << 1) & 30u;
        const uint32_t old = atom_or_shared_if(&f.sw[(unsigned)u[j] >> 4], (uint32_t)f.knew << sh, un[j]);
        won[j] = un[j] && ((old >> sh) & 3u) == 0u;
    }
    if (f.gnb) {
#pragma unroll
        for (int j = 0; j < 4; ++j) red_or_global_if(&f.gnb[(unsigned)u[j] >> 5], 1u << (u[j] & 31), won[j]);
        return;
    }
    const int lane = threadIdx.x & 31;
    const int cnt = (int)won[0] + (int)won[1] + (int)won[2] + (int)won[3];
    int incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    const int tot = __shfl_sync(FULL, incl, 31);
    if (tot == 0) return;
    int base = 0;
    if (lane == 31) base = atomicAdd(f.cnt, tot);
    base = __shfl_sync(FULL, base, 31) + incl - cnt;
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (won[j]) f.Snext[base++] = u[j];
}

// Successor-bit window of a one-thread row: bits of words w0, w0 + 1 (64 arcs).
__device__ __forceinline__ void sb_flush(uint32_t *sb, int w0, uint64_t win) {
    red_or_global_if(&sb[w0], (uint32_t)win, (uint32_t)win != 0u);
    red_or_global_if(&sb[w0 + 1], (uint32_t)(win >> 32), (win >> 32) != 0ull);
}
__device__ __forceinline__ uint64_t sb_window(const uint32_t *sb, int w0, int end, bool any) {
    uint64_t win = 0;
    if (any) {
        win = __ldcg(&sb[w0]);
        if (end > (w0 + 1) * 32) win |= (uint64_t)__ldcg(&sb[w0 + 1]) << 32;
    }
    return win;
}

// acc + g[0] + g[1] + g[2] + g[3] in CSR order.  (BC_TREE_ADD=1, a tuning build: as
// acc + ((g0 + g1) + (g2 + g3)), one dependent DADD per quad on the accumulator instead of
// four -- measured neutral on B200: c4 460.0 -> 460.5 ms, c2d 251.2 -> 254.1, c5k 1921 ->
// 1908; not kept, the CSR order stays.)
#ifndef BC_TREE_ADD
#define BC_TREE_ADD 0
#endif
__device__ __forceinline__ double add4(double acc, const double (&g)[4]) {
#if BC_TREE_ADD
    return acc + ((g[0] + g[1]) + (g[2] + g[3]));
#else
#pragma unroll
    for (int j = 0; j < 4; ++j) acc += g[j];
    return acc;
#endif
}

// Backward sum of one row [beg, end) over its successor arcs only, taken from the
// successor bitmap four at a time (find-first-set on a 64-arc window): the columns and
// omega gathers of up to four successors are issued together, so a row costs one window
// load + one column round trip + one gather round trip per four successors, whatever its
// length (the quad walk paid a loop trip per four arcs).  Sums in CSR order.
#ifndef BC_SUCC_EXTRACT
#define BC_SUCC_EXTRACT 1
#endif
__device__ __forceinline__ double succ_sum(const uint32_t *sb, const int *__restrict__ cols, const double *sig,
                                           int beg, int end) {
    double acc = 0.0;
    if (end <= beg) return acc;
    int base = (beg >> 5) << 5;  // window [base, base + 64)
    auto window = [&](int b) -> uint64_t {
        uint64_t w = __ldcg(&sb[b >> 5]);
        if (end > b + 32) w |= (uint64_t)__ldcg(&sb[(b >> 5) + 1]) << 32;
        if (end - b < 64) w &= (1ull << (end - b)) - 1ull;
        return w;
    };
    uint64_t win = window(base) & (~0ull << (beg - base));
    for (;;) {
        int a[4];
        bool ok[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            while (win == 0ull && base + 64 < end) {  // rows longer than the window
                base += 64;
                win = window(base);
            }
            ok[j] = win != 0ull;
            a[j] = base + (ok[j] ? __ffsll((long long)win) - 1 : 0);
            win &= win - 1ull;
        }
        if (!ok[0]) break;
        int u[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) u[j] = ok[j] ? ld_col(cols + a[j]) : 0;
        double g[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) g[j] = ldca_if(sig + u[j], ok[j]);
        acc = add4(acc, g);
        if (!ok[3]) break;
    }
    return acc;
}

// Quads of the one-thread rows of a 32-vertex chunk; lane = row [beg, end) (deg <= seq_max,
// deg = 0 for lanes without a row).  Warp-uniform trip count.  Returns the lane's sum of
// gathers in CSR order.
template <bool G, bool FWD>
__device__ __forceinline__ double fast_seq_rows(const FastLevel &f, const int *__restrict__ cols, int beg,
                                                int end, Counters &c) {
    const int q0 = beg & ~3;
    const int nq = end > beg ? ((end + 3) >> 2) - (beg >> 2) : 0;
    const int maxq = __reduce_max_sync(FULL, (unsigned)nq);
    double acc = 0.0;
    const bool bits = G && f.sb;
    if (bits && !FWD) {
        // backward: only the successor arcs the forward marked; no probe
        // (per-lane trip count: no warp collective in here, and a lane whose quads hold no
        // successor skips them)
        if (BC_SUCC_EXTRACT) return succ_sum(f.sb, cols, f.sig, beg, end);
        int w0 = beg >> 5;
        uint64_t win = sb_window(f.sb, w0, end, nq > 0);
        for (int q = 0; q < nq; ++q) {
            const int pos = q0 + 4 * q;
            int off = pos - 32 * w0;
            if (off >= 64) {
                w0 += 2;
                off -= 64;
                win = sb_window(f.sb, w0, end, true);
            }
            unsigned valid = 0xFu;
            if (pos < beg) valid &= 0xFu << (beg - pos);
            if (pos + 4 > end) valid &= 0xFu >> min(4, pos + 4 - end);
            const unsigned sbits = (unsigned)(win >> off) & valid;
            if (!sbits) continue;
            const int4 c4 = ld_col4(cols + pos);
            const int u[4] = {c4.x, c4.y, c4.z, c4.w};
            double g[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) g[j] = ldca_if(f.sig + u[j], (sbits >> j) & 1u);
            acc = add4(acc, g);
        }
        return acc;
    }
    int4 nx = make_int4(0, 0, 0, 0);
    if (nq > 0) nx = ld_col4(cols + q0);
    unsigned dag = 0;
    int w0 = beg >> 5;
    uint64_t win = 0;
    for (int q = 0; q < maxq; ++q) {
        const int pos = q0 + 4 * q;
        const int4 c4 = nx;
        if (q + 1 < nq) nx = ld_col4(cols + pos + 4);
        unsigned valid = q < nq ? 0xFu : 0u;
        if (pos < beg) valid &= 0xFu << (beg - pos);
        if (pos + 4 > end) valid &= 0xFu >> min(4, pos + 4 - end);
        // slots outside the row hold other rows' columns (or the zeroed slack after col[nnz-1]):
        // valid vertex ids, probed harmlessly and masked out of every predicate
        const int u[4] = {c4.x, c4.y, c4.z, c4.w};
        int k[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) k[j] = fcode<G>(f, u[j]);
        bool pg[4];
        double g[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            pg[j] = ((valid >> j) & 1u) && k[j] == f.kmatch;
            g[j] = ldca_if(f.sig + u[j], pg[j]);
        }
        if (FWD) {
            bool un[4];
            bool any = false;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                un[j] = ((valid >> j) & 1u) && k[j] == 0;
                any |= un[j];
            }
            if (__any_sync(FULL, any)) fast_claims<G>(f, u, un);
            dag += (unsigned)pg[0] + (unsigned)pg[1] + (unsigned)pg[2] + (unsigned)pg[3];
            if (bits) {  // successors: unvisited or already on level L+1
                int off = pos - 32 * w0;
                if (off >= 64) {
                    sb_flush(f.sb, w0, win);
                    w0 += 2;
                    off -= 64;
                    win = 0;
                }
                unsigned sm4 = 0;
#pragma unroll
                for (int j = 0; j < 4; ++j) sm4 |= (((valid >> j) & 1u) && (k[j] == 0 || k[j] == f.knew)) ? 1u << j : 0u;
                win |= (uint64_t)sm4 << off;
            }
        }
        acc = add4(acc, g);
    }
    if (FWD && bits) sb_flush(f.sb, w0, win);
    if (FWD) c.dag += dag;
    return acc;
}

// One row [b, e) expanded by `stride` cooperating threads (a warp or the CTA), thread t
// taking arcs t, t + stride, ... (four in flight).  Warp-uniform within each warp.  Returns
// the thread's partial sum (the caller reduces).
// (With codes in shared memory, successor bits for these rows were measured slower on B200:
// c4 161 -> 188 ms per 4,096 sources, the forward paying more than the backward saved; the
// group engine, whose probes are global loads, keeps them.)
template <bool G, bool FWD>
__device__ __forceinline__ double fast_coop_row(const FastLevel &f, const int *__restrict__ cols, int b, int e,
                                                int t, int stride, Counters &c) {
    double acc = 0.0;
    const int lane = threadIdx.x & 31;
    const bool bits = G && f.sb;
    if (bits && !FWD) {
        uint32_t wn[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int a = b + t + j * stride;
            wn[j] = a < e ? __ldcg(&f.sb[a >> 5]) : 0u;
        }
        for (int base = b; base < e; base += 4 * stride) {
            bool s[4];
            int a[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                a[j] = base + t + j * stride;
                s[j] = a[j] < e && ((wn[j] >> (a[j] & 31)) & 1u);
            }
            const int bn = base + 4 * stride;
            if (bn < e) {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int an = bn + t + j * stride;
                    wn[j] = an < e ? __ldcg(&f.sb[an >> 5]) : 0u;
                }
            }
            if (!__any_sync(FULL, s[0] | s[1] | s[2] | s[3])) continue;
            int u[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) u[j] = s[j] ? ld_col(cols + a[j]) : 0;
            double g[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) g[j] = ldca_if(f.sig + u[j], s[j]);
            acc = add4(acc, g);
        }
        return acc;
    }
    unsigned dag = 0;
    int un_[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) un_[j] = b + t + j * stride < e ? ld_col(cols + b + t + j * stride) : 0;
    // each step's gathers are added one step late, after the next step's gathers are issued
    // (same order of additions, so the same sums; B200: c4 160.3 -> 157.3 ms per 4,096
    // sources, c5k group 1960 -> 1947 ms per 2,048)
    double gp[4] = {0.0, 0.0, 0.0, 0.0};
    for (int base = b; base < e; base += 4 * stride) {
        int u[4];
        bool ok[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            u[j] = un_[j];
            ok[j] = base + t + j * stride < e;
        }
        const int bn = base + 4 * stride;
        if (bn < e) {
#pragma unroll
            for (int j = 0; j < 4; ++j) un_[j] = bn + t + j * stride < e ? ld_col(cols + bn + t + j * stride) : 0;
        }
        int k[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) k[j] = fcode<G>(f, u[j]);
        bool pg[4];
        double g[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            pg[j] = ok[j] && k[j] == f.kmatch;
            g[j] = ldca_if(f.sig + u[j], pg[j]);
        }
        if (FWD) {
            bool un[4];
            bool any = false;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                un[j] = ok[j] && k[j] == 0;
                any |= un[j];
            }
            if (__any_sync(FULL, any)) fast_claims<G>(f, u, un);
            dag += (unsigned)pg[0] + (unsigned)pg[1] + (unsigned)pg[2] + (unsigned)pg[3];
            if (bits) {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const unsigned m = __ballot_sync(FULL, ok[j] && (k[j] == 0 || k[j] == f.knew));
                    if (lane == 0 && m) {  // the warp's 32 arcs are consecutive
                        const int A = base + j * stride + (t - lane);
                        const int sh = A & 31;
                        atomicOr(&f.sb[A >> 5], m << sh);  // RED: result unused
                        if (sh) atomicOr(&f.sb[(A >> 5) + 1], m >> (32 - sh));
                    }
                }
            }
        }
        acc = add4(acc, gp);
#pragma unroll
        for (int j = 0; j < 4; ++j) gp[j] = g[j];
    }
    acc = add4(acc, gp);
    if (FWD) c.dag += dag;
    return acc;
}

template <bool G, bool FWD>
__device__ __forceinline__ void fast_medium_row(const KParams &p, const FastLevel &f, int w, int b, int e, int L,
                                                Counters &c) {
    const int lane = threadIdx.x & 31;
    double swm = 0.0;
    if (!FWD && lane == 0) swm = __ldcg(&f.sig[w]);
    const double a = warp_sum(fast_coop_row<G, FWD>(f, p.col, b, e, lane, 32, c));
    if (lane == 0) {
        if (FWD) {
            if (L > 0) {
                f.sig[w] = a;
                if (a >= TWO53) c.inexact = 1;
            }
        } else {
            finish_dependency(p, swm, f.sig, w, a);
        }
    }
}

// One forward (FWD) or backward level over S[lo, hi): phase A (warps take 32-vertex chunks --
// warp sm.gw0 + wid of sm.gwn sharing the pass -- and sum their one-thread rows, queueing the
// medium rows), phase M (medium rows dealt to warps dynamically; B200: c4 159.9 -> 154.5 ms
// per 4,096 sources; graphs without medium rows skip it), phase B (rows > warp_max, whole
// CTA).  Forward finish: sigma[v] = sum (L > 0).  Backward finish: finish_dependency (omega
// in place, bc += delta).  Ends with a CTA barrier (in phase B's test).
template <int NT, bool G, bool FWD>
__device__ __forceinline__ void fast_pass(const KParams &p, const FastLevel &f, const int *__restrict__ S, int lo,
                                          int hi, int L, int *bigq, Smem<NT> &sm, Counters &c, int par) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int *__restrict__ rows = p.ro;
    const int *__restrict__ cols = p.col;
    const int seq_max = p.seq_max_deg, warp_max = p.warp_max_deg;
    const int gstep = sm.gwn * 32;
    for (int base = lo + (sm.gw0 + wid) * 32; base < hi; base += gstep) {
        const int i = base + lane;
        int v = -1, beg = 0, deg = 0;
        if (i < hi) {
            v = S[i];
            beg = rows[v];
            deg = rows[v + 1] - beg;
        }
        c.scanned += deg;
        if (FWD && !G && p.bpush && L < NLEV_ARCS) {  // arcs of level L's rows (backward push choice)
            const unsigned a = __reduce_add_sync(FULL, (unsigned)deg);
            if (lane == 0 && a) atomicAdd(&sm.alev[L], a);
        }
        const bool seq = v >= 0 && deg <= seq_max;
        double sw = 0.0;
        if (!FWD && seq) sw = __ldcg(&f.sig[v]);  // sigma[w], issued early
        const double acc = fast_seq_rows<G, FWD>(f, cols, beg, seq ? beg + deg : beg, c);
        if (seq) {
            if (FWD) {
                if (L > 0) f.sig[v] = acc;
            } else {
                finish_dependency(p, sw, f.sig, v, acc);
            }
        }
        unsigned med = __ballot_sync(FULL, v >= 0 && deg > seq_max && deg <= warp_max);
        if (p.medq && med) {  // to the CTA's medium queue (back of bigq)
            int q = 0;
            if (lane == 0) q = atomicAdd(&sm.medc[par], __popc(med));
            q = __shfl_sync(FULL, q, 0);
            if ((med >> lane) & 1u) bigq[p.stride_big - 1 - (q + __popc(med & ((1u << lane) - 1u)))] = v;
            med = 0u;
        }
        while (med) {
            const int leader = __ffs(med) - 1;
            med &= med - 1;
            const int w = __shfl_sync(FULL, v, leader);
            const int b = __shfl_sync(FULL, beg, leader);
            const int e = b + __shfl_sync(FULL, deg, leader);
            double swm = 0.0;
            if (!FWD && lane == leader) swm = __ldcg(&f.sig[w]);
            const double a = warp_sum(fast_coop_row<G, FWD>(f, cols, b, e, lane, 32, c));
            if (lane == leader) {
                if (FWD) {
                    if (L > 0) {
                        f.sig[w] = a;
                        if (a >= TWO53) c.inexact = 1;
                    }
                } else {
                    finish_dependency(p, swm, f.sig, w, a);
                }
            }
        }
        if (v >= 0 && deg > warp_max) bigq[atomicAdd(&sm.nbig, 1)] = v;
    }
    if (p.medq) {
        __syncthreads();
        if (threadIdx.x == 0) sm.medc[par ^ 1] = sm.medn[par ^ 1] = 0;  // the other parity's pass is over
        const int nmed = sm.medc[par];
        for (;;) {
            int r = 0;
            if (lane == 0) r = atomicAdd(&sm.medn[par], 1);
            r = __shfl_sync(FULL, r, 0);
            if (r >= nmed) break;
            const int w = __ldcg(&bigq[p.stride_big - 1 - r]);
            fast_medium_row<G, FWD>(p, f, w, rows[w], rows[w + 1], L, c);
        }
    }
    if (__syncthreads_or(sm.nbig > 0)) {
        const int nb = sm.nbig;
        for (int r = 0; r < nb; ++r) {
            const int v = __ldcg(&bigq[r]);
            const int b = rows[v], e = rows[v + 1];
            double swb = 0.0;
            if (!FWD && threadIdx.x == 0) swb = __ldcg(&f.sig[v]);
            const double a = warp_sum(fast_coop_row<G, FWD>(f, cols, b, e, threadIdx.x, NT, c));
            if (lane == 0) sm.red[wid] = a;
            __syncthreads();
            if (threadIdx.x == 0) {
                double t = 0.0;
#pragma unroll
                for (int q = 0; q < NW; ++q) t += sm.red[q];
                if (FWD) {
                    if (L > 0) {
                        f.sig[v] = t;
                        if (t >= TWO53) c.inexact = 1;
                    }
                } else {
                    finish_dependency(p, swb, f.sig, v, t);
                }
                if (r == nb - 1) sm.nbig = 0;
            }
            __syncthreads();
        }
    }
}

__device__ __forceinline__ void red_add_f64_if(double *addr, double val, bool c) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.global.add.f64 [%0], %1;\n\t}"
                 :
                 : "l"(addr), "d"(val), "r"((unsigned)c)
                 : "memory");
}

// Backward level L finished by PUSHING (the dependency sum of Alg. 3 l.5-9, P:202-227,
// accumulated from the other side of each DAG arc, with atomics as the paper notes an
// edge-parallel backward needs): every level-(L+1) vertex w adds omega[w] to
// acc[v] of each predecessor v (code key(L), a shared-memory probe), then every level-L
// vertex finishes from acc: delta = sigma * acc, omega = (1 + delta) / sigma, bc += delta
// (Eq. 3).  Scans A_{L+1} arcs instead of A_L: on Kronecker graphs the big middle level's
// rows hold most arcs, the level below it few.  The sums are the same up to order (fp64
// atomics; checked at 1e-9).  S[lo, hi) = level L, S[hi, hi2) = level L+1.  Ends with a
// barrier.
// Pushes of the rows S[lo2, hi2) (level L+1) by warps gw0 + wid of gwn; codes in shared memory.
template <int NT>
__device__ __forceinline__ void push_rows(const KParams &p, const uint32_t *sw, const double *sig_om, double *acc,
                                          const int *__restrict__ S, int lo2, int hi2, int kpred, int gw0, int gwn,
                                          Counters &c) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int *__restrict__ rows = p.ro;
    const int *__restrict__ cols = p.col;
    auto code = [&](int u) -> int { return code_at(sw, u); };
    for (int base = lo2 + (gw0 + wid) * 32; base < hi2; base += gwn * 32) {
        const int i = base + lane;
        int v = -1, beg = 0, end = 0;
        double om = 0.0;
        if (i < hi2) {
            v = S[i];
            beg = rows[v];
            end = rows[v + 1];
            om = __ldcg(&sig_om[v]);  // omega[w] (level L+1 is finished)
        }
        c.scanned += end - beg;
        const bool one = end - beg <= 32;
        const int e1 = one ? end : beg;
        const int nq = (e1 - beg + 3) >> 2;
        const int maxq = (int)__reduce_max_sync(FULL, (unsigned)nq);
        for (int q = 0; q < maxq; ++q) {
            int u[4];
            bool ok[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int a = beg + 4 * q + j;
                ok[j] = a < e1;
                u[j] = ok[j] ? ld_col(cols + a) : 0;
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) red_add_f64_if(acc + u[j], om, ok[j] && code(u[j]) == kpred);
        }
        unsigned wide = __ballot_sync(FULL, v >= 0 && !one);
        while (wide) {  // longer rows: the whole warp, 32 arcs per step
            const int ld = __ffs(wide) - 1;
            wide &= wide - 1u;
            const int b = __shfl_sync(FULL, beg, ld), e = __shfl_sync(FULL, end, ld);
            const double w = __shfl_sync(FULL, om, ld);
            for (int a = b + lane; a < e; a += 32) {
                const int u = ld_col(cols + a);
                red_add_f64_if(acc + u, w, code(u) == kpred);
            }
        }
    }
}

// Finish of the level-L vertices S[lo, hi) from their pushed sums.
template <int NT>
__device__ __forceinline__ void finish_from_acc(const KParams &p, double *sig_om, double *acc,
                                                const int *__restrict__ S, int lo, int hi) {
    for (int i = lo + threadIdx.x; i < hi; i += NT) {
        const int v = S[i];
        const double a = __ldcg(&acc[v]);
        finish_dependency(p, __ldcg(&sig_om[v]), sig_om, v, a);
    }
}

template <int NT>
__device__ __forceinline__ void push_level(const KParams &p, const uint32_t *sw, double *sig_om, double *acc,
                                           const int *__restrict__ S, int lo, int hi, int hi2, int kpred,
                                           Counters &c) {
    // acc is the per-slot omega array, which EP levels of other launches leave dirty
    for (int i = lo + threadIdx.x; i < hi; i += NT) acc[S[i]] = 0.0;
    __syncthreads();
    push_rows<NT>(p, sw, sig_om, acc, S, hi, hi2, kpred, 0, NT / 32, c);
    __syncthreads();
    finish_from_acc<NT>(p, sig_om, acc, S, lo, hi);
    __syncthreads();
}

}  // namespace bcdev
