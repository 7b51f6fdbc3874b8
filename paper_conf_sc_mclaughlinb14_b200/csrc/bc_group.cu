// bc_group.cu -- the group engine (design in bc_group.cuh).
//
// One cooperative persistent kernel.  The grid is cut into G groups of C CTAs; each group
// pulls sources from the global counter and runs Alg. 1-3 for one source at a
// time with all its CTAs, meeting at a group barrier (a counter in global memory) once per
// level.  The level code (forward_we / backward_we / row_pass) is bc_kernel's.
#define BC_INSTANCE_TU
#include "bc_kernels.cuh"
#include "bc_group.cuh"
#include "bc_thin.cuh"

namespace bcgroup {

using namespace bcdev;

__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Barrier of the C CTAs of one group (monotone counter, one arrival per CTA).  The fence
// before the arrival publishes the CTA's writes; the acquire load / fence after it
// invalidate this SM's L1 (CCTL.IVALL), so plain loads after the barrier see every write
// made before it.
// `wait` (thread 0) accumulates the cycles from this CTA's arrival to the release.
__device__ __forceinline__ void group_sync(unsigned long long *bar, unsigned long long &target, int C,
                                           unsigned long long *wait) {
    __syncthreads();
    if (threadIdx.x == 0) {
        const long long t0 = clock64();
        target += (unsigned long long)C;
        __threadfence();
        atomicAdd(bar, 1ull);
        while (ld_acquire(bar) < target) {
        }
        __threadfence();
        *wait += (unsigned long long)(clock64() - t0);
    }
    __syncthreads();
}

// Bits of the discovery bitmap `nb` owned by CTA r of C, as a list of items: item i < H
// (H = min(C, words) "hub" words) is word i restricted to the vertices v = 32 i + j with
// v mod C == r; the words after the hub words are dealt out in blocks of OB words, block
// b to CTA b mod C; item H + k is word k mod OB of this CTA's (k / OB)-th block.  Items
// are in ascending vertex order.  OB = GParams::own_block: 32 words (1,024 vertices) keeps
// neighbouring ids -- the local neighbours of spatial / ring-ordered graphs -- with one
// CTA and its L1 (c5ws 1604 -> 1547 ms); 1 word on degree-relabelled graphs, whose
// consecutive ids have similar degrees (c5k: 32 words 2479 -> 2629 ms).
// Levels whose per-CTA share is remembered for the backward (deeper levels -- only on
// graphs of diameter > RCAP -- are cut in 32-vertex chunks over the whole group).
constexpr int RCAP = 1024;
struct Owned {
    const uint32_t *nb;
    int words, r, C, OB, H, items;
    __device__ __forceinline__ Owned(const uint32_t *nb_, int words_, int r_, int C_, int ob_)
        : nb(nb_), words(words_), r(r_), C(C_), OB(ob_) {
        H = min(C, words);
        const int T = words - H, nbk = T / OB, rem = T % OB;
        const int full = nbk > r ? (nbk - 1 - r) / C + 1 : 0;        // whole blocks owned
        const int part = (rem > 0 && nbk % C == r) ? rem : 0;          // the ragged last block
        items = H + full * OB + part;
    }
    __device__ __forceinline__ int word(int i) const {
        if (i < H) return i;
        const int k = i - H;
        return H + (r + (k / OB) * C) * OB + (k % OB);
    }
    __device__ __forceinline__ uint32_t bits(int i) const {
        if (i >= items) return 0u;
        if (i >= H) return __ldcg(&nb[word(i)]);  // (word order = item order)
        uint32_t m = 0u;
        int j = (int)(((long long)r - 32LL * i) % C);
        if (j < 0) j += C;
        for (; j < 32; j += C) m |= 1u << j;
        return __ldcg(&nb[i]) & m;
    }
};

// Compact the owned bits of `nb` into out[off ...] in ascending vertex order, where off is
// reserved with one atomicAdd on *ctr; clears the owned whole words (hub words are cleared
// later by rank 0, once every CTA has read them).  Returns this CTA's count; sets off.
template <int NT>
__device__ __forceinline__ int group_compact(uint32_t *nb, int words, int r, int C, int ob, int *out,
                                             int *ctr, Smem<NT> &sm, int &off) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const Owned ow(nb, words, r, C, ob);
    const int per = ((ow.items + NW - 1) / NW + 31) & ~31;  // items per warp, multiple of 32
    const int i0 = min(wid * per, ow.items), i1 = min(i0 + per, ow.items);
    int cnt = 0;
    for (int i = i0 + lane; i < i1; i += 32) cnt += __popc(ow.bits(i));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(FULL, cnt, o);
    if (lane == 0) sm.wtot[wid] = cnt;
    __syncthreads();
    int base = 0, total = 0;
    for (int q = 0; q < NW; ++q) {
        if (q < wid) base += sm.wtot[q];
        total += sm.wtot[q];
    }
    if (threadIdx.x == 0) sm.goff = total ? atomicAdd(ctr, total) : 0;
    __syncthreads();
    off = sm.goff;
    for (int i = i0; i < i1; i += 32) {
        const int ii = i + lane;
        uint32_t b = ii < i1 ? ow.bits(ii) : 0u;
        const int c = __popc(b);
        int incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        int pos = off + base + incl - c;
        if (b) {
            const int w = ow.word(ii);
            if (ii >= ow.H) nb[w] = 0u;
            while (b) {
                const int j = __ffs(b) - 1;
                out[pos++] = w * 32 + j;
                b &= b - 1u;
            }
        }
        base += __shfl_sync(FULL, incl, 31);
    }
    __syncthreads();
    return total;
}

// FASTG: work-efficient levels through the fast path (bc_fast.cuh, G = true) instead of the
// generic row_pass.  Measured per graph kind on B200: faster on the skewed,
// degree-relabelled Kronecker graph (c5k 2100 -> 2024 ms per 2,048 sources; 1954 with 18
// CTAs per group), slower on the unskewed small world (c5ws 1500 -> 1568 ms, the backward).
// MODE: GM_GENERIC (row_pass), GM_FAST (bc_fast.cuh), GM_THIN (bc_thin.cuh, virtual warps).
#ifndef BC_THIN_MINB
#define BC_THIN_MINB 2
#endif
template <int NT, int MODE>
__global__ void __launch_bounds__(NT, NT >= 1024 ? 1 : NT >= 512 ? (MODE == GM_THIN ? BC_THIN_MINB : 2) : 4)
group_kernel(KParams p, GParams gp) {
    constexpr bool FASTG = MODE == GM_FAST;
    constexpr bool THIN = MODE == GM_THIN;
    constexpr int NW = NT / 32;
    __shared__ Smem<NT> sm;
    __shared__ int2 s_reg[RCAP];  // this CTA's share of level L in S: (offset, count), L < RCAP
    const int T = gridDim.x, G = gp.groups;
    const int g = (int)((long long)blockIdx.x * G / T);
    const int b0 = (int)(((long long)g * T + G - 1) / G);
    const int b1 = (int)(((long long)(g + 1) * T + G - 1) / G);
    const int r = (int)blockIdx.x - b0, C = b1 - b0;
    const int tid = threadIdx.x;
    unsigned long long *ctl = gp.ctl + (size_t)g * CTL_WORDS;
    unsigned long long *bar = ctl;
    long long *next_idx = reinterpret_cast<long long *>(ctl + 8);
    int *lvl = reinterpret_cast<int *>(ctl + 16);  // level counts, ring of 4
    GlobalCodes lv;
    lv.w = p.gcodes + (size_t)g * p.stride_codes;
    lv.fb = nullptr;
    double *sigma = p.sigma + (size_t)g * p.stride_n;
    int *S = p.S + (size_t)g * p.stride_n;
    int *ends = p.ends + (size_t)g * p.stride_e;
    uint32_t *nbb = p.nbits + (size_t)g * p.stride_nb;  // 3 buffers of nb_words
    uint32_t *sb = p.sbits ? p.sbits + (size_t)g * p.stride_sb : nullptr;
    int *bigq = p.bigq + (size_t)blockIdx.x * p.stride_big;
    const int nbw = p.nb_words;
    unsigned long long target = 0;
    Counters c;
    if (tid == 0) {
        sm.nbig = 0;
        sm.st = CtaStats{};
        sm.gw0 = 0;
        sm.gwn = NW;
        sm.cnt[0] = sm.cnt[1] = sm.cnt[2] = 0;
        sm.medc[0] = sm.medc[1] = sm.medn[0] = sm.medn[1] = 0;
    }
    int fpass = 0;  // fast-path passes (medium-queue counters alternate by parity)
    // fast path (bc_fast.cuh, G = true): global codes, idempotent marks, successor bits
    auto mk = [&](uint32_t *gnb, int kmatch, int knew) {
        FastLevel f;
        f.sw = lv.w;
        f.gnb = gnb;
        f.sb = sb;
        f.sig = sigma;
        f.Snext = nullptr;
        f.cnt = nullptr;
        f.kmatch = kmatch;
        f.knew = knew;
        return f;
    };
    auto tl_ = [&](uint32_t *gnb, int kmatch, int knew) {
        ThinLevel t;
        t.ro = p.ro;
        t.col = p.col;
        t.sbr = sb;
        t.codes = lv.w;
        t.nb = gnb;
        t.sb = sb;
        t.sig = sigma;
        t.kmatch = kmatch;
        t.knew = knew;
        return t;
    };
    const long long K = p.k;
    if (r == 0 && tid == 0) *next_idx = (long long)atomicAdd(p.work_counter, 1ULL);
    group_sync(bar, target, C, &sm.st.gwait);

    for (;;) {
        const long long idx = *(volatile long long *)next_idx;
        if (idx >= K) break;
        int s = p.sources ? p.sources[p.src_base + idx] : (int)(p.src_base + idx);
        if (p.perm) s = p.perm[s];
        const long long tsrc = clock64();
        // Alg. 1 by rank 0; every other entry is already unvisited / zero.
        if (r == 0 && tid == 0) {
            lv.set_source(s);
            sigma[s] = 1.0;
            S[0] = s;
            ends[0] = 0;
            ends[1] = 1;
            lvl[0] = 1;
            lvl[1] = 0;
        }
        if constexpr (THIN) __syncthreads();  // Alg. 1 stores above, read by other lanes below
        int mylo = 0, mycnt = r == 0 ? 1 : 0;  // this CTA's vertices of level L: S[mylo, +mycnt)
        if (tid == 0) s_reg[0] = make_int2(mylo, mycnt);
        int prevlo = 0, prevcnt = 0;
        int startL = 0;                        // ends[L]
        int L = 0;
        long long tl = clock64();
        for (;;) {
            uint32_t *nbw_next = nbb + (size_t)((L + 1) % 3) * nbw;
            // (a) Alg. 2 over this CTA's share of level L (ends with a CTA barrier)
            if (mycnt > 0) {
                if constexpr (THIN) {
                    thin_pass<NT, true>(p, tl_(nbw_next, GlobalCodes::key(L - 1), GlobalCodes::key(L + 1)), S, mylo,
                                        mylo + mycnt, L, bigq, sm, c);
                } else if constexpr (!FASTG) {
                    forward_we<false, NT, GlobalCodes, true>(p, lv, sigma, S, bigq, nbw_next, sb, L, mylo,
                                                             mylo + mycnt, sm, c);
                } else {
                    const unsigned before = c.scanned;
                    fast_pass<NT, true, true>(p, mk(nbw_next, GlobalCodes::key(L - 1), GlobalCodes::key(L + 1)), S,
                                              mylo, mylo + mycnt, L, bigq, sm, c, fpass++ & 1);
                    c.arcs_reached += c.scanned - before;
                }
            }
            // (b) level L+1 is complete once every CTA got here
            group_sync(bar, target, C, &sm.st.gwait);
            const int tot = *(volatile int *)&lvl[L & 3];
            if (r == 0 && tid == 0 && p.dbg_fcyc && L > 0 && L - 1 < p.dbg_max_levels) {
                const long long now = clock64();
                p.dbg_fcyc[L - 1] = now - tl;
                tl = now;
            }
            if (tot == 0) break;  // level L is empty (Alg. 2 l.11): maxdepth = L - 1
            const int endL1 = startL + tot;
            if (r == 0) {
                if (tid == 0) {
                    ends[L + 1] = endL1;
                    sm.st.dsum += (unsigned long long)L * (unsigned long long)tot;  // level L
                    lvl[(L + 2) & 3] = 0;  // next used for level L+2, reserved after barrier L+1
                }
                // hub words of level L's bitmap: every CTA read them before barrier L
                uint32_t *old = nbb + (size_t)(L % 3) * nbw;
                for (int i = tid; i < min(C, nbw); i += NT) old[i] = 0u;
            }
            // (c) this CTA's part of level L+1, in vertex order, straight into S
            int off = 0;
            const int cnt = group_compact<NT>(nbw_next, nbw, r, C, gp.own_block, S + endL1, &lvl[(L + 1) & 3], sm, off);
            prevlo = mylo;
            prevcnt = mycnt;
            mylo = endL1 + off;
            mycnt = cnt;
            if (tid == 0 && L + 1 < RCAP) s_reg[L + 1] = make_int2(mylo, mycnt);
            startL = endL1;
            ++L;
        }
        const int maxdepth = L - 1;
        const int S_len = startL;
        const long long tfwd = clock64();
        if (p.keys && idx < p.nkeys && r == 0 && tid == 0) p.keys[idx] = maxdepth;
        if (p.dbg_d) {  // debug export of d and sigma before omega overwrites sigma
            for (int l = 0; l <= maxdepth; ++l) {
                const int lo = ends[l], hi = ends[l + 1];
                for (int i = lo + r * NT + tid; i < hi; i += C * NT) {
                    const int v = S[i];
                    p.dbg_d[v] = l;
                    p.dbg_sigma[v] = __ldcg(&sigma[v]);
                }
            }
            group_sync(bar, target, C, &sm.st.gwait);
        }
        // Stage 2 (Alg. 3).  Deepest level: delta = 0, omega = 1/sigma (in place), by owner.
        if (maxdepth >= 1) {
            for (int i = prevlo + tid; i < prevlo + prevcnt; i += NT) {
                const int v = S[i];
                sigma[v] = 1.0 / __ldcg(&sigma[v]);
            }
            group_sync(bar, target, C, &sm.st.gwait);
        }
        // Backward levels: each CTA finishes the vertices it expanded in the forward (same
        // ownership, same locality); levels >= RCAP in 32-vertex chunks over the group.
        for (int Lb = maxdepth - 1; Lb >= 1; --Lb) {
            const long long t0 = clock64();
            if (Lb < RCAP) {
                const int2 rg = s_reg[Lb];
                if constexpr (THIN) {
                    thin_pass<NT, false>(p, tl_(nullptr, GlobalCodes::key(Lb + 1), 0), S, rg.x, rg.x + rg.y, Lb, bigq,
                                         sm, c);
                } else if constexpr (!FASTG) {
                    backward_we<NT, GlobalCodes, true>(p, lv, sigma, S, bigq, sb, Lb, rg.x, rg.x + rg.y, sm, c);
                } else {
                    fast_pass<NT, true, false>(p, mk(nullptr, GlobalCodes::key(Lb + 1), 0), S, rg.x, rg.x + rg.y, Lb,
                                               bigq, sm, c, fpass++ & 1);
                }
            } else {
                if (tid == 0) {
                    sm.gw0 = r * NW;
                    sm.gwn = C * NW;
                }
                __syncthreads();
                if constexpr (THIN) {
                    thin_pass<NT, false>(p, tl_(nullptr, GlobalCodes::key(Lb + 1), 0), S, ends[Lb], ends[Lb + 1], Lb,
                                         bigq, sm, c);
                } else if constexpr (!FASTG) {
                    backward_we<NT, GlobalCodes, true>(p, lv, sigma, S, bigq, sb, Lb, ends[Lb], ends[Lb + 1], sm, c);
                } else {
                    fast_pass<NT, true, false>(p, mk(nullptr, GlobalCodes::key(Lb + 1), 0), S, ends[Lb], ends[Lb + 1],
                                               Lb, bigq, sm, c, fpass++ & 1);
                }
                __syncthreads();
                if (tid == 0) {
                    sm.gw0 = 0;
                    sm.gwn = NW;
                }
            }
            group_sync(bar, target, C, &sm.st.gwait);
            if (r == 0 && tid == 0 && p.dbg_bcyc && Lb < p.dbg_max_levels) p.dbg_bcyc[Lb] = clock64() - t0;
        }
        // Reset of this source's codes and successor bits (the bitmaps are clear already),
        // then the next source.
        {
            uint4 *w4 = reinterpret_cast<uint4 *>(lv.w);
            for (int i = r * NT + tid; i < (p.code_words >> 2); i += C * NT) w4[i] = make_uint4(0u, 0u, 0u, 0u);
            if (sb) {
                uint4 *s4 = reinterpret_cast<uint4 *>(sb);
                for (int i = r * NT + tid; i < (p.sb_words >> 2); i += C * NT) s4[i] = make_uint4(0u, 0u, 0u, 0u);
            }
        }
        flush_counters(c, sm.st);
        if (r == 0 && tid == 0) {
            if (p.dbg_d) {
                for (int l = 0; l <= maxdepth && l < p.dbg_max_levels; ++l) {
                    p.dbg_modes[l] = (unsigned char)MODE_WE;
                    if (p.dbg_lsizes) p.dbg_lsizes[l] = ends[l + 1] - ends[l];
                }
                *p.dbg_nlevels = maxdepth + 1;
            }
            const long long now = clock64();
            sm.st.cyc[0] += (unsigned long long)(tfwd - tsrc);
            sm.st.cyc[2] += (unsigned long long)(now - tfwd);
            sm.st.lv[0] += (unsigned long long)(maxdepth + 1);
            sm.st.src += 1;
            sm.st.reached += (unsigned long long)S_len;
            *next_idx = (long long)atomicAdd(p.work_counter, 1ULL);
        }
        group_sync(bar, target, C, &sm.st.gwait);
    }

    if (tid == 0) {
        DevStats *gs = p.stats;
        if (sm.st.src) {
            atomicAdd(&gs->sources, sm.st.src);
            atomicAdd(&gs->levels, sm.st.lv[0]);
            atomicAdd(&gs->we_levels, sm.st.lv[0]);
            atomicAdd(&gs->n_reached, sm.st.reached);
            atomicAdd(&gs->dist_sum, sm.st.dsum);
            atomicAdd(&gs->phase_cycles[0], sm.st.cyc[0]);
            atomicAdd(&gs->phase_cycles[2], sm.st.cyc[2]);
        }
        atomicAdd(&gs->group_wait, sm.st.gwait);
        atomicAdd(&gs->arcs_reached, sm.st.ar);
        atomicAdd(&gs->dag_arcs, sm.st.dg);
        atomicAdd(&gs->arcs_scanned, sm.st.sc);
        if (sm.st.inexact) atomicOr(&gs->sigma_inexact, 1);
    }
}

const void *group_kernel_fn(int nt, int mode) {
#if defined(BC_GROUP_1024) && BC_GROUP_1024
    if (nt == 1024) {  // tuning build only (BC_GROUP_NT=1024)
        if (mode == GM_FAST) return (const void *)group_kernel<1024, GM_FAST>;
        if (mode == GM_THIN) return (const void *)group_kernel<1024, GM_THIN>;
        return (const void *)group_kernel<1024, GM_GENERIC>;
    }
#endif
    if (mode == GM_FAST) return nt == 256 ? (const void *)group_kernel<256, GM_FAST> : (const void *)group_kernel<512, GM_FAST>;
    if (mode == GM_THIN) return nt == 256 ? (const void *)group_kernel<256, GM_THIN> : (const void *)group_kernel<512, GM_THIN>;
    return nt == 256 ? (const void *)group_kernel<256, GM_GENERIC> : (const void *)group_kernel<512, GM_GENERIC>;
}

}  // namespace bcgroup
