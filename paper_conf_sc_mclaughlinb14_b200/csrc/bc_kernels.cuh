// bc_kernels.cuh -- sm_100a device code for per-source Brandes BC.
//
// One CTA owns one source at a time ("coarse-grained" root parallelism, P:118,
// P:198) and loops: Alg. 1 init -> forward levels (Alg. 2) in WE or
// EP mode -> backward levels (Alg. 3) -> BC update (Eq. 3) ->
// reset of the touched state.  Sources are pulled from a global atomic counter,
// so the grid is persistent (one CTA per workspace slot).
//
// B200 choices:
//  * Level state policy.  Undirected graphs whose 2-bit level codes fit in shared
//    memory keep d as a code per vertex in SMEM (0 = unvisited, 1 + L mod 3):
//    every neighbour of a level-L vertex lies on L-1, L or L+1, so the code
//    decides the predecessor / successor / unvisited tests exactly, and every
//    probe of Alg. 2 l.5/l.7 and Alg. 3 l.7 is a shared-memory load instead of a
//    random HBM sector.  Directed or large graphs keep exact int32 d in HBM.
//  * sigma is PULLED (sigma[w] = sum of sigma over w's level-(L-1) neighbours)
//    when w itself is expanded, fused with w's discovery scan: one CSR row read
//    serves both, no sigma atomics in WE mode, and rows of degree <= seq_max_deg
//    are summed by one thread in CSR order = the oracle's order (bit-exact).
//  * the queue is S itself: level L+1 is appended at S[ends[L+1]...] with a
//    warp-aggregated atomic, so Alg. 2's Q_next -> Q_curr copy disappears.
//  * rows of degree > seq_max_deg are expanded cooperatively (Merrill et al.'s
//    scan+warp+CTA gather): one warp per row up to warp_max_deg, the whole
//    CTA for longer rows, two arcs in flight per thread, one reduction per row.
//  * EP levels stream src[]/col[] with 16-byte vector loads and test frontier
//    membership in a shared-memory bitmap.
//  * backward uses omega[v] = (1 + delta[v]) / sigma[v], stored in place of
//    sigma[v]: one 8-byte gather per DAG arc, delta[w] = sigma[w] * sum(omega).
#pragma once

#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace bcdev {

constexpr int INF = 0x7F7F7F7F;  // "infinity" distance (memset-able byte pattern)
constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr double TWO53 = 9007199254740992.0;

enum : int { MODE_WE = 0, MODE_EP = 1 };
enum : int { LM_WE = 0, LM_EP = 1, LM_HYBRID = 2, LM_SAMPLED = 3 };

struct DevStats {
    unsigned long long sources, levels, we_levels, ep_levels;
    unsigned long long n_reached, arcs_reached, dag_arcs, arcs_scanned;
    unsigned long long phase_cycles[4];  // SM cycles (CTA thread 0): fwd WE, fwd EP, bwd WE, bwd EP
    int sigma_inexact;
    int sampling_ep;
    int sampling_median;
    int pad;
    unsigned long long batches, batch_overflows;  // multi-source engine (bc_batch.cu)
    unsigned long long dist_sum;  // sum over sources of sum_t d(s,t) over reached t (self-check)
    unsigned long long group_wait;  // group engine: CTA cycles waiting at group barriers
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
    const int *__restrict__ perm;     // caller id -> internal id (NULL: identity)
    long long src_base;
    long long k;                      // sources in this launch
    const long long *k_dev;           // non-NULL: k is read from device memory (batch overflows)
    int skip_if_ep;                   // 1: do nothing when Alg. 5 chose EP (batched / EP-capable kernel runs)
    int skip_if_we;                   // 1: do nothing when Alg. 5 chose WE (the WE-only kernel runs)
    int *fallback_src;                // fast WE-only kernel: sources whose selector picks an EP
    unsigned long long *fallback_n;   // level are abandoned and appended here (caller ids)
    unsigned long long *work_counter;
    // workspace (slot-major)
    int *d;                           // GlobalLevels only
    double *sigma;
    double *omega;
    int *S;
    int *ends;
    unsigned char *modes;
    int *bigq;           // rows queued for CTA-cooperative expansion (per slot)
    size_t stride_big;   // per-slot bigq entries: CTA rows from the front, medium rows from the back
    size_t stride_n;     // elements per slot for d/sigma/omega/S
    size_t stride_e;     // elements per slot for ends/modes
    double *bc;
    // shared-memory level codes (SmemCodes): 32-bit words of codes / of the EP bitmap
    int code_words;
    uint32_t *gcodes;    // GlobalCodes: per-slot code words / EP bitmap words in HBM
    uint32_t *gfb;
    size_t stride_codes, stride_fb;
    int fb_words;        // 0: this launch never runs an EP level
    uint32_t *nbits;     // per-slot bitmap of the level being discovered (sorted frontiers)
    size_t stride_nb;
    int nb_words;
    int sort_min;        // rebuild a level in vertex order when it has >= sort_min vertices
    uint32_t *sbits;     // per-slot successor bitmap over arcs (ArcBits), NULL = off
    size_t stride_sb;
    int sb_words;        // multiple of 4
    int seq_max_deg;     // rows up to this degree: owner thread, CSR order
    int medq;            // fast path: rows in (seq_max_deg, warp_max_deg] are queued and dealt to
                         // warps dynamically after the one-thread rows (graph has such rows)
    int warp_max_deg;    // rows up to this degree: one warp; longer: whole CTA
    int bpush;           // fast path backward: level L's dependencies are PUSHED from level L+1's
                         // rows (RED into omega-as-accumulator) when bpush * A_{L+1} < A_L
                         // (A = arcs of the level's rows); 0 = always pulled (Alg. 3)
    // strategy
    int launch_mode;
    const int *sampled_flag;  // LM_SAMPLED: 1 = EP run
    int alpha, beta, ep_min_frontier;
    int backward_we;
    int *keys;                // sampling phase: keys[idx] = max depth, for idx < nkeys
    long long nkeys;
    DevStats *stats;
    // debug export (single source), may be NULL
    int *dbg_d;
    double *dbg_sigma;
    double *dbg_delta;
    unsigned char *dbg_modes;
    int dbg_max_levels;
    int *dbg_nlevels;
    // per-level trace, may be NULL: frontier sizes and SM cycles
    int *dbg_lsizes;
    long long *dbg_fcyc;
    long long *dbg_bcyc;
};

// Per-thread counters for the byte model / stats, flushed into shared memory once
// per source (32-bit: at most a few rows' worth of arcs per thread per source).
struct Counters {
    unsigned arcs_reached = 0, dag = 0, scanned = 0;
    int inexact = 0;
};

// Per-CTA counters in shared memory (updated by thread 0 or by warp leaders).
struct CtaStats {
    unsigned long long src, reached, ar, dg, sc;
    unsigned long long lv[2];   // levels expanded WE / EP
    unsigned long long cyc[4];  // fwd WE, fwd EP, bwd WE, bwd EP
    unsigned long long dsum;    // sum of d(s,t) over the reached t of this CTA's sources
    unsigned long long gwait;   // group engine: cycles waiting at group barriers (thread 0)
    int inexact;
};

__device__ __forceinline__ void flush_counters(Counters &c, CtaStats &st) {
    unsigned long long ar = c.arcs_reached, dg = c.dag, sc = c.scanned;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        ar += __shfl_down_sync(0xFFFFFFFFu, ar, o);
        dg += __shfl_down_sync(0xFFFFFFFFu, dg, o);
        sc += __shfl_down_sync(0xFFFFFFFFu, sc, o);
    }
    const int inex = __any_sync(0xFFFFFFFFu, c.inexact);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&st.ar, ar);
        atomicAdd(&st.dg, dg);
        atomicAdd(&st.sc, sc);
        if (inex) st.inexact = 1;
    }
    c = Counters{};
}

constexpr int NLEV_ARCS = 64;  // levels whose arc counts the fast path keeps (deeper: pulled)

template <int NT>
struct Smem {
    long long idx;
    int cnt[3];           // level L appends at S[hi + cnt[L % 3]] (triple-buffered, see kernel)
    int nbig;             // rows queued for CTA-cooperative expansion in this tile
    int medc[2], medn[2]; // fast path: medium rows queued / grabbed, by pass parity
    int gw0, gwn;         // row_pass chunk distribution: this CTA's first warp index, warps
                          // sharing the pass (0 / NT/32, except in the group engine's backward)
    int goff;             // group engine: this CTA's offset in the level being compacted
    unsigned alev[NLEV_ARCS];  // fast path: arcs of the rows of forward level L (L < NLEV_ARCS)
    CtaStats st;
    double red[NT / 32];  // block reduction scratch
    int wtot[NT / 32];    // per-warp totals (frontier compaction)
    int big_v[NT];
    int big_beg[NT];
    int big_deg[NT];
};

// ------------------------------------------------------------ level policies

// Exact int32 distances in HBM (directed graphs, or graphs too large for SMEM codes).
struct GlobalLevels {
    static constexpr int UNVISITED = INF;
    static constexpr bool SPEC_GATHER = false;  // gathers wait for the probe (see GlobalCodes)
    static constexpr bool RESET_VERTICES = true;
    static constexpr bool BITMAP_DISCOVERY = false;
    __device__ __forceinline__ void mark(int, int) const {}
    __device__ __forceinline__ void level_fence() const {}
    int *d;
    uint32_t *fb;  // unused
    __device__ __forceinline__ int probe(int u) const { return __ldcg(&d[u]); }
    __device__ __forceinline__ static int key(int L) { return L; }  // L = -1: matches nothing
    __device__ __forceinline__ bool discover(int u, int L1) const {
        return atomicCAS(&d[u], INF, L1) == INF;
    }
    __device__ __forceinline__ bool in_frontier(int x, int L) const { return __ldcg(&d[x]) == L; }
    __device__ __forceinline__ void set_source(int s) const { d[s] = 0; }
    __device__ __forceinline__ void reset_vertex(int v) const { d[v] = INF; }
    template <int NT> __device__ __forceinline__ void reset_all(int) const {}
    template <int NT> __device__ __forceinline__ void prepare_frontier(const int *, int, int, int) const {}
};

// 2-bit level codes in HBM/L2, per slot, for undirected graphs too large for
// shared memory (n/4 bytes per source: 1 MB at n = 2^22, L2-resident for ~100
// sources in flight instead of 16 MB of int32 distances).  Same code semantics
// as SmemCodes; discoveries are global atomicOr.
struct GlobalCodes {
    static constexpr int UNVISITED = 0;
    // Speculative gathers (issued beside the probe, one round trip per arc quad instead of
    // two) were measured slower on B200 (c5ws 2491 -> 2983 ms, c5k group 2479 -> 3430 ms):
    // the extra sector requests cost more than the latency they hide.
    static constexpr bool SPEC_GATHER = false;
    static constexpr bool RESET_VERTICES = false;
    // Discovery without winner election: mark() is an idempotent OR (RED, no return)
    // and the level is rebuilt from the per-level bitmap (compact_level).
    static constexpr bool BITMAP_DISCOVERY = true;
    __device__ __forceinline__ void mark(int u, int L1) const {
        atomicOr(&w[u >> 4], (uint32_t)key(L1) << ((u & 15) << 1));
    }
    uint32_t *w;
    uint32_t *fb;
    // Probes go through L1 (neighbouring vertices share code words).  A stale L1
    // line can only hide discoveries made by atomics; level_fence() invalidates L1
    // (gpu-scope fence -> CCTL.IVALL) at every forward level start, so codes of
    // earlier levels are always current.  Within a level a stale "unvisited" only
    // costs a failed atomicOr (whose old value is authoritative); the backward
    // stage performs no discoveries.
    __device__ __forceinline__ int probe(int u) const {
        return (__ldca(&w[u >> 4]) >> ((u & 15) << 1)) & 3;
    }
    __device__ __forceinline__ void level_fence() const { __threadfence(); }
    __device__ __forceinline__ static int key(int L) { return L < 0 ? 4 : (L % 3) + 1; }
    __device__ __forceinline__ bool discover(int u, int L1) const {
        const uint32_t sh = (uint32_t)(u & 15) << 1;
        const uint32_t old = atomicOr(&w[u >> 4], (uint32_t)key(L1) << sh);
        return ((old >> sh) & 3u) == 0u;
    }
    __device__ __forceinline__ bool in_frontier(int x, int) const {
        return (__ldcg(&fb[x >> 5]) >> (x & 31)) & 1u;
    }
    __device__ __forceinline__ void set_source(int s) const {
        atomicOr(&w[s >> 4], (uint32_t)key(0) << ((s & 15) << 1));
    }
    __device__ __forceinline__ void reset_vertex(int) const {}
    template <int NT> __device__ __forceinline__ void reset_all(int words) const {
        uint4 *w4 = reinterpret_cast<uint4 *>(w);
        for (int i = threadIdx.x; i < (words >> 2); i += NT) w4[i] = make_uint4(0u, 0u, 0u, 0u);
    }
    template <int NT>
    __device__ __forceinline__ void prepare_frontier(const int *S, int lo, int hi, int words) const {
        for (int i = threadIdx.x; i < words; i += NT) fb[i] = 0u;
        __syncthreads();
        for (int i = lo + threadIdx.x; i < hi; i += NT) {
            const int v = S[i];
            atomicOr(&fb[v >> 5], 1u << (v & 31));
        }
        __syncthreads();
    }
};

// 2-bit level codes in shared memory, undirected graphs only (see header).
struct SmemCodes {
    static constexpr int UNVISITED = 0;
    static constexpr bool SPEC_GATHER = false;  // shared-memory probes are cheap
    static constexpr bool RESET_VERTICES = false;
    static constexpr bool BITMAP_DISCOVERY = false;
    __device__ __forceinline__ void mark(int, int) const {}
    __device__ __forceinline__ void level_fence() const {}
    uint32_t *w;   // codes, 16 vertices per word
    uint32_t *fb;  // EP frontier bitmap, 32 vertices per word
    __device__ __forceinline__ int probe(int u) const { return (w[u >> 4] >> ((u & 15) << 1)) & 3; }
    __device__ __forceinline__ static int key(int L) { return L < 0 ? 4 : (L % 3) + 1; }
    __device__ __forceinline__ bool discover(int u, int L1) const {
        const uint32_t sh = (uint32_t)(u & 15) << 1;
        const uint32_t old = atomicOr(&w[u >> 4], (uint32_t)key(L1) << sh);
        return ((old >> sh) & 3u) == 0u;
    }
    __device__ __forceinline__ bool in_frontier(int x, int) const { return (fb[x >> 5] >> (x & 31)) & 1u; }
    __device__ __forceinline__ void set_source(int s) const { w[s >> 4] |= (uint32_t)key(0) << ((s & 15) << 1); }
    __device__ __forceinline__ void reset_vertex(int) const {}
    template <int NT> __device__ __forceinline__ void reset_all(int words) const {
        uint4 *w4 = reinterpret_cast<uint4 *>(w);  // words is a multiple of 4 (host pads)
        for (int i = threadIdx.x; i < (words >> 2); i += NT) w4[i] = make_uint4(0u, 0u, 0u, 0u);
    }
    // Bitmap of S[lo, hi) (one EP level).  Ends with a barrier.
    template <int NT>
    __device__ __forceinline__ void prepare_frontier(const int *S, int lo, int hi, int words) const {
        for (int i = threadIdx.x; i < words; i += NT) fb[i] = 0u;
        __syncthreads();
        for (int i = lo + threadIdx.x; i < hi; i += NT) {
            const int v = S[i];
            atomicOr(&fb[v >> 5], 1u << (v & 31));
        }
        __syncthreads();
    }
};

// ------------------------------------------------------------------ helpers

// Append u to S (Q_next) with one shared atomic per group of converged lanes.
__device__ __forceinline__ void enqueue(int *S, int *s_len, int u) {
    const unsigned m = __activemask();
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(m) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(s_len, __popc(m));
    base = __shfl_sync(m, base, leader);
    S[base + __popc(m & ((1u << lane) - 1u))] = u;
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}


// Column loads of the CSR.  (An L2 evict-first / L1 no-allocate hint on them was measured
// slower on B200: c4 159 -> 178 ms per 4,096 sources, c5ws 1500 -> 1715, c5k 1956 -> 2212 ms
// per 2,048 -- neighbouring rows share L1 lines and concurrent sources share L2 lines.)
__device__ __forceinline__ int4 ld_col4(const int *p) { return *reinterpret_cast<const int4 *>(p); }
__device__ __forceinline__ int ld_col(const int *p) { return *p; }

#ifndef BC_UNROLL
#define BC_UNROLL 4
#endif

// Successor bitmap over the arcs of one source (one bit per CSR position): the
// O(m) boolean array of Jia et al., kept for SUCCESSORS.  mode 1 (forward,
// WE level L): bit a is set when col[a] is, or is about to become, a level-(L+1)
// vertex -- known exactly while the row is scanned (an unvisited neighbour of a
// level-L vertex can only be discovered at L+1).  mode 2 (backward level L): only
// arcs whose bit is set are visited, without a probe, and col is read only for
// them.  mode 0: not used (EP levels, option off).
struct ArcBits {
    uint32_t *sb = nullptr;
    int mode = 0;
    int knext = 0;  // code of level L+1
    int unv = 0;    // code of "unvisited"
};

// Arcs t, t+stride, ... of row [b, e) for `stride` cooperating threads (a warp or the
// CTA).  The loop trip count is uniform over the cooperating threads (ballots).
// Forward: col loads of step i+1 are issued before the gathers of step i are
// consumed; padding slots probe vertex 0 and add +0.0.
template <int U, class Probe, class Gather, class Claim, class Visit>
__device__ __forceinline__ double coop_sum(const int *__restrict__ cols, int b, int e, int t, int stride,
                                           const ArcBits &ab, Probe &probe, Gather &gather,
                                           Claim &claim, Visit &visit) {
    double acc = 0.0;
    const int lane = threadIdx.x & 31;
    if (ab.mode == 2) {
        for (int base = b; base < e; base += U * stride) {
            int u[U];
            bool ok[U];
            double g[U];
#pragma unroll
            for (int j = 0; j < U; ++j) {
                const int a = base + t + j * stride;
                ok[j] = a < e && ((__ldcg(&ab.sb[a >> 5]) >> (a & 31)) & 1u);
            }
#pragma unroll
            for (int j = 0; j < U; ++j) u[j] = ok[j] ? ld_col(cols + base + t + j * stride) : 0;
#pragma unroll
            for (int j = 0; j < U; ++j) g[j] = ok[j] ? gather(u[j], ab.knext) : 0.0;
#pragma unroll
            for (int j = 0; j < U; ++j) acc += g[j];
        }
        return acc;
    }
    int un[U];
#pragma unroll
    for (int j = 0; j < U; ++j) un[j] = b + t + j * stride < e ? ld_col(cols + b + t + j * stride) : 0;
    for (int base = b; base < e; base += U * stride) {
        int u[U], k[U];
        bool ok[U];
        double g[U];
#pragma unroll
        for (int j = 0; j < U; ++j) {
            u[j] = un[j];
            ok[j] = base + t + j * stride < e;
        }
        const int bn = base + U * stride;
        if (bn < e) {
#pragma unroll
            for (int j = 0; j < U; ++j) un[j] = bn + t + j * stride < e ? ld_col(cols + bn + t + j * stride) : 0;
        }
#pragma unroll
        for (int j = 0; j < U; ++j) k[j] = probe(u[j]);
#pragma unroll
        for (int j = 0; j < U; ++j) g[j] = ok[j] ? gather(u[j], k[j]) : 0.0;
        bool won[U];  // all discovery atomics are issued before any result is used
#pragma unroll
        for (int j = 0; j < U; ++j) won[j] = ok[j] && claim(u[j], k[j]);
#pragma unroll
        for (int j = 0; j < U; ++j)
            if (ok[j]) visit(u[j], k[j], won[j]);
        if (ab.mode == 1) {
#pragma unroll
            for (int j = 0; j < U; ++j) {
                const unsigned m = __ballot_sync(FULL, ok[j] && (k[j] == ab.unv || k[j] == ab.knext));
                if (lane == 0 && m) {  // the warp's 32 arcs are consecutive
                    const int A = base + j * stride + (t - lane);
                    const int sh = A & 31;
                    atomicOr(&ab.sb[A >> 5], m << sh);
                    if (sh) atomicOr(&ab.sb[(A >> 5) + 1], m >> (32 - sh));
                }
            }
        }
#pragma unroll
        for (int j = 0; j < U; ++j) acc += g[j];
    }
    return acc;
}

// One row owned by one thread, read as aligned 16-byte quads of col (one LDG.128
// per 4 arcs instead of four LDG.32 that each touch a different sector per lane).
// Slots outside [a, e) probe vertex 0 and add +0.0, so the sum keeps the CSR order
// (also in mode 2, which skips non-successor slots: they only ever added 0.0).
// cols must be 16-byte aligned with >= 3 ints of readable slack after the end.
template <class Probe, class Gather, class Claim, class Visit>
__device__ __forceinline__ double seq_row_bits(const int *__restrict__ cols, int a, int e, const ArcBits &ab,
                                          Probe &probe, Gather &gather, Claim &claim, Visit &visit) {
    double acc = 0.0;
    // Successor bits of the row through a 64-arc window of two bitmap words starting at
    // word w0: loaded once (mode 2) / OR-ed once (mode 1) per row of <= 32 arcs.
    int w0 = a >> 5;
    uint64_t win = 0;
    if (ab.mode == 2) {
        win = __ldcg(&ab.sb[w0]);
        if (e > (w0 + 1) * 32) win |= (uint64_t)__ldcg(&ab.sb[w0 + 1]) << 32;
    }
    for (int q = a & ~3; q < e; q += 4) {
        // in-row slots of this quad as a 4-bit mask
        unsigned valid = 0xFu;
        if (q < a) valid &= 0xFu << (a - q);
        if (q + 4 > e) valid &= 0xFu >> (q + 4 - e);
        int off = q - w0 * 32;
        if (off >= 64) {  // rows longer than the window (seq_max_deg > 32)
            if (ab.mode == 1) {
                if ((uint32_t)win) atomicOr(&ab.sb[w0], (uint32_t)win);
                if (win >> 32) atomicOr(&ab.sb[w0 + 1], (uint32_t)(win >> 32));
            }
            w0 += 2;
            off -= 64;
            win = 0;
            if (ab.mode == 2) {
                win = __ldcg(&ab.sb[w0]);
                if (e > (w0 + 1) * 32) win |= (uint64_t)__ldcg(&ab.sb[w0 + 1]) << 32;
            }
        }
        if (ab.mode == 2) {
            const unsigned bits = (unsigned)(win >> off) & valid;
            if (!bits) continue;
            const int4 c4 = ld_col4(cols + q);
            const int u[4] = {c4.x, c4.y, c4.z, c4.w};
            double g[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) g[j] = (bits >> j) & 1u ? gather(u[j], ab.knext) : 0.0;
#pragma unroll
            for (int j = 0; j < 4; ++j) acc += g[j];
            continue;
        }
        const int4 c4 = ld_col4(cols + q);
        int u[4] = {c4.x, c4.y, c4.z, c4.w}, k[4];
        bool ok[4];
        double g[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            ok[j] = (valid >> j) & 1u;
            u[j] = ok[j] ? u[j] : 0;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) k[j] = probe(u[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) g[j] = ok[j] ? gather(u[j], k[j]) : 0.0;
        bool won[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) won[j] = ok[j] && claim(u[j], k[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (ok[j]) visit(u[j], k[j], won[j]);
        if (ab.mode == 1) {
            unsigned bits = 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) bits |= (ok[j] && (k[j] == ab.unv || k[j] == ab.knext)) ? 1u << j : 0u;
            win |= (uint64_t)bits << off;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) acc += g[j];
    }
    if (ab.mode == 1) {
        if ((uint32_t)win) atomicOr(&ab.sb[w0], (uint32_t)win);
        if (win >> 32) atomicOr(&ab.sb[w0 + 1], (uint32_t)(win >> 32));
    }
    return acc;
}

// Mode-0 row (no successor bitmap), software-pipelined: the column quad of step i+1 is
// loaded while the probes / gathers / discoveries of step i are in flight.  Same slot
// order and +0.0 padding as seq_row_bits, so the sum is unchanged.
template <class Probe, class Gather, class Claim, class Visit>
__device__ __forceinline__ double seq_row(const int *__restrict__ cols, int a, int e, const ArcBits &ab,
                                          Probe &probe, Gather &gather, Claim &claim, Visit &visit) {
    if (ab.mode != 0) return seq_row_bits(cols, a, e, ab, probe, gather, claim, visit);
    double acc = 0.0;
    int q = a & ~3;
    if (q >= e) return acc;
    int4 nx = ld_col4(cols + q);
    for (; q < e; q += 4) {
        const int4 c4 = nx;
        if (q + 4 < e) nx = ld_col4(cols + q + 4);
        unsigned valid = 0xFu;
        if (q < a) valid &= 0xFu << (a - q);
        if (q + 4 > e) valid &= 0xFu >> (q + 4 - e);
        int u[4] = {c4.x, c4.y, c4.z, c4.w}, k[4];
        bool ok[4];
        double g[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            ok[j] = (valid >> j) & 1u;
            u[j] = ok[j] ? u[j] : 0;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) k[j] = probe(u[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) g[j] = ok[j] ? gather(u[j], k[j]) : 0.0;
        bool won[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) won[j] = ok[j] && claim(u[j], k[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (ok[j]) visit(u[j], k[j], won[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) acc += g[j];
    }
    return acc;
}

// Row pass over the vertices S[lo, hi) (Merrill et al.'s scan+warp+CTA gather,
// cited at P:196, with the per-vertex sum the pull needs): every row
// [rows[v], rows[v+1]) of `cols` is inspected; gather(u, probe(u)) is summed per
// row, visit(u, probe(u)) performs side effects (discovery), finish(v, sum, coop)
// is called once per vertex.  Rows of degree <= seq_max are summed by their owner
// thread in CSR order (the oracle's order); rows up to warp_max by one warp; longer
// rows are queued in bigq and expanded by the whole CTA after one barrier.  Warps
// take 32-vertex chunks independently, so there is no barrier per chunk.
template <int NT, class Probe, class Gather, class Claim, class Visit, class Pre, class Finish>
__device__ __forceinline__ void row_pass(const int *__restrict__ S, int lo, int hi,
                                         const int *__restrict__ rows,
                                         const int *__restrict__ cols, int seq_max, int warp_max,
                                         int *__restrict__ bigq, Smem<NT> &sm, Counters &c,
                                         const ArcBits &ab, Probe probe, Gather gather, Claim claim,
                                         Visit visit, Pre pre, Finish finish) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    // Phase A: each warp walks its own 32-vertex chunks; no CTA barrier.
    // (Pipelining the S / row-bound loads of the next chunks was measured neutral on B200:
    // c4 728 -> 725 ms, c3 270 -> 274 ms; not kept.)
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
        // (1) short rows: owner thread, CSR order; gathers issued before side effects
        if (v >= 0 && deg <= seq_max) {
            const double pv = pre(v);
            const double acc = seq_row(cols, beg, beg + deg, ab, probe, gather, claim, visit);
            finish(v, acc, false, pv);
        }
        // (2) medium rows: the lanes of this warp take their rows one at a time
        unsigned med = __ballot_sync(FULL, v >= 0 && deg > seq_max && deg <= warp_max);
        while (med) {
            const int leader = __ffs(med) - 1;
            med &= med - 1;
            const int w = __shfl_sync(FULL, v, leader);
            const int b = __shfl_sync(FULL, beg, leader);
            const int e = b + __shfl_sync(FULL, deg, leader);
            const double pv = pre(w);
            const double acc =
                warp_sum(coop_sum<BC_UNROLL>(cols, b, e, lane, 32, ab, probe, gather, claim, visit));
            if (lane == leader) finish(w, acc, true, pv);
        }
        // (3) long rows: queued for the CTA-cooperative phase B
        if (v >= 0 && deg > warp_max) bigq[atomicAdd(&sm.nbig, 1)] = v;
    }
    // Phase B: long rows, the whole CTA per row (block reduction of the partials).
    if (__syncthreads_or(sm.nbig > 0)) {
        const int nb = sm.nbig;
        for (int r = 0; r < nb; ++r) {
            const int v = __ldcg(&bigq[r]);
            const int b = rows[v], e = rows[v + 1];
            const double pv = pre(v);
            const double acc =
                warp_sum(coop_sum<BC_UNROLL>(cols, b, e, threadIdx.x, NT, ab, probe, gather, claim, visit));
            if (lane == 0) sm.red[wid] = acc;
            __syncthreads();
            if (threadIdx.x == 0) {
                double t = 0.0;
#pragma unroll
                for (int q = 0; q < NW; ++q) t += sm.red[q];
                finish(v, t, true, pv);
                if (r == nb - 1) sm.nbig = 0;  // before the barrier: the next pass may push
            }
            __syncthreads();
        }
    }
}


__device__ __forceinline__ int next_mode(const KParams &p, int mode, int run_ep, int q_curr,
                                         int q_next) {
    switch (p.launch_mode) {
    case LM_WE: return MODE_WE;
    case LM_EP: return MODE_EP;
    case LM_HYBRID: {  // Alg. 4
        const int change = q_next > q_curr ? q_next - q_curr : q_curr - q_next;
        if (change > p.alpha) return q_next > p.beta ? MODE_EP : MODE_WE;
        return mode;
    }
    default:  // LM_SAMPLED: Alg. 5 run mode with the P:301 guard
        return (run_ep && q_next >= p.ep_min_frontier) ? MODE_EP : MODE_WE;
    }
}

// Rewrite out[0 .. popcount(nb)) with the set bits of nb in ascending order and
// clear nb.  Each warp owns a contiguous range of words and reads it coalesced;
// one block scan of the warp totals.  Returns popcount(nb); ends with a barrier.
template <int NT>
__device__ __forceinline__ int compact_level(uint32_t *nb, int words, int *out, Smem<NT> &sm) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int per = ((words + NW - 1) / NW + 31) & ~31;  // words per warp, multiple of 32
    const int w0 = min(wid * per, words), w1 = min(w0 + per, words);
    int cnt = 0;
    for (int w = w0 + lane; w < w1; w += 32) cnt += __popc(__ldcg(&nb[w]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(FULL, cnt, o);
    if (lane == 0) sm.wtot[wid] = cnt;
    __syncthreads();
    int base = 0, total = 0;
    for (int q = 0; q < NW; ++q) {
        if (q < wid) base += sm.wtot[q];
        total += sm.wtot[q];
    }
    for (int w = w0; w < w1; w += 32) {
        const int wi = w + lane;
        uint32_t bits = wi < w1 ? __ldcg(&nb[wi]) : 0u;
        const int c = __popc(bits);
        int incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        int pos = base + incl - c;
        if (bits) {
            nb[wi] = 0u;
            while (bits) {
                const int b = __ffs(bits) - 1;
                out[pos++] = wi * 32 + b;
                bits &= bits - 1u;
            }
        }
        base += __shfl_sync(FULL, incl, 31);
    }
    __syncthreads();
    return total;
}

// ------------------------------------------------------------------ forward

// L1G: sigma / omega gathers through L1 (ld.ca) instead of L2 only (ld.cg).  Safe where
// every entry a level gathers was written by plain stores of this SM or before an L1
// invalidation (work-efficient-only kernels; the group engine's barriers): neighbouring
// lanes then share sectors of local neighbours and hub entries in L1.  EP-capable kernels
// keep ld.cg, since EP levels accumulate sigma with L2 atomics.
__device__ __forceinline__ double ld_sig(const double *a, bool l1) { return l1 ? __ldca(a) : __ldcg(a); }

template <bool DIR, int NT, class LV, bool L1G = false>
__device__ void forward_we(const KParams &p, const LV &lv, double *sigma, int *S, int *bigq,
                           uint32_t *nb, uint32_t *sb, int L, int lo, int hi, Smem<NT> &sm,
                           Counters &c) {
    const int L1 = L + 1;
    const int kprev = LV::key(L - 1);
    ArcBits ab;  // successor bits written during the discovery scan (mode 1)
    ab.sb = sb;
    ab.mode = sb ? 1 : 0;
    ab.knext = LV::key(L1);
    ab.unv = LV::UNVISITED;
    const ArcBits none_ab;
    auto probe = [&](int u) -> int { return lv.probe(u); };
    auto pull = [&](int u, int k) -> double {
        if (LV::SPEC_GATHER) {
            const double sv = ld_sig(&sigma[u], L1G);
            return k == kprev ? sv : 0.0;
        }
        return k == kprev ? ld_sig(&sigma[u], L1G) : 0.0;
    };
    auto claim = [&](int u, int k) -> bool {
        if (LV::BITMAP_DISCOVERY) {
            // no winner election: idempotent OR of the code and of the level bitmap
            // (fire-and-forget RED); the level is compacted from the bitmap afterwards
            if (k == LV::UNVISITED) {
                lv.mark(u, L1);
                atomicOr(&nb[u >> 5], 1u << (u & 31));
            }
            return false;
        }
        return k == LV::UNVISITED && lv.discover(u, L1);
    };
    auto noclaim = [&](int, int) -> bool { return false; };
    auto discover = [&](int u, int, bool won) {
        if (won) {
            enqueue(S + hi, &sm.cnt[L % 3], u);
            if (nb) atomicOr(&nb[u >> 5], 1u << (u & 31));  // RED: result unused
        }
    };
    auto fin = [&](int v, double acc, bool coop, double) {
        sigma[v] = acc;
        if (coop && acc >= TWO53) c.inexact = 1;
    };
    auto nopre = [&](int) -> double { return 0.0; };
    if (!DIR) {
        // fused: discovery of level L+1 and sigma pull for level L in one row scan
        auto visit = [&](int u, int k, bool won) {
            if (k == kprev) c.dag++;
            discover(u, k, won);
        };
        auto fin0 = [&](int v, double acc, bool coop, double) {
            if (L > 0) fin(v, acc, coop, 0.0);
        };
        const unsigned before = c.scanned;
        row_pass<NT>(S, lo, hi, p.ro, p.col, p.seq_max_deg, p.warp_max_deg, bigq, sm, c, ab, probe,
                     pull, claim, visit, nopre, fin0);
        c.arcs_reached += c.scanned - before;
    } else {
        auto none = [&](int, int) -> double { return 0.0; };
        auto fin1 = [&](int, double, bool, double) {};
        const unsigned before = c.scanned;
        row_pass<NT>(S, lo, hi, p.ro, p.col, p.seq_max_deg, p.warp_max_deg, bigq, sm, c, ab, probe,
                     none, claim, discover, nopre, fin1);
        c.arcs_reached += c.scanned - before;
        if (L > 0) {
            auto count = [&](int, int k, bool) {
                if (k == kprev) c.dag++;
            };
            row_pass<NT>(S, lo, hi, p.iro, p.icol, p.seq_max_deg, p.warp_max_deg, bigq, sm, c, none_ab,
                         probe, pull, noclaim, count, nopre, fin);
        }
    }
}

// Thread-per-arc scan of ALL arcs (a_src[i] -> a_dst[i]) restricted to sources in
// the current frontier (Jia et al. EP): 16-byte loads of src[], col[]
// loaded only when one of the four arcs starts in the frontier.
template <int NT, class LV, class Arc>
__device__ __forceinline__ void ep_scan(const int *__restrict__ a_src, const int *__restrict__ a_dst,
                                        int nnz, const LV &lv, int L, Arc arc) {
    const int n4 = nnz >> 2;
    const int4 *s4 = reinterpret_cast<const int4 *>(a_src);
    const int4 *d4 = reinterpret_cast<const int4 *>(a_dst);
    auto quad = [&](const int4 xs, int q) {
        const bool f0 = lv.in_frontier(xs.x, L), f1 = lv.in_frontier(xs.y, L);
        const bool f2 = lv.in_frontier(xs.z, L), f3 = lv.in_frontier(xs.w, L);
        if (f0 | f1 | f2 | f3) {
            const int4 ys = d4[q];
            if (f0) arc(xs.x, ys.x);
            if (f1) arc(xs.y, ys.y);
            if (f2) arc(xs.z, ys.z);
            if (f3) arc(xs.w, ys.w);
        }
    };
    const int4 none = make_int4(0, 0, 0, 0);
    for (int q = threadIdx.x; q < n4; q += 4 * NT) {  // four 16-byte src loads in flight
        const bool v1 = q + NT < n4, v2 = q + 2 * NT < n4, v3 = q + 3 * NT < n4;
        const int4 x0 = s4[q];
        const int4 x1 = v1 ? s4[q + NT] : none;
        const int4 x2 = v2 ? s4[q + 2 * NT] : none;
        const int4 x3 = v3 ? s4[q + 3 * NT] : none;
        quad(x0, q);
        if (v1) quad(x1, q + NT);
        if (v2) quad(x2, q + 2 * NT);
        if (v3) quad(x3, q + 3 * NT);
    }
    for (int a = (n4 << 2) + threadIdx.x; a < nnz; a += NT) {
        const int x = a_src[a];
        if (lv.in_frontier(x, L)) arc(x, a_dst[a]);
    }
}

template <bool DIR, int NT, class LV>
__device__ void forward_ep(const KParams &p, const LV &lv, double *sigma, int *S, int L, int lo,
                           int hi, Smem<NT> &sm, Counters &c) {
    const int L1 = L + 1;
    const int kprev = LV::key(L - 1);
    for (int i = lo + threadIdx.x; i < hi; i += NT) {
        const int v = S[i];
        c.arcs_reached += (unsigned long long)(p.ro[v + 1] - p.ro[v]);  // byte model
        if (L > 0) sigma[v] = 0.0;  // accumulated with atomics below
    }
    __syncthreads();
    lv.template prepare_frontier<NT>(S, lo, hi, p.fb_words);
    auto arc = [&](int x, int y) {
        const int k = lv.probe(y);
        if (k == LV::UNVISITED) {
            if (lv.discover(y, L1)) enqueue(S + hi, &sm.cnt[L % 3], y);
        } else if (!DIR && k == kprev) {
            atomicAdd(&sigma[x], __ldcg(&sigma[y]));  // result unused -> RED (no return trip)
            c.dag++;
        }
    };
    ep_scan<NT>(p.src, p.col, p.nnz, lv, L, arc);
    if (threadIdx.x == 0) sm.st.sc += (unsigned long long)p.nnz;
    if (DIR && L > 0) {
        auto arc_in = [&](int x, int y) {
            if (lv.probe(y) == kprev) {
                atomicAdd(&sigma[x], __ldcg(&sigma[y]));
                c.dag++;
            }
        };
        ep_scan<NT>(p.isrc, p.icol, p.nnz, lv, L, arc_in);
        if (threadIdx.x == 0) sm.st.sc += (unsigned long long)p.nnz;
    }
    __syncthreads();
    // atomic (order-dependent) sums that reached 2^53 may differ in the last bits
    for (int i = lo + threadIdx.x; i < hi; i += NT)
        if (__ldcg(&sigma[S[i]]) >= TWO53) c.inexact = 1;
    __syncthreads();  // every level function ends with a barrier
}

// ------------------------------------------------------------------ backward

// omega[w] = (1 + delta[w]) / sigma[w] is stored IN PLACE of sigma[w]: sigma[w]
// is only needed to finish w itself, and every gather of the backward stage
// reads a vertex one level deeper, whose entry already holds omega.  One f64
// array per source instead of two (smaller working set in L2).
__device__ __forceinline__ void finish_dependency(const KParams &p, double sw, double *sig_om,
                                                  int w, double acc) {
    const double delta = sw * acc;                 // delta[w] = sum sw/sigma[v] (1+delta[v])
    sig_om[w] = (1.0 + delta) / sw;
    if (delta != 0.0) atomicAdd(&p.bc[w], delta);  // Eq. 3
    if (p.dbg_delta) p.dbg_delta[w] = delta;
}

template <int NT, class LV, bool L1G = false>
__device__ void backward_we(const KParams &p, const LV &lv, double *sig_om, const int *S, int *bigq,
                            uint32_t *sb, int L, int lo, int hi, Smem<NT> &sm, Counters &c) {
    const int knext = LV::key(L + 1);
    ArcBits ab;  // successors from the forward's bits (mode 2): no probe, col only for them
    ab.sb = sb;
    ab.mode = sb ? 2 : 0;
    ab.knext = knext;
    ab.unv = LV::UNVISITED;
    auto probe = [&](int v) -> int { return lv.probe(v); };
    auto gather = [&](int v, int k) -> double {
        if (LV::SPEC_GATHER && !sb) {
            const double ov = ld_sig(&sig_om[v], L1G);
            return k == knext ? ov : 0.0;
        }
        return k == knext ? ld_sig(&sig_om[v], L1G) : 0.0;
    };
    auto noclaim = [&](int, int) -> bool { return false; };
    auto none = [&](int, int, bool) {};
    auto pre = [&](int w) -> double { return __ldcg(&sig_om[w]); };  // sigma[w], issued early
    auto fin = [&](int w, double acc, bool, double sw) { finish_dependency(p, sw, sig_om, w, acc); };
    row_pass<NT>(S, lo, hi, p.ro, p.col, p.seq_max_deg, p.warp_max_deg, bigq, sm, c, ab, probe, gather,
                 noclaim, none, pre, fin);
}

template <int NT, class LV>
__device__ void backward_ep(const KParams &p, const LV &lv, double *sig_om, double *acc_ep,
                            const int *S, int L, int lo, int hi, Smem<NT> &sm, Counters &c) {
    const int knext = LV::key(L + 1);
    for (int i = lo + threadIdx.x; i < hi; i += NT) acc_ep[S[i]] = 0.0;  // atomic accumulators
    __syncthreads();
    lv.template prepare_frontier<NT>(S, lo, hi, p.fb_words);
    auto arc = [&](int x, int y) {
        if (lv.probe(y) == knext) atomicAdd(&acc_ep[x], __ldcg(&sig_om[y]));
    };
    ep_scan<NT>(p.src, p.col, p.nnz, lv, L, arc);
    if (threadIdx.x == 0) sm.st.sc += (unsigned long long)p.nnz;
    __syncthreads();
    for (int i = lo + threadIdx.x; i < hi; i += NT) {
        const int w = S[i];
        finish_dependency(p, __ldcg(&sig_om[w]), sig_om, w, __ldcg(&acc_ep[w]));
    }
    __syncthreads();  // every level function ends with a barrier
}

// ------------------------------------------------------------------ kernel

}  // namespace bcdev
#include "bc_fast.cuh"
namespace bcdev {

template <class LV> __device__ __forceinline__ LV make_levels(const KParams &p, size_t slot, uint32_t *dyn);
template <> __device__ __forceinline__ GlobalLevels make_levels<GlobalLevels>(const KParams &p, size_t slot,
                                                                              uint32_t *) {
    GlobalLevels lv;
    lv.d = p.d + slot * p.stride_n;
    lv.fb = nullptr;
    return lv;
}
template <> __device__ __forceinline__ SmemCodes make_levels<SmemCodes>(const KParams &p, size_t,
                                                                        uint32_t *dyn) {
    SmemCodes lv;
    lv.w = dyn;
    lv.fb = dyn + p.code_words;
    return lv;
}
template <> __device__ __forceinline__ GlobalCodes make_levels<GlobalCodes>(const KParams &p, size_t slot,
                                                                            uint32_t *) {
    GlobalCodes lv;
    lv.w = p.gcodes + slot * p.stride_codes;
    lv.fb = p.gfb + slot * p.stride_fb;
    return lv;
}

// EPOK = false instantiates a work-efficient-only kernel (no EP code, fewer
// registers) for launches that never run an EP level.  SB = false compiles the
// successor bitmap out (it costs registers even when p.sbits is NULL).
template <bool DIR, class LV, int NT, bool EPOK, bool SB>
#ifndef BC_MINB512
#define BC_MINB512 2
#endif
__global__ void __launch_bounds__(NT, NT >= 1024 ? 1 : (NT == 512 ? BC_MINB512 : (NT == 256 ? 4 : (NT == 128 ? 8 : 16))))
bc_kernel(KParams p) {
    __shared__ Smem<NT> sm;
    extern __shared__ __align__(16) uint32_t dyn_smem[];
    const size_t slot = blockIdx.x;
    const LV lv = make_levels<LV>(p, slot, dyn_smem);
    double *sigma = p.sigma + slot * p.stride_n;
    // opaque from here on: the slot's base stays in two registers instead of being
    // rematerialised (constant-bank load + 64-bit multiply-add) at every gather
    asm volatile("" : "+l"(sigma));
    double *omega = p.omega + slot * p.stride_n;
    int *S = p.S + slot * p.stride_n;
    int *ends = p.ends + slot * p.stride_e;
    unsigned char *modes = p.modes + slot * p.stride_e;
    int *bigq = p.bigq + slot * p.stride_big;
    uint32_t *nb = p.nbits ? p.nbits + slot * p.stride_nb : nullptr;
    uint32_t *sb = SB && p.sbits ? p.sbits + slot * p.stride_sb : nullptr;
    // Fast path (bc_fast.cuh): undirected graphs, shared-memory codes, WE-only kernels.
    // (Also running the EP-capable kernels' WE levels through it was measured slower on B200:
    // c4 hybrid 234 -> 348 ms.)
#ifdef BC_NO_FAST
    constexpr bool FAST = false;
#else
    constexpr bool FAST = !DIR && !SB && !EPOK && std::is_same<LV, SmemCodes>::value;
#endif

    Counters c;
    const int run_ep = (p.launch_mode == LM_SAMPLED && p.sampled_flag) ? *p.sampled_flag : 0;
    if (p.skip_if_ep && run_ep) return;  // uniform over the grid
    if (p.skip_if_we && !run_ep) return;
    const long long K = p.k_dev ? *p.k_dev : p.k;
    lv.template reset_all<NT>(p.code_words);
    if (threadIdx.x == 0) {
        sm.nbig = 0;
        sm.st = CtaStats{};
        sm.gw0 = 0;
        sm.gwn = NT / 32;
        sm.medc[0] = sm.medc[1] = sm.medn[0] = sm.medn[1] = 0;
    }
    int fpass = 0;  // fast-path passes so far (medium-queue counters alternate by parity)

    for (;;) {
        if (threadIdx.x == 0) sm.idx = (long long)atomicAdd(p.work_counter, 1ULL);
        __syncthreads();
        const long long idx = sm.idx;
        if (idx >= K) break;
        int s = p.sources ? p.sources[p.src_base + idx] : (int)(p.src_base + idx);
        const int s_caller = s;
        if (p.perm) s = p.perm[s];  // caller's id -> internal id
        // per-source statistics (thread 0), rolled back if the source is handed over
        const unsigned long long sv_lv = sm.st.lv[0], sv_cyc = sm.st.cyc[0], sv_dsum = sm.st.dsum;
        bool handed_over = false;
        // Alg. 1; all other entries are already unvisited / zero.
        if (threadIdx.x == 0) {
            lv.set_source(s);
            sigma[s] = 1.0;
            S[0] = s;
            ends[0] = 0;
            ends[1] = 1;
            sm.cnt[0] = sm.cnt[1] = sm.cnt[2] = 0;
        }
        if (FAST && threadIdx.x < NLEV_ARCS) sm.alev[threadIdx.x] = 0u;
        __syncthreads();

        int L = 0, lo = 0, hi = 1;
        int mode = p.launch_mode == LM_HYBRID ? MODE_WE  // Alg. 4 starts WE
                                              : next_mode(p, MODE_WE, run_ep, 0, 1);
        for (;;) {
            const long long t0 = clock64();
            lv.level_fence();
            // mark discoveries in the bitmap only when the next level is likely to be
            // large enough to be rebuilt (levels grow/shrink gradually)
            uint32_t *const nbl =
                LV::BITMAP_DISCOVERY ? nb
                                     : ((nb && (long long)(hi - lo) * 4 >= p.sort_min) ? nb : nullptr);
            if constexpr (FAST) {
                FastLevel f;
                f.sw = dyn_smem;
                f.gnb = nbl;
                f.sb = nullptr;
                f.sig = sigma;
                f.Snext = S + hi;
                f.cnt = &sm.cnt[L % 3];
                f.kmatch = LV::key(L - 1);
                f.knew = LV::key(L + 1);
                const unsigned before = c.scanned;
                fast_pass<NT, false, true>(p, f, S, lo, hi, L, bigq, sm, c, fpass++ & 1);
                c.arcs_reached += c.scanned - before;
            } else if (!EPOK || mode == MODE_WE) {
                forward_we<DIR, NT, LV, !EPOK>(p, lv, sigma, S, bigq, nbl, sb, L, lo, hi, sm, c);
            } else {
                forward_ep<DIR, NT>(p, lv, sigma, S, L, lo, hi, sm, c);
            }
            // (the level functions end with a barrier: every discovery is recorded)
            int nhi;
            if (FAST && nbl) {
                // fast path, large level: level L+1 = the bitmap, in vertex order
                nhi = hi + compact_level<NT>(nbl, p.nb_words, S + hi, sm);
            } else if (LV::BITMAP_DISCOVERY && mode == MODE_WE) {
                // level L+1 = the discovery bitmap, written to S in vertex order
                nhi = hi + compact_level<NT>(nb, p.nb_words, S + hi, sm);
            } else {
                nhi = hi + sm.cnt[L % 3];
                if (nbl && mode == MODE_WE && nhi > hi) {
                    // Level L+1 in vertex order (any order is a valid S, R14): consecutive
                    // threads then touch neighbouring rows, codes and sigma entries.
                    if (nhi - hi >= p.sort_min) {
                        compact_level<NT>(nb, p.nb_words, S + hi, sm);
                    } else {
                        for (int i = hi + threadIdx.x; i < nhi; i += NT) nb[S[i] >> 5] = 0u;
                        __syncthreads();
                    }
                }
            }
            if (threadIdx.x == 0) {
                modes[L] = (unsigned char)mode;
                ends[L + 2] = nhi;
                // cnt[(L+2)%3] was last used by level L-1 and read by every thread
                // before level L started; it is next used by level L+2.
                sm.cnt[(L + 2) % 3] = 0;
                const long long dt = clock64() - t0;
                sm.st.cyc[mode] += (unsigned long long)dt;
                if (p.dbg_fcyc && L < p.dbg_max_levels) p.dbg_fcyc[L] = dt;
                sm.st.lv[mode] += 1;
                sm.st.dsum += (unsigned long long)(L + 1) * (unsigned long long)(nhi - hi);
            }
            if (nhi == hi) break;  // Q_next_len == 0 (Alg. 2 l.11)
            mode = next_mode(p, mode, run_ep, hi - lo, nhi - hi);
            if (FAST && mode == MODE_EP && p.fallback_src) {
                // the selector asks for an EP level this WE-only kernel cannot run: hand the
                // source over to the EP-capable launch (uniform decision over the CTA)
                handed_over = true;
                break;
            }
            lo = hi;
            hi = nhi;
            ++L;
        }
        if (handed_over) {
            if (threadIdx.x == 0) {
                p.fallback_src[atomicAdd(p.fallback_n, 1ull)] = s_caller;
                sm.st.lv[0] = sv_lv;
                sm.st.cyc[0] = sv_cyc;
                sm.st.dsum = sv_dsum;
            }
            c = Counters{};
            lv.template reset_all<NT>(p.code_words);  // sigma needs no reset (written before read)
            __syncthreads();
            continue;
        }
        const int maxdepth = L;
        const int S_len = hi;
        if (p.keys && idx < p.nkeys && threadIdx.x == 0) p.keys[idx] = maxdepth;

        if (p.dbg_d) {  // debug export of d and sigma before omega overwrites sigma
            for (int l = 0; l <= maxdepth; ++l)
                for (int i = ends[l] + threadIdx.x; i < ends[l + 1]; i += NT) {
                    const int v = S[i];
                    p.dbg_d[v] = l;
                    p.dbg_sigma[v] = __ldcg(&sigma[v]);
                }
        }
        // Stage 2 (Alg. 3).  Deepest level: delta = 0, omega = 1/sigma (in place).
        if (maxdepth >= 1)
            for (int i = lo + threadIdx.x; i < hi; i += NT) {
                const int v = S[i];
                sigma[v] = 1.0 / __ldcg(&sigma[v]);
            }
        __syncthreads();
        for (int Lb = maxdepth - 1; Lb >= 1; --Lb) {
            const int blo = ends[Lb], bhi = ends[Lb + 1];
            const int bmode = p.backward_we ? MODE_WE : (int)modes[Lb];
            const long long t0 = clock64();
            // the forward's successor bits exist only if forward level Lb ran WE
            uint32_t *const sbl = (sb && (!EPOK || modes[Lb] == MODE_WE)) ? sb : nullptr;
            if constexpr (FAST) {
                if (p.bpush && Lb + 1 < NLEV_ARCS &&
                    (unsigned long long)p.bpush * sm.alev[Lb + 1] < (unsigned long long)sm.alev[Lb]) {
                    // level Lb+1's rows are the cheaper side: push its omega to the predecessors
                    push_level<NT>(p, dyn_smem, sigma, p.omega + slot * p.stride_n, S, blo, bhi, ends[Lb + 2],
                                   LV::key(Lb), c);
                } else {
                    FastLevel f;
                    f.sw = dyn_smem;
                    f.gnb = nullptr;
                    f.sb = nullptr;
                    f.sig = sigma;
                    f.Snext = nullptr;
                    f.cnt = nullptr;
                    f.kmatch = LV::key(Lb + 1);
                    f.knew = 0;
                    fast_pass<NT, false, false>(p, f, S, blo, bhi, Lb, bigq, sm, c, fpass++ & 1);
                }
            } else if (!EPOK || bmode == MODE_WE) {
                backward_we<NT, LV, !EPOK>(p, lv, sigma, S, bigq, sbl, Lb, blo, bhi, sm, c);
            } else {
                backward_ep<NT>(p, lv, sigma, omega, S, Lb, blo, bhi, sm, c);
            }
            if (threadIdx.x == 0) {
                const long long dt = clock64() - t0;
                sm.st.cyc[2 + bmode] += (unsigned long long)dt;
                if (p.dbg_bcyc && Lb < p.dbg_max_levels) p.dbg_bcyc[Lb] = dt;
            }
        }

        // Debug export, then reset of the touched state.
        if (p.dbg_d) {
            if (threadIdx.x == 0) {
                for (int l = 0; l <= maxdepth && l < p.dbg_max_levels; ++l) {
                    p.dbg_modes[l] = modes[l];
                    if (p.dbg_lsizes) p.dbg_lsizes[l] = ends[l + 1] - ends[l];
                }
                *p.dbg_nlevels = maxdepth + 1;
            }
            __syncthreads();
        }
        // sigma / omega need no reset: every entry is written before it is read
        // (pull writes sigma[w], finish overwrites it with omega; EP zeroes its
        // accumulators).
        if (LV::RESET_VERTICES)
            for (int i = threadIdx.x; i < S_len; i += NT) lv.reset_vertex(S[i]);
        lv.template reset_all<NT>(p.code_words);
        if (sb) {  // successor bits of this source
            uint4 *s4 = reinterpret_cast<uint4 *>(sb);
            for (int i = threadIdx.x; i < (p.sb_words >> 2); i += NT) s4[i] = make_uint4(0u, 0u, 0u, 0u);
        }
        flush_counters(c, sm.st);
        if (threadIdx.x == 0) {
            sm.st.src += 1;
            sm.st.reached += (unsigned long long)S_len;
        }
        __syncthreads();
    }

    if (threadIdx.x == 0) {
        DevStats *g = p.stats;
        atomicAdd(&g->sources, sm.st.src);
        atomicAdd(&g->levels, sm.st.lv[0] + sm.st.lv[1]);
        atomicAdd(&g->we_levels, sm.st.lv[0]);
        atomicAdd(&g->ep_levels, sm.st.lv[1]);
        atomicAdd(&g->n_reached, sm.st.reached);
        atomicAdd(&g->arcs_reached, sm.st.ar);
        atomicAdd(&g->dag_arcs, sm.st.dg);
        atomicAdd(&g->arcs_scanned, sm.st.sc);
#pragma unroll
        for (int q = 0; q < 4; ++q) atomicAdd(&g->phase_cycles[q], sm.st.cyc[q]);
        atomicAdd(&g->dist_sum, sm.st.dsum);
        if (sm.st.inexact) atomicOr(&g->sigma_inexact, 1);
    }
}

// Address of bc_kernel<DIR, LV, nt, epok, sb> (host side).  Each level store is
// instantiated in its own translation unit (bc_inst_*.cu) so the library builds in
// parallel; bc_api.cu reaches them through the kernel_* functions declared below.
template <bool DIR, class LV, int NT>
const void *kernel_nt(bool epok, bool sb) {
    return epok ? (sb ? (const void *)bc_kernel<DIR, LV, NT, true, true>
                      : (const void *)bc_kernel<DIR, LV, NT, true, false>)
                : (sb ? (const void *)bc_kernel<DIR, LV, NT, false, true>
                      : (const void *)bc_kernel<DIR, LV, NT, false, false>);
}
template <bool DIR, class LV>
const void *kernel_table(int nt, bool epok, bool sb) {
    return nt == 1024  ? kernel_nt<DIR, LV, 1024>(epok, sb)
           : nt == 512 ? kernel_nt<DIR, LV, 512>(epok, sb)
           : nt == 128 ? kernel_nt<DIR, LV, 128>(epok, sb)
                       : kernel_nt<DIR, LV, 256>(epok, sb);
}
const void *kernel_directed(int nt, bool epok, bool sb);       // GlobalLevels, DIR
const void *kernel_levels(int nt, bool epok, bool sb);         // GlobalLevels, undirected
const void *kernel_gcodes(int nt, bool epok, bool sb);         // GlobalCodes
const void *kernel_scodes(int nt, bool epok, bool sb);         // SmemCodes

#ifndef BC_INSTANCE_TU
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
                const int j = i ^ stride;
                if (j > i) {
                    const bool up = (i & size) == 0;
                    const int a = sk[i], b = sk[j];
                    if ((a > b) == up) { sk[i] = b; sk[j] = a; }
                }
            }
            __syncthreads();
        }
    }
    if (threadIdx.x == 0) {
        const int med = sk[nk / 2];
        const int ep = (double)med < thresh ? 1 : 0;
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
            const int mid = (lo + hi + 1) >> 1;
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

// out[v] = f * bc_internal[perm[v]]: back to the caller's vertex ids (and halving).
__global__ void unpermute_kernel(const double *__restrict__ bc_int, const int *__restrict__ perm,
                                 int n, double f, double *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        out[i] = f * bc_int[perm[i]];
}

#endif  // BC_INSTANCE_TU

}  // namespace bcdev
