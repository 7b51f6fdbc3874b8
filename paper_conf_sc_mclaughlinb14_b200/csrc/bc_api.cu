// bc_api.cu -- host side of libbc.so: the C ABI declared in include/bc.h.
//
// Graph ingest, workspace sizing, the launch sequence of one
// bc_compute (sampling phase -> decision -> main phase -> halving, Alg. 5
// P:283-301), stats and errors.  All arithmetic of the method runs in the
// kernels of bc_kernels.cuh; this file only validates, copies and launches.
#include "bc.h"
#include "bc_kernels.cuh"
#include "bc_batch.cuh"
#include "bc_group.cuh"

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

using namespace bcdev;

namespace {

thread_local char g_err[512] = "";

int fail(int code, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return code;
}

#define CK(call)                                                                         \
    do {                                                                                 \
        cudaError_t e_ = (call);                                                         \
        if (e_ != cudaSuccess)                                                           \
            return fail(e_ == cudaErrorMemoryAllocation ? BC_ENOMEM : BC_ECUDA,          \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, \
                        __LINE__);                                                       \
    } while (0)

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

// The persisting-L2 carve-out (cudaLimitPersistingL2CacheSize) is device-global state
// shared by every handle on a device.  Handles register while they use a window; the
// limit only grows while any handle holds it, and is reset (persisting lines released,
// limit 0) when the last holder on the device lets go.
struct L2Share {
    int users = 0;
    size_t carve = 0;
};
std::mutex g_l2_mu;
L2Share g_l2[128];

cudaError_t l2_acquire(int dev, size_t carve, bool held) {
    std::lock_guard<std::mutex> lk(g_l2_mu);
    L2Share &sh = g_l2[dev & 127];
    if (!held) sh.users++;
    if (carve > sh.carve) {
        const cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, carve);
        if (e != cudaSuccess) {
            if (!held) sh.users--;
            return e;
        }
        sh.carve = carve;
    }
    return cudaSuccess;
}

void l2_release(int dev) {
    std::lock_guard<std::mutex> lk(g_l2_mu);
    L2Share &sh = g_l2[dev & 127];
    if (sh.users > 0 && --sh.users == 0) {
        cudaCtxResetPersistingL2Cache();
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
        sh.carve = 0;
    }
}

}  // namespace

struct bc_graph {
    int device = 0;
    int n = 0;
    int nnz = 0;
    int directed = 0;
    int num_sms = 0;
    // kernel configuration (see configure()): one without / one with the EP bitmap
    struct KCfg {
        const void *fn = nullptr;
        int nt = 256;
        size_t dyn = 0;   // dynamic shared memory bytes
        int per_sm = 1;   // resident CTAs per SM
    } cfg_we, cfg_ep;
    int lstore = 1;       // level store: 1 int32 d (HBM), 2 codes in SMEM, 3 codes in HBM/L2
    uint32_t *gcodes = nullptr, *gfb = nullptr;
    int sort_frontier = 0, sort_min = 0, nb_words = 0;  // sorted-frontier rebuild (configure())
    uint32_t *nbits = nullptr;
    int succ_bits = 0, sb_words = 0;                    // successor bitmap over arcs (generic kernels)
    uint32_t *sbits = nullptr;
    int code_words = 0, fb_words = 0;
    int seq_max_deg = 32;
    int max_deg = 0;      // largest out-degree of the graph
    int thin_wide = 0;    // rows longer than bcgroup::THIN_MAX_ROW
    int bpush = 2;        // fast path backward push ratio (KParams::bpush; BC_BPUSH overrides)
    int warp_max_deg = 4096;
    // graph
    char *graph_buf = nullptr;          // ro | col | src
    size_t csr_bytes = 0, graph_bytes = 0;
    cudaAccessPolicyWindow l2win{};     // persisting-L2 window over the CSR (num_bytes 0 = off)
    bool l2_held = false;               // registered as a user of the device's carve-out (L2Share)
    int *ro = nullptr, *col = nullptr, *src = nullptr;
    int *iro = nullptr, *icol = nullptr, *isrc = nullptr;
    // internal relabelling (see want_reorder): perm[old] = new; NULL = identity
    int *perm = nullptr;
    std::vector<int> h_perm;
    double *bc_tmp = nullptr;           // BC in internal ids before mapping back
    // workspace
    int slots = 0;
    int *d = nullptr;
    double *sigma = nullptr, *omega = nullptr;
    int *S = nullptr, *ends = nullptr;
    unsigned char *modes = nullptr;
    int *bigq = nullptr;
    size_t stride_big = 0;
    size_t stride_n = 0, stride_e = 0;
    // per-call buffers
    int *src_buf = nullptr;
    long long src_cap = 0;
    int *fb_src = nullptr;                   // sources handed from the WE-only to the EP kernel
    long long fb_cap = 0;
    unsigned long long *fb_n = nullptr;      // [0] handed over, [1] work counter of the EP launch
    int fb_used = 0;                         // the last compute call used the hand-over path
    double *bc_buf = nullptr;
    unsigned long long *counters = nullptr;  // [0] sampling phase, [1] main phase
    int *keys = nullptr;
    int *flag = nullptr;                     // Alg. 5 decision (persists for single-source)
    DevStats *stats = nullptr;
    cudaStream_t stream = nullptr;           // own stream for the host-buffer API
    cudaEvent_t done = nullptr;              // end of the last enqueued call
    bc_options opt{};
    int sampling_ran = 0;
    int last_inflight = 0;
    int launches = 0;        // kernels launched by the last compute call
    int bc_launches = 0;     // ... of which bc_kernel
    cudaEvent_t tev[4] = {nullptr, nullptr, nullptr, nullptr};  // around the bc_kernel launches
    int tev_used[2] = {0, 0};
    // multi-source batched engine (bc_batch.cu); allocated on first use
    std::vector<int> h_ro;              // internal CSR offsets (hub counts for any chunk size)
    struct Batch {
        int ready = 0, failed = 0;
        int Lcap = 0, LS = 0, nt = 256, grid = 0, nwarps = 0;
        long long qcap = 0;
        unsigned long long *F = nullptr, *qctr = nullptr, *lvor = nullptr;
        double *sig = nullptr, *dacc = nullptr;
        int *Q = nullptr, *qoff = nullptr;
        int *ovf_src = nullptr;
        long long ovf_cap = 0;
        long long *ovf_n = nullptr;
    } bt;
    int batch_ran = 0;       // the last compute call launched the batched engine
    int engines = 0;         // engines launched by the last compute call (bc_stats.engines)
    // group engine (bc_group.cu); allocated on first use
    struct Group {
        int ready = 0, failed = 0, nt = 512, grid = 0, G = 0, code_words = 0, sb = 0;
        unsigned long long *ctl = nullptr;
        double *sigma = nullptr;
        int *S = nullptr, *ends = nullptr, *bigq = nullptr;
        uint32_t *codes = nullptr, *nb = nullptr, *sbits = nullptr;
    } gr;
};

extern "C" void bc_default_options(bc_options *o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));  // every field (and any padding) defined, whatever the caller left
    o->strategy = BC_STRATEGY_SAMPLING;
    o->alpha = 768;
    o->beta = 512;
    o->gamma = 4.0;
    o->n_samps = 512;
    o->ep_min_frontier = 512;
    o->inflight = 0;
    o->backward_we = 0;
    o->block_threads = 0;
    o->seq_max_deg = 0;
    o->warp_max_deg = 0;
    o->l2_persist = 0;
    o->sort_frontier = 0;
    o->extrapolate = 0;
    o->succ_bits = 0;
    o->normalize = 0;
    o->level_store = 0;
    o->engine = BC_ENGINE_AUTO;
    o->batch_levels = 0;
    o->hub_chunk = 0;
    o->group_ctas = 0;
}

extern "C" const char *bc_last_error(void) { return g_err; }

static void free_workspace(bc_graph *g) {
    cudaFree(g->d);
    cudaFree(g->sigma);
    cudaFree(g->omega);
    cudaFree(g->S);
    cudaFree(g->ends);
    cudaFree(g->modes);
    cudaFree(g->bigq);
    cudaFree(g->gcodes);
    cudaFree(g->gfb);
    cudaFree(g->nbits);
    cudaFree(g->sbits);
    g->nbits = nullptr;
    g->sbits = nullptr;
    g->bigq = nullptr;
    g->gcodes = g->gfb = nullptr;
    g->d = nullptr;
    g->sigma = g->omega = nullptr;
    g->S = g->ends = nullptr;
    g->modes = nullptr;
    g->slots = 0;
}

static size_t slot_bytes(const bc_graph *g) {
    const size_t gc = g->lstore == 3 ? 4 * ((size_t)g->code_words + (size_t)g->fb_words) : 0;
    return g->stride_n * ((g->lstore == 1 ? sizeof(int) : 0) + 2 * sizeof(double) + sizeof(int)) +
           g->stride_e * (sizeof(int) + 1) + g->stride_big * sizeof(int) + gc +
           (g->sort_frontier ? 4 * (size_t)g->nb_words : 0) +
           (g->succ_bits ? 4 * (size_t)g->sb_words : 0);
}

template <bool EPOK>
static const void *pick_kernel(const bc_graph *g, int nt) {
    const bool sb = g->succ_bits != 0;
    if (g->directed) return kernel_directed(nt, EPOK, sb);
    if (g->lstore == 2) return kernel_scodes(nt, EPOK, sb);
    if (g->lstore == 3) return kernel_gcodes(nt, EPOK, sb);
    return kernel_levels(nt, EPOK, sb);
}

// Choose level store, block size and shared memory for both launch kinds
// (with / without the EP frontier bitmap) and their occupancy.
static int configure(bc_graph *g) {
    const bc_options &o = g->opt;
    const size_t code_bytes = (((size_t)g->n + 63) / 64) * 16;  // words padded to a multiple of 4
    const size_t fb_bytes = (((size_t)g->n + 31) / 32) * 4;
    const size_t smem_cap = 200 * 1024;  // leaves room for the static part (< 16 KB)
    const bool fits = !g->directed && code_bytes + fb_bytes <= smem_cap;
    if (o.level_store == 2 && !fits)
        return fail(BC_EINVAL, "level_store=2 needs an undirected graph with n <= ~%zu", smem_cap * 8 / 3);
    if (o.level_store == 3 && g->directed)
        return fail(BC_EINVAL, "level_store=3 (2-bit codes) needs an undirected graph");
    if (o.level_store != 0) g->lstore = o.level_store;
    else g->lstore = g->directed ? 1 : (fits ? 2 : 3);
    int nt = o.block_threads;
    if (nt == 0) {
        // Measured on B200 (tools/sweep.py): graphs of 2^17+ vertices (frontiers of
        // 10^3..10^5 vertices, hub rows) want wide CTAs; small graphs want many
        // narrow ones (frontiers of a few hundred vertices, more roots in flight).
        nt = g->n >= (1 << 17) ? 512 : 128;
        // degree-relabelled (skewed) graphs since the backward push: 1,024 threads, one
        // source per SM (c4: 487 -> 466 ms per 16,384 sources; c3, unskewed, 227 -> 286 ms)
        if (g->perm && g->n >= (1 << 17) && g->lstore == 2) nt = 1024;
    }
    if (nt != 128 && nt != 256 && nt != 512 && nt != 1024)
        return fail(BC_EINVAL, "block_threads must be 0, 128, 256, 512 or 1024");
    // defaults from tools/sweep_rows.sh on B200 (c4: 110.7 -> 103.8 ms, c3 82 -> 79 ms):
    // one-thread rows keep 32 independent rows in flight per warp, which beats warp
    // cooperation up to degree ~128; CTA cooperation pays for rows > 8192 (re-swept with the
    // group engine, tools/gpu/sweep_rows2.txt: c4 735.7 -> 731.7 ms, c5k 2335 -> 2195 ms;
    // 2048 / 4096 lose on c4, 64 / 256 one-thread rows lose on c4)
    g->seq_max_deg = o.seq_max_deg > 0 ? o.seq_max_deg : 128;
    g->warp_max_deg = std::max(g->seq_max_deg, o.warp_max_deg > 0 ? o.warp_max_deg : 8192);
    // Sorted frontiers: a level is rebuilt in vertex order from the per-level bitmap
    // when it holds >= sort_min vertices (the scan costs n/32 words, so small levels
    // keep their append order).
    g->sort_frontier = o.sort_frontier > 0 ? 1 : (o.sort_frontier < 0 ? 0 : (g->n >= (1 << 17)));
    if (g->lstore == 3) g->sort_frontier = 1;  // codes in HBM/L2 discover through the bitmap
    g->nb_words = (int)((((size_t)g->n + 31) / 32 + 31) & ~(size_t)31);
    // the bitmap replaces a probe of the level store per backward arc by one bit read,
    // at the price of an atomic OR per row in the forward pass: measured +6% on c5k
    // (codes in HBM/L2), neutral on c5ws, -10..-16% against shared-memory codes
    // (c2/c3/c4), so auto enables it only with level store 3
    g->succ_bits = o.succ_bits > 0 || (o.succ_bits == 0 && g->lstore == 3);
    g->sb_words = (int)((((size_t)g->nnz + 31) / 32 + 2 + 3) & ~(size_t)3);
    g->sort_min = std::max(1024, g->n / 64);
    g->code_words = g->lstore >= 2 ? (int)(code_bytes / 4) : 0;
    g->fb_words = g->lstore >= 2 ? (int)(fb_bytes / 4) : 0;

    // Persisting-L2 window over the CSR (plus src[] when EP levels can run): every
    // in-flight source re-reads the same rows, while sigma/omega gathers stream.
    g->l2win = cudaAccessPolicyWindow{};
    // auto: on, except for skewed graphs on the shared-memory-codes engine, whose CSR reads
    // hit L2 anyway once fewer sources are in flight (c4 at 1,024 threads: 466 -> 460 ms
    // without the window; c3 / c2d neutral)
    const bool l2_on = o.l2_persist > 0 || (o.l2_persist == 0 && !(g->perm && g->lstore == 2));
    if (!l2_on && g->l2_held) {  // window switched off: stop holding the carve-out
        l2_release(g->device);
        g->l2_held = false;
    }
    if (l2_on && g->graph_buf) {
        int max_persist = 0, max_win = 0;
        CK(cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, g->device));
        CK(cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, g->device));
        if (max_persist > 0 && max_win > 0) {
            const size_t span = o.strategy == BC_STRATEGY_WE ? g->csr_bytes : g->graph_bytes;
            const size_t want = std::min<size_t>(span, (size_t)max_win);
            const size_t carve = std::min<size_t>(want, (size_t)max_persist);
            CK(l2_acquire(g->device, carve, g->l2_held));
            g->l2_held = true;
            g->l2win.base_ptr = g->graph_buf;
            g->l2win.num_bytes = want;
            g->l2win.hitRatio = (float)((double)carve / (double)want);
            g->l2win.hitProp = cudaAccessPropertyPersisting;
            g->l2win.missProp = cudaAccessPropertyStreaming;
        }
    }
    g->cfg_we.fn = pick_kernel<false>(g, nt);
    g->cfg_ep.fn = pick_kernel<true>(g, nt);
    g->cfg_we.nt = g->cfg_ep.nt = nt;
    g->cfg_we.dyn = g->lstore == 2 ? code_bytes : 0;
    g->cfg_ep.dyn = g->lstore == 2 ? code_bytes + fb_bytes : 0;
    CK(cudaFuncSetAttribute(g->cfg_we.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->cfg_we.dyn));
    CK(cudaFuncSetAttribute(g->cfg_ep.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->cfg_ep.dyn));
    for (auto *c : {&g->cfg_we, &g->cfg_ep}) {
        int per_sm = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, c->fn, c->nt, c->dyn));
        if (per_sm < 1) return fail(BC_EINTERNAL, "kernel cannot be resident (dyn smem %zu)", c->dyn);
        c->per_sm = per_sm;
    }
    return BC_OK;
}

// Per-slot capacity of bigq (rows queued for CTA-cooperative expansion): a level queues at
// most nnz / (warp_max + 1) rows, warp_max being the EFFECTIVE threshold configure() derived
// (max(seq_max_deg, warp_max_deg)), so the stride must follow every change of either knob.
static size_t big_stride(const bc_graph *g) {
    // CTA rows (> warp_max) from the front and medium rows (> seq_max, fast path) from the
    // back: a level holds at most nnz / (seq_max + 1) of them together
    return (((size_t)g->nnz / ((size_t)g->seq_max_deg + 1) + 2) + 31) & ~(size_t)31;
}

static int alloc_workspace(bc_graph *g) {
    free_workspace(g);
    g->stride_n = (size_t)std::max(g->n, 1);
    g->stride_n = (g->stride_n + 31) & ~(size_t)31;  // 128-byte aligned slots
    g->stride_e = g->stride_n + 32;
    g->stride_big = big_stride(g);
    const int occ = std::max(g->cfg_we.per_sm, g->cfg_ep.per_sm) * g->num_sms;
    int want = g->opt.inflight > 0 ? std::min(g->opt.inflight, occ) : occ;
    size_t free_b = 0, total_b = 0;
    CK(cudaMemGetInfo(&free_b, &total_b));
    size_t per = slot_bytes(g);
    size_t budget = (size_t)(0.6 * (double)free_b);
    int cap = (int)std::max<size_t>(1, budget / std::max<size_t>(per, 1));
    g->slots = std::max(1, std::min(want, cap));
    size_t ns = (size_t)g->slots;
    if (g->lstore == 1) CK(cudaMalloc(&g->d, ns * g->stride_n * sizeof(int)));
    if (g->lstore == 3) {
        CK(cudaMalloc(&g->gcodes, ns * (size_t)g->code_words * 4));
        CK(cudaMalloc(&g->gfb, ns * (size_t)g->fb_words * 4));
        CK(cudaMemset(g->gcodes, 0, ns * (size_t)g->code_words * 4));
    }
    CK(cudaMalloc(&g->sigma, ns * g->stride_n * sizeof(double)));
    CK(cudaMalloc(&g->omega, ns * g->stride_n * sizeof(double)));
    CK(cudaMalloc(&g->S, ns * g->stride_n * sizeof(int)));
    CK(cudaMalloc(&g->ends, ns * g->stride_e * sizeof(int)));
    CK(cudaMalloc(&g->modes, ns * g->stride_e));
    CK(cudaMalloc(&g->bigq, ns * g->stride_big * sizeof(int)));
    if (g->succ_bits) {
        CK(cudaMalloc(&g->sbits, ns * (size_t)g->sb_words * 4));
        CK(cudaMemset(g->sbits, 0, ns * (size_t)g->sb_words * 4));
    }
    if (g->sort_frontier) {
        CK(cudaMalloc(&g->nbits, ns * (size_t)g->nb_words * 4));
        CK(cudaMemset(g->nbits, 0, ns * (size_t)g->nb_words * 4));
    }
    if (g->lstore == 1) CK(cudaMemset(g->d, 0x7F, ns * g->stride_n * sizeof(int)));  // INF = 0x7F7F7F7F
    CK(cudaMemset(g->sigma, 0, ns * g->stride_n * sizeof(double)));
    CK(cudaMemset(g->omega, 0, ns * g->stride_n * sizeof(double)));
    CK(cudaDeviceSynchronize());
    return BC_OK;
}

static void free_batch(bc_graph *g) {
    bc_graph::Batch &b = g->bt;
    cudaFree(b.F);
    cudaFree(b.qctr);
    cudaFree(b.lvor);
    cudaFree(b.sig);
    cudaFree(b.dacc);
    cudaFree(b.Q);
    cudaFree(b.qoff);
    cudaFree(b.ovf_src);
    cudaFree(b.ovf_n);
    b = bc_graph::Batch{};
}

// Workspace of the batched engine: vertex-major level masks F[(Lcap + 2) n], sigma/omega
// and accumulators [n][64], the union-frontier lists Q + their arc offsets (a vertex is
// in at most min(64, Lcap + 2) of them).  ~2 KB per vertex at Lcap 64.
static int alloc_batch(bc_graph *g, long long max_sources) {
    bc_graph::Batch &b = g->bt;
    const int Lcap = g->opt.batch_levels > 0 ? g->opt.batch_levels : 64;
    const long long ovf_need = std::max<long long>(max_sources, 64);
    if (b.ready && b.Lcap == Lcap && b.ovf_cap >= ovf_need) return BC_OK;
    free_batch(g);
    if ((long long)g->n >= (1LL << 24)) return fail(BC_EINVAL, "batched engine: n must be < 2^24");
    const size_t n = (size_t)std::max(g->n, 1);
    b.Lcap = Lcap;
    b.LS = Lcap + 2;
    const long long per_v = std::min(bcbatch::BW, b.LS);
    b.qcap = (long long)n * per_v;
    b.ovf_cap = ovf_need;
    b.nt = 256;
    const void *fn = bcbatch::batch_kernel_fn(b.nt);
    int per_sm = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, b.nt, 0));
    if (per_sm < 1) return fail(BC_EINTERNAL, "batched kernel cannot be resident");
    b.grid = per_sm * g->num_sms;
    b.nwarps = b.grid * b.nt / 32;
    CK(cudaMalloc(&b.F, n * (size_t)b.LS * 8));
    const size_t sn = (n + 31) & ~(size_t)31;
    CK(cudaMalloc(&b.sig, sn * bcbatch::BW * sizeof(double)));
    CK(cudaMalloc(&b.Q, (size_t)b.qcap * sizeof(int)));
    CK(cudaMalloc(&b.qoff, (size_t)b.qcap * sizeof(int)));
    CK(cudaMalloc(&b.qctr, (size_t)b.LS * 8));
    CK(cudaMalloc(&b.lvor, (size_t)b.LS * 8));
    CK(cudaMalloc(&b.dacc, sn * bcbatch::BW * sizeof(double)));
    CK(cudaMalloc(&b.ovf_src, (size_t)b.ovf_cap * sizeof(int)));
    CK(cudaMalloc(&b.ovf_n, sizeof(long long)));
    CK(cudaMemset(b.F, 0, n * (size_t)b.LS * 8));
    CK(cudaMemset(b.qctr, 0, (size_t)b.LS * 8));
    CK(cudaMemset(b.lvor, 0, (size_t)b.LS * 8));
    CK(cudaMemset(b.ovf_n, 0, sizeof(long long)));
    CK(cudaDeviceSynchronize());
    b.ready = 1;
    return BC_OK;
}

// Whether this call may run the batched engine (undirected graphs only: the
// three-mask visited test relies on neighbours being on adjacent levels).  Auto mode
// follows the engine comparison of DESIGN.md §7 (tools/cmp_engines.sh): the batched
// engine wins only where the per-source state of the in-flight sources (24 B x n each)
// is far beyond L2 AND the degree distribution is skewed (relabelled graphs: c5k
// 1.26x), loses on c4 (n = 2^18), on the unskewed small world c5ws and on every
// high-diameter graph; the device-side Alg. 5 flag still has to say EP.
static bool main_on_group(const bc_graph *g);

static bool batch_wanted(const bc_graph *g) {
    if (g->directed || g->n == 0) return false;
    if (g->opt.engine == BC_ENGINE_BATCHED) return true;
    return g->opt.engine == BC_ENGINE_AUTO && g->opt.strategy == BC_STRATEGY_SAMPLING &&
           g->perm != nullptr && g->n >= (1 << 21) && !main_on_group(g);
}

static void free_group(bc_graph *g) {
    bc_graph::Group &q = g->gr;
    cudaFree(q.ctl);
    cudaFree(q.sigma);
    cudaFree(q.S);
    cudaFree(q.ends);
    cudaFree(q.bigq);
    cudaFree(q.codes);
    cudaFree(q.nb);
    cudaFree(q.sbits);
    q = bc_graph::Group{};
}

// Groups for the group engine: as many as keep every group's per-source state
// (sigma 8n + codes n/4 + bitmaps 3n/8 + successor bits 2m/8 bytes) within ~48 MB of L2
// together, at least one; group_ctas > 0 fixes the CTAs per group instead.
static int group_count(const bc_graph *g, int grid) {
    if (g->opt.group_ctas > 0) return std::max(1, std::min(grid, grid / g->opt.group_ctas));
    // Auto, from the B200 sweeps (kernel ms for 2,048 sources): the unskewed
    // small world c5ws is fastest with 4 groups of 74 CTAs (1509 ms; 148 CTAs 1590, 37:
    // 1609), the skewed Kronecker c5k with groups of 12 CTAs (2103 ms; 9: 2149, 6: 2308,
    // 18: 2552).  Skewed = internally relabelled by degree (want_reorder).
    const int ctas = g->perm ? 18 : std::max(1, grid / 4);
    return std::max(1, std::min(grid, grid / ctas));
}

// The group engine's work-efficient levels run through the fast path on degree-relabelled
// (skewed) graphs and through the generic row_pass otherwise (measured).
// Thin rows (bc_thin.cuh) need the successor bitmap and a per-CTA queue (bigq, stride_big
// entries) that holds every row longer than THIN_MAX_ROW.
static bool thin_ok(const bc_graph *g) {
    return g->opt.succ_bits >= 0 && (size_t)g->thin_wide + 2 <= g->stride_big;
}

static int group_mode(const bc_graph *g) {
    int m = -1;
    if (const char *e = getenv("BC_GROUP_MODE")) m = atoi(e);  // tuning override
    else if (const char *e = getenv("BC_GROUP_FAST")) m = atoi(e) != 0 ? bcgroup::GM_FAST : bcgroup::GM_GENERIC;
    // auto (B200, c5ws 2,048 sources, kernel ms): degree-relabelled graphs take the fast path
    // (c5k 1959 against 2104 generic, 4036+ thin); graphs in their own order with >= 2^21
    // vertices take thin rows (c5ws 1416 against 1503 generic, 1548 fast), smaller ones the
    // generic row_pass (CSR-order sums)
    if (m < 0) m = g->perm ? bcgroup::GM_FAST : (g->n >= (1 << 21) ? bcgroup::GM_THIN : bcgroup::GM_GENERIC);
    if (m == bcgroup::GM_THIN && !thin_ok(g)) m = bcgroup::GM_GENERIC;
    return m;
}

static int alloc_group(bc_graph *g) {
    bc_graph::Group &q = g->gr;
    int nt = g->n >= (1 << 17) ? 512 : 256;
    if (const char *e = getenv("BC_GROUP_NT")) nt = atoi(e);  // tuning override (1024: tuning build)
    int per_sm = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bcgroup::group_kernel_fn(nt, group_mode(g)), nt, 0));
    if (per_sm < 1) return fail(BC_EINTERNAL, "group kernel cannot be resident");
    const int grid = per_sm * g->num_sms;
    const int G = group_count(g, grid);
    const int sbw = g->opt.succ_bits >= 0;  // on unless switched off
    if (q.ready && q.nt == nt && q.grid == grid && q.G == G && q.sb == sbw) return BC_OK;
    free_group(g);
    q.nt = nt;
    q.grid = grid;
    q.G = G;
    q.sb = sbw;
    q.code_words = (int)((((size_t)g->n + 63) / 64) * 4);
    const size_t ng = (size_t)G;
    CK(cudaMalloc(&q.ctl, ng * bcgroup::CTL_WORDS * 8));
    CK(cudaMalloc(&q.sigma, ng * g->stride_n * sizeof(double)));
    CK(cudaMalloc(&q.S, ng * g->stride_n * sizeof(int)));
    CK(cudaMalloc(&q.ends, ng * g->stride_e * sizeof(int)));
    CK(cudaMalloc(&q.bigq, (size_t)grid * g->stride_big * sizeof(int)));
    CK(cudaMalloc(&q.codes, ng * (size_t)q.code_words * 4));
    CK(cudaMalloc(&q.nb, ng * 3 * (size_t)g->nb_words * 4));
    CK(cudaMemset(q.codes, 0, ng * (size_t)q.code_words * 4));
    CK(cudaMemset(q.nb, 0, ng * 3 * (size_t)g->nb_words * 4));
    if (sbw) {
        CK(cudaMalloc(&q.sbits, ng * (size_t)g->sb_words * 4));
        CK(cudaMemset(q.sbits, 0, ng * (size_t)g->sb_words * 4));
    }
    CK(cudaMemset(q.sigma, 0, ng * g->stride_n * sizeof(double)));
    CK(cudaDeviceSynchronize());
    q.ready = 1;
    return BC_OK;
}

// Whether a launch may run on the group engine: undirected, every level work-efficient
// (WE strategy, or Alg. 5 with a guard no frontier can reach), no device-side count.
static bool group_eligible(const bc_graph *g, const KParams &p) {
    if (g->directed || g->n == 0 || p.k_dev || p.skip_if_ep) return false;
    return p.launch_mode == LM_WE ||
           (p.launch_mode == LM_SAMPLED && (long long)p.ep_min_frontier > (long long)g->n);
}

// Auto mode picks the group engine for large undirected graphs (n >= 2^21: the c5
// configs, where it beats the per-source engine 1.55x (c5ws) and 1.36x (c5k) and the
// batched engine 2.2x / 1.14x); on smaller graphs the per-source engine
// (codes in shared memory, ~300 sources in flight) is faster (c4: 728 vs 1374 ms).
static bool group_auto(const bc_graph *g) {
    return g->opt.engine == BC_ENGINE_AUTO && !g->directed && g->n >= (1 << 21) && !g->gr.failed;
}

static bool group_wanted(const bc_graph *g, const KParams &p) {
    return (g->opt.engine == BC_ENGINE_GROUP || group_auto(g)) && group_eligible(g, p);
}

// Whether the main phase of a compute call runs entirely on the group engine.
static bool main_on_group(const bc_graph *g) {
    const int st = g->opt.strategy;
    const bool all_we = st == BC_STRATEGY_WE ||
                        (st == BC_STRATEGY_SAMPLING && (long long)g->opt.ep_min_frontier > (long long)g->n);
    return (g->opt.engine == BC_ENGINE_GROUP || group_auto(g)) && !g->directed && g->n > 0 && all_we;
}

static int launch_group(bc_graph *g, const KParams &p0, cudaStream_t st) {
    int rc = alloc_group(g);
    if (rc) return rc;
    const bc_graph::Group &q = g->gr;
    KParams p = p0;
    p.sigma = q.sigma;
    // the group engine always pulls (pushing from level L+1 was measured slower on c5k:
    // 2085 -> 2556 ms per 2,048 sources, its successor-bit backward is already cheap per arc)
    p.bpush = 0;
    p.S = q.S;
    p.ends = q.ends;
    p.bigq = q.bigq;
    p.gcodes = q.codes;
    p.stride_codes = (size_t)q.code_words;
    p.code_words = q.code_words;
    p.nbits = q.nb;
    p.stride_nb = 3 * (size_t)g->nb_words;
    p.nb_words = g->nb_words;
    p.sbits = q.sbits;
    p.stride_sb = (size_t)g->sb_words;
    p.sb_words = g->sb_words;
    p.fb_words = 0;
    bcgroup::GParams gp;
    gp.groups = q.G;
    gp.ctl = q.ctl;
    gp.own_block = g->perm ? 1 : 32;  // see bcgroup::Owned (measured per graph kind)
    if (const char *ob = getenv("BC_OWN_BLOCK")) gp.own_block = std::max(1, atoi(ob));  // tuning
    CK(cudaMemsetAsync(q.ctl, 0, (size_t)q.G * bcgroup::CTL_WORDS * 8, st));
    void *args[] = {&p, &gp};
    cudaLaunchConfig_t lc{};
    lc.gridDim = dim3(q.grid);
    lc.blockDim = dim3(q.nt);
    lc.dynamicSmemBytes = 0;
    lc.stream = st;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    int na = 1;
    if (g->l2win.num_bytes) {
        attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[1].val.accessPolicyWindow = g->l2win;
        na = 2;
    }
    lc.attrs = attr;
    lc.numAttrs = na;
    CK(cudaLaunchKernelExC(&lc, bcgroup::group_kernel_fn(q.nt, group_mode(g)), args));
    CK(cudaGetLastError());
    g->launches++;
    g->bc_launches++;
    g->engines |= 4;
    g->last_inflight = std::max(g->last_inflight, q.G);
    return BC_OK;
}

static int launch_batch(bc_graph *g, const bcbatch::BParams &bp0, cudaStream_t st) {
    if (bp0.k <= 0) return BC_OK;
    bcbatch::BParams bp = bp0;
    void *args[] = {&bp};
    cudaLaunchConfig_t lc{};
    lc.gridDim = dim3(g->bt.grid);
    lc.blockDim = dim3(g->bt.nt);
    lc.dynamicSmemBytes = 0;
    lc.stream = st;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    int na = 1;
    if (g->l2win.num_bytes) {
        attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[1].val.accessPolicyWindow = g->l2win;
        na = 2;
    }
    lc.attrs = attr;
    lc.numAttrs = na;
    // BC_BATCH_TRACE=1: per-level cycle trace of the launch's first batch on stderr
    // (debug tooling; synchronises the stream)
    const char *tr = getenv("BC_BATCH_TRACE");
    long long *dtrace = nullptr;
    const size_t ntr = 2 * (size_t)g->bt.LS * 12;
    if (tr && *tr == '1') {
        CK(cudaMalloc(&dtrace, ntr * sizeof(long long)));
        CK(cudaMemsetAsync(dtrace, 0, ntr * sizeof(long long), st));
        bp.trace = dtrace;
    }
    CK(cudaLaunchKernelExC(&lc, bcbatch::batch_kernel_fn(g->bt.nt), args));
    if (dtrace) {
        std::vector<long long> h(ntr);
        CK(cudaMemcpyAsync(h.data(), dtrace, ntr * sizeof(long long), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        cudaFree(dtrace);
        const int nw = g->bt.nwarps;
        for (int dir = 0; dir < 2; ++dir)
            for (int L = 0; L < g->bt.LS; ++L) {
                const long long *t = &h[((size_t)dir * g->bt.LS + L) * 12];
                if (!t[0] && !t[1]) continue;
                fprintf(stderr, "[trace] %s L=%2d arcs=%9lld wall=%9lld maxwarp=%9lld meanwarp=%9.0f | "
                        "rowwin %lld x %.0f cyc, pairwin %lld x %.0f cyc, pairs %lld, range %.0f cyc/warp\n",
                        dir ? "bwd" : "fwd", L, t[3], t[0], t[1], (double)t[2] / nw,
                        t[6], t[6] ? (double)t[4] / t[6] : 0.0, t[7], t[7] ? (double)t[5] / t[7] : 0.0, t[8],
                        (double)t[9] / nw);
            }
    }
    g->launches++;
    g->bc_launches++;
    g->engines |= 2;
    g->batch_ran = 1;
    g->last_inflight = std::max(g->last_inflight, g->bt.grid);
    return BC_OK;
}

static bcbatch::BParams batch_params(bc_graph *g, const int *d_sources, long long base, long long k,
                                     double *acc_bc) {
    const bc_graph::Batch &b = g->bt;
    bcbatch::BParams bp;
    memset(&bp, 0, sizeof(bp));
    bp.n = g->n;
    bp.ro = g->ro;
    bp.col = g->col;
    bp.src = g->src;
    bp.nnz = g->nnz;
    // multi-source EP levels: Alg. 5 runs (guard ep_min_frontier, only after an EP decision)
    // and the EP strategy (every level); WE / hybrid batches stay work-efficient
    bp.ep_guard = g->opt.strategy == BC_STRATEGY_SAMPLING ? g->opt.ep_min_frontier
                : g->opt.strategy == BC_STRATEGY_EP ? 1 : 0;
    bp.ep_flag = g->opt.strategy == BC_STRATEGY_SAMPLING ? g->flag : nullptr;
    bp.sources = d_sources;
    bp.perm = g->perm;
    bp.src_base = base;
    bp.k = k;
    bp.Lcap = b.Lcap;
    bp.LS = b.LS;
    bp.min_range = g->opt.hub_chunk > 0 ? g->opt.hub_chunk : 64;
    bp.F = b.F;
    bp.sig = b.sig;
    bp.Q = b.Q;
    bp.qoff = b.qoff;
    bp.qcap = b.qcap;
    bp.qctr = b.qctr;
    bp.lvor = b.lvor;
    bp.dacc = b.dacc;
    bp.sn = ((size_t)std::max(g->n, 1) + 31) & ~(size_t)31;
    bp.bc = acc_bc;
    bp.stats = g->stats;
    bp.ovf_src = b.ovf_src;
    bp.ovf_n = b.ovf_n;
    return bp;
}

extern "C" void bc_destroy(bc_graph *g) {
    if (!g) return;
    DeviceGuard dg(g->device);
    if (g->done) cudaEventSynchronize(g->done);
    free_workspace(g);
    free_batch(g);
    free_group(g);
    if (g->l2_held) l2_release(g->device);  // the last holder on the device resets the carve-out
    cudaFree(g->graph_buf);
    cudaFree(g->perm);
    cudaFree(g->bc_tmp);
    cudaFree(g->iro);
    cudaFree(g->icol);
    cudaFree(g->isrc);
    cudaFree(g->src_buf);
    cudaFree(g->fb_src);
    cudaFree(g->fb_n);
    cudaFree(g->bc_buf);
    cudaFree(g->counters);
    cudaFree(g->keys);
    cudaFree(g->flag);
    cudaFree(g->stats);
    if (g->done) cudaEventDestroy(g->done);
    for (auto &e : g->tev)
        if (e) cudaEventDestroy(e);
    if (g->stream) cudaStreamDestroy(g->stream);
    delete g;
}

// Internal vertex order.  For skewed degree distributions the vertices are
// relabelled by descending degree (stable): the sigma/omega entries that the
// shortest-path DAG gathers most (hub predecessors) then share a few KB per
// source instead of one 32-byte sector each, and isolated vertices move to the
// end.  Each row keeps its original neighbour order (so one-thread sums follow
// the caller's CSR order).  Sources are mapped old -> new on the device and BC is
// mapped back when it is written out.  BC_REORDER=0/1 overrides the heuristic.
static bool want_reorder(const bc_graph *g, const int64_t *ro64) {
    const char *env = getenv("BC_REORDER");
    if (env && *env) return atoi(env) != 0;
    if (g->n < 1024) return false;
    int64_t maxdeg = 0;
    for (int v = 0; v < g->n; ++v) maxdeg = std::max<int64_t>(maxdeg, ro64[v + 1] - ro64[v]);
    const double avg = (double)g->nnz / g->n;
    return (double)maxdeg >= 32.0 * std::max(avg, 1.0);
}

static int create_impl(bc_graph *g, const int64_t *ro64, const int32_t *col_in) {
    const int n = g->n;
    const int nnz = g->nnz;
    std::vector<int> ro32((size_t)n + 1);
    std::vector<int> col_re;
    const int32_t *col = col_in;
    if (want_reorder(g, ro64)) {
        std::vector<int> order((size_t)n);
        for (int v = 0; v < n; ++v) order[v] = v;
        std::stable_sort(order.begin(), order.end(), [&](int a, int b) {
            return ro64[a + 1] - ro64[a] > ro64[b + 1] - ro64[b];
        });
        g->h_perm.assign((size_t)n, 0);
        for (int i = 0; i < n; ++i) g->h_perm[order[i]] = i;  // old -> new
        col_re.resize((size_t)std::max(nnz, 1));
        ro32[0] = 0;
        for (int i = 0; i < n; ++i) {
            const int v = order[i];
            int k = ro32[i];
            for (int64_t e = ro64[v]; e < ro64[v + 1]; ++e) col_re[k++] = g->h_perm[col_in[e]];
            ro32[i + 1] = k;
        }
        col = col_re.data();
        CK(cudaMalloc(&g->perm, sizeof(int) * (size_t)n));
        CK(cudaMemcpy(g->perm, g->h_perm.data(), sizeof(int) * (size_t)n, cudaMemcpyHostToDevice));
        CK(cudaMalloc(&g->bc_tmp, sizeof(double) * (size_t)n));
    } else {
        for (int v = 0; v <= n; ++v) ro32[v] = (int)ro64[v];
    }
    g->h_ro = ro32;
    for (int v = 0; v < n; ++v) {
        g->max_deg = std::max(g->max_deg, ro32[v + 1] - ro32[v]);
        if (ro32[v + 1] - ro32[v] > bcgroup::THIN_MAX_ROW) g->thin_wide++;
    }
    CK(cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&g->done, cudaEventDisableTiming));
    for (auto &e : g->tev) CK(cudaEventCreate(&e));
    // ro | col | src in one allocation so one L2 access-policy window covers the CSR
    auto al = [](size_t b) { return (b + 255) & ~(size_t)255; };
    const size_t b_ro = al(sizeof(int) * ((size_t)n + 1));
    const size_t b_col = al(sizeof(int) * (size_t)std::max(nnz, 1) + 16);
    CK(cudaMalloc(&g->graph_buf, b_ro + 2 * b_col));
    g->ro = reinterpret_cast<int *>(g->graph_buf);
    g->col = reinterpret_cast<int *>(g->graph_buf + b_ro);
    g->src = reinterpret_cast<int *>(g->graph_buf + b_ro + b_col);
    g->csr_bytes = b_ro + b_col;
    g->graph_bytes = b_ro + 2 * b_col;
    CK(cudaMemcpy(g->ro, ro32.data(), sizeof(int) * ((size_t)n + 1), cudaMemcpyHostToDevice));
    if (nnz) CK(cudaMemcpy(g->col, col, sizeof(int) * (size_t)nnz, cudaMemcpyHostToDevice));
    // zeroed slack after the last column: 16-byte quad reads past a row's end (one-thread
    // rows) then always see valid vertex ids
    CK(cudaMemset(g->col + nnz, 0, 16));
    if (nnz && n) {
        build_src_kernel<<<std::min((nnz + 255) / 256, 148 * 16), 256>>>(g->ro, n, nnz, g->src);
        CK(cudaGetLastError());
    }
    if (g->directed) {
        // transpose on the host (counting sort keeps in-rows in ascending source order)
        std::vector<int> iro((size_t)n + 1, 0), icol((size_t)std::max(nnz, 1)), fill((size_t)n);
        for (int e = 0; e < nnz; ++e) iro[col[e] + 1]++;
        for (int v = 0; v < n; ++v) iro[v + 1] += iro[v];
        for (int v = 0; v < n; ++v) fill[v] = iro[v];
        for (int u = 0; u < n; ++u)
            for (int e = ro32[u]; e < ro32[u + 1]; ++e) icol[fill[col[e]]++] = u;
        CK(cudaMalloc(&g->iro, sizeof(int) * ((size_t)n + 1)));
        CK(cudaMalloc(&g->icol, sizeof(int) * ((size_t)std::max(nnz, 1) + 4)));  // quad-read slack
        CK(cudaMalloc(&g->isrc, sizeof(int) * (size_t)std::max(nnz, 1)));
        CK(cudaMemcpy(g->iro, iro.data(), sizeof(int) * ((size_t)n + 1), cudaMemcpyHostToDevice));
        if (nnz) {
            CK(cudaMemcpy(g->icol, icol.data(), sizeof(int) * (size_t)nnz, cudaMemcpyHostToDevice));
            build_src_kernel<<<std::min((nnz + 255) / 256, 148 * 16), 256>>>(g->iro, n, nnz, g->isrc);
            CK(cudaGetLastError());
        }
    }
    CK(cudaMalloc(&g->counters, 3 * sizeof(unsigned long long)));
    CK(cudaMalloc(&g->fb_n, 2 * sizeof(unsigned long long)));
    CK(cudaMalloc(&g->keys, sizeof(int) * 8192));
    CK(cudaMalloc(&g->flag, sizeof(int)));
    CK(cudaMemset(g->flag, 0, sizeof(int)));
    CK(cudaMalloc(&g->stats, sizeof(DevStats)));
    CK(cudaMemset(g->stats, 0, sizeof(DevStats)));
    CK(cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device));
    bc_default_options(&g->opt);
    int rc = configure(g);
    if (rc) return rc;
    rc = alloc_workspace(g);
    if (rc) return rc;
    CK(cudaDeviceSynchronize());
    return BC_OK;
}

extern "C" int bc_graph_create(int32_t n, int64_t nnz, const int64_t *row_offsets,
                               const int32_t *col_indices, int directed, int device,
                               bc_graph **out) {
    if (!out) return fail(BC_EINVAL, "out is NULL");
    *out = nullptr;
    if (n < 0 || n > 0x7FFFFFFF - 64) return fail(BC_EINVAL, "n=%d out of range", n);
    if (nnz < 0 || nnz > 0x7FFFFFFFLL - 1) return fail(BC_EINVAL, "nnz=%lld out of range (< 2^31)", (long long)nnz);
    if (!row_offsets) return fail(BC_EINVAL, "row_offsets is NULL");
    if (nnz > 0 && !col_indices) return fail(BC_EINVAL, "col_indices is NULL");
    if (row_offsets[0] != 0) return fail(BC_EINVAL, "row_offsets[0] != 0");
    if (row_offsets[n] != nnz) return fail(BC_EINVAL, "row_offsets[n]=%lld != nnz=%lld",
                                           (long long)row_offsets[n], (long long)nnz);
    for (int v = 0; v < n; ++v)
        if (row_offsets[v + 1] < row_offsets[v])
            return fail(BC_EINVAL, "row_offsets decreases at vertex %d", v);
    for (int64_t e = 0; e < nnz; ++e)
        if (col_indices[e] < 0 || col_indices[e] >= n)
            return fail(BC_EINVAL, "col_indices[%lld]=%d out of range", (long long)e, col_indices[e]);
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return fail(BC_ECUDA, "no CUDA device available");
    if (device < 0 || device >= ndev) return fail(BC_EINVAL, "device %d out of range", device);
    bc_graph *g = new (std::nothrow) bc_graph();
    if (!g) return fail(BC_ENOMEM, "host allocation failed");
    g->device = device;
    g->n = n;
    g->nnz = (int)nnz;
    g->directed = directed ? 1 : 0;
    DeviceGuard dg(device);
    int rc = create_impl(g, row_offsets, col_indices);
    if (rc) {
        bc_destroy(g);
        return rc;
    }
    *out = g;
    g_err[0] = 0;
    return BC_OK;
}

extern "C" int bc_set_options(bc_graph *g, const bc_options *o) {
    if (!g || !o) return fail(BC_EINVAL, "NULL argument");
    if (o->strategy < 0 || o->strategy > 3) return fail(BC_EINVAL, "bad strategy %d", o->strategy);
    if (o->n_samps < 1 || o->n_samps > 8192) return fail(BC_EINVAL, "n_samps must be in [1, 8192]");
    if (o->alpha < 0 || o->beta < 0 || o->ep_min_frontier < 0 || o->inflight < 0 || !(o->gamma >= 0) ||
        o->seq_max_deg < 0 || o->warp_max_deg < 0 || o->level_store < 0 || o->level_store > 3 ||
        o->engine < 0 || o->engine > 3 || o->group_ctas < 0 || o->batch_levels < 0 || o->batch_levels > bcbatch::MAX_LCAP ||
        o->hub_chunk < 0)
        return fail(BC_EINVAL, "invalid parameter");
    if (o->block_threads != 0 && o->block_threads != 128 && o->block_threads != 256 &&
        o->block_threads != 512 && o->block_threads != 1024)
        return fail(BC_EINVAL, "block_threads must be 0, 128, 256, 512 or 1024");
    DeviceGuard dg(g->device);
    if (g->done) CK(cudaEventSynchronize(g->done));
    const bc_options old = g->opt;
    g->opt = *o;
    free_group(g);  // re-sized on its next use
    int rc = configure(g);
    if (rc) {
        g->opt = old;
        configure(g);
        return rc;
    }
    const int old_slots = g->slots;
    // bigq follows the effective row-split threshold (seq_max_deg AND warp_max_deg): a
    // smaller threshold queues more rows per level, so the workspace must grow with it
    const int realloc = o->inflight != old.inflight || o->level_store != old.level_store ||
                        o->block_threads != old.block_threads || big_stride(g) != g->stride_big ||
                        o->sort_frontier != old.sort_frontier || o->succ_bits != old.succ_bits;
    if (realloc) {
        rc = alloc_workspace(g);
        if (rc) return rc;
    }
    (void)old_slots;
    return BC_OK;
}

extern "C" int bc_get_options(const bc_graph *g, bc_options *o) {
    if (!g || !o) return fail(BC_EINVAL, "NULL argument");
    *o = g->opt;
    return BC_OK;
}

static KParams base_params(bc_graph *g, double *d_bc) {
    KParams p;
    memset(&p, 0, sizeof(p));
    p.n = g->n;
    p.nnz = g->nnz;
    p.ro = g->ro;
    p.col = g->col;
    p.src = g->src;
    p.iro = g->directed ? g->iro : g->ro;
    p.icol = g->directed ? g->icol : g->col;
    p.isrc = g->directed ? g->isrc : g->src;
    p.d = g->d;
    p.sigma = g->sigma;
    p.omega = g->omega;
    p.S = g->S;
    p.ends = g->ends;
    p.modes = g->modes;
    p.bigq = g->bigq;
    p.stride_big = g->stride_big;
    p.stride_n = g->stride_n;
    p.stride_e = g->stride_e;
    p.bc = d_bc;
    p.alpha = g->opt.alpha;
    p.beta = g->opt.beta;
    p.ep_min_frontier = g->opt.ep_min_frontier;
    p.backward_we = g->opt.backward_we;
    p.code_words = g->code_words;
    p.gcodes = g->gcodes;
    p.gfb = g->gfb;
    p.stride_codes = (size_t)g->code_words;
    p.stride_fb = (size_t)g->fb_words;
    p.nbits = g->sort_frontier ? g->nbits : nullptr;
    p.stride_nb = (size_t)g->nb_words;
    p.nb_words = g->nb_words;
    p.sort_min = g->sort_min;
    p.sbits = g->succ_bits ? g->sbits : nullptr;
    p.stride_sb = (size_t)g->sb_words;
    p.sb_words = g->sb_words;
    p.seq_max_deg = g->seq_max_deg;
    p.medq = g->max_deg > g->seq_max_deg ? 1 : 0;
    p.bpush = g->bpush;
    if (const char *e = getenv("BC_BPUSH")) p.bpush = std::max(0, atoi(e));  // tuning override
    p.warp_max_deg = g->warp_max_deg;
    p.stats = g->stats;
    p.sampled_flag = g->flag;
    p.perm = g->perm;
    return p;
}

// Raw launch of bc_kernel with configuration c (grid = resident CTAs, at most k).
static int launch_cfg(bc_graph *g, KParams p, const bc_graph::KCfg &c, bool ep_kernel, cudaStream_t st) {
    p.fb_words = ep_kernel ? g->fb_words : 0;
    const long long cap = std::min<long long>(g->slots, (long long)c.per_sm * g->num_sms);
    const int grid = (int)std::min<long long>(cap, p.k);
    void *args[] = {&p};
    cudaLaunchConfig_t lc{};
    lc.gridDim = dim3(grid);
    lc.blockDim = dim3(c.nt);
    lc.dynamicSmemBytes = c.dyn;
    lc.stream = st;
    cudaLaunchAttribute attr[1];
    if (g->l2win.num_bytes) {
        attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[0].val.accessPolicyWindow = g->l2win;
        lc.attrs = attr;
        lc.numAttrs = 1;
    }
    CK(cudaLaunchKernelExC(&lc, c.fn, args));
    g->last_inflight = std::max(g->last_inflight, grid);
    g->launches++;
    g->bc_launches++;
    g->engines |= 1;
    CK(cudaGetLastError());
    return BC_OK;
}

// Whether cfg_we is the fast-path kernel (bc_fast.cuh), which can hand a source whose
// selector asks for an EP level over to an EP-capable launch.
static bool we_kernel_is_fast(const bc_graph *g) { return g->lstore == 2 && !g->directed && !g->succ_bits; }

static int launch(bc_graph *g, const KParams &p0, cudaStream_t st) {
    if (p0.k <= 0) return BC_OK;
    if (group_wanted(g, p0)) {
        const int rc = launch_group(g, p0, st);
        if (rc == BC_OK || g->opt.engine == BC_ENGINE_GROUP) return rc;
        free_group(g);
        g->gr.failed = 1;  // auto: e.g. no memory for the group workspace -> per-source engine
        cudaGetLastError();
    }
    KParams p = p0;
    // An EP level needs a frontier of >= ep_min_frontier (Alg. 5 guard) or > beta
    // (Alg. 4) vertices; when no frontier can be that large, the work-efficient-only
    // kernel (no EP code, no bitmap) is launched instead.
    const bool ep_possible =
        !p.skip_if_ep &&
        (p.launch_mode == LM_EP ||
         (p.launch_mode == LM_SAMPLED && (long long)p.ep_min_frontier <= (long long)g->n) ||
         (p.launch_mode == LM_HYBRID && (long long)p.beta < (long long)g->n));
    if (!ep_possible) return launch_cfg(g, p, g->cfg_we, false, st);
    // Alg. 4 / Alg. 5 run that MAY ask for EP levels: optimistic work-efficient launch.  The
    // fast WE-only kernel runs every source; a source whose selector picks EP for its next
    // level is abandoned before its backward stage (nothing of it reaches bc) and queued; an
    // EP-capable launch then runs the queued sources from scratch with the same selector.  A
    // run that never picks EP (Alg. 4 on high-diameter graphs, Alg. 5 with a WE decision)
    // therefore never pays for the EP code path (the selectors taxed WE levels).
    if ((p.launch_mode == LM_HYBRID || p.launch_mode == LM_SAMPLED) && we_kernel_is_fast(g) && !p.dbg_d &&
        !p.k_dev && !p.skip_if_we) {
        if (p.k > g->fb_cap) {
            cudaFree(g->fb_src);
            g->fb_src = nullptr;
            g->fb_cap = 0;
            CK(cudaMalloc(&g->fb_src, sizeof(int) * (size_t)p.k));
            g->fb_cap = p.k;
        }
        CK(cudaMemsetAsync(g->fb_n, 0, 2 * sizeof(unsigned long long), st));
        g->fb_used = 1;
        KParams pw = p;
        pw.fallback_src = g->fb_src;
        pw.fallback_n = g->fb_n;
        int rc = launch_cfg(g, pw, g->cfg_we, false, st);
        if (rc) return rc;
        KParams pe = p;
        pe.sources = g->fb_src;  // caller ids
        pe.src_base = 0;
        pe.k_dev = reinterpret_cast<const long long *>(g->fb_n);
        pe.work_counter = g->fb_n + 1;
        return launch_cfg(g, pe, g->cfg_ep, true, st);
    }
    // Otherwise (other level stores): an Alg. 5 run whose decision is still on the device
    // enqueues BOTH kernels, each gated on the flag (the other exits at once).
    if (p.launch_mode == LM_SAMPLED && p.sampled_flag && !p.skip_if_we) {
        KParams pw = p;
        pw.skip_if_ep = 1;
        int rc = launch_cfg(g, pw, g->cfg_we, false, st);
        if (rc) return rc;
        p.skip_if_we = 1;
    }
    return launch_cfg(g, p, g->cfg_ep, true, st);
}

// Enqueue one full BC computation on `st`.  d_sources may be NULL (all n).
static int enqueue_compute(bc_graph *g, const int *d_sources, long long k, double *d_bc,
                           cudaStream_t st) {
    CK(cudaStreamWaitEvent(st, g->done, 0));
    g->sampling_ran = 0;
    if (g->n == 0) {
        CK(cudaMemsetAsync(g->stats, 0, sizeof(DevStats), st));
        CK(cudaEventRecord(g->done, st));
        return BC_OK;
    }
    double *acc_bc = g->perm ? g->bc_tmp : d_bc;  // accumulate in internal ids
    CK(cudaMemsetAsync(acc_bc, 0, sizeof(double) * (size_t)g->n, st));
    CK(cudaMemsetAsync(g->counters, 0, 3 * sizeof(unsigned long long), st));
    CK(cudaMemsetAsync(g->stats, 0, sizeof(DevStats), st));
    g->last_inflight = 0;
    g->launches = g->bc_launches = 0;
    g->tev_used[0] = g->tev_used[1] = 0;
    g->batch_ran = 0;
    g->engines = 0;
    g->fb_used = 0;
    KParams p = base_params(g, acc_bc);
    p.sources = d_sources;
    int rc = BC_OK;
    const int strat = g->opt.strategy;
    const int mode_main = strat == BC_STRATEGY_WE ? LM_WE : strat == BC_STRATEGY_EP ? LM_EP
                        : strat == BC_STRATEGY_HYBRID ? LM_HYBRID : LM_SAMPLED;
    long long ks = 0;
    // Alg. 5 with a guard no frontier can reach (ep_min_frontier > n, the bench's B200
    // guard): the decision cannot change how any source runs (every level is WE either
    // way), so the sampling sources and the rest go in ONE launch -- the first n_samps still
    // record their max depth and the decision is still taken and reported afterwards --
    // instead of two launches with a tail each (c1: two waves of 512 sources -> one).
    const bool merged = strat == BC_STRATEGY_SAMPLING && (long long)g->opt.ep_min_frontier > (long long)g->n &&
                        !batch_wanted(g) && !getenv("BC_NO_MERGE");
    if (merged) {
        ks = std::min<long long>(k, g->opt.n_samps);
        KParams pm = p;
        pm.launch_mode = LM_WE;
        pm.src_base = 0;
        pm.k = k;
        pm.keys = g->keys;
        pm.nkeys = ks;
        pm.work_counter = g->counters + 1;
        if (k > 0) {
            CK(cudaEventRecord(g->tev[2], st));
            if ((rc = launch(g, pm, st))) return rc;
            CK(cudaEventRecord(g->tev[3], st));
            g->tev_used[1] = 1;
        }
        if (ks > 0) {
            int P = 1;
            while (P < ks) P <<= 1;
            const double thresh = g->opt.gamma * std::log2((double)std::max(g->n, 1));
            sampling_decide_kernel<<<1, 1024, sizeof(int) * (size_t)P, st>>>(g->keys, (int)ks, thresh,
                                                                           g->flag, g->stats);
            CK(cudaGetLastError());
            g->launches++;
            g->sampling_ran = 1;
        }
        ks = k;  // nothing left for the main phase below
    } else if (strat == BC_STRATEGY_SAMPLING) {
        // Alg. 5: first n_samps sources WE, record max depth, decide, then the rest.
        ks = std::min<long long>(k, g->opt.n_samps);
        KParams ps = p;
        ps.launch_mode = LM_WE;
        ps.src_base = 0;
        ps.k = ks;
        ps.keys = g->keys;
        ps.nkeys = ks;
        ps.work_counter = g->counters;
        if (ks > 0) {
            CK(cudaEventRecord(g->tev[0], st));
            if ((rc = launch(g, ps, st))) return rc;
            CK(cudaEventRecord(g->tev[1], st));
            g->tev_used[0] = 1;
        }
        if (ks > 0) {
            int P = 1;
            while (P < ks) P <<= 1;
            const double thresh = g->opt.gamma * std::log2((double)std::max(g->n, 1));
            sampling_decide_kernel<<<1, 1024, sizeof(int) * (size_t)P, st>>>(g->keys, (int)ks, thresh,
                                                                           g->flag, g->stats);
            CK(cudaGetLastError());
            g->launches++;
            g->sampling_ran = 1;
        }
    }
    // Main phase.  With the batched engine in auto mode, both engines are enqueued and
    // the device-side Alg. 5 decision picks one: an EP ("small-world") run goes to the
    // multi-source batched kernel, a WE run to bc_kernel; sources of batches deeper than
    // the level cap are rerun by bc_kernel (count read on the device).
    const long long km = k - ks;
    bool batched = km > 0 && batch_wanted(g);
    if (batched && !g->bt.failed) {
        rc = alloc_batch(g, km);
        if (rc) {
            if (g->opt.engine == BC_ENGINE_BATCHED) return rc;
            g->bt.failed = 1;  // auto: keep the per-source engine
            free_batch(g);
        }
    }
    batched = batched && g->bt.ready;
    const bool gated = batched && g->opt.engine == BC_ENGINE_AUTO;  // decided by the Alg. 5 flag
    if (km > 0) {
        CK(cudaEventRecord(g->tev[2], st));
        if (!batched || gated) {
            KParams pm = p;
            pm.launch_mode = mode_main;
            pm.src_base = ks;
            pm.k = km;
            pm.work_counter = g->counters + 1;
            pm.skip_if_ep = gated ? 1 : 0;
            if ((rc = launch(g, pm, st))) return rc;
        }
        if (batched) {
            CK(cudaMemsetAsync(g->bt.ovf_n, 0, sizeof(long long), st));
            bcbatch::BParams bp = batch_params(g, d_sources, ks, km, acc_bc);
            bp.sampled_flag = gated ? g->flag : nullptr;
            if ((rc = launch_batch(g, bp, st))) return rc;
            KParams po = p;  // overflow rerun (usually zero sources: the CTAs exit at once)
            po.launch_mode = mode_main;
            po.sources = g->bt.ovf_src;
            po.perm = g->perm;
            po.src_base = 0;
            po.k = km;
            po.k_dev = g->bt.ovf_n;
            po.work_counter = g->counters + 2;
            if ((rc = launch(g, po, st))) return rc;
        }
        CK(cudaEventRecord(g->tev[3], st));
        g->tev_used[1] = 1;
    }
    double h = g->directed ? 1.0 : 0.5;
    // optional k-source estimator scaling (n/k, refs [3],[9]) and the
    // (n-1)(n-2) normalisation of P:74 (applied literally as written in the paper).
    if (g->opt.extrapolate && k > 0) h *= (double)g->n / (double)k;
    if (g->opt.normalize && g->n > 2) h /= ((double)g->n - 1.0) * ((double)g->n - 2.0);
    const int eb = std::min((g->n + 255) / 256, 148 * 8);
    if (g->perm) {
        unpermute_kernel<<<eb, 256, 0, st>>>(acc_bc, g->perm, g->n, h, d_bc);
        CK(cudaGetLastError());
        g->launches++;
    } else if (h != 1.0) {
        scale_kernel<<<eb, 256, 0, st>>>(d_bc, g->n, h);
        CK(cudaGetLastError());
        g->launches++;
    }
    CK(cudaEventRecord(g->done, st));
    return BC_OK;
}

extern "C" int bc_compute_device(bc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc,
                                 void *cuda_stream) {
    if (!g || !d_bc) return fail(BC_EINVAL, "NULL argument");
    if (!d_sources) k = g->n;
    if (k < 0) return fail(BC_EINVAL, "k < 0");
    DeviceGuard dg(g->device);
    int rc = enqueue_compute(g, d_sources, k, d_bc, (cudaStream_t)cuda_stream);
    if (rc == BC_OK) g_err[0] = 0;
    return rc;
}

extern "C" int bc_compute(bc_graph *g, const int32_t *sources, int64_t num_sources, double *bc) {
    if (!g || !bc) return fail(BC_EINVAL, "NULL argument");
    long long k = sources ? num_sources : g->n;
    if (k < 0) return fail(BC_EINVAL, "num_sources < 0");
    if (sources)
        for (long long i = 0; i < k; ++i)
            if (sources[i] < 0 || sources[i] >= g->n)
                return fail(BC_EINVAL, "sources[%lld]=%d out of range", i, sources[i]);
    DeviceGuard dg(g->device);
    CK(cudaEventSynchronize(g->done));
    if (sources && k > g->src_cap) {
        cudaFree(g->src_buf);
        g->src_buf = nullptr;
        g->src_cap = 0;
        CK(cudaMalloc(&g->src_buf, sizeof(int) * (size_t)k));
        g->src_cap = k;
    }
    if (!g->bc_buf) CK(cudaMalloc(&g->bc_buf, sizeof(double) * (size_t)std::max(g->n, 1)));
    if (sources && k > 0)
        CK(cudaMemcpyAsync(g->src_buf, sources, sizeof(int) * (size_t)k, cudaMemcpyHostToDevice, g->stream));
    int rc = enqueue_compute(g, sources ? g->src_buf : nullptr, k, g->bc_buf, g->stream);
    if (rc) return rc;
    if (g->n > 0)
        CK(cudaMemcpyAsync(bc, g->bc_buf, sizeof(double) * (size_t)g->n, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
    g_err[0] = 0;
    return BC_OK;
}

static int single_source_impl(bc_graph *g, int32_t s, int32_t *d, double *sigma, double *delta,
                              uint8_t *level_modes, int32_t max_levels, int32_t *num_levels,
                              int32_t *level_sizes, int64_t *fwd_cycles, int64_t *bwd_cycles) {
    if (!g) return fail(BC_EINVAL, "NULL graph");
    if (s < 0 || s >= g->n) return fail(BC_EINVAL, "source %d out of range", s);
    if (max_levels < 0) return fail(BC_EINVAL, "max_levels < 0");
    DeviceGuard dg(g->device);
    CK(cudaEventSynchronize(g->done));
    const size_t n = (size_t)g->n;
    const bool trace = level_sizes || fwd_cycles || bwd_cycles;
    const int ml = (level_modes || trace) ? max_levels : 0;
    int *dd = nullptr, *dn = nullptr, *dsrc = nullptr, *dls = nullptr;
    double *ds = nullptr, *ddel = nullptr, *dbc = nullptr;
    long long *dfc = nullptr, *dbcyc = nullptr;
    unsigned char *dm = nullptr;
    int rc = BC_OK;
    cudaError_t e = cudaSuccess;
    if (trace) {
        const size_t lv = (size_t)std::max(ml, 1);
        e = cudaMalloc(&dls, lv * sizeof(int));
        if (e == cudaSuccess) e = cudaMalloc(&dfc, lv * sizeof(long long));
        if (e == cudaSuccess) e = cudaMalloc(&dbcyc, lv * sizeof(long long));
        if (e == cudaSuccess) e = cudaMemsetAsync(dbcyc, 0, lv * sizeof(long long), g->stream);
    }
    if (e == cudaSuccess) e = cudaMalloc(&dd, n * sizeof(int));
    if (e == cudaSuccess) e = cudaMalloc(&ds, n * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&ddel, n * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&dbc, n * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&dm, (size_t)std::max(ml, 1));
    if (e == cudaSuccess) e = cudaMalloc(&dn, sizeof(int));
    if (e == cudaSuccess) e = cudaMalloc(&dsrc, sizeof(int));
    if (e == cudaSuccess) e = cudaMemsetAsync(dd, 0xFF, n * sizeof(int), g->stream);  // -1
    if (e == cudaSuccess) e = cudaMemsetAsync(ds, 0, n * sizeof(double), g->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(ddel, 0, n * sizeof(double), g->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(dbc, 0, n * sizeof(double), g->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(dn, 0, sizeof(int), g->stream);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dsrc, &s, sizeof(int), cudaMemcpyHostToDevice, g->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(g->counters, 0, 3 * sizeof(unsigned long long), g->stream);
    DevStats *dst = nullptr;
    if (e == cudaSuccess) e = cudaMalloc(&dst, sizeof(DevStats));
    if (e == cudaSuccess) e = cudaMemsetAsync(dst, 0, sizeof(DevStats), g->stream);
    if (e != cudaSuccess) rc = fail(e == cudaErrorMemoryAllocation ? BC_ENOMEM : BC_ECUDA, "%s", cudaGetErrorString(e));
    if (rc == BC_OK) {
        KParams p = base_params(g, dbc);
        const int strat = g->opt.strategy;
        p.launch_mode = strat == BC_STRATEGY_WE ? LM_WE : strat == BC_STRATEGY_EP ? LM_EP
                      : strat == BC_STRATEGY_HYBRID ? LM_HYBRID : LM_SAMPLED;
        p.sources = dsrc;
        p.src_base = 0;
        p.k = 1;
        p.work_counter = g->counters;
        p.dbg_d = dd;
        p.dbg_sigma = ds;
        p.dbg_delta = ddel;
        p.dbg_modes = dm;
        p.dbg_max_levels = ml;
        p.dbg_nlevels = dn;
        p.dbg_lsizes = dls;
        p.dbg_fcyc = dfc;
        p.dbg_bcyc = dbcyc;
        p.stats = dst;  // keep the last compute call's stats intact
        rc = launch(g, p, g->stream);
    }
    int nl = 0;
    if (rc == BC_OK) {
        e = cudaStreamSynchronize(g->stream);
        // the debug arrays are in internal ids: gather them back to the caller's ids
        const std::vector<int> &pm = g->h_perm;
        auto fetch = [&](void *host, const void *dev, size_t elem) -> cudaError_t {
            if (!host) return cudaSuccess;
            if (!g->perm) return cudaMemcpy(host, dev, n * elem, cudaMemcpyDeviceToHost);
            std::vector<char> tmp(n * elem);
            cudaError_t r = cudaMemcpy(tmp.data(), dev, n * elem, cudaMemcpyDeviceToHost);
            if (r != cudaSuccess) return r;
            char *h = static_cast<char *>(host);
            for (size_t v = 0; v < n; ++v) memcpy(h + v * elem, tmp.data() + (size_t)pm[v] * elem, elem);
            return cudaSuccess;
        };
        if (e == cudaSuccess) e = fetch(d, dd, sizeof(int));
        if (e == cudaSuccess) e = fetch(sigma, ds, sizeof(double));
        if (e == cudaSuccess) e = fetch(delta, ddel, sizeof(double));
        if (e == cudaSuccess) e = cudaMemcpy(&nl, dn, sizeof(int), cudaMemcpyDeviceToHost);
        const size_t nlc = (size_t)std::max(0, std::min(ml, nl));
        if (e == cudaSuccess && level_modes && nlc)
            e = cudaMemcpy(level_modes, dm, nlc, cudaMemcpyDeviceToHost);
        if (e == cudaSuccess && level_sizes && nlc)
            e = cudaMemcpy(level_sizes, dls, nlc * sizeof(int), cudaMemcpyDeviceToHost);
        if (e == cudaSuccess && fwd_cycles && nlc)
            e = cudaMemcpy(fwd_cycles, dfc, nlc * sizeof(long long), cudaMemcpyDeviceToHost);
        if (e == cudaSuccess && bwd_cycles && nlc)
            e = cudaMemcpy(bwd_cycles, dbcyc, nlc * sizeof(long long), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) rc = fail(BC_ECUDA, "%s", cudaGetErrorString(e));
    }
    if (rc == BC_OK && num_levels) *num_levels = nl;
    cudaFree(dls);
    cudaFree(dfc);
    cudaFree(dbcyc);
    cudaFree(dd);
    cudaFree(ds);
    cudaFree(ddel);
    cudaFree(dbc);
    cudaFree(dm);
    cudaFree(dn);
    cudaFree(dsrc);
    cudaFree(dst);
    if (rc == BC_OK) g_err[0] = 0;
    return rc;
}

extern "C" int bc_single_source(bc_graph *g, int32_t s, int32_t *d, double *sigma, double *delta,
                                uint8_t *level_modes, int32_t max_levels, int32_t *num_levels) {
    return single_source_impl(g, s, d, sigma, delta, level_modes, level_modes ? max_levels : 0,
                              num_levels, nullptr, nullptr, nullptr);
}

extern "C" int bc_trace_source(bc_graph *g, int32_t s, int32_t *level_sizes, int64_t *fwd_cycles,
                               int64_t *bwd_cycles, int32_t max_levels, int32_t *num_levels) {
    if (!level_sizes || !fwd_cycles || !bwd_cycles) return fail(BC_EINVAL, "NULL trace array");
    return single_source_impl(g, s, nullptr, nullptr, nullptr, nullptr, max_levels, num_levels,
                              level_sizes, fwd_cycles, bwd_cycles);
}

extern "C" int bc_batch_sources(bc_graph *g, const int32_t *sources, int32_t k, int32_t *d, double *sigma,
                                double *delta) {
    if (!g || !sources) return fail(BC_EINVAL, "NULL argument");
    if (g->directed) return fail(BC_EINVAL, "the batched engine needs an undirected graph");
    if (k < 1 || k > bcbatch::BW) return fail(BC_EINVAL, "k=%d outside 1..64", k);
    for (int i = 0; i < k; ++i)
        if (sources[i] < 0 || sources[i] >= g->n) return fail(BC_EINVAL, "sources[%d]=%d out of range", i, sources[i]);
    DeviceGuard dg(g->device);
    CK(cudaEventSynchronize(g->done));
    int rc = alloc_batch(g, k);
    if (rc) return rc;
    const size_t n = (size_t)g->n, kn = (size_t)k * n;
    int *dsrc = nullptr, *dd = nullptr;
    double *ds = nullptr, *ddel = nullptr, *dbc = nullptr;
    DevStats *dst = nullptr;
    cudaError_t e = cudaMalloc(&dsrc, (size_t)k * sizeof(int));
    if (e == cudaSuccess) e = cudaMalloc(&dd, kn * sizeof(int));
    if (e == cudaSuccess) e = cudaMalloc(&ds, kn * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&ddel, kn * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&dbc, n * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&dst, sizeof(DevStats));
    if (e == cudaSuccess) e = cudaMemcpy(dsrc, sources, (size_t)k * sizeof(int), cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemset(dd, 0xFF, kn * sizeof(int));
    if (e == cudaSuccess) e = cudaMemset(ds, 0, kn * sizeof(double));
    if (e == cudaSuccess) e = cudaMemset(ddel, 0, kn * sizeof(double));
    if (e == cudaSuccess) e = cudaMemset(dbc, 0, n * sizeof(double));
    if (e == cudaSuccess) e = cudaMemset(dst, 0, sizeof(DevStats));
    if (e == cudaSuccess) e = cudaMemset(g->bt.ovf_n, 0, sizeof(long long));
    if (e == cudaSuccess) e = cudaDeviceSynchronize();  // the launch stream does not wait on memsets
    if (e != cudaSuccess) rc = fail(e == cudaErrorMemoryAllocation ? BC_ENOMEM : BC_ECUDA, "%s", cudaGetErrorString(e));
    if (rc == BC_OK) {
        bcbatch::BParams bp = batch_params(g, dsrc, 0, k, dbc);
        bp.stats = dst;
        bp.dbg_d = dd;
        bp.dbg_sigma = ds;
        bp.dbg_delta = ddel;
        const int saved = g->launches, saved_bc = g->bc_launches, saved_ran = g->batch_ran;
        rc = launch_batch(g, bp, g->stream);
        g->launches = saved;
        g->bc_launches = saved_bc;
        g->batch_ran = saved_ran;
    }
    if (rc == BC_OK) {
        long long novf = 0;
        e = cudaStreamSynchronize(g->stream);
        if (e == cudaSuccess) e = cudaMemcpy(&novf, g->bt.ovf_n, sizeof(long long), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) rc = fail(BC_ECUDA, "%s", cudaGetErrorString(e));
        else if (novf) rc = fail(BC_EINVAL, "batch deeper than batch_levels=%d", g->bt.Lcap);
    }
    if (rc == BC_OK) {
        // rows are in internal ids: gather back to the caller's ids
        std::vector<char> tmp(n * sizeof(double));
        auto fetch = [&](void *host, const void *dev, size_t elem) -> cudaError_t {
            if (!host) return cudaSuccess;
            for (int b = 0; b < k; ++b) {
                char *h = static_cast<char *>(host) + (size_t)b * n * elem;
                const char *dv = static_cast<const char *>(dev) + (size_t)b * n * elem;
                if (!g->perm) {
                    cudaError_t r = cudaMemcpy(h, dv, n * elem, cudaMemcpyDeviceToHost);
                    if (r != cudaSuccess) return r;
                    continue;
                }
                cudaError_t r = cudaMemcpy(tmp.data(), dv, n * elem, cudaMemcpyDeviceToHost);
                if (r != cudaSuccess) return r;
                for (size_t v = 0; v < n; ++v) memcpy(h + v * elem, tmp.data() + (size_t)g->h_perm[v] * elem, elem);
            }
            return cudaSuccess;
        };
        e = fetch(d, dd, sizeof(int));
        if (e == cudaSuccess) e = fetch(sigma, ds, sizeof(double));
        if (e == cudaSuccess) e = fetch(delta, ddel, sizeof(double));
        if (e != cudaSuccess) rc = fail(BC_ECUDA, "%s", cudaGetErrorString(e));
    }
    cudaFree(dsrc);
    cudaFree(dd);
    cudaFree(ds);
    cudaFree(ddel);
    cudaFree(dbc);
    cudaFree(dst);
    if (rc == BC_OK) g_err[0] = 0;
    return rc;
}

extern "C" int bc_get_stats(bc_graph *g, bc_stats *st) {
    if (!g || !st) return fail(BC_EINVAL, "NULL argument");
    DeviceGuard dg(g->device);
    CK(cudaEventSynchronize(g->done));
    CK(cudaStreamSynchronize(g->stream));
    DevStats h;
    CK(cudaMemcpy(&h, g->stats, sizeof(h), cudaMemcpyDeviceToHost));
    st->sources = (int64_t)h.sources;
    st->levels = (int64_t)h.levels;
    st->we_levels = (int64_t)h.we_levels;
    st->ep_levels = (int64_t)h.ep_levels;
    st->n_reached = (int64_t)h.n_reached;
    st->arcs_reached = (int64_t)h.arcs_reached;
    st->dag_arcs = (int64_t)h.dag_arcs;
    st->arcs_scanned = (int64_t)h.arcs_scanned;
    const int samp = g->opt.strategy == BC_STRATEGY_SAMPLING && g->sampling_ran;
    st->sampling_ep = samp ? h.sampling_ep : -1;
    st->sampling_median = samp ? h.sampling_median : -1;
    st->sigma_inexact = h.sigma_inexact;
    st->inflight = g->last_inflight;
    st->kernel_launches = g->launches;
    st->bc_kernel_launches = g->bc_launches;
    for (int q = 0; q < 4; ++q) st->phase_cycles[q] = (int64_t)h.phase_cycles[q];
    st->batches = (int64_t)h.batches;
    st->batch_overflows = (int64_t)h.batch_overflows;
    st->engines = g->engines;
    st->pad_ = 0;
    st->dist_sum = (int64_t)h.dist_sum;
    st->handovers = 0;
    st->group_wait_cycles = (int64_t)h.group_wait;
    st->group_mode = (g->engines & 4) ? group_mode(g) : -1;
    st->pad2_ = 0;
    if (g->fb_used) {
        unsigned long long fb = 0;
        CK(cudaMemcpy(&fb, g->fb_n, sizeof(fb), cudaMemcpyDeviceToHost));
        st->handovers = (int64_t)fb;
    }
    st->kernel_ms = 0.0;
    for (int i = 0; i < 2; ++i)
        if (g->tev_used[i]) {
            float ms = 0.f;
            CK(cudaEventElapsedTime(&ms, g->tev[2 * i], g->tev[2 * i + 1]));
            st->kernel_ms += ms;
        }
    return BC_OK;
}
