// bc_group.cuh -- the group engine: G groups of CTAs, each group traversing one source at a
// time.
//
// The same per-source Brandes computation as bc_kernel (Alg. 1-3, work-efficient
// levels only), with a source's levels spread over the C = grid / G CTAs of its group
// instead of one CTA.  Only G sources are in flight, so their per-source state (sigma /
// omega f64[n], 2-bit level codes, successor bits) can stay in L2 on graphs whose state is
// far too large for the ~300 sources the per-source engine keeps in flight (n = 2^22:
// 32 MB of sigma per source).  Undirected graphs only (2-bit level codes).
//
// Forward level L (one group barrier per level):
//   (a) every CTA expands the level-L vertices IT owns (row_pass of bc_kernels.cuh: fused
//       discovery + sigma pull); discoveries set the 2-bit code and a bit of the level's
//       discovery bitmap (idempotent ORs, no winner election)
//   (b) group barrier: level L+1 is complete
//   (c) every CTA compacts the bitmap words it owns into S (one atomicAdd on the level's
//       counter reserves its range) and goes straight on to expand them: no second barrier.
// Ownership: vertex v < 32 C (the highest-degree vertices after the internal relabelling)
// belongs to CTA v mod C, the other vertices in blocks of own_block bitmap words dealt out
// round-robin, so hubs spread over the group.  Bitmaps are triple-buffered by level (marks
// of level L+3 may start before every CTA has read level L+1's bits).  Backward level L is
// finished by the CTAs that expanded its vertices in the forward (same ownership), one
// barrier per level.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace bcdev {
struct KParams;
}

namespace bcgroup {

constexpr int CTL_WORDS = 32;  // u64 per group control block (256 B)

struct GParams {
    int groups;                  // G; group g owns CTAs [ceil(g T / G), ceil((g+1) T / G))
    unsigned long long *ctl;     // [G][CTL_WORDS]: [0] barrier count, [8] next source index,
                                 // [16..17] four int32 level counters (ring); zero at launch
    int own_block;               // bitmap words per ownership block (>= 1), see Owned
};

// Level passes of the group kernel: generic row_pass, the fast path (bc_fast.cuh, degree-
// relabelled graphs) or thin rows on virtual warps (bc_thin.cuh, graphs without hubs).
enum : int { GM_GENERIC = 0, GM_FAST = 1, GM_THIN = 2 };
constexpr int THIN_MAX_ROW = 32;  // GM_THIN: longer rows are queued (<= stride_big per CTA), one warp each

// Kernel symbol for a block size (256 or 512 threads); launched cooperatively with
// arguments (KParams, GParams).  KParams: sigma / S / ends / gcodes / nbits (3 buffers of
// nb_words) / sbits are per GROUP (strides stride_n, stride_e, stride_codes, stride_nb,
// stride_sb); bigq is per CTA (stride_big).
const void *group_kernel_fn(int nt, int mode);

}  // namespace bcgroup
