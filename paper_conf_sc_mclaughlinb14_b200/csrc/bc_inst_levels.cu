// bc_inst_levels.cu -- instantiates bc_kernel for the GlobalLevels level store in
// all block sizes / EP / successor-bitmap variants (one translation unit per store so
// the library compiles in parallel).  No code of its own: see bc_kernels.cuh.
#define BC_INSTANCE_TU
#include "bc_kernels.cuh"

namespace bcdev {
const void *kernel_levels(int nt, bool epok, bool sb) { return kernel_table<false, GlobalLevels>(nt, epok, sb); }
}  // namespace bcdev
