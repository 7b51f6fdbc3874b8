"""B200-native betweenness centrality (McLaughlin & Bader, SC'14 hot path).

The compute path is libbc.so (CUDA, sm_100a) behind the C ABI in include/bc.h;
`_bc` is its ctypes binding, `graphgen` the seeded synthetic inputs and
`distributed` the multi-GPU source sharding + NCCL reduction.
"""
from ._bc import (BATCH_WIDTH, BCError, BCGraph, ENGINES, LIB_PATH, STRATEGIES, bc_batch_sources, bc_compute, bc_compute_device,  # noqa: F401
                  bc_default_options, bc_destroy, bc_get_options, bc_get_stats, bc_graph_create,
                  bc_last_error, bc_set_options, bc_single_source, bc_trace_source,
                  load_library)

__all__ = ["BCGraph", "BCError", "bc_graph_create", "bc_compute", "bc_compute_device",
           "bc_single_source", "bc_trace_source", "bc_batch_sources", "ENGINES", "BATCH_WIDTH", "bc_default_options", "bc_set_options", "bc_get_options",
           "bc_get_stats", "bc_destroy", "bc_last_error", "load_library", "LIB_PATH", "STRATEGIES"]
