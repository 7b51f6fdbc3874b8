"""Multi-GPU betweenness centrality: one process per GPU, graph replicated,
sources split across ranks, ONE all-reduce of the per-GPU BC vectors.

This is the paper's scale-out: "distributing a subset of roots to
each GPU", the graph "replicated across all GPUs", local BC vectors combined by
MPI_Reduce -- here a single ncclAllReduce (sum, fp64, n) over NVLink/NVSwitch
through torch.distributed.  Each rank runs Alg. 5's sampling on its own first
n_samps sources (the paper is silent on where samples are taken).

Halving is done by every rank before the reduce; fl(a/2 + b/2) =
fl(a + b)/2 exactly, so this equals halving once after the sum.
"""
from __future__ import annotations

from typing import Callable, Optional

import numpy as np

from . import graphgen


def shard_sources(sources: np.ndarray, rank: int, world: int, seed: int = 0) -> np.ndarray:
    """Seeded permutation, then strided assignment sources[rank::world] so cheap
    (isolated / small-component) sources spread evenly over ranks."""
    if not 0 <= rank < world:
        raise ValueError("rank out of range")
    perm = graphgen.permute_sources(np.asarray(sources, dtype=np.int32), seed)
    return np.ascontiguousarray(perm[rank::world])


def bc_distributed(g, sources: Optional[np.ndarray], *, seed: int = 0, group=None,
                   compute: Optional[Callable] = None, device=None, bcgraph=None):
    """BC over `sources` (None = all vertices) on all ranks of the default process
    group; every rank returns the full reduced BC vector as a torch tensor.

    compute(local_sources) -> float64 tensor [n] (on the reduce device) defaults to
    the CUDA path through `bcgraph` (a BCGraph on this rank's GPU).  Tests inject a
    CPU compute to exercise the sharding and reduction with the gloo backend.
    """
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group) if dist.is_initialized() else 0
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    all_src = np.arange(g.n, dtype=np.int32) if sources is None else np.asarray(sources, np.int32)
    local = shard_sources(all_src, rank, world, seed)
    if compute is None:
        if bcgraph is None:
            raise ValueError("bcgraph (a BCGraph on this rank's device) is required")
        dev = device or torch.device("cuda", bcgraph.device)
        d_src = torch.from_numpy(local).to(dev)
        out = torch.empty(g.n, dtype=torch.float64, device=dev)
        bcgraph.compute_device(d_src, out, stream=torch.cuda.current_stream(dev))
    else:
        out = compute(local)
    if world > 1:
        dist.all_reduce(out, op=dist.ReduceOp.SUM, group=group)
    return out
