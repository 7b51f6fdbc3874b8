"""Multi-GPU betweenness centrality: one process per GPU, graph replicated,
sources split across ranks, ONE all-reduce of the per-GPU BC vectors.

This is the paper's scale-out: "distributing a subset of roots to
each GPU", the graph "replicated across all GPUs", local BC vectors combined by
MPI_Reduce -- here a single ncclAllReduce (sum, fp64, n) over NVLink/NVSwitch
through torch.distributed.  Each rank runs Alg. 5's sampling on its own first
n_samps sources (the paper is silent on where samples are taken).

Halving is done by every rank before the reduce; fl(a/2 + b/2) =
fl(a + b)/2 exactly, so this equals halving once after the sum.

`bc_step` is THE multi-GPU step: bench.py times it, `bc_distributed` calls it, and
the gloo tests (tests/test_distributed_cpu.py) drive it with a CPU compute.
"""
from __future__ import annotations

from typing import Callable, Optional

import numpy as np

from . import graphgen


def shard_sources(sources: np.ndarray, rank: int, world: int, seed: int = 0) -> np.ndarray:
    """Seeded permutation, then strided assignment sources[rank::world] so cheap
    (isolated / small-component) sources spread evenly over ranks.  A rank may get an
    empty shard (fewer sources than ranks): its partial BC is all zero."""
    if not 0 <= rank < world:
        raise ValueError("rank out of range")
    perm = graphgen.permute_sources(np.asarray(sources, dtype=np.int32), seed)
    return np.ascontiguousarray(perm[rank::world])


def world_info(group=None):
    """(rank, world size) of `group` (the default group), (0, 1) without one."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized():
        return 0, 1
    return dist.get_rank(group), dist.get_world_size(group)


def bc_step(compute_into: Callable, out, group=None):
    """One step of the multi-GPU method: compute_into(out) writes this
    rank's partial BC (its shard of the sources) into `out` (float64[n]), then ONE
    all-reduce (SUM) leaves the full BC on every rank.  Nothing else crosses GPUs."""
    import torch.distributed as dist
    compute_into(out)
    _, world = world_info(group)
    if world > 1:
        dist.all_reduce(out, op=dist.ReduceOp.SUM, group=group)
    return out


def bc_distributed(g, sources: Optional[np.ndarray], *, seed: int = 0, group=None,
                   compute: Optional[Callable] = None, device=None, bcgraph=None):
    """BC over `sources` (None = all vertices) on all ranks of the default process
    group; every rank returns the full reduced BC vector as a torch tensor.

    compute(local_sources) -> float64 tensor [n] (on the reduce device) defaults to
    the CUDA path through `bcgraph` (a BCGraph on this rank's GPU).  Tests inject a
    CPU compute to exercise the sharding and reduction with the gloo backend.

    The n/k estimator option (`extrapolate`, N3) is rejected here: every rank would
    scale its partial sum by n / k_local and the reduced vector would be ~world times
    too large.  Scale the reduced vector by n / len(sources) instead.
    """
    import torch

    rank, world = world_info(group)
    all_src = np.arange(g.n, dtype=np.int32) if sources is None else np.asarray(sources, np.int32)
    local = shard_sources(all_src, rank, world, seed)
    if compute is None:
        if bcgraph is None:
            raise ValueError("bcgraph (a BCGraph on this rank's device) is required")
        if bcgraph.options().get("extrapolate"):
            raise ValueError("extrapolate (n/k per call) is not additive over ranks: switch it "
                             "off and scale the reduced BC by n / len(sources)")
        dev = device or torch.device("cuda", bcgraph.device)
        d_src = torch.from_numpy(local).to(dev)
        out = torch.empty(g.n, dtype=torch.float64, device=dev)
        stream = torch.cuda.current_stream(dev)
        return bc_step(lambda o: bcgraph.compute_device(d_src, o, stream=stream), out, group)
    out = compute(local)  # this rank's partial BC, on the device the group reduces on
    return bc_step(lambda o: None, out, group)
