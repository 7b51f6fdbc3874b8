"""Multi-process (gloo, world_size 2, CPU) test of the sharding + reduction path.

The per-rank compute is injected (the CPU oracle here, test infrastructure
only); the product path passes a BCGraph on the rank's GPU instead.  Checks that
the strided shards partition the source multiset and that the all-reduced result
equals the single-process BC.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_sc_mclaughlinb14_b200 import distributed as bdist
from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    import torch
    import torch.distributed as dist
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.rmat(9, 16, seed=21)
    S = gg.sample_sources(g, 301, seed=2)
    res = bdist.bc_distributed(g, S, seed=5,
                               compute=lambda loc: torch.from_numpy(oracle.bc(g, loc)))
    np.save(os.path.join(out_dir, f"r{rank}.npy"), res.numpy())
    dist.destroy_process_group()


def test_shards_partition_sources():
    S = np.arange(1000, dtype=np.int32)
    for P in (1, 2, 3, 8):
        parts = [bdist.shard_sources(S, r, P, seed=1) for r in range(P)]
        assert sorted(np.concatenate(parts).tolist()) == S.tolist()
        assert max(p.size for p in parts) - min(p.size for p in parts) <= 1
    with pytest.raises(ValueError):
        bdist.shard_sources(S, 2, 2)


def test_gloo_world2_equals_single_process(tmp_path, oracle_mod):
    port = _free_port()
    mp.spawn(_worker, args=(2, port, str(tmp_path)), nprocs=2, join=True)
    r0 = np.load(tmp_path / "r0.npy")
    r1 = np.load(tmp_path / "r1.npy")
    g = gg.rmat(9, 16, seed=21)
    whole = oracle_mod.bc(g, gg.sample_sources(g, 301, seed=2))
    assert np.array_equal(r0, r1)
    assert np.max(np.abs(r0 - whole) / np.maximum(np.abs(whole), 1)) < 1e-12


def _worker_step(rank, world, port, out_dir, nsrc):
    """Drives distributed.bc_step -- the function bench.py times -- with a CPU compute;
    nsrc < world leaves some ranks with an EMPTY shard (their partial BC must be zero,
    not "all vertices")."""
    import torch
    import torch.distributed as dist
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    cfg, g, total, local = bench.make_workload("c1", world, rank, "strong", nsrc)
    out = torch.empty(g.n, dtype=torch.float64)
    bdist.bc_step(lambda o: o.copy_(torch.from_numpy(oracle.bc(g, local))), out)
    np.save(os.path.join(out_dir, f"s{rank}.npy"), out.numpy())
    np.save(os.path.join(out_dir, f"src{rank}.npy"), local)
    dist.destroy_process_group()


@pytest.mark.parametrize("world,nsrc", [(2, 301), (3, 2)])
def test_gloo_bench_step(tmp_path, oracle_mod, world, nsrc):
    port = _free_port()
    mp.spawn(_worker_step, args=(world, port, str(tmp_path), nsrc), nprocs=world, join=True)
    outs = [np.load(tmp_path / f"s{r}.npy") for r in range(world)]
    shards = [np.load(tmp_path / f"src{r}.npy") for r in range(world)]
    g = gg.CONFIGS["c1"].graph()
    total = gg.sample_sources(g, nsrc, gg.CONFIGS["c1"].seed + 7)
    assert sorted(np.concatenate(shards).tolist()) == sorted(total.tolist())
    if nsrc < world:
        assert min(s.size for s in shards) == 0
    whole = oracle_mod.bc(g, total)
    for o in outs:
        assert np.array_equal(o, outs[0])
        assert np.max(np.abs(o - whole) / np.maximum(np.abs(whole), 1)) < 1e-12
