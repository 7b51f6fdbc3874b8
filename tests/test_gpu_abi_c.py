"""The boundary as a C caller sees it: tests/c/abi_c1.c (plain C, include/bc.h only)
runs bc_graph_create / bc_default_options on a garbage-filled struct / bc_set_options /
bc_compute / bc_get_stats / bc_destroy on c1 and compares every BC value with an
expected file written here by the ORACLE (exact BC, all 1,024 sources)."""
import os
import subprocess

import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
from test_abi import build_c_caller

pytestmark = pytest.mark.gpu


def write_graph(path, g):
    with open(path, "w") as f:
        f.write(f"{g.n} {g.col_indices.size} {int(g.directed)}\n")
        f.write(" ".join(map(str, np.asarray(g.row_offsets, dtype=np.int64).tolist())) + "\n")
        f.write(" ".join(map(str, np.asarray(g.col_indices, dtype=np.int32).tolist())) + "\n")


@pytest.mark.parametrize("key", ["c1", "dir"])
def test_c_caller_against_oracle(tmp_path, oracle_mod, key):
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    g = gg.CONFIGS["c1"].graph() if key == "c1" else gg.rmat(9, 8, seed=4, directed=True)
    gp, ep = tmp_path / "g.txt", tmp_path / "want.txt"
    write_graph(gp, g)
    np.savetxt(ep, oracle_mod.bc(g, None, nthreads=8), fmt="%.17g")
    exe = str(tmp_path / "abi_c1")
    build_c_caller(exe)
    r = subprocess.run([exe, str(gp), str(ep), "1e-9"], capture_output=True, text=True, timeout=300)
    print(r.stdout, r.stderr)
    assert r.returncode == 0, r.stdout + r.stderr
