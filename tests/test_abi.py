"""C-ABI checks that need no GPU: libbc.so loads, exports every symbol that
include/bc.h declares, the binding's struct layouts match the header, and the
host-side validation of bc_graph_create rejects malformed CSR input."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bc.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    if not os.path.exists(_bc.LIB_PATH):
        subprocess.check_call(["make", "-C", ROOT, "paper_conf_sc_mclaughlinb14_b200/libbc.so"])
    return _bc.load_library()


def declared_functions():
    text = open(HEADER).read()
    return re.findall(r"BC_API\s+[\w\s\*]+?\b(bc_\w+)\s*\(", text)


def test_header_declares_the_boundary():
    names = set(declared_functions())
    # north_star's three calls plus the build's extensions
    assert {"bc_graph_create", "bc_compute", "bc_destroy"} <= names
    assert {"bc_compute_device", "bc_single_source", "bc_set_options", "bc_get_stats",
            "bc_last_error"} <= names


def test_every_declared_symbol_is_exported(lib):
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    out = subprocess.check_output(["nm", "-D", "--defined-only", _bc.LIB_PATH]).decode()
    exported = set(re.findall(r"\sT\s(bc_\w+)", out))
    for name in declared_functions():
        assert name in exported, name
        assert hasattr(lib, name)
    assert set(_bc.EXPORTED) == set(declared_functions())
    # nothing else leaks (hidden visibility for internals)
    assert exported == set(declared_functions())


def test_struct_layouts_match_header():
    """Compile a tiny C program against bc.h and compare sizeof/offsetof with ctypes."""
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    src = r"""
#include <stdio.h>
#include <stddef.h>
#include "bc.h"
int main(void){
  printf("%zu %zu %zu %zu\n", sizeof(bc_options), offsetof(bc_options, gamma),
         offsetof(bc_options, level_store), sizeof(bc_stats));
  printf("%zu %zu %zu\n", offsetof(bc_stats, sampling_ep), offsetof(bc_stats, inflight),
         offsetof(bc_stats, kernel_ms));
  printf("%zu %zu %d\n", offsetof(bc_options, engine), offsetof(bc_options, group_ctas), BC_ENGINE_GROUP);
  printf("%zu %zu\n", offsetof(bc_stats, dist_sum), offsetof(bc_stats, handovers));
  printf("%zu %zu\n", offsetof(bc_stats, group_wait_cycles), offsetof(bc_stats, group_mode));
  return 0; }
"""
    import tempfile
    with tempfile.TemporaryDirectory() as td:
        c = os.path.join(td, "t.c")
        exe = os.path.join(td, "t")
        open(c, "w").write(src)
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), "-o", exe, c])
        vals = [int(x) for x in subprocess.check_output([exe]).split()]
    O, S = _bc.bc_options, _bc.bc_stats
    assert vals == [ctypes.sizeof(O), O.gamma.offset, O.level_store.offset, ctypes.sizeof(S),
                    S.sampling_ep.offset, S.inflight.offset, S.kernel_ms.offset,
                    O.engine.offset, O.group_ctas.offset, _bc.ENGINES["group"], S.dist_sum.offset, S.handovers.offset,
                    S.group_wait_cycles.offset, S.group_mode.offset]


def test_default_options_are_the_papers(lib):
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    o = _bc.bc_default_options()
    assert (o.strategy, o.alpha, o.beta, o.gamma, o.n_samps, o.ep_min_frontier) == \
        (_bc.BC_STRATEGY_SAMPLING, 768, 512, 4.0, 512, 512)


def test_default_options_overwrite_garbage(lib):
    """A C caller's stack struct holds garbage: bc_default_options must set EVERY field
    (round-1 bug: group_ctas was left as it was)."""
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    o = _bc.bc_options()
    ctypes.memset(ctypes.byref(o), 0xFF, ctypes.sizeof(o))
    lib.bc_default_options(ctypes.byref(o))
    z = _bc.bc_options()
    lib.bc_default_options(ctypes.byref(z))          # from a zeroed struct
    assert bytes(o) == bytes(z)
    assert o.group_ctas == 0 and o.engine == _bc.BC_ENGINE_AUTO and o.hub_chunk == 0


def test_pure_c_caller_compiles_and_links(lib, tmp_path):
    """tests/c/abi_c1.c (a plain C program using only include/bc.h) links against libbc.so;
    the GPU test test_gpu_abi_c.py runs it against the oracle."""
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    exe = tmp_path / "abi_c1"
    build_c_caller(str(exe))
    out = subprocess.check_output(["ldd", str(exe)]).decode()
    assert os.path.realpath(_bc.LIB_PATH) in out or "libbc.so" in out


def build_c_caller(exe):
    pkg = os.path.join(ROOT, "paper_conf_sc_mclaughlinb14_b200")
    subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
                           "-o", exe, os.path.join(ROOT, "tests", "c", "abi_c1.c"),
                           "-L", pkg, "-lbc", "-Wl,-rpath," + pkg, "-lm"])


@pytest.mark.parametrize("case", ["ro0", "ron", "decreasing", "col_range", "neg_n", "big_nnz"])
def test_create_rejects_bad_csr(lib, case):
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    ro = np.array([0, 2, 3, 4], dtype=np.int64)
    col = np.array([1, 2, 0, 1], dtype=np.int32)
    n, nnz = 3, 4
    if case == "ro0":
        ro = ro + 1
    elif case == "ron":
        nnz = 3
    elif case == "decreasing":
        ro = np.array([0, 3, 2, 4], dtype=np.int64)
    elif case == "col_range":
        col = np.array([1, 2, 0, 3], dtype=np.int32)
    elif case == "neg_n":
        n = -1
    elif case == "big_nnz":
        nnz = 1 << 31
    h = ctypes.c_void_p()
    rc = lib.bc_graph_create(n, nnz, ro.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                             col.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), 0, 0,
                             ctypes.byref(h))
    assert rc == _bc.BC_EINVAL
    assert h.value is None
    assert len(_bc.bc_last_error()) > 0


def test_null_arguments(lib):
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    assert lib.bc_graph_create(3, 0, None, None, 0, 0, None) == _bc.BC_EINVAL
    assert lib.bc_compute(None, None, 0, None) == _bc.BC_EINVAL
    assert lib.bc_get_stats(None, None) == _bc.BC_EINVAL
    lib.bc_destroy(None)  # NULL-safe


def test_binding_raises_without_library(tmp_path):
    from paper_conf_sc_mclaughlinb14_b200 import _bc
    saved = _bc._lib
    try:
        _bc._lib = None
        with pytest.raises(RuntimeError):
            _bc.load_library(str(tmp_path / "missing.so"))
    finally:
        _bc._lib = saved
