"""CPU-side checks of the boundary: libsym.so builds for sm_100a, loads without a
GPU, exports every function include/sym.h declares, and its host-only calls
(workspace query, argument errors, version) behave as documented.  No kernel is
launched here."""
import ctypes
import os
import re
import subprocess

import pytest
import torch

import paper_conf_ipps_nayyaroddeengk17_b200 as sb
from paper_conf_ipps_nayyaroddeengk17_b200 import _lib as L
from paper_conf_ipps_nayyaroddeengk17_b200 import build as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sym.h")


@pytest.fixture(scope="module")
def lib():
    B.build()
    return L.load()


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(sym_[a-z_]+)\s*\(", text)))


def test_header_declares_the_survey_boundary():
    names = declared_functions()
    for f in ("sym_decompose", "sym_mis", "sym_mm", "sym_color", "sym_workspace_bytes", "sym_validate"):
        assert f in names


def test_every_declared_symbol_is_exported(lib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", L.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (sym_\w+)", out))
    missing = [f for f in declared_functions() if f not in exported]
    assert not missing, missing
    assert set(L.EXPORTS) == set(declared_functions())


def test_cubin_is_sm100a(lib):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", L.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_version_and_errors(lib):
    assert "sm_100a" in sb.sym_version()
    assert lib.sym_error_string(0) == b"success"
    assert lib.sym_error_string(2) == b"workspace too small"


def _g(n, nnz):
    return L.SymGraph(n, nnz, 0x1000 if n else 0, 0x2000 if nnz else 0)


def test_workspace_query_is_host_only_and_monotone(lib):
    p = L.SymParams(L.DEGK, 2, 42, 0, 0)
    sizes = []
    for n, nnz in ((10, 20), (1000, 20000), (1 << 20, 1 << 24)):
        g = _g(n, nnz)
        s = [lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), prob) for prob in range(5)]
        assert all(x > 0 for x in s)
        sizes.append(s)
    for a, b in zip(sizes, sizes[1:]):
        assert all(x < y for x, y in zip(a[:4], b[:4]))   # validate needs a constant block
        assert a[4] == b[4]
    # an external decomposition shrinks the problem workspaces
    g = _g(1 << 20, 1 << 24)
    pe = L.SymParams(L.DEGK, 2, 42, L.F_EXT_DECOMP, 0)
    assert lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(pe), L.PROBLEM_MIS) < \
        lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), L.PROBLEM_MIS) - 8 * (1 << 24)


def test_argument_errors_before_any_launch(lib):
    g = _g(10, 20)
    bad_p = L.SymParams(L.RAND, 0, 42, 0, 0)       # RAND with p = 0
    assert lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(bad_p), L.PROBLEM_MIS) == 0
    rc = lib.sym_mis(ctypes.byref(g), ctypes.byref(bad_p), None, None, 0, None, None, None)
    assert rc == L.SYM_EINVAL
    assert b"RAND" in lib.sym_last_error()
    ok_p = L.SymParams(L.NONE, 0, 42, 0, 0)
    rc = lib.sym_mis(ctypes.byref(g), ctypes.byref(ok_p), None, None, 0, 0x3000, None, None)
    assert rc == L.SYM_EWORKSPACE
    neg = L.SymGraph(-1, 0, 0, 0)
    assert lib.sym_mm(ctypes.byref(neg), ctypes.byref(ok_p), None, None, 0, None, None, None) == L.SYM_EINVAL
    nullrow = L.SymGraph(5, 0, 0, 0)
    assert lib.sym_color(ctypes.byref(nullrow), ctypes.byref(ok_p), None, None, 0, 0x1, None, None) == L.SYM_EINVAL
    big_p = L.SymParams(L.RAND, 70000, 42, 0, 0)
    assert lib.sym_decompose(ctypes.byref(g), ctypes.byref(big_p), None, 0, None, None) == L.SYM_EINVAL
    # EXT_DECOMP without a decomposition
    ext = L.SymParams(L.DEGK, 2, 42, L.F_EXT_DECOMP, 0)
    assert lib.sym_mis(ctypes.byref(g), ctypes.byref(ext), None, None, 0, 0x3000, None, None) == L.SYM_EINVAL


def test_empty_graph_is_a_noop(lib):
    g = L.SymGraph(0, 0, 0, 0)
    p = L.SymParams(L.NONE, 0, 42, 0, 0)
    ws = lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), L.PROBLEM_MIS)
    assert ws > 0


def test_python_binding_rejects_wrong_dtypes():
    rp = torch.zeros(3, dtype=torch.int32)
    ci = torch.zeros(0, dtype=torch.int32)
    with pytest.raises(TypeError):
        sb.sym_workspace_bytes(rp, ci, L.PROBLEM_MIS)
