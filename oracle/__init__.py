"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / ``--impl
reference`` leg may import this package.  It shares no code with the CUDA path
(`paper_conf_ipps_nayyaroddeengk17_b200`), and the product never imports it.

The arithmetic lives in `oracle/oracle.c` (plain single-threaded C, each function
citing PAPER.md); this file only compiles/loads it with gcc and marshals numpy
arrays.  `oracle/brute.py` holds the exhaustive tiny-graph forms used to pin it.

Every function follows one row of DESIGN.md §3 (= SURVEY.md §8(c)):
  decompose  -> D1 RAND (Alg 2), D2 DEGk (Alg 3)
  mis        -> M1 NONE, M2 DEGk, M3 RAND
  mm         -> MM1 NONE, MM2 RAND (Alg 5), MM3 DEGk (Alg 6)
  color      -> C1 NONE, C2 DEGk (Alg 9), C3 RAND (Alg 8)
Parity pins: tests/test_oracle_*.py (none of these functions is "parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

NONE, RAND, DEGK, BRIDGE = 0, 1, 2, 3
# f1 variant flags (the same numbers as SYM_F_* in include/sym.h)
F_PER_ROUND, F_CONFLICT_DROP, F_SPARSER_FIRST, F_LOWER_ONLY = 0x10, 0x20, 0x40, 0x80
F_COLOR_EB, F_COLOR_VB = 0x100, 0x200  # f3: the paper's speculative colouring subroutines
F_ORDER_LF, F_ORDER_SF = 0x400, 0x800  # f2: JP with largest / smallest degree first
KINDS = {"none": NONE, "rand": RAND, "degk": DEGK, "bridge": BRIDGE}
TAG_VERTEX, TAG_EDGE, TAG_RAND = 1, 2, 3

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


_SRC_OMP = os.path.join(_HERE, "oracle_omp.c")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")
_lib_omp = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, single-threaded) -> liboracle.so, and the
    round-based all-core forms (oracle_omp.c + oracle.c, -fopenmp) -> liboracle_omp.so."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    t_omp = os.path.getmtime(_LIB_OMP) if os.path.exists(_LIB_OMP) else -1
    if force or t_omp < max(os.path.getmtime(_SRC), os.path.getmtime(_SRC_OMP)):
        tmp = _LIB_OMP + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-o", tmp, _SRC_OMP, _SRC])
        os.replace(tmp, _LIB_OMP)
    return _LIB


def lib_omp():
    """liboracle_omp.so: LubyMIS / LMAX / JP as synchronous rounds on all host cores."""
    global _lib_omp
    if _lib_omp is None:
        build()
        l = ctypes.CDLL(_LIB_OMP)
        for name in ("oro_mis", "oro_mm", "oro_color"):
            f = getattr(l, name)
            f.restype = None
            f.argtypes = [_I64, _P, _P, _INT, _U32, _U64, _P]
        l.oro_threads.restype = _INT
        l.oro_threads.argtypes = []
        _lib_omp = l
    return _lib_omp


def omp_threads() -> int:
    """Threads the OpenMP round oracle uses (OMP_NUM_THREADS, else every host core)."""
    return int(lib_omp().oro_threads())


_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_U32 = ctypes.c_uint32
_U64 = ctypes.c_uint64
_INT = ctypes.c_int

_SIGS = {
    "or_mix64": (_U64, [_U64]),
    "or_fmix32": (_U32, [_U32]),
    "or_stream_key": (_U64, [_U64, _U32, _U32]),
    "or_pv": (_U32, [_U64, _U32]),
    "or_pe": (_U32, [_U64, _U32, _U32]),
    "or_label": (_U32, [_U64, _U32, _U32]),
    "or_classes": (None, [_I64, _P, _P, _INT, _U32, _U64, _P]),
    "or_decompose": (None, [_I64, _P, _P, _INT, _U32, _U64, _P, _P, _P, _P]),
    "or_mis": (None, [_I64, _P, _P, _INT, _U32, _U64, _P]),
    "or_mm": (None, [_I64, _P, _P, _INT, _U32, _U64, _P]),
    "or_color": (None, [_I64, _P, _P, _INT, _U32, _U64, _P]),
    "or_luby_rounds": (_INT, [_I64, _P, _P, _P, _U64, _P]),
    "or_lmax_rounds": (_INT, [_I64, _P, _P, _U64, _P]),
    "or_jp_rounds": (_INT, [_I64, _P, _P, _U64, _P]),
    "or_cert_mis": (_I64, [_I64, _P, _P, _P, _U64, _P]),
    "or_cert_mm": (_I64, [_I64, _P, _P, _P, _INT, _P, _U64, _P]),
    "or_cert_col": (_I64, [_I64, _P, _P, _P, _P, _INT, _U64, _P]),
    "or_cert_col_rand": (_I64, [_I64, _P, _P, _U32, _U64, _P, _P]),
    "or_cert_flow": (_I64, [_INT, _I64, _P, _P, _INT, _U32, _U64, _P]),
    "or_mis_ex": (None, [_I64, _P, _P, _INT, _U32, _U64, _U32, _P]),
    "or_color_ex": (None, [_I64, _P, _P, _INT, _U32, _U64, _U32, _P]),
    "or_color_spec": (None, [_I64, _P, _P, _INT, _U32, _U64, _U32, _P]),
    "or_color_ord": (None, [_I64, _P, _P, _INT, _U32, _U64, _U32, _P]),
}


def lib():
    global _lib
    if _lib is None:
        l = ctypes.CDLL(build())
        for name, (res, args) in _SIGS.items():
            f = getattr(l, name)
            f.restype = res
            f.argtypes = args
        _lib = l
    return _lib


def _np(x, dtype):
    """torch tensor / array -> contiguous numpy array of dtype (CPU)."""
    if hasattr(x, "detach"):
        x = x.detach().cpu().numpy()
    return np.ascontiguousarray(np.asarray(x, dtype=dtype))


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _graph(rp, ci):
    rp = _np(rp, np.int64)
    ci = _np(ci, np.int32)
    return rp.size - 1, rp, ci


def _kind(kind):
    return KINDS[kind] if isinstance(kind, str) else int(kind)


# ---------------------------------------------------------------- hash contract
def mix64(z: int) -> int:
    return lib().or_mix64(z & (2**64 - 1))


def fmix32(h: int) -> int:
    return lib().or_fmix32(h & 0xFFFFFFFF)


def stream_key(seed: int, tag: int, rnd: int = 0) -> int:
    return lib().or_stream_key(seed & (2**64 - 1), tag, rnd)


def pv(seed: int, v: int) -> int:
    return lib().or_pv(stream_key(seed, TAG_VERTEX), v)


def pe(seed: int, a: int, b: int) -> int:
    lo, hi = min(a, b), max(a, b)
    return lib().or_pe(stream_key(seed, TAG_EDGE), lo, hi)


def label(seed: int, v: int, p: int) -> int:
    return lib().or_label(stream_key(seed, TAG_RAND), v, p)


# ---------------------------------------------------------------- decomposition
def classes(rp, ci, kind, param, seed):
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 0), dtype=np.uint32)
    lib().or_classes(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out


def decompose(rp, ci, kind, param, seed):
    """-> (row_ptr_in, col_in, row_ptr_x, col_x) as numpy arrays."""
    n, rp, ci = _graph(rp, ci)
    nnz = ci.size
    rp_in = np.zeros(n + 1, np.int64)
    rp_x = np.zeros(n + 1, np.int64)
    c_in = np.zeros(max(nnz, 1), np.int32)
    c_x = np.zeros(max(nnz, 1), np.int32)
    lib().or_decompose(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1),
                       _ptr(rp_in), _ptr(c_in), _ptr(rp_x), _ptr(c_x))
    return rp_in, c_in[: rp_in[-1]].copy(), rp_x, c_x[: rp_x[-1]].copy()


# ---------------------------------------------------------------- flows
def mis(rp, ci, kind="none", param=0, seed=42, flags=0):
    """MIS flows (or_mis); flags: the f1 variants (or_mis_ex)."""
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.uint8)
    if flags:
        lib().or_mis_ex(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), flags, _ptr(out))
    else:
        lib().or_mis(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


def mm(rp, ci, kind="none", param=0, seed=42):
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.int32)
    lib().or_mm(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


def color(rp, ci, kind="none", param=0, seed=42, flags=0):
    """COLOR flows (or_color); flags: the f1 variant (or_color_ex) or the f3 speculative
    subroutines EB / VB (or_color_spec)."""
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.uint32)
    if flags & (F_ORDER_LF | F_ORDER_SF):
        lib().or_color_ord(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), flags, _ptr(out))
    elif flags & (F_COLOR_EB | F_COLOR_VB):
        lib().or_color_spec(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), flags, _ptr(out))
    elif flags:
        lib().or_color_ex(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), flags, _ptr(out))
    else:
        lib().or_color(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


def omp_mis(rp, ci, kind="none", param=0, seed=42):
    """MIS flows as synchronous LubyMIS rounds on all cores (oracle_omp.c)."""
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.uint8)
    lib_omp().oro_mis(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


def omp_mm(rp, ci, kind="none", param=0, seed=42):
    """MM flows as synchronous LMAX rounds on all cores (oracle_omp.c)."""
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.int32)
    lib_omp().oro_mm(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


def omp_color(rp, ci, kind="none", param=0, seed=42):
    """COLOR flows as JP levels on all cores (oracle_omp.c)."""
    n, rp, ci = _graph(rp, ci)
    out = np.zeros(max(n, 1), np.uint32)
    lib_omp().oro_color(n, _ptr(rp), _ptr(ci), _kind(kind), param, seed & (2**64 - 1), _ptr(out))
    return out[:n]


# ---------------------------------------------------------------- round forms
def luby_rounds(rp, ci, seed=42, inS=None, status=None):
    n, rp, ci = _graph(rp, ci)
    S = np.ones(max(n, 1), np.uint8) if inS is None else _np(inS, np.uint8)
    st = np.zeros(max(n, 1), np.uint8) if status is None else _np(status, np.uint8).copy()
    r = lib().or_luby_rounds(n, _ptr(rp), _ptr(ci), _ptr(S), seed & (2**64 - 1), _ptr(st))
    return (st[:n] == 1).astype(np.uint8), r


def lmax_rounds(rp, ci, seed=42):
    n, rp, ci = _graph(rp, ci)
    mate = np.zeros(max(n, 1), np.int32)
    r = lib().or_lmax_rounds(n, _ptr(rp), _ptr(ci), seed & (2**64 - 1), _ptr(mate))
    return mate[:n], r


def jp_rounds(rp, ci, seed=42):
    n, rp, ci = _graph(rp, ci)
    C = np.zeros(max(n, 1), np.uint32)
    r = lib().or_jp_rounds(n, _ptr(rp), _ptr(ci), seed & (2**64 - 1), _ptr(C))
    return C[:n], r


# ---------------------------------------------------------------- certificates (full-size parity)
ADMIT_ALL, ADMIT_SAME, ADMIT_DIFF, ADMIT_HH, ADMIT_LX = 0, 1, 2, 3, 4


def cert_mis(rp, ci, in_set, seed, inS=None):
    n, rp, ci = _graph(rp, ci)
    S = np.ones(max(n, 1), np.uint8) if inS is None else _np(inS, np.uint8)
    I = _np(in_set, np.uint8)
    return lib().or_cert_mis(n, _ptr(rp), _ptr(ci), _ptr(S), seed & (2**64 - 1), _ptr(I))


def cert_mm(rp, ci, mate, seed, cls=None, admit=ADMIT_ALL, elig=None):
    n, rp, ci = _graph(rp, ci)
    c = np.zeros(max(n, 1), np.uint32) if cls is None else _np(cls, np.uint32)
    E = np.ones(max(n, 1), np.uint8) if elig is None else _np(elig, np.uint8)
    M = _np(mate, np.int32)
    return lib().or_cert_mm(n, _ptr(rp), _ptr(ci), _ptr(c), admit, _ptr(E), seed & (2**64 - 1), _ptr(M))


def cert_col(rp, ci, C, seed, inS=None, cls=None, admit=ADMIT_ALL):
    n, rp, ci = _graph(rp, ci)
    S = np.ones(max(n, 1), np.uint8) if inS is None else _np(inS, np.uint8)
    c = np.zeros(max(n, 1), np.uint32) if cls is None else _np(cls, np.uint32)
    Cc = _np(C, np.uint32)
    return lib().or_cert_col(n, _ptr(rp), _ptr(ci), _ptr(S), _ptr(c), admit, seed & (2**64 - 1), _ptr(Cc))


def cert_col_rand(rp, ci, C, p, seed):
    """COLOR-Rand certificate in O(m + n) -> (violations, |V'|)."""
    n, rp, ci = _graph(rp, ci)
    Cc = _np(C, np.uint32)
    nconf = ctypes.c_int64(0)
    bad = lib().or_cert_col_rand(n, _ptr(rp), _ptr(ci), int(p), seed & (2**64 - 1), _ptr(Cc), ctypes.byref(nconf))
    return int(bad), int(nconf.value)


def cert_flow(problem, rp, ci, kind, param, seed, result):
    """O(m)-time, O(n)-memory exact check that `result` equals the oracle flow's output,
    phase by phase (oracle.c or_cert_flow; used at full sizes -- up to R-MAT scale 27
    -- where the sequential run's sort is too slow).  Returns the number of violations
    (0 = identical to the oracle)."""
    n, rp, ci = _graph(rp, ci)
    code, dt = {"mis": (1, np.uint8), "mm": (2, np.int32), "color": (3, np.uint32)}[problem]
    R = _np(result, dt)
    return int(lib().or_cert_flow(code, n, _ptr(rp), _ptr(ci), _kind(kind), int(param), seed & (2**64 - 1), _ptr(R)))
