"""ctypes view of include/sym.h (argument marshalling only; every step runs in libsym.so).

Loading fails loudly if the extension was not built: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SYM_LIB") or os.path.join(HERE, "libsym.so")  # SYM_LIB: diagnostic builds

SYM_OK, SYM_EINVAL, SYM_EWORKSPACE, SYM_EGRAPH, SYM_ECUDA, SYM_ENCCL, SYM_EROUNDS = range(7)
NONE, RAND, DEGK, BRIDGE = 0, 1, 2, 3
PROBLEM_DECOMPOSE, PROBLEM_MIS, PROBLEM_MM, PROBLEM_COLOR, PROBLEM_VALIDATE = range(5)
F_VALIDATE, F_STATS, F_EXT_DECOMP = 0x1, 0x2, 0x4

# every symbol include/sym.h declares (checked by tests/test_abi.py)
EXPORTS = (
    "sym_workspace_bytes", "sym_decompose", "sym_mis", "sym_mm", "sym_color", "sym_validate",
    "sym_error_string", "sym_last_error", "sym_version", "sym_profile_enable", "sym_profile_collect",
    "sym_comm_unique_id", "sym_comm_create", "sym_comm_create_local", "sym_comm_destroy", "sym_comm_size",
    "sym_sharded_workspace_bytes", "sym_mis_sharded", "sym_mm_sharded", "sym_color_sharded",
)
COMM_ID_BYTES = 128


class SymShardStats(ctypes.Structure):
    _fields_ = [("rounds", ctypes.c_uint32 * 3), ("exchanges", ctypes.c_uint32), ("boundary", ctypes.c_int64),
                ("sent_bytes", ctypes.c_int64), ("gathered_bytes", ctypes.c_int64),
                ("max_exchange_bytes", ctypes.c_int64)]

    def as_dict(self):
        return {"rounds": list(self.rounds), "exchanges": self.exchanges, "boundary": self.boundary,
                "sent_bytes": self.sent_bytes, "gathered_bytes": self.gathered_bytes,
                "max_exchange_bytes": self.max_exchange_bytes}


class SymGraphShard(ctypes.Structure):
    _fields_ = [("n_global", ctypes.c_int64), ("v_begin", ctypes.c_int64), ("v_end", ctypes.c_int64),
                ("nnz", ctypes.c_int64), ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p)]


class SymKernelProfile(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 24), ("launches", ctypes.c_int64), ("ms", ctypes.c_double),
                ("alg_bytes", ctypes.c_double), ("impl_bytes", ctypes.c_double)]


class SymGraph(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p)]


class SymParams(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("param", ctypes.c_uint32), ("seed", ctypes.c_uint64),
                ("flags", ctypes.c_uint32), ("max_rounds", ctypes.c_uint32)]


class SymDecomp(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("kind", ctypes.c_int32), ("param", ctypes.c_uint32),
                ("seed", ctypes.c_uint64),
                ("row_ptr_in", ctypes.c_void_p), ("col_in", ctypes.c_void_p),
                ("row_ptr_x", ctypes.c_void_p), ("col_x", ctypes.c_void_p),
                ("nnz_in", ctypes.c_int64), ("nnz_x", ctypes.c_int64),
                ("label", ctypes.c_void_p)]


class SymStats(ctypes.Structure):
    _fields_ = [("rounds", ctypes.c_uint32 * 3), ("phase_vertices", ctypes.c_int64 * 3),
                ("result_size", ctypes.c_int64), ("conflicts", ctypes.c_int64),
                ("max_color", ctypes.c_uint32), ("ms", ctypes.c_float * 4)]

    def as_dict(self):
        return {"rounds": list(self.rounds), "phase_vertices": list(self.phase_vertices),
                "result_size": self.result_size, "conflicts": self.conflicts,
                "max_color": self.max_color}


_lib = None


def load(build_if_missing: bool = False):
    """Load libsym.so (optionally building it first).  Raises if unavailable."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing:
        from . import build as _b
        _b.build()
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libsym.so not built ({LIB_PATH}); run "
                           "`python -m paper_conf_ipps_nayyaroddeengk17_b200.build` -- no CPU fallback exists")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    G = ctypes.POINTER(SymGraph)
    PR = ctypes.POINTER(SymParams)
    D = ctypes.POINTER(SymDecomp)
    S = ctypes.POINTER(SymStats)
    sigs = {
        "sym_workspace_bytes": (ctypes.c_size_t, [G, PR, ctypes.c_int]),
        "sym_decompose": (ctypes.c_int, [G, PR, P, ctypes.c_size_t, D, P]),
        "sym_mis": (ctypes.c_int, [G, PR, D, P, ctypes.c_size_t, P, S, P]),
        "sym_mm": (ctypes.c_int, [G, PR, D, P, ctypes.c_size_t, P, S, P]),
        "sym_color": (ctypes.c_int, [G, PR, D, P, ctypes.c_size_t, P, S, P]),
        "sym_validate": (ctypes.c_int, [G, P, ctypes.c_size_t, ctypes.POINTER(ctypes.c_int64), P]),
        "sym_error_string": (ctypes.c_char_p, [ctypes.c_int]),
        "sym_last_error": (ctypes.c_char_p, []),
        "sym_version": (ctypes.c_char_p, []),
        "sym_comm_unique_id": (ctypes.c_int, [P]),
        "sym_comm_create": (ctypes.c_int, [ctypes.POINTER(P), ctypes.c_int, ctypes.c_int, P]),
        "sym_comm_create_local": (ctypes.c_int, [ctypes.POINTER(P), ctypes.c_int, ctypes.c_int, ctypes.c_uint64]),
        "sym_comm_destroy": (ctypes.c_int, [P]),
        "sym_comm_size": (ctypes.c_int, [P, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_int)]),
        "sym_sharded_workspace_bytes": (ctypes.c_size_t, [ctypes.POINTER(SymGraphShard), PR, P, ctypes.c_int]),
        "sym_mis_sharded": (ctypes.c_int, [ctypes.POINTER(SymGraphShard), PR, P, P, ctypes.c_size_t, P,
                                           ctypes.POINTER(SymShardStats), P]),
        "sym_mm_sharded": (ctypes.c_int, [ctypes.POINTER(SymGraphShard), PR, P, P, ctypes.c_size_t, P,
                                          ctypes.POINTER(SymShardStats), P]),
        "sym_color_sharded": (ctypes.c_int, [ctypes.POINTER(SymGraphShard), PR, P, P, ctypes.c_size_t, P,
                                             ctypes.POINTER(SymShardStats), P]),
        "sym_profile_enable": (ctypes.c_int, [ctypes.c_int]),
        "sym_profile_collect": (ctypes.c_int, [ctypes.POINTER(SymKernelProfile), ctypes.c_int,
                                               ctypes.POINTER(ctypes.c_int)]),
    }
    for name, (res, args) in sigs.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib
