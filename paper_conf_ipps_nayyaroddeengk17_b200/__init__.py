"""symbreak-b200: decomposition-based parallel symmetry breaking on B200 (sm_100a).

Python binding of the C-ABI in include/sym.h (same names; argument marshalling
only -- every step of the hot path runs in the CUDA kernels of libsym.so).  PyTorch
supplies device memory and the current stream.

    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    in_set = sb.sym_mis(row_ptr, col_idx, kind="degk", param=2, seed=42)
    mate   = sb.sym_mm(row_ptr, col_idx, kind="rand", param=4, seed=42)
    color  = sb.sym_color(row_ptr, col_idx, kind="degk", param=2, seed=42)

Graphs are symmetric simple CSRs: row_ptr int64[n+1], col_idx int32[nnz] (rows
sorted).  CUDA tensors are used in place; CPU tensors are copied to the device and
the result is copied back (the end-to-end host path).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import torch

from . import _lib as L

__all__ = ["sym_workspace_bytes", "sym_decompose", "sym_mis", "sym_mm", "sym_color", "sym_validate",
           "sym_version", "Decomposition", "SymError", "KINDS"]

KINDS = {"none": L.NONE, "rand": L.RAND, "degk": L.DEGK, "bridge": L.BRIDGE}


class SymError(RuntimeError):
    def __init__(self, code, where):
        lib = L.load()
        msg = lib.sym_last_error().decode() or lib.sym_error_string(code).decode()
        super().__init__(f"{where}: {lib.sym_error_string(code).decode()} ({code}): {msg}")
        self.code = code


def _kind(kind) -> int:
    return KINDS[kind] if isinstance(kind, str) else int(kind)


def _stream_ptr(device) -> int:
    return torch.cuda.current_stream(device).cuda_stream


_WS: dict = {}


def _workspace(nbytes: int, device) -> torch.Tensor:
    """Per (device, stream) scratch: calls on different streams (e.g. independent problems
    run concurrently from several host threads) never share a workspace."""
    device = torch.device(device)
    key = (device.index, torch.cuda.current_stream(device).cuda_stream)
    buf = _WS.get(key)
    if buf is None or buf.numel() < nbytes:
        _WS.pop(key, None)
        buf = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=device)
        _WS[key] = buf
    return buf


def _graph(row_ptr: torch.Tensor, col_idx: torch.Tensor):
    if row_ptr.dtype != torch.int64 or col_idx.dtype != torch.int32:
        raise TypeError("row_ptr must be int64 and col_idx int32")
    if not (row_ptr.is_contiguous() and col_idx.is_contiguous()):
        raise ValueError("row_ptr / col_idx must be contiguous")
    g = L.SymGraph(row_ptr.numel() - 1, col_idx.numel(), row_ptr.data_ptr(), col_idx.data_ptr() if col_idx.numel() else 0)
    return g


def _to_device(row_ptr, col_idx, device):
    host = not row_ptr.is_cuda
    if host:
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        row_ptr = row_ptr.to(dev, non_blocking=True)
        col_idx = col_idx.to(dev, non_blocking=True)
    return row_ptr, col_idx, host


def _params(kind, param, seed, flags, max_rounds):
    return L.SymParams(_kind(kind), int(param), int(seed) & (2**64 - 1), int(flags), int(max_rounds))


def sym_version() -> str:
    return L.load().sym_version().decode()


def sym_workspace_bytes(row_ptr, col_idx, problem, kind="none", param=0, seed=42, flags=0) -> int:
    g = _graph(row_ptr, col_idx)
    p = _params(kind, param, seed, flags, 0)
    return int(L.load().sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), int(problem)))


@dataclass
class Decomposition:
    """sym_decompose output: intra CSR (induced subgraphs) + cross CSR (cross edges)."""
    kind: int
    param: int
    seed: int
    row_ptr_in: torch.Tensor
    col_in: torch.Tensor
    row_ptr_x: torch.Tensor
    col_x: torch.Tensor
    nnz_in: int
    nnz_x: int
    label: torch.Tensor | None = None

    def c_struct(self) -> L.SymDecomp:
        return L.SymDecomp(self.row_ptr_in.numel() - 1, self.kind, self.param, self.seed,
                           self.row_ptr_in.data_ptr(), self.col_in.data_ptr(),
                           self.row_ptr_x.data_ptr(), self.col_x.data_ptr(),
                           self.nnz_in, self.nnz_x, self.label.data_ptr() if self.label is not None else 0)


def sym_decompose(row_ptr, col_idx, kind, param, seed=42, label=False, flags=0) -> Decomposition:
    lib = L.load()
    g = _graph(row_ptr, col_idx)
    p = _params(kind, param, seed, flags, 0)
    dev = row_ptr.device
    n, nnz = g.n, g.nnz
    out = Decomposition(_kind(kind), int(param), int(seed) & (2**64 - 1),
                        torch.empty(n + 1, dtype=torch.int64, device=dev), torch.empty(max(nnz, 1), dtype=torch.int32, device=dev),
                        torch.empty(n + 1, dtype=torch.int64, device=dev), torch.empty(max(nnz, 1), dtype=torch.int32, device=dev),
                        0, 0, torch.empty(max(n, 1), dtype=torch.int16, device=dev) if label else None)
    ws_n = lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), L.PROBLEM_DECOMPOSE)
    ws = _workspace(ws_n, dev)
    d = out.c_struct()
    with torch.cuda.device(dev):  # the library launches on the current device
        rc = lib.sym_decompose(ctypes.byref(g), ctypes.byref(p), ws.data_ptr(), ws.numel(), ctypes.byref(d),
                               _stream_ptr(dev))
    if rc != L.SYM_OK:
        raise SymError(rc, "sym_decompose")
    out.nnz_in, out.nnz_x = int(d.nnz_in), int(d.nnz_x)
    return out


def _flow(name, problem, out_dtype, row_ptr, col_idx, kind, param, seed, decomp, stats, flags, max_rounds, validate,
          device=None):
    lib = L.load()
    row_ptr, col_idx, host = _to_device(row_ptr, col_idx, device)
    if validate:
        flags |= L.F_VALIDATE
    if decomp is not None:
        flags |= L.F_EXT_DECOMP
    g = _graph(row_ptr, col_idx)
    p = _params(kind, param, seed, flags, max_rounds)
    dev = row_ptr.device
    out = torch.empty(max(g.n, 1), dtype=out_dtype, device=dev)
    ws_n = lib.sym_workspace_bytes(ctypes.byref(g), ctypes.byref(p), problem)
    if ws_n == 0:
        raise SymError(L.SYM_EINVAL, name)
    ws = _workspace(ws_n, dev)
    st = L.SymStats()
    dptr = ctypes.byref(decomp.c_struct()) if decomp is not None else None
    fn = getattr(lib, name)
    with torch.cuda.device(dev):  # the library launches on the current device
        rc = fn(ctypes.byref(g), ctypes.byref(p), dptr, ws.data_ptr(), ws.numel(), out.data_ptr(),
                ctypes.byref(st) if stats else None, _stream_ptr(dev))
    if rc != L.SYM_OK:
        raise SymError(rc, name)
    out = out[: g.n]
    if host:
        out = out.cpu()
    return (out, st.as_dict()) if stats else out


def sym_mis(row_ptr, col_idx, kind="none", param=0, seed=42, decomp=None, stats=False, flags=0, max_rounds=0,
            validate=False, device=None):
    """MIS (LubyMIS / MIS-Rand / MIS-Deg2) -> uint8[n], 1 = in the set."""
    return _flow("sym_mis", L.PROBLEM_MIS, torch.uint8, row_ptr, col_idx, kind, param, seed, decomp, stats, flags,
                 max_rounds, validate, device)


def sym_mm(row_ptr, col_idx, kind="none", param=0, seed=42, decomp=None, stats=False, flags=0, max_rounds=0,
           validate=False, device=None):
    """Maximal matching (LMAX / MM-Rand / MM-Degk) -> int32[n] mate, -1 = unmatched."""
    return _flow("sym_mm", L.PROBLEM_MM, torch.int32, row_ptr, col_idx, kind, param, seed, decomp, stats, flags,
                 max_rounds, validate, device)


def sym_color(row_ptr, col_idx, kind="none", param=0, seed=42, decomp=None, stats=False, flags=0, max_rounds=0,
              validate=False, device=None):
    """Colouring (JP / COLOR-Rand / COLOR-Degk) -> int32[n] colours >= 1 (uint32 in the C-ABI)."""
    return _flow("sym_color", L.PROBLEM_COLOR, torch.int32, row_ptr, col_idx, kind, param, seed, decomp, stats,
                 flags, max_rounds, validate, device)


def sym_profile_enable(on=True) -> None:
    """Record CUDA-event device times per hot-kernel class (measurement hook).
    True / 1: events and the kernels' device byte counters; 2: events only (timing
    without the counters' atomics); False / 0: off."""
    L.load().sym_profile_enable(int(on) if not isinstance(on, bool) else (1 if on else 0))


def sym_profile_collect() -> dict:
    """{class: {"launches", "ms", "alg_bytes", "impl_bytes"}} accumulated since the last collect
    (alg = SURVEY §8(d) algorithmic bytes, impl = the implementation's own words)."""
    lib = L.load()
    buf = (L.SymKernelProfile * 64)()
    cnt = ctypes.c_int(0)
    rc = lib.sym_profile_collect(buf, 64, ctypes.byref(cnt))
    if rc != L.SYM_OK:
        raise SymError(rc, "sym_profile_collect")
    return {buf[i].name.decode(): {"launches": int(buf[i].launches), "ms": float(buf[i].ms),
                                   "alg_bytes": float(buf[i].alg_bytes), "impl_bytes": float(buf[i].impl_bytes)}
            for i in range(min(cnt.value, 64))}


def sym_validate(row_ptr, col_idx) -> int:
    """Number of CSR-precondition violations found on the device (0 = valid)."""
    lib = L.load()
    g = _graph(row_ptr, col_idx)
    ws_n = lib.sym_workspace_bytes(ctypes.byref(g), None, L.PROBLEM_VALIDATE)
    ws = _workspace(ws_n, row_ptr.device)
    bad = ctypes.c_int64(0)
    with torch.cuda.device(row_ptr.device):
        rc = lib.sym_validate(ctypes.byref(g), ws.data_ptr(), ws.numel(), ctypes.byref(bad),
                              _stream_ptr(row_ptr.device))
    if rc not in (L.SYM_OK, L.SYM_EGRAPH):
        raise SymError(rc, "sym_validate")
    return int(bad.value)
