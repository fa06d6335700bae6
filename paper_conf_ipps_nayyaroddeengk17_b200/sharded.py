"""Sharded MIS, MM and COLOR over several GPUs.

Python binding of include/sym.h's `sym_comm_*` and `sym_{mis,mm,color}_sharded`
(argument marshalling only).  One process per GPU: rank r owns the 32-aligned vertex
block [r*B, min(n, (r+1)*B)), B = ceil(n/N) rounded up to 32, and passes those rows
with global column ids.  Each call runs the whole flow inside libsym -- every round,
every fix-up, and after every round the exchange of the state changes of the rank's
boundary vertices (NCCL all-gathers on the caller's stream; csrc/shard.cu).  The
result for the owned rows equals the single-GPU call bit for bit.

    comm = Comm.nccl()                    # torch.distributed initialised; one rank per GPU
    sh = make_shards(row_ptr, col_idx, comm.nranks, ranks=[comm.rank])[0]
    in_set_owned = sym_mis_sharded(sh, comm, "degk", 2, seed=42)

`run_local(shards, problem, ...)` runs N ranks in ONE process (a host thread and a CUDA
stream per rank, `Comm.local` communicators), which is how the multi-rank path is
tested on a single GPU.
"""
from __future__ import annotations

import ctypes
import itertools
import math
import threading
from dataclasses import dataclass

import torch

from . import _lib as L

ALIGN = 32
_KINDS = {"none": L.NONE, "rand": L.RAND, "degk": L.DEGK}


def shard_block(n_global: int, nranks: int) -> int:
    """Vertices per rank: ceil(n / nranks) rounded up to a multiple of 32."""
    b = max(1, math.ceil(n_global / max(nranks, 1)))
    return ((b + ALIGN - 1) // ALIGN) * ALIGN


def shard_range(n_global: int, nranks: int, rank: int) -> tuple[int, int]:
    b = shard_block(n_global, nranks)
    v0 = min(n_global, rank * b)
    return v0, min(n_global, v0 + b)


def extract_rows(row_ptr: torch.Tensor, col_idx: torch.Tensor, v0: int, v1: int):
    """Rows [v0, v1) of a global CSR as a local CSR with global column ids."""
    a, b = int(row_ptr[v0]), int(row_ptr[v1])
    return (row_ptr[v0:v1 + 1] - a).contiguous(), col_idx[a:b].contiguous()


@dataclass
class Shard:
    n_global: int
    nranks: int
    rank: int
    row_ptr: torch.Tensor  # local rows, int64[v1 - v0 + 1]
    col_idx: torch.Tensor  # global ids, int32
    v0: int = 0
    v1: int = 0

    def __post_init__(self):
        self.v0, self.v1 = shard_range(self.n_global, self.nranks, self.rank)

    def c_struct(self) -> L.SymGraphShard:
        return L.SymGraphShard(self.n_global, self.v0, self.v1, self.col_idx.numel(), self.row_ptr.data_ptr(),
                               self.col_idx.data_ptr() if self.col_idx.numel() else 0)


def make_shards(row_ptr, col_idx, nranks, ranks=None):
    """Shards of a global CSR (on its device) for the given ranks (default: all)."""
    n = row_ptr.numel() - 1
    out = []
    for r in (range(nranks) if ranks is None else ranks):
        v0, v1 = shard_range(n, nranks, r)
        rp, ci = extract_rows(row_ptr, col_idx, v0, v1)
        out.append(Shard(n, nranks, r, rp, ci))
    return out


def _check(rc, what):
    if rc != L.SYM_OK:
        from . import SymError
        raise SymError(rc, what)


class Comm:
    """A libsym communicator (sym_comm*)."""

    _local_keys = itertools.count(1)

    def __init__(self, handle, nranks, rank):
        self.handle, self.nranks, self.rank = handle, nranks, rank

    @classmethod
    def nccl(cls, group=None, device=None):
        """NCCL communicator over the ranks of torch.distributed's (default) group: rank 0
        makes the unique id, torch.distributed broadcasts its 128 bytes."""
        import torch.distributed as dist
        lib = L.load()
        rank, nranks = dist.get_rank(group), dist.get_world_size(group)
        uid = (ctypes.c_char * L.COMM_ID_BYTES)()
        if rank == 0:
            _check(lib.sym_comm_unique_id(uid), "sym_comm_unique_id")
        box = [bytes(uid)]
        dist.broadcast_object_list(box, src=0, group=group)
        uid = (ctypes.c_char * L.COMM_ID_BYTES).from_buffer_copy(box[0])
        h = ctypes.c_void_p()
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        with torch.cuda.device(dev):
            _check(lib.sym_comm_create(ctypes.byref(h), nranks, rank, uid), "sym_comm_create")
        return cls(h, nranks, rank)

    @classmethod
    def local_group(cls, nranks):
        """N communicators of one in-process group (ranks driven by N host threads)."""
        lib = L.load()
        key = next(cls._local_keys)
        out = []
        for r in range(nranks):
            h = ctypes.c_void_p()
            _check(lib.sym_comm_create_local(ctypes.byref(h), nranks, r, key), "sym_comm_create_local")
            out.append(cls(h, nranks, r))
        return out

    def close(self):
        if self.handle:
            L.load().sym_comm_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # interpreter shutdown
            pass


_PROBLEMS = {"mis": (L.PROBLEM_MIS, "sym_mis_sharded", torch.uint8),
             "mm": (L.PROBLEM_MM, "sym_mm_sharded", torch.int32),
             "color": (L.PROBLEM_COLOR, "sym_color_sharded", torch.int32)}


def _sharded(problem, shard: Shard, comm: Comm, kind, param, seed, stats, max_rounds):
    lib = L.load()
    code, name, dt = _PROBLEMS[problem]
    kind = _KINDS[kind] if isinstance(kind, str) else int(kind)
    g = shard.c_struct()
    p = L.SymParams(kind, int(param), int(seed) & (2**64 - 1), 0, int(max_rounds))
    dev = shard.row_ptr.device
    nbytes = lib.sym_sharded_workspace_bytes(ctypes.byref(g), ctypes.byref(p), comm.handle, code)
    if nbytes == 0:
        _check(L.SYM_EINVAL, name)
    ws = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = torch.empty(max(shard.v1 - shard.v0, 1), dtype=dt, device=dev)
    st = L.SymShardStats()
    with torch.cuda.device(dev):
        rc = getattr(lib, name)(ctypes.byref(g), ctypes.byref(p), comm.handle, ws.data_ptr(), ws.numel(),
                                out.data_ptr(), ctypes.byref(st), torch.cuda.current_stream(dev).cuda_stream)
    _check(rc, name)
    out = out[: shard.v1 - shard.v0]
    return (out, st.as_dict()) if stats else out


def sym_mis_sharded(shard, comm, kind="none", param=0, seed=42, stats=False, max_rounds=0):
    """MIS (LubyMIS / MIS-Deg2 / MIS-Rand) of the owned rows -> uint8[v1 - v0]."""
    return _sharded("mis", shard, comm, kind, param, seed, stats, max_rounds)


def sym_mm_sharded(shard, comm, kind="none", param=0, seed=42, stats=False, max_rounds=0):
    """Maximal matching (LMAX / MM-Rand) of the owned rows -> int32[v1 - v0] global mates."""
    return _sharded("mm", shard, comm, kind, param, seed, stats, max_rounds)


def sym_color_sharded(shard, comm, kind="none", param=0, seed=42, stats=False, max_rounds=0):
    """Colouring (JP / COLOR-Degk / COLOR-Rand) of the owned rows -> int32[v1 - v0] (uint32 >= 1)."""
    return _sharded("color", shard, comm, kind, param, seed, stats, max_rounds)


def run_local(shards, problem, kind="none", param=0, seed=42, stats=False, max_rounds=0):
    """All ranks of `shards` in this process: one host thread, CUDA stream and local
    communicator per rank (the library's exchange runs between the threads).  Returns
    the owned outputs in shard order (and the per-rank stats)."""
    comms = Comm.local_group(len(shards))
    res, err = [None] * len(shards), [None] * len(shards)

    def work(i):
        try:
            dev = shards[i].row_ptr.device
            s = torch.cuda.Stream(dev)
            s.wait_stream(torch.cuda.current_stream(dev))
            with torch.cuda.stream(s):
                res[i] = _sharded(problem, shards[i], comms[i], kind, param, seed, True, max_rounds)
            s.synchronize()
        except BaseException as e:  # surfaced below
            err[i] = e

    ts = [threading.Thread(target=work, args=(i,)) for i in range(len(shards))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for c in comms:
        c.close()
    for e in err:
        if e is not None:
            raise e
    outs = [r[0] for r in res]
    return (outs, [r[1] for r in res]) if stats else outs
