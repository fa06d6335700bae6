"""Sharded MIS over several GPUs (C-ABI: include/sym.h `sym_shard_*`).

One process per GPU.  Rank r owns the 32-aligned vertex block [r*B, min(n, (r+1)*B))
and holds those rows with global column ids; every rank keeps a full replica of the
1-byte MIS status.  Per round each rank runs the Luby round kernel on its owned
frontier (`sym_shard_mis_round`), then the owned status segments are all-gathered
and the next-frontier counts all-reduced -- the only data exchanged (north_star:
"only the boundary vertex-status ... exchanged each round, using NCCL allgather").
MIS-Deg2 applies the DEGk decomposition as a class predicate on the owned
rows: the global V_H bitmap is all-gathered once; phase L on V_L, the fix-up
`sym_shard_mis_kill`, phase R on V_H.  Results equal the single-GPU sym_mis() bit
for bit (fixed priorities make every schedule give the lexicographically-first MIS).

This module is orchestration only: every step of the method runs in libsym.so
kernels (`GpuBackend`); the exchange is a `Transport`:
  * `DistTransport`  -- torch.distributed (NCCL over NVLink on GPUs; gloo in CPU tests)
  * `LocalTransport` -- several shards in one process (single-GPU multi-shard tests)
"""
from __future__ import annotations

import ctypes
import math
from dataclasses import dataclass, field

import torch

from . import _lib as L

ALIGN = 32


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
    row_ptr: torch.Tensor        # local rows, int64[v1 - v0 + 1]
    col_idx: torch.Tensor        # global ids, int32
    v0: int = 0
    v1: int = 0
    block: int = 0
    status: torch.Tensor = None  # replica, uint8[nranks * block]
    hbits: torch.Tensor = None   # int32 words over nranks * block bits
    cur: torch.Tensor = None
    nxt: torch.Tensor = None
    cur_cnt: torch.Tensor = None
    nxt_cnt: torch.Tensor = None
    ws: torch.Tensor = None
    extra: dict = field(default_factory=dict)

    def __post_init__(self):
        self.block = shard_block(self.n_global, self.nranks)
        self.v0, self.v1 = shard_range(self.n_global, self.nranks, self.rank)
        dev = self.row_ptr.device
        pad = self.nranks * self.block
        self.status = torch.zeros(pad, dtype=torch.uint8, device=dev)
        self.hbits = torch.zeros(pad // 32, dtype=torch.int32, device=dev)
        m = max(self.v1 - self.v0, 1)
        self.cur = torch.empty(m, dtype=torch.int32, device=dev)
        self.nxt = torch.empty(m, dtype=torch.int32, device=dev)
        self.cur_cnt = torch.zeros(1, dtype=torch.int32, device=dev)
        self.nxt_cnt = torch.zeros(1, dtype=torch.int32, device=dev)

    @property
    def owned(self) -> slice:
        return slice(self.rank * self.block, (self.rank + 1) * self.block)

    def c_struct(self) -> L.SymGraphShard:
        return L.SymGraphShard(self.n_global, self.v0, self.v1, self.col_idx.numel(), self.row_ptr.data_ptr(),
                               self.col_idx.data_ptr() if self.col_idx.numel() else 0)


# ------------------------------------------------------------------ transports
class LocalTransport:
    """All shards live in this process: the exchange copies owned segments."""

    def allgather(self, shards, attr):
        for s in shards:
            src = getattr(s, attr)
            seg = s.owned if attr == "status" else slice(s.owned.start // 32, s.owned.stop // 32)
            for o in shards:
                if o is not s:
                    getattr(o, attr)[seg].copy_(src[seg])

    def allreduce_sum(self, shards, attr) -> int:
        return int(sum(int(getattr(s, attr)[0]) for s in shards))


class DistTransport:
    """One shard per process; torch.distributed collectives (NCCL on GPUs)."""

    def __init__(self, group=None):
        self.group = group

    def allgather(self, shards, attr):
        import torch.distributed as dist
        (s,) = shards
        full = getattr(s, attr)
        seg = s.owned if attr == "status" else slice(s.owned.start // 32, s.owned.stop // 32)
        mine = full[seg].clone()
        dist.all_gather_into_tensor(full, mine, group=self.group)

    def allreduce_sum(self, shards, attr) -> int:
        import torch.distributed as dist
        (s,) = shards
        t = getattr(s, attr).clone()
        dist.all_reduce(t, group=self.group)
        return int(t[0])


# ------------------------------------------------------------------ GPU backend (libsym.so)
class GpuBackend:
    def __init__(self):
        self.lib = L.load()

    def _s(self, sh):
        return torch.cuda.current_stream(sh.row_ptr.device).cuda_stream

    def _chk(self, rc, what):
        if rc != L.SYM_OK:
            from . import SymError
            raise SymError(rc, what)

    def classify(self, sh: Shard, k: int):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_classify(ctypes.byref(g), k, sh.hbits.data_ptr(), self._s(sh)), "classify")

    def frontier(self, sh: Shard, cls: int):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_frontier(ctypes.byref(g), sh.hbits.data_ptr(), cls, sh.status.data_ptr(),
                                              sh.cur.data_ptr(), sh.cur_cnt.data_ptr(), self._s(sh)), "frontier")

    def round(self, sh: Shard, seed: int, cls: int):
        g = sh.c_struct()
        if sh.ws is None:
            nbytes = self.lib.sym_shard_workspace_bytes(ctypes.byref(g))
            sh.ws = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=sh.row_ptr.device)
        p = L.SymParams(L.NONE, 0, seed & (2**64 - 1), 0, 0)
        self._chk(self.lib.sym_shard_mis_round(ctypes.byref(g), ctypes.byref(p), sh.hbits.data_ptr(), cls,
                                               sh.status.data_ptr(), sh.cur.data_ptr(), sh.cur_cnt.data_ptr(),
                                               sh.nxt.data_ptr(), sh.nxt_cnt.data_ptr(), sh.ws.data_ptr(),
                                               sh.ws.numel(), self._s(sh)), "mis_round")

    def kill(self, sh: Shard):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_mis_kill(ctypes.byref(g), sh.hbits.data_ptr(), sh.status.data_ptr(),
                                              self._s(sh)), "kill")

    def finish(self, sh: Shard) -> torch.Tensor:
        g = sh.c_struct()
        out = torch.empty(max(sh.v1 - sh.v0, 1), dtype=torch.uint8, device=sh.row_ptr.device)
        self._chk(self.lib.sym_shard_mis_finish(ctypes.byref(g), sh.status.data_ptr(), out.data_ptr(), self._s(sh)),
                  "finish")
        return out[: sh.v1 - sh.v0]


# ------------------------------------------------------------------ the flow
def sym_mis_sharded(shards, kind="none", param=0, seed=42, transport=None, backend=None, stats=None):
    """MIS-NONE / MIS-Deg2 over the given shards (all of them in one process with
    LocalTransport, or this rank's single shard with DistTransport).  Returns the
    owned in-set (uint8) of every shard, in the order given."""
    kind = {"none": L.NONE, "degk": L.DEGK}.get(kind, kind) if isinstance(kind, str) else int(kind)
    if kind not in (L.NONE, L.DEGK):
        raise ValueError("sharded MIS supports the NONE and DEGk decompositions")
    transport = transport or LocalTransport()
    backend = backend or GpuBackend()
    for s in shards:
        s.status.zero_()
    if kind == L.DEGK:
        for s in shards:
            backend.classify(s, int(param))
        transport.allgather(shards, "hbits")
        phases = [0, "kill", 1]
    else:
        phases = [-1]
    rounds = []
    for ph in phases:
        if ph == "kill":
            for s in shards:
                backend.kill(s)
            transport.allgather(shards, "status")
            continue
        for s in shards:
            backend.frontier(s, ph)
        r = 0
        while True:
            for s in shards:
                backend.round(s, seed, ph)
            transport.allgather(shards, "status")
            r += 1
            left = transport.allreduce_sum(shards, "nxt_cnt")
            for s in shards:
                s.cur, s.nxt = s.nxt, s.cur
                s.cur_cnt, s.nxt_cnt = s.nxt_cnt, s.cur_cnt
            if left == 0:
                break
        rounds.append(r)
    if stats is not None:
        stats["rounds"] = rounds
    return [backend.finish(s) for s in shards]


def make_shards(row_ptr, col_idx, nranks, ranks=None):
    """Shards of a global CSR (on its device) for the given ranks (default: all)."""
    n = row_ptr.numel() - 1
    out = []
    for r in (range(nranks) if ranks is None else ranks):
        v0, v1 = shard_range(n, nranks, r)
        rp, ci = extract_rows(row_ptr, col_idx, v0, v1)
        out.append(Shard(n, nranks, r, rp, ci))
    return out
