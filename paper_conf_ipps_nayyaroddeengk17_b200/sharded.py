"""Sharded MIS, MM and COLOR over several GPUs (C-ABI: include/sym.h `sym_shard_*`).

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

MM-NONE / MM-Rand (Alg 5) keep replicas of `mate` and of the two pick
buffers; per handshake round (`sym_shard_mm_round`) the owned segments of
the current picks and of mate are all-gathered.  MM-Rand decomposes the owned rows
locally (`sym_shard_decompose`; labels hash the global id): phase 1 on the local
intra CSR, phase 2 on the local cross CSR.  Results equal sym_mm() bit for bit.

COLOR-NONE / COLOR-Degk / COLOR-Rand (Alg 9, Alg 8) keep a
replica of the colour array; per Jones-Plassmann round (`sym_shard_jp_round`) the
owned colour segments are all-gathered.  COLOR-Degk colours G_H and G_L at once
(same-class arcs), all-reduces max C_H and shifts the V_L colours; COLOR-Rand colours
the induced subgraphs, marks and clears V' (monochromatic cross arcs), all-gathers,
and recolours V' against G.  Results equal sym_color() bit for bit.

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
    mate: torch.Tensor = None    # MM: replica, int32[nranks * block]
    picks: list = None           # MM: two pick replicas (round r writes picks[r & 1])
    pick_cur: torch.Tensor = None
    color: torch.Tensor = None   # COLOR: replica, int32 view of uint32[nranks * block]
    cmax: torch.Tensor = None    # COLOR-Degk: owned max colour over V_H (1 element)
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

    def segment(self, attr) -> slice:
        """Owned part of a replica: per-vertex arrays by vertex, the bitmap by word."""
        if attr == "hbits":
            return slice(self.owned.start // 32, self.owned.stop // 32)
        return self.owned

    def c_struct(self) -> L.SymGraphShard:
        return L.SymGraphShard(self.n_global, self.v0, self.v1, self.col_idx.numel(), self.row_ptr.data_ptr(),
                               self.col_idx.data_ptr() if self.col_idx.numel() else 0)

    def init_mm(self):
        dev = self.row_ptr.device
        pad = self.nranks * self.block
        self.mate = torch.full((pad,), -1, dtype=torch.int32, device=dev)
        self.picks = [torch.full((pad,), -1, dtype=torch.int32, device=dev) for _ in range(2)]

    def init_color(self):
        dev = self.row_ptr.device
        self.color = torch.zeros(self.nranks * self.block, dtype=torch.int32, device=dev)
        self.cmax = torch.zeros(1, dtype=torch.int32, device=dev)


@dataclass
class PhaseView:
    """A local phase CSR over the shard's owned rows (global column ids)."""
    shard: Shard
    row_ptr: torch.Tensor
    col_idx: torch.Tensor
    nnz: int

    def c_struct(self) -> L.SymGraphShard:
        sh = self.shard
        return L.SymGraphShard(sh.n_global, sh.v0, sh.v1, self.nnz, self.row_ptr.data_ptr(),
                               self.col_idx.data_ptr() if self.col_idx.numel() else 0)


# ------------------------------------------------------------------ transports
class LocalTransport:
    """All shards live in this process: the exchange copies owned segments."""

    def allgather(self, shards, attr):
        for s in shards:
            src = getattr(s, attr)
            seg = s.segment(attr)
            for o in shards:
                if o is not s:
                    getattr(o, attr)[seg].copy_(src[seg])

    def allreduce_sum(self, shards, attr) -> int:
        return int(sum(int(getattr(s, attr)[0]) for s in shards))

    def allreduce_max(self, shards, attr) -> int:
        return int(max(int(getattr(s, attr)[0]) for s in shards))


class DistTransport:
    """One shard per process; torch.distributed collectives (NCCL on GPUs)."""

    def __init__(self, group=None):
        self.group = group

    def allgather(self, shards, attr):
        import torch.distributed as dist
        (s,) = shards
        full = getattr(s, attr)
        seg = s.segment(attr)
        mine = full[seg].clone()
        dist.all_gather_into_tensor(full, mine, group=self.group)

    def allreduce_sum(self, shards, attr) -> int:
        import torch.distributed as dist
        (s,) = shards
        t = getattr(s, attr).clone()
        dist.all_reduce(t, group=self.group)
        return int(t[0])

    def allreduce_max(self, shards, attr) -> int:
        import torch.distributed as dist
        (s,) = shards
        t = getattr(s, attr).clone()
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=self.group)
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

    # ---- MM
    def decompose(self, sh: Shard, param: int, seed: int):
        """Local RAND decomposition of the owned rows -> (intra, cross) PhaseViews."""
        g = sh.c_struct()
        dev = sh.row_ptr.device
        nl, nnz = sh.v1 - sh.v0, sh.col_idx.numel()
        nbytes = self.lib.sym_shard_decompose_workspace_bytes(ctypes.byref(g))
        ws = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=dev)
        rp_in = torch.empty(nl + 1, dtype=torch.int64, device=dev)
        rp_x = torch.empty(nl + 1, dtype=torch.int64, device=dev)
        ci_in = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)
        ci_x = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)
        p = L.SymParams(L.RAND, int(param), seed & (2**64 - 1), 0, 0)
        self._chk(self.lib.sym_shard_decompose(ctypes.byref(g), ctypes.byref(p), ws.data_ptr(), ws.numel(),
                                               rp_in.data_ptr(), ci_in.data_ptr(), rp_x.data_ptr(), ci_x.data_ptr(),
                                               self._s(sh)), "decompose")
        n_in = int(rp_in[-1])
        return PhaseView(sh, rp_in, ci_in, n_in), PhaseView(sh, rp_x, ci_x, nnz - n_in)

    def mm_frontier(self, view: PhaseView):
        sh = view.shard
        g = view.c_struct()
        self._chk(self.lib.sym_shard_mm_frontier(ctypes.byref(g), sh.mate.data_ptr(), sh.cur.data_ptr(),
                                                 sh.cur_cnt.data_ptr(), self._s(sh)), "mm_frontier")

    def mm_round(self, view: PhaseView, seed: int, r: int):
        sh = view.shard
        g = view.c_struct()
        if sh.extra.get("mm_ws") is None:
            nbytes = self.lib.sym_shard_mm_workspace_bytes(ctypes.byref(sh.c_struct()))
            sh.extra["mm_ws"] = torch.empty(max(nbytes, 256), dtype=torch.uint8, device=sh.row_ptr.device)
        ws = sh.extra["mm_ws"]
        p = L.SymParams(L.NONE, 0, seed & (2**64 - 1), 0, 0)
        self._chk(self.lib.sym_shard_mm_round(ctypes.byref(g), ctypes.byref(p), r, sh.mate.data_ptr(),
                                              sh.picks[(r + 1) & 1].data_ptr(), sh.picks[r & 1].data_ptr(),
                                              sh.cur.data_ptr(), sh.cur_cnt.data_ptr(), sh.nxt.data_ptr(),
                                              sh.nxt_cnt.data_ptr(), ws.data_ptr(), ws.numel(), self._s(sh)),
                  "mm_round")

    # ---- COLOR
    def color_frontier(self, sh: Shard):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_color_frontier(ctypes.byref(g), sh.color.data_ptr(), sh.cur.data_ptr(),
                                                    sh.cur_cnt.data_ptr(), self._s(sh)), "color_frontier")

    def jp_round(self, sh: Shard, kind: int, param: int, seed: int, admit: int):
        g = sh.c_struct()
        p = L.SymParams(kind, int(param), seed & (2**64 - 1), 0, 0)
        self._chk(self.lib.sym_shard_jp_round(ctypes.byref(g), ctypes.byref(p), sh.hbits.data_ptr(), admit,
                                              sh.color.data_ptr(), sh.cur.data_ptr(), sh.cur_cnt.data_ptr(),
                                              sh.nxt.data_ptr(), sh.nxt_cnt.data_ptr(), self._s(sh)), "jp_round")

    def color_conflicts(self, sh: Shard, kind: int, param: int, seed: int):
        g = sh.c_struct()
        p = L.SymParams(kind, int(param), seed & (2**64 - 1), 0, 0)
        self._chk(self.lib.sym_shard_color_conflicts(ctypes.byref(g), ctypes.byref(p), sh.hbits.data_ptr(),
                                                     sh.color.data_ptr(), sh.cur.data_ptr(), sh.cur_cnt.data_ptr(),
                                                     self._s(sh)), "color_conflicts")
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_color_clear(ctypes.byref(g), sh.color.data_ptr(), sh.cur.data_ptr(),
                                                 sh.cur_cnt.data_ptr(), self._s(sh)), "color_clear")

    def color_maxh(self, sh: Shard):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_color_maxh(ctypes.byref(g), sh.hbits.data_ptr(), sh.color.data_ptr(),
                                                sh.cmax.data_ptr(), self._s(sh)), "color_maxh")

    def color_shift(self, sh: Shard, M: int):
        g = sh.c_struct()
        self._chk(self.lib.sym_shard_color_shift(ctypes.byref(g), sh.hbits.data_ptr(), sh.color.data_ptr(), int(M),
                                                 self._s(sh)), "color_shift")


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


def sym_mm_sharded(shards, kind="none", param=0, seed=42, transport=None, backend=None, stats=None):
    """MM-NONE / MM-Rand over the given shards.  Returns the owned mate (int32, -1 =
    unmatched) of every shard, in the order given."""
    kind = {"none": L.NONE, "rand": L.RAND}.get(kind, kind) if isinstance(kind, str) else int(kind)
    if kind not in (L.NONE, L.RAND):
        raise ValueError("sharded MM supports the NONE and RAND decompositions")
    transport = transport or LocalTransport()
    backend = backend or GpuBackend()
    for s in shards:
        s.init_mm()
    if kind == L.RAND:
        views = [backend.decompose(s, int(param), seed) for s in shards]  # per shard: (intra, cross)
        phases = [[v[0] for v in views], [v[1] for v in views]]
    else:
        phases = [[PhaseView(s, s.row_ptr, s.col_idx, s.col_idx.numel()) for s in shards]]
    rounds = []
    for pv in phases:
        for v in pv:
            backend.mm_frontier(v)
        r = 0
        while True:
            for v in pv:
                backend.mm_round(v, seed, r)
            for s in shards:
                s.pick_cur = s.picks[r & 1]
            transport.allgather(shards, "pick_cur")
            transport.allgather(shards, "mate")
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
    return [s.mate[s.v0:s.v1].clone() for s in shards]


def sym_color_sharded(shards, kind="none", param=0, seed=42, transport=None, backend=None, stats=None):
    """COLOR-NONE / COLOR-Degk / COLOR-Rand over the given shards (Jones-Plassmann
    rounds; Alg 9; Alg 8).  Returns the owned colours (int32
    view of uint32, >= 1) of every shard, in the order given; equal to sym_color()."""
    kind = {"none": L.NONE, "rand": L.RAND, "degk": L.DEGK}.get(kind, kind) if isinstance(kind, str) else int(kind)
    if kind not in (L.NONE, L.RAND, L.DEGK):
        raise ValueError("unknown decomposition kind")
    if kind == L.RAND and not 1 <= int(param) <= 65535:
        raise ValueError("RAND needs 1 <= p <= 65535")
    transport = transport or LocalTransport()
    backend = backend or GpuBackend()
    for s in shards:
        s.init_color()
    if kind == L.DEGK:
        for s in shards:
            s.hbits.zero_()
            backend.classify(s, int(param))
        transport.allgather(shards, "hbits")

    def run_phase(admit, fresh):
        if fresh:
            for s in shards:
                backend.color_frontier(s)
        r = 0
        while True:
            for s in shards:
                backend.jp_round(s, kind, param, seed, admit)
            transport.allgather(shards, "color")
            r += 1
            left = transport.allreduce_sum(shards, "nxt_cnt")
            for s in shards:
                s.cur, s.nxt = s.nxt, s.cur
                s.cur_cnt, s.nxt_cnt = s.nxt_cnt, s.cur_cnt
            if left == 0:
                return r

    rounds = [run_phase(0 if kind == L.NONE else 1, True)]
    conflicts = 0
    if kind == L.DEGK:
        for s in shards:
            backend.color_maxh(s)
        M = transport.allreduce_max(shards, "cmax")
        for s in shards:
            backend.color_shift(s, M)
        transport.allgather(shards, "color")
    elif kind == L.RAND:
        for s in shards:
            backend.color_conflicts(s, kind, param, seed)   # V' -> s.cur, then cleared
        transport.allgather(shards, "color")
        conflicts = transport.allreduce_sum(shards, "cur_cnt")
        rounds.append(run_phase(0, False) if conflicts else 0)
    if stats is not None:
        stats["rounds"] = rounds
        stats["conflicts"] = conflicts
    return [s.color[s.v0:s.v1].clone() for s in shards]


def make_shards(row_ptr, col_idx, nranks, ranks=None):
    """Shards of a global CSR (on its device) for the given ranks (default: all)."""
    n = row_ptr.numel() - 1
    out = []
    for r in (range(nranks) if ranks is None else ranks):
        v0, v1 = shard_range(n, nranks, r)
        rp, ci = extract_rows(row_ptr, col_idx, v0, v1)
        out.append(Shard(n, nranks, r, rp, ci))
    return out
