"""CPU test double of the library's sharded flows (TEST INFRASTRUCTURE).

`csrc/{mis,mm,color_shard,shard}.cu` run each rank's round loop inside libsym and,
after every round, exchange only the state changes of the rank's BOUNDARY vertices
(owned vertices with a remote neighbour): an all-gather of {delta count, frontier
count} pairs, then an all-gather of the delta lists padded to the largest count,
applied to the local replicas (shard.cu header).  This module re-implements that
per-rank loop with numpy -- the same shard plan, phase sequences (MIS-Deg2 P:288,
MIS-Rand P:286, MM-Rand Alg 5, COLOR-Degk Alg 9, COLOR-Rand Alg 8), round rules
(Luby P:272-274, handshake P:152-154, JP P:214 with the FIXED priorities of DESIGN §3
H, taken from the oracle's hash contract) and delta protocol -- so that the protocol
can be checked on a machine without a GPU, in one process or over torch.distributed
(gloo) with several processes.  If the boundary deltas did not carry every state a
remote kernel reads, the results would differ from the oracle.
"""
import numpy as np
import torch

import oracle as O
from paper_conf_ipps_nayyaroddeengk17_b200.sharded import shard_block, shard_range

UNDEC, IN, OUT, INACTIVE = 0, 1, 2, 3
NONE, RAND, DEGK = 0, 1, 2
KINDS = {"none": NONE, "rand": RAND, "degk": DEGK}


# ------------------------------------------------------------------ transports
class LocalTransport:
    """All ranks in this process (their steps are called in rank order)."""

    def __init__(self, nranks):
        self.nranks = nranks
        self.pending = {}

    def allgather(self, rank, arr):
        # called for every rank in turn by run_ranks' lock-step driver
        self.pending[rank] = arr
        if len(self.pending) < self.nranks:
            return None
        out = [self.pending[q] for q in range(self.nranks)]
        self.pending = {}
        return out


class GlooTransport:
    """One rank per process: torch.distributed all_gather_into_tensor (gloo)."""

    def __init__(self, nranks):
        self.nranks = nranks

    def allgather(self, rank, arr):
        import torch.distributed as dist
        t = torch.as_tensor(np.ascontiguousarray(arr, dtype=np.int64))
        full = torch.zeros(self.nranks * t.numel(), dtype=torch.int64)
        dist.all_gather_into_tensor(full, t)
        return [full[q * t.numel():(q + 1) * t.numel()].numpy() for q in range(self.nranks)]


# ------------------------------------------------------------------ one rank
class Rank:
    def __init__(self, rp, ci, nranks, rank, kind, param, seed):
        rp, ci = np.asarray(rp), np.asarray(ci)
        self.n = rp.size - 1
        self.N, self.rank = nranks, rank
        self.B = shard_block(self.n, nranks)
        self.v0, self.v1 = shard_range(self.n, nranks, rank)
        a, b = int(rp[self.v0]), int(rp[self.v1])
        self.rp = rp[self.v0:self.v1 + 1] - a  # owned rows, global column ids
        self.ci = ci[a:b]
        self.kind, self.param, self.seed = KINDS[kind] if isinstance(kind, str) else kind, param, seed
        self.pv = {}
        self.exchanged = 0  # delta entries this rank sent
        self.bnd = {v for v in self.owned() if any(not self.v0 <= int(w) < self.v1 for w in self.row(v))}

    def owned(self):
        return range(self.v0, self.v1)

    def row(self, v):
        return self.ci[self.rp[v - self.v0]:self.rp[v - self.v0 + 1]]

    def vkey(self, v):
        if v not in self.pv:
            self.pv[v] = (O.pv(self.seed, int(v)) << 32) | int(v)
        return self.pv[v]

    def label(self, v):
        return O.label(self.seed, int(v), self.param)


def run_ranks(ranks, transport, flow):
    """Drive the flow generator of every rank in lock step (in-process) or the single
    rank of this process (gloo): each `yield (deltas, front)` is one exchange."""
    gens = [flow(r) for r in ranks]
    results = [None] * len(gens)
    sends = [None] * len(gens)
    for i, g in enumerate(gens):
        sends[i] = next(g)
    while True:
        replies = []
        for i, r in enumerate(ranks):
            deltas, front = sends[i]
            r.exchanged += len(deltas)
            pair = np.array([len(deltas), front], dtype=np.int64)
            replies.append(transport.allgather(r.rank, pair))
        pairs = replies[-1]  # every rank receives the same gathered pairs
        maxd = max(int(p[0]) for p in pairs)
        gfront = sum(int(p[1]) for p in pairs)
        gathered = None
        for i, r in enumerate(ranks):
            deltas = sends[i][0]
            width = 2
            pad = np.zeros((maxd, width), dtype=np.int64)
            if deltas:
                pad[:len(deltas)] = np.asarray(deltas, dtype=np.int64).reshape(-1, width)
            gathered = transport.allgather(r.rank, pad.reshape(-1)) if maxd else [np.zeros(0)] * r.N
        done = True
        for i, r in enumerate(ranks):
            received = [(gathered[q].reshape(-1, 2)[:int(pairs[q][0])] if q != r.rank else None)
                        for q in range(r.N)]
            try:
                sends[i] = gens[i].send((gfront, received))
                done = False
            except StopIteration as e:
                results[i] = e.value
        if done:
            return results


# ------------------------------------------------------------------ MIS
def mis_flow(r):
    st = np.zeros(r.N * r.B, dtype=np.uint8)
    hb = {}  # DEGk class of every vertex: owned computed, remote from the setup exchange

    def apply(received):
        for seg in received:
            if seg is None:
                continue
            for v, s in seg:
                st[v] = s

    def in_phase(w, cls):
        return cls < 0 or hb[int(w)] == cls

    def phase(cls):
        lst = [v for v in r.owned() if st[v] == UNDEC and (cls < 0 or hb[v] == cls)]
        while True:
            nxt, deltas = [], []
            for v in lst:
                has_in = blk = False
                for w in r.row(v):
                    w = int(w)
                    if not in_phase(w, cls):
                        continue
                    if st[w] == IN:
                        has_in = True
                    elif st[w] == UNDEC and r.vkey(w) > r.vkey(v):
                        blk = True
                if has_in:
                    st[v] = OUT
                elif blk:
                    nxt.append(v)
                    continue
                else:
                    st[v] = IN
                if v in r.bnd:
                    deltas.append((v, int(st[v])))
            gfront, received = yield deltas, len(nxt)
            apply(received)
            lst = nxt
            if gfront == 0:
                return

    if r.kind == DEGK:
        own = [(v, int(len(r.row(v)) > r.param)) for v in r.owned()]
        for v, c in own:
            hb[v] = c
        _, received = yield [(v, c) for v, c in own], 0  # the class bitmap, gathered once
        for seg in received:
            if seg is not None:
                for v, c in seg:
                    hb[int(v)] = int(c)
        yield from phase(0)
        deltas = []
        for v in r.owned():
            if hb[v] == 1 and st[v] == UNDEC and any(hb[int(w)] == 0 and st[w] == IN for w in r.row(v)):
                st[v] = OUT
                if v in r.bnd:
                    deltas.append((v, OUT))
        _, received = yield deltas, 0
        apply(received)
        yield from phase(1)
    elif r.kind == RAND:
        deltas = []
        for v in r.owned():
            if any(r.label(w) != r.label(v) for w in r.row(v)):
                st[v] = INACTIVE
                if v in r.bnd:
                    deltas.append((v, INACTIVE))
        _, received = yield deltas, 0
        apply(received)
        yield from phase(-1)
        deltas = []
        for v in r.owned():
            if st[v] == INACTIVE:
                st[v] = OUT if any(st[w] == IN for w in r.row(v)) else UNDEC
                if v in r.bnd:
                    deltas.append((v, int(st[v])))
        _, received = yield deltas, 0
        apply(received)
        yield from phase(-1)
    else:
        yield from phase(-1)
    return np.array([1 if st[v] == IN else 0 for v in r.owned()], dtype=np.uint8)


# ------------------------------------------------------------------ MM
def mm_flow(r):
    mate = np.full(r.N * r.B, -1, dtype=np.int64)
    picks = [np.full(r.N * r.B, -1, dtype=np.int64) for _ in range(2)]

    def ekey(u, w):
        return (O.pe(r.seed, int(u), int(w)) << 32) | int(w)

    def phase(admit):
        lst = [u for u in r.owned() if mate[u] < 0 and any(admit(u, w) for w in r.row(u))]
        rnd = 0
        while True:
            prev, cur = picks[(rnd + 1) & 1], picks[rnd & 1]
            nxt, deltas = [], []
            for u in lst:
                reuse = False
                if rnd > 0:
                    p = int(prev[u])
                    if p >= 0 and prev[p] == u:
                        mate[u] = p
                        cur[u] = -1
                    elif mate[u] >= 0:
                        cur[u] = -1
                    elif p >= 0 and mate[p] < 0:
                        cur[u] = p  # the pick is still live: kept (mm.cu)
                        reuse = True
                        nxt.append(u)
                if mate[u] < 0 and not reuse:
                    best = None
                    for w in r.row(u):
                        w = int(w)
                        if admit(u, w) and mate[w] < 0 and (best is None or ekey(u, w) > best):
                            best = ekey(u, w)
                    cur[u] = -1 if best is None else best & 0xFFFFFFFF
                    if best is not None:
                        nxt.append(u)
                if u in r.bnd:
                    deltas.append((u | ((1 << 31) if mate[u] >= 0 else 0), int(cur[u])))
            gfront, received = yield deltas, len(nxt)
            for seg in received:
                if seg is None:
                    continue
                for e, pk in seg:
                    u = int(e) & 0x7FFFFFFF
                    cur[u] = pk
                    if int(e) >> 31:
                        mate[u] = u  # remote entries: only the sign is read
            lst = nxt
            rnd += 1
            if gfront == 0:
                return

    if r.kind == RAND:
        yield from phase(lambda u, w: r.label(u) == r.label(w))
        yield from phase(lambda u, w: r.label(u) != r.label(w))
    else:
        yield from phase(lambda u, w: True)
    return np.array([mate[v] for v in r.owned()], dtype=np.int32)


# ------------------------------------------------------------------ COLOR
def color_flow(r):
    col = np.zeros(r.N * r.B, dtype=np.int64)
    hb = {}

    def cls(v):
        if r.kind == RAND:
            return r.label(v)
        if r.kind == DEGK:
            return hb[int(v)]
        return 0

    def phase(lst, admit_all):
        while True:
            nxt, deltas = [], []
            for v in lst:
                nb = [int(w) for w in r.row(v) if admit_all or cls(w) == cls(v)]
                if any(r.vkey(w) > r.vkey(v) and col[w] == 0 for w in nb):
                    nxt.append(v)
                    continue
                used = {int(col[w]) for w in nb}
                c = 1
                while c in used:
                    c += 1
                col[v] = c
                if v in r.bnd:
                    deltas.append((v, c))
            gfront, received = yield deltas, len(nxt)
            for seg in received:
                if seg is not None:
                    for v, c in seg:
                        col[v] = c
            lst = nxt
            if gfront == 0:
                return

    if r.kind == DEGK:
        own = [(v, int(len(r.row(v)) > r.param)) for v in r.owned()]
        for v, c in own:
            hb[v] = c
        _, received = yield [(v, c) for v, c in own], 0
        for seg in received:
            if seg is not None:
                for v, c in seg:
                    hb[int(v)] = int(c)
    yield from phase(list(r.owned()), r.kind == NONE)
    if r.kind == DEGK:
        mh = max([int(col[v]) for v in r.owned() if hb[v] == 1] or [0])
        _, received = yield [(0, mh)], 0  # all-max of max C_H
        M = max([mh] + [int(c) for seg in received if seg is not None for _, c in seg])
        for v in r.owned():
            if hb[v] == 0:
                col[v] += M
    elif r.kind == RAND:
        vp = [v for v in r.owned() if any(cls(w) != cls(v) and col[w] == col[v] for w in r.row(v))]
        deltas = []
        for v in vp:
            col[v] = 0
            if v in r.bnd:
                deltas.append((v, 0))
        _, received = yield deltas, 0
        for seg in received:
            if seg is not None:
                for v, c in seg:
                    col[v] = c
        yield from phase(vp, True)
    return np.array([col[v] for v in r.owned()], dtype=np.int64)


FLOWS = {"mis": mis_flow, "mm": mm_flow, "color": color_flow}


def run_local(rp, ci, nranks, problem, kind, param, seed):
    ranks = [Rank(rp, ci, nranks, q, kind, param, seed) for q in range(nranks)]
    out = run_ranks(ranks, LocalTransport(nranks), FLOWS[problem])
    return np.concatenate(out), ranks
