"""CPU test double of the sharded MIS / MM backend (TEST INFRASTRUCTURE).

Implements the `sym_shard_*` operations with numpy on CPU tensors, following the
same round rules as the CUDA kernels (Luby P:272-274, handshake P:152-154, RAND
labels Alg 2, all with fixed priorities), so
that the multi-process orchestration in `paper_conf_ipps_nayyaroddeengk17_b200.sharded`
(shard plan, status/bitmap/mate/pick all-gathers, count all-reduce, termination,
the MIS-Deg2 and MM-Rand phase sequences) can be exercised with torch.distributed/gloo on a machine without a
GPU.  Priorities come from the oracle's hash contract.
"""
import numpy as np
import torch

import oracle as O

IN, OUT, UNDEC = 1, 2, 0


class CpuBackend:
    def __init__(self, n_global, seed):
        self.n_global, self.seed = n_global, seed
        self._ekeys = {}
        key = O.stream_key(seed, O.TAG_VERTEX)
        self.pv = np.array([O.lib().or_pv(key, v) for v in range(n_global)], dtype=np.uint64)
        self.key = (self.pv << np.uint64(32)) | np.arange(n_global, dtype=np.uint64)

    @staticmethod
    def _bit(hb, v):
        return (int(hb[v >> 5]) >> (v & 31)) & 1

    def classify(self, sh, k):
        rp = sh.row_ptr.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        for v in range(sh.v0, sh.v1):
            if rp[v - sh.v0 + 1] - rp[v - sh.v0] > k:
                hb[v >> 5] |= np.uint32(1 << (v & 31))

    def frontier(self, sh, cls):
        st = sh.status.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        vs = [v for v in range(sh.v0, sh.v1) if st[v] == UNDEC and (cls < 0 or self._bit(hb, v) == cls)]
        sh.cur[: len(vs)] = torch.tensor(vs, dtype=torch.int32)
        sh.cur_cnt[0] = len(vs)

    def round(self, sh, seed, cls):
        rp, ci = sh.row_ptr.numpy(), sh.col_idx.numpy()
        st = sh.status.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        nxt = []
        for v in sh.cur[: int(sh.cur_cnt[0])].tolist():
            if st[v] != UNDEC:
                continue
            has_in = blk = False
            for w in ci[rp[v - sh.v0]: rp[v - sh.v0 + 1]]:
                if cls >= 0 and self._bit(hb, int(w)) != cls:
                    continue
                if st[w] == IN:
                    has_in = True
                elif st[w] == UNDEC and self.key[w] > self.key[v]:
                    blk = True
            if has_in:
                st[v] = OUT
            elif blk:
                nxt.append(v)
            else:
                st[v] = IN
        if nxt:
            sh.nxt[: len(nxt)] = torch.tensor(nxt, dtype=torch.int32)
        sh.nxt_cnt[0] = len(nxt)

    def kill(self, sh):
        rp, ci = sh.row_ptr.numpy(), sh.col_idx.numpy()
        st = sh.status.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        for v in range(sh.v0, sh.v1):
            if self._bit(hb, v) == 1 and st[v] == UNDEC:
                row = ci[rp[v - sh.v0]: rp[v - sh.v0 + 1]]
                if any(self._bit(hb, int(w)) == 0 and st[w] == IN for w in row):
                    st[v] = OUT

    def finish(self, sh):
        return (sh.status[sh.v0:sh.v1] == IN).to(torch.uint8)

    # ---- MM
    def decompose(self, sh, param, seed):
        from paper_conf_ipps_nayyaroddeengk17_b200.sharded import PhaseView
        rp, ci = sh.row_ptr.numpy(), sh.col_idx.numpy()
        lab = {}

        def label(v):
            if v not in lab:
                lab[v] = O.label(seed, v, param)
            return lab[v]
        rin, rx, cin, cx = [0], [0], [], []
        for v in range(sh.v0, sh.v1):
            for w in ci[rp[v - sh.v0]: rp[v - sh.v0 + 1]]:
                (cin if label(int(w)) == label(v) else cx).append(int(w))
            rin.append(len(cin))
            rx.append(len(cx))
        mk = lambda a, dt: torch.tensor(a, dtype=dt)
        return (PhaseView(sh, mk(rin, torch.int64), mk(cin, torch.int32), len(cin)),
                PhaseView(sh, mk(rx, torch.int64), mk(cx, torch.int32), len(cx)))

    def mm_frontier(self, view):
        sh = view.shard
        rp, mate = view.row_ptr.numpy(), sh.mate.numpy()
        vs = [v for v in range(sh.v0, sh.v1) if mate[v] < 0 and rp[v - sh.v0 + 1] > rp[v - sh.v0]]
        sh.cur[: len(vs)] = torch.tensor(vs, dtype=torch.int32)
        sh.cur_cnt[0] = len(vs)

    def _arc_keys(self, view):
        k = id(view.col_idx)
        if k not in self._ekeys:
            sh = view.shard
            rp, ci = view.row_ptr.numpy(), view.col_idx.numpy()
            keys = np.zeros(len(ci), dtype=np.uint64)
            for v in range(sh.v0, sh.v1):
                for a in range(rp[v - sh.v0], rp[v - sh.v0 + 1]):
                    w = int(ci[a])
                    keys[a] = (O.pe(self.seed, v, w) << 32) | w
            self._ekeys[k] = (view.col_idx, keys)  # keep the tensor alive so its id stays unique
        return self._ekeys[k][1]

    def mm_round(self, view, seed, r):
        sh = view.shard
        rp, ci = view.row_ptr.numpy(), view.col_idx.numpy()
        keys = self._arc_keys(view)
        mate = sh.mate.numpy()
        prev, cur = sh.picks[(r + 1) & 1].numpy(), sh.picks[r & 1].numpy()
        nxt = []
        for u in sh.cur[: int(sh.cur_cnt[0])].tolist():
            if r > 0:
                p = prev[u]
                if p >= 0 and prev[p] == u:
                    mate[u] = p
                    cur[u] = -1
                    continue
                if mate[u] >= 0:
                    cur[u] = -1
                    continue
            best = None
            for a in range(rp[u - sh.v0], rp[u - sh.v0 + 1]):
                if mate[ci[a]] < 0 and (best is None or keys[a] > best):
                    best = keys[a]
            cur[u] = -1 if best is None else int(best & np.uint64(0xFFFFFFFF))
            if best is not None:
                nxt.append(u)
        if nxt:
            sh.nxt[: len(nxt)] = torch.tensor(nxt, dtype=torch.int32)
        sh.nxt_cnt[0] = len(nxt)

    # ---- COLOR (JP rounds P:214; Alg 8; Alg 9)
    def _cls(self, kind, param, seed, hb, v):
        if kind == 1:  # RAND
            return O.label(seed, v, param)
        if kind == 2:  # DEGK
            return self._bit(hb, v)
        return 0

    def color_frontier(self, sh):
        col = sh.color.numpy()
        vs = [v for v in range(sh.v0, sh.v1) if col[v] == 0]
        if vs:
            sh.cur[: len(vs)] = torch.tensor(vs, dtype=torch.int32)
        sh.cur_cnt[0] = len(vs)

    def jp_round(self, sh, kind, param, seed, admit):
        rp, ci = sh.row_ptr.numpy(), sh.col_idx.numpy()
        col = sh.color.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        snap = col.copy()  # synchronous round (the kernel may see in-round colours: same result)
        nxt = []
        for v in sh.cur[: int(sh.cur_cnt[0])].tolist():
            cv = self._cls(kind, param, seed, hb, v)
            nb = [int(w) for w in ci[rp[v - sh.v0]: rp[v - sh.v0 + 1]]
                  if admit == 0 or self._cls(kind, param, seed, hb, int(w)) == cv]
            if any(self.key[w] > self.key[v] and snap[w] == 0 for w in nb):
                nxt.append(v)
                continue
            used = {int(snap[w]) for w in nb}
            c = 1
            while c in used:
                c += 1
            col[v] = c
        if nxt:
            sh.nxt[: len(nxt)] = torch.tensor(nxt, dtype=torch.int32)
        sh.nxt_cnt[0] = len(nxt)

    def color_conflicts(self, sh, kind, param, seed):
        rp, ci = sh.row_ptr.numpy(), sh.col_idx.numpy()
        col = sh.color.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        vs = [v for v in range(sh.v0, sh.v1)
              if any(self._cls(kind, param, seed, hb, int(w)) != self._cls(kind, param, seed, hb, v)
                     and col[w] == col[v] for w in ci[rp[v - sh.v0]: rp[v - sh.v0 + 1]])]
        for v in vs:
            col[v] = 0
        if vs:
            sh.cur[: len(vs)] = torch.tensor(vs, dtype=torch.int32)
        sh.cur_cnt[0] = len(vs)

    def color_maxh(self, sh):
        col = sh.color.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        sh.cmax[0] = max([int(col[v]) for v in range(sh.v0, sh.v1) if self._bit(hb, v)] or [0])

    def color_shift(self, sh, M):
        col = sh.color.numpy()
        hb = sh.hbits.numpy().view(np.uint32)
        for v in range(sh.v0, sh.v1):
            if not self._bit(hb, v):
                col[v] += M
