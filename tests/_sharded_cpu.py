"""CPU test double of the sharded-MIS backend (TEST INFRASTRUCTURE).

Implements the five `sym_shard_*` operations with numpy on CPU tensors, following the
same round rule as the CUDA kernels (P:272-274 with fixed priorities), so
that the multi-process orchestration in `paper_conf_ipps_nayyaroddeengk17_b200.sharded`
(shard plan, status/bitmap all-gathers, count all-reduce, termination, the MIS-Deg2
phase sequence) can be exercised with torch.distributed/gloo on a machine without a
GPU.  Priorities come from the oracle's hash contract.
"""
import numpy as np
import torch

import oracle as O

IN, OUT, UNDEC = 1, 2, 0


class CpuBackend:
    def __init__(self, n_global, seed):
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
