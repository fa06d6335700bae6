"""Concurrent schedule of one step of the hot path (MIS-Deg2 + COLOR-Deg2 + MM-Rand4).

The three problems are independent once the DEG2 decomposition exists (P:288, P:234
use it; MM-Rand has its own RAND decomposition), so they run on two CUDA
streams from two host threads (ctypes releases the GIL; the library keeps no
per-call global state and every stream gets its own workspace):

    stream A (high priority): DEG2 decomposition -> COLOR-Deg2.
    stream B:                 RAND4 decomposition -> MM-Rand4 -> MIS-Deg2 (after
                              stream A's decomposition).

This paid off while COLOR's persistent kernel held one 512-thread CTA per SM (levels
JP, 60.4 vs 65.9 ms per step); the early-commit rounds kernel holds two CTAs of 64
registers per thread -- every SM's register file -- so stream B can only interleave
and the step is slower than the five calls in order (51.2 vs 48.8 ms).  bench.py
therefore runs the calls in order by default (--concurrent selects this schedule).

Every call is the public API (sym_decompose / sym_mis / sym_mm / sym_color); results
are bit-identical to running the five calls in order (tests/test_gpu_concurrent.py).
"""
from __future__ import annotations

import concurrent.futures as cf

import torch

from . import sym_color, sym_decompose, sym_mis, sym_mm


class ConcurrentStep:
    def __init__(self, device, seed: int, k: int = 2, p: int = 4):
        self.dev = torch.device(device)
        self.seed, self.k, self.p = seed, k, p
        self.sA = torch.cuda.Stream(self.dev, priority=-1)
        self.sB = torch.cuda.Stream(self.dev)
        self.pool = cf.ThreadPoolExecutor(1)

    def __call__(self, rp: torch.Tensor, ci: torch.Tensor):
        """-> (in_set, color, mate) of MIS-Deg{k}, COLOR-Deg{k}, MM-Rand{p} on (rp, ci)."""
        seed, k, p = self.seed, self.k, self.p
        main = torch.cuda.current_stream(self.dev)
        self.sA.wait_stream(main)
        self.sB.wait_stream(main)
        with torch.cuda.stream(self.sA):
            dD = sym_decompose(rp, ci, "degk", k, seed)
            evD = torch.cuda.Event()
            evD.record(self.sA)

        def side():
            with torch.cuda.device(self.dev), torch.cuda.stream(self.sB):
                dR = sym_decompose(rp, ci, "rand", p, seed)
                M = sym_mm(rp, ci, "rand", p, seed, decomp=dR)
                self.sB.wait_event(evD)
                I = sym_mis(rp, ci, "degk", k, seed, decomp=dD)
            return I, M

        fut = self.pool.submit(side)
        with torch.cuda.stream(self.sA):
            C = sym_color(rp, ci, "degk", k, seed, decomp=dD)
        I, M = fut.result()
        # tensors used on both streams: keep the caching allocator from reusing them early
        for t in (dD.row_ptr_in, dD.col_in, dD.row_ptr_x, dD.col_x, rp, ci):
            t.record_stream(self.sA)
            t.record_stream(self.sB)
        for t in (I, M):
            t.record_stream(self.sB)
        C.record_stream(self.sA)
        main.wait_stream(self.sA)
        main.wait_stream(self.sB)
        return I, C, M


class OverlapStep:
    """The latency-bound prefix of the step on two streams, the colouring alone:

        stream A: DEG2 decomposition -> MIS-Deg2
        stream B: RAND4 decomposition -> MM-Rand4        (a second host thread)
        then, after both:  COLOR-Deg2 on the caller's stream

    The MIS/MM round kernels leave most of the GPU idle (dependent gathers: DRAM 14 %,
    L2 26-28 % busy) and the two splits have different bottlenecks (L2 for DEGk, issue
    for RAND), so the two chains interleave; the JP rounds kernel, which holds every
    SM's register file, runs alone (co-running with it was slower, see ConcurrentStep).
    Every call is the public API; results are bit-identical to the calls in order."""

    def __init__(self, device, seed: int, k: int = 2, p: int = 4):
        self.dev = torch.device(device)
        self.seed, self.k, self.p = seed, k, p
        self.sA = torch.cuda.Stream(self.dev)
        self.sB = torch.cuda.Stream(self.dev)
        self.pool = cf.ThreadPoolExecutor(1)

    def __call__(self, rp: torch.Tensor, ci: torch.Tensor):
        """-> (in_set, color, mate) of MIS-Deg{k}, COLOR-Deg{k}, MM-Rand{p} on (rp, ci)."""
        seed, k, p = self.seed, self.k, self.p
        main = torch.cuda.current_stream(self.dev)
        self.sA.wait_stream(main)
        self.sB.wait_stream(main)

        def side():
            with torch.cuda.device(self.dev), torch.cuda.stream(self.sB):
                dR = sym_decompose(rp, ci, "rand", p, seed)
                return sym_mm(rp, ci, "rand", p, seed, decomp=dR)

        fut = self.pool.submit(side)
        with torch.cuda.stream(self.sA):
            dD = sym_decompose(rp, ci, "degk", k, seed)
            I = sym_mis(rp, ci, "degk", k, seed, decomp=dD)
        M = fut.result()
        for t in (rp, ci):
            t.record_stream(self.sA)
            t.record_stream(self.sB)
        for t in (dD.row_ptr_in, dD.col_in, dD.row_ptr_x, dD.col_x, I):
            t.record_stream(self.sA)
        M.record_stream(self.sB)
        main.wait_stream(self.sA)
        main.wait_stream(self.sB)
        C = sym_color(rp, ci, "degk", k, seed, decomp=dD)
        return I, C, M
