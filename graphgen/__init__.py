"""Seeded synthetic graph generators (shared test/bench input infrastructure).

This module is the ONLY code shared by the CPU oracle side and the CUDA side: it
produces inputs and holds none of the method's arithmetic (no priorities, labels,
MIS/MM/COLOR logic).  Its hash is the generator's own counter-based RNG.

All arithmetic is integer (int64 tensors, 32-bit values masked), so the same call
gives bit-identical CSRs on CPU and on CUDA.  Every graph is returned as a
*canonical* symmetric simple CSR (the precondition of PAPER.md P:126: directed
edges symmetrised, self-loops dropped; rows sorted, no duplicates):

    row_ptr int64[n+1], col_idx int32[nnz]

Families (shapes of the paper's workloads):
  * rmat(scale, ef, seed)          Graph500-parameter R-MAT (a=.57,b=.19,c=.19),
                                   ids permuted by a scale-bit bijection
                                   (kron-g500 analogue)
  * grid(w, h, keep, seed)         4-neighbour grid keeping each edge with prob
                                   `keep` (road-like analogue of road-central,
                                   P:112: avg degree 2.4, %DEG2 50.9)
  * near_regular(n, d, seed)       union of d/2 hash permutations (rgg analogue)
  * tiny families                  path, cycle, star, complete, empty, matching,
                                   gnp (brute-force tier, n <= 12)
"""
from __future__ import annotations

import torch

M32 = 0xFFFFFFFF
GOLDEN64 = 0x9E3779B97F4A7C15


# ----------------------------------------------------------------------------
# generator RNG (its own copy; not the method's priority hash)
# ----------------------------------------------------------------------------
def _py_mix64(z: int) -> int:
    z &= (1 << 64) - 1
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & ((1 << 64) - 1)
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & ((1 << 64) - 1)
    z ^= z >> 31
    return z


def _mul32(a: torch.Tensor, c: int) -> torch.Tensor:
    """(a * c) mod 2^32 for int64 tensors holding values in [0, 2^32), without
    int64 overflow: split a into 16-bit halves."""
    c &= M32
    lo = (a & 0xFFFF) * c
    hi = (((a >> 16) * c) & 0xFFFF) << 16
    return (lo + hi) & M32


def _gmix32(h: torch.Tensor) -> torch.Tensor:
    h = h ^ (h >> 16)
    h = _mul32(h, 0x85EBCA6B)
    h = h ^ (h >> 13)
    h = _mul32(h, 0xC2B2AE35)
    h = h ^ (h >> 16)
    return h


def _stream(seed: int, tag: int, idx: int) -> tuple[int, int]:
    k = _py_mix64(_py_mix64(seed ^ GOLDEN64) ^ ((tag << 40) | idx))
    return k & M32, k >> 32


def _rand32(seed: int, tag: int, idx: int, i: torch.Tensor) -> torch.Tensor:
    """u32 pseudo-random value for counter i (int64 tensor, i < 2^63)."""
    a, b = _stream(seed, tag, idx)
    lo = i & M32
    hi = i >> 32
    return _gmix32(_gmix32(lo ^ a) ^ hi ^ b)


# ----------------------------------------------------------------------------
# CSR assembly
# ----------------------------------------------------------------------------
def csr_from_edges(n: int, src: torch.Tensor, dst: torch.Tensor):
    """Symmetrise, drop self-loops, dedup, sort -> (row_ptr int64[n+1], col_idx int32[nnz])."""
    dev = src.device
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    a = torch.cat([src, dst])
    b = torch.cat([dst, src])
    del src, dst
    key = torch.unique(a * n + b, sorted=True)
    del a, b
    s = key // n
    col = (key - s * n).to(torch.int32)
    deg = torch.bincount(s, minlength=n)
    del s, key
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    torch.cumsum(deg, 0, out=row_ptr[1:])
    return row_ptr, col


def csr_from_edges_bucketed(n: int, src: torch.Tensor, dst: torch.Tensor, nbuckets: int):
    """csr_from_edges for graphs whose arc list does not fit a global sort in memory:
    the arcs are grouped by source-vertex bucket, each bucket is deduplicated and
    sorted on its own.  The result is identical (same canonical CSR)."""
    dev = src.device
    keep = src != dst
    src, dst = src[keep], dst[keep]
    B = (n + nbuckets - 1) // nbuckets
    deg = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    parts = []
    for b in range(nbuckets):
        lo, hi = b * B, min(n, (b + 1) * B)
        if lo >= hi:
            break
        m1 = (src >= lo) & (src < hi)
        m2 = (dst >= lo) & (dst < hi)
        a = torch.cat([src[m1], dst[m2]]).to(torch.int64)
        c = torch.cat([dst[m1], src[m2]]).to(torch.int64)
        del m1, m2
        key = torch.unique((a - lo) * n + c, sorted=True)
        del a, c
        s = key // n
        parts.append((key - s * n).to(torch.int32))
        deg[lo + 1:hi + 1] = torch.bincount(s, minlength=hi - lo)
        del key, s
    row_ptr = torch.cumsum(deg, 0)
    col = torch.empty(int(row_ptr[-1]), dtype=torch.int32, device=dev)
    off = 0
    for p in parts:
        col[off:off + p.numel()] = p
        off += p.numel()
    return row_ptr, col


def _perm_bits(x: torch.Tensor, scale: int, seed: int) -> torch.Tensor:
    """A bijection on [0, 2^scale): two rounds of (odd multiply mod 2^s, xorshift)."""
    if scale == 0:
        return x
    mask = (1 << scale) - 1
    sh = (scale + 1) // 2
    for r in range(2):
        a, b = _stream(seed, 7, r)
        x = _mul32(x, a | 1) & mask
        x = x ^ (b & mask)
        x = x ^ (x >> sh)
    return x


# ----------------------------------------------------------------------------
# families
# ----------------------------------------------------------------------------
RMAT_A, RMAT_B, RMAT_C = 0.57, 0.19, 0.19  # Graph500 parameters
_T1 = int(RMAT_A * 2**32)
_T2 = int((RMAT_A + RMAT_B) * 2**32)
_T3 = int((RMAT_A + RMAT_B + RMAT_C) * 2**32)


def rmat(scale: int, ef: int, seed: int = 1, device="cpu", chunk: int = 1 << 26, buckets: int | None = None):
    """buckets: assemble the CSR in source buckets (default: 1 below scale 26, else 16)
    so that scale 27 (2^31 edges) fits in one GPU's memory; same output either way."""
    n = 1 << scale
    ne = ef << scale
    if buckets is None:
        buckets = 1 if scale < 26 else 16
    small_ids = buckets > 1 and n < 2**31
    srcs, dsts = [], []
    for c0 in range(0, ne, chunk):
        i = torch.arange(c0, min(ne, c0 + chunk), dtype=torch.int64, device=device)
        s = torch.zeros_like(i)
        d = torch.zeros_like(i)
        for lvl in range(scale):
            r = _rand32(seed, 1, lvl, i)
            sb = (r >= _T2).to(torch.int64)                       # quadrants c,d
            db = ((r >= _T1) & (r < _T2)) | (r >= _T3)            # quadrants b,d
            s = (s << 1) | sb
            d = (d << 1) | db.to(torch.int64)
        ps, pd = _perm_bits(s, scale, seed), _perm_bits(d, scale, seed)
        srcs.append(ps.to(torch.int32) if small_ids else ps)
        dsts.append(pd.to(torch.int32) if small_ids else pd)
        del i, s, d, ps, pd
    src = torch.cat(srcs)
    del srcs
    dst = torch.cat(dsts)
    del dsts
    if buckets > 1:
        return csr_from_edges_bucketed(n, src, dst, buckets)
    return csr_from_edges(n, src, dst)


def grid(w: int, h: int, keep: float = 1.0, seed: int = 1, device="cpu"):
    n = w * h
    r = torch.arange(h, dtype=torch.int64, device=device).view(-1, 1)
    c = torch.arange(w, dtype=torch.int64, device=device).view(1, -1)
    hs = (r * w + c)[:, : w - 1].reshape(-1)          # (r,c)-(r,c+1)
    vs = (r * w + c)[: h - 1, :].reshape(-1)          # (r,c)-(r+1,c)
    src = torch.cat([hs, vs])
    dst = torch.cat([hs + 1, vs + w])
    if keep < 1.0:
        eid = torch.cat([hs, vs + n])
        thr = int(keep * 2**32)
        m = _rand32(seed, 2, 0, eid) < thr
        src, dst = src[m], dst[m]
    return csr_from_edges(n, src, dst)


def _hash_perm(n: int, seed: int, j: int, device) -> torch.Tensor:
    i = torch.arange(n, dtype=torch.int64, device=device)
    keys = _rand32(seed, 3, j, i) * (1 << 31) + i   # unique keys
    return torch.argsort(keys)


def near_regular(n: int, d: int, seed: int = 1, device="cpu"):
    i = torch.arange(n, dtype=torch.int64, device=device)
    src = torch.cat([i for _ in range(d // 2)])
    dst = torch.cat([_hash_perm(n, seed, j, device) for j in range(d // 2)])
    return csr_from_edges(n, src, dst)


def path(n, device="cpu"):
    i = torch.arange(max(n - 1, 0), dtype=torch.int64, device=device)
    return csr_from_edges(n, i, i + 1)


def cycle(n, device="cpu"):
    i = torch.arange(n, dtype=torch.int64, device=device)
    return csr_from_edges(n, i, (i + 1) % n)


def star(n, device="cpu"):
    i = torch.arange(1, n, dtype=torch.int64, device=device)
    return csr_from_edges(n, torch.zeros_like(i), i)


def complete(n, device="cpu"):
    a = torch.arange(n, dtype=torch.int64, device=device)
    s, t = torch.meshgrid(a, a, indexing="ij")
    return csr_from_edges(n, s.reshape(-1), t.reshape(-1))


def empty(n, device="cpu"):
    e = torch.zeros(0, dtype=torch.int64, device=device)
    return csr_from_edges(n, e, e)


def matching(n, device="cpu"):
    i = torch.arange(0, n - 1, 2, dtype=torch.int64, device=device)
    return csr_from_edges(n, i, i + 1)


def gnp(n: int, p: float, seed: int = 1, device="cpu"):
    a = torch.arange(n, dtype=torch.int64, device=device)
    s, t = torch.meshgrid(a, a, indexing="ij")
    s, t = s.reshape(-1), t.reshape(-1)
    up = s < t
    s, t = s[up], t[up]
    m = _rand32(seed, 4, n, s * n + t) < int(p * 2**32)
    return csr_from_edges(n, s[m], t[m])


def disjoint_union(*graphs):
    """Disjoint union of CSRs (vertex ids shifted)."""
    rps, cis, off_v, off_e = [], [], 0, 0
    for rp, ci in graphs:
        rps.append(rp[:-1] + off_e)
        cis.append(ci.to(torch.int64) + off_v)
        off_v += rp.numel() - 1
        off_e += int(rp[-1])
    rp = torch.cat(rps + [torch.tensor([off_e], dtype=torch.int64, device=graphs[0][0].device)])
    return rp, torch.cat(cis).to(torch.int32)


def tiny_families(seed: int = 1):
    """(name, (row_ptr, col_idx)) for the brute-force tier (n <= 12)."""
    out = []
    for n in (0, 1, 2, 3, 5, 8):
        out.append((f"path{n}", path(n)))
    for n in (3, 4, 7, 10):
        out.append((f"cycle{n}", cycle(n)))
    for n in (2, 5, 9):
        out.append((f"star{n}", star(n)))
    for n in (1, 4, 6):
        out.append((f"K{n}", complete(n)))
    out.append(("empty6", empty(6)))
    out.append(("matching8", matching(8)))
    for j in range(12):
        n = 5 + (j % 6)
        out.append((f"gnp{n}_{j}", gnp(n, 0.25 + 0.05 * (j % 5), seed=seed + j)))
    out.append(("path3+cycle5+K4", disjoint_union(path(3), cycle(5), complete(4))))
    return out


def checksum(row_ptr: torch.Tensor, col_idx: torch.Tensor) -> int:
    """Order-sensitive 32-bit fold used to compare CPU- and GPU-generated CSRs."""
    def fold(x: torch.Tensor, tag: int) -> int:
        x = x.to(torch.int64)
        i = torch.arange(x.numel(), dtype=torch.int64, device=x.device)
        h = _rand32(tag, 9, 0, (x & M32) ^ _mul32(i & M32, 0x9E3779B1))
        return int((h.sum() & M32).item())
    return fold(row_ptr, 1) ^ (fold(col_idx, 2) * 3 & M32)
