"""Exhaustive tiny-graph forms (n <= 12) -- TEST INFRASTRUCTURE ONLY.

These characterise the lexicographically-first results by enumeration rather than
by the greedy loop, so they pin `oracle/oracle.c` from outside:

* LF-MIS(G)  = the maximal independent set whose indicator vector, read in
               decreasing (pv, id) order, is lexicographically largest
               (fixed-priority LubyMIS == greedy MIS, Blelloch et al. [6]);
* LF-MM(G)   = the maximal matching whose indicator vector over edges in
               decreasing (pe, lo, hi) order is lexicographically largest
               (GM / LMAX with fixed edge priorities);
* LF-COL(G)  = the proper colouring with colours >= 1 whose colour vector, read in
               decreasing (pv, id) order, is lexicographically smallest (first-fit
               JP).

Priorities come from the oracle's hash contract (pinned separately by published
test vectors).
"""
from __future__ import annotations

import itertools

import numpy as np

from . import pe, pv


def adjacency(rp, ci):
    rp = np.asarray(rp, dtype=np.int64)
    ci = np.asarray(ci, dtype=np.int64)
    n = rp.size - 1
    return n, [set(int(w) for w in ci[rp[v]:rp[v + 1]]) for v in range(n)]


def vertex_order(n, seed):
    return sorted(range(n), key=lambda v: (pv(seed, v), v), reverse=True)


def edge_list(adj):
    return sorted({(min(u, w), max(u, w)) for u in range(len(adj)) for w in adj[u]})


def all_mis(adj):
    n = len(adj)
    for mask in range(1 << n):
        S = [v for v in range(n) if mask >> v & 1]
        if any(w in adj[v] for v in S for w in S):
            continue
        if all((mask >> v & 1) or any(mask >> w & 1 for w in adj[v]) for v in range(n)):
            yield frozenset(S)


def brute_lf_mis(rp, ci, seed):
    n, adj = adjacency(rp, ci)
    order = vertex_order(n, seed)
    best = max(all_mis(adj), key=lambda S: tuple(1 if v in S else 0 for v in order))
    out = np.zeros(n, np.uint8)
    for v in best:
        out[v] = 1
    return out


def all_maximal_matchings(adj):
    E = edge_list(adj)
    for mask in range(1 << len(E)):
        M = [E[i] for i in range(len(E)) if mask >> i & 1]
        used = [x for e in M for x in e]
        if len(used) != len(set(used)):
            continue
        cov = set(used)
        if all(u in cov or w in cov for (u, w) in E):
            yield M


def brute_lf_mm(rp, ci, seed):
    n, adj = adjacency(rp, ci)
    E = edge_list(adj)
    assert len(E) <= 18, "brute force limited to <= 18 edges"
    order = sorted(E, key=lambda e: (pe(seed, *e), e[0], e[1]), reverse=True)
    best = max(all_maximal_matchings(adj), key=lambda M: tuple(1 if e in M else 0 for e in order))
    mate = np.full(n, -1, np.int32)
    for u, w in best:
        mate[u], mate[w] = w, u
    return mate


def brute_lf_col(rp, ci, seed):
    """lexicographically smallest proper colouring (colours 1..n) in priority order;
    exhaustive over n^n assignments (n <= 6)."""
    n, adj = adjacency(rp, ci)
    assert n <= 6
    order = vertex_order(n, seed)
    best = None
    for cols in itertools.product(range(1, n + 1), repeat=n):   # cols[i] = colour of order[i]
        c = {order[i]: cols[i] for i in range(n)}
        if all(c[u] != c[w] for u in range(n) for w in adj[u]):
            best = cols          # product() enumerates in lexicographic order
            break
    out = np.zeros(n, np.uint32)
    if best is not None:
        for i, v in enumerate(order):
            out[v] = best[i]
    return out
