"""Brute-force tier (n <= 12): the oracle's sequential forms against exhaustive
enumeration (oracle/brute.py) and networkx, for every tiny family and method seed.

Pins:
* M1/MM1/C1  == lexicographically-first MIS / maximal matching / colouring found
  by enumeration (Blelloch et al. [6]);
* C1         == networkx greedy_color with the same vertex order (+1, colour base 1);
* M2/M3/MM2/MM3/C2/C3 == the two-stage definitions of P:162-178, P:226-234,
  P:286-288 evaluated by enumeration on the explicit subgraphs.
"""
import networkx as nx
import numpy as np
import pytest

import graphgen as G
import oracle as O
from oracle import brute as B
from conftest import SEEDS

FAMS = G.tiny_families()


def _nx(rp, ci):
    n, adj = B.adjacency(rp, ci)
    g = nx.Graph()
    g.add_nodes_from(range(n))
    g.add_edges_from(B.edge_list(adj))
    return g


def _sub_csr(n, edges):
    """CSR on n vertices from an undirected edge list."""
    adj = [[] for _ in range(n)]
    for u, w in edges:
        adj[u].append(w)
        adj[w].append(u)
    rp = np.zeros(n + 1, np.int64)
    ci = []
    for v in range(n):
        ci += sorted(adj[v])
        rp[v + 1] = len(ci)
    return rp, np.array(ci, np.int32)


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_mis_none_is_lexfirst(name, g, seed):
    rp, ci = g
    assert (O.mis(rp, ci, "none", 0, seed) == B.brute_lf_mis(rp, ci, seed)).all()


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_mm_none_is_lexfirst(name, g, seed):
    rp, ci = g
    n, adj = B.adjacency(rp, ci)
    if len(B.edge_list(adj)) > 16:
        pytest.skip("too many edges for enumeration")
    mate = O.mm(rp, ci, "none", 0, seed)
    assert (mate == B.brute_lf_mm(rp, ci, seed)).all()
    M = {(min(u, int(w)), max(u, int(w))) for u, w in enumerate(mate) if w >= 0}
    assert nx.is_maximal_matching(_nx(rp, ci), M)


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_color_none_matches_networkx_greedy(name, g, seed):
    rp, ci = g
    n = rp.numel() - 1
    C = O.color(rp, ci, "none", 0, seed)
    order = B.vertex_order(n, seed)
    ref = nx.greedy_color(_nx(rp, ci), strategy=lambda G_, c: iter(order))
    assert all(C[v] == ref[v] + 1 for v in range(n))
    if n <= 6:
        assert (C == B.brute_lf_col(rp, ci, seed)).all()


def _two_stage_mis(rp, ci, kind, param, seed):
    """P:286/P:288 evaluated by enumeration on explicit subgraphs."""
    n, adj = B.adjacency(rp, ci)
    cls = O.classes(rp, ci, kind, param, seed)
    if kind == "degk":
        S1 = [v for v in range(n) if cls[v] == 0]                  # V_L
    else:
        S1 = [v for v in range(n) if all(cls[w] == cls[v] for w in adj[v])]  # interior
    E1 = [(u, w) for u in S1 for w in adj[u] if w in S1 and u < w]
    I1 = B.brute_lf_mis(*_sub_csr(n, E1), seed)
    I1 = {v for v in S1 if I1[v]}            # isolated non-S1 vertices excluded
    dead = set(I1) | {w for v in I1 for w in adj[v]}
    X = [v for v in range(n) if v not in dead and v not in S1]
    E2 = [(u, w) for u in X for w in adj[u] if w in X and u < w]
    I2 = B.brute_lf_mis(*_sub_csr(n, E2), seed)
    out = np.zeros(n, np.uint8)
    for v in I1:
        out[v] = 1
    for v in X:
        out[v] |= I2[v]
    return out


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,param", [("degk", 2), ("degk", 1), ("rand", 2), ("rand", 3)])
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_mis_two_stage_flows(name, g, kind, param, seed):
    rp, ci = g
    assert (O.mis(rp, ci, kind, param, seed) == _two_stage_mis(rp, ci, kind, param, seed)).all()


def _two_stage_mm(rp, ci, kind, param, seed):
    """Alg 5 / Alg 6 by enumeration."""
    n, adj = B.adjacency(rp, ci)
    cls = O.classes(rp, ci, kind, param, seed)
    E = B.edge_list(adj)
    if kind == "rand":
        E1 = [e for e in E if cls[e[0]] == cls[e[1]]]
    else:
        E1 = [e for e in E if cls[e[0]] == 1 and cls[e[1]] == 1]
    m1 = B.brute_lf_mm(*_sub_csr(n, E1), seed)
    free = [m1[v] < 0 for v in range(n)]
    E2 = [e for e in E if e not in E1 and free[e[0]] and free[e[1]]]
    m2 = B.brute_lf_mm(*_sub_csr(n, E2), seed)
    return np.where(m1 >= 0, m1, m2).astype(np.int32)


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,param", [("degk", 2), ("rand", 2), ("rand", 3)])
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_mm_two_stage_flows(name, g, kind, param, seed):
    rp, ci = g
    n, adj = B.adjacency(rp, ci)
    if len(B.edge_list(adj)) > 16:
        pytest.skip("too many edges for enumeration")
    assert (O.mm(rp, ci, kind, param, seed) == _two_stage_mm(rp, ci, kind, param, seed)).all()


def _two_stage_col(rp, ci, kind, param, seed):
    """Alg 9 and Alg 8 with networkx greedy colouring as the
    subroutine (first-fit in priority order)."""
    n, adj = B.adjacency(rp, ci)
    cls = O.classes(rp, ci, kind, param, seed)
    order = B.vertex_order(n, seed)

    def ff(vertices, edges, pre):
        C = dict(pre)
        for v in [u for u in order if u in vertices]:
            used = {C.get(w, 0) for (a, w) in edges if a == v} | {C.get(a, 0) for (a, w) in edges if w == v}
            c = 1
            while c in used:
                c += 1
            C[v] = c
        return C

    E = B.edge_list(adj)
    if kind == "degk":
        H = {v for v in range(n) if cls[v] == 1}
        L = set(range(n)) - H
        CH = ff(H, [e for e in E if e[0] in H and e[1] in H], {})
        M = max(CH.values(), default=0)
        CL = ff(L, [e for e in E if e[0] in L and e[1] in L], {})
        C = {**CH, **{v: M + CL[v] for v in L}}
    else:
        C1 = ff(set(range(n)), [e for e in E if cls[e[0]] == cls[e[1]]], {})
        Vp = {v for (u, w) in E if cls[u] != cls[w] and C1[u] == C1[w] for v in (u, w)}
        pre = {v: c for v, c in C1.items() if v not in Vp}
        C = ff(Vp, E, pre)
    return np.array([C[v] for v in range(n)], np.uint32)


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,param", [("degk", 2), ("degk", 1), ("rand", 2), ("rand", 4)])
@pytest.mark.parametrize("name,g", FAMS, ids=[f[0] for f in FAMS])
def test_color_two_stage_flows(name, g, kind, param, seed):
    rp, ci = g
    assert (O.color(rp, ci, kind, param, seed) == _two_stage_col(rp, ci, kind, param, seed)).all()
