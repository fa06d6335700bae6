"""Pins of the BRIDGE decomposition oracle (Alg 1) and of the
Bridge flows (MM-Bridge Alg 4 / P:160, COLOR-Bridge Alg 7 / P:224, MIS-Bridge Alg 10 /
P:280-284, which the oracle runs as the RAND flows with the 2-edge-connected
components as the classes):
* the bridges equal networkx.bridges, and by brute force on tiny graphs an edge is a
  bridge iff deleting it disconnects its endpoints ("any bridge in a graph can never be
  a part of a cycle");
* the classes are the connected components of G - B (networkx) labelled by their
  smallest vertex; an arc is intra iff it is not a bridge;
* reductions: a tree (every edge a bridge) and a 2-edge-connected graph (no bridge)
  give the undecomposed results for all three problems.
"""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

nx = pytest.importorskip("networkx")


def _nx(rp, ci):
    n = rp.size - 1
    g = nx.Graph()
    g.add_nodes_from(range(n))
    src = np.repeat(np.arange(n), np.diff(rp))
    g.add_edges_from((int(a), int(b)) for a, b in zip(src, ci) if a < b)
    return g


GRAPHS = {
    "rmat11": lambda: G.rmat(11, 4, 2),
    "road40": lambda: G.grid(40, 40, 0.5, 3),
    "mix": lambda: G.disjoint_union(G.path(30), G.cycle(17), G.star(12), G.complete(9), G.empty(4), G.rmat(8, 2, 5)),
}


@pytest.mark.parametrize("name", list(GRAPHS))
def test_bridge_classes_match_networkx(name):
    rp, ci = (x.numpy() for x in GRAPHS[name]())
    n = rp.size - 1
    g = _nx(rp, ci)
    bridges = {frozenset(e) for e in nx.bridges(g)}
    cls = O.classes(rp, ci, "bridge", 0, 42)
    src = np.repeat(np.arange(n), np.diff(rp))
    cross = {frozenset((int(a), int(b))) for a, b in zip(src, ci) if cls[a] != cls[b]}
    assert cross == bridges
    h = g.copy()
    h.remove_edges_from(tuple(e) for e in bridges)
    for comp in nx.connected_components(h):
        assert {int(cls[v]) for v in comp} == {min(comp)}


def test_bridges_brute_force_tiny():
    for name, (rp, ci) in G.tiny_families()[:40]:
        rp, ci = rp.numpy(), ci.numpy()
        n = rp.size - 1
        g = _nx(rp, ci)
        cls = O.classes(rp, ci, "bridge", 0, 1)
        for a, b in list(g.edges()):
            h = g.copy()
            h.remove_edge(a, b)
            is_bridge = not nx.has_path(h, a, b)
            assert is_bridge == (cls[a] != cls[b]), (name, a, b)


@pytest.mark.parametrize("seed", SEEDS)
def test_bridge_flow_reductions(seed):
    """Trees: every edge a bridge; cycles / cliques / grids without dead ends: none."""
    for g in (G.path(50), G.star(40)):
        rp, ci = (x.numpy() for x in g)
        for prob, fn in (("mis", O.mis), ("mm", O.mm), ("color", O.color)):
            assert np.array_equal(fn(rp, ci, "bridge", 0, seed), fn(rp, ci, "none", 0, seed)), prob
    for g in (G.cycle(41), G.complete(20), G.grid(12, 12, 1.0)):
        rp, ci = (x.numpy() for x in g)
        assert len(set(O.classes(rp, ci, "bridge", 0, seed).tolist())) == 1
        for prob, fn in (("mis", O.mis), ("mm", O.mm), ("color", O.color)):
            assert np.array_equal(fn(rp, ci, "bridge", 0, seed), fn(rp, ci, "none", 0, seed)), prob


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("name", list(GRAPHS))
def test_bridge_flows_invariants_and_certificates(name, seed):
    rp, ci = (x.numpy() for x in GRAPHS[name]())
    n = rp.size - 1
    src = np.repeat(np.arange(n), np.diff(rp))
    I = O.mis(rp, ci, "bridge", 0, seed)
    assert not np.any((I[src] == 1) & (I[ci] == 1))
    cov = I.astype(bool).copy()
    cov[src[I[ci] == 1]] = True
    assert cov.all()
    M = O.mm(rp, ci, "bridge", 0, seed)
    assert all(M[M[v]] == v for v in range(n) if M[v] >= 0)
    assert not np.any((M[src] < 0) & (M[ci] < 0))
    C = O.color(rp, ci, "bridge", 0, seed).astype(np.int64)
    assert (C >= 1).all() and not np.any(C[src] == C[ci])
    for prob, res in (("mis", I), ("mm", M), ("color", C)):
        assert O.cert_flow(prob, rp, ci, "bridge", 0, seed, res) == 0
    assert np.array_equal(O.omp_mis(rp, ci, "bridge", 0, seed), I)
    assert np.array_equal(O.omp_mm(rp, ci, "bridge", 0, seed), M)
    assert np.array_equal(O.omp_color(rp, ci, "bridge", 0, seed).astype(np.int64), C)
