"""Pins of the f1 variant oracles (oracle/oracle.c §VAR).

Each variant is checked against something other than its own code:
* PER_ROUND (classic LubyMIS with priorities re-drawn every round):
  independence + maximality (the MIS definition) for every flow; closed forms
  (empty graph -> V, K_n -> {argmax of the round-0 draw}, a star); every local
  maximum of the round-0 draw is In (Luby's first round selects exactly those); the
  re-draw is real (the result differs from the FIXED-priority one on R-MAT) and a
  fixed-priority run is NOT what it computes.  [partially pinned: the later rounds'
  selections are checked only through the invariants]
* MIS-RAND CONFLICT_DROP (reading G10 (i)): recomposed from pinned primitives -- the
  parts' MIS = the FIXED LF-MIS of the intra CSR (oracle.decompose + oracle.mis NONE,
  pinned by brute force), minus the lower In end of every In-In cross arc, then the
  MIS of the induced subgraph of the undecided rest by the oracle's literal Luby
  rounds (or_luby_rounds with a vertex mask, pinned to LF-MIS).
* MIS-RAND SPARSER_FIRST (reading G10 (ii)): the standard flow when the
  cross graph is not sparser; otherwise recomposed the same way (MIS of G[B] first).
* COLOR-RAND LOWER_ONLY: proper; V' = lower ends only is a subset of both ends; the
  colouring off V' equals the parts' greedy colouring (oracle.color NONE on the intra
  CSR, pinned by networkx); p = 1 reduces to COLOR-NONE.
"""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

GRAPHS = {
    "rmat12": lambda: G.rmat(12, 8, 1),
    "road48": lambda: G.grid(48, 48, 0.6, 2),
    "nreg": lambda: G.near_regular(1500, 6, 3),
}


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    rp, ci = GRAPHS[request.param]()
    return rp.numpy(), ci.numpy()


def _is_mis(rp, ci, I):
    src = np.repeat(np.arange(rp.size - 1), np.diff(rp))
    independent = not np.any((I[src] == 1) & (I[ci] == 1))
    covered = I.astype(bool).copy()
    covered[src[I[ci] == 1]] = True
    return independent and covered.all()


def _lf_mis_of(rp, ci, keep, seed):
    """MIS of G[keep] by the oracle's literal fixed-priority Luby rounds (or_luby_rounds,
    an independent function pinned to LF-MIS by tests/test_oracle_rounds.py)"""
    I, _ = O.luby_rounds(rp, ci, seed, inS=keep.astype(np.uint8))
    return (I.astype(bool) & keep).astype(np.uint8)


# ------------------------------------------------------------------ PER_ROUND
@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4)])
def test_per_round_is_an_mis(graph, kind, p, seed):
    rp, ci = graph
    assert _is_mis(rp, ci, O.mis(rp, ci, kind, p, seed, flags=O.F_PER_ROUND))


@pytest.mark.parametrize("seed", SEEDS)
def test_per_round_closed_forms(seed):
    rp, ci = (x.numpy() for x in G.empty(9))
    assert (O.mis(rp, ci, "none", 0, seed, flags=O.F_PER_ROUND) == 1).all()
    rp, ci = (x.numpy() for x in G.complete(30))
    I = O.mis(rp, ci, "none", 0, seed, flags=O.F_PER_ROUND)
    top = max(range(30), key=lambda v: (O.pv(seed, v), v))  # round 0's draw = the FIXED key
    assert I.tolist() == [int(v == top) for v in range(30)]
    rp, ci = (x.numpy() for x in G.star(12))  # centre 0 and leaves 1..n-1
    n = rp.size - 1
    I = O.mis(rp, ci, "none", 0, seed, flags=O.F_PER_ROUND)
    centre_wins = all(O.pv(seed, 0) > O.pv(seed, v) for v in range(1, n))
    assert I.tolist() == ([1] + [0] * (n - 1) if centre_wins else [0] + [1] * (n - 1))


@pytest.mark.parametrize("seed", SEEDS)
def test_per_round_first_round_local_maxima(graph, seed):
    """Luby's round 0 selects every local maximum of the round-0 draw."""
    rp, ci = graph
    I = O.mis(rp, ci, "none", 0, seed, flags=O.F_PER_ROUND)
    key = np.array([(O.pv(seed, v) << 32) | v for v in range(rp.size - 1)], dtype=np.uint64)
    src = np.repeat(np.arange(rp.size - 1), np.diff(rp))
    beaten = np.zeros(rp.size - 1, bool)
    beaten[src[key[ci] > key[src]]] = True
    assert (I[~beaten] == 1).all()


def test_per_round_redraws():
    rp, ci = (x.numpy() for x in G.rmat(12, 8, 1))
    differs = [not np.array_equal(O.mis(rp, ci, "none", 0, s, flags=O.F_PER_ROUND), O.mis(rp, ci, "none", 0, s))
               for s in SEEDS]
    assert all(differs)


# ------------------------------------------------------------------ MIS-RAND variants
@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("p", [1, 2, 4])
def test_conflict_drop_recomposed(graph, p, seed):
    rp, ci = graph
    n = rp.size - 1
    got = O.mis(rp, ci, "rand", p, seed, flags=O.F_CONFLICT_DROP)
    assert _is_mis(rp, ci, got)
    if p == 1:
        assert np.array_equal(got, O.mis(rp, ci, "none", 0, seed))
    rin, cin, _, _ = O.decompose(rp, ci, "rand", p, seed)
    IP = O.mis(rin, cin, "none", 0, seed)                     # the parts' LF-MIS
    cls = O.classes(rp, ci, "rand", p, seed)
    key = np.array([(O.pv(seed, v) << 32) | v for v in range(n)], dtype=np.uint64)
    src = np.repeat(np.arange(n), np.diff(rp))
    drop = np.zeros(n, bool)
    hit = (cls[src] != cls[ci]) & (IP[src] == 1) & (IP[ci] == 1) & (key[ci] > key[src])
    drop[src[hit]] = True
    Ip = (IP == 1) & ~drop
    killed = np.zeros(n, bool)
    killed[src[Ip[ci]]] = True
    X = ~Ip & ~killed
    want = Ip.astype(np.uint8) | _lf_mis_of(rp, ci, X, seed)
    assert np.array_equal(got, want)


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("p", [2, 3, 4])
def test_sparser_first_recomposed(graph, p, seed):
    rp, ci = graph
    n = rp.size - 1
    got = O.mis(rp, ci, "rand", p, seed, flags=O.F_SPARSER_FIRST)
    assert _is_mis(rp, ci, got)
    cls = O.classes(rp, ci, "rand", p, seed)
    src = np.repeat(np.arange(n), np.diff(rp))
    cross = cls[src] != cls[ci]
    if not cross.sum() < (~cross).sum():
        assert np.array_equal(got, O.mis(rp, ci, "rand", p, seed))  # the standard order
        return
    B = np.zeros(n, bool)
    B[src[cross]] = True
    I1 = _lf_mis_of(rp, ci, B, seed)
    killed = np.zeros(n, bool)
    killed[src[I1[ci] == 1]] = True
    X = ~B & ~killed
    assert np.array_equal(got, I1 | _lf_mis_of(rp, ci, X, seed))


def test_sparser_first_takes_both_branches():
    seen = set()
    for g in GRAPHS.values():
        rp, ci = (x.numpy() for x in g())
        for p in (2, 3, 4):
            for seed in SEEDS:
                cls = O.classes(rp, ci, "rand", p, seed)
                src = np.repeat(np.arange(rp.size - 1), np.diff(rp))
                cross = cls[src] != cls[ci]
                seen.add(bool(cross.sum() < (~cross).sum()))
    assert seen == {True, False}


# ------------------------------------------------------------------ COLOR-RAND lower-only
@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("p", [1, 2, 4, 64])
def test_color_lower_only(graph, p, seed):
    rp, ci = graph
    n = rp.size - 1
    C = O.color(rp, ci, "rand", p, seed, flags=O.F_LOWER_ONLY).astype(np.int64)
    src = np.repeat(np.arange(n), np.diff(rp))
    assert (C >= 1).all() and not np.any(C[src] == C[ci])  # proper
    if p == 1:
        assert np.array_equal(C, O.color(rp, ci, "none", 0, seed).astype(np.int64))
    rin, cin, _, _ = O.decompose(rp, ci, "rand", p, seed)
    C1 = O.color(rin, cin, "none", 0, seed).astype(np.int64)  # the parts' greedy colouring
    cls = O.classes(rp, ci, "rand", p, seed)
    key = np.array([(O.pv(seed, v) << 32) | v for v in range(n)], dtype=np.uint64)
    mono = (cls[src] != cls[ci]) & (C1[src] == C1[ci])
    both = np.zeros(n, bool)
    both[src[mono]] = True
    lower = np.zeros(n, bool)
    lower[src[mono & (key[ci] > key[src])]] = True
    assert not np.any(lower & ~both)
    assert np.array_equal(C[~lower], C1[~lower])  # only V' is recoloured


# ------------------------------------------------------------------ f3: the paper's subroutines
SPEC = [("eb", O.F_COLOR_EB), ("vb", O.F_COLOR_VB)]


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("name,flag", SPEC)
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 1), ("rand", 4), ("rand", 64)])
def test_speculative_colouring_is_proper(graph, name, flag, kind, p, seed):
    """EB / VB and the literal G_L loop (Alg 9): every vertex coloured, no
    edge monochromatic; COLOR-Degk's G_L colours lie in max(C_H)+1 .. max(C_H)+k+1
    ("an additional k+1 colors"); RAND p = 1 is the plain speculative colouring."""
    rp, ci = graph
    n = rp.size - 1
    C = O.color(rp, ci, kind, p, seed, flags=flag).astype(np.int64)
    src = np.repeat(np.arange(n), np.diff(rp))
    assert (C >= 1).all() and not np.any(C[src] == C[ci])
    if kind == "degk":
        cls = O.classes(rp, ci, kind, p, seed)
        M = int(C[cls == 1].max()) if (cls == 1).any() else 0
        assert ((C[cls == 0] > M) & (C[cls == 0] <= M + p + 1)).all()
    if kind == "rand" and p == 1:
        assert np.array_equal(C, O.color(rp, ci, "none", 0, seed, flags=flag).astype(np.int64))


@pytest.mark.parametrize("name,flag", SPEC)
@pytest.mark.parametrize("n", [5, 33, 70])
def test_speculative_closed_forms(name, flag, n):
    """K_n: round r leaves exactly the highest remaining id with its colour (every
    other clique edge resets its lower end), so C(v) = n - v -- whatever the window
    (EB 32, VB n - 1) and its OFFSET moves; the empty graph is coloured 1 in one round."""
    rp, ci = (x.numpy() for x in G.complete(n))
    C = O.color(rp, ci, "none", 0, 42, flags=flag)
    assert C.tolist() == [n - v for v in range(n)]
    rp, ci = (x.numpy() for x in G.empty(9))
    assert (O.color(rp, ci, "none", 0, 42, flags=flag) == 1).all()


def test_speculative_is_not_greedy():
    """The speculative colourings are not the greedy (JP) one -- the variant really
    replaces the subroutine.  (EB's and VB's windows only change a colour when a
    colour below a vertex's moved window is freed later by a reset, which is rare:
    on these R-MAT graphs they coincide.)"""
    rp, ci = (x.numpy() for x in G.rmat(12, 8, 1))
    for flag in (O.F_COLOR_EB, O.F_COLOR_VB):
        for kind, p in (("none", 0), ("degk", 2), ("rand", 4)):
            assert not np.array_equal(O.color(rp, ci, kind, p, 42, flags=flag), O.color(rp, ci, kind, p, 42))


# ------------------------------------------------------------------ f2: JP orderings
@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("order", ["lf", "sf"])
def test_jp_orderings_equal_networkx_first_fit(order, seed):
    """JP with largest / smallest degree first (Hasenplaugh et al. [14]) =
    first-fit in that order, computed by networkx's greedy_color (an independent
    first-fit) with the same (degree, pv, id) order."""
    nx = pytest.importorskip("networkx")
    flag = {"lf": O.F_ORDER_LF, "sf": O.F_ORDER_SF}[order]
    for g in (G.rmat(10, 8, 1), G.grid(24, 24, 0.6, 2), G.near_regular(400, 6, 1)):
        rp, ci = (x.numpy() for x in g)
        n = rp.size - 1
        deg = np.diff(rp)
        Gx = nx.Graph()
        Gx.add_nodes_from(range(n))
        src = np.repeat(np.arange(n), deg)
        Gx.add_edges_from(zip(src.tolist(), ci.tolist()))
        sign = 1 if order == "lf" else -1
        orderv = sorted(range(n), key=lambda v: (sign * int(deg[v]), O.pv(seed, v), v), reverse=True)
        want = nx.greedy_color(Gx, strategy=lambda _g, _c: iter(orderv))
        got = O.color(rp, ci, "none", 0, seed, flags=flag)
        assert got.tolist() == [want[v] + 1 for v in range(n)]


@pytest.mark.parametrize("seed", SEEDS)
def test_lf_welsh_powell_bound(graph, seed):
    """Largest-first colouring obeys the Welsh-Powell bound max_i min(d_i + 1, i) over
    the degree-sorted vertices; every ordering is proper in every flow."""
    rp, ci = graph
    n = rp.size - 1
    d = np.sort(np.diff(rp))[::-1]
    bound = int(max(min(int(d[i]) + 1, i + 1) for i in range(n)))
    C = O.color(rp, ci, "none", 0, seed, flags=O.F_ORDER_LF)
    assert int(C.max()) <= bound
    src = np.repeat(np.arange(n), np.diff(rp))
    for flag in (O.F_ORDER_LF, O.F_ORDER_SF):
        for kind, p in (("degk", 2), ("rand", 4)):
            C = O.color(rp, ci, kind, p, seed, flags=flag).astype(np.int64)
            assert (C >= 1).all() and not np.any(C[src] == C[ci])
