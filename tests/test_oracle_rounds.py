"""Pins: the literal round-based algorithms reach the sequential greedy results
(fixed priorities).  These are the facts the paper builds on:

* fixed-priority LubyMIS rounds == greedy MIS in priority order (Blelloch et al.
  [6], cited at P:274);
* LMAX rounds (mutual heaviest edge) == greedy matching GM in decreasing
  edge priority;
* Jones-Plassmann rounds == first-fit greedy colouring in priority order,
  and its colour class 1 is the greedy MIS;
on R-MAT, road-like grid and near-regular graphs shaped like the paper's workloads.
"""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

GRAPHS = {
    "rmat10": lambda: G.rmat(10, 8, 3),
    "rmat12": lambda: G.rmat(12, 16, 1),
    "grid64_road": lambda: G.grid(64, 64, 0.6, 1),
    "grid32": lambda: G.grid(32, 32, 1.0),
    "nreg": lambda: G.near_regular(3000, 6, 5),
}


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    return GRAPHS[request.param]()


@pytest.mark.parametrize("seed", SEEDS)
def test_luby_rounds_equal_greedy_mis(graph, seed):
    rp, ci = graph
    I_rounds, r = O.luby_rounds(rp, ci, seed)
    assert (I_rounds == O.mis(rp, ci, "none", 0, seed)).all()
    assert r >= 1


@pytest.mark.parametrize("seed", SEEDS)
def test_lmax_rounds_equal_greedy_mm(graph, seed):
    rp, ci = graph
    mate, r = O.lmax_rounds(rp, ci, seed)
    assert (mate == O.mm(rp, ci, "none", 0, seed)).all()


@pytest.mark.parametrize("seed", SEEDS)
def test_jp_rounds_equal_greedy_color(graph, seed):
    rp, ci = graph
    C, depth = O.jp_rounds(rp, ci, seed)
    Cg = O.color(rp, ci, "none", 0, seed)
    assert (C == Cg).all()
    # colour class 1 of greedy colouring == greedy MIS
    assert ((Cg == 1).astype(np.uint8) == O.mis(rp, ci, "none", 0, seed)).all()


def test_luby_rounds_on_subset_equal_two_stage():
    """The MIS-DEG2 phases as round-based Luby on V_L then on X == the oracle flow."""
    rp, ci = G.rmat(12, 8, 7)
    seed = 42
    n = rp.numel() - 1
    deg = np.diff(rp.numpy())
    L = (deg <= 2).astype(np.uint8)
    I1, _ = O.luby_rounds(rp, ci, seed, inS=L)
    I1 = I1 * L
    rpn, cin = rp.numpy(), ci.numpy()
    st = np.zeros(n, np.uint8)
    X = np.zeros(n, np.uint8)
    for v in range(n):
        if L[v]:
            st[v] = 1 if I1[v] else 2
            continue
        if any(L[w] and I1[w] for w in cin[rpn[v]:rpn[v + 1]]):
            st[v] = 2
        else:
            X[v] = 1
    I2, _ = O.luby_rounds(rp, ci, seed, inS=X)
    I = (I1 | (I2 * X)).astype(np.uint8)
    assert (I == O.mis(rp, ci, "degk", 2, seed)).all()
