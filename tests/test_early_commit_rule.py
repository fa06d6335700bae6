"""Pins the early-commit rule the CUDA colouring path runs (jp.cu header)
against the oracle's first-fit greedy colouring (LF-COL).

Rule: with m = mex of the colours of v's coloured higher-priority neighbours, v may
take m once every higher neighbour u is coloured with a colour != m, or uncoloured
with m already forbidden for u (a coloured higher neighbour of u holds m) or
m > cap(u) = #higher(u) + 1.  The claim is that this reaches exactly the greedy
colouring under ANY schedule.  This file implements the rule independently of the
CUDA code (plain Python sets, CPU) in two schedules -- synchronous rounds and a
random asynchronous order with immediate updates -- and checks both against the
oracle, plus that the synchronous rounds never exceed the JP dependency depth.
"""
import random

import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS


def _prio(n, seed):
    pv = np.array([O.pv(seed, v) for v in range(n)], dtype=np.uint64)
    return (pv << np.uint64(32)) | np.arange(n, dtype=np.uint64)  # larger = higher priority


def _lists(rp, ci, key):
    rp, ci = rp.numpy(), ci.numpy()
    n = len(rp) - 1
    higher = [[int(w) for w in ci[rp[v]:rp[v + 1]] if key[w] > key[v]] for v in range(n)]
    return higher


def _try(v, higher, col, forb):
    """The rule: returns v's colour if it can commit now, else 0."""
    m = 1
    while m in forb[v]:
        m += 1
    for u in higher[v]:
        if col[u]:
            if col[u] == m:
                return 0
        elif not (m in forb[u] or m > len(higher[u]) + 1):
            return 0
    return m


def _commit(v, c, col, forb, lower):
    col[v] = c
    for w in lower[v]:
        forb[w].add(c)


def early_commit_rounds(rp, ci, seed):
    n = len(rp) - 1
    key = _prio(n, seed)
    higher = _lists(rp, ci, key)
    lower = [[] for _ in range(n)]
    for v in range(n):
        for u in higher[v]:
            lower[u].append(v)
    col = [0] * n
    forb = [set() for _ in range(n)]
    left, rounds = set(range(n)), 0
    while left:
        decided = {v: c for v in left for c in [_try(v, higher, col, forb)] if c}
        assert decided, "no progress"
        for v, c in decided.items():
            _commit(v, c, col, forb, lower)
        left -= decided.keys()
        rounds += 1
    return np.array(col, dtype=np.uint32), rounds


def early_commit_async(rp, ci, seed, order_seed):
    n = len(rp) - 1
    key = _prio(n, seed)
    higher = _lists(rp, ci, key)
    lower = [[] for _ in range(n)]
    for v in range(n):
        for u in higher[v]:
            lower[u].append(v)
    col = [0] * n
    forb = [set() for _ in range(n)]
    rng = random.Random(order_seed)
    left = list(range(n))
    while left:
        rng.shuffle(left)
        nxt = []
        for v in left:  # immediate updates: later vertices see earlier commits
            c = _try(v, higher, col, forb)
            if c:
                _commit(v, c, col, forb, lower)
            else:
                nxt.append(v)
        assert len(nxt) < len(left), "no progress"
        left = nxt
    return np.array(col, dtype=np.uint32)


GRAPHS = {
    "rmat10": lambda: G.rmat(10, 8, 3),
    "grid32_road": lambda: G.grid(32, 32, 0.6, 1),
    "nreg": lambda: G.near_regular(800, 6, 5),
    "complete40": lambda: G.complete(40),
    "star50": lambda: G.star(50),
    "cycle31": lambda: G.cycle(31),
}


@pytest.mark.parametrize("name", list(GRAPHS))
@pytest.mark.parametrize("seed", SEEDS)
def test_early_commit_rounds_equal_greedy(name, seed):
    rp, ci = GRAPHS[name]()
    got, rounds = early_commit_rounds(rp, ci, seed)
    assert (got == O.color(rp, ci, "none", 0, seed)).all()
    _, depth = O.jp_rounds(rp, ci, seed)
    assert rounds <= depth


@pytest.mark.parametrize("name", ["rmat10", "grid32_road", "nreg"])
def test_early_commit_any_order_equals_greedy(name):
    rp, ci = GRAPHS[name]()
    ref = O.color(rp, ci, "none", 0, 42)
    for order_seed in range(3):
        assert (early_commit_async(rp, ci, 42, order_seed) == ref).all()


def test_early_commit_cuts_rounds_on_rmat():
    """The point of the rule: far fewer dependent rounds than JP levels on R-MAT."""
    rp, ci = G.rmat(11, 16, 1)
    _, rounds = early_commit_rounds(rp, ci, 42)
    _, depth = O.jp_rounds(rp, ci, 42)
    assert rounds * 2 <= depth


def test_negative_control_ignoring_uncoloured_neighbours_breaks_greedy(monkeypatch):
    """A plausible mistake -- treating an uncoloured higher neighbour as harmless --
    must be caught: the colouring then differs from greedy."""
    def sloppy(v, higher, col, forb):
        m = 1
        while m in forb[v]:
            m += 1
        return 0 if any(col[u] == m for u in higher[v]) else m
    monkeypatch.setattr(__import__(__name__), "_try", sloppy)
    rp, ci = GRAPHS["rmat10"]()
    got, _ = early_commit_rounds(rp, ci, 42)
    assert not (got == O.color(rp, ci, "none", 0, 42)).all()
