"""Oracle flow pins at sizes brute force cannot reach (SURVEY.md §4 / DESIGN.md §3):

* invariants of every output: independent + maximal,
  valid + maximal matching, proper colouring with colours >= 1;
* degenerate reductions: RAND p=1 and DEGk with k >= max degree collapse to the
  undecomposed method (NONE);
* the paper's claims: P:23/P:234 -- a DEG2 colouring of G_H and G_L coloured
  independently is valid once L is shifted by max(C_H) (negative control: without
  the shift cross edges conflict), and G_L needs only k+1 = 3 colours;
  P:188 -- RAND with p parts leaves ~1/p of the edges intra;
  Table II shape -- road-like grid %DEG2 from the closed form;
* closed forms on K_n, stars, empty graphs;
* decomposition structure (Alg 2/3): intra u cross = G per row, in input order;
* certificates (used for full-size parity) reject perturbed results.
"""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

KINDS = [("none", 0), ("degk", 2), ("rand", 4), ("rand", 10)]


def _arrays(g):
    rp, ci = g
    return rp.numpy(), ci.numpy()


@pytest.fixture(scope="module")
def rmat14():
    return _arrays(G.rmat(14, 8, 1))


@pytest.fixture(scope="module")
def road():
    return _arrays(G.grid(256, 256, 0.6, 1))


def _src(rp):
    return np.repeat(np.arange(rp.size - 1), np.diff(rp))


def check_mis(rp, ci, I):
    s = _src(rp)
    assert not (I[s] & I[ci]).any(), "not independent"
    covered = I.astype(bool).copy()
    covered[s[I[ci] == 1]] = True
    assert covered.all(), "not maximal"


def check_mm(rp, ci, mate):
    n = rp.size - 1
    s = _src(rp)
    m = mate >= 0
    assert (mate[mate[m]] == np.arange(n)[m]).all()
    # each mate pair is an edge
    key = set(zip(s.tolist(), ci.tolist()))
    assert all((v, int(mate[v])) in key for v in np.nonzero(m)[0][:2000])
    # maximal: no edge with both endpoints free
    assert not ((~m[s]) & (~m[ci])).any()


def check_col(rp, ci, C):
    s = _src(rp)
    assert (C >= 1).all()
    assert not (C[s] == C[ci]).any(), "not proper"


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", KINDS)
def test_invariants_rmat(rmat14, kind, p, seed):
    rp, ci = rmat14
    check_mis(rp, ci, O.mis(rp, ci, kind, p, seed))
    check_mm(rp, ci, O.mm(rp, ci, kind, p, seed))
    check_col(rp, ci, O.color(rp, ci, kind, p, seed))


@pytest.mark.parametrize("kind,p", KINDS + [("rand", 64)])
def test_invariants_road(road, kind, p):
    rp, ci = road
    check_mis(rp, ci, O.mis(rp, ci, kind, p, 42))
    check_mm(rp, ci, O.mm(rp, ci, kind, p, 42))
    check_col(rp, ci, O.color(rp, ci, kind, p, 42))


@pytest.mark.parametrize("problem", ["mis", "mm", "color"])
def test_degenerate_reductions(rmat14, problem):
    rp, ci = rmat14
    f = getattr(O, problem)
    ref = f(rp, ci, "none", 0, 42)
    assert (f(rp, ci, "rand", 1, 42) == ref).all()            # p = 1: no cross edges
    dmax = int(np.diff(rp).max())
    assert (f(rp, ci, "degk", dmax, 42) == ref).all()         # k >= Delta: V_H empty
    # k < min degree: V_L empty (cycle graphs: every degree is 2)
    crp, cci = _arrays(G.cycle(101))
    assert (f(crp, cci, "degk", 1, 42) == f(crp, cci, "none", 0, 42)).all()


@pytest.mark.parametrize("seed", SEEDS)
def test_paper_claim_deg2_independent_colouring_is_valid(rmat14, seed):
    """P:23 / P:234: colour G_H, then G_L with the k+1 colours max(C_H)+1..max(C_H)+k+1:
    the union is a valid colouring of G (no recolouring needed).  Negative control:
    without the shift, cross edges G_C conflict."""
    rp, ci = rmat14
    k = 2
    C = O.color(rp, ci, "degk", k, seed)
    check_col(rp, ci, C)
    deg = np.diff(rp)
    H = deg > k
    M = int(C[H].max())
    CL = C[~H] - M
    assert CL.min() >= 1 and CL.max() <= k + 1            # G_L uses <= k+1 colours
    unshifted = C.astype(np.int64).copy()
    unshifted[~H] -= M
    s = _src(rp)
    assert (unshifted[s] == unshifted[ci]).sum() > 0     # the shift is necessary


@pytest.mark.parametrize("p", [4, 10])
def test_paper_rand_intra_fraction(p):
    """with p (=10) partitions the induced subgraphs hold ~1/p of the edges."""
    rp, ci = _arrays(G.rmat(16, 16, 2))
    rp_in, c_in, rp_x, c_x = O.decompose(rp, ci, "rand", p, 42)
    frac = c_in.size / ci.size
    assert abs(frac - 1 / p) < 0.01


def test_road_like_grid_deg2_fraction_closed_form():
    """Road-like grid (keep 0.6): interior vertex degree ~ Bin(4, 0.6), so
    P[deg <= 2] = 1 - 4(.6^3)(.4) - .6^4 = 0.5248 (cf. road-central 50.91 %)."""
    w = 512
    rp, ci = _arrays(G.grid(w, w, 0.6, 3))
    deg = np.diff(rp).reshape(w, w)[1:-1, 1:-1]
    frac = (deg <= 2).mean()
    expect = 1 - 4 * 0.6**3 * 0.4 - 0.6**4
    assert abs(expect - 0.5248) < 1e-12
    sd = np.sqrt(expect * (1 - expect) / deg.size)
    assert abs(frac - expect) < 6 * sd * 2   # neighbouring degrees share edges: x2


@pytest.mark.parametrize("kind,p", [("rand", 4), ("rand", 1), ("degk", 2), ("none", 0)])
def test_decomposition_structure(rmat14, kind, p):
    rp, ci = rmat14
    rp_in, c_in, rp_x, c_x = O.decompose(rp, ci, kind, p, 42)
    cls = O.classes(rp, ci, kind, p, 42)
    n = rp.size - 1
    assert rp_in[-1] + rp_x[-1] == ci.size
    for v in range(0, n, 7):
        row = ci[rp[v]:rp[v + 1]]
        same = cls[row] == cls[v]
        assert (c_in[rp_in[v]:rp_in[v + 1]] == row[same]).all()
        assert (c_x[rp_x[v]:rp_x[v + 1]] == row[~same]).all()
    # induced subgraphs are symmetric
    s_in = np.repeat(np.arange(n), np.diff(rp_in))
    a = set(zip(s_in.tolist(), c_in.tolist()))
    assert all((w, v) in a for (v, w) in list(a)[:5000])


@pytest.mark.parametrize("seed", SEEDS)
def test_closed_forms(seed):
    # K_n: MIS = {argmax pv}; colours = rank in priority order; MM perfect for even n
    n = 9
    rp, ci = _arrays(G.complete(n))
    pv = np.array([O.pv(seed, v) for v in range(n)], np.int64)
    I = O.mis(rp, ci, "none", 0, seed)
    assert I.sum() == 1 and I[np.argmax(pv)] == 1
    rank = np.empty(n, np.int64)
    rank[np.argsort(-pv)] = np.arange(1, n + 1)
    assert (O.color(rp, ci, "none", 0, seed) == rank).all()
    rp8, ci8 = _arrays(G.complete(8))
    assert (O.mm(rp8, ci8, "none", 0, seed) >= 0).all()
    # star: MIS = {centre} iff centre has the top priority, else the leaves;
    # MM = the single heaviest edge
    rp, ci = _arrays(G.star(11))
    pv = np.array([O.pv(seed, v) for v in range(11)])
    I = O.mis(rp, ci, "none", 0, seed)
    if pv[0] == pv.max():
        assert I.tolist() == [1] + [0] * 10
    else:
        assert I.tolist() == [0] + [1] * 10
    mate = O.mm(rp, ci, "none", 0, seed)
    best = max(range(1, 11), key=lambda w: (O.pe(seed, 0, w), w))
    assert mate[0] == best and (mate >= 0).sum() == 2
    # empty graph: everything In, colour 1, unmatched
    rp, ci = _arrays(G.empty(7))
    assert (O.mis(rp, ci, "none", 0, seed) == 1).all()
    assert (O.color(rp, ci, "none", 0, seed) == 1).all()
    assert (O.mm(rp, ci, "none", 0, seed) == -1).all()


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4), ("rand", 64)])
def test_flow_certificates_accept_oracle_outputs(rmat14, road, kind, p, seed):
    """or_cert_flow (O(n) memory, used up to scale 27) returns 0 on the oracle's own
    output of every flow, on R-MAT and on the road grid."""
    for rp, ci in (rmat14, road):
        for prob, fn in (("mis", O.mis), ("mm", O.mm), ("color", O.color)):
            assert O.cert_flow(prob, rp, ci, kind, p, seed, fn(rp, ci, kind, p, seed)) == 0, prob


@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4)])
def test_certificates_accept_oracle_and_reject_perturbations(rmat14, kind, p):
    rp, ci = rmat14
    I = O.mis(rp, ci, kind, p, 42)
    assert O.cert_flow("mis", rp, ci, kind, p, 42, I) == 0
    for v in (0, 17, 4000, 9999):
        J = I.copy()
        J[v] ^= 1
        assert O.cert_flow("mis", rp, ci, kind, p, 42, J) > 0
    M = O.mm(rp, ci, kind, p, 42)
    assert O.cert_flow("mm", rp, ci, kind, p, 42, M) == 0
    u = int(np.nonzero(M >= 0)[0][5])
    M2 = M.copy()
    M2[M2[u]] = -1
    M2[u] = -1
    assert O.cert_flow("mm", rp, ci, kind, p, 42, M2) > 0
    C = O.color(rp, ci, kind, p, 42)
    assert O.cert_flow("color", rp, ci, kind, p, 42, C) == 0
    C2 = C.copy()
    C2[int(np.argmax(np.diff(rp)))] += 1
    assert O.cert_flow("color", rp, ci, kind, p, 42, C2) > 0


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("p", [1, 2, 4, 64])
def test_color_rand_certificate(rmat14, road, seed, p):
    """The O(m) COLOR-Rand certificate (Alg 8; C1 by a topological sweep
    instead of the sort) accepts exactly the oracle's output: every single-vertex
    change -- in V' or outside it, up or down -- is rejected; p = 1 (no cross edges,
    V' empty) reduces it to the JP/greedy certificate of COLOR-NONE; |V'| is the
    fraction the paper reports the recolouring works on (~45 % at p = 2 on its
    graphs; [sim] 25-37 % for R-MAT at p = 2..4)."""
    for rp, ci in (rmat14, road):
        n = rp.size - 1
        C = O.color(rp, ci, "rand", p, seed)
        bad, nconf = O.cert_col_rand(rp, ci, C, p, seed)
        assert bad == 0
        if p == 1:
            assert nconf == 0
            assert np.array_equal(C, O.color(rp, ci, "none", 0, seed))
        elif (rp, ci) is rmat14 and p <= 4:
            assert 0.15 < nconf / n < 0.5
        rng = np.random.default_rng(seed & 0xFFFF)
        for v in rng.choice(n, 12, replace=False):
            for d in (1, -1):
                if int(C[v]) + d < 1:
                    continue
                C2 = C.copy()
                C2[v] = int(C[v]) + d
                assert O.cert_col_rand(rp, ci, C2, p, seed)[0] > 0
    # the NONE colouring is rejected as a COLOR-Rand result once cross edges exist
    rp, ci = rmat14
    assert O.cert_col_rand(rp, ci, O.color(rp, ci, "none", 0, seed), 4, seed)[0] > 0


def test_round_counts_are_logarithmic(rmat14):
    """LubyMIS needs O(log n) rounds in expectation; LMAX converges in a
    handful of rounds with random (hash) priorities (no 'vain tendency')."""
    rp, ci = rmat14
    _, r = O.luby_rounds(rp, ci, 42)
    assert r <= 4 * np.log2(rp.size)
    _, r = O.lmax_rounds(rp, ci, 42)
    assert r <= 4 * np.log2(rp.size)
