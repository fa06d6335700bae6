"""GPU parity: the CUDA path (through the C-ABI, via the Python binding) against the
CPU oracle, element by element, bit-exact (all data is integer: SURVEY §8 / DESIGN §6).

Sizes: the oracle finishes in seconds and the graphs span many tiles (2048-arc split
tiles, 32-vertex warps) with ragged tails; the families include the degenerate cases
(empty graph, isolated vertices, stars whose hub exceeds the warp budgets and hits
the CTA kernels, cliques, paths/cycles for G_L) and the paper's workload shapes
(R-MAT, road-like grid, near-regular).  Full BASELINE sizes are in
tests/test_gpu_fullsize.py.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O
from conftest import SEEDS

pytestmark = pytest.mark.gpu

sb = pytest.importorskip("paper_conf_ipps_nayyaroddeengk17_b200")

DEV = "cuda"


def _graphs():
    big_star = G.star(9000)                    # hub degree 8999 > every warp budget
    return {
        "rmat14_ef8": G.rmat(14, 8, 1),        # config C1 shape
        "rmat12_ef16": G.rmat(12, 16, 3),
        "road128": G.grid(128, 128, 0.6, 1),   # road-like (C2 shape, smaller)
        "grid64": G.grid(64, 64, 1.0),
        "nreg": G.near_regular(5000, 8, 2),
        "star9000": big_star,
        "hubs": G.disjoint_union(G.star(5000), G.complete(60), G.path(700), G.cycle(301), G.empty(50),
                                 G.rmat(10, 8, 9)),
        "K200": G.complete(200),
        "tiny_mix": G.disjoint_union(*[g for _, g in G.tiny_families()[:20]]),
        "empty7": G.empty(7),
        "single": G.empty(1),
    }


GRAPHS = _graphs()
FLOWS = [("none", 0), ("degk", 2), ("rand", 4), ("rand", 1), ("degk", 1), ("rand", 64)]


def _dev(g):
    rp, ci = g
    return rp.to(DEV), ci.to(DEV)


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    g = GRAPHS[request.param]
    return request.param, g, _dev(g)


def _eq(got, ref, what):
    got = got.cpu().numpy().astype(np.int64)
    ref = np.asarray(ref).astype(np.int64)
    bad = np.nonzero(got != ref)[0]
    assert bad.size == 0, f"{what}: {bad.size} mismatches, first at v={bad[:5].tolist()} got={got[bad[:5]].tolist()} ref={ref[bad[:5]].tolist()}"


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", FLOWS)
def test_mis_parity(graph, kind, p, seed):
    name, g, (rp, ci) = graph
    _eq(sb.sym_mis(rp, ci, kind=kind, param=p, seed=seed), O.mis(*g, kind, p, seed), f"MIS {kind}{p} {name}")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", FLOWS)
def test_mm_parity(graph, kind, p, seed):
    name, g, (rp, ci) = graph
    _eq(sb.sym_mm(rp, ci, kind=kind, param=p, seed=seed), O.mm(*g, kind, p, seed), f"MM {kind}{p} {name}")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", FLOWS)
def test_color_parity(graph, kind, p, seed):
    name, g, (rp, ci) = graph
    _eq(sb.sym_color(rp, ci, kind=kind, param=p, seed=seed), O.color(*g, kind, p, seed), f"COLOR {kind}{p} {name}")


@pytest.mark.parametrize("kind,p", [("rand", 4), ("degk", 2), ("none", 0), ("rand", 1), ("rand", 65535)])
def test_decompose_parity(graph, kind, p):
    name, g, (rp, ci) = graph
    d = sb.sym_decompose(rp, ci, kind, p, seed=42, label=True)
    rp_in, c_in, rp_x, c_x = O.decompose(*g, kind, p, 42)
    _eq(d.row_ptr_in, rp_in, "row_ptr_in")
    _eq(d.row_ptr_x, rp_x, "row_ptr_x")
    assert d.nnz_in == c_in.size and d.nnz_x == c_x.size
    _eq(d.col_in[: d.nnz_in], c_in, "col_in")
    _eq(d.col_x[: d.nnz_x], c_x, "col_x")
    cls = O.classes(*g, kind, p, 42)
    _eq(d.label.to(torch.int32) & 0xFFFF, cls, "label")


@pytest.mark.parametrize("kind,p", [("degk", 2), ("rand", 4)])
def test_precomputed_decomposition_is_reused(kind, p):
    g = GRAPHS["rmat14_ef8"]
    rp, ci = _dev(g)
    d = sb.sym_decompose(rp, ci, kind, p, seed=7)
    _eq(sb.sym_mis(rp, ci, kind, p, 7, decomp=d), O.mis(*g, kind, p, 7), "MIS ext decomp")
    _eq(sb.sym_mm(rp, ci, kind, p, 7, decomp=d), O.mm(*g, kind, p, 7), "MM ext decomp")
    _eq(sb.sym_color(rp, ci, kind, p, 7, decomp=d), O.color(*g, kind, p, 7), "COLOR ext decomp")
    with pytest.raises(sb.SymError):
        sb.sym_mis(rp, ci, kind, p, 8, decomp=d)    # seed mismatch is rejected


def test_host_buffers_end_to_end():
    g = GRAPHS["road128"]
    out = sb.sym_mis(g[0].pin_memory(), g[1].pin_memory(), "degk", 2, 42)
    assert out.device.type == "cpu"
    _eq(out, O.mis(*g, "degk", 2, 42), "host path")


def test_shuffled_rows_and_repeats_are_bit_identical():
    """FIXED-priority results are schedule- and order-independent."""
    rp, ci = GRAPHS["rmat14_ef8"]
    n = rp.numel() - 1
    perm_ci = ci.clone()
    gen = torch.Generator().manual_seed(0)
    deg = rp[1:] - rp[:-1]
    for v in torch.nonzero(deg > 1).flatten()[:4000].tolist():
        a, b = int(rp[v]), int(rp[v + 1])
        perm_ci[a:b] = ci[a:b][torch.randperm(b - a, generator=gen)]
    rpd, cid, pcd = rp.to(DEV), ci.to(DEV), perm_ci.to(DEV)
    for fn in (sb.sym_mis, sb.sym_mm, sb.sym_color):
        for kind, p in (("degk", 2), ("rand", 4), ("none", 0)):
            ref = fn(rpd, cid, kind, p, 42)
            for _ in range(3):
                assert torch.equal(fn(rpd, cid, kind, p, 42), ref)
            assert torch.equal(fn(rpd, pcd, kind, p, 42), ref)
    assert n > 0


def test_validate():
    rp, ci = _dev(GRAPHS["rmat12_ef16"])
    assert sb.sym_validate(rp, ci) == 0
    bad = ci.clone()
    bad[5] = (bad[5] + 1) % (rp.numel() - 1)      # breaks symmetry / order
    assert sb.sym_validate(rp, bad) > 0
    loop = ci.clone()
    v = int(torch.nonzero(rp[1:] > rp[:-1])[0])
    loop[int(rp[v])] = v
    assert sb.sym_validate(rp, loop) > 0
    with pytest.raises(sb.SymError):
        sb.sym_mis(rp, bad, validate=True)


def test_stats_are_reported():
    rp, ci = _dev(GRAPHS["rmat14_ef8"])
    I, st = sb.sym_mis(rp, ci, "degk", 2, 42, stats=True, flags=2)
    assert st["result_size"] == int(I.sum())
    assert st["rounds"][0] >= 1 and st["rounds"][1] >= 1
    M, st = sb.sym_mm(rp, ci, "rand", 4, 42, stats=True, flags=2)
    assert st["result_size"] == int((M >= 0).sum()) // 2
    C, st = sb.sym_color(rp, ci, "rand", 4, 42, stats=True, flags=2)
    assert st["max_color"] == int(C.max())
    assert st["conflicts"] > 0


def test_generator_cpu_gpu_identical():
    a = G.rmat(16, 16, 5)
    b = G.rmat(16, 16, 5, device=DEV)
    assert torch.equal(a[0], b[0].cpu()) and torch.equal(a[1], b[1].cpu())
    assert G.checksum(*a) == G.checksum(*b)
    c = G.grid(300, 200, 0.6, 2)
    d = G.grid(300, 200, 0.6, 2, device=DEV)
    assert torch.equal(c[1], d[1].cpu())


@pytest.mark.parametrize("fn", ["sym_color", "sym_mis", "sym_mm"])
def test_max_rounds_is_reported(fn):
    """params.max_rounds caps the round loop: SYM_EROUNDS, not a wrong result.  The
    early-commit colouring needs tens of rounds on R-MAT s12 (plain JP: more)."""
    rp, ci = G.rmat(12, 16, 1)
    rpd, cid = rp.cuda(), ci.cuda()
    with pytest.raises(sb.SymError) as ei:
        getattr(sb, fn)(rpd, cid, "none", 0, 42, max_rounds=2)
    assert ei.value.code == 6  # SYM_EROUNDS
    # and with room to finish, the result equals the oracle
    got = getattr(sb, fn)(rpd, cid, "none", 0, 42, max_rounds=100000).cpu().numpy()
    ref = getattr(O, fn[4:])(rp, ci, "none", 0, 42)
    assert (got.astype(np.int64) == ref.astype(np.int64)).all()
