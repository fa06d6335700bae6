"""GPU parity of the f1 variants (include/sym.h SYM_F_PER_ROUND,
SYM_F_CONFLICT_DROP, SYM_F_SPARSER_FIRST, SYM_F_LOWER_ONLY) against the variant
oracles (oracle/oracle.c §VAR, pinned in tests/test_oracle_variants.py), element by
element, bit-exact.  Classic per-round Luby is NOT schedule-independent, so this also
checks that the GPU runs its two-step rounds exactly synchronously.
"""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

pytestmark = pytest.mark.gpu

sb = pytest.importorskip("paper_conf_ipps_nayyaroddeengk17_b200")

GRAPHS = {
    "rmat14_ef8": lambda: G.rmat(14, 8, 1),
    "road128": lambda: G.grid(128, 128, 0.6, 1),
    "nreg": lambda: G.near_regular(5000, 8, 2),
    "hubs": lambda: G.disjoint_union(G.star(5000), G.complete(60), G.path(700), G.cycle(301), G.empty(50)),
}


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    g = GRAPHS[request.param]()
    return request.param, g, (g[0].cuda(), g[1].cuda())


def _eq(got, ref, what):
    got = got.cpu().numpy().astype(np.int64)
    ref = np.asarray(ref).astype(np.int64)
    assert np.array_equal(got, ref), f"{what}: {(got != ref).sum()} mismatches"


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4), ("rand", 64)])
def test_per_round_luby(graph, kind, p, seed):
    name, g, (rp, ci) = graph
    f = O.F_PER_ROUND
    _eq(sb.sym_mis(rp, ci, kind, p, seed, flags=f), O.mis(*g, kind, p, seed, flags=f), f"PER_ROUND {kind}{p} {name}")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("flag", ["conflict_drop", "sparser_first"])
@pytest.mark.parametrize("p", [1, 2, 4, 64])
def test_mis_rand_variants(graph, flag, p, seed):
    name, g, (rp, ci) = graph
    f = {"conflict_drop": O.F_CONFLICT_DROP, "sparser_first": O.F_SPARSER_FIRST}[flag]
    _eq(sb.sym_mis(rp, ci, "rand", p, seed, flags=f), O.mis(*g, "rand", p, seed, flags=f), f"{flag} p{p} {name}")
    # combined with per-round Luby steps
    f |= O.F_PER_ROUND
    _eq(sb.sym_mis(rp, ci, "rand", p, seed, flags=f), O.mis(*g, "rand", p, seed, flags=f), f"{flag}+PR p{p} {name}")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("p", [1, 2, 4, 64])
def test_color_lower_only(graph, p, seed):
    name, g, (rp, ci) = graph
    f = O.F_LOWER_ONLY
    _eq(sb.sym_color(rp, ci, "rand", p, seed, flags=f), O.color(*g, "rand", p, seed, flags=f), f"LOWER p{p} {name}")


def test_variant_flags_rejected_where_undefined():
    rp, ci = (x.cuda() for x in G.rmat(10, 8, 1))
    with pytest.raises(sb.SymError):
        sb.sym_mis(rp, ci, "rand", 4, 42, flags=O.F_CONFLICT_DROP | O.F_SPARSER_FIRST)


def test_variants_scale20_match_the_oracle():
    """R-MAT scale 20 (16 M arcs; per-round Luby on the full flow set)."""
    g = G.rmat(20, 16, 1, device="cuda")
    h = (g[0].cpu().numpy(), g[1].cpu().numpy())
    for kind, p, f in (("none", 0, O.F_PER_ROUND), ("degk", 2, O.F_PER_ROUND), ("rand", 4, O.F_CONFLICT_DROP),
                       ("rand", 2, O.F_SPARSER_FIRST)):
        _eq(sb.sym_mis(*g, kind, p, 42, flags=f), O.mis(*h, kind, p, 42, flags=f), f"s20 {kind}{p} {f:#x}")
    _eq(sb.sym_color(*g, "rand", 4, 42, flags=O.F_LOWER_ONLY), O.color(*h, "rand", 4, 42, flags=O.F_LOWER_ONLY),
        "s20 lower-only")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("flag", ["eb", "vb"])
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4), ("rand", 64)])
def test_speculative_colouring(graph, flag, kind, p, seed):
    """f3: the paper's EB / VB subroutines and the literal G_L loop, bit-exact."""
    name, g, (rp, ci) = graph
    f = {"eb": O.F_COLOR_EB, "vb": O.F_COLOR_VB}[flag]
    _eq(sb.sym_color(rp, ci, kind, p, seed, flags=f), O.color(*g, kind, p, seed, flags=f), f"{flag} {kind}{p} {name}")
    if kind == "rand":
        f |= O.F_LOWER_ONLY
        _eq(sb.sym_color(rp, ci, kind, p, seed, flags=f), O.color(*g, kind, p, seed, flags=f),
            f"{flag}+lower {kind}{p} {name}")


def test_speculative_scale20():
    g = G.rmat(20, 16, 1, device="cuda")
    h = (g[0].cpu().numpy(), g[1].cpu().numpy())
    for kind, p in (("none", 0), ("degk", 2), ("rand", 4)):
        _eq(sb.sym_color(*g, kind, p, 42, flags=O.F_COLOR_EB), O.color(*h, kind, p, 42, flags=O.F_COLOR_EB),
            f"s20 EB {kind}")


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("order", ["lf", "sf"])
@pytest.mark.parametrize("kind,p", [("none", 0), ("degk", 2), ("rand", 4)])
def test_jp_orderings(graph, order, kind, p, seed):
    """f2: early-commit JP with the largest / smallest degree first orders, bit-exact."""
    name, g, (rp, ci) = graph
    f = {"lf": O.F_ORDER_LF, "sf": O.F_ORDER_SF}[order]
    _eq(sb.sym_color(rp, ci, kind, p, seed, flags=f), O.color(*g, kind, p, seed, flags=f), f"{order} {kind}{p} {name}")
    if kind == "rand":
        f |= O.F_LOWER_ONLY
        _eq(sb.sym_color(rp, ci, kind, p, seed, flags=f), O.color(*g, kind, p, seed, flags=f), f"{order}+lower {name}")


def test_jp_orderings_scale20():
    g = G.rmat(20, 16, 1, device="cuda")
    h = (g[0].cpu().numpy(), g[1].cpu().numpy())
    for f in (O.F_ORDER_LF, O.F_ORDER_SF):
        _eq(sb.sym_color(*g, "degk", 2, 42, flags=f), O.color(*h, "degk", 2, 42, flags=f), f"s20 order {f:#x}")
