"""GPU parity of the BRIDGE decomposition (Alg 1) and the
Bridge flows (MM-Bridge Alg 4, COLOR-Bridge Alg 7, MIS-Bridge Alg 10) against the
oracle (tests/test_oracle_bridge.py pins it to networkx.bridges and brute force):
the intra / cross CSRs element by element, and every output bit-exact."""
import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import SEEDS

pytestmark = pytest.mark.gpu

sb = pytest.importorskip("paper_conf_ipps_nayyaroddeengk17_b200")

GRAPHS = {
    "rmat14_ef4": lambda: G.rmat(14, 4, 1),
    "road128_sparse": lambda: G.grid(128, 128, 0.5, 1),   # long BFS paths, many bridges
    "hubs": lambda: G.disjoint_union(G.star(5000), G.complete(60), G.path(700), G.cycle(301), G.empty(50),
                                     G.rmat(10, 2, 9)),
    "tiny_mix": lambda: G.disjoint_union(*[g for _, g in G.tiny_families()[:30]]),
    "empty": lambda: G.empty(5),
}


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    g = GRAPHS[request.param]()
    return request.param, g, (g[0].cuda(), g[1].cuda())


def _eq(got, ref, what):
    got = got.cpu().numpy().astype(np.int64)
    ref = np.asarray(ref).astype(np.int64)
    assert np.array_equal(got, ref), f"{what}: {(got != ref).sum() if got.shape == ref.shape else 'shape'} mismatches"


def test_bridge_decomposition(graph):
    name, g, (rp, ci) = graph
    d = sb.sym_decompose(rp, ci, "bridge", 0, seed=42)
    rin, cin, rx, cx = O.decompose(*g, "bridge", 0, 42)
    _eq(d.row_ptr_in, rin, f"row_ptr_in {name}")
    _eq(d.row_ptr_x, rx, f"row_ptr_x {name}")
    assert d.nnz_in == cin.size and d.nnz_x == cx.size
    _eq(d.col_in[: d.nnz_in], cin, f"col_in {name}")
    _eq(d.col_x[: d.nnz_x], cx, f"col_x {name}")


@pytest.mark.parametrize("seed", SEEDS)
def test_bridge_flows(graph, seed):
    name, g, (rp, ci) = graph
    for prob, fn in (("mis", sb.sym_mis), ("mm", sb.sym_mm), ("color", sb.sym_color)):
        _eq(fn(rp, ci, "bridge", 0, seed), getattr(O, prob)(*g, "bridge", 0, seed), f"{prob}-bridge {name}")
    _eq(sb.sym_mis(rp, ci, "bridge", 0, seed, flags=O.F_PER_ROUND),
        O.mis(*g, "bridge", 0, seed, flags=O.F_PER_ROUND), f"mis-bridge per-round {name}")
    _eq(sb.sym_color(rp, ci, "bridge", 0, seed, flags=O.F_ORDER_LF),
        O.color(*g, "bridge", 0, seed, flags=O.F_ORDER_LF), f"color-bridge LF {name}")


def test_bridge_scale20():
    g = G.rmat(20, 4, 1, device="cuda")
    h = (g[0].cpu().numpy(), g[1].cpu().numpy())
    d = sb.sym_decompose(*g, "bridge", 0, 42)
    rin, cin, rx, cx = O.decompose(*h, "bridge", 0, 42)
    assert d.nnz_x == cx.size and cx.size > 0
    _eq(d.row_ptr_in, rin, "s20 row_ptr_in")
    _eq(d.col_x[: d.nnz_x], cx, "s20 col_x")
    for prob, fn in (("mis", sb.sym_mis), ("mm", sb.sym_mm), ("color", sb.sym_color)):
        res = fn(*g, "bridge", 0, 42, decomp=d).cpu().numpy()
        assert O.cert_flow(prob, *h, "bridge", 0, 42, res) == 0, prob
