"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(same C-ABI calls, same decomposition reuse).

* C3  R-MAT scale 24 ef16, MIS-Deg2: every output byte vs the sequential oracle.
* C4  R-MAT scale 24 ef16, COLOR with DEG2 and RAND p=4: every colour vs the oracle.
* MM-Rand p=4 at scale 24 (the MM rows of the bench step): the oracle's full sort of
  2.6e8 edges is too slow here, so the result is checked with the oracle's O(m)
  certificate, which holds iff the matching equals LF-MM phase by phase
  (oracle/oracle.c §CRT; exact, not a sample).
* C2  road-like grid 2048^2 (keep 0.6), MM-Rand p=64: every mate vs the oracle.
* C1  R-MAT scale 14, MIS-Rand p=4 is in test_gpu_parity.py.
Graphs are generated on the GPU (graphgen, bit-identical to the CPU generator,
checked in test_gpu_parity.py) and copied to the host for the oracle.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = pytest.mark.gpu

sb = pytest.importorskip("paper_conf_ipps_nayyaroddeengk17_b200")
SEED = 42


@pytest.fixture(scope="module")
def rmat24():
    rp, ci = G.rmat(24, 16, seed=1, device="cuda")
    torch.cuda.synchronize()
    return (rp, ci), (rp.cpu().numpy(), ci.cpu().numpy())


def _mismatch(got, ref):
    got = got.cpu().numpy().astype(np.int64)
    ref = np.asarray(ref).astype(np.int64)
    return int((got != ref).sum())


def test_c3_mis_deg2_scale24(rmat24):
    (rp, ci), (hrp, hci) = rmat24
    d = sb.sym_decompose(rp, ci, "degk", 2, SEED)
    I = sb.sym_mis(rp, ci, "degk", 2, SEED, decomp=d)
    assert _mismatch(I, O.mis(hrp, hci, "degk", 2, SEED)) == 0
    # the undecomposed LubyMIS baseline too (certificate: O(m), exact)
    I0 = sb.sym_mis(rp, ci, "none", 0, SEED)
    assert O.cert_flow("mis", hrp, hci, "none", 0, SEED, I0.cpu().numpy()) == 0


def test_c4_color_deg2_and_rand_scale24(rmat24):
    (rp, ci), (hrp, hci) = rmat24
    for kind, p in (("degk", 2), ("rand", 4)):
        d = sb.sym_decompose(rp, ci, kind, p, SEED)
        C = sb.sym_color(rp, ci, kind, p, SEED, decomp=d)
        assert _mismatch(C, O.color(hrp, hci, kind, p, SEED)) == 0, kind


def test_mm_rand4_scale24_certificate(rmat24):
    (rp, ci), (hrp, hci) = rmat24
    d = sb.sym_decompose(rp, ci, "rand", 4, SEED)
    M = sb.sym_mm(rp, ci, "rand", 4, SEED, decomp=d).cpu().numpy()
    assert O.cert_flow("mm", hrp, hci, "rand", 4, SEED, M) == 0
    assert (M >= 0).sum() > 0


def test_c2_road_grid_mm_rand64():
    rp, ci = G.grid(2048, 2048, 0.6, seed=1, device="cuda")
    M = sb.sym_mm(rp, ci, "rand", 64, SEED)
    ref = O.mm(rp.cpu().numpy(), ci.cpu().numpy(), "rand", 64, SEED)
    assert _mismatch(M, ref) == 0


def test_decomposition_scale24_sampled_rows(rmat24):
    """sym_decompose at full size vs the oracle's split of sampled rows (plus the
    global totals)."""
    (rp, ci), (hrp, hci) = rmat24
    for kind, p in (("degk", 2), ("rand", 4)):
        d = sb.sym_decompose(rp, ci, kind, p, SEED)
        cls = O.classes(hrp, hci, kind, p, SEED)
        rin, cin = d.row_ptr_in.cpu().numpy(), d.col_in.cpu().numpy()
        rx, cx = d.row_ptr_x.cpu().numpy(), d.col_x.cpu().numpy()
        src = np.repeat(np.arange(hrp.size - 1), np.diff(hrp))
        n_intra = int((cls[src] == cls[hci]).sum())
        assert d.nnz_in == n_intra and d.nnz_x == hci.size - n_intra
        rng = np.random.default_rng(0)
        deg = np.diff(hrp)
        rows = np.concatenate([rng.integers(0, hrp.size - 1, 20000), np.argsort(-deg)[:50]])
        for v in rows:
            row = hci[hrp[v]:hrp[v + 1]]
            same = cls[row] == cls[v]
            assert np.array_equal(cin[rin[v]:rin[v + 1]], row[same])
            assert np.array_equal(cx[rx[v]:rx[v + 1]], row[~same])
