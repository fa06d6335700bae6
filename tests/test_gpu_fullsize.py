"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(same C-ABI calls, same decomposition reuse).

* C3  R-MAT scale 24 ef16, MIS-Deg2: every output byte vs the sequential oracle.
* C4  R-MAT scale 24 ef16, COLOR with DEG2 and RAND p=4: every colour vs the oracle.
* MM-Rand p=4 at scale 24 (the MM rows of the bench step): the oracle's full sort of
  2.6e8 edges is too slow here, so the result is checked with the oracle's O(m)
  certificate, which holds iff the matching equals LF-MM phase by phase
  (oracle/oracle.c §CRT; exact, not a sample).
* C2  road-like grid 2048^2 (keep 0.6), MM-Rand p=64: every mate vs the oracle.
* the DEG2 and RAND-4 decompositions at scale 24: all four CSR arrays, every element.
* MM-NONE and COLOR-NONE (the undecomposed baselines) at scale 24: O(m) certificates.
* C1  R-MAT scale 14, MIS-Rand p=4 is in test_gpu_parity.py; C5 (scale 27) in
  test_gpu_scale27.py.
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
        # and the O(m) certificate agrees (it is what the scale-27 test relies on)
        assert O.cert_flow("color", hrp, hci, kind, p, SEED, C.cpu().numpy()) == 0, kind


def test_c4_mm_none_and_color_none_scale24(rmat24):
    """The undecomposed baselines the bench reports beside C3/C4 (MM-NONE = LMAX,
    COLOR-NONE = JP): exact O(m) certificates."""
    (rp, ci), (hrp, hci) = rmat24
    M = sb.sym_mm(rp, ci, "none", 0, SEED).cpu().numpy()
    assert O.cert_flow("mm", hrp, hci, "none", 0, SEED, M) == 0
    C = sb.sym_color(rp, ci, "none", 0, SEED).cpu().numpy()
    assert O.cert_flow("color", hrp, hci, "none", 0, SEED, C) == 0


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


def test_decomposition_scale24_full(rmat24):
    """sym_decompose at full size vs the oracle's split (Alg 2 / Alg 3):
    all four arrays (row_ptr_in, col_in, row_ptr_x, col_x) compared element by
    element -- 2 x 520.8 M column entries and 2 x 16.8 M row offsets."""
    (rp, ci), (hrp, hci) = rmat24
    for kind, p in (("degk", 2), ("rand", 4)):
        d = sb.sym_decompose(rp, ci, kind, p, SEED)
        rin, cin, rx, cx = O.decompose(hrp, hci, kind, p, SEED)
        assert d.nnz_in == cin.size and d.nnz_x == cx.size
        assert np.array_equal(d.row_ptr_in.cpu().numpy(), rin), kind
        assert np.array_equal(d.row_ptr_x.cpu().numpy(), rx), kind
        assert np.array_equal(d.col_in[: d.nnz_in].cpu().numpy(), cin), kind
        assert np.array_equal(d.col_x[: d.nnz_x].cpu().numpy(), cx), kind
        del d
