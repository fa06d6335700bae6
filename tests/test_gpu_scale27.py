"""C5 (BASELINE.json configs[4]) on one B200: R-MAT scale 27, edge factor 16
(n = 134.2 M, 4.22 G arcs -- int64 row offsets, col_idx 16.9 GB), in the launch
configuration of bench.py (one decomposition per kind, reused by the problems).

Parity is exact and complete (every vertex), by the oracle's O(m)-time,
O(n)-memory flow certificates (oracle/oracle.c or_cert_flow: each holds iff the
output equals the oracle's lexicographically-first result phase by phase; pinned in
tests/test_oracle_flows.py and cross-checked against the full oracle at scale 24 in
test_gpu_fullsize.py):
  * MIS-Deg2, COLOR-Deg2 (Alg 9) on the DEG2 decomposition;
  * MM-Rand p = 8 (Alg 5) and COLOR-Rand p = 8 (Alg 8) on RAND-8;
  * the 8-way sharded MIS-Deg2, MM-Rand8 and COLOR-Deg2 (one process, in-process
    exchange, the multi-GPU path's kernels) equal the single-GPU outputs bit for bit.
Scale 27 is where the JP compact ids and extra-bitmap offsets are closest to their
27-bit fields (jp.cu JP_HMASK), and where nnz > 2^32 exercises int64 offsets.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = [pytest.mark.gpu, pytest.mark.scale27]

sb = pytest.importorskip("paper_conf_ipps_nayyaroddeengk17_b200")
SEED = 42
SCALE = 27


@pytest.fixture(scope="module")
def rmat27():
    free, _ = torch.cuda.mem_get_info()
    if free < 120e9:
        pytest.fail(f"scale 27 needs ~120 GB of free device memory, {free / 1e9:.0f} GB free")
    rp, ci = G.rmat(SCALE, 16, seed=1, device="cuda")
    torch.cuda.synchronize()
    hrp, hci = rp.cpu().numpy(), ci.cpu().numpy()
    assert hci.size > 2**31  # arc offsets beyond int32: int64 row_ptr really used
    yield (rp, ci), (hrp, hci)
    del rp, ci
    torch.cuda.empty_cache()


def _free():
    torch.cuda.synchronize()
    torch.cuda.empty_cache()


def test_c5_deg2_mis_color(rmat27):
    (rp, ci), (hrp, hci) = rmat27
    d = sb.sym_decompose(rp, ci, "degk", 2, SEED)
    I = sb.sym_mis(rp, ci, "degk", 2, SEED, decomp=d).cpu().numpy()
    C, st = sb.sym_color(rp, ci, "degk", 2, SEED, decomp=d, stats=True)
    C = C.cpu().numpy()
    del d
    _free()
    assert O.cert_flow("mis", hrp, hci, "degk", 2, SEED, I) == 0
    assert O.cert_flow("color", hrp, hci, "degk", 2, SEED, C) == 0
    assert st["rounds"][0] > 0 and C.min() >= 1


def test_c5_rand8_mm_color(rmat27):
    (rp, ci), (hrp, hci) = rmat27
    d = sb.sym_decompose(rp, ci, "rand", 8, SEED)
    M = sb.sym_mm(rp, ci, "rand", 8, SEED, decomp=d).cpu().numpy()
    C = sb.sym_color(rp, ci, "rand", 8, SEED, decomp=d).cpu().numpy()
    del d
    _free()
    assert O.cert_flow("mm", hrp, hci, "rand", 8, SEED, M) == 0
    assert (M >= 0).sum() > 0
    assert O.cert_flow("color", hrp, hci, "rand", 8, SEED, C) == 0


def test_c5_sharded8_equals_single_gpu(rmat27):
    """8 ranks (the C5 multi-GPU layout) through the library's sharded calls, one host
    thread and local communicator per rank on this GPU: bit-identical to the
    single-GPU calls (FIXED priorities are schedule-independent)."""
    from paper_conf_ipps_nayyaroddeengk17_b200 import sharded as S
    (rp, ci), _ = rmat27
    ref_I = sb.sym_mis(rp, ci, "degk", 2, SEED)
    ref_M = sb.sym_mm(rp, ci, "rand", 8, SEED)
    _free()
    shards = S.make_shards(rp, ci, 8)
    out = S.run_local(shards, "mis", "degk", 2, SEED)
    assert torch.equal(torch.cat(out), ref_I)
    del out
    _free()
    out = S.run_local(shards, "mm", "rand", 8, SEED)
    assert torch.equal(torch.cat(out), ref_M)
    del out, shards
    _free()
