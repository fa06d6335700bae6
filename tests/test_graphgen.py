"""Generator checks (test infrastructure): the bucketed CSR assembly used for
scale >= 26 (so that R-MAT scale 27 fits one GPU) yields exactly the same canonical
CSR as the global sort; CSRs are canonical (symmetric, loop-free, sorted rows)."""
import numpy as np
import pytest
import torch

import graphgen as G


@pytest.mark.parametrize("buckets", [2, 7, 16])
def test_bucketed_assembly_is_identical(buckets):
    a = G.rmat(13, 8, 3)
    b = G.rmat(13, 8, 3, buckets=buckets)
    assert torch.equal(a[0], b[0]) and torch.equal(a[1], b[1])


@pytest.mark.parametrize("g", [G.rmat(12, 16, 2), G.grid(40, 30, 0.6, 1), G.near_regular(999, 6, 4)])
def test_canonical_csr(g):
    rp, ci = g[0].numpy(), g[1].numpy()
    n = rp.size - 1
    src = np.repeat(np.arange(n), np.diff(rp))
    assert (src != ci).all()
    for v in range(0, n, 17):
        row = ci[rp[v]:rp[v + 1]]
        assert (np.diff(row) > 0).all()
    fwd = set(zip(src.tolist(), ci.tolist()))
    assert all((w, v) in fwd for v, w in list(fwd)[:4000])
