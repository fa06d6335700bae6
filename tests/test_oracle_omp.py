"""The all-core round-based oracle (oracle/oracle_omp.c: LubyMIS rounds P:272-274,
LMAX rounds P:150-154, JP levels P:214, in the decomposition flows of P:162-178,
P:226-234) is pinned to the sequential oracle: with fixed priorities the
round forms reach the lexicographically-first results (Blelloch et al. [6]),
so every flow must agree bit for bit -- on every graph family, seed, decomposition
and thread count (the rounds are synchronous, so the thread count cannot matter)."""
import os
import subprocess
import sys

import numpy as np
import pytest

import graphgen as G
import oracle as O
from conftest import ROOT, SEEDS

FLOWS = [("none", 0), ("degk", 2), ("rand", 1), ("rand", 4), ("rand", 64)]
GRAPHS = {
    "rmat12": lambda: G.rmat(12, 8, 1),
    "road64": lambda: G.grid(64, 64, 0.6, 2),
    "nreg": lambda: G.near_regular(2000, 6, 3),
    "mix": lambda: G.disjoint_union(G.star(300), G.cycle(61), G.path(40), G.complete(12), G.empty(9)),
}


@pytest.fixture(scope="module", params=list(GRAPHS))
def graph(request):
    rp, ci = GRAPHS[request.param]()
    return rp.numpy(), ci.numpy()


@pytest.mark.parametrize("seed", SEEDS)
@pytest.mark.parametrize("kind,p", FLOWS)
def test_round_oracle_equals_sequential(graph, kind, p, seed):
    rp, ci = graph
    assert np.array_equal(O.omp_mis(rp, ci, kind, p, seed), O.mis(rp, ci, kind, p, seed))
    assert np.array_equal(O.omp_mm(rp, ci, kind, p, seed), O.mm(rp, ci, kind, p, seed))
    assert np.array_equal(O.omp_color(rp, ci, kind, p, seed), O.color(rp, ci, kind, p, seed))


def test_round_oracle_thread_count_invariant():
    """1 thread and 4 threads give the same bits on R-MAT scale 14 (subprocesses, so
    OMP_NUM_THREADS takes effect)."""
    code = ("import sys; sys.path.insert(0, %r); import numpy as np, graphgen as G, oracle as O; "
            "rp, ci = G.rmat(14, 8, 1); rp, ci = rp.numpy(), ci.numpy(); "
            "print(O.omp_threads(), int(O.omp_mis(rp, ci, 'degk', 2, 7).sum()), "
            "int((O.omp_mm(rp, ci, 'rand', 4, 7) >= 0).sum()), int(O.omp_color(rp, ci, 'rand', 4, 7).astype(np.int64).sum()))"
            % ROOT)
    outs = []
    for t in (1, 4):
        env = dict(os.environ, OMP_NUM_THREADS=str(t))
        outs.append(subprocess.check_output([sys.executable, "-c", code], env=env, text=True).split())
    assert outs[0][0] == "1" and outs[1][0] == "4"
    assert outs[0][1:] == outs[1][1:]
