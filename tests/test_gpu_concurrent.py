"""The two-stream steps (schedule.ConcurrentStep, schedule.OverlapStep) equal the
sequential calls bit for bit, and both equal the oracle on a small graph."""
import pytest
import torch

import graphgen
import oracle as O

pytestmark = pytest.mark.gpu


def _seq(sb, rp, ci, seed):
    dD = sb.sym_decompose(rp, ci, "degk", 2, seed)
    I = sb.sym_mis(rp, ci, "degk", 2, seed, decomp=dD)
    C = sb.sym_color(rp, ci, "degk", 2, seed, decomp=dD)
    dR = sb.sym_decompose(rp, ci, "rand", 4, seed)
    M = sb.sym_mm(rp, ci, "rand", 4, seed, decomp=dR)
    return I, C, M


@pytest.mark.parametrize("scale", [12, 18])
@pytest.mark.parametrize("kind", ["concurrent", "overlap"])
def test_concurrent_step_equals_sequential(scale, kind):
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    from paper_conf_ipps_nayyaroddeengk17_b200.schedule import ConcurrentStep, OverlapStep
    dev = torch.device("cuda", 0)
    rp, ci = graphgen.rmat(scale, 8, seed=3, device=dev)
    ref = _seq(sb, rp, ci, 42)
    step = (ConcurrentStep if kind == "concurrent" else OverlapStep)(dev, 42)
    for _ in range(3):
        got = step(rp, ci)
        torch.cuda.synchronize()
        for a, b in zip(ref, got):
            assert torch.equal(a, b)
    if scale == 12:
        rpc, cic = rp.cpu().numpy(), ci.cpu().numpy()
        I, C, M = (x.cpu().numpy() for x in got)
        assert (I == O.mis(rpc, cic, "degk", 2, 42)).all()
        assert (C == O.color(rpc, cic, "degk", 2, 42)).all()
        assert (M == O.mm(rpc, cic, "rand", 4, 42)).all()
