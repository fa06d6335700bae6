"""Step time of the five calls in order vs OverlapStep (schedule.py) at R-MAT s24, with
a bit-identity check of the outputs.   python tools/overlap_probe.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402
from paper_conf_ipps_nayyaroddeengk17_b200.schedule import OverlapStep  # noqa: E402

dev = torch.device("cuda", 0)
rp, ci = graphgen.rmat(24, 16, seed=1, device=dev)
seed = 42


def seq():
    dD = sb.sym_decompose(rp, ci, "degk", 2, seed)
    I = sb.sym_mis(rp, ci, "degk", 2, seed, decomp=dD)
    C = sb.sym_color(rp, ci, "degk", 2, seed, decomp=dD)
    dR = sb.sym_decompose(rp, ci, "rand", 4, seed)
    M = sb.sym_mm(rp, ci, "rand", 4, seed, decomp=dR)
    return I, C, M


ov = OverlapStep(dev, seed)


def timeit(f, k=10, w=3):
    for _ in range(w):
        f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(k):
        f()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / k


a = [x.cpu() for x in seq()]
b = [x.cpu() for x in ov(rp, ci)]
same = all(torch.equal(x, y) for x, y in zip(a, b))
res = {"sequential_ms": timeit(seq), "overlap_ms": timeit(lambda: ov(rp, ci)), "bit_identical": same}
res["sequential_ms_again"] = timeit(seq)
print(json.dumps(res))
