"""The bench step, sequential vs the two-stream schedule (schedule.ConcurrentStep),
with the JP rounds kernel at SYM_JR_CTAS_PER_SM CTAs per SM (set in the environment).

    SYM_JR_CTAS_PER_SM=1 python tools/concurrency_probe.py
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402
from paper_conf_ipps_nayyaroddeengk17_b200.schedule import ConcurrentStep  # noqa: E402


def main():
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

    cs = ConcurrentStep(dev, seed)
    out = {"SYM_JR_CTAS_PER_SM": os.environ.get("SYM_JR_CTAS_PER_SM")}
    ref = [x.clone() for x in seq()]
    for name, fn in (("sequential", seq), ("concurrent", lambda: cs(rp, ci))):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(7):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            res = fn()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        out[name] = {"ms": statistics.median(ts), "equal": all(torch.equal(x, y) for x, y in zip(res, ref))}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
