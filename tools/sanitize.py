"""compute-sanitizer driver: every C-ABI flow once on small graphs (R-MAT s12 and a
road grid): MIS/MM/COLOR x NONE/DEG2/RAND4, decompose, validate.

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402

dev = torch.device("cuda", 0)
for name, (rp, ci) in {"rmat12": G.rmat(12, 16, 1), "grid64": G.grid(64, 64, 0.6, 1)}.items():
    rp, ci = rp.to(dev), ci.to(dev)
    assert sb.sym_validate(rp, ci) == 0
    for kind, p in (("none", 0), ("degk", 2), ("rand", 4)):
        if kind != "none":
            sb.sym_decompose(rp, ci, kind, p, 7)
        for fn in (sb.sym_mis, sb.sym_mm, sb.sym_color):
            fn(rp, ci, kind, p, 7)
            fn(rp, ci, kind, p, 7, stats=True)
    torch.cuda.synchronize()
    print(name, "done", flush=True)
