"""compute-sanitizer driver: every C-ABI flow once on small graphs (R-MAT s12 and a
road grid): MIS/MM/COLOR x NONE/DEG2/RAND4/BRIDGE, decompose, validate, the f1/f2/f3
variant flags, and the sharded calls (2 ranks in one process, local communicator).

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402
from paper_conf_ipps_nayyaroddeengk17_b200 import sharded as S  # noqa: E402

dev = torch.device("cuda", 0)
for name, (rp, ci) in {"rmat12": G.rmat(12, 16, 1), "grid64": G.grid(64, 64, 0.6, 1)}.items():
    rp, ci = rp.to(dev), ci.to(dev)
    assert sb.sym_validate(rp, ci) == 0
    for kind, p in (("none", 0), ("degk", 2), ("rand", 4), ("bridge", 0)):
        if kind != "none":
            sb.sym_decompose(rp, ci, kind, p, 7, label=True)
        for fn in (sb.sym_mis, sb.sym_mm, sb.sym_color):
            fn(rp, ci, kind, p, 7)
            fn(rp, ci, kind, p, 7, stats=True)
    for f in (0x10,):  # per-round Luby
        sb.sym_mis(rp, ci, "degk", 2, 7, flags=f)
    for f in (0x20, 0x40):  # conflict-drop, sparser-first
        sb.sym_mis(rp, ci, "rand", 2, 7, flags=f)
    for kind, p in (("none", 0), ("degk", 2), ("rand", 4)):
        for f in (0x100, 0x200, 0x400, 0x800):  # EB, VB, LF, SF
            sb.sym_color(rp, ci, kind, p, 7, flags=f)
    sb.sym_color(rp, ci, "rand", 4, 7, flags=0x80)
    for prob, kind, p in (("mis", "degk", 2), ("mis", "rand", 4), ("mm", "rand", 4), ("color", "degk", 2),
                          ("color", "rand", 4)):
        S.run_local(S.make_shards(rp, ci, 2), prob, kind, p, 7)
    torch.cuda.synchronize()
    print(name, "done", flush=True)
