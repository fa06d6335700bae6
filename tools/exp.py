"""Experiment driver (GPU box): R-MAT s24 ef16, time selected problems through the
public API (median of R runs, CUDA events) and print the library's per-class profile
(ms, alg / impl bytes).  Used for A/B runs of kernel changes; not a bench line.
    python tools/exp.py [--scale 24] [--reps 5] split_degk mis_none mm_none ...
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=24)
ap.add_argument("--ef", type=int, default=16)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--once", action="store_true", help="one call each, no timing (for ncu)")
ap.add_argument("what", nargs="+")
a = ap.parse_args()
dev = torch.device("cuda", 0)
rp, ci = graphgen.rmat(a.scale, a.ef, seed=1, device=dev)
m = int(ci.numel()) // 2
d2 = sb.sym_decompose(rp, ci, "degk", 2, 42)
d4 = sb.sym_decompose(rp, ci, "rand", 4, 42)
CASES = {
    "split_degk": lambda: sb.sym_decompose(rp, ci, "degk", 2, 42),
    "split_rand4": lambda: sb.sym_decompose(rp, ci, "rand", 4, 42),
    "mis_none": lambda: sb.sym_mis(rp, ci, "none", 0, 42),
    "mis_deg2": lambda: sb.sym_mis(rp, ci, "degk", 2, 42, decomp=d2),
    "mm_none": lambda: sb.sym_mm(rp, ci, "none", 0, 42),
    "mm_rand4": lambda: sb.sym_mm(rp, ci, "rand", 4, 42, decomp=d4),
    "color_deg2": lambda: sb.sym_color(rp, ci, "degk", 2, 42, decomp=d2),
}
out = {}
for w in a.what:
    f = CASES[w]
    if a.once:
        f()
        torch.cuda.synchronize()
        continue
    f()
    ts = []
    for _ in range(a.reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    sb.sym_profile_enable(True)
    sb.sym_profile_collect()
    f()
    torch.cuda.synchronize()
    prof = sb.sym_profile_collect()
    sb.sym_profile_enable(False)
    ts.sort()
    out[w] = {"ms_med": round(ts[len(ts) // 2], 4), "ms_min": round(ts[0], 4), "classes": prof}
    print(w, json.dumps(out[w]), flush=True)
