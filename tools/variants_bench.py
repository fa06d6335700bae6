"""Device time of the variants next to the default flows on R-MAT s24 (one line per
setting): per-round Luby, MIS-Rand conflict-drop / sparser-first, COLOR-Rand lower-only,
the speculative EB / VB subroutines, JP with LF / SF orders.

    python tools/variants_bench.py  ->  gpurun_out/variants_bench.json
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_nayyaroddeengk17_b200 as sb  # noqa: E402

F = {"default": 0, "per_round": 0x10, "conflict_drop": 0x20, "sparser_first": 0x40, "lower_only": 0x80,
     "eb": 0x100, "vb": 0x200, "lf": 0x400, "sf": 0x800}
RUNS = [("mis", "none", 0, "default"), ("mis", "none", 0, "per_round"), ("mis", "degk", 2, "default"),
        ("mis", "degk", 2, "per_round"), ("mis", "rand", 4, "default"), ("mis", "rand", 4, "conflict_drop"),
        ("mis", "rand", 2, "sparser_first"), ("color", "none", 0, "default"), ("color", "none", 0, "eb"),
        ("color", "none", 0, "vb"), ("color", "none", 0, "lf"), ("color", "none", 0, "sf"),
        ("color", "degk", 2, "default"), ("color", "degk", 2, "eb"), ("color", "degk", 2, "lf"),
        ("color", "rand", 4, "default"), ("color", "rand", 4, "lower_only"), ("color", "rand", 4, "eb"),
        ("mis", "bridge", 0, "default"), ("mm", "bridge", 0, "default"), ("color", "bridge", 0, "default"),
        ("mm", "rand", 4, "default"), ("mm", "none", 0, "default")]


def main():
    rp, ci = G.rmat(24, 16, 1, device="cuda")
    m = ci.numel() // 2
    fns = {"mis": sb.sym_mis, "mm": sb.sym_mm, "color": sb.sym_color}
    out = {}
    for prob, kind, p, var in RUNS:
        dms = None
        if kind != "none":
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            sb.sym_decompose(rp, ci, kind, p, 42)
            a.record()
            d = sb.sym_decompose(rp, ci, kind, p, 42)
            b.record()
            torch.cuda.synchronize()
            dms = a.elapsed_time(b)
        else:
            d = None
        call = lambda: fns[prob](rp, ci, kind, p, 42, decomp=d, flags=F[var])  # noqa: E731
        call()
        ts = []
        for _ in range(3):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            call()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        res, st = fns[prob](rp, ci, kind, p, 42, decomp=d, stats=True, flags=F[var] | 2)
        key = f"{prob}_{kind}{p}_{var}"
        out[key] = {"ms": statistics.median(ts), "decompose_ms": dms, "edges_per_s": m / statistics.median(ts) * 1e3,
                    "rounds": st["rounds"], "result_size": st["result_size"]}
        print(key, out[key], flush=True)
        del d
    with open(os.path.join(ROOT, "gpurun_out", "variants_bench.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
