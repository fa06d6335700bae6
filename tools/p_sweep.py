"""Partition-count sweep ("as the number of partitions
increases there is slowdown in the performance of Algorithm MM-Rand", P:254 the same
for COLOR-Rand): MM-Rand and COLOR-Rand device time (decomposition included), rounds,
and the paper's mechanism (intra fraction, conflicts) for p = 2, 4, 10, 64, 100 on
R-MAT s24 and the road grid, next to the undecomposed MM-NONE / COLOR-NONE.

    python tools/p_sweep.py  ->  gpurun_out/p_sweep.json
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


def timed(fn, reps=5):
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    out = {}
    for gname, (rp, ci) in (("rmat24_ef16", G.rmat(24, 16, 1, device="cuda")),
                            ("road2048", G.grid(2048, 2048, 0.6, 1, device="cuda"))):
        m = ci.numel() // 2
        rec = {"m": m}
        for prob, fn in (("mm", sb.sym_mm), ("color", sb.sym_color)):
            fn(rp, ci, "none", 0, 42)
            ms = timed(lambda: fn(rp, ci, "none", 0, 42))
            _, st = fn(rp, ci, "none", 0, 42, stats=True, flags=2)
            rec[f"{prob}_none"] = {"ms": ms, "edges_per_s": m / ms * 1e3, "rounds": st["rounds"],
                                   "result_size": st["result_size"]}
            for p in (2, 4, 10, 64, 100):
                def call():
                    d = sb.sym_decompose(rp, ci, "rand", p, 42)
                    return fn(rp, ci, "rand", p, 42, decomp=d)
                call()
                ms = timed(call)
                d = sb.sym_decompose(rp, ci, "rand", p, 42)
                _, st = fn(rp, ci, "rand", p, 42, decomp=d, stats=True, flags=2)
                rec[f"{prob}_rand{p}"] = {"ms": ms, "edges_per_s": m / ms * 1e3, "rounds": st["rounds"],
                                          "result_size": st["result_size"], "conflicts": st["conflicts"],
                                          "intra_fraction": d.nnz_in / max(1, ci.numel())}
                print(gname, prob, p, rec[f"{prob}_rand{p}"], flush=True)
                del d
        out[gname] = rec
        del rp, ci
        torch.cuda.empty_cache()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "p_sweep.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
