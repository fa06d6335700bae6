"""Diagnostic: per-level floor of the JP levels kernel -- a path whose vertex order is
the priority order has depth n and one tiny task per level."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle as O
import paper_conf_ipps_nayyaroddeengk17_b200 as sb
n = int(sys.argv[1]) if len(sys.argv) > 1 else 5000
pv = np.array([O.pv(42, v) for v in range(n)], dtype=np.uint64)
order = np.argsort(-(pv.astype(np.int64) << 32 | np.arange(n)))  # decreasing (pv, id)
src, dst = order[:-1], order[1:]
a = np.concatenate([src, dst]); b = np.concatenate([dst, src])
idx = np.lexsort((b, a))
a, b = a[idx], b[idx]
rp = np.zeros(n + 1, dtype=np.int64); np.add.at(rp, a + 1, 1); rp = np.cumsum(rp)
dev = torch.device("cuda", 0)
rpt, cit = torch.from_numpy(rp).to(dev), torch.from_numpy(b.astype(np.int32)).to(dev)
for it in range(3):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); c, st = sb.sym_color(rpt, cit, "none", 0, 42, stats=True); e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
print(json.dumps({"n": n, "levels": st["rounds"][0], "ms": ms, "us_per_level": ms * 1e3 / max(1, st["rounds"][0]),
                  "max_color": int(c.max())}))
