"""Diagnostic: per-level task counts, start times and (SYM_JP_TRACE=1) spans of the
persistent JP levels kernel: the slowest CTA's work span and flush+arrival span."""
import os, sys
os.environ.setdefault("SYM_JP_TRACE", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
for _ in range(2):
    col, st = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d, stats=True)
torch.cuda.synchronize()
ws = sb._WS[(0, torch.cuda.current_stream(dev).cuda_stream)]
off = ((ws.data_ptr() + 255) & ~255) - ws.data_ptr()
h = ws[off + 136: off + 136 + 16384].cpu().numpy().view(np.uint32)
cnt, ts = h[:1024].astype(np.int64), h[1024:2048].astype(np.int64) * 32 / 1000.0
work, flush = h[2048:3072] * 32 / 1000.0, h[3072:4096] * 32 / 1000.0
print("levels", st["rounds"])
dt = np.diff(ts)
for r in list(range(0, 12)) + list(range(40, 1023, 80)):
    print(f"L{r:5d} tasks {cnt[r]:8d} t {ts[r]:9.1f} us  dt {dt[r]:7.2f} us  work(max CTA) {work[r]:6.2f}  flush(max) {flush[r]:6.2f}")
sel = slice(20, 1023)
print("median dt", np.median(dt[sel]), "work", np.median(work[sel]), "flush", np.median(flush[sel]),
      "rest (barrier+skew)", np.median(dt[sel] - work[sel] - flush[sel]))
