"""Diagnostic: per-level task counts and start times of the persistent JP levels kernel."""
import os, sys
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
h = ws[off + 136: off + 136 + 8192].cpu().numpy().view(np.uint32)
cnt, ts = h[:1024].astype(np.int64), h[1024:2048].astype(np.int64) * 32 / 1000.0
print("levels", st["rounds"])
dt = np.diff(ts)
for r in list(range(0, 40)) + list(range(40, 1023, 40)):
    print(f"L{r:5d} tasks {cnt[r]:8d} t {ts[r]:9.1f} us  dt {dt[r]:7.2f} us")
print("median dt", np.median(dt), "mean", dt.mean(), "p90", np.percentile(dt, 90))
big = np.argsort(-dt)[:15]
print("slowest levels:", [(int(r), float(dt[r]), int(cnt[r])) for r in big])
