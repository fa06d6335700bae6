"""Diagnostic: per-round list sizes and start times of the persistent JP rounds kernel
(COLOR-Deg2 on R-MAT), and the COLOR-Deg2 device time."""
import os, sys
os.environ.setdefault("SYM_JP_TRACE", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
ts = []
for _ in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); sb.sym_color(rp, ci, "degk", 2, 42, decomp=d); e1.record(); torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
sb.sym_profile_enable(True)
sb.sym_color(rp, ci, "degk", 2, 42, decomp=d)
torch.cuda.synchronize()
print("profile", sb.sym_profile_collect())
sb.sym_profile_enable(False)
col, st = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d, stats=True)
torch.cuda.synchronize()
print("COLOR-Deg2 ms", ts, "max colour", int(col.max()))
ws = sb._WS[(0, torch.cuda.current_stream(dev).cuda_stream)]
off = ((ws.data_ptr() + 255) & ~255) - ws.data_ptr()
h = ws[off + 136: off + 136 + 16384].cpu().numpy().view(np.uint32)
tr = h[2048:4096].astype(np.int64)
pa = tr[:512] * 32 / 1000.0
cnt, t = h[:1024].astype(np.int64), h[1024:2048].astype(np.int64) * 32 / 1000.0
R = st["rounds"][0]
print("rounds", st["rounds"])
dt = np.diff(t[:min(R, 1024)])
for r in list(range(0, 16)) + list(range(20, min(R, 1023), 40)):
    if r < len(dt):
        if os.environ.get("SYM_JP_TRACE") == "4":  # slowest big push: atomics returned, hot loads, activations
            extra = (f" A {pa[r]-t[r]:7.2f} us atom {tr[512+r]*0.032:6.2f} hot {tr[1024+r]*0.032:6.2f}"
                     f" activ {tr[1536+r]*0.032:7.2f}") if r < 512 else ""
        elif os.environ.get("SYM_JP_TRACE") == "2":  # slowest warp's push / build span of phase B
            extra = (f" A {pa[r]-t[r]:7.2f} us push {tr[512+r]*0.032:6.2f} build {tr[1024+r]*0.032:6.2f}"
                     f" Bwork {tr[1536+r]*0.032:7.2f}") if r < 512 else ""
        else:
            extra = f" A {pa[r]-t[r]:7.2f} us pushT {tr[512+r]:7d} buildT {tr[1024+r]:7d} Bwork {tr[1536+r]*0.032:7.2f}" if r < 512 else ""
        print(f"R{r:5d} |U| {cnt[r]:9d} t {t[r]:9.1f} us  dt {dt[r]:7.2f} us" + extra)
if len(dt) > 40:
    print("median dt (rounds >= 20)", np.median(dt[20:]), "mean", dt[20:].mean())
