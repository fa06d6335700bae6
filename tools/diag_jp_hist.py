"""Diagnostic: JP task count per round (first 2048 rounds) read from the Ctl block."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
C, st = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d, stats=True)
ws = sb._WS[0]
base = (ws.data_ptr() + 255) & ~255
off = base - ws.data_ptr()
hist = ws[off + 136: off + 136 + 8192].cpu().numpy().view(np.uint32)
print("rounds", st["rounds"], "colours", int(C.max()))
h = hist[:2048]
print("first 40:", h[:40].tolist())
print("percentiles tasks/round (rounds 0..2047):", np.percentile(h[h > 0], [10, 50, 90, 99]).tolist(), "sum", int(h.sum()))
print("rounds 1000..1040:", h[1000:1040].tolist())
