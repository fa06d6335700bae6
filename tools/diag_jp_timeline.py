"""Diagnostic: async JP timeline (us at which each 1/64 of the vertices is coloured)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["SYM_DEBUG_JP"] = "1"
import numpy as np, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
rp, ci = graphgen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 24, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
for _ in range(2):
    sb.sym_color(rp, ci, "degk", 2, 42, decomp=d)
torch.cuda.synchronize()
ws = sb._WS[0]
off = ((ws.data_ptr() + 255) & ~255) - ws.data_ptr()
h = ws[off + 136: off + 136 + 16384].cpu().numpy().view(np.uint32)
print("timeline us per 1/64:", h[2048:2048 + 64].tolist())
