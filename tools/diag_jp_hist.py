"""Diagnostic: JP tasks and lower-neighbour pushes per round (first 2048 rounds),
read from the control block (needs SYM_DEBUG_JP=1 for pushes)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
C, st = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d, stats=True)
ws = sb._WS[0]
off = ((ws.data_ptr() + 255) & ~255) - ws.data_ptr()
hist = ws[off + 136: off + 136 + 16384].cpu().numpy().view(np.uint32)
np.save(os.path.join(os.environ.get("GRAFT_REPO_ROOT", "."), "gpurun_out", "jp_hist.npy"), hist)
print("rounds", st["rounds"], "tasks[:10]", hist[:10].tolist(), "pushes[:10]", hist[2048:2058].tolist())
