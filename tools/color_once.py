"""One COLOR call on R-MAT (for ncu launch lists): python tools/color_once.py [scale] [kind] [param]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
kind = sys.argv[2] if len(sys.argv) > 2 else "degk"
param = int(sys.argv[3]) if len(sys.argv) > 3 else 2
dev = torch.device("cuda", 0)
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, kind, param, 42) if kind != "none" else None
col = sb.sym_color(rp, ci, kind, param, 42, decomp=d)
torch.cuda.synchronize()
print("max colour", int(col.max()))
