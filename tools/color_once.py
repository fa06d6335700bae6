"""One COLOR-Deg2 call on R-MAT (for ncu captures of the JP kernels)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
col = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d)
torch.cuda.synchronize()
print("max colour", int(col.max()))
