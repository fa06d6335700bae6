import os, sys; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import sys, torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device("cuda", 0)
rp, ci = graphgen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 24, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, "degk", 2, 42)
for _ in range(2):
    sb.sym_color(rp, ci, "degk", 2, 42, decomp=d)
torch.cuda.synchronize()
