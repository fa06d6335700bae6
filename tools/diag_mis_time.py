import sys, time, torch
sys.path.insert(0, '/root/repo')
import graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
dev = torch.device('cuda', 0)
rp, ci = graphgen.rmat(24, 16, seed=1, device=dev)
d = sb.sym_decompose(rp, ci, 'degk', 2, 42)
def t(f, k=3):
    out = []
    for _ in range(k):
        torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        h0 = time.perf_counter(); e0.record(); f(); e1.record(); torch.cuda.synchronize(); out.append((round(e0.elapsed_time(e1), 2), round((time.perf_counter() - h0) * 1e3, 2)))
    return out
print('mis first', t(lambda: sb.sym_mis(rp, ci, 'degk', 2, 42, decomp=d)))
print('color', t(lambda: sb.sym_color(rp, ci, 'degk', 2, 42, decomp=d), 1))
print('mis after color', t(lambda: sb.sym_mis(rp, ci, 'degk', 2, 42, decomp=d)))
sb.sym_profile_enable(True)
print('mis profiled', t(lambda: sb.sym_mis(rp, ci, 'degk', 2, 42, decomp=d)))
print(sb.sym_profile_collect())
