"""Diagnostic: time the JP drivers (levels / async / rounds) on R-MAT; parity vs levels."""
import os, subprocess, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

if len(sys.argv) > 1 and sys.argv[1] == "child":
    import torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
    scale, kind, param = int(sys.argv[2]), sys.argv[3], int(sys.argv[4])
    dev = torch.device("cuda", 0)
    rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
    d = sb.sym_decompose(rp, ci, kind, param, 42) if kind != "none" else None
    out = None
    ts = []
    for it in range(4):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        res = sb.sym_color(rp, ci, kind, param, 42, decomp=d, stats=(it == 0))
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        if it == 0:
            col, st = res
            out = col
    import hashlib
    h = hashlib.sha1(out.cpu().numpy().tobytes()).hexdigest()[:16]
    print(json.dumps({"mode": os.environ.get("SYM_JP_MODE", "levels"), "scale": scale, "kind": kind,
                      "ms": ts, "sha": h, "rounds": st.get("rounds"),
                      "max_color": int(out.max())}), flush=True)
    sys.exit(0)

scale = sys.argv[1] if len(sys.argv) > 1 else "24"
for kind, param in (("degk", "2"), ("none", "0")):
    for mode in ("levels", "async", "rounds"):
        env = dict(os.environ, SYM_JP_MODE=mode)
        subprocess.run([sys.executable, __file__, "child", scale, kind, param], env=env, timeout=600)
