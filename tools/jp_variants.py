"""Diagnostic: build libsym variants with -D overrides and time COLOR-Deg2 on R-MAT.

    python tools/jp_variants.py build            # here (nvcc), into build/variants/
    python tools/jp_variants.py run [scale]      # on the GPU box
"""
import json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
OUT = os.path.join(ROOT, "build", "variants")
VARIANTS = {  # the last comparison run (DESIGN §7 records the others)
    "base": [],
    "t256x4": ["-DSYM_JR_THREADS=256", "-DSYM_JR_MINB=4"],
    "t1024x1": ["-DSYM_JR_THREADS=1024", "-DSYM_JR_MINB=1"],
    "lc2": ["-DSYM_JP_LANE_CHECKS=2"],
}

if sys.argv[1] == "build":
    from paper_conf_ipps_nayyaroddeengk17_b200 import build as b
    os.makedirs(OUT, exist_ok=True)
    for name, defs in VARIANTS.items():
        cmd = [b.NVCC, *b.ARCH, *b.FLAGS, *defs, "-I", os.path.join(ROOT, "include"),
               "-o", os.path.join(OUT, f"libsym_{name}.so"), *b.sources()]
        subprocess.check_call(cmd)
        print("built", name, flush=True)
elif sys.argv[1] == "child":
    import torch, graphgen, paper_conf_ipps_nayyaroddeengk17_b200 as sb
    scale = int(sys.argv[2])
    dev = torch.device("cuda", 0)
    rp, ci = graphgen.rmat(scale, 16, seed=1, device=dev)
    d = sb.sym_decompose(rp, ci, "degk", 2, 42)
    ts, ref = [], None
    for it in range(4):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); col = sb.sym_color(rp, ci, "degk", 2, 42, decomp=d); e1.record(); torch.cuda.synchronize()
        ts.append(round(e0.elapsed_time(e1), 2))
    import hashlib
    print(json.dumps({"lib": os.path.basename(os.environ["SYM_LIB"]), "ms": ts,
                      "sha": hashlib.sha1(col.cpu().numpy().tobytes()).hexdigest()[:12]}), flush=True)
else:
    scale = sys.argv[2] if len(sys.argv) > 2 else "24"
    for name in VARIANTS:
        env = dict(os.environ, SYM_LIB=os.path.join(OUT, f"libsym_{name}.so"))
        subprocess.run([sys.executable, __file__, "child", scale], env=env, timeout=600)
