"""Benchmark: decomposition-based symmetry breaking on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

One STEP = one pass of the whole hot path (every SURVEY §8(a) row) over the
synthetic workload of BASELINE.json configs[2]/[3] -- R-MAT scale 24, edge factor
16 (Graph500 parameters; m = 260.4 M undirected edges, 520.8 M arcs):
    DEG2 decomposition -> MIS-Deg2 -> COLOR-Deg2   (one shared decomposition)
    RAND p=4 decomposition -> MM-Rand               (p = 4 is the paper's GPU value)
value = m / (device time of one step) [edges/s].  Inputs (col_idx 2.08 GB) exceed
the 126 MB L2, so no flush is needed between steps.

Also in the one JSON line:
  roofline     the dominant kernel class, achieved = §8(d) ALGORITHMIC bytes per launch
               (counted by the kernels / known on the host) / its average launch time
               (CUDA events on the launch stream); impl_bytes = the implementation's
               own words; traffic = ncu DRAM bytes per launch from the committed
               `--cache-control none` capture of this step (profiles/*traffic*.json)
  configs      one entry per BASELINE config: C1 s14 MIS-Rand4, C2 road grid
               MM-Rand64, C3 s24 MIS-Deg2 + MIS-NONE, C4 s24 COLOR-Deg2 / COLOR-Rand4
               / MM-Rand4 / MM-NONE (C5, scale 27, with --c5), each with the
               rooflines of its round kernels on §8(d) bytes
  cpu_baseline the round-based oracle on all host cores (oracle_rounds_omp) and the
               sequential oracle on 1 core, both on the SAME s24 CSR and the same step,
               both checked bit-exact against the GPU outputs
  paper_context PAPER.md Table I speedups with their hardware (context, not targets)
  e2e          the same step through the public API with the CSR copied from pinned
               host memory and the results copied back, every step
Multi-GPU (torchrun, N > 1): every rank owns a 1/N vertex block of ONE graph and
the step runs sharded through the library (sym_*_sharded, NCCL exchange inside
libsym); "scaling": "strong" at scale 24.
"""
from __future__ import annotations

import argparse
import glob
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MIS/MM/COLOR edges/s at 1/2/4/8 B200; % of HBM roofline; vs CPU oracle"

# PAPER.md Table I and §III-V text: the paper's speedups over its own
# non-decomposed baselines, with the hardware they were measured on.  Context only.
PAPER_CONTEXT = {
    "source": "PAPER.md Table I (P:31-38), P:186-196, P:246-250, P:298-300",
    "hardware": {"cpu": "Intel Xeon E5-2650, 2x10 cores, 2.3 GHz, 68 GB/s, 80 threads",
                 "gpu": "NVIDIA Tesla K40c (Kepler, 15 SMs, 745 MHz, 288 GB/s)"},
    "speedups": {"MM-Rand vs GM (CPU)": "3.5x", "MM-Rand vs LMAX (GPU)": "2.53x",
                 "COLOR-Deg2 vs VB (CPU)": "1.27x", "COLOR-Rand vs EB (GPU)": "1x",
                 "MIS-Deg2 vs LubyMIS (CPU)": "3.39x", "MIS-Deg2 vs LubyMIS (GPU)": "2.16x"},
    "note": "speedups of decomposed over non-decomposed runs on the paper's Table II graphs; "
            "no absolute edges/s are published (BASELINE.md §1)",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--ef", type=int, default=16)
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--no-cpu", action="store_true", help="skip the CPU oracle baselines")
    ap.add_argument("--no-seq", action="store_true", help="skip the 1-core sequential oracle (~1 min at s24)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-configs", action="store_true")
    ap.add_argument("--c5", action="store_true", help="also run C5 (R-MAT scale 27) on this GPU")
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--reps", type=int, default=7, help="timed repetitions per config problem (median)")
    ap.add_argument("--profile-only", action="store_true", help="short run for ncu (no JSON contract)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        try:
            p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                  "--format=csv,noheader,nounits", "-lms", "200"],
                                 stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            return
        while not self._stop.is_set():
            line = p.stdout.readline()
            if not line:
                break
            self.samples.append([x.strip() for x in line.split(",")])
        p.terminate()

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        time.sleep(0.25)
        self._stop.set()
        self._t.join(timeout=2)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if len(s) > i + 2 and s[i + 2].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def cpu_model():
    try:
        for line in subprocess.check_output(["lscpu"], text=True).splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except (OSError, subprocess.CalledProcessError):
        pass
    return None


# ------------------------------------------------------------------ CPU oracle step
def oracle_step(rp, ci, seed, omp):
    """The bench step (MIS-Deg2 + COLOR-Deg2 + MM-Rand4) by the CPU oracle: the
    round-based all-core form (omp) or the sequential greedy form (1 core)."""
    import oracle as O
    fm, fc, fmm = (O.omp_mis, O.omp_color, O.omp_mm) if omp else (O.mis, O.color, O.mm)
    t = time.perf_counter()
    I = fm(rp, ci, "degk", 2, seed)
    C = fc(rp, ci, "degk", 2, seed)
    M = fmm(rp, ci, "rand", 4, seed)
    return time.perf_counter() - t, (I, C, M)


def host_graph(scale, ef):
    """The bench graph on the host: generated with torch on the GPU when one is visible
    (graphgen: input infrastructure, not the library; bit-identical to the CPU
    generator), else on the CPU."""
    import torch
    import graphgen
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    rp, ci = graphgen.rmat(scale, ef, seed=1, device=dev)
    return rp.cpu().numpy(), ci.cpu().numpy()


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as it stands -- the round-based form on all host
    cores (oracle_rounds_omp) -- on the SAME workload as our arm (R-MAT s24 ef16, the
    full step), rank 0 only."""
    if rank != 0:
        return
    import oracle as O
    O.build()
    rp, ci = host_graph(args.scale, args.ef)
    m = ci.size // 2
    for _ in range(max(0, min(args.warmup, 1))):
        oracle_step(rp, ci, args.seed, True)
    ts = [oracle_step(rp, ci, args.seed, True)[0] for _ in range(args.steps)]
    T = statistics.median(ts)
    v = m / T
    cores = O.omp_threads()
    sample = (f"R-MAT scale {args.scale} ef {args.ef} (m={m}), the full step (MIS-Deg2 + COLOR-Deg2 + MM-Rand4) "
              f"by oracle_rounds_omp (LubyMIS / JP / LMAX rounds) on {cores} threads; warm-up capped at 1")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "edges/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": T * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"rmat{args.scale}-ef{args.ef}: DEG2{{MIS,COLOR}} + RAND4{{MM}}"},
        "cpu_baseline": {"value": v, "unit": "edges/s", "cores": cores, "kind": "oracle", "sample": sample,
                         "cpu_model": cpu_model()},
        "e2e": {"value": v, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ------------------------------------------------------------------ measurement helpers
def load_traffic():
    """ncu DRAM bytes per launch per kernel class, from the newest committed capture
    (`tools/ncu_traffic.py`: --cache-control none, this step)."""
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "*traffic*.json")))
    if not files:
        return {}, None
    try:
        d = json.load(open(files[-1]))
    except (OSError, ValueError):
        return {}, None
    return d.get("classes", {}), os.path.relpath(files[-1], ROOT)


def merge_classes(prof, groups):
    """{group: [classes]} -> summed {launches, ms, alg_bytes, impl_bytes} (classes absent
    from prof are skipped; the launch count is that of the first present class)."""
    out = {}
    for g, names in groups.items():
        present = [c for c in names if c in prof]
        if not present:
            continue
        out[g] = {"launches": prof[present[0]]["launches"], "ms": sum(prof[c]["ms"] for c in present),
                  "alg_bytes": sum(max(0.0, prof[c]["alg_bytes"]) for c in present),
                  "impl_bytes": sum(max(0.0, prof[c]["impl_bytes"]) for c in present),
                  "classes": present}
    return out


def roofline(name, v, calls, peak, peak_src, traffic, traffic_src, step_ms=None):
    """Roofline object of one kernel class (v: profile sums over `calls` calls)."""
    if v["launches"] <= 0 or v["ms"] <= 0:
        return None
    per_launch_s = v["ms"] / v["launches"] * 1e-3
    alg = v["alg_bytes"] / v["launches"]
    impl = v["impl_bytes"] / v["launches"]
    ach = alg / per_launch_s / 1e9
    classes = v.get("classes", [name])
    tr = None
    if traffic:
        have = [traffic[c]["dram_bytes_per_launch"] for c in classes if c in traffic]
        tr = sum(have) if have else None
    r = {"kernel": name, "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
         "traffic": tr, "traffic_source": traffic_src if tr is not None else None, "peak_source": peak_src,
         "alg_bytes_per_launch": alg, "impl_bytes_per_launch": impl,
         "impl_frac": impl / per_launch_s / 1e9 / peak,
         "ms_per_launch": per_launch_s * 1e3, "launches_per_call": v["launches"] / calls}
    if len(classes) > 1:
        r["classes"] = classes
    if traffic:
        # ncu's own view of the same class in the same capture: L2 / DRAM throughput
        # fractions (time-weighted lts__throughput / dram__throughput) -- the gather-bound
        # round kernels are judged against the L2 as well as HBM
        l2 = [(traffic[c]["l2_frac"], traffic[c]["us"]) for c in classes if c in traffic and "l2_frac" in traffic[c]]
        if l2 and sum(t for _, t in l2) > 0:
            r["l2_frac_ncu"] = sum(f * t for f, t in l2) / sum(t for _, t in l2)
        dr = [(traffic[c]["dram_frac"], traffic[c]["us"]) for c in classes if c in traffic and "dram_frac" in traffic[c]]
        if dr and sum(t for _, t in dr) > 0:
            r["dram_frac_ncu"] = sum(f * t for f, t in dr) / sum(t for _, t in dr)
    if step_ms:
        r["share_of_step"] = (v["ms"] / calls) / step_ms
    return r


# ------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist

    import graphgen
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    from paper_conf_ipps_nayyaroddeengk17_b200 import build as B

    if rank == 0:
        B.build()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        dist.barrier()
    if rank != 0:
        B.build()
    if world > 1:
        from paper_conf_ipps_nayyaroddeengk17_b200 import shardstep
        shardstep.bench(args, rank, world, dev, METRIC, ClockSampler)
        dist.destroy_process_group()
        return

    t0 = time.time()
    rp, ci = graphgen.rmat(args.scale, args.ef, seed=1, device=dev)
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    n, nnz = rp.numel() - 1, ci.numel()
    m = nnz // 2
    seed = args.seed

    def step(rp=rp, ci=ci):
        dD = sb.sym_decompose(rp, ci, "degk", 2, seed)
        I = sb.sym_mis(rp, ci, "degk", 2, seed, decomp=dD)
        C = sb.sym_color(rp, ci, "degk", 2, seed, decomp=dD)
        dR = sb.sym_decompose(rp, ci, "rand", 4, seed)
        M = sb.sym_mm(rp, ci, "rand", 4, seed, decomp=dR)
        return I, C, M

    if args.profile_only:
        for _ in range(max(0, args.warmup)):
            step()
        torch.cuda.synchronize()
        for _ in range(max(1, args.steps)):
            step()
        torch.cuda.synchronize()
        return

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    stream = torch.cuda.current_stream(dev)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
    ms_step = ev0.elapsed_time(ev1) / args.steps
    value = m / (ms_step * 1e-3)
    I_gpu, C_gpu, M_gpu = [x.cpu().numpy() for x in step()]

    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    peak_src = "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if "hbm_gbs" in peaks else "B200_PROFILING fallback 6.65 TB/s"
    traffic, traffic_src = load_traffic()

    def timed(fn, reps):
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)

    def profiled(fn, calls):
        """Per-class profile over `calls` calls: device times from an events-only pass
        (mode 2: the kernels' byte counters cost time -- MIS rounds ran 2.4x slower with
        them), byte counts from one counting pass (mode 1), scaled per launch."""
        sb.sym_profile_enable(1)
        fn()  # the first profiled call allocates the hook's counters
        torch.cuda.synchronize()
        sb.sym_profile_collect()
        fn()
        torch.cuda.synchronize()
        counted = sb.sym_profile_collect()
        sb.sym_profile_enable(2)
        for _ in range(calls):
            fn()
        torch.cuda.synchronize()
        prof = sb.sym_profile_collect()
        sb.sym_profile_enable(False)
        for c, v in prof.items():
            b = counted.get(c)
            for key in ("alg_bytes", "impl_bytes"):
                if b is None or b[key] < 0 or b["launches"] <= 0:
                    v[key] = -1.0
                else:  # bytes of one counted call, spread over this pass's launches
                    v[key] = b[key] * calls
        return prof

    # ---- per-problem breakdown of the step (events between the calls)
    steps_p = max(1, min(args.steps, 3))
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
    brk = {"decompose_deg2": 0.0, "mis_deg2": 0.0, "color_deg2": 0.0, "decompose_rand4": 0.0, "mm_rand4": 0.0}
    for _ in range(steps_p):
        evs[0].record(stream)
        dD = sb.sym_decompose(rp, ci, "degk", 2, seed)
        evs[1].record(stream)
        sb.sym_mis(rp, ci, "degk", 2, seed, decomp=dD)
        evs[2].record(stream)
        sb.sym_color(rp, ci, "degk", 2, seed, decomp=dD)
        evs[3].record(stream)
        dR = sb.sym_decompose(rp, ci, "rand", 4, seed)
        evs[4].record(stream)
        sb.sym_mm(rp, ci, "rand", 4, seed, decomp=dR)
        evs[5].record(stream)
        torch.cuda.synchronize()
        for i, k in enumerate(brk):
            brk[k] += evs[i].elapsed_time(evs[i + 1]) / steps_p
    del dD, dR

    # ---- per-kernel-class device times and bytes through the library's event hook
    prof = profiled(step, steps_p)
    merged = merge_classes(prof, {c: [c] for c in prof})
    rooflines = {k: roofline(k, v, steps_p, hbm_peak, peak_src, traffic, traffic_src, ms_step)
                 for k, v in merged.items()}
    rooflines = {k: v for k, v in rooflines.items() if v}
    dominant = max(merged, key=lambda k: merged[k]["ms"]) if merged else None
    roof = rooflines.get(dominant)
    _, st_mis = sb.sym_mis(rp, ci, "degk", 2, seed, stats=True, flags=2)
    _, st_col = sb.sym_color(rp, ci, "degk", 2, seed, stats=True, flags=2)
    _, st_mm = sb.sym_mm(rp, ci, "rand", 4, seed, stats=True, flags=2)
    if roof is not None and dominant == "jp_rounds":
        rounds = st_col["rounds"][0]
        roof["latency_model"] = {
            "rounds": rounds, "plain_jp_levels": 5063, "us_per_round": roof["ms_per_launch"] * 1e3 / max(1, rounds),
            "note": "round-bound: rounds x (dependent L2/DRAM round trips + 2 grid barriers); early-commit JP in "
                    "one cooperative grid kernel (DESIGN §7)"}

    # ---- per-config lines (BASELINE.json configs)
    configs = None
    if not args.no_configs:
        configs = run_configs(args, sb, graphgen, torch, dev, rp, ci, timed, profiled, hbm_peak, peak_src,
                              traffic, traffic_src)

    # ---- e2e through the public API with pinned host buffers
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, torch, dev, stream, rp, ci, step, m, n)

    # ---- CPU oracle baselines on the SAME CSR (rank 0, N = 1)
    cpu = None
    if not args.no_cpu:
        cpu = run_cpu(args, rp, ci, seed, m, (I_gpu, C_gpu, M_gpu))

    launches = sum(v["launches"] for v in prof.values()) / steps_p
    out = {
        "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"rmat{args.scale}-ef{args.ef}: DEG2{{MIS,COLOR}} + RAND4{{MM}}",
                   "n": n, "m": m, "arcs": nnz, "seed": seed, "graph_seed": 1, "parallelism": "single",
                   "schedule": "sequential (one stream)",
                   "l2": "inputs exceed L2 (col_idx %.2f GB > 126 MB), no flush" % (nnz * 4 / 1e9),
                   "generate_s": round(gen_s, 2)},
        "breakdown_ms": brk,
        "breakdown_edges_per_s": {"mis_deg2_incl_decomp": m / ((brk["decompose_deg2"] + brk["mis_deg2"]) * 1e-3),
                                  "color_deg2_incl_decomp": m / ((brk["decompose_deg2"] + brk["color_deg2"]) * 1e-3),
                                  "mm_rand4_incl_decomp": m / ((brk["decompose_rand4"] + brk["mm_rand4"]) * 1e-3)},
        "dominant_kernel": dominant, "roofline": roof, "rooflines": rooflines,
        "roofline_bytes": "alg = SURVEY §8(d): rounds 4 B/scanned arc + 9 B/active vertex; split 8 B/arc + "
                          "24 B/row pointer; JP 8 B/arc + 12 B/vertex (DESIGN §7); impl = the kernels' own words",
        "configs": configs, "cpu_baseline": cpu, "paper_context": PAPER_CONTEXT, "e2e": e2e,
        "gpu_launches": int(round(launches)),
        "clocks": clk.summary(),
        "stats": {"mis": st_mis, "color": st_col, "mm": st_mm},
    }
    print(json.dumps(out), flush=True)


def run_configs(args, sb, graphgen, torch, dev, rp24, ci24, timed, profiled, peak, peak_src, traffic, traffic_src):
    """One entry per BASELINE config.  Each problem: median device time of
    (decomposition + problem) over --reps calls, edges/s = m / that, rounds, and the
    rooflines of its kernel classes on §8(d) bytes (one profiled call)."""
    seed = args.seed
    round_groups = {"mis": {"rounds": ["mis_round", "mis_huge", "mis_round0"]},
                    "mm": {"rounds": ["mm_round0", "mm_round", "mm_huge"], "round0": ["mm_round0"],
                           "later_rounds": ["mm_round", "mm_huge"]},
                    "color": {"jp_rounds": ["jp_rounds"], "jp_build": ["jp_build"]}}
    fns = {"mis": sb.sym_mis, "mm": sb.sym_mm, "color": sb.sym_color}

    def problem(rp, ci, prob, kind, p):
        m = ci.numel() // 2

        def call():
            d = sb.sym_decompose(rp, ci, kind, p, seed) if kind != "none" else None
            return fns[prob](rp, ci, kind, p, seed, decomp=d)
        call()
        ms = timed(call, args.reps)
        d = sb.sym_decompose(rp, ci, kind, p, seed) if kind != "none" else None
        ms_solve = timed(lambda: fns[prob](rp, ci, kind, p, seed, decomp=d), args.reps)
        prof = profiled(lambda: fns[prob](rp, ci, kind, p, seed, decomp=d), 1)
        _, st = fns[prob](rp, ci, kind, p, seed, decomp=d, stats=True, flags=2)
        merged = merge_classes(prof, round_groups[prob])
        rl = {k: roofline(k, v, 1, peak, peak_src, traffic, traffic_src) for k, v in merged.items()}
        per_class = {k: {"launches": v["launches"], "ms": v["ms"], "alg_bytes": v["alg_bytes"],
                         "impl_bytes": v["impl_bytes"]} for k, v in prof.items()}
        del d
        return {"ms_incl_decomp": ms, "ms_problem_only": ms_solve, "edges_per_s": m / (ms * 1e-3),
                "rounds": st["rounds"], "result_size": st["result_size"],
                "rooflines": {k: v for k, v in rl.items() if v}, "classes": per_class}

    out = {}
    rp, ci = graphgen.rmat(14, 8, seed=1, device=dev)
    out["C1"] = {"graph": "R-MAT s14 ef8", "n": rp.numel() - 1, "m": ci.numel() // 2,
                 "note": "L2-resident, latency-bound: edges/s, no meaningful roofline (SURVEY §8(d))",
                 "mis_rand4": problem(rp, ci, "mis", "rand", 4)}
    rp, ci = graphgen.grid(2048, 2048, 0.6, seed=1, device=dev)
    out["C2"] = {"graph": "road-like grid 2048^2 keep 0.6", "n": rp.numel() - 1, "m": ci.numel() // 2,
                 "mm_rand64": problem(rp, ci, "mm", "rand", 64)}
    del rp, ci
    out["C3"] = {"graph": "R-MAT s24 ef16 (the step's graph)", "mis_deg2": problem(rp24, ci24, "mis", "degk", 2),
                 "mis_none": problem(rp24, ci24, "mis", "none", 0)}
    out["C4"] = {"graph": "R-MAT s24 ef16 (the step's graph)",
                 "color_deg2": problem(rp24, ci24, "color", "degk", 2),
                 "color_rand4": problem(rp24, ci24, "color", "rand", 4),
                 "mm_rand4": problem(rp24, ci24, "mm", "rand", 4),
                 "mm_none": problem(rp24, ci24, "mm", "none", 0)}
    torch.cuda.empty_cache()
    if args.c5:
        rp, ci = graphgen.rmat(27, 16, seed=1, device=dev)
        out["C5"] = {"graph": "R-MAT s27 ef16 (1 GPU)", "n": rp.numel() - 1, "m": ci.numel() // 2,
                     "mis_deg2": problem(rp, ci, "mis", "degk", 2),
                     "color_deg2": problem(rp, ci, "color", "degk", 2),
                     "mm_rand8": problem(rp, ci, "mm", "rand", 8)}
        del rp, ci
        torch.cuda.empty_cache()
    return out


def run_e2e(args, torch, dev, stream, rp, ci, step, m, n):
    """Every step copies its input CSR host->device (pinned) and its three results
    device->host.  Double-buffered: step i+1's input is copied on a copy stream while
    step i computes."""
    rp_h = rp.cpu().pin_memory()
    ci_h = ci.cpu().pin_memory()
    dbuf = [(torch.empty_like(rp), torch.empty_like(ci)) for _ in range(2)]
    out_h = (torch.empty(n, dtype=torch.uint8).pin_memory(), torch.empty(n, dtype=torch.int32).pin_memory(),
             torch.empty(n, dtype=torch.int32).pin_memory())
    sc = torch.cuda.Stream(dev)
    copied = [torch.cuda.Event() for _ in range(2)]
    consumed = [torch.cuda.Event() for _ in range(2)]
    K = args.e2e_steps

    def h2d(slot):
        with torch.cuda.stream(sc):
            dbuf[slot][0].copy_(rp_h, non_blocking=True)
            dbuf[slot][1].copy_(ci_h, non_blocking=True)
            copied[slot].record(sc)

    # warm-up (untimed): both input buffers and the result copies once -- the first DMA
    # from freshly pinned pages ran 2.5x slower on one box (115 vs 46 ms per step)
    for slot in range(2):
        h2d(slot)
    sc.synchronize()
    I, C, M = step(*dbuf[0])
    for h, d in zip(out_h, (I, C, M)):
        h.copy_(d)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    sc.wait_stream(stream)
    h2d(0)
    for i in range(K):
        cur = i % 2
        if i + 1 < K:
            if i >= 1:
                sc.wait_event(consumed[(i + 1) % 2])  # that buffer fed step i-1
            h2d((i + 1) % 2)
        stream.wait_event(copied[cur])
        I, C, M = step(*dbuf[cur])
        consumed[cur].record(stream)
        sc.wait_event(consumed[cur])
        with torch.cuda.stream(sc):
            for h, d in zip(out_h, (I, C, M)):
                d.record_stream(sc)  # keep the block alive until sc's copy has run
                h.copy_(d, non_blocking=True)
    stream.wait_stream(sc)
    e1.record(stream)
    torch.cuda.synchronize()
    e_ms = e0.elapsed_time(e1) / K
    return {"value": m / (e_ms * 1e-3), "unit": "edges/s",
            "h2d_bytes_per_step": rp_h.numel() * 8 + ci_h.numel() * 4,
            "d2h_bytes_per_step": sum(x.numel() * x.element_size() for x in out_h),
            "ms_per_step": e_ms, "steps": K, "pipeline": "double-buffered: step i+1's H2D copy overlaps step i"}


def run_cpu(args, rp, ci, seed, m, gpu_out):
    """The oracle on the SAME CSR as the GPU step: all-core round form and 1-core
    sequential form; each result compared bit for bit with the GPU's."""
    import numpy as np
    import oracle as O
    O.build()
    hrp, hci = rp.cpu().numpy(), ci.cpu().numpy()
    I, C, M = gpu_out

    def same(res):
        return bool(np.array_equal(res[0], I) and np.array_equal(res[1].astype(np.int64), C.astype(np.int64))
                    and np.array_equal(res[2], M))
    T, res = oracle_step(hrp, hci, seed, True)
    cores = O.omp_threads()
    sample = (f"the SAME R-MAT s{args.scale} ef{args.ef} CSR as the GPU step (m={m}), the full step "
              f"(MIS-Deg2 + COLOR-Deg2 + MM-Rand4), one run")
    cpu = {"value": m / T, "unit": "edges/s", "cores": cores, "kind": "oracle",
           "oracle": "oracle_rounds_omp (LubyMIS / JP levels / LMAX rounds, OpenMP)", "seconds": T,
           "sample": sample, "matches_gpu": same(res), "cpu_model": cpu_model(), "host_cpus": os.cpu_count()}
    if not args.no_seq:
        T1, res1 = oracle_step(hrp, hci, seed, False)
        cpu["single_core"] = {"value": m / T1, "unit": "edges/s", "cores": 1, "seconds": T1,
                              "oracle": "oracle_seq (sequential greedy, the parity authority)",
                              "matches_gpu": same(res1)}
    return cpu


if __name__ == "__main__":
    main()
