"""Benchmark: decomposition-based symmetry breaking on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

One STEP = one pass of the whole hot path (every SURVEY §8(a) row) over the
synthetic workload of BASELINE.json configs[2]/[3] -- R-MAT scale 24, edge factor
16 (Graph500 parameters; m = 260.4 M undirected edges, 520.8 M arcs):
    DEG2 decomposition -> MIS-Deg2 -> COLOR-Deg2   (one shared decomposition)
    RAND p=4 decomposition -> MM-Rand               (p = 4 is the paper's GPU value)
value = m / (device time of one step) [edges/s]; per-problem edges/s are in
"breakdown".  Inputs (col_idx 2.08 GB) exceed the 126 MB L2, so no flush is needed
between steps.  Multi-GPU (torchrun): every rank runs an independent replica of the
step (weak scaling, "replicas"; the sharded exchange path is not yet built).
"""
from __future__ import annotations

import argparse
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

# per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) of each kernel
# class from one `ncu --set full` capture of this step (profiles/r1*_ncu*.md);
# None where no capture was taken for the current code.
TRAFFIC = {
    "split": 4.51e9,       # k_split<DEGK> / <RAND> at R-MAT s24 (profiles/r1b_ncu.md): 2.22 GB read + 2.29 GB written
    "mm_round0": 0.719e9,  # k_round0<MM> on the RAND-4 intra CSR
    # COLOR-Deg2 at R-MAT s24 (profiles/r1i_color_launches.csv): the build kernels
    # (k_jpc_*: compact ids, counts, lists) and the early-commit rounds kernel
    "jp_build": 8.46e9,
    "jp_rounds": 17.12e9,  # k_jp_rounds: 14.72 GB read + 2.40 GB written (lists, meta, hot records)
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
    ap.add_argument("--cpu-scale", type=int, default=20, help="R-MAT scale of the bounded oracle sample")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--profile-only", action="store_true", help="short run for ncu (no JSON contract)")
    ap.add_argument("--sequential", action="store_true", help="one stream, the five calls in order (default)")
    ap.add_argument("--concurrent", action="store_true",
                    help="two streams (schedule.ConcurrentStep); slower since the early-commit JP kernel "
                         "holds every SM's register file")
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


# ------------------------------------------------------------------ CPU oracle sample
def oracle_step(rp, ci, seed):
    import oracle as O
    t = time.perf_counter()
    O.mis(rp, ci, "degk", 2, seed)
    O.color(rp, ci, "degk", 2, seed)
    O.mm(rp, ci, "rand", 4, seed)
    return time.perf_counter() - t


def cpu_sample(scale, ef):
    import graphgen
    rp, ci = graphgen.rmat(scale, ef, seed=1)
    return rp.numpy(), ci.numpy()


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (as it stands, 1 thread) on a bounded sample."""
    if rank != 0:
        return
    import oracle as O
    O.build()
    rp, ci = cpu_sample(args.cpu_scale, args.ef)
    m = ci.size // 2
    for _ in range(max(0, min(args.warmup, 1))):
        oracle_step(rp, ci, args.seed)
    ts = [oracle_step(rp, ci, args.seed) for _ in range(args.steps)]
    T = sum(ts) / len(ts)
    v = m / T
    sample = f"R-MAT scale {args.cpu_scale} ef {args.ef} (m={m}), same step (MIS-Deg2 + COLOR-Deg2 + MM-Rand4)"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "edges/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": T * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"rmat{args.scale}-ef{args.ef}: DEG2{{MIS,COLOR}} + RAND4{{MM}}",
                   "sample_workload": sample},
        "cpu_baseline": {"value": v, "unit": "edges/s", "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": v, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


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

    t0 = time.time()
    rp, ci = graphgen.rmat(args.scale, args.ef, seed=1, device=dev)
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    n, nnz = rp.numel() - 1, ci.numel()
    m = nnz // 2
    seed = args.seed + rank

    def step_sequential(rp=rp, ci=ci):
        dD = sb.sym_decompose(rp, ci, "degk", 2, seed)
        I = sb.sym_mis(rp, ci, "degk", 2, seed, decomp=dD)
        C = sb.sym_color(rp, ci, "degk", 2, seed, decomp=dD)
        dR = sb.sym_decompose(rp, ci, "rand", 4, seed)
        M = sb.sym_mm(rp, ci, "rand", 4, seed, decomp=dR)
        return I, C, M

    from paper_conf_ipps_nayyaroddeengk17_b200.schedule import ConcurrentStep
    _cs = ConcurrentStep(dev, seed)

    def step_concurrent(rp=rp, ci=ci):
        return _cs(rp, ci)

    args.sequential = not args.concurrent
    step = step_sequential if args.sequential else step_concurrent

    if args.profile_only:
        for _ in range(max(1, args.warmup)):
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
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = ev0.elapsed_time(ev1)
    if world > 1:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / args.steps
    value = world * m / (ms_step * 1e-3)

    # ---- per-problem breakdown (events between the calls, no profiling hook) ...
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
    # ... and per-kernel-class device times through the library's event hook (separate pass)
    sb.sym_profile_enable(True)
    step_sequential()  # first profiled call allocates the hook's counters
    torch.cuda.synchronize()
    sb.sym_profile_collect()
    for _ in range(steps_p):
        step_sequential()
    torch.cuda.synchronize()
    prof = sb.sym_profile_collect()
    sb.sym_profile_enable(False)
    _, st_mis = sb.sym_mis(rp, ci, "degk", 2, seed, stats=True, flags=2)
    _, st_col = sb.sym_color(rp, ci, "degk", 2, seed, stats=True, flags=2)
    _, st_mm = sb.sym_mm(rp, ci, "rand", 4, seed, stats=True, flags=2)

    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    peak_src = "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if "hbm_gbs" in peaks else "B200_PROFILING fallback 6.65 TB/s"
    # dominant kernel among the classes with exactly known algorithmic bytes
    per_step = {k: {"ms_per_step": v["ms"] / steps_p, "launches_per_step": v["launches"] / steps_p,
                    "alg_bytes_per_step": (v["alg_bytes"] / steps_p) if v["alg_bytes"] >= 0 else None}
                for k, v in prof.items()}
    def roof_of(name):
        v = prof[name]
        if v["alg_bytes"] <= 0 or v["ms"] <= 0:
            return None
        per_launch_bytes = v["alg_bytes"] / v["launches"]
        per_launch_s = v["ms"] / v["launches"] * 1e-3
        ach = per_launch_bytes / per_launch_s / 1e9
        return {"kernel": name, "bound": "hbm", "achieved": ach, "peak": hbm_peak, "unit": "GB/s",
                "frac": ach / hbm_peak, "traffic": TRAFFIC.get(name), "peak_source": peak_src,
                "alg_bytes_per_launch": per_launch_bytes, "ms_per_launch": per_launch_s * 1e3,
                "launches_per_step": v["launches"] / steps_p, "share_of_step": (v["ms"] / steps_p) / ms_step}

    # the dominant kernel = the class with the most device time in the step
    dominant_overall = max(prof, key=lambda k: prof[k]["ms"]) if prof else None
    roof = roof_of(dominant_overall) if dominant_overall else None
    if roof is not None and dominant_overall == "jp_rounds":
        # the colouring is bound by its number of dependent rounds, not by bytes: a
        # round = checks, grid barrier, pushes, grid barrier
        rounds = st_col["rounds"][0]
        roof["latency_model"] = {
            "rounds": rounds, "plain_jp_levels": 5063, "us_per_round": roof["ms_per_launch"] * 1e3 / max(1, rounds),
            "grid_barriers_per_round": 2, "note": "round-bound: rounds x (dependent L2/DRAM round trips + 2 grid "
            "barriers); HBM frac is reported for the algorithmic bytes only"}
    rooflines = {k: roof_of(k) for k in prof if roof_of(k)}

    # ---- e2e through the public API with pinned host buffers: every step copies its
    #      input CSR host->device and its three results device->host.  Double-buffered:
    #      step i+1's input is copied on a copy stream while step i computes.
    e2e = None
    if not args.no_e2e:
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
        if world > 1:
            t = torch.tensor([e_ms], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_ms = float(t.item())
        e2e = {"value": world * m / (e_ms * 1e-3), "unit": "edges/s",
               "h2d_bytes_per_step": rp_h.numel() * 8 + ci_h.numel() * 4,
               "d2h_bytes_per_step": sum(x.numel() * x.element_size() for x in out_h),
               "ms_per_step": e_ms, "steps": K,
               "pipeline": "double-buffered: step i+1's H2D copy overlaps step i"}
        del dbuf

    # ---- sharded MIS-Deg2 of ONE graph across the N ranks (the exchange path,
    #      SURVEY §8(e)): per round, NCCL all-gather of the owned 1-byte status segments
    from paper_conf_ipps_nayyaroddeengk17_b200 import sharded as S
    shards = S.make_shards(rp, ci, world, ranks=[rank])
    tr = S.DistTransport() if world > 1 else S.LocalTransport()
    sst = {}
    S.sym_mis_sharded(shards, "degk", 2, args.seed, tr, None, sst)  # warm-up
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 3
    s0.record(stream)
    for _ in range(reps):
        S.sym_mis_sharded(shards, "degk", 2, args.seed, tr, None, sst)
    s1.record(stream)
    torch.cuda.synchronize()
    sh_ms = s0.elapsed_time(s1) / reps
    if world > 1:
        t = torch.tensor([sh_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        sh_ms = float(t.item())
    sharded = {"problem": "MIS-Deg2 (no decomposition materialised; DEGk as a class predicate)",
               "ranks": world, "ms": sh_ms, "edges_per_s": m / (sh_ms * 1e-3), "rounds": sst.get("rounds"),
               "exchange": "all_gather_into_tensor of owned status segments + all_reduce of frontier counts per round",
               "scaling": "strong (one graph)"}
    del shards

    # ---- CPU oracle (rank 0, N = 1 only), bounded sample
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        import oracle as O
        O.build()
        rps, cis = cpu_sample(args.cpu_scale, args.ef)
        T = oracle_step(rps, cis, seed)
        cpu = {"value": (cis.size // 2) / T, "unit": "edges/s", "cores": 1, "kind": "oracle",
               "sample": f"R-MAT scale {args.cpu_scale} ef {args.ef} (m={cis.size // 2}), same step, "
                         f"single-threaded C oracle, {T:.1f} s"}

    if rank == 0:
        launches = sum(v["launches"] for v in prof.values()) / steps_p
        out = {
            "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"rmat{args.scale}-ef{args.ef}: DEG2{{MIS,COLOR}} + RAND4{{MM}}",
                       "n": n, "m": m, "arcs": nnz, "seed": seed, "graph_seed": 1,
                       "parallelism": "replicas" if world > 1 else "single",
                       "schedule": "sequential (one stream)" if args.sequential else
                       "2 streams: [DEG2 decomposition -> COLOR-Deg2] || [RAND4 decomposition -> MM-Rand4 -> MIS-Deg2]",
                       "l2": "inputs exceed L2 (col_idx %.2f GB > 126 MB)" % (nnz * 4 / 1e9),
                       "generate_s": round(gen_s, 2)},
            "breakdown_ms": brk,
            "breakdown_edges_per_s": {"mis_deg2_incl_decomp": m / ((brk["decompose_deg2"] + brk["mis_deg2"]) * 1e-3),
                                      "color_deg2_incl_decomp": m / ((brk["decompose_deg2"] + brk["color_deg2"]) * 1e-3),
                                      "mm_rand4_incl_decomp": m / ((brk["decompose_rand4"] + brk["mm_rand4"]) * 1e-3)},
            "kernels": per_step, "dominant_kernel": dominant_overall,
            "roofline": roof, "rooflines": rooflines, "cpu_baseline": cpu, "e2e": e2e, "sharded_mis": sharded,
            "gpu_launches": int(round(launches)),
            "clocks": clk.summary(),
            "stats": {"mis": st_mis, "color": st_col, "mm": st_mm},
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
