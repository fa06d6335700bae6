"""bench.py --gpus N (N > 1): the bench step sharded over the N ranks (one per GPU).

Every rank generates the same R-MAT graph, keeps only its vertex block (SURVEY
§8(e): ownership = contiguous 32-aligned blocks of the permuted R-MAT ids) and runs
the step through the library's sharded calls with one NCCL communicator:
    MIS-Deg2 -> COLOR-Deg2 -> MM-Rand4      (sym_{mis,color,mm}_sharded)
One graph for all N ranks: strong scaling.  The timed region is bracketed by a
barrier + synchronize on both sides, device-timed with CUDA events, max over ranks.
"""
from __future__ import annotations

import json
import time


def bench(args, rank, world, dev, metric, ClockSampler):
    import torch
    import torch.distributed as dist

    import graphgen
    from . import sharded as S

    t0 = time.time()
    rp, ci = graphgen.rmat(args.scale, args.ef, seed=1, device=dev)
    n, nnz = rp.numel() - 1, ci.numel()
    m = nnz // 2
    (sh,) = S.make_shards(rp, ci, world, ranks=[rank])
    rp_h, ci_h = sh.row_ptr.cpu().pin_memory(), sh.col_idx.cpu().pin_memory()  # for the e2e leg
    del rp, ci
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    comm = S.Comm.nccl(device=dev)
    seed = args.seed
    stream = torch.cuda.current_stream(dev)
    stats = {}

    def step(shard=sh, keep=False):
        I, a = S.sym_mis_sharded(shard, comm, "degk", 2, seed, stats=True)
        C, b = S.sym_color_sharded(shard, comm, "degk", 2, seed, stats=True)
        M, c = S.sym_mm_sharded(shard, comm, "rand", 4, seed, stats=True)
        if keep:
            stats.update({"mis_deg2": a, "color_deg2": b, "mm_rand4": c})
        return I, C, M

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev.index) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([e0.elapsed_time(e1) / args.steps], device=dev, dtype=torch.float64)
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_step = float(ms.item())

    # per-problem times (events between the calls; max over ranks) and exchange stats
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    dist.barrier()
    evs[0].record(stream)
    S.sym_mis_sharded(sh, comm, "degk", 2, seed)
    evs[1].record(stream)
    S.sym_color_sharded(sh, comm, "degk", 2, seed)
    evs[2].record(stream)
    S.sym_mm_sharded(sh, comm, "rand", 4, seed)
    evs[3].record(stream)
    torch.cuda.synchronize()
    brk = torch.tensor([evs[i].elapsed_time(evs[i + 1]) for i in range(3)], device=dev, dtype=torch.float64)
    dist.all_reduce(brk, op=dist.ReduceOp.MAX)
    step(keep=True)

    # e2e: the owned rows copied host->device and the owned results back, every step
    e2e = None
    if not args.no_e2e:
        K = max(1, min(args.steps, 3))
        dist.barrier()
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(K):
            shd = S.Shard(sh.n_global, sh.nranks, sh.rank, rp_h.to(dev, non_blocking=True),
                          ci_h.to(dev, non_blocking=True))
            outs = step(shd)
            host = [o.to("cpu", non_blocking=True) for o in outs]
        f1.record(stream)
        torch.cuda.synchronize()
        e_ms = torch.tensor([f0.elapsed_time(f1) / K], device=dev, dtype=torch.float64)
        dist.all_reduce(e_ms, op=dist.ReduceOp.MAX)
        e2e = {"value": m / (float(e_ms.item()) * 1e-3), "unit": "edges/s",
               "h2d_bytes_per_step": rp_h.numel() * 8 + ci_h.numel() * 4,
               "d2h_bytes_per_step": sum(h.numel() * h.element_size() for h in host),
               "ms_per_step": float(e_ms.item()), "steps": K, "note": "per rank (rank 0's bytes)"}
    comm.close()
    if rank == 0:
        out = {
            "metric": metric, "value": m / (ms_step * 1e-3), "unit": "edges/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"rmat{args.scale}-ef{args.ef}: DEG2{{MIS,COLOR}} + RAND4{{MM}}, sharded",
                       "n": n, "m": m, "arcs": nnz, "seed": seed, "graph_seed": 1,
                       "parallelism": f"sharded over {world} ranks (32-aligned vertex blocks, NCCL delta exchange)",
                       "l2": "inputs exceed L2", "generate_s": round(gen_s, 2)},
            "breakdown_ms": {"mis_deg2": float(brk[0]), "color_deg2": float(brk[1]), "mm_rand4": float(brk[2])},
            "exchange": {k: dict(v, exchanged_bytes_per_exchange=(v["gathered_bytes"] / max(1, v["exchanges"])))
                         for k, v in stats.items()},
            "note": "sharded COLOR runs plain Jones-Plassmann levels with one exchange per level (DESIGN §9)",
            "e2e": e2e, "gpu_launches": None, "clocks": clk.summary(),
        }
        print(json.dumps(out), flush=True)
