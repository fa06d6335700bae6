"""Multi-GPU sharded MIS, MM and COLOR (include/sym.h
`sym_comm_*`, `sym_{mis,mm,color}_sharded`).

CPU (no GPU needed):
  * the shard plan covers [0, n) with disjoint 32-aligned blocks;
  * the library's per-rank protocol (tests/_sharded_cpu.py: the same phase sequences
    and round rules, and after every round ONLY the boundary vertices' state changes
    exchanged as padded delta lists) reproduces the oracle bit for bit for every flow,
    in one process with 1..4 ranks and over torch.distributed/gloo with 2 processes.
GPU (-m gpu): the library itself -- 1..8 ranks in one process (a host thread, CUDA
stream and local communicator per rank) and a 1-rank NCCL communicator -- equals the
oracle and the single-GPU calls bit for bit, with the exchanged bytes reported.
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import graphgen as G
import oracle as O
from paper_conf_ipps_nayyaroddeengk17_b200 import sharded as S

import _sharded_cpu as D

GRAPHS = {
    "rmat10": lambda: G.rmat(10, 8, 3),
    "road32": lambda: G.grid(32, 32, 0.6, 2),
    "mix": lambda: G.disjoint_union(G.star(300), G.cycle(61), G.path(40), G.complete(12), G.empty(9)),
}
ORACLE = {"mis": O.mis, "mm": O.mm, "color": O.color}
FLOWS = [("mis", "none", 0), ("mis", "degk", 2), ("mis", "rand", 4), ("mm", "none", 0), ("mm", "rand", 4),
         ("color", "none", 0), ("color", "degk", 2), ("color", "rand", 4)]


@pytest.mark.parametrize("n,ranks", [(1, 1), (31, 2), (100, 3), (1000, 8), (5, 8)])
def test_shard_plan(n, ranks):
    covered = []
    for r in range(ranks):
        v0, v1 = S.shard_range(n, ranks, r)
        assert (v0 % 32 == 0 or v0 == v1 == n) and v0 <= v1
        covered += list(range(v0, v1))
    assert covered == list(range(n))


@pytest.mark.parametrize("problem,kind,p", FLOWS)
@pytest.mark.parametrize("nranks", [1, 2, 3, 4])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_protocol_local_cpu(name, nranks, problem, kind, p):
    rp, ci = (x.numpy() for x in GRAPHS[name]())
    got, ranks = D.run_local(rp, ci, nranks, problem, kind, p, 42)
    want = ORACLE[problem](rp, ci, kind, p, 42)
    assert np.array_equal(got.astype(np.int64), want.astype(np.int64))
    if nranks == 1:
        assert not ranks[0].bnd  # one rank has no boundary: nothing but class bits moves


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, problem, kind, k, outdir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rp, ci = (x.numpy() for x in G.rmat(11, 8, 5))
        n = rp.size - 1
        r = D.Rank(rp, ci, world, rank, kind, k, 7)
        (mine,) = D.run_ranks([r], D.GlooTransport(world), D.FLOWS[problem])
        block = S.shard_block(n, world)
        pad = torch.zeros(block, dtype=torch.int64)
        pad[: mine.size] = torch.as_tensor(mine.astype(np.int64))
        full = torch.zeros(world * block, dtype=torch.int64)
        dist.all_gather_into_tensor(full, pad)
        if rank == 0:
            want = ORACLE[problem](rp, ci, kind, k, 7).astype(np.int64)
            ok = np.array_equal(full[:n].numpy(), want)
            with open(os.path.join(outdir, "result"), "w") as f:
                f.write(f"{ok} boundary={len(r.bnd)} sent={r.exchanged}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("problem,kind,k", FLOWS)
def test_gloo_world_size_2(problem, kind, k):
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(2, _free_port(), problem, kind, k, d), nprocs=2, join=True)
        res = open(os.path.join(d, "result")).read()
    assert res.startswith("True"), res


# ------------------------------------------------------------------ GPU (the library)
GPU_GRAPHS = {"rmat14": lambda: G.rmat(14, 8, 1), "road128": lambda: G.grid(128, 128, 0.6, 1),
              "hubs": lambda: G.disjoint_union(G.star(9000), G.complete(1100), G.cycle(301), G.empty(50))}


@pytest.mark.gpu
@pytest.mark.parametrize("problem,kind,p", FLOWS + [("mm", "rand", 64), ("color", "rand", 64)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 8])
@pytest.mark.parametrize("name", list(GPU_GRAPHS))
def test_gpu_sharded_local(name, nranks, problem, kind, p):
    g = GPU_GRAPHS[name]()
    rp, ci = g[0].cuda(), g[1].cuda()
    outs, stats = S.run_local(S.make_shards(rp, ci, nranks), problem, kind, p, 42, stats=True)
    got = torch.cat(outs).cpu().numpy().astype(np.int64)
    assert np.array_equal(got, ORACLE[problem](*g, kind, p, 42).astype(np.int64))
    for st in stats:
        if nranks == 1:
            assert st["boundary"] == 0 and st["sent_bytes"] == 0
        assert st["exchanges"] >= 1


@pytest.mark.gpu
def test_gpu_sharded_scale20_equals_single_gpu():
    """R-MAT scale 20 (16 M arcs): 2 and 5 ranks in one process == the single-GPU calls,
    and MIS-Deg2's boundary-only exchange stays within n/4 bytes per exchange on average
    (the C3 flow; SURVEY §8(e) budgets n/4 B per round for the dense 2-bit status)."""
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    rp, ci = G.rmat(20, 16, 1, device="cuda")
    n = rp.numel() - 1
    for problem, fn, kind, p in (("mis", sb.sym_mis, "degk", 2), ("mis", sb.sym_mis, "rand", 4),
                                 ("mm", sb.sym_mm, "none", 0), ("mm", sb.sym_mm, "rand", 8),
                                 ("color", sb.sym_color, "degk", 2), ("color", sb.sym_color, "rand", 4)):
        ref = fn(rp, ci, kind, p, 42)
        for nranks in (2, 5):
            outs, stats = S.run_local(S.make_shards(rp, ci, nranks), problem, kind, p, 42, stats=True)
            assert torch.equal(torch.cat(outs).to(ref.dtype), ref), (problem, kind, nranks)
            if problem == "mis" and kind == "degk":
                sent = sum(s["sent_bytes"] for s in stats)
                assert sent / stats[0]["exchanges"] <= n / 4, (kind, nranks, stats)


@pytest.mark.gpu
def test_gpu_nccl_single_rank():
    """The NCCL communicator (one rank: ncclCommInitRank + ncclAllGather on the stream)."""
    import torch.distributed as dist
    g = G.rmat(14, 8, 1)
    rp, ci = g[0].cuda(), g[1].cuda()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{_free_port()}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        comm = S.Comm.nccl()
        (sh,) = S.make_shards(rp, ci, 1)
        for problem, fn, kind, p in (("mis", S.sym_mis_sharded, "degk", 2), ("mm", S.sym_mm_sharded, "rand", 4),
                                     ("color", S.sym_color_sharded, "rand", 4)):
            got = fn(sh, comm, kind, p, 42).cpu().numpy().astype(np.int64)
            assert np.array_equal(got, ORACLE[problem](*g, kind, p, 42).astype(np.int64)), problem
        comm.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_gpu_sharded_bad_plan_is_rejected():
    from paper_conf_ipps_nayyaroddeengk17_b200 import SymError
    rp, ci = (x.cuda() for x in G.rmat(10, 8, 1))
    sh = S.make_shards(rp, ci, 2)[0]
    (comm,) = S.Comm.local_group(1)
    with pytest.raises(SymError):  # a 2-rank shard handed to a 1-rank communicator
        S.sym_mis_sharded(sh, comm)
    comm.close()
