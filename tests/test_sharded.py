"""Multi-GPU sharded MIS, MM and COLOR: host logic on CPU, kernels on GPU.

CPU (no GPU needed):
  * the shard plan covers [0, n) with disjoint 32-aligned blocks;
  * the orchestration (status / class-bitmap all-gathers, count all-reduce, the
    MIS-Deg2 phase sequence, termination) with the CPU test double, in one process
    (1..4 shards) and over torch.distributed/gloo with world size 2, equals the oracle.
GPU (-m gpu): the sym_shard_* kernels with 1..4 shards in one process (in-process
exchange) equal the oracle and the single-GPU sym_mis, bit for bit.
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

from _sharded_cpu import CpuBackend

GRAPHS = {
    "rmat10": lambda: G.rmat(10, 8, 3),
    "road32": lambda: G.grid(32, 32, 0.6, 2),
    "mix": lambda: G.disjoint_union(G.star(300), G.cycle(61), G.path(40), G.complete(12), G.empty(9)),
}


@pytest.mark.parametrize("n,ranks", [(1, 1), (31, 2), (100, 3), (1000, 8), (5, 8)])
def test_shard_plan(n, ranks):
    covered = []
    for r in range(ranks):
        v0, v1 = S.shard_range(n, ranks, r)
        assert (v0 % 32 == 0 or v0 == v1 == n) and v0 <= v1
        covered += list(range(v0, v1))
    assert covered == list(range(n))


@pytest.mark.parametrize("kind,k", [("none", 0), ("degk", 2)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 4])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_orchestration_local_cpu(name, nranks, kind, k):
    rp, ci = GRAPHS[name]()
    n = rp.numel() - 1
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_mis_sharded(shards, kind, k, 42, S.LocalTransport(), CpuBackend(n, 42))
    got = torch.cat(out).numpy()
    assert np.array_equal(got, O.mis(rp, ci, kind, k, 42))


@pytest.mark.parametrize("kind,k", [("none", 0), ("degk", 2), ("rand", 4)])
@pytest.mark.parametrize("nranks", [1, 2, 3])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_color_orchestration_local_cpu(name, nranks, kind, k):
    rp, ci = GRAPHS[name]()
    n = rp.numel() - 1
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_color_sharded(shards, kind, k, 42, S.LocalTransport(), CpuBackend(n, 42))
    got = torch.cat(out).numpy()
    assert np.array_equal(got, O.color(rp, ci, kind, k, 42))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("kind,p", [("none", 0), ("rand", 4)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 4])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_mm_orchestration_local_cpu(name, nranks, kind, p):
    rp, ci = GRAPHS[name]()
    n = rp.numel() - 1
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_mm_sharded(shards, kind, p, 42, S.LocalTransport(), CpuBackend(n, 42))
    got = torch.cat(out).numpy()
    assert np.array_equal(got, O.mm(rp, ci, kind, p, 42))


def _worker(rank, world, port, kind, k, outdir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rp, ci = G.rmat(11, 8, 5)
        n = rp.numel() - 1
        (sh,) = S.make_shards(rp, ci, world, ranks=[rank])
        stats = {}
        mm = kind in ("mm-none", "mm-rand")
        col = kind.startswith("col-")
        if col:
            (mine,) = S.sym_color_sharded([sh], kind[4:], k, 7, S.DistTransport(), CpuBackend(n, 7), stats)
        elif mm:
            (mine,) = S.sym_mm_sharded([sh], kind[3:], k, 7, S.DistTransport(), CpuBackend(n, 7), stats)
        else:
            (mine,) = S.sym_mis_sharded([sh], kind, k, 7, S.DistTransport(), CpuBackend(n, 7), stats)
        block = S.shard_block(n, world)
        pad = torch.zeros(block, dtype=mine.dtype)
        pad[: mine.numel()] = mine
        full = torch.zeros(world * block, dtype=mine.dtype)
        dist.all_gather_into_tensor(full, pad)
        if rank == 0:
            want = (O.color(rp, ci, kind[4:], k, 7) if col else
                    O.mm(rp, ci, kind[3:], k, 7) if mm else O.mis(rp, ci, kind, k, 7))
            ok = np.array_equal(full[:n].numpy(), want)
            with open(os.path.join(outdir, "result"), "w") as f:
                f.write(f"{ok} {stats['rounds']}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind,k", [("none", 0), ("degk", 2), ("mm-none", 0), ("mm-rand", 4),
                                    ("col-none", 0), ("col-degk", 2), ("col-rand", 4)])
def test_gloo_world_size_2(kind, k):
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(2, _free_port(), kind, k, d), nprocs=2, join=True)
        res = open(os.path.join(d, "result")).read()
    assert res.startswith("True"), res


# ------------------------------------------------------------------ GPU
@pytest.mark.gpu
@pytest.mark.parametrize("kind,k", [("none", 0), ("degk", 2)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("name", ["rmat14", "road128", "hubs"])
def test_gpu_sharded_mis(name, nranks, kind, k):
    g = {"rmat14": lambda: G.rmat(14, 8, 1), "road128": lambda: G.grid(128, 128, 0.6, 1),
         "hubs": lambda: G.disjoint_union(G.star(9000), G.complete(60), G.cycle(301), G.empty(50))}[name]()
    rp, ci = g[0].cuda(), g[1].cuda()
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_mis_sharded(shards, kind, k, 42, S.LocalTransport(), S.GpuBackend())
    got = torch.cat(out).cpu().numpy()
    assert np.array_equal(got, O.mis(*g, kind, k, 42))


@pytest.mark.gpu
def test_gpu_sharded_scale20_equals_single_gpu():
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    rp, ci = G.rmat(20, 16, 1, device="cuda")
    ref = sb.sym_mis(rp, ci, "degk", 2, 42)
    for nranks in (2, 5):
        out = S.sym_mis_sharded(S.make_shards(rp, ci, nranks), "degk", 2, 42)
        assert torch.equal(torch.cat(out), ref)


@pytest.mark.gpu
@pytest.mark.parametrize("kind,p", [("none", 0), ("rand", 4), ("rand", 64)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("name", ["rmat14", "road128", "hubs"])
def test_gpu_sharded_mm(name, nranks, kind, p):
    g = {"rmat14": lambda: G.rmat(14, 8, 1), "road128": lambda: G.grid(128, 128, 0.6, 1),
         "hubs": lambda: G.disjoint_union(G.star(9000), G.complete(60), G.cycle(301), G.empty(50))}[name]()
    rp, ci = g[0].cuda(), g[1].cuda()
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_mm_sharded(shards, kind, p, 42, S.LocalTransport(), S.GpuBackend())
    got = torch.cat(out).cpu().numpy()
    assert np.array_equal(got, O.mm(*g, kind, p, 42))


@pytest.mark.gpu
def test_gpu_sharded_mm_scale20_equals_single_gpu():
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    rp, ci = G.rmat(20, 16, 1, device="cuda")
    for kind, p in (("none", 0), ("rand", 8)):
        ref = sb.sym_mm(rp, ci, kind, p, 42)
        for nranks in (2, 5):
            out = S.sym_mm_sharded(S.make_shards(rp, ci, nranks), kind, p, 42)
            assert torch.equal(torch.cat(out), ref), (kind, nranks)


@pytest.mark.gpu
@pytest.mark.parametrize("kind,k", [("none", 0), ("degk", 2), ("rand", 4), ("rand", 64)])
@pytest.mark.parametrize("nranks", [1, 2, 3, 8])
@pytest.mark.parametrize("name", ["rmat14", "road128", "hubs"])
def test_gpu_sharded_color(name, nranks, kind, k):
    g = {"rmat14": lambda: G.rmat(14, 8, 1), "road128": lambda: G.grid(128, 128, 0.6, 1),
         "hubs": lambda: G.disjoint_union(G.star(9000), G.complete(1100), G.cycle(301), G.empty(50))}[name]()
    rp, ci = g[0].cuda(), g[1].cuda()
    shards = S.make_shards(rp, ci, nranks)
    out = S.sym_color_sharded(shards, kind, k, 42, S.LocalTransport(), S.GpuBackend())
    got = torch.cat(out).cpu().numpy()
    assert np.array_equal(got, O.color(*g, kind, k, 42))


@pytest.mark.gpu
def test_gpu_sharded_color_scale18_equals_single_gpu():
    import paper_conf_ipps_nayyaroddeengk17_b200 as sb
    rp, ci = G.rmat(18, 16, 1, device="cuda")
    for kind, k in (("degk", 2), ("rand", 4)):
        ref = sb.sym_color(rp, ci, kind, k, 42)
        for nranks in (2, 5):
            out = S.sym_color_sharded(S.make_shards(rp, ci, nranks), kind, k, 42)
            assert torch.equal(torch.cat(out), ref), (kind, nranks)
