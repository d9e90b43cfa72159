"""N>1 host logic on CPU (-m "not gpu"): world_size-2 gloo process groups exercise
the source sharding, the rank-0 build + save/load sharing of the hierarchy, and the
MAX all-reduce used for the diameter and for max-over-ranks timing."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_dellinggnw11_b200.parallel import shard


def test_shard_covers_exactly():
    for count in (0, 1, 7, 64, 8192, 1_000_003):
        for world in (1, 2, 3, 8):
            parts = [shard(count, world, r) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == count
            for (a, b), (c, d) in zip(parts, parts[1:]):
                assert b == c
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard(10, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, tmpdir, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import phastgen
        import paper_conf_ipps_dellinggnw11_b200 as P
        from paper_conf_ipps_dellinggnw11_b200.parallel import allreduce_max_u32, share_hierarchy, shard
        g = phastgen.road(20_000, seed=5)
        h = share_hierarchy(lambda: P.Phast.from_graph(g, host_only=True),
                            lambda p: P.Phast.load(p, host_only=True),
                            os.path.join(tmpdir, "h.phast"), rank, dist.barrier)
        ex = h.export()
        digest = int(np.bitwise_xor.reduce(ex["dn_tail"].astype(np.uint64) * 2654435761 % (1 << 32)))
        lo, hi = shard(1000, world, rank)
        m = allreduce_max_u32(0xFFFFFFF0 - rank)          # uint32 values survive the int64 carrier
        t = allreduce_max_u32(1000 + 7 * rank)
        q.put((rank, digest, h.levels, lo, hi, m, t))
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_sharing_and_allreduce(tmp_path):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, str(tmp_path), q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    res = sorted(q.get(timeout=10) for _ in range(world))
    assert res[0][1] == res[1][1] and res[0][2] == res[1][2]      # identical hierarchy on both ranks
    assert (res[0][3], res[0][4], res[1][3], res[1][4]) == (0, 500, 500, 1000)
    assert all(r[5] == 0xFFFFFFF0 for r in res)
    assert all(r[6] == 1007 for r in res)
    assert not os.path.exists(tmp_path / "h.phast")               # rank 0 cleaned up


def _centrality_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import phastgen
        from paper_conf_ipps_dellinggnw11_b200.parallel import combine_centrality, shard
        g = phastgen.grid(9, 7, 1, 5, seed=12)
        lo, hi = shard(g.n, world, rank)
        src = np.arange(lo, hi, dtype=np.uint32)
        cb = torch.from_numpy(oracle.betweenness(g, src))
        r = torch.from_numpy(oracle.reach(g, src).view(np.int32).copy())
        combine_centrality(cb, reach=False)
        combine_centrality(r, reach=True)
        q.put((rank, cb.numpy(), r.numpy().view(np.uint32)))
    finally:
        dist.destroy_process_group()


def test_two_rank_centrality_shards_combine():
    """Betweenness / reach over disjoint source shards (NEXT-3): SUM and MAX over the
    ranks give the all-sources values (the combine bench_betweenness.py uses)."""
    import oracle
    import phastgen
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_centrality_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    res = sorted((q.get(timeout=10) for _ in range(world)), key=lambda x: x[0])
    g = phastgen.grid(9, 7, 1, 5, seed=12)
    allv = np.arange(g.n)
    for _, cb, r in res:
        np.testing.assert_allclose(cb, oracle.betweenness(g, allv), rtol=1e-12)
        assert np.array_equal(r, oracle.reach(g, allv))


def _bench_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import bench
        import phastgen
        cfg = phastgen.CONFIGS["C4"]
        n = 24_000_000
        # strong scaling (BASELINE configs[3]): 8192 sources sharded; 8000 = ragged last batch
        out = {}
        for total in (8192, 8000):
            warm, timed, trees = bench.rank_batches(n, cfg, 64, world, rank, 5, 3, total)
            got = [None] * world
            dist.all_gather_object(got, (rank, [b.tolist() for b in timed], trees))
            out[total] = got
        # weak scaling: `steps` batches of this rank's own sources
        warm, timed, trees = bench.rank_batches(n, cfg, 64, world, rank, 5, 3, 0)
        weak = [None] * world
        dist.all_gather_object(weak, (rank, [b.tolist() for b in timed], [b.tolist() for b in warm], trees))
        # max-over-ranks timing (the bench's rule for every multi-GPU number)
        t = torch.tensor([10.0 + rank], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        q.put((rank, out, weak, float(t.item())))
    finally:
        dist.destroy_process_group()


def test_two_rank_bench_source_plan():
    """bench.py's rank logic on a world-2 gloo group: in strong-scaling mode the two
    ranks' batches cover the one seeded list of T sources exactly once (a ragged last
    batch is padded with duplicates that are not counted); in weak mode each rank
    sweeps `steps` batches of k sources of its own; timings combine by MAX."""
    import phastgen
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    # drain the queue before joining: a worker cannot exit while its large result
    # is still in the pipe
    res = sorted((q.get(timeout=300) for _ in range(world)), key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cfg = phastgen.CONFIGS["C4"]
    for total in (8192, 8000):
        full = phastgen.sources(24_000_000, total, seed=cfg["src_seed"] * 7919 + 1).tolist()
        per_rank = sorted(res[0][1][total])
        assert per_rank == sorted(res[1][1][total])           # all_gather agrees on both ranks
        flat, counted = [], 0
        for r, batches, trees in per_rank:
            assert all(len(b) == 64 for b in batches)
            real = sum((b for b in batches), [])[:trees]
            flat += real
            counted += trees
        assert flat == full and counted == total
    weak = res[0][2]
    assert [w[3] for w in weak] == [320, 320]
    a, b = weak[0][1], weak[1][1]
    assert len(a) == len(b) == 5 and all(len(x) == 64 for x in a + b)
    assert a != b and weak[0][2] != a                          # own sources per rank; warm-up differs
    assert all(r[3] == 11.0 for r in res)


def test_bench_relaunches_under_torchrun(monkeypatch):
    """`python bench.py --gpus 8` outside torchrun re-executes itself under
    torch.distributed.run with 8 ranks, 127.0.0.1 rendezvous, NCCL init logging."""
    import sys
    import bench
    seen = {}

    def fake_call(cmd, env):
        seen["cmd"], seen["env"] = cmd, env
        return 0
    monkeypatch.setattr(bench.subprocess, "call", fake_call)
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "8", "--steps", "5"])
    assert bench.main() == 0
    cmd = seen["cmd"]
    assert cmd[1:4] == ["-m", "torch.distributed.run", "--nnodes=1"]
    assert "--nproc-per-node=8" in cmd and "127.0.0.1" in cmd
    assert cmd[-4:] == ["--gpus", "8", "--steps", "5"] and cmd[-5].endswith("bench.py")
    assert seen["env"]["NCCL_DEBUG"] == "INFO"
