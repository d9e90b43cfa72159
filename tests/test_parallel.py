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
