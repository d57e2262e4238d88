"""Partitioned multi-GPU host logic on CPU with gloo,
world_size 2: partitions tile the accounts and transactions exactly once,
seeds differ per rank, and the statistics reduction is SUM / MAX."""
import os
import socket

import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_nunesc022_b200 import partition as P


def test_partition_tiles_everything():
    for world in (1, 2, 3, 8):
        parts = [P.partition(1_000_003, 10_000_019, 7, r, world) for r in range(world)]
        assert sum(p.n_items for p in parts) == 1_000_003
        assert sum(p.n_tx for p in parts) == 10_000_019
        for a, b in zip(parts, parts[1:]):
            assert a.item_lo + a.n_items == b.item_lo and a.tx_lo + a.n_tx == b.tx_lo
        seeds = {p.seed for p in parts}
        assert len(seeds) == world
    assert P.partition(10, 10, 7, 0, 1).seed == 7
    with pytest.raises(ValueError):
        P.partition(10, 10, 1, 2, 2)


def test_weak_partition_fixes_per_rank_work():
    for world in (1, 2, 4, 8):
        parts = [P.partition(1 << 20, 1 << 24, 1, r, world, mode="weak") for r in range(world)]
        assert all(p.n_items == 1 << 20 and p.n_tx == 1 << 24 for p in parts)
        assert [p.item_lo for p in parts] == [r << 20 for r in range(world)]   # disjoint key ranges
        assert len({p.seed for p in parts}) == world
    assert P.partition(10, 10, 7, 0, 1, mode="weak").seed == 7
    with pytest.raises(ValueError):
        P.partition(10, 10, 1, 0, 1, mode="diagonal")


def test_mix64_vector():
    assert P.mix64(0) == 0xE220A8397B1DCDAF


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    st = {"committed_update": 10 + rank, "committed_ro": 20 + rank, "batches": 3, "rounds": 4,
          "total_aborts": rank, "committed": 30 + 2 * rank, "elapsed_ns": 1000 * (rank + 1)}
    out = P.reduce_stats(st)
    q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


def test_reduce_stats_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in (0, 1):
        o = res[r]
        assert o["committed_update"] == 21 and o["committed_ro"] == 41 and o["committed"] == 62
        assert o["elapsed_ns"] == 2000 and o["total_aborts"] == 1
        assert abs(o["tx_per_s"] - 62 / 2e-6) < 1e-3


def _bench_rank(rank, world, port, q):
    """What each rank of `bench.py --gpus N` computes before touching a GPU:
    its weak partition of the C2 job, and the statistics reduction."""
    import types

    import torch
    import torch.distributed as dist

    import bench
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cfg, lcfg, part = bench.make_cfg(types.SimpleNamespace(config="C2", n_tx=0), world, rank)
    mine = torch.tensor([part.item_lo, part.n_items, lcfg.n_tx, lcfg.seed & 0x7FFFFFFF], dtype=torch.int64)
    allp = [torch.zeros_like(mine) for _ in range(world)]
    dist.all_gather(allp, mine)
    q.put((rank, [t.tolist() for t in allp], lcfg.workload.client_group))
    dist.barrier()
    dist.destroy_process_group()


def test_bench_ranks_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_rank, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict((r, (a, g)) for r, a, g in (q.get(timeout=180) for _ in procs))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    parts, group = res[0]
    assert parts == res[1][0] and group == 4
    (lo0, n0, tx0, s0), (lo1, n1, tx1, s1) = parts
    assert (lo0, lo1) == (0, 1 << 20) and n0 == n1 == 1 << 20      # disjoint key ranges, full per-GPU size
    assert tx0 == tx1 == 1 << 24 and s0 != s1                       # weak scaling, per-rank seeds


def test_bench_rejects_world_size_mismatch():
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2"], env=env,
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 2 and "WORLD_SIZE" in r.stderr
