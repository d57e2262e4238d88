"""Partitioned multi-GPU mode.

CSMV serialises every update through one CTS sequence and one GTS (P:65,
P:101), so a single store does not shard.  For G GPUs the framework
runs G *independent key-range-partitioned instances*: rank g owns its own
key range of the job's accounts as its own store (local ids 0..N_g-1), runs
its own server and GTS, generates its transactions with seed_g = mix64(seed ^
g) inside its partition, and never exchanges data with another rank.  The
only collective is the end-of-run statistics reduction (SUM of counters, MAX
of elapsed time) -- every figure is labelled "partitioned, no cross-GPU
transactions".

Two ways to split a job (``mode``):
  * "weak" (bench.py's): every rank runs the full per-GPU workload -- n_items
    accounts and n_tx transactions -- on key range [g*n_items, (g+1)*n_items)
    of a G*n_items-account job; per-GPU work is fixed as G grows;
  * "strong": a fixed job of n_items accounts and n_tx transactions is split
    into G near-equal key and transaction ranges.
"""
from __future__ import annotations

from dataclasses import dataclass, replace

M64 = (1 << 64) - 1

SUM_KEYS = ("committed_update", "committed_ro", "batches", "rounds", "total_aborts", "committed")
MAX_KEYS = ("elapsed_ns",)


def mix64(x: int) -> int:
    """splitmix64 output function (docs/GENERATOR.md section 1)."""
    z = (x + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


@dataclass(frozen=True)
class Part:
    rank: int
    world: int
    item_lo: int        # first global account owned
    n_items: int        # accounts in this partition
    tx_lo: int          # first global transaction index of this rank
    n_tx: int
    seed: int


def partition(n_items: int, n_tx: int, seed: int, rank: int, world: int, mode: str = "strong") -> Part:
    if not 0 <= rank < world:
        raise ValueError("rank out of range")
    s = seed if world == 1 else mix64(seed ^ rank)
    if mode == "weak":
        return Part(rank, world, n_items * rank, n_items, n_tx * rank, n_tx, s)
    if mode != "strong":
        raise ValueError(f"unknown partition mode {mode!r}")
    lo = n_items * rank // world
    hi = n_items * (rank + 1) // world
    t_lo = n_tx * rank // world
    t_hi = n_tx * (rank + 1) // world
    return Part(rank, world, lo, hi - lo, t_lo, t_hi - t_lo, s)


def local_config(cfg, part: Part):
    """The workload preset restricted to one partition."""
    return replace(cfg, n_items=part.n_items, n_tx=part.n_tx, seed=part.seed)


def stats_vector(stats: dict) -> list:
    return [float(stats[k]) for k in SUM_KEYS] + [float(stats[k]) for k in MAX_KEYS]


def reduce_stats(stats: dict, device=None) -> dict:
    """All-reduce per-rank stats over torch.distributed (SUM counters, MAX
    elapsed).  Works with the nccl (GPU) and gloo (CPU tests) backends."""
    import torch
    import torch.distributed as dist

    v = stats_vector(stats)
    ns, nm = len(SUM_KEYS), len(MAX_KEYS)
    t_sum = torch.tensor(v[:ns], dtype=torch.float64, device=device)
    t_max = torch.tensor(v[ns:], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t_sum, op=dist.ReduceOp.SUM)
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
    out = {k: int(x) for k, x in zip(SUM_KEYS, t_sum.tolist())}
    out.update({k: int(x) for k, x in zip(MAX_KEYS, t_max.tolist())})
    att = out["committed"] + out["total_aborts"]
    out["abort_rate"] = out["total_aborts"] / att if att else 0.0
    out["tx_per_s"] = out["committed"] / (out["elapsed_ns"] * 1e-9) if out["elapsed_ns"] else 0.0
    return out
