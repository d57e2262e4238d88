"""The five configurations of BASELINE.json as concrete workloads
(readings Q10-Q13, Q26-Q29 listed in DESIGN.md).

Each preset returns (n_items, n_versions, Workload, n_tx, seed, init).
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass, replace

import numpy as np

from .csmv import (DIST_UNIFORM, DIST_ZIPF, KIND_BANK, KIND_KV, LOG_DIGEST, LOG_FULL,
                   SERVER_CLUSTER, SERVER_CTA, Workload)

BANK_INIT = 1000


@dataclass
class Config:
    name: str
    n_items: int
    n_versions: int
    workload: Workload
    n_tx: int
    seed: int
    kv_slots: int = 0

    def init_values(self) -> np.ndarray:
        return np.full(self.n_items, BANK_INIT, dtype=np.int32)

    def with_(self, **kw) -> "Config":
        wk = {k: v for k, v in kw.items() if hasattr(self.workload, k)}
        ck = {k: v for k, v in kw.items() if not hasattr(self.workload, k)}
        return replace(self, workload=replace(self.workload, **wk), **ck)


def c1(**kw) -> Config:
    """bank: 1,024 accounts, K=4, 8 client warps, 10k transfers + 10% total-sum
    ROTs (1,111 of 11,111, slot i read-only iff i % 10 == 9, Q13), seed 1."""
    w = Workload(kind=KIND_BANK, dist=DIST_UNIFORM, ro_period=10, ro_reads=0,
                 client_warps=8, log_mode=LOG_FULL)
    return Config("C1", 1024, 4, w, 11_111, 1).with_(**kw)


def c2(**kw) -> Config:
    """bank: 1M accounts, K=4, full-GPU client grid, 50% update, uniform,
    read-only = 64-read contiguous scan (Q10)."""
    w = Workload(kind=KIND_BANK, dist=DIST_UNIFORM, p_update_ppm=500_000, ro_reads=64,
                 client_warps=0, log_mode=LOG_DIGEST)
    return Config("C2", 1 << 20, 4, w, 1 << 24, 1).with_(**kw)


def c3(**kw) -> Config:
    """bank: 4,096 accounts (the whole store is the hot set, Q26), 90%
    read-only 64-read scans from a uniform start, zipf 0.99 update endpoints."""
    w = Workload(kind=KIND_BANK, dist=DIST_ZIPF, zipf_theta_milli=990, p_update_ppm=100_000,
                 ro_reads=64, client_warps=0, log_mode=LOG_DIGEST)
    return Config("C3", 4096, 4, w, 1 << 22, 1).with_(**kw)


def c4(**kw) -> Config:
    """MemcachedGPU-style KV: 4M slots / 4M keys, 16 ways (Q16, Q27), 99% GET,
    zipf 0.99 keys, 16 B keys, 32 B values, K=4.  n_items = slots."""
    w = Workload(kind=KIND_KV, dist=DIST_ZIPF, zipf_theta_milli=990, p_update_ppm=10_000,
                 kv_ways=16, kv_keys=1 << 22, client_warps=0, log_mode=LOG_DIGEST)
    cfg = Config("C4", 1 << 22, 4, w, 1 << 24, 1, kv_slots=1 << 22).with_(**kw)
    if "n_items" in kw and "kv_keys" not in kw:   # shrunk configs: key space = slots
        cfg = cfg.with_(kv_keys=cfg.n_items)
    return cfg


C5_UPDATE = (100_000, 300_000, 500_000, 700_000, 900_000)          # Q28
C5_ITEMS = (1 << 10, 1 << 14, 1 << 18, 1 << 22, 1 << 24)
C5_VERSIONS = (2, 4, 8)
C5_SERVERS = (SERVER_CTA, SERVER_CLUSTER)


def c5_points(n_tx: int = 1 << 22, servers=C5_SERVERS):
    """sweep: update rate 10-90% x contention (1K-16M items) x K = 2/4/8 x
    single-SM vs cluster server = 150 points (Q28)."""
    for pu, n, k, srv in itertools.product(C5_UPDATE, C5_ITEMS, C5_VERSIONS, servers):
        w = Workload(kind=KIND_BANK, dist=DIST_UNIFORM, p_update_ppm=pu, ro_reads=64,
                     server=srv, log_mode=LOG_DIGEST)
        yield Config(f"C5-u{pu // 10_000}-n{n}-k{k}-s{srv}", n, k, w, n_tx, 1)


PRESETS = {"C1": c1, "C2": c2, "C3": c3, "C4": c4}
