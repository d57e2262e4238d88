"""Partitioned multi-GPU mode on one GPU: the per-rank
configurations bench.py builds for a 2- and a 4-GPU job (weak partitions:
rank g owns key range [g*N, (g+1)*N) of the job, runs the full per-GPU
workload with seed mix64(seed ^ g)) are each run through the C ABI with a
DIGEST log and checked by the oracle on their own log, exactly as each rank
of `bench.py --gpus N` would be; ranks never share a transaction or an
account."""
import os
import sys
import types

import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from tests.test_gpu_kv import as_state, ocfg_of  # noqa: E402
from tests.test_gpu_parity import check  # noqa: E402


def rank_cfg(name, world, rank, n_tx):
    _, lcfg, part = bench.make_cfg(types.SimpleNamespace(config=name, n_tx=n_tx), world, rank)
    return lcfg.with_(log_mode=csmv.LOG_DIGEST, client_warps=bench.tuned_client_warps(name, 148)), part


@pytest.mark.parametrize("world", [2, 4])
def test_bank_ranks_each_pass_their_oracle(world):
    seeds, los = set(), set()
    for r in range(world):
        cfg, part = rank_cfg("C2", world, r, 1 << 20)
        assert cfg.n_items == 1 << 20 and part.item_lo == r << 20
        seeds.add(cfg.seed)
        los.add(part.item_lo)
        rep, stats, *_ = check(cfg)
        assert stats["committed"] == cfg.n_tx
    assert len(seeds) == world and len(los) == world


def test_kv_ranks_each_pass_their_oracle():
    for r in range(2):
        cfg, part = rank_cfg("C4", 2, r, 1 << 18)
        w = cfg.workload
        with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
            st.load(w.kv_keys)
            stats = st.run(w, cfg.n_tx, cfg.seed)
            log = st.log(cfg.n_tx)
            fin = st.dump()
        oc = ocfg_of(cfg)
        rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log,
                              final=as_state(fin, cfg.n_items, w.kv_ways),
                              claims=dict(committed_update=stats["committed_update"],
                                          committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                          total_aborts=stats["total_aborts"]))
        assert rep["ok"], (r, rep)
