"""GPU parity at BASELINE.json's full sizes, in the launch configuration
bench.py times (its tuned per-config launch, the full client grid): every
committed transaction's snapshot, CTS, attempts and read/write digest checked
by the oracle's replay, the final store against the
oracle's, and the claimed counters (C2: 2^24 transactions over 1M accounts;
C3: 2^22 over 4,096; C4: 2^24 over the 4M-slot cache, preload included)."""
import os
import sys
import types

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
torch = pytest.importorskip("torch")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from tests.test_gpu_kv import as_state, ocfg_of  # noqa: E402
from tests.test_gpu_parity import oracle_cfg  # noqa: E402


def bench_cfg(name, n_tx=0):
    _, lcfg, _ = bench.make_cfg(types.SimpleNamespace(config=name, n_tx=n_tx), 1, 0)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    return lcfg.with_(client_warps=bench.tuned_client_warps(name, sms), log_mode=csmv.LOG_DIGEST)


@pytest.mark.parametrize("name", ["C2", "C3"])
def test_bank_full_size_bench_launch(name):
    cfg = bench_cfg(name)
    init = cfg.init_values()
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(init)
        stats = st.run(cfg.workload, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx)
        rings = st.dump()
    ocfg = oracle_cfg(cfg)
    rep = oracle.bank_check(ocfg, init, oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx), log, rings=rings,
                            claims=dict(committed_update=stats["committed_update"],
                                        committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                        total_aborts=stats["total_aborts"]))
    assert rep["ok"], (name, rep, stats)
    assert stats["committed"] == cfg.n_tx
    assert stats["gts_final"] == stats["committed_update"]


def test_kv_full_size_bench_launch():
    cfg = bench_cfg("C4")
    w = cfg.workload
    with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
        st.load(w.kv_keys)
        pre = st.dump()
        stats = st.run(w, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx)
        fin = st.dump()
    oc = ocfg_of(cfg)
    init = oracle.kv_preload(oc)
    for a, b in zip(pre, (init.keys, init.vals, init.lru, init.clocks)):
        assert np.array_equal(a, b)
    rep = oracle.kv_check(oc, init, oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log,
                          final=as_state(fin, cfg.n_items, w.kv_ways),
                          claims=dict(committed_update=stats["committed_update"],
                                      committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                      total_aborts=stats["total_aborts"]))
    assert rep["ok"], (rep, stats)
    assert stats["committed"] == cfg.n_tx
