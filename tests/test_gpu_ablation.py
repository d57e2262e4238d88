"""GPU parity of the paper's own ATR design (NEXT-1 ablations): the ATR as
a CTS-indexed list of write-sets validated by a warp-cooperative scan
(collaborative validation) or one lane per transaction (CSMV-NoCV,
P:264-266)."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_parity import check, closed_form, newest, run_gpu, oracle_cfg  # noqa: E402


@pytest.mark.parametrize("mode", [csmv.ATR_LIST, csmv.ATR_LIST_NOCV])
@pytest.mark.parametrize("combine", [1, 4])
def test_list_atr_parity(mode, combine):
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 17, atr_mode=mode, client_warps=48, server_combine=combine,
               server_workers=6, ro_streak=8, publish=csmv.PUBLISH_SERVER)
    rep, stats, log, rings, descs = check(cfg)
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))


@pytest.mark.parametrize("mode", [csmv.ATR_LIST, csmv.ATR_LIST_NOCV])
def test_list_atr_c1_full(mode):
    check(W.c1(atr_mode=mode))


def test_list_atr_overflow():
    """A 64-entry ring: snapshots older than the ring abort with OVERFLOW."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 16, atr_mode=csmv.ATR_LIST, atr_capacity=64, client_warps=64)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["overflow"]["update"] > 0


def test_list_atr_one_warp_deterministic():
    cfg = W.c1(client_warps=1, n_tx=2000, atr_mode=csmv.ATR_LIST_NOCV, ro_streak=4)
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    assert np.array_equal(log, plog) and np.array_equal(rings, prings)


def test_list_atr_rejects_kv_and_cluster():
    with pytest.raises(csmv.CsmvError):
        cfg = W.c2(n_items=1 << 10, n_tx=100, atr_mode=csmv.ATR_LIST, server=csmv.SERVER_CLUSTER, cluster_size=2)
        run_gpu(cfg)


# ---- commit-protocol ablations ----
COMMITS = [csmv.COMMIT_ONLYCS, csmv.COMMIT_JVSTM]


@pytest.mark.parametrize("commit", COMMITS)
def test_commit_ablation_c1_full(commit):
    """C1 in full, FULL log: every read value, snapshot, CTS and ring slot
    replayed by the oracle."""
    check(W.c1(commit=commit))


@pytest.mark.parametrize("commit", COMMITS)
@pytest.mark.parametrize("publish", [csmv.PUBLISH_CLIENT, csmv.PUBLISH_SERVER])
def test_commit_ablation_c2(commit, publish):
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 17, commit=commit, client_warps=96, publish=publish, ro_streak=8)
    rep, stats, log, rings, descs = check(cfg)
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))
    if commit == csmv.COMMIT_ONLYCS:
        assert stats["aborts"]["preval"]["update"] == 0  # no client pre-validation


@pytest.mark.parametrize("commit", COMMITS)
def test_commit_ablation_contended(commit):
    """Zipf 0.99 over 256 accounts: most updates conflict."""
    cfg = W.c3(n_items=256, n_tx=1 << 15, commit=commit, client_warps=64)
    rep, stats, log, rings, descs = check(cfg)
    assert stats["aborts"]["conflict"]["update"] + stats["aborts"]["early"]["update"] > 0


def test_onlycs_one_warp_matches_predictor():
    """One client warp: snapshots are always current, so sequential server
    validation keeps exactly the lanes greedy pre-validation keeps;
    only the abort label moves from PREVAL to CONFLICT."""
    cfg = W.c1(client_warps=1, n_tx=2000, commit=csmv.COMMIT_ONLYCS, ro_streak=4)
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    assert np.array_equal(log, plog) and np.array_equal(rings, prings)
    assert stats["aborts"]["conflict"]["update"] == pst["aborts_preval"]
    assert stats["aborts"]["preval"]["update"] == 0


@pytest.mark.parametrize("commit", COMMITS)
def test_commit_ablation_negative_control(commit):
    """Validation switched off: the oracle must reject the history."""
    cfg = W.c3(n_items=64, n_tx=1 << 14, commit=commit, client_warps=64, debug_flags=csmv.DBG_NO_VALIDATE)
    rep, *_ = check(cfg, expect_ok=False)
    assert not rep["ok"]


def test_jvstm_counts_cas_failures():
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 16, commit=csmv.COMMIT_JVSTM, client_warps=256)
    rep, stats, *_ = check(cfg)
    assert stats["cas_failures"] > 0
