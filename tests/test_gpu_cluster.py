"""GPU parity of the thread-block-cluster server (receivers and workers in
every CTA of the cluster, the bank commit through the commit ring to one
committer warp in CTA 0; KV and the A/B flag: the recent-commit table striped
over the CTAs' shared memory through DSMEM under a ticket lock in CTA 0) and
of the single-CTA server on the same workloads (C5's server axis)."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_parity import check, closed_form, newest  # noqa: E402
from tests.test_gpu_kv import ocfg_of, as_state, run as run_kv  # noqa: E402


@pytest.mark.parametrize("cs,flags", [(2, 0), (4, 0), (8, 0), (16, 0), (2, csmv.DBG_ALT_COMMIT),
                                      (16, csmv.DBG_ALT_COMMIT)])
def test_bank_cluster_parity(cs, flags):
    cfg = W.c2(n_items=1 << 16, n_tx=1 << 18, server=csmv.SERVER_CLUSTER, cluster_size=cs,
               publish=csmv.PUBLISH_SERVER, ro_streak=8, server_workers=6, server_combine=4,
               client_warps=256, debug_flags=flags)
    rep, stats, log, rings, descs = check(cfg)
    assert stats["server_ctas"] == cs
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))


def test_bank_cluster_contention_and_tiny_table():
    """Hot items and a tiny striped table: OVERFLOW aborts appear, parity holds."""
    cfg = W.c2(n_items=1 << 10, n_tx=1 << 17, server=csmv.SERVER_CLUSTER, cluster_size=4,
               atr_capacity=64, p_update_ppm=700_000, client_warps=128, server_combine=4, server_workers=6)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["overflow"]["update"] > 0


def test_c3_cluster_parity():
    cfg = W.c3(n_tx=1 << 17, server=csmv.SERVER_CLUSTER, cluster_size=8, client_warps=128,
               ro_streak=8, server_combine=4, server_workers=6)
    check(cfg)


def test_kv_cluster_parity():
    cfg = W.c4(n_items=1 << 13, n_tx=1 << 16, p_update_ppm=100_000, server=csmv.SERVER_CLUSTER,
               cluster_size=4, client_warps=128, server_workers=6)
    pre, stats, log, fin = run_kv(cfg)
    oc = ocfg_of(cfg)
    init = oracle.kv_preload(oc)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    rep = oracle.kv_check(oc, init, d, log, final=as_state(fin, cfg.n_items, cfg.workload.kv_ways),
                          claims=dict(committed_update=stats["committed_update"], committed_ro=stats["committed_ro"],
                                      gts_final=stats["gts_final"], total_aborts=stats["total_aborts"]))
    assert rep["ok"], rep


def test_cluster_one_client_warp_is_deterministic():
    """P7 holds with the cluster server too (the server's shape is invisible)."""
    cfg = W.c1(client_warps=1, n_tx=2000, server=csmv.SERVER_CLUSTER, cluster_size=2, ro_streak=4)
    from tests.test_gpu_parity import run_gpu, oracle_cfg
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    assert np.array_equal(log, plog) and np.array_equal(rings, prings)


@pytest.mark.parametrize("publish", [0, 1])
def test_bank_commit_ring_single_cta(publish):
    """The commit ring on the single-CTA server (CSMV_DBG_ALT_COMMIT): same
    history checks, closed-form final store."""
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 18, publish=publish, ro_streak=8, server_workers=6,
               server_combine=4, client_warps=256, debug_flags=csmv.DBG_ALT_COMMIT)
    rep, stats, log, rings, descs = check(cfg)
    assert stats["server_workers"] == 5  # the last warp of CTA 0 is the committer
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))


@pytest.mark.parametrize("server,flags", [(0, 32), (1, 0), (1, 32)])
def test_commit_designs_one_client_warp_deterministic(server, flags):
    """P7 through every commit design: ring or lock, one CTA or a cluster."""
    cfg = W.c1(client_warps=1, n_tx=2000, server=server, cluster_size=4, ro_streak=4, debug_flags=flags)
    from tests.test_gpu_parity import run_gpu, oracle_cfg
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    assert np.array_equal(log, plog) and np.array_equal(rings, prings)


@pytest.mark.parametrize("workers", [1, 3, 7])
def test_bank_self_receiving_workers(workers):
    """Self-receiving worker warps (CSMV_RECV_SELF) with 1, 3 and 7 workers,
    and the receiver-warp design on the same workload."""
    for recv in (csmv.RECV_SELF, csmv.RECV_WARP):
        cfg = W.c2(n_items=1 << 14, n_tx=1 << 17, publish=1, ro_streak=8, server_workers=workers,
                   server_combine=8, client_warps=200, server_recv=recv)
        rep, stats, log, rings, descs = check(cfg)
        # a receiver warp takes one of the 8; the publisher another unless it runs on a client CTA
        assert stats["server_workers"] == (workers if recv == csmv.RECV_SELF else min(workers, 7))
        assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions),
                              closed_form(cfg, descs, cfg.init_values()))


def test_self_receiving_one_warp_deterministic_and_c3():
    """P7 and a contended C3 run through the self-receiving server."""
    cfg = W.c1(client_warps=1, n_tx=2000, ro_streak=4, server_recv=csmv.RECV_SELF)
    from tests.test_gpu_parity import run_gpu, oracle_cfg
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    assert np.array_equal(log, plog) and np.array_equal(rings, prings)
    check(W.c3(n_tx=1 << 17, client_warps=128, ro_streak=8, server_combine=8, server_workers=7,
               server_recv=csmv.RECV_SELF, publish=1, ro_adaptive=1))
