"""GPU parity of the MemcachedGPU workload (C4) against the CPU
oracle: preload, every GET's and PUT's digests, snapshots and CTS, the
final store, the counters; the 1-warp deterministic schedule exactly."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402


def ocfg_of(cfg):
    w = cfg.workload
    return oracle.kv_cfg(cfg.n_items, w.kv_ways, n_keys=w.kv_keys, n_versions=cfg.n_versions,
                         dist=w.dist, zipf_theta_milli=w.zipf_theta_milli, p_update_ppm=w.p_update_ppm,
                         ro_streak=w.ro_streak)


def as_state(dump, S, A):
    st = oracle.KvStore(S, A)
    st.keys[:], st.vals[:], st.lru[:], st.clocks[:] = dump
    return st


def run(cfg):
    w = cfg.workload
    with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
        st.load(w.kv_keys)
        pre = st.dump()
        stats = st.run(w, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx) if w.log_mode else None
        fin = st.dump()
    return pre, stats, log, fin


@pytest.mark.parametrize("S,A,keys", [(1 << 12, 16, 0), (1 << 10, 4, 0), (1 << 12, 16, 3 << 12),
                                      (1 << 12, 16, 1000), (1 << 10, 1, 0), (1 << 12, 256, 5 << 12),
                                      (256, 256, 3000), (1 << 22, 16, 0), (1 << 22, 16, 3 << 21)])
def test_preload_parity(S, A, keys):
    """The library's device preload (count, bucket, keep each set's A largest
    keys: a set's r-th insertion takes way r mod A) against the oracle's
    literal PUT-by-PUT preload, with fewer, as many and more keys than slots,
    one set (T = 1) and C4's full 4M slots."""
    cfg = W.c4(n_items=S, kv_ways=A, n_tx=0, **({"kv_keys": keys} if keys else {}))
    pre, *_ = run(cfg)
    ref = oracle.kv_preload(ocfg_of(cfg))
    for a, b in zip(pre, (ref.keys, ref.vals, ref.lru, ref.clocks)):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("p_update,streak,k,flags", [(10_000, 0, 4, 0), (10_000, 8, 4, 0), (200_000, 4, 4, 0),
                                                     (500_000, 0, 2, 0), (50_000, 8, 8, 0), (10_000, 8, 4, 16),
                                                     (200_000, 4, 4, 16)])
def test_kv_parity(p_update, streak, k, flags):
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, p_update_ppm=p_update, ro_streak=streak, n_versions=k,
               client_warps=256, server_workers=6, debug_flags=flags)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    init = oracle.kv_preload(oc)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    rep = oracle.kv_check(oc, init, d, log, final=as_state(fin, cfg.n_items, cfg.workload.kv_ways),
                          claims=dict(committed_update=stats["committed_update"],
                                      committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                      total_aborts=stats["total_aborts"]))
    assert rep["ok"], (rep, stats)
    assert stats["committed_update"] == int(d["is_update"].sum())


@pytest.mark.parametrize("flags", [0, csmv.DBG_KV_ITEMSETS])
@pytest.mark.parametrize("streak", [0, 4])
def test_kv_one_warp_deterministic(streak, flags):
    """Both request forms ({set clock} u WS by default, item by item with
    DBG_KV_ITEMSETS) keep and abort exactly the lanes the oracle's item-level
    predictor does."""
    cfg = W.c4(n_items=1 << 11, kv_ways=8, n_tx=4000, p_update_ppm=300_000, client_warps=1,
               ro_streak=streak, debug_flags=flags)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    init = oracle.kv_preload(oc)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    plog, pfin, ps = oracle.kv_predict(oc, init, d, 32)
    bad = np.nonzero(log != plog)[0]
    assert len(bad) == 0, (bad[:5], log[bad[:5]], plog[bad[:5]])
    for a, b in zip(fin, (pfin.keys, pfin.vals, pfin.lru, pfin.clocks)):
        assert np.array_equal(a, b)
    assert stats["total_aborts"] == ps["aborts_preval"] and stats["batches"] == ps["batches"]


def test_kv_generator_parity():
    cfg = W.c4()
    oc = ocfg_of(cfg)
    od = oracle.kv_gen(oc, 99, 20_000, tx0=5)
    with csmv.KvStore(1 << 10, 16, 4) as st:
        gd = st.gen_descs(cfg.workload, 99, 20_000, tx0=5)
    assert np.array_equal(gd[:, 0], od["is_update"]) and np.array_equal(gd[:, 1], od["key"])
    assert np.array_equal(gd[:, 2:], od["val"])


def test_kv_no_validate_is_caught():
    cfg = W.c4(n_items=1 << 8, kv_ways=4, n_tx=1 << 14, p_update_ppm=600_000, client_warps=64,
               debug_flags=csmv.DBG_NO_VALIDATE, dist=0)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log)
    assert not rep["ok"]


# ---- compact PUT read-sets ({set clock} u WS) and wide sets (4..256 ways) ----
def _check_kv(cfg):
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    init = oracle.kv_preload(oc)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    rep = oracle.kv_check(oc, init, d, log, final=as_state(fin, cfg.n_items, cfg.workload.kv_ways),
                          claims=dict(committed_update=stats["committed_update"],
                                      committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                      total_aborts=stats["total_aborts"]))
    assert rep["ok"], (rep, stats)
    return stats


@pytest.mark.parametrize("ways", [4, 16])
def test_kv_itemsets_one_warp_matches_item_level_predictor(ways):
    cfg = W.c4(n_items=1 << 11, kv_ways=ways, n_tx=4000, p_update_ppm=300_000, client_warps=1, ro_streak=4,
               debug_flags=csmv.DBG_KV_ITEMSETS)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    plog, pfin, ps = oracle.kv_predict(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), 32)
    assert np.array_equal(log, plog)
    for a, b in zip(fin, (pfin.keys, pfin.vals, pfin.lru, pfin.clocks)):
        assert np.array_equal(a, b)
    assert stats["total_aborts"] == ps["aborts_preval"]


@pytest.mark.parametrize("ways", [32, 256])
def test_kv_wide_sets_one_warp(ways):
    cfg = W.c4(n_items=ways * 64, kv_ways=ways, kv_keys=ways * 64, n_tx=3000, p_update_ppm=300_000,
               client_warps=1, ro_streak=4)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    plog, pfin, ps = oracle.kv_predict(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), 32)
    assert np.array_equal(log, plog)
    for a, b in zip(fin, (pfin.keys, pfin.vals, pfin.lru, pfin.clocks)):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("ways,p_update,flags", [(16, 50_000, 0), (16, 50_000, 16), (64, 2_000, 0),
                                                 (256, 2_000, 0), (256, 100_000, 0)])
def test_kv_wide_sets_parity(ways, p_update, flags):
    cfg = W.c4(n_items=1 << 16, kv_ways=ways, kv_keys=1 << 16, n_tx=1 << 16, p_update_ppm=p_update,
               client_warps=256, server_workers=6, ro_streak=4, debug_flags=flags)
    _check_kv(cfg)


def test_kv_wide_negative_control():
    cfg = W.c4(n_items=1 << 10, kv_ways=64, kv_keys=1 << 10, n_tx=1 << 14, p_update_ppm=600_000, client_warps=64,
               debug_flags=csmv.DBG_NO_VALIDATE, dist=0)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log)
    assert not rep["ok"]


def test_kv_ro_adaptive_parity():
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, p_update_ppm=20_000, client_warps=256, server_workers=6,
               ro_streak=32, ro_adaptive=1)
    _check_kv(cfg)


def test_kv_small_atr():
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, p_update_ppm=100_000, client_warps=256, server_workers=6,
               atr_capacity=256, dist=0)
    _check_kv(cfg)


@pytest.mark.parametrize("workers,jitter", [(7, 0), (3, 0), (7, csmv.DBG_JITTER)])
def test_kv_self_receiving_workers(workers, jitter):
    """The KV filter worker with self-receiving worker warps
    (CSMV_RECV_SELF): each sweeps its slice of the doorbells, no receiver."""
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, p_update_ppm=100_000, ro_streak=8, client_warps=256,
               server_workers=workers, server_recv=csmv.RECV_SELF, publish=1, debug_flags=jitter)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log,
                          final=as_state(fin, cfg.n_items, cfg.workload.kv_ways),
                          claims=dict(committed_update=stats["committed_update"],
                                      committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                      total_aborts=stats["total_aborts"]))
    assert rep["ok"], (rep, stats)
    assert stats["server_workers"] == workers


# ---- CSMV_RETRY_FIFO: per-set PUT tickets (client-side contention management) ----
@pytest.mark.parametrize("kw", [
    dict(p_update_ppm=10_000, ro_streak=32, ro_adaptive=2),                          # C4-shaped, zipf
    dict(p_update_ppm=300_000, ro_streak=4, ro_adaptive=1),                          # many PUTs per set
    dict(p_update_ppm=100_000, ro_streak=8, ro_adaptive=2, publish=1),               # server publisher
    dict(p_update_ppm=100_000, ro_streak=8, ro_adaptive=2, debug_flags=csmv.DBG_JITTER),
    dict(p_update_ppm=100_000, ro_streak=8, server_recv=csmv.RECV_SELF, server_workers=7, publish=1),
    dict(p_update_ppm=50_000, ro_streak=8, ro_adaptive=2, debug_flags=csmv.DBG_KV_ITEMSETS),
    dict(p_update_ppm=50_000, ro_streak=8, ro_adaptive=2, server=csmv.SERVER_CLUSTER, cluster_size=4),
])
def test_kv_retry_fifo_parity(kw):
    """PUTs on a set attempt in ticket order: the history is still the one
    the replaying oracle accepts (validation is unchanged), every PUT commits
    once, and no PUT loses to another PUT of its set (no PREVAL, no EARLY)."""
    kw = dict(dict(server_workers=6), **kw)
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, client_warps=256, retry_order=csmv.RETRY_FIFO, **kw)
    stats = _check_kv(cfg)
    ab = stats["aborts"]
    assert ab["preval"]["update"] == 0 and ab["early"]["update"] == 0 and ab["conflict"]["update"] == 0, ab


def test_kv_retry_fifo_one_set():
    """Every PUT on one cache set (T = 1): a single ticket queue of 64 warps."""
    cfg = W.c4(n_items=16, kv_ways=16, kv_keys=64, n_tx=1 << 14, p_update_ppm=200_000, client_warps=64,
               ro_streak=4, ro_adaptive=2, retry_order=csmv.RETRY_FIFO)
    stats = _check_kv(cfg)
    assert stats["aborts"]["preval"]["update"] == 0


def test_kv_retry_fifo_orders_each_set():
    """The tickets alone serialise the PUTs of a set (each reads at a
    snapshot covering the previous ticket's commit, and nothing else writes
    the set): even with the server's validation and the clients'
    pre-validation switched off the history is one the oracle accepts --
    whereas the same run without tickets is rejected
    (test_kv_no_validate_is_caught)."""
    cfg = W.c4(n_items=1 << 8, kv_ways=4, n_tx=1 << 14, p_update_ppm=600_000, client_warps=64, dist=0,
               retry_order=csmv.RETRY_FIFO, debug_flags=csmv.DBG_NO_VALIDATE | csmv.DBG_NO_PREVAL)
    pre, stats, log, fin = run(cfg)
    oc = ocfg_of(cfg)
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), log,
                          final=as_state(fin, cfg.n_items, cfg.workload.kv_ways))
    assert rep["ok"], rep


# ---- the warp-cooperative PUT read (default) against the lane's own scan ----
@pytest.mark.parametrize("ways,k", [(16, 4), (8, 2), (4, 8), (16, 16), (2, 4)])
def test_kv_coop_read_one_warp_matches_predictor(ways, k):
    """The one-trip cooperative read decides every PUT as the oracle's
    item-level predictor does (same victims, digests, aborts), at several
    associativities and version counts, with and without the lane's own scan."""
    for flags in (0, csmv.DBG_KV_SEQREAD):
        cfg = W.c4(n_items=ways * 128, kv_ways=ways, n_versions=k, n_tx=3000, p_update_ppm=300_000,
                   client_warps=1, ro_streak=4, debug_flags=flags)
        pre, stats, log, fin = run(cfg)
        oc = ocfg_of(cfg)
        plog, pfin, ps = oracle.kv_predict(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), 32)
        assert np.array_equal(log, plog), flags
        for a, b in zip(fin, (pfin.keys, pfin.vals, pfin.lru, pfin.clocks)):
            assert np.array_equal(a, b)


@pytest.mark.parametrize("kw", [dict(kv_keys=3 << 12), dict(kv_keys=1000), dict(n_versions=2), dict(n_versions=8),
                                dict(debug_flags=csmv.DBG_JITTER)])
def test_kv_coop_read_parity(kw):
    """Contended runs with the cooperative read: misses (more keys than
    slots: LRU victims), fewer keys than slots (empty ways), K = 2/8, jitter."""
    kw = dict(dict(n_items=1 << 12, n_tx=1 << 16, p_update_ppm=100_000, ro_streak=8, ro_adaptive=2,
                   client_warps=256, server_workers=6), **kw)
    _check_kv(W.c4(**kw))


# ---- server write-back (csmv_workload.server_writeback): the worker writes the PUT's versions and publishes ----
@pytest.mark.parametrize("kw", [
    dict(p_update_ppm=10_000, ro_streak=32, ro_adaptive=2, backoff_max=16, publish=1),
    dict(p_update_ppm=300_000, ro_streak=4, ro_adaptive=1, publish=0),
    dict(p_update_ppm=100_000, ro_streak=8, ro_adaptive=2, publish=1, debug_flags=csmv.DBG_JITTER),
    dict(p_update_ppm=100_000, ro_streak=8, ro_adaptive=2, publish=0, debug_flags=csmv.DBG_JITTER),
    dict(p_update_ppm=100_000, ro_streak=8, server_recv=csmv.RECV_SELF, server_workers=7, publish=1, req_tagged=1),
    dict(p_update_ppm=50_000, ro_streak=8, ro_adaptive=2, server=csmv.SERVER_CLUSTER, cluster_size=4, publish=1),
    dict(p_update_ppm=50_000, ro_streak=8, ro_adaptive=2, n_versions=2, publish=0),
    dict(p_update_ppm=10_000, ro_streak=32, ro_adaptive=2, backoff_max=16, publish=1, req_tagged=1),
    dict(p_update_ppm=200_000, ro_streak=8, ro_adaptive=2, publish=1, req_tagged=1, debug_flags=csmv.DBG_JITTER),
    dict(p_update_ppm=200_000, ro_streak=8, ro_adaptive=2, publish=0, req_tagged=1, debug_flags=csmv.DBG_JITTER),
])
def test_kv_server_writeback_parity(kw):
    kw = dict(dict(server_workers=6), **kw)
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, client_warps=256, server_writeback=1, **kw)
    _check_kv(cfg)


def test_kv_server_writeback_one_warp():
    """With one client warp the schedule is the client's own: the server
    writing the versions back changes no snapshot, CTS or ring slot."""
    for swb in (0, 1):
        cfg = W.c4(n_items=1 << 11, kv_ways=8, n_tx=4000, p_update_ppm=300_000, client_warps=1, ro_streak=4,
                   server_writeback=swb)
        pre, stats, log, fin = run(cfg)
        oc = ocfg_of(cfg)
        plog, pfin, ps = oracle.kv_predict(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, cfg.n_tx), 32)
        assert np.array_equal(log, plog), swb
        for a, b in zip(fin, (pfin.keys, pfin.vals, pfin.lru, pfin.clocks)):
            assert np.array_equal(a, b)
