"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element -- every committed transaction's snapshot, CTS, attempts,
read digest and written values, every value a FULL log records, the final
version rings, and the claimed counters."""
import numpy as np
import pytest

import oracle
from tests import _ref as R

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402


def oracle_cfg(cfg):
    w = cfg.workload
    return oracle.bank_cfg(cfg.n_items, cfg.n_versions, dist=w.dist,
                           zipf_theta_milli=w.zipf_theta_milli, p_update_ppm=w.p_update_ppm,
                           ro_period=w.ro_period, ro_reads=w.ro_reads, amount_max=w.amount_max,
                           ro_streak=w.ro_streak)


def run_gpu(cfg, init=None):
    init = cfg.init_values() if init is None else init
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(init)
        stats = st.run(cfg.workload, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx) if cfg.workload.log_mode else None
        vals = st.vals() if cfg.workload.log_mode == csmv.LOG_FULL else (None, 0)
        rings = st.dump()
    return stats, log, vals, rings


def check(cfg, init=None, expect_ok=True):
    init = cfg.init_values() if init is None else init
    stats, log, (vals, mv), rings = run_gpu(cfg, init)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    rep = oracle.bank_check(ocfg, init, descs, log, vals=vals, max_vals=mv, rings=rings,
                            claims=dict(committed_update=stats["committed_update"],
                                        committed_ro=stats["committed_ro"],
                                        gts_final=stats["gts_final"],
                                        total_aborts=stats["total_aborts"]))
    if expect_ok:
        assert rep["ok"], (cfg.name, rep, stats)
    return rep, stats, log, rings, descs


def closed_form(cfg, descs, init):
    upd = descs["is_update"] == 1
    final = init.astype(np.int64).copy()
    np.add.at(final, descs["src"][upd], -descs["amt"][upd].astype(np.int64))
    np.add.at(final, descs["dst"][upd], descs["amt"][upd].astype(np.int64))
    return final.astype(np.int32)


def newest(rings, n, k):
    rr = rings.reshape(n, k)
    ts = (rr >> np.uint64(32)).astype(np.int64)
    ts[ts == R.EMPTY] = -1
    return (rr[np.arange(n), ts.argmax(axis=1)] & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)


@pytest.mark.parametrize("publish", [csmv.PUBLISH_CLIENT, csmv.PUBLISH_SERVER])
def test_c1_full_parity(publish):
    cfg = W.c1(publish=publish)
    rep, stats, log, rings, descs = check(cfg)
    init = cfg.init_values()
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, init))  # P1
    assert np.all(log["aux"][descs["is_update"] == 0].view(np.int64) == 1024 * 1000)  # P2
    assert stats["gts_final"] == 10000 and stats["committed_ro"] == 1111           # P3
    assert sum(stats["aborts"][r]["ro"] for r in ("preval", "conflict", "early", "overflow")) == 0


@pytest.mark.parametrize("k,streak,ro_reads", [(1, 0, 0), (2, 0, 0), (4, 0, 0), (8, 0, 0), (16, 0, 0),
                                               (4, 4, 0), (4, 8, 16), (2, 1, 16),
                                               # ragged warp-cooperative scans: 2-3 rows with a
                                               # partial last row, more rows than fit in flight
                                               (2, 4, 70), (4, 8, 33), (4, 2, 300)])
def test_one_warp_is_deterministic(k, streak, ro_reads):
    """with one client warp the oracle predicts every snapshot,
    CTS, attempt count and ring exactly."""
    cfg = W.c1(client_warps=1, n_versions=k, n_tx=3000, log_mode=csmv.LOG_FULL,
               ro_streak=streak, ro_reads=ro_reads)
    stats, log, (vals, mv), rings = run_gpu(cfg)
    ocfg = oracle_cfg(cfg)
    descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
    plog, pvals, prings, pst = oracle.bank_predict(ocfg, cfg.init_values(), descs, 32, max_vals=mv)
    bad = np.nonzero(log != plog)[0]
    assert len(bad) == 0, (bad[:5], log[bad[:5]], plog[bad[:5]])
    assert np.array_equal(vals, pvals)
    assert np.array_equal(rings, prings)
    assert stats["aborts"]["preval"]["update"] == pst["aborts_preval"]
    assert stats["total_aborts"] == pst["aborts_preval"]
    assert stats["batches"] == pst["batches"] and stats["rounds"] == pst["rounds"]


@pytest.mark.parametrize("publish,streak,workers,combine", [
    (csmv.PUBLISH_CLIENT, 0, 4, 1), (csmv.PUBLISH_SERVER, 0, 6, 1), (csmv.PUBLISH_SERVER, 8, 6, 4),
    (csmv.PUBLISH_CLIENT, 8, 2, 2), (csmv.PUBLISH_SERVER, 8, 6, 3)])
def test_c2_shrunk_parity(publish, streak, workers, combine):
    cfg = W.c2(n_items=1 << 16, n_tx=1 << 18, publish=publish, ro_streak=streak,
               server_workers=workers, server_combine=combine, client_warps=512)
    rep, stats, log, rings, descs = check(cfg)
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions),
                          closed_form(cfg, descs, cfg.init_values()))


@pytest.mark.parametrize("streak", [0, 8])
def test_c3_shrunk_parity(streak):
    cfg = W.c3(n_tx=1 << 18, ro_streak=streak, client_warps=256, server_combine=4, server_workers=6)
    rep, stats, log, rings, descs = check(cfg)
    assert stats["aborts"]["conflict"]["ro"] == 0 and stats["aborts"]["early"]["ro"] == 0  # P6/Q7


def test_version_misses_k1():
    """K = 1 under contention: read-only transactions restart only with
    VERSION_MISS, and parity still holds."""
    cfg = W.c3(n_versions=1, n_tx=1 << 16)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["version"]["ro"] > 0
    assert stats["aborts"]["conflict"]["ro"] == 0


@pytest.mark.parametrize("combine", [1, 4])
def test_tiny_atr_overflow(combine):
    """A tiny ATR forces evictions: spurious aborts appear only with the
    labelled OVERFLOW reason and never let a conflicting commit through."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 17, atr_capacity=16, server_combine=combine, client_warps=256)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["overflow"]["update"] > 0


def test_read_only_workload():
    """P5: p_update = 0 leaves the store unchanged; zero aborts and no batches."""
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 16, p_update_ppm=0)
    rep, stats, log, rings, _ = check(cfg)
    assert stats["total_aborts"] == 0 and stats["batches"] == 0 and stats["gts_final"] == 0
    assert np.all((rings.reshape(-1, cfg.n_versions)[:, 0] >> np.uint64(32)) == 0)


def test_empty_run():
    cfg = W.c2(n_items=1 << 10, n_tx=0)
    stats, *_ = run_gpu(cfg)
    assert stats["committed"] == 0 and stats["gts_final"] == 0


@pytest.mark.parametrize("combine", [1, 4])
def test_update_only_high_contention(combine):
    cfg = W.c2(n_items=64, n_tx=1 << 15, p_update_ppm=1_000_000, client_warps=64, server_combine=combine)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["preval"]["update"] > 0


def test_no_validate_is_caught():
    """Negative control: a server that skips validation produces
    a history the oracle rejects."""
    cfg = W.c2(n_items=128, n_tx=1 << 15, p_update_ppm=900_000, client_warps=64,
               debug_flags=csmv.DBG_NO_VALIDATE)
    rep, *_ = check(cfg, expect_ok=False)
    assert not rep["ok"]
    # the same through the commit ring (one CTA, then a cluster)
    for srv, fl in ((csmv.SERVER_CTA, csmv.DBG_ALT_COMMIT), (csmv.SERVER_CLUSTER, 0)):
        rep, *_ = check(cfg.with_(server=srv, cluster_size=4, debug_flags=csmv.DBG_NO_VALIDATE | fl),
                        expect_ok=False)
        assert not rep["ok"]


def test_generator_parity():
    """the device generator equals the oracle's regenerated
    descriptors, and the zipf tables are byte-equal."""
    for cfg in (W.c1(), W.c2(n_items=1 << 20), W.c3()):
        ocfg = oracle_cfg(cfg)
        od = oracle.bank_gen(ocfg, 77, 50_000, tx0=123)
        with csmv.Store(cfg.n_items, cfg.n_versions) as st:
            gd = st.gen_descs(cfg.workload, 77, 50_000, tx0=123)
        for j, f in enumerate(("is_update", "src", "dst", "amt", "start", "len")):
            assert np.array_equal(gd[:, j], od[f].astype(np.uint32)), f
    for n, th in ((4096, 990), (1 << 22, 990), (1000, 500)):
        assert np.array_equal(csmv.zipf_table(n, th), oracle.zipf_cdf(n, th))


def test_runs_continue_from_store():
    """Two runs back to back continue the store and GTS."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 14, log_mode=csmv.LOG_NONE)
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(cfg.init_values())
        s1 = st.run(cfg.workload, cfg.n_tx, 1)
        s2 = st.run(cfg.workload, cfg.n_tx, 2)
        assert s2["gts_start"] == s1["gts_final"]
        assert s2["gts_final"] == s1["gts_final"] + s2["committed_update"]


@pytest.mark.parametrize("publish", [csmv.PUBLISH_CLIENT, csmv.PUBLISH_SERVER])
def test_reload_then_rerun(publish):
    """csmv_load restarts CTS at 1: nothing left from the previous run (done
    flags of the server publisher, lastw) may leak into the next one."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 15, publish=publish, client_warps=32, ro_streak=4, watchdog_ms=20_000)
    init = cfg.init_values()
    ocfg = oracle_cfg(cfg)
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        for seed in (1, 2):
            st.load(init)
            stats = st.run(cfg.workload, cfg.n_tx, seed)
            log = st.log(cfg.n_tx)
            rings = st.dump()
            descs = oracle.bank_gen(ocfg, seed, cfg.n_tx)
            rep = oracle.bank_check(ocfg, init, descs, log, rings=rings,
                                    claims=dict(committed_update=stats["committed_update"],
                                                committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                                total_aborts=stats["total_aborts"]))
            assert rep["ok"], (seed, rep)


@pytest.mark.parametrize("preset,streak", [("c2", 16), ("c3", 32)])
def test_ro_adaptive_parity(preset, streak):
    """ro_adaptive: read-only runs end when the batch is answered (a
    timing-dependent schedule) -- still every history replays exactly."""
    mk = getattr(W, preset)
    cfg = mk(n_items=1 << 12, n_tx=1 << 17, client_warps=128, ro_streak=streak, ro_adaptive=1,
             server_workers=6, server_combine=4, publish=csmv.PUBLISH_SERVER)
    rep, stats, log, rings, descs = check(cfg)
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))


@pytest.mark.parametrize("cap", [256, 1024])
def test_small_atr_bucket_races(cap):
    """A small recent-write filter (server.cuh filt_idx): lanes of one batch
    often share slots and the window saturates it, so many updates abort
    OVERFLOW -- but a write inside the window is never missed."""
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 17, atr_capacity=cap, server_combine=4, server_workers=6,
               client_warps=256, ro_streak=4, publish=csmv.PUBLISH_SERVER)
    rep, stats, log, rings, descs = check(cfg)
    assert np.array_equal(newest(rings, cfg.n_items, cfg.n_versions), closed_form(cfg, descs, cfg.init_values()))


@pytest.mark.parametrize("ro_reads,k", [(40, 4), (97, 2), (1, 4)])
def test_ragged_read_only_scans(ro_reads, k):
    """Warp-cooperative read-only scans (kernel.cu rot_coop) with lengths that
    are not a multiple of the 32-account row, wrapping past the last account,
    with version misses at K = 2, many warps, FULL log (every value read)."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 15, ro_reads=ro_reads, n_versions=k, log_mode=csmv.LOG_FULL,
               client_warps=64, ro_streak=8, p_update_ppm=300_000)
    check(cfg)


@pytest.mark.parametrize("publish", [0, 1])
def test_filter16_wraps(publish):
    """The 16-bit filter slots (server.cuh) wrap several times: > 4 x 2^16
    commits through the smallest filter (2K slots, so slots alias often) on a
    contended store.  Aliasing may only add OVERFLOW aborts -- a missed
    conflict would be a history the oracle rejects."""
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 19, p_update_ppm=700_000, atr_capacity=16, server_combine=8,
               server_workers=6, client_warps=256, publish=publish, ro_streak=8, ro_adaptive=1)
    rep, stats, *_ = check(cfg)
    assert stats["gts_final"] - stats["gts_start"] > 4 * 65536
    assert stats["aborts"]["overflow"]["update"] > 0


def test_blind_write_elision():
    """without blind writes the write-write check can be omitted.
    The bank qualifies (RS = WS): with elide_ww the history is still
    opaque, and with one client warp it is the very same history; the KV
    workload (blind value/LRU writes) is refused."""
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 16, client_warps=256, elide_ww=1, ro_streak=4)
    check(cfg)
    one = W.c1(client_warps=1, n_tx=3000, log_mode=csmv.LOG_FULL)
    a = run_gpu(one)
    b = run_gpu(one.with_(elide_ww=1))
    assert np.array_equal(a[1], b[1]) and np.array_equal(a[3], b[3])
    kv = W.c4(n_items=1 << 12, n_tx=1 << 10, elide_ww=1)
    with csmv.KvStore(kv.n_items, kv.workload.kv_ways, kv.n_versions) as st:
        st.load(kv.workload.kv_keys)
        with pytest.raises(csmv.CsmvError) as e:
            st.run(kv.workload, kv.n_tx, kv.seed)
        assert e.value.code == csmv.EINVAL


def test_tagged_requests_fall_back_above_24_bit_items():
    """Round-tagged requests carry the round in id bits 24-30, so a store
    with item ids >= 2^24 must run fenced requests instead -- and still pass
    the oracle (the self-receiving worker, where tags are otherwise taken)."""
    n = (1 << 24) + 4096
    cfg = W.c2(n_items=n, n_tx=1 << 15, client_warps=128, ro_reads=64, server_recv=csmv.RECV_SELF,
               server_workers=7, server_combine=2, publish=csmv.PUBLISH_CLIENT, req_tagged=1)
    rep, stats, *_ = check(cfg)
    assert stats["committed"] == cfg.n_tx


@pytest.mark.parametrize("kw", [dict(), dict(debug_flags=csmv.DBG_JITTER), dict(n_versions=2), dict(n_versions=8),
                                dict(publish=csmv.PUBLISH_CLIENT), dict(publish=csmv.PUBLISH_CLIENT, debug_flags=csmv.DBG_JITTER),
                                dict(req_tagged=1), dict(req_tagged=1, publish=csmv.PUBLISH_CLIENT, debug_flags=csmv.DBG_JITTER)])
def test_bank_server_writeback(kw):
    """Bank, self-receiving workers with server_writeback: the worker writes
    each committed transfer's versions and lastw and sets its done flag; the
    oracle replays the history and the final rings match the closed form."""
    kw = dict(dict(publish=csmv.PUBLISH_SERVER), **kw)
    cfg = W.c3(n_tx=1 << 16, client_warps=128, server_recv=csmv.RECV_SELF, server_workers=7, server_combine=2,
               ro_streak=4, ro_adaptive=1, server_writeback=1, **kw)
    rep, stats, log, rings, descs = check(cfg)
    assert stats["committed"] == cfg.n_tx
    c2 = W.c2(n_items=1 << 14, n_tx=1 << 16, client_warps=256, server_recv=csmv.RECV_SELF, server_workers=7,
              server_writeback=1, **kw)
    rep, stats, log, rings, descs = check(c2)
    assert np.array_equal(newest(rings, c2.n_items, c2.n_versions), closed_form(c2, descs, c2.init_values()))
