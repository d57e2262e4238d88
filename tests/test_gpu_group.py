"""CTA-level batches (csmv_workload.client_group): the G
client warps of a group pre-validate against each other in shared memory
(P:118 across warps) and submit one request the server commits in one step
of its critical section.  Every committed transaction is
replayed by the oracle (batches conflict-free, P4), with ragged
groups (CTAs with fewer warps than G), both publish modes, contention and
race widening."""
import pytest

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_parity import check, closed_form, newest  # noqa: E402


@pytest.mark.parametrize("group,warps", [(2, 294), (2, 256), (4, 588), (4, 500), (8, 1176), (8, 700), (2, 3)])
@pytest.mark.parametrize("publish", [csmv.PUBLISH_SERVER, csmv.PUBLISH_CLIENT])
def test_group_c2_shrunk(group, warps, publish):
    cfg = W.c2(n_items=1 << 16, n_tx=1 << 18, client_warps=warps, client_group=group, publish=publish,
               ro_streak=8, ro_adaptive=1, server_workers=6, server_combine=8)
    rep, stats, log, rings, descs = check(cfg)
    assert (newest(rings, cfg.n_items, cfg.n_versions) == closed_form(cfg, descs, cfg.init_values())).all()
    assert stats["committed"] == cfg.n_tx


@pytest.mark.parametrize("group", [2, 4, 8])
def test_group_contention(group):
    """256 accounts and 588 warps: most groups hold conflicting transfers
    across their warps, which the cross-warp pre-validation must drop."""
    cfg = W.c2(n_items=256, n_tx=1 << 16, client_warps=588, client_group=group, p_update_ppm=900_000,
               ro_streak=2, server_combine=8, server_workers=6)
    rep, stats, *_ = check(cfg)
    assert stats["aborts"]["preval"]["update"] > 0


@pytest.mark.parametrize("group", [2, 4])
def test_group_c1_full_log_and_jitter(group):
    check(W.c1(client_warps=150 * group, client_group=group))
    check(W.c1(client_warps=150 * group, client_group=group, debug_flags=csmv.DBG_JITTER))
    check(W.c3(n_tx=1 << 16, client_warps=296, client_group=group, debug_flags=csmv.DBG_JITTER, ro_streak=4,
               server_combine=8))


def test_group_negative_control():
    """The cross-warp check is what keeps a group's request conflict-free:
    without any pre-validation the oracle rejects the history."""
    cfg = W.c2(n_items=128, n_tx=1 << 14, client_warps=296, client_group=2, p_update_ppm=900_000,
               debug_flags=csmv.DBG_NO_PREVAL)
    rep, *_ = check(cfg, expect_ok=False)
    assert not rep["ok"]


@pytest.mark.parametrize("group", [2, 4])
@pytest.mark.parametrize("kw", [dict(server=csmv.SERVER_CLUSTER, cluster_size=4),
                                dict(server=csmv.SERVER_CLUSTER, cluster_size=16),
                                dict(debug_flags=csmv.DBG_ALT_COMMIT),
                                dict(server=csmv.SERVER_CLUSTER, cluster_size=8, debug_flags=csmv.DBG_JITTER)])
def test_group_commit_ring(group, kw):
    """Client groups into the commit ring (cluster server, or one CTA with
    DBG_ALT_COMMIT): a request's G batches take G consecutive ring slots and
    the committer commits them in one step of its chain."""
    cfg = W.c2(n_items=1 << 16, n_tx=1 << 18, client_warps=148 * group, client_group=group,
               publish=csmv.PUBLISH_SERVER, ro_streak=8, ro_adaptive=1, server_combine=8, **kw)
    rep, stats, log, rings, descs = check(cfg)
    assert (newest(rings, cfg.n_items, cfg.n_versions) == closed_form(cfg, descs, cfg.init_values())).all()
    check(W.c3(n_tx=1 << 16, client_warps=148 * group, client_group=group, server=csmv.SERVER_CLUSTER,
               cluster_size=4, ro_streak=4))


@pytest.mark.parametrize("kw", [dict(server_recv=csmv.RECV_SELF), dict(atr_mode=csmv.ATR_LIST),
                                dict(commit=csmv.COMMIT_JVSTM), dict(client_group=3),
                                dict(server=csmv.SERVER_CLUSTER, cluster_size=4, client_group=8)])
def test_group_rejects_other_servers(kw):
    kw = dict(kw)
    g = kw.pop("client_group", 2)
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 10, client_warps=64, client_group=g, **kw)
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(cfg.init_values())
        with pytest.raises(csmv.CsmvError) as e:
            st.run(cfg.workload, cfg.n_tx, cfg.seed)
        assert e.value.code == csmv.EINVAL
