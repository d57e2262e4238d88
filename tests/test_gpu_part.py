"""Item-partitioned servers (CSMV_SERVER_PART; NEXT-3; DESIGN.md
11; server_part.cuh): S server CTAs each own the items hashing to them; a
batch prepares at every owner (validate that part, mark it pending), takes
its CTS from one global counter, and decides at each.  The protocol was
checked by exhaustive interleavings first (tests/test_oracle_protocols.py);
here every committed transaction of the GPU runs is replayed by the oracle
(CTS dense and contiguous per batch)."""
import pytest

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_parity import check, closed_form, newest  # noqa: E402

P = csmv.SERVER_PART


@pytest.mark.parametrize("servers", [2, 4, 8])
@pytest.mark.parametrize("publish", [csmv.PUBLISH_SERVER, csmv.PUBLISH_CLIENT])
def test_part_c2_shrunk(servers, publish):
    cfg = W.c2(n_items=1 << 16, n_tx=1 << 18, client_warps=288, server=P, cluster_size=servers, publish=publish,
               ro_streak=8, ro_adaptive=1, server_workers=6)
    rep, stats, log, rings, descs = check(cfg)
    assert (newest(rings, cfg.n_items, cfg.n_versions) == closed_form(cfg, descs, cfg.init_values())).all()
    assert stats["committed"] == cfg.n_tx and stats["server_ctas"] == servers


@pytest.mark.parametrize("servers", [2, 4])
def test_part_hot_and_full_log(servers):
    """Contention (zipf 0.99 over 4,096 accounts) and C1 with every value read."""
    check(W.c3(n_tx=1 << 16, client_warps=256, server=P, cluster_size=servers, ro_streak=4))
    check(W.c1(server=P, cluster_size=servers))
    check(W.c2(n_items=256, n_tx=1 << 15, client_warps=288, p_update_ppm=900_000, server=P, cluster_size=servers))


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_part_no_starvation(seed):
    """288 warps on 4,096 accounts: with a fixed sweep order the servers
    starved the last rows of their slices -- decides included, whose pending
    marks then rejected every other prepare (a livelock the watchdog ended
    in about half of the seeds).  The round-robin sweep finishes all."""
    check(W.c2(n_items=1 << 12, n_tx=1 << 16, client_warps=288, server=P, cluster_size=2, publish=csmv.PUBLISH_CLIENT,
               watchdog_ms=5000, seed=seed))


@pytest.mark.parametrize("servers", [2, 8])
def test_part_under_jitter(servers):
    check(W.c2(n_items=1 << 12, n_tx=1 << 16, client_warps=256, server=P, cluster_size=servers,
               debug_flags=csmv.DBG_JITTER, ro_streak=4))


def test_part_negative_control():
    """Without validation at the servers (the pending marks and the
    records) conflicting transfers commit together: the oracle rejects."""
    cfg = W.c2(n_items=128, n_tx=1 << 14, client_warps=288, p_update_ppm=900_000, server=P, cluster_size=2,
               debug_flags=csmv.DBG_NO_VALIDATE)
    rep, *_ = check(cfg, expect_ok=False)
    assert not rep["ok"]


@pytest.mark.parametrize("kw", [dict(cluster_size=3), dict(cluster_size=16), dict(client_group=4),
                                dict(atr_mode=csmv.ATR_LIST), dict(commit=csmv.COMMIT_ONLYCS)])
def test_part_rejects(kw):
    kw = dict(kw)
    cfg = W.c2(n_items=1 << 12, n_tx=1 << 10, client_warps=64, server=P, **dict(dict(cluster_size=2), **kw))
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(cfg.init_values())
        with pytest.raises(csmv.CsmvError) as e:
            st.run(cfg.workload, cfg.n_tx, cfg.seed)
        assert e.value.code == csmv.EINVAL
