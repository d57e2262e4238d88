"""Race widening (SURVEY 4 layers 5-6): the parity of every commit design
re-checked under CSMV_DBG_JITTER -- each warp sleeps a seeded 0..2 us at
every protocol step that hands data to another warp or SM (doorbell,
response poll, write-back, GTS publish, receiver sweep, payload load, lock
entry, the KV workers' e_pre -> lastw window, the committer, the publisher)
-- so that orderings the ordering argument of P:113-116 relies on are
exercised far from the schedule a quiet run takes.  The oracle replays every
committed transaction.  Plus the negative control for client
pre-validation: without it, conflicting transactions of one batch
commit together and the oracle must reject the history."""
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_kv import as_state, ocfg_of, run as run_kv  # noqa: E402
from tests.test_gpu_parity import check  # noqa: E402

J = csmv.DBG_JITTER


@pytest.mark.parametrize("name,kw", [
    ("lock+publisher", dict(publish=csmv.PUBLISH_SERVER, ro_streak=8, server_workers=6, server_combine=8,
                            ro_adaptive=1)),
    ("lock+client-chain", dict(publish=csmv.PUBLISH_CLIENT, ro_streak=8, server_workers=6, server_combine=4)),
    ("self-receiving", dict(publish=csmv.PUBLISH_CLIENT, server_recv=csmv.RECV_SELF, server_workers=7,
                            server_combine=2)),
    ("commit-ring one CTA", dict(publish=csmv.PUBLISH_SERVER, debug_flags=csmv.DBG_ALT_COMMIT, server_workers=4)),
    ("cluster-4 ring", dict(publish=csmv.PUBLISH_SERVER, server=csmv.SERVER_CLUSTER, cluster_size=4)),
    ("cluster-2 lock", dict(publish=csmv.PUBLISH_CLIENT, server=csmv.SERVER_CLUSTER, cluster_size=2,
                            debug_flags=csmv.DBG_ALT_COMMIT)),
    ("list ATR", dict(atr_mode=csmv.ATR_LIST, server_combine=2)),
    ("list ATR NoCV", dict(atr_mode=csmv.ATR_LIST_NOCV)),
    ("grouped G=4", dict(publish=csmv.PUBLISH_SERVER, client_group=4, ro_streak=8, server_workers=6,
                         server_combine=8, ro_adaptive=1)),
    ("self-receiving tagged requests", dict(publish=csmv.PUBLISH_CLIENT, server_recv=csmv.RECV_SELF,
                                            server_workers=7, server_combine=2, req_tagged=1)),
    ("self-receiving tagged, publisher", dict(publish=csmv.PUBLISH_SERVER, server_recv=csmv.RECV_SELF,
                                              server_workers=6, server_combine=4, ro_adaptive=1, req_tagged=1)),
    ("onlyCS", dict(commit=csmv.COMMIT_ONLYCS)),
    ("JVSTM-GPU", dict(commit=csmv.COMMIT_JVSTM)),
])
def test_bank_c2_shrunk_under_jitter(name, kw):
    kw = dict(kw)
    flags = kw.pop("debug_flags", 0) | J
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 16, client_warps=256, debug_flags=flags, **kw)
    rep, stats, *_ = check(cfg)
    assert stats["committed"] == cfg.n_tx, name


@pytest.mark.parametrize("server", [csmv.SERVER_CTA, csmv.SERVER_CLUSTER])
def test_bank_c3_hot_set_under_jitter(server):
    """Zipf 0.99 over 4,096 accounts: every hot transfer chains on the last."""
    cfg = W.c3(n_tx=1 << 16, client_warps=128, server=server, cluster_size=4, debug_flags=J,
               ro_streak=4, server_combine=2)
    check(cfg)


def test_bank_c1_full_log_under_jitter():
    """C1 with a FULL log: every value every committed transaction read."""
    check(W.c1(debug_flags=J))


@pytest.mark.parametrize("server,flags", [(csmv.SERVER_CTA, 0), (csmv.SERVER_CTA, csmv.DBG_KV_ITEMSETS),
                                          (csmv.SERVER_CLUSTER, 0), (csmv.SERVER_CLUSTER, csmv.DBG_KV_ITEMSETS),
                                          (csmv.SERVER_CTA, csmv.DBG_KV_SEQREAD)])
@pytest.mark.parametrize("tagged", [0, 1])
@pytest.mark.parametrize("p_update", [10_000, 300_000])
def test_kv_c4_shrunk_under_jitter(server, flags, p_update, tagged):
    """KV workers read e_pre = tail outside the lock and then load lastw: the
    jitter sits exactly in that window (cs_leave's fence covers it)."""
    cfg = W.c4(n_items=1 << 12, n_tx=1 << 15, p_update_ppm=p_update, ro_streak=4, client_warps=192,
               server_workers=6, server=server, cluster_size=4, debug_flags=flags | J, req_tagged=tagged)
    pre, stats, log, fin = run_kv(cfg)
    oc = ocfg_of(cfg)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), d, log, final=as_state(fin, cfg.n_items, cfg.workload.kv_ways),
                          claims=dict(committed_update=stats["committed_update"],
                                      committed_ro=stats["committed_ro"], gts_final=stats["gts_final"],
                                      total_aborts=stats["total_aborts"]))
    assert rep["ok"], (rep, stats)


def test_jitter_is_on():
    """The flag really slows the protocol down (it is not a silent no-op)."""
    cfg = W.c2(n_items=1 << 14, n_tx=1 << 16, client_warps=256)
    _, quiet, *_ = check(cfg)
    _, jit, *_ = check(cfg.with_(debug_flags=J))
    assert jit["elapsed_ns"] > 1.2 * quiet["elapsed_ns"], (quiet["elapsed_ns"], jit["elapsed_ns"])


@pytest.mark.parametrize("jitter", [0, J])
def test_no_preval_is_caught(jitter):
    """Negative control for P:118: the server validates a batch's lanes in
    parallel against earlier commits only, so without client pre-validation
    two conflicting transfers of one batch both commit and the replay must
    find a read of a version overwritten after the snapshot."""
    cfg = W.c1(n_items=256, n_tx=4000, debug_flags=csmv.DBG_NO_PREVAL | jitter)
    rep, stats, *_ = check(cfg, expect_ok=False)
    assert not rep["ok"], stats
    assert stats["aborts"]["preval"]["update"] == 0
