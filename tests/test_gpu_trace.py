"""CSMV_DBG_TRACE (tools/chain.py): the traced records are exactly the
committed writers of the traced item -- the CTS set equals the one the
DIGEST log and the regenerated descriptors give (bank: account 0; KV: the
set of key 0) -- with ordered timestamps, and tracing keeps parity."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu

csmv = pytest.importorskip("paper_conf_ipps_nunesc022_b200.csmv")
from paper_conf_ipps_nunesc022_b200 import workloads as W  # noqa: E402
from tests.test_gpu_kv import ocfg_of  # noqa: E402
from tests.test_gpu_parity import oracle_cfg  # noqa: E402


def check_times(tr):
    assert np.all(tr["t_begin"] <= tr["t_submit"]) and np.all(tr["t_submit"] <= tr["t_response"])
    assert np.all(tr["t_response"] <= tr["t_publish"])
    assert np.all(tr["snapshot"] < tr["cts"])


@pytest.mark.parametrize("server_recv,publish", [(0, 1), (1, 0)])
def test_bank_trace_is_the_hot_account_chain(server_recv, publish):
    cfg = W.c3(n_tx=1 << 16, client_warps=256, server_recv=server_recv, publish=publish, ro_streak=4,
               server_combine=2, server_workers=7 if server_recv else 6, debug_flags=csmv.DBG_TRACE)
    init = cfg.init_values()
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        st.load(init)
        st.run(cfg.workload, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx)
        tr = st.trace()
    d = oracle.bank_gen(oracle_cfg(cfg), cfg.seed, cfg.n_tx)
    hot = (d["is_update"] == 1) & ((d["src"] == 0) | (d["dst"] == 0))
    assert sorted(tr["cts"].tolist()) == sorted(log["cts"][hot].tolist())
    check_times(tr)


def test_kv_trace_is_the_hot_set_chain():
    cfg = W.c4(n_items=1 << 14, n_tx=1 << 17, p_update_ppm=50_000, ro_streak=8, client_warps=256,
               debug_flags=csmv.DBG_TRACE)
    w = cfg.workload
    with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
        st.load(w.kv_keys)
        st.run(w, cfg.n_tx, cfg.seed)
        log = st.log(cfg.n_tx)
        tr = st.trace()
    oc = ocfg_of(cfg)
    d = oracle.kv_gen(oc, cfg.seed, cfg.n_tx)
    T = cfg.n_items // w.kv_ways
    t0 = oracle.kv_set(0, T)
    upd = np.nonzero(d["is_update"] == 1)[0]
    hot = np.zeros(len(d), dtype=bool)
    hot[[i for i in upd if oracle.kv_set(int(d["key"][i]), T) == t0]] = True
    assert hot.sum() > 0
    assert sorted(tr["cts"].tolist()) == sorted(log["cts"][hot].tolist())
    check_times(tr)
