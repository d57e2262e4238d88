"""Hot-item commit chain (CSMV_DBG_TRACE): every committed writer of the
traced item (bank account 0 / the KV set of key 0, zipf rank 0) logs its
CTS, snapshot and device-wide timestamps.  Consecutive writers form the
chain the paper's ordering implies (the next writer's
snapshot must include the previous commit).  Per link i -> i+1 this prints
the median of
  link      t_response(i+1) - t_response(i)
  publish   t_publish(i) - t_response(i)          write-back + publish of i
  restart   t_begin(i+1) - t_publish(i)           until the next winner's round starts
  read      t_submit(i+1) - t_begin(i+1)          its snapshot + reads + pre-validation
  server    t_response(i+1) - t_submit(i+1)       request -> response, split by the
            server's stamps into to_claim (doorbell -> a worker took it),
            worker (claim -> response stored), to_client (-> client saw it)
(restart can be negative: the winner's round began before i was
published, e.g. when GTS was advanced by the server publisher meanwhile).

usage: python tools/chain.py C3|C4 [key=value ...]
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402

def base(name: str) -> dict:
    """bench.py's tuned launch of the config (so a trace describes the benchmarked run)."""
    import bench
    t = dict(bench.tuned(name))
    return dict({k: v for k, v in t.items() if k != "client_warps_per_sm"},
                client_warps=t["client_warps_per_sm"] * 147)


def main(argv):
    kw = base(argv[0])
    kw.update({k: int(v) for k, v in (a.split("=") for a in argv[1:])})
    kw["debug_flags"] = kw.get("debug_flags", 0) | csmv.DBG_TRACE
    cfg = workloads.PRESETS[argv[0]](**kw)
    if cfg.workload.kind == csmv.KIND_KV:
        st = csmv.KvStore(cfg.n_items, cfg.workload.kv_ways, cfg.n_versions)
        st.load(cfg.workload.kv_keys)
    else:
        st = csmv.Store(cfg.n_items, cfg.n_versions)
        st.load(cfg.init_values())
    with st:
        s = st.run(cfg.workload, cfg.n_tx, cfg.seed)
        tr = st.trace()
    tr = np.sort(tr, order="cts")
    f = lambda a: float(np.median(a)) / 1e3 if len(a) else None  # noqa: E731
    r, p, b, sub, tc, tv, tsn, trd = (tr[k].astype(np.int64) for k in (
        "t_response", "t_publish", "t_begin", "t_submit", "t_claim", "t_served", "t_snap", "t_read"))
    okc = (tsn >= b) & (trd >= tsn) & (sub >= trd)  # client stamps present
    ok = (tc > 0) & (tv >= tc) & (tc >= sub - 1000) & (tv <= r)  # server stamps present and consistent
    out = {"cfg": argv, "tx_per_s_M": round(s["tx_per_s"] / 1e6, 2), "kernel_ms": s["elapsed_ns"] / 1e6,
           "hot_commits": int(len(tr)), "span_ms": float((r[-1] - r[0]) / 1e6) if len(tr) > 1 else None,
           "median_us": {"link": f(np.diff(r)), "publish": f(p - r), "restart": f(b[1:] - p[:-1]),
                         "read": f(sub - b), "server": f(r - sub)},
           "server_us": {"stamped": int(ok.sum()), "to_claim": f((tc - sub)[ok]), "worker": f((tv - tc)[ok]),
                         "to_client": f((r - tv)[ok])},
           "read_us": {"stamped": int(okc.sum()), "snapshot": f((tsn - b)[okc]), "reads": f((trd - tsn)[okc]),
                       "submit": f((sub - trd)[okc])},
           "readers_mean": float(np.mean(tr["n_readers"])) if len(tr) else None,
           "kept_mean": float(np.mean(tr["n_kept"])) if len(tr) else None,
           "mean_link_us": float(np.mean(np.diff(r))) / 1e3 if len(tr) > 1 else None,
           "snapshot_lag_median": float(np.median(tr["cts"][1:].astype(np.int64) - tr["snapshot"][1:]))
           if len(tr) > 1 else None}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
