"""C5 sweep (BASELINE.json configs[4]): update rate 10-90% x contention
(1K-16M items) x K = 2/4/8 versions x single-SM vs cluster server.

For every point (SURVEY 8(d) protocol): one DIGEST-logged run (seed 1)
checked element by element against the CPU oracle (--check), then timed runs
without logging for seeds 1..--seeds (mean, min, max of tx/s).  The launch
is bench.py's tuned one scaled to the point: client warps = max(16,
min(588, N/64)) so that in-flight updates stay well below the item count
(Q29), in CTA-level groups of 4 when a CTA hosts at least two client warps
(both servers: the cluster's commit ring takes grouped requests).  Writes
one JSON line per point.

usage: python tools/sweep_c5.py [--n-tx N] [--check] [--seeds 3] [--out FILE] [--servers 0,1]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402

TUNED = dict(server_workers=7, server_combine=8, ro_streak=2, ro_adaptive=0, publish=csmv.PUBLISH_SERVER)  # bench.py's C2 launch


def run_point(cfg, check: bool, seeds: int):
    import numpy as np
    w = cfg.workload
    out = {"name": cfg.name, "n_items": cfg.n_items, "K": cfg.n_versions, "p_update_ppm": w.p_update_ppm,
           "server": ["cta", "cluster"][w.server], "cluster_size": w.cluster_size if w.server else 1}
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        init = cfg.init_values()
        if check:
            import oracle
            st.load(init)
            s = st.run(w, cfg.n_tx, cfg.seed)
            log = st.log(cfg.n_tx)
            rings = st.dump()
            ocfg = oracle.bank_cfg(cfg.n_items, cfg.n_versions, dist=w.dist, p_update_ppm=w.p_update_ppm,
                                   ro_reads=w.ro_reads, amount_max=w.amount_max, ro_streak=w.ro_streak)
            descs = oracle.bank_gen(ocfg, cfg.seed, cfg.n_tx)
            rep = oracle.bank_check(ocfg, init, descs, log, rings=rings,
                                    claims=dict(committed_update=s["committed_update"], committed_ro=s["committed_ro"],
                                                gts_final=s["gts_final"], total_aborts=s["total_aborts"]))
            out["parity"] = rep["ok"]
            out["oracle_s"] = rep["seconds"]
            if not rep["ok"]:
                out["parity_msg"] = rep["msg"]
        rates, last = [], None
        for sd in range(1, seeds + 1):
            st.load(init)
            wt = workloads.Config(cfg.name, cfg.n_items, cfg.n_versions, cfg.workload, cfg.n_tx, sd).with_(log_mode=0)
            last = st.run(wt.workload, cfg.n_tx, sd)
            rates.append(last["tx_per_s"])
    s = last
    out["tx_per_s_mean"], out["tx_per_s_min"], out["tx_per_s_max"] = sum(rates) / len(rates), min(rates), max(rates)
    out["seeds_timed"] = list(range(1, seeds + 1))
    for k in ("tx_per_s", "abort_rate", "committed_update", "committed_ro", "batches", "server_ctas", "client_warps",
              "elapsed_ns"):
        out[k] = s[k]
    out["aborts"] = {k: v for k, v in s["aborts"].items() if v["ro"] or v["update"]}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-tx", type=int, default=1 << 22)
    ap.add_argument("--seeds", type=int, default=3)
    ap.add_argument("--check", action="store_true")
    ap.add_argument("--out", default="")
    ap.add_argument("--servers", default="0,1")
    ap.add_argument("--cluster-size", type=int, default=16)
    args = ap.parse_args()
    servers = tuple(int(x) for x in args.servers.split(","))
    f = open(args.out, "w") if args.out else None
    for cfg in workloads.c5_points(args.n_tx, servers=servers):
        single = cfg.workload.server == csmv.SERVER_CTA
        cw = max(16, min(588, cfg.n_items // 64))  # in-flight updates << items (Q29)
        group = 4 if cw >= 296 else 1  # CTA-level batches (the commit ring takes them too)
        cfg = cfg.with_(cluster_size=args.cluster_size, watchdog_ms=60_000, client_group=group,
                        **dict(TUNED, client_warps=cw))
        try:
            r = run_point(cfg, args.check, args.seeds)
            r["client_group"] = group
        except Exception as e:  # report and continue the sweep
            r = {"name": cfg.name, "error": str(e)}
        line = json.dumps(r)
        print(line, flush=True)
        if f:
            f.write(line + "\n")
            f.flush()


if __name__ == "__main__":
    main()
