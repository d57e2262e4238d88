"""Tuning sweep on one preset: every argument is a comma-separated override
set; each runs `reps` times in one process (store reloaded per set).
usage: python tools/tune.py C2 reps=2 "ro_adaptive=1" "server_workers=4,server_combine=4" ..."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402

BASE = dict(client_warps=294, publish=1, server_workers=6, server_combine=8, ro_streak=8, ro_adaptive=1, log_mode=0)


def main(argv):
    name, reps, sets = argv[0], 2, []
    for a in argv[1:]:
        if a.startswith("reps="):
            reps = int(a[5:])
        else:
            sets.append(a)
    for s in sets or [""]:
        kw = dict(BASE)
        for kv in filter(None, s.split(",")):
            k, v = kv.split("=")
            kw[k] = int(v)
        cfg = workloads.PRESETS[name](**kw)
        if cfg.workload.kind == csmv.KIND_KV:
            st = csmv.KvStore(cfg.n_items, cfg.workload.kv_ways, cfg.n_versions)
            st.load(cfg.workload.kv_keys)
        else:
            st = csmv.Store(cfg.n_items, cfg.n_versions)
            st.load(cfg.init_values())
        with st:
            for r in range(reps):
                x = st.run(cfg.workload, cfg.n_tx, cfg.seed + r)
                ab = {k: v["update"] + v["ro"] for k, v in x["aborts"].items() if v["ro"] or v["update"]}
                ph = {k: v // max(1, x["server_groups"]) for k, v in x["server_phase_cycles"].items()}
                print(json.dumps({"set": s, "Mtx_s": round(x["tx_per_s"] / 1e6, 1),
                                  "abort": round(x["abort_rate"], 4), "upd_per_batch":
                                  round(x["committed_update"] / max(1, x["batches"]), 1),
                                  "aborts": ab, "crit": ph.get("critical"), "lockw": ph.get("lock_wait"),
                                  "srv": ph, "client_us_per_round": {k: round(v / max(1, x["rounds"]) / 1965, 2)
                                                                     for k, v in x["client_phase_cycles"].items() if v}}),
                      flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
