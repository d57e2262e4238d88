"""Exploration helper: run a preset with overrides and print stats as JSON.
usage: python tools/probe.py C2 n_tx=1048576 client_warps=512 publish=1 [reps=3]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402


def main(argv):
    name = argv[0]
    kw = {}
    reps = 1
    for a in argv[1:]:
        k, v = a.split("=")
        if k == "reps":
            reps = int(v)
        else:
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
            t = time.time()
            s = st.run(cfg.workload, cfg.n_tx, cfg.seed + r)
            s["wall_s"] = time.time() - t
            out = {k: s[k] for k in ("committed", "committed_update", "tx_per_s", "abort_rate",
                                     "batches", "rounds", "elapsed_ns", "client_warps",
                                     "server_lock_cycles", "server_busy_cycles", "wall_s")}
            b = max(1, s["batches"])
            out["phase_per_batch"] = {k: v // max(1, s["server_groups"]) for k, v in s["server_phase_cycles"].items()}
            out["aborts"] = {k: v for k, v in s["aborts"].items() if v["ro"] or v["update"]}
            out["cfg"] = dict(name=name, **kw)
            print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
