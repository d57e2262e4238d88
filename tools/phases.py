"""Client/server phase breakdown of one run (CSMV_DBG_PHASES): per client
round, cycles by phase (mean lane), and the server's per-group phases.
usage: python tools/phases.py C2 key=value ..."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402


def main(argv):
    kw = {k: int(v) for k, v in (a.split("=") for a in argv[1:])}
    kw["debug_flags"] = kw.get("debug_flags", 0) | csmv.DBG_PHASES
    cfg = workloads.PRESETS[argv[0]](**kw)
    if cfg.workload.kind == csmv.KIND_KV:
        st = csmv.KvStore(cfg.n_items, cfg.workload.kv_ways, cfg.n_versions)
        st.load(cfg.workload.kv_keys)
    else:
        st = csmv.Store(cfg.n_items, cfg.n_versions)
        st.load(cfg.init_values())
    with st:
        s = st.run(cfg.workload, cfg.n_tx, cfg.seed)
    rounds = max(1, s["rounds"])
    groups = max(1, s["server_groups"])
    out = {"cfg": argv, "tx_per_s_M": round(s["tx_per_s"] / 1e6, 1), "abort_rate": round(s["abort_rate"], 4),
           "rounds": rounds, "batches": s["batches"], "updates_per_batch": round(s["committed_update"] / max(1, s["batches"]), 2),
           "client_cycles_per_round": {k: round(v / rounds) for k, v in s["client_phase_cycles"].items()},
           "server_cycles_per_group": {k: round(v / groups) for k, v in s["server_phase_cycles"].items() if v},
           "kernel_ms": round(s["elapsed_ns"] / 1e6, 2), "client_warps": s["client_warps"]}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
