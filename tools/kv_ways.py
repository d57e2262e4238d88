"""MemcachedGPU associativity sweep (Fig. 3 / Tables III-IV shape, P:189-214,
P:250-258): 1M-slot cache, 1M zipf(0.99) keys, 99.8%
GET, ways 4..256.  Per point: an optional DIGEST-logged run checked by the
CPU oracle (--check, small n_tx), a timed run, and a CSMV_DBG_PHASES run
giving the per-phase client and server cycle breakdown per committed PUT /
per transaction.

usage: python tools/kv_ways.py [--n-tx N] [--check] [--out FILE] [--ways 4,8,...]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402

WAYS = (4, 8, 16, 32, 64, 128, 256)
TUNED = dict(server_workers=6, ro_streak=32, ro_adaptive=2, backoff_max=16, req_tagged=1, client_warps=294,
             publish=csmv.PUBLISH_SERVER)  # bench.py's C4 launch


def cfg_for(ways: int, n_tx: int, slots: int, **kw):
    return workloads.c4(n_items=slots, kv_ways=ways, kv_keys=slots, p_update_ppm=2_000, n_tx=n_tx,
                        watchdog_ms=120_000, **dict(TUNED, **kw)).with_(name=f"kv-{ways}w")


def one(cfg, seed, flags=0):
    w = cfg.with_(log_mode=csmv.LOG_NONE, debug_flags=flags).workload
    with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
        st.load(w.kv_keys)
        return st.run(w, cfg.n_tx, seed)


def check(cfg, n_chk):
    import oracle
    w = cfg.workload
    oc = oracle.kv_cfg(cfg.n_items, w.kv_ways, n_keys=w.kv_keys, n_versions=cfg.n_versions, dist=w.dist,
                       zipf_theta_milli=w.zipf_theta_milli, p_update_ppm=w.p_update_ppm, ro_streak=w.ro_streak)
    with csmv.KvStore(cfg.n_items, w.kv_ways, cfg.n_versions) as st:
        st.load(w.kv_keys)
        s = st.run(w, n_chk, cfg.seed)
        log = st.log(n_chk)
        fin = st.dump()
    final = oracle.KvStore(cfg.n_items, w.kv_ways)
    final.keys[:], final.vals[:], final.lru[:], final.clocks[:] = fin
    rep = oracle.kv_check(oc, oracle.kv_preload(oc), oracle.kv_gen(oc, cfg.seed, n_chk), log, final=final,
                          claims=dict(committed_update=s["committed_update"], committed_ro=s["committed_ro"],
                                      gts_final=s["gts_final"], total_aborts=s["total_aborts"]))
    return rep


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-tx", type=int, default=1 << 22)
    ap.add_argument("--slots", type=int, default=1 << 20)
    ap.add_argument("--ways", default=",".join(map(str, WAYS)))
    ap.add_argument("--check", action="store_true")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    f = open(args.out, "w") if args.out else None
    for a in (int(x) for x in args.ways.split(",")):
        cfg = cfg_for(a, args.n_tx, args.slots)
        r = {"ways": a, "slots": args.slots, "n_tx": args.n_tx, "p_update_ppm": cfg.workload.p_update_ppm}
        try:
            if args.check:
                rep = check(cfg, 1 << 16)
                r["parity"] = rep["ok"]
                if not rep["ok"]:
                    r["parity_msg"] = rep["msg"]
            s = one(cfg, cfg.seed + 1)
            for k in ("tx_per_s", "abort_rate", "committed_update", "committed_ro", "batches", "elapsed_ns",
                      "client_warps"):
                r[k] = s[k]
            r["aborts"] = {k: v for k, v in s["aborts"].items() if v["ro"] or v["update"]}
            sp = one(cfg, cfg.seed + 1, csmv.DBG_PHASES)
            rounds = max(1, sp["rounds"])
            r["phases_tx_per_s"] = sp["tx_per_s"]
            r["client_cycles_per_round"] = {k: v / rounds for k, v in sp["client_phase_cycles"].items()}
            g = max(1, sp["server_groups"])
            r["server_cycles_per_batch"] = {k: v / g for k, v in sp["server_phase_cycles"].items()}
            r["rounds"] = sp["rounds"]
        except Exception as e:  # report and continue
            r["error"] = str(e)
        line = json.dumps(r)
        print(line, flush=True)
        if f:
            f.write(line + "\n")
            f.flush()


if __name__ == "__main__":
    main()
