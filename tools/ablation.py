"""Commit-design ablation on the paper's Bank setting (Fig. 2 / Fig. 4,
P:232-281): 6,000 accounts, read-only transactions
that sum every account, % read-only in {1, 10, 50, 90, 99}, for

  csmv-b200   this build's defaults (item-indexed ATR, ROT streaming,
              combining, server publisher)
  csmv        the paper's CSMV: list ATR + collaborative validation, one
              batch per critical section, one tx per lane per round,
              client publish chain
  nocv        CSMV-NoCV: as csmv, one lane scans per transaction
  onlycs      CSMV-onlyCS: NoCV without batched insert, client
              pre-validation and client write-back
  jvstm       JVSTM-GPU: decentralized per-thread commit over a
              global-memory ATR and a global CAS

Each point: optionally one DIGEST-logged run checked by the CPU oracle
(--check, small n_tx), then one timed run.  One JSON line per point.

usage: python tools/ablation.py [--n-tx N] [--check] [--out FILE] [--warps W]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ipps_nunesc022_b200 import csmv, workloads  # noqa: E402

VARIANTS = {
    "csmv-b200": dict(atr_mode=csmv.ATR_HASH, server_combine=8, server_workers=7, ro_streak=2, ro_adaptive=0,
                      publish=csmv.PUBLISH_SERVER),  # bench.py's C2 launch (per-warp batches)
    "csmv": dict(atr_mode=csmv.ATR_LIST, server_combine=1, ro_streak=0, publish=csmv.PUBLISH_CLIENT),
    "nocv": dict(atr_mode=csmv.ATR_LIST_NOCV, server_combine=1, ro_streak=0, publish=csmv.PUBLISH_CLIENT),
    "onlycs": dict(commit=csmv.COMMIT_ONLYCS, ro_streak=0, publish=csmv.PUBLISH_CLIENT),
    "jvstm": dict(commit=csmv.COMMIT_JVSTM, ro_streak=0, publish=csmv.PUBLISH_CLIENT),
}
RO_PCT = (1, 10, 50, 90, 99)


def bank_6k(ro_pct: int, n_tx: int, warps: int, **kw) -> workloads.Config:
    """P:183 / Fig. 2: 6k accounts, total-sum ROTs, uniform transfers."""
    return workloads.c2(n_items=6000, n_versions=4, n_tx=n_tx, ro_reads=0,
                        p_update_ppm=(100 - ro_pct) * 10_000, client_warps=warps,
                        watchdog_ms=120_000, **kw).with_(name=f"bank6k-ro{ro_pct}")


def run_point(cfg, check: bool):
    w = cfg.workload
    out = {}
    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
        init = cfg.init_values()
        if check:
            import oracle
            n_chk = min(cfg.n_tx, 1 << 14)
            st.load(init)
            s = st.run(w, n_chk, cfg.seed)
            log = st.log(n_chk)
            rings = st.dump()
            ocfg = oracle.bank_cfg(cfg.n_items, cfg.n_versions, dist=w.dist, p_update_ppm=w.p_update_ppm,
                                   ro_reads=w.ro_reads, amount_max=w.amount_max, ro_streak=w.ro_streak)
            descs = oracle.bank_gen(ocfg, cfg.seed, n_chk)
            rep = oracle.bank_check(ocfg, init, descs, log, rings=rings,
                                    claims=dict(committed_update=s["committed_update"],
                                                committed_ro=s["committed_ro"], gts_final=s["gts_final"],
                                                total_aborts=s["total_aborts"]))
            out["parity"] = rep["ok"]
            out["parity_n_tx"] = n_chk
            if not rep["ok"]:
                out["parity_msg"] = rep["msg"]
        st.load(init)
        wt = cfg.with_(log_mode=csmv.LOG_NONE).workload
        s = st.run(wt, cfg.n_tx, cfg.seed + 1)
    for k in ("tx_per_s", "abort_rate", "committed_update", "committed_ro", "batches", "client_warps",
              "elapsed_ns", "cas_failures"):
        out[k] = s[k]
    out["aborts"] = {k: v for k, v in s["aborts"].items() if v["ro"] or v["update"]}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-tx", type=int, default=1 << 18)
    ap.add_argument("--reads", type=float, default=2e8, help="item-read budget per point (caps n_tx)")
    ap.add_argument("--warps", type=int, default=0, help="client warps (0 = full grid)")
    ap.add_argument("--check", action="store_true")
    ap.add_argument("--out", default="")
    ap.add_argument("--variants", default=",".join(VARIANTS))
    ap.add_argument("--ro", default=",".join(map(str, RO_PCT)))
    args = ap.parse_args()
    f = open(args.out, "w") if args.out else None
    for ro in (int(x) for x in args.ro.split(",")):
        for name in args.variants.split(","):
            n_tx = int(min(args.n_tx, args.reads / (2 + ro / 100 * 6000)))
            cfg = bank_6k(ro, n_tx, args.warps, **VARIANTS[name])
            try:
                r = run_point(cfg, args.check)
            except Exception as e:  # report and continue
                r = {"error": str(e)}
            r = dict({"variant": name, "ro_pct": ro, "n_items": cfg.n_items, "n_tx": cfg.n_tx}, **r)
            line = json.dumps(r)
            print(line, flush=True)
            if f:
                f.write(line + "\n")
                f.flush()


if __name__ == "__main__":
    main()
