"""Sweep of the item-partitioned servers (CSMV_SERVER_PART) against the tuned
single-CTA launch on full-size presets: python tools/part_perf.py C2,C3
(profiles/r02/part_perf.txt)."""
import sys
sys.path.insert(0, '.')
from paper_conf_ipps_nunesc022_b200 import csmv, workloads as W
import bench
names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C2", "C3"]
for name in names:
    t = bench.tuned(name)
    cfg0 = W.PRESETS[name]().with_(log_mode=0, ro_streak=t["ro_streak"], publish=t["publish"], server_workers=t["server_workers"],
                                  server_combine=t["server_combine"], ro_adaptive=t["ro_adaptive"], server_recv=t["server_recv"],
                                  client_group=t["client_group"], backoff_max=t.get("backoff_max", 0))
    for srv in [None, 2, 4, 8]:
        for wpsm in ([t["client_warps_per_sm"]] if not srv else [2, 4]):
            for pub in ([t["publish"]] if not srv else [0, 1]):
                cfg = cfg0.with_(client_warps=wpsm * (148 - (srv or 1)))
                if srv:
                    cfg = cfg.with_(server=csmv.SERVER_PART, cluster_size=srv, client_group=1, server_recv=0, publish=pub,
                                    server_workers=7 if pub == 0 else 6)
                try:
                    with csmv.Store(cfg.n_items, cfg.n_versions) as st:
                        st.load(cfg.init_values())
                        best, ab = 0, 0
                        for rep in range(3):
                            st.run(cfg.workload, cfg.n_tx, cfg.seed)
                            s = st.stats()
                            if s["tx_per_s"] > best:
                                best, ab = s["tx_per_s"], s["abort_rate"]
                        print(name, "part" if srv else "cta", srv, "wpsm", wpsm, "pub", pub, f"{best/1e6:.1f} M tx/s abort {ab:.3f}", flush=True)
                except Exception as e:
                    print(name, srv, wpsm, pub, "ERR", str(e)[:150], flush=True)
