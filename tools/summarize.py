"""Turn the JSONL output of tools/ablation.py, tools/kv_ways.py and
tools/sweep_c5.py into the markdown tables kept under profiles/.

usage: python tools/summarize.py ablation|kv_ways|c5 FILE.jsonl [> out.md]
"""
import json
import sys


def rows(path):
    return [json.loads(line) for line in open(path) if line.strip()]


def fmt_rate(x):
    return f"{x / 1e6:.3g} M" if x >= 1e5 else f"{x / 1e3:.3g} k"


def ablation(path):
    rs = rows(path)
    variants = list(dict.fromkeys(r["variant"] for r in rs))
    ros = sorted({r["ro_pct"] for r in rs})
    print("committed tx/s (parity of a 16K-tx DIGEST run vs the oracle: ok / FAIL / -)\n")
    print("| % ROT | " + " | ".join(variants) + " |")
    print("|---|" + "---|" * len(variants))
    for ro in ros:
        cells = []
        for v in variants:
            r = next((x for x in rs if x["variant"] == v and x["ro_pct"] == ro), None)
            if r is None:
                cells.append("")
            elif "error" in r:
                cells.append("timeout" if "watchdog" in r["error"] else "error")
            else:
                par = {True: "ok", False: "FAIL"}.get(r.get("parity"), "-")
                cells.append(f"{fmt_rate(r['tx_per_s'])} ({par}, abort {r['abort_rate']:.2f})")
        print(f"| {ro} | " + " | ".join(cells) + " |")


def kv_ways(path):
    rs = rows(path)
    print("| ways | tx/s | abort rate | parity | client cycles/round: read, preval, submit, GETs, wait server, "
          "write-back, publish | server cycles/batch: load, lock wait, critical, respond |")
    print("|---|---|---|---|---|---|")
    for r in rs:
        if "error" in r:
            print(f"| {r['ways']} | error: {r['error'][:60]} | | | | |")
            continue
        c = r.get("client_cycles_per_round", {})
        s = r.get("server_cycles_per_batch", {})
        cc = ", ".join(f"{c.get(k, 0):.0f}" for k in ("read", "preval", "submit", "rot", "wait_server",
                                                      "writeback", "publish"))
        ss = ", ".join(f"{s.get(k, 0):.0f}" for k in ("load", "lock_wait", "critical", "respond"))
        par = {True: "ok", False: "FAIL"}.get(r.get("parity"), "-")
        print(f"| {r['ways']} | {fmt_rate(r['tx_per_s'])} | {r['abort_rate']:.3f} | {par} | {cc} | {ss} |")


def c5(path):
    rs = rows(path)
    ok = [r for r in rs if "error" not in r]
    n_par = sum(1 for r in ok if r.get("parity") is True)
    print(f"{len(rs)} points, {n_par} parity-ok, {len(rs) - len(ok)} errors\n")
    pairs = {}
    for r in ok:
        pairs.setdefault(r["name"][:-3], {})[r["server"]] = r.get("tx_per_s_mean", r["tx_per_s"])
    ratios = sorted(v["cluster"] / v["cta"] for v in pairs.values() if "cta" in v and "cluster" in v)
    if ratios:
        print(f"cluster/CTA throughput ratio over {len(ratios)} pairs: median {ratios[len(ratios) // 2]:.2f}, "
              f"min {ratios[0]:.2f}, max {ratios[-1]:.2f}\n")
    print("| point | items | K | update % | server | group | tx/s mean (min-max, seeds) | abort rate | parity |")
    print("|---|---|---|---|---|---|---|---|---|")
    for r in rs:
        if "error" in r:
            print(f"| {r['name']} | | | | | | error: {r['error'][:50]} | | |")
            continue
        par = {True: "ok", False: "FAIL"}.get(r.get("parity"), "-")
        mean = r.get("tx_per_s_mean", r["tx_per_s"])
        rng = f" ({fmt_rate(r['tx_per_s_min'])}-{fmt_rate(r['tx_per_s_max'])}, {len(r['seeds_timed'])})" \
            if "tx_per_s_min" in r else ""
        print(f"| {r['name']} | {r['n_items']} | {r['K']} | {r['p_update_ppm'] / 1e4:.0f} | "
              f"{r['server']}{'' if r['server'] == 'cta' else r['cluster_size']} | {r.get('client_group', 1)} | "
              f"{fmt_rate(mean)}{rng} | {r['abort_rate']:.3f} | {par} |")


if __name__ == "__main__":
    {"ablation": ablation, "kv_ways": kv_ways, "c5": c5}[sys.argv[1]](sys.argv[2])
