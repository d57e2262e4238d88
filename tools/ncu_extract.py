"""Summarise ncu captures of csmv_fused into profiles/ncu_summary.json.

usage: python tools/ncu_extract.py CONFIG RAW.csv CAPTURE_DESCRIPTION [N_TX]
  RAW.csv  = `ncu -i X.ncu-rep --page raw --csv` of a capture of one timed
             bench.py step (tools/gpu_profile.sh).
Writes/updates the entry `CONFIG` (c2, c3, c4) with per-launch counters:
duration, DRAM bytes (the contract's `traffic`), L2 bytes requested, L2
atomic/reduction sectors (the commit path should have ~none) and shared
atomics (the server's).  bench.py reads these to put the roofline's
`traffic`, `l2_traffic` and `server_smem_atomics` on the bench line.
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles", "ncu_summary.json")

WANT = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_bytes_read",
    "dram__bytes_write.sum": "dram_bytes_write",
    "lts__t_bytes.sum": "l2_bytes_per_launch",
    "lts__t_sectors_op_atom.sum": "l2_atomic_sectors",
    "lts__t_sectors_op_red.sum": "l2_reduction_sectors",
    "sm__sass_inst_executed_op_shared_atom.sum": "shared_atomics_per_launch",
    "launch__registers_per_thread": "registers_per_thread",
    "launch__grid_size": "grid_ctas",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
}


def num(x):
    x = x.replace(",", "")
    try:
        return float(x)
    except ValueError:
        return None


def parse(path):
    rows = list(csv.reader(open(path)))
    head = rows[0]
    units = rows[1] if len(rows) > 1 and rows[1] and rows[1][0] == "" else None
    data = [r for r in rows[1 + (units is not None):] if len(r) == len(head)]
    out = []
    for r in data:
        d = dict(zip(head, r))
        if "csmv_fused" not in d.get("Kernel Name", ""):
            continue
        e = {"kernel": d.get("Kernel Name")}
        for m, k in WANT.items():
            if m in d:
                v = num(d[m])
                if v is None:
                    continue
                u = units[head.index(m)] if units else ""
                if m == "gpu__time_duration.sum":
                    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "msecond": 1.0, "ms": 1.0, "s": 1e3,
                             "nsecond": 1e-6, "second": 1e3}.get(u, 1e-6)
                    e["duration_ms"] = v * scale
                elif "bytes" in m:
                    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6,
                             "GB": 1e9}.get(u, 1)
                    e[k] = v * scale
                else:
                    e[k] = v
        if "dram_bytes_read" in e and "dram_bytes_write" in e:
            e["dram_bytes_per_launch"] = e["dram_bytes_read"] + e["dram_bytes_write"]
        out.append(e)
    return out


def main():
    cfg, path, desc = sys.argv[1].lower(), sys.argv[2], sys.argv[3]
    n_tx = int(sys.argv[4]) if len(sys.argv) > 4 else 1 << 24
    launches = parse(path)
    if not launches:
        sys.exit(f"no csmv_fused launch in {path}")
    e = launches[-1]
    e["capture"] = desc
    e["raw_csv"] = os.path.relpath(path, ROOT)
    e["n_tx_per_launch"] = n_tx
    d = json.load(open(OUT)) if os.path.exists(OUT) else {}
    d[cfg] = e
    json.dump(d, open(OUT, "w"), indent=1, sort_keys=True)
    print(json.dumps(e, indent=1))


if __name__ == "__main__":
    main()
