#!/usr/bin/env python
"""Benchmark: committed transactions/s and abort rate of the CSMV batched
commit pipeline (BASELINE.json metric) on the config it is quoted on,
configs[1] = C2: bank, 1M accounts, K=4 versions, full-GPU client grid, 50%
update, uniform access, read-only = 64-read scans.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config C2|C3|C4|C1]

A step is one csmv_run over n_tx = 2^24 freshly generated transactions
(every one commits exactly once; aborted attempts are retried inside the
step).  The store and GTS persist across steps.  L2 is flushed (a 512 MiB
write) before every timed step.

--gpus N > 1 runs one process per GPU (torchrun; bench.py spawns it itself
when started without one) as independent key-range-partitioned instances:
rank g runs the full per-GPU workload on its own key range of an N x larger
job (weak scaling), its own server and GTS, no cross-GPU transactions; NCCL
only reduces the statistics.

--impl reference times the CPU oracle (the deterministic 1-warp schedule of
oracle/, single-threaded C) on bounded samples of the same workload: the
tier's reference arm is the oracle, there is no GPU reference to install.

Roofs: the measured L2 / cross-SM / shared-atomic roofs of
tools/ubench/roofs.cu and the critical-section chain floor of
tools/ubench/filt16_ubench.cu are read from profiles/roofs_b200.json; the
per-launch DRAM / L2 bytes and shared atomics from profiles/ncu_summary.json
(tools/ncu_extract.py over the committed ncu captures).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "committed tx/sec and abort rate at 1 B200 (+partitioned 2/4/8)"
UNIT = "tx/s"

# tuned launch configuration of the C2 workload: 4 client warps
# per SM submitting CTA-level batches of 4 warps (client_group, 355 -> 490 M
# tx/s with the 2-hash filter, profiles/r02/tune_group.md)
# (round-2 retune at 801ce07: a read-only run of 2 per round (was 8), the
# fixed-length rounds (ro_adaptive 0) and a 7th worker: 501 -> 555 M in tune
# runs, profiles/r02/raw/r02bf_c2_retune.txt)
TUNED = dict(client_warps_per_sm=4, client_group=4, server_workers=7, server_combine=8, ro_streak=2, publish=1,
             ro_adaptive=0, server_recv=0)
# per-workload overrides of the tuned launch (tools/tune.py on B200): the hot-item
# chains of C3 want the lower-latency self-receiving server combining at most 2
# batches per critical section (3.3M -> 4.5M tx/s against 8) and the clients'
# own ordered GTS publish (no publisher hop on the chain: 4.4M -> 5.0M), the PUT
# convoys of C4 longer read-only runs ahead of a blocked PUT, and a PUT that met
# a newer version of its set sits out up to 16 rounds but its warp's GET run
# ends once GTS covers that version (ro_adaptive 2: 52 -> 55 M tx/s, abort rate
# 54 % -> 13 %); both keep per-warp batches (the self-receiving server and the
# KV workload take no groups) and send round-tagged requests (no fence between
# payload and doorbell: a shorter link; C4 103 -> 113 M tx/s, while C2's
# server-bound step prefers fenced payloads, 494 vs 505 M); C4's server
# worker writes the committed PUTs back itself and the publisher advances
# GTS (server_writeback: 115 -> 125 M fenced, 135 M tagged, the client's
# answer and write-back off the hot set's chain); C3's self-receiving workers
# write back too and advance GTS themselves in CTS order (4.9 -> 5.3 M on one
# box)
TUNED_PER_CONFIG = {"C3": dict(server_recv=1, server_workers=7, server_combine=2, publish=0, client_warps_per_sm=2,
                               client_group=1, req_tagged=1, ro_streak=8, ro_adaptive=1, server_writeback=1),
                    "C4": dict(ro_streak=32, client_warps_per_sm=2, client_group=1, ro_adaptive=2, backoff_max=16,
                               req_tagged=1, server_workers=7, server_writeback=1)}


def tuned(config: str) -> dict:
    return dict(TUNED, **TUNED_PER_CONFIG.get(config, {}))


def tuned_client_warps(config: str, sms: int) -> int:
    """client warps of the tuned launch: every SM but the server's hosts
    client_warps_per_sm of them."""
    return tuned(config)["client_warps_per_sm"] * (sms - 1)

# algorithmic bytes (paper VBox layout P:289): a read moves the
# VBox head, the visited version's ts and the value (4+4+4); a write-back the
# same; a request 4 B per RS and per WS id, a response 4 B per tx and a batch
# header 16 B per 32 transactions.
BYTES_READ = 12.0
BYTES_WRITE = 12.0
BYTES_TRANSFER = 2 * BYTES_READ + 2 * BYTES_WRITE + 4 * 4 + 4 + 16 / 32   # 68.5


def algorithmic_bytes(stats: dict, ro_reads: int, n_items: int) -> float:
    L = ro_reads if ro_reads else n_items
    return stats["committed_update"] * BYTES_TRANSFER + stats["committed_ro"] * BYTES_READ * L


def _load_json(*parts):
    p = os.path.join(ROOT, *parts)
    if not os.path.exists(p):
        return {}
    with open(p) as f:
        return json.load(f)


def hbm_peak():
    d = _load_json("MEASURED_PEAKS.json")
    if "hbm_gbs" in d:
        return float(d["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (copy bandwidth, driver-measured)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def roofs():
    """Measured roofs of this B200 (tools/ubench/roofs.cu, filt16_ubench.cu)."""
    return _load_json("profiles", "roofs_b200.json")


def ncu_entry(config: str):
    """Per-launch counters of csmv_fused for this config's bench step."""
    return _load_json("profiles", "ncu_summary.json").get(config.lower(), {})


def serial_chain(batches_per_s, cs_cycles, upd_per_batch, clocks, floor_cycles):
    """The commit critical section is one serial chain on the server SM.  Its
    floor is the same chain (filter loads -> recency test -> ballot -> CTS ->
    filter stores) for one request (a batch, or a client group's G batches)
    timed alone on an idle SM (filt16_ubench): one request per `floor_cycles`
    at the SM clock.  `frac` = requests/s reached / that bound."""
    d = {"batches_per_s": batches_per_s, "critical_section_cycles_per_batch": cs_cycles,
         "updates_per_batch": upd_per_batch,
         "critical_section_cycles_per_update": cs_cycles / upd_per_batch if upd_per_batch else None}
    mhz = clocks.get("sm_mhz") or clocks.get("sm_max_mhz")
    if mhz and floor_cycles:
        bound = mhz * 1e6 / floor_cycles
        d.update({"floor_cycles_per_batch": floor_cycles,
                  "floor_source": "profiles/roofs_b200.json cs_floor_cycles_per_request[g<group>k2]",
                  "bound_batches_per_s": bound, "frac": batches_per_s / bound,
                  "updates_bound_per_s": bound * upd_per_batch})
    return d


def cpu_info():
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.path = None

    def __enter__(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except (FileNotFoundError, OSError):
            self.proc = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if getattr(self, "_summary", None) is not None:
            return self._summary
        self._summary = self._read()
        return self._summary

    def _read(self):
        if not self.path or not os.path.exists(self.path):
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm, smax, reasons = [], None, set()
        names = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        os.unlink(self.path)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


DESCR = {"C1": "C1: bank, 1,024 accounts, K=4, 8 client warps, 10k transfers + 10% total-sum ROTs",
         "C2": "C2: bank, 1M accounts, K=4, 50% update, uniform, 64-read ROT scans",
         "C3": "C3: bank, 4,096 accounts, K=4, 90% 64-read ROT scans, zipf 0.99 updates",
         "C4": "C4: MemcachedGPU KV, 4M slots/keys, 16 ways, K=4, 99% GET, zipf 0.99"}


def oracle_sample_rate(cfg, budget_s: float, chunk: int, tx_start: int = 0):
    """CPU oracle (1-warp deterministic schedule, single thread) on bounded
    chunks of the workload; returns (tx/s, txs, seconds)."""
    import numpy as np

    import oracle

    w = cfg.workload
    if w.kind == 1:  # KV (MemcachedGPU)
        ocfg = oracle.kv_cfg(cfg.n_items, w.kv_ways, n_keys=w.kv_keys, n_versions=cfg.n_versions, dist=w.dist,
                             zipf_theta_milli=w.zipf_theta_milli, p_update_ppm=w.p_update_ppm,
                             ro_streak=w.ro_streak)
        init = oracle.kv_preload(ocfg)
        gen, predict = oracle.kv_gen, oracle.kv_predict
    else:
        ocfg = oracle.bank_cfg(cfg.n_items, cfg.n_versions, dist=w.dist, zipf_theta_milli=w.zipf_theta_milli,
                               p_update_ppm=w.p_update_ppm, ro_period=w.ro_period, ro_reads=w.ro_reads,
                               amount_max=w.amount_max, ro_streak=w.ro_streak)
        init = np.full(cfg.n_items, 1000, dtype=np.int32)
        gen, predict = oracle.bank_gen, oracle.bank_predict
    done, spent, tx0 = 0, 0.0, tx_start
    while True:
        descs = gen(ocfg, cfg.seed, chunk, tx0=tx0)
        t = time.perf_counter()
        predict(ocfg, init, descs, 32)
        spent += time.perf_counter() - t
        done += chunk
        tx0 += chunk
        if spent >= budget_s:
            break
    return done / spent, done, spent


def make_cfg(args, world: int, rank: int):
    """The preset with the tuned launch; for world > 1 this rank's weak
    partition: the full per-GPU workload on key range [rank*N, (rank+1)*N)
    of the job, seed mix64(seed ^ rank) (partition.py)."""
    from paper_conf_ipps_nunesc022_b200 import partition, workloads
    cfg = workloads.PRESETS[args.config]()
    n_tx = args.n_tx or cfg.n_tx
    t = tuned(args.config)
    cfg = cfg.with_(n_tx=n_tx, log_mode=0, **{k: v for k, v in t.items() if k != "client_warps_per_sm"})
    part = partition.partition(cfg.n_items, n_tx, cfg.seed, rank, world, mode="weak")
    lcfg = partition.local_config(cfg, part)
    return cfg, lcfg, part


# KV algorithmic bytes (paper VBox layout): a GET hitting at
# the average way (A+1)/2 reads that many keys (head+ts+16 B) and the value
# (head+ts+32 B); a PUT at most 2A+1 reads + 4 write-backs + ids.
def kv_bytes(stats: dict, ways: int) -> float:
    get = (ways + 1) / 2 * 24 + 40
    put = (ways + 1) / 2 * 24 + 12 + (24 + 40 + 12 + 12) + 4 * ((ways + 1) / 2 + 4) + 4
    return stats["committed_ro"] * get + stats["committed_update"] * put


def bench_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    cfg, _, _ = make_cfg(args, 1, 0)
    chunk = 1 << 18
    for i in range(args.warmup):
        oracle_sample_rate(cfg, 0.0, chunk, tx_start=i * chunk)
    rates, total_tx, total_s = [], 0, 0.0
    for i in range(args.steps):
        r, n, s = oracle_sample_rate(cfg, 0.0, chunk, tx_start=(args.warmup + i) * chunk)
        rates.append(r)
        total_tx += n
        total_s += s
    value = total_tx / total_s
    sample = f"{args.steps} chunks of {chunk} consecutive {cfg.name} transactions ({cfg.n_items} items)"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total_s / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic", "config": {"workload": DESCR.get(cfg.name, cfg.name), "n_items": cfg.n_items,
                                            "n_versions": cfg.n_versions, "sample": sample},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             **cpu_info()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def roofline_block(args, cfg, lcfg, steps, kern_ns, is_kv, world):
    """Roofline of the dominant (only) kernel csmv_fused against the roof
    that binds its configuration (SURVEY 8(d) rooflines 1-3):
      C2 / C3 (store L2-resident): L2 bandwidth -- algorithmic bytes per
        launch / launch time against the measured L2 read roof;
      C4 (store 1.7 GB, HBM-resident): HBM bandwidth against MEASURED_PEAKS;
    plus the sector-granular L2 traffic and the server SM's shared-memory
    atomics from the committed ncu capture of the same bench step."""
    w = lcfg.workload
    algo = sum(kv_bytes(s, w.kv_ways) if is_kv else algorithmic_bytes(s, w.ro_reads, lcfg.n_items)
               for _, _, s in steps) / len(steps)
    kmean_s = sum(kern_ns) / len(kern_ns) * 1e-9
    achieved = algo / kmean_s / 1e9
    rf = roofs()
    nc = ncu_entry(args.config) if world == 1 else {}
    store_bytes = steps[-1][2]["store_bytes"]
    l2_resident = store_bytes < 64 << 20
    if l2_resident and rf.get("l2_read_gbs"):
        bound, peak = "l2", rf["l2_read_gbs"]
        peak_src = "profiles/roofs_b200.json l2_read_gbs (tools/ubench/roofs.cu, all SMs, 256-bit loads, L2-resident)"
    else:
        bound = "hbm"
        peak, peak_src = hbm_peak()
    out = {"bound": bound, "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
           "traffic": nc.get("dram_bytes_per_launch"), "peak_source": peak_src, "kernel": "csmv_fused",
           "algorithmic_bytes_per_launch": algo, "kernel_ms": kmean_s * 1e3,
           "store_bytes": store_bytes}
    if nc:
        out["ncu"] = {k: nc[k] for k in ("capture", "n_tx_per_launch", "duration_ms", "dram_bytes_per_launch",
                                          "l2_bytes_per_launch", "shared_atomics_per_launch") if k in nc}
        scale = lcfg.n_tx / nc.get("n_tx_per_launch", lcfg.n_tx)
        if nc.get("l2_bytes_per_launch"):
            l2b = nc["l2_bytes_per_launch"] * scale
            out["l2_traffic"] = {"bytes_per_launch": l2b, "achieved_gbs": l2b / kmean_s / 1e9,
                                 "peak_gbs": rf.get("l2_read_gbs"),
                                 "frac": (l2b / kmean_s / 1e9) / rf["l2_read_gbs"] if rf.get("l2_read_gbs") else None,
                                 "x_algorithmic": l2b / algo if algo else None}
        if nc.get("shared_atomics_per_launch") and rf.get("smem_atom_per_s_sm"):
            a = nc["shared_atomics_per_launch"] * scale / kmean_s
            out["server_smem_atomics"] = {"per_s": a, "peak_per_s_one_sm": rf["smem_atom_per_s_sm"],
                                          "frac": a / rf["smem_atom_per_s_sm"],
                                          "note": "all shared atomics of the launch (server dispatch-queue claims,"
                                                  " lock tickets) against one SM's measured atomic throughput"}
    return out


def spawn_ranks(args):
    """--gpus N > 1 without a launcher: re-run this command under torchrun
    (one process per GPU, 127.0.0.1 rendezvous); rank 0 prints the line."""
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def bench_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_nunesc022_b200 import csmv, partition

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}\n")
        return 2
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    cfg, lcfg, part = make_cfg(args, world, rank)
    props = torch.cuda.get_device_properties(dev)
    n_cw = args.client_warps or lcfg.workload.client_warps or \
        tuned_client_warps(args.config, props.multi_processor_count)
    lcfg = lcfg.with_(client_warps=n_cw)
    w = lcfg.workload
    is_kv = w.kind == csmv.KIND_KV

    stream = torch.cuda.current_stream()
    if is_kv:
        store = csmv.KvStore(lcfg.n_items, w.kv_ways, lcfg.n_versions)
        init = None  # the preload is computed on the device from n_keys: no H2D
        store.load(w.kv_keys)
    else:
        store = csmv.Store(lcfg.n_items, lcfg.n_versions)
        init = np.full(lcfg.n_items, 1000, dtype=np.int32)
        store.load(init)
    store.set_stream(stream.cuda_stream)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()

    for i in range(args.warmup):
        store.run(w, lcfg.n_tx, lcfg.seed + 1000 + i)

    barrier()
    torch.cuda.synchronize()
    steps = []
    with Clocks(dev.index) as clk:
        for i in range(args.steps):
            flush.zero_()                                   # L2 flush, outside the events
            ev0 = torch.cuda.Event(enable_timing=True)
            ev1 = torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            st = store.run(w, lcfg.n_tx, lcfg.seed + i)
            ev1.record(stream)
            steps.append((ev0, ev1, st))
        torch.cuda.synchronize()
    barrier()
    step_ms = [a.elapsed_time(b) for a, b, _ in steps]
    kern_ns = [s["elapsed_ns"] for _, _, s in steps]
    agg = {k: sum(s[k] for _, _, s in steps) for k in ("committed", "committed_update", "committed_ro",
                                                        "total_aborts", "batches", "rounds")}
    agg["elapsed_ns"] = int(sum(step_ms) * 1e6)
    red = partition.reduce_stats(agg, device=dev if world > 1 else None)
    total_ms_max = red["elapsed_ns"] / 1e6
    value = red["committed"] / (total_ms_max * 1e-3)
    roof = roofline_block(args, cfg, lcfg, steps, kern_ns, is_kv, world)
    last = steps[-1][2]
    cs_cycles = last["server_phase_cycles"]["critical"] / max(1, last["batches"])

    # end to end through the public API with host buffers: load (H2D of the
    # initial balances), run, stats (D2H)
    e2e_steps = max(1, min(3, args.steps))
    init_pinned = None if is_kv else torch.from_numpy(init).pin_memory()
    torch.cuda.synchronize()
    barrier()
    t0 = time.perf_counter()
    e2e_committed = 0
    t_load = 0.0
    for i in range(e2e_steps):
        tl = time.perf_counter()
        store.load(w.kv_keys if is_kv else init_pinned.numpy())
        t_load += time.perf_counter() - tl
        s = store.run(w, lcfg.n_tx, lcfg.seed + 500 + i)
        e2e_committed += s["committed"]
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    e2e_red = partition.reduce_stats({"committed_update": 0, "committed_ro": 0, "batches": 0, "rounds": 0,
                                      "total_aborts": 0, "committed": e2e_committed,
                                      "elapsed_ns": int(e2e_s * 1e9)}, device=dev if world > 1 else None)
    e2e_value = e2e_red["committed"] / (e2e_red["elapsed_ns"] * 1e-9)
    store.close()

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        r, n, s = oracle_sample_rate(cfg, args.cpu_budget, 1 << 18)
        cpu = {"value": r, "unit": UNIT, "cores": 1, "kind": "oracle", **cpu_info(),
               "sample": f"{n} consecutive {cfg.name} transactions ({s:.1f} s, 1-warp schedule, {cfg.n_items} items)"}
    rf = roofs()
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total_ms_max / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "abort_rate": red["abort_rate"],
        "config": {"workload": DESCR.get(cfg.name, cfg.name),
                   "n_items_per_gpu": lcfg.n_items, "n_items_job": lcfg.n_items * world,
                   "n_versions": cfg.n_versions, "n_tx_per_step_per_gpu": lcfg.n_tx,
                   "client_warps_per_gpu": n_cw, "client_group": w.client_group, "server_workers": w.server_workers,
                   "server_combine": w.server_combine,
                   "ro_streak": w.ro_streak, "ro_adaptive": w.ro_adaptive, "backoff_max": w.backoff_max,
                   "publish": ["client", "server"][w.publish],
                   "server_recv": ["receiver warp", "self-receiving workers"][w.server_recv],
                   "parallelism": f"partitioned x{world}" if world > 1 else "single-gpu",
                   "multi_gpu": "independent key-range partitions (rank g: keys [g*N, (g+1)*N), full per-GPU "
                                "workload), no cross-GPU transactions, NCCL stats only",
                   "l2": "flushed (512 MiB write) before every timed step"},
        "roofline": roof,
        "serial_chain": serial_chain(red["batches"] / (total_ms_max * 1e-3), cs_cycles,
                                     red["committed_update"] / max(1, red["batches"]), clk.summary(),
                                     rf.get("cs_floor_cycles_per_request", {}).get(
                                         f"g{max(1, w.client_group)}k2", rf.get("cs_floor_cycles"))),
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": 0 if is_kv else int(init.nbytes),
                "d2h_bytes_per_step": 400, "steps": e2e_steps,
                "load_ms_per_step": 1e3 * t_load / e2e_steps, "wall_ms_per_step": 1e3 * e2e_s / e2e_steps},
        "gpu_launches": args.steps * int(last["kernel_launches"]),
        "clocks": clk.summary(),
        "kernel_ms_per_step": statistics.mean(kern_ns) / 1e6,
        "aborts": last["aborts"],
    }
    if args.config in ("C3", "C4") and rf.get("xsm_roundtrip_ns"):
        line["hot_chain"] = hot_chain(last, lcfg, rf, statistics.mean(kern_ns))
    if cpu:
        line["cpu_baseline"] = cpu
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def hot_chain(st, lcfg, rf, kern_ns):
    """C3 / C4: every committed transfer touching the hottest account (C4:
    every PUT on the hottest cache set) must see the previous one in its
    snapshot, so those commits form a chain whose link is at
    least publish -> snapshot -> read -> request -> server -> response: two
    cross-SM round trips (client->server->client, and the GTS publish -> next
    client's acquire) plus the read (one L2 round trip: the bank's two rings,
    the KV set read by the warp together).  Floor per link = 2 x
    xsm_roundtrip + l2_load (tools/ubench/roofs.cu)."""
    import numpy as np
    w = lcfg.workload
    theta = w.zipf_theta_milli / 1000.0
    if w.kind == 1:
        # C4: every PUT on the hottest cache set (the set of key 0, zipf rank
        # 0) reads and writes its clock, so those PUTs form the chain; the
        # set of key k is uniform(mix64(k ^ 0xA5..A5), T) (docs/GENERATOR.md)
        n = w.kv_keys
        r = np.arange(1, n + 1, dtype=np.float64) ** -theta
        k = np.arange(n, dtype=np.uint64) ^ np.uint64(0xA5A5A5A5A5A5A5A5)
        with np.errstate(over="ignore"):
            z = k + np.uint64(0x9E3779B97F4A7C15)
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            z = z ^ (z >> np.uint64(31))
        T = lcfg.n_items // w.kv_ways
        sets = ((z >> np.uint64(32)) * np.uint64(T) + (((z & np.uint64(0xFFFFFFFF)) * np.uint64(T)) >> np.uint64(32))) \
            >> np.uint64(32)
        p_touch = float(r[sets == sets[0]].sum() / r.sum())
    else:
        n = lcfg.n_items
        r = np.arange(1, n + 1, dtype=np.float64) ** -theta
        p0 = r[0] / r.sum()
        # a transfer touches account 0 if src or dst is 0 (dst = src+1 on a collision)
        p_touch = 1 - (1 - p0) ** 2
    links = st["committed_update"] * p_touch
    floor_ns = 2 * rf["xsm_roundtrip_ns"] + rf["l2_load_ns"]
    link_ns = kern_ns / links if links else None
    return {"hot_commits": links, "link_ns": link_ns, "floor_link_ns": floor_ns,
            "frac": floor_ns / link_ns if link_ns else None,
            "floor": "2 x xsm_roundtrip_ns + l2_load_ns (profiles/roofs_b200.json)"}


def main():
    ap = argparse.ArgumentParser(description=__doc__.split("\n")[0])
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=("ours", "reference"), default="ours")
    ap.add_argument("--n-tx", type=int, default=0)
    ap.add_argument("--config", choices=("C1", "C2", "C3", "C4"), default="C2",
                    help="workload (default C2, the config BASELINE.json's metric is quoted on)")
    ap.add_argument("--client-warps", type=int, default=0)
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args)
    if args.impl == "reference":
        return bench_reference(args)
    return bench_ours(args)


if __name__ == "__main__":
    sys.exit(main())
