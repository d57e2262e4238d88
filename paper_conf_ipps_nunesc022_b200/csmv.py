"""Thin ctypes binding of include/csmv.h -- argument marshalling only.

Every step of the commit pipeline runs inside libcsmv.so's kernels; this
module only converts Python/numpy arguments into the C ABI's plain pointers
and sizes, and raises on error codes.  It fails loudly when the library is
missing or when no sm_100a device is present: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass, fields

import numpy as np

from . import build as _build

OK, EINVAL, ENOMEM, ECUDA, ESTATE, ETIMEOUT, EOVERFLOW = 0, -1, -2, -3, -4, -5, -6
KIND_BANK, KIND_KV = 0, 1
DIST_UNIFORM, DIST_ZIPF = 0, 1
LOG_NONE, LOG_DIGEST, LOG_FULL = 0, 1, 2
SERVER_CTA, SERVER_CLUSTER, SERVER_PART = 0, 1, 2
PUBLISH_CLIENT, PUBLISH_SERVER = 0, 1
RETRY_FREE, RETRY_FIFO = 0, 1
ATR_HASH, ATR_LIST, ATR_LIST_NOCV = 0, 1, 2
COMMIT_CSMV, COMMIT_ONLYCS, COMMIT_JVSTM = 0, 1, 2
DBG_NO_PREVAL, DBG_NO_VALIDATE, DBG_JITTER, DBG_PHASES, DBG_KV_ITEMSETS, DBG_ALT_COMMIT, DBG_TRACE = 1, 2, 4, 8, 16, 32, 64
DBG_KV_SEQREAD = 128
RECV_WARP, RECV_SELF = 0, 1
CLIENT_PHASES = ("read", "preval", "submit", "rot", "wait_server", "writeback", "publish", "divergence")
ABORT_REASONS = ("preval", "conflict", "early", "overflow", "version")

TRACE_DTYPE = np.dtype([("cts", "<u4"), ("snapshot", "<u4"), ("t_begin", "<u8"), ("t_submit", "<u8"),
                        ("t_response", "<u8"), ("t_publish", "<u8"), ("t_claim", "<u8"), ("t_served", "<u8"),
                        ("t_snap", "<u8"), ("t_read", "<u8"), ("n_readers", "<u4"), ("n_kept", "<u4")])
LOG_DTYPE = np.dtype([("tx", "<u4"), ("snapshot", "<u4"), ("cts", "<u4"),
                      ("attempts", "<u4"), ("read_digest", "<u8"), ("aux", "<u8")])


class CsmvError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"csmv error {code}: {msg}")
        self.code = code


class _Workload(C.Structure):
    _fields_ = [(n, C.c_uint32) for n in (
        "kind", "dist", "zipf_theta_milli", "p_update_ppm", "ro_period", "ro_reads",
        "amount_max", "kv_ways", "kv_keys", "client_warps", "server", "cluster_size", "server_workers", "server_combine",
        "atr_capacity", "atr_mode", "publish", "ro_streak", "backoff_max", "log_mode", "debug_flags", "watchdog_ms", "commit",
        "ro_adaptive", "server_recv", "client_group", "trace_item", "elide_ww", "retry_order", "server_writeback", "req_tagged")]


class _Stats(C.Structure):
    _fields_ = [("committed_update", C.c_uint64), ("committed_ro", C.c_uint64),
                ("aborts", (C.c_uint64 * 2) * 5), ("batches", C.c_uint64),
                ("server_groups", C.c_uint64),
                ("rounds", C.c_uint64), ("gts_start", C.c_uint64), ("gts_final", C.c_uint64),
                ("elapsed_ns", C.c_uint64), ("ro_checksum", C.c_uint64),
                ("store_bytes", C.c_uint64), ("store_bytes_paper", C.c_uint64),
                ("server_lock_cycles", C.c_uint64), ("server_busy_cycles", C.c_uint64),
                ("server_phase_cycles", C.c_uint64 * 8), ("cas_failures", C.c_uint64),
                ("client_phase_cycles", C.c_uint64 * 8),
                ("client_warps", C.c_uint32), ("server_ctas", C.c_uint32),
                ("server_workers", C.c_uint32), ("atr_entries", C.c_uint32),
                ("sm_count", C.c_uint32), ("kernel_launches", C.c_uint32)]


@dataclass
class Workload:
    """Mirror of csmv_workload (include/csmv.h)."""
    kind: int = KIND_BANK
    dist: int = DIST_UNIFORM
    zipf_theta_milli: int = 990
    p_update_ppm: int = 500_000
    ro_period: int = 0
    ro_reads: int = 64
    amount_max: int = 100
    kv_ways: int = 16
    kv_keys: int = 0
    client_warps: int = 0
    server: int = SERVER_CTA
    cluster_size: int = 16
    server_workers: int = 0
    server_combine: int = 0
    atr_capacity: int = 0
    atr_mode: int = ATR_HASH
    publish: int = PUBLISH_CLIENT
    ro_streak: int = 0
    backoff_max: int = 0
    log_mode: int = LOG_NONE
    debug_flags: int = 0
    watchdog_ms: int = 0
    commit: int = COMMIT_CSMV
    ro_adaptive: int = 0
    server_recv: int = 0
    client_group: int = 0
    trace_item: int = 0xFFFFFFFF
    elide_ww: int = 0
    retry_order: int = 0
    server_writeback: int = 0
    req_tagged: int = 0

    def to_c(self) -> _Workload:
        return _Workload(*[getattr(self, f.name) for f in fields(self)])


_lib = None


def lib() -> C.CDLL:
    """Load libcsmv.so (building it in-tree first if it is stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = _build.LIB
    if not os.path.exists(path) or _build.stale():
        _build.build()
    L = C.CDLL(path)
    vp, u64, u32, i32 = C.c_void_p, C.c_uint64, C.c_uint32, C.c_int
    L.csmv_abi_version.restype = i32
    L.csmv_last_error.restype = C.c_char_p
    L.csmv_create.restype = vp
    L.csmv_create.argtypes = [u64, u32]
    L.csmv_create_kv.restype = vp
    L.csmv_create_kv.argtypes = [u64, u32, u32]
    L.csmv_load.argtypes = [vp, vp, u64]
    L.csmv_load_kv.argtypes = [vp, u64]
    L.csmv_set_stream.argtypes = [vp, vp]
    L.csmv_run.argtypes = [vp, C.POINTER(_Workload), u64, u64]
    L.csmv_stats.argtypes = [vp, C.POINTER(_Stats)]
    L.csmv_get_log.argtypes = [vp, vp, u64, C.POINTER(u64)]
    L.csmv_get_vals.argtypes = [vp, vp, u64, C.POINTER(u32)]
    L.csmv_dump_store.argtypes = [vp, vp, u64]
    L.csmv_dump_kv.argtypes = [vp, vp, vp, vp, vp]
    L.csmv_gen_descs.argtypes = [vp, C.POINTER(_Workload), u64, u64, u64, vp]
    L.csmv_zipf_table.argtypes = [u32, u32, vp]
    L.csmv_get_trace.argtypes = [vp, vp, u64, C.POINTER(u64)]
    L.csmv_destroy.argtypes = [vp]
    L.csmv_destroy.restype = None
    _lib = L
    return L


def _check(rc: int):
    if rc != OK:
        raise CsmvError(rc, lib().csmv_last_error().decode())


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def stats_dict(s: _Stats) -> dict:
    d = {f: getattr(s, f) for f, _ in _Stats._fields_
         if f not in ("aborts", "server_phase_cycles", "client_phase_cycles")}
    d["client_phase_cycles"] = dict(zip(CLIENT_PHASES, list(s.client_phase_cycles)))
    d["server_phase_cycles"] = dict(zip(("queue", "load", "lock_wait", "critical", "respond", "cs_validate", "cs_insert0", "cs_insert1"),
                                        list(s.server_phase_cycles)))
    d["aborts"] = {ABORT_REASONS[i]: {"ro": s.aborts[i][0], "update": s.aborts[i][1]}
                   for i in range(5)}
    d["total_aborts"] = sum(s.aborts[i][k] for i in range(5) for k in range(2))
    d["committed"] = s.committed_update + s.committed_ro
    att = d["committed"] + d["total_aborts"]
    d["abort_rate"] = d["total_aborts"] / att if att else 0.0
    d["tx_per_s"] = d["committed"] / (s.elapsed_ns * 1e-9) if s.elapsed_ns else 0.0
    return d


class Store:
    """A CSMV store on the current CUDA device (csmv_t)."""

    def __init__(self, n_items: int, n_versions: int = 4):
        h = lib().csmv_create(n_items, n_versions)
        if not h:
            raise CsmvError(ECUDA, lib().csmv_last_error().decode())
        self.h = h
        self.n_items, self.n_versions = n_items, n_versions

    def close(self):
        if self.h:
            lib().csmv_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def set_stream(self, stream_handle: int | None):
        _check(lib().csmv_set_stream(self.h, stream_handle))

    def load(self, init_values):
        a = np.ascontiguousarray(init_values, dtype=np.int32)
        _check(lib().csmv_load(self.h, _ptr(a), a.size))

    def run(self, w: Workload, n_tx: int, seed: int) -> dict:
        wc = w.to_c()
        _check(lib().csmv_run(self.h, C.byref(wc), n_tx, seed))
        return self.stats()

    def stats(self) -> dict:
        s = _Stats()
        _check(lib().csmv_stats(self.h, C.byref(s)))
        return stats_dict(s)

    def log(self, n_tx: int) -> np.ndarray:
        out = np.zeros(n_tx, dtype=LOG_DTYPE)
        n = C.c_uint64()
        _check(lib().csmv_get_log(self.h, _ptr(out), n_tx, C.byref(n)))
        return out[: n.value]

    def vals(self):
        mv = C.c_uint32()
        _check(lib().csmv_get_vals(self.h, None, 0, C.byref(mv)))
        n = self.stats()["committed"]
        out = np.zeros(n * mv.value, dtype=np.uint32)
        _check(lib().csmv_get_vals(self.h, _ptr(out), out.size, C.byref(mv)))
        return out, mv.value

    def trace(self, cap: int = 1 << 18) -> np.ndarray:
        """CSMV_DBG_TRACE records of the last run (csmv_get_trace)."""
        out = np.zeros(cap, dtype=TRACE_DTYPE)
        n = C.c_uint64()
        _check(lib().csmv_get_trace(self.h, _ptr(out), cap, C.byref(n)))
        return out[: min(cap, n.value)]

    def dump(self) -> np.ndarray:
        out = np.zeros(self.n_items * self.n_versions, dtype=np.uint64)
        _check(lib().csmv_dump_store(self.h, _ptr(out), out.size))
        return out

    def gen_descs(self, w: Workload, seed: int, n: int, tx0: int = 0) -> np.ndarray:
        out = np.zeros(n * 6, dtype=np.uint32)
        wc = w.to_c()
        _check(lib().csmv_gen_descs(self.h, C.byref(wc), seed, tx0, n, _ptr(out)))
        return out.reshape(n, 6)


def zipf_table(n: int, theta_milli: int) -> np.ndarray:
    out = np.zeros(n, dtype=np.uint64)
    _check(lib().csmv_zipf_table(n, theta_milli, _ptr(out)))
    return out


class KvStore(Store):
    """A MemcachedGPU store (csmv_create_kv): n_slots slots, `ways` ways."""

    def __init__(self, n_slots: int, ways: int = 16, n_versions: int = 4):
        h = lib().csmv_create_kv(n_slots, ways, n_versions)
        if not h:
            raise CsmvError(ECUDA, lib().csmv_last_error().decode())
        self.h = h
        self.n_slots, self.ways, self.n_versions = n_slots, ways, n_versions
        self.n_items = 3 * n_slots + n_slots // ways

    def load(self, n_keys: int):
        _check(lib().csmv_load_kv(self.h, n_keys))

    def dump(self):
        S, T = self.n_slots, self.n_slots // self.ways
        keys = np.zeros((S, 4), dtype=np.uint32)
        vals = np.zeros((S, 8), dtype=np.uint32)
        lru = np.zeros(S, dtype=np.uint32)
        clocks = np.zeros(T, dtype=np.uint32)
        _check(lib().csmv_dump_kv(self.h, _ptr(keys), _ptr(vals), _ptr(lru), _ptr(clocks)))
        return keys, vals, lru, clocks

    def gen_descs(self, w: Workload, seed: int, n: int, tx0: int = 0) -> np.ndarray:
        out = np.zeros(n * 10, dtype=np.uint32)
        wc = w.to_c()
        _check(lib().csmv_gen_descs(self.h, C.byref(wc), seed, tx0, n, _ptr(out)))
        return out.reshape(n, 10)
