"""CPU oracle for the CSMV batched commit pipeline -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_ipps_nunesc022_b200`` never imports it, and this
package never imports the product package (they share no code; each
implements ``docs/GENERATOR.md`` on its own).

The arithmetic lives in ``oracle.c`` (plain C99, single-threaded); this module
is ctypes marshalling plus a build helper.  See ``oracle.h`` for what each
function computes and which PAPER.md passage it follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
SRC_KV = os.path.join(HERE, "oracle_kv.c")
HDR = os.path.join(HERE, "oracle.h")
LIB = os.path.join(HERE, "liboracle.so")

EMPTY_TS = 0xFFFFFFFF
DIST_UNIFORM, DIST_ZIPF = 0, 1

LOG_DTYPE = np.dtype([("tx", "<u4"), ("snapshot", "<u4"), ("cts", "<u4"),
                      ("attempts", "<u4"), ("read_digest", "<u8"), ("aux", "<u8")])
BANK_DESC_DTYPE = np.dtype([("is_update", "<u4"), ("src", "<u4"), ("dst", "<u4"),
                            ("amt", "<i4"), ("start", "<u4"), ("len", "<u4")])

ERR_NAMES = {0: "OK", 1: "MISSING", 2: "CTS", 3: "SNAPSHOT", 4: "VALIDITY",
             5: "READ", 6: "WRITE", 7: "RING", 8: "STATS", 9: "ARGS"}


class BankCfg(C.Structure):
    _fields_ = [("n_items", C.c_uint32), ("n_versions", C.c_uint32),
                ("dist", C.c_uint32), ("zipf_theta_milli", C.c_uint32),
                ("p_update_ppm", C.c_uint32), ("ro_period", C.c_uint32),
                ("ro_reads", C.c_uint32), ("amount_max", C.c_uint32),
                ("ro_streak", C.c_uint32)]


class Report(C.Structure):
    _fields_ = [("ok", C.c_int), ("code", C.c_int), ("tx", C.c_uint64),
                ("expected", C.c_uint64), ("got", C.c_uint64),
                ("replayed", C.c_uint64), ("seconds", C.c_double),
                ("msg", C.c_char * 200)]

    def as_dict(self):
        return {"ok": bool(self.ok), "code": ERR_NAMES.get(self.code, self.code),
                "tx": self.tx, "expected": self.expected, "got": self.got,
                "replayed": self.replayed, "seconds": self.seconds,
                "msg": self.msg.decode()}


class Claims(C.Structure):
    _fields_ = [("committed_update", C.c_uint64), ("committed_ro", C.c_uint64),
                ("gts_final", C.c_uint64), ("total_aborts", C.c_uint64)]


class PredStats(C.Structure):
    _fields_ = [("rounds", C.c_uint64), ("batches", C.c_uint64),
                ("aborts_preval", C.c_uint64), ("committed_update", C.c_uint64),
                ("committed_ro", C.c_uint64), ("gts_final", C.c_uint64),
                ("seconds", C.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class KvCfg(C.Structure):
    _fields_ = [(n, C.c_uint32) for n in ("n_slots", "ways", "n_keys", "n_versions", "dist",
                                         "zipf_theta_milli", "p_update_ppm", "ro_streak")]


class KvState(C.Structure):
    _fields_ = [("keys", C.c_void_p), ("vals", C.c_void_p), ("lru", C.c_void_p),
                ("clocks", C.c_void_p)]


KV_DESC_DTYPE = np.dtype([("is_update", "<u4"), ("key", "<u4"), ("val", "<u4", (8,))])


class KvStore:
    """numpy-backed or_kv_state (keys S x 4, vals S x 8, lru S, clocks S/A)."""

    def __init__(self, n_slots, ways):
        self.keys = np.zeros((n_slots, 4), dtype=np.uint32)
        self.vals = np.zeros((n_slots, 8), dtype=np.uint32)
        self.lru = np.zeros(n_slots, dtype=np.uint32)
        self.clocks = np.zeros(n_slots // ways, dtype=np.uint32)

    def c(self) -> KvState:
        return KvState(self.keys.ctypes.data, self.vals.ctypes.data, self.lru.ctypes.data,
                       self.clocks.ctypes.data)

    def copy(self):
        o = KvStore.__new__(KvStore)
        o.keys, o.vals, o.lru, o.clocks = (self.keys.copy(), self.vals.copy(), self.lru.copy(),
                                           self.clocks.copy())
        return o


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C99)."""
    stale = force or not os.path.exists(LIB) or any(
        os.path.getmtime(p) > os.path.getmtime(LIB) for p in (SRC, SRC_KV, HDR))
    if stale:
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-Wextra", "-fPIC",
                               "-shared", "-o", LIB, SRC, SRC_KV, "-lm"])
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        u64, u32, vp = C.c_uint64, C.c_uint32, C.c_void_p
        L.or_mix64.restype = u64
        L.or_mix64.argtypes = [u64]
        L.or_draw.restype = u64
        L.or_draw.argtypes = [u64, u64, u64]
        L.or_uniform.restype = u64
        L.or_uniform.argtypes = [u64, u64]
        L.or_zipf_cdf.argtypes = [u32, u32, vp]
        L.or_upper_bound.restype = u32
        L.or_upper_bound.argtypes = [vp, u32, u64]
        L.or_bank_gen.argtypes = [C.POINTER(BankCfg), u64, u64, u64, vp, vp]
        L.or_bank_check.argtypes = [C.POINTER(BankCfg), vp, u64, vp, vp, vp, u32, vp,
                                    C.POINTER(Claims), C.POINTER(Report)]
        L.or_bank_predict.argtypes = [C.POINTER(BankCfg), vp, u64, vp, u32, vp, vp, u32,
                                      vp, C.POINTER(PredStats)]
        L.or_vbox_bytes.restype = u64
        L.or_vbox_bytes.argtypes = [u64, u32, u32]
        L.or_kv_key16.argtypes = [u32, vp]
        L.or_kv_set.restype = u32
        L.or_kv_set.argtypes = [u32, u32]
        L.or_kv_gen.argtypes = [C.POINTER(KvCfg), u64, u64, u64, vp, vp]
        L.or_kv_preload.argtypes = [C.POINTER(KvCfg), C.POINTER(KvState)]
        L.or_kv_check.argtypes = [C.POINTER(KvCfg), C.POINTER(KvState), u64, vp, vp,
                                  C.POINTER(KvState), C.POINTER(Claims), C.POINTER(Report)]
        L.or_kv_predict.argtypes = [C.POINTER(KvCfg), C.POINTER(KvState), u64, vp, u32, vp,
                                    C.POINTER(KvState), C.POINTER(PredStats)]
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def mix64(x: int) -> int:
    return lib().or_mix64(x)


def draw(seed: int, tx: int, k: int) -> int:
    return lib().or_draw(seed, tx, k)


def uniform(u: int, n: int) -> int:
    return lib().or_uniform(u, n)


def zipf_cdf(n: int, theta_milli: int) -> np.ndarray:
    out = np.zeros(n, dtype=np.uint64)
    rc = lib().or_zipf_cdf(n, theta_milli, _ptr(out))
    assert rc == 0, rc
    return out


def bank_cfg(n_items, n_versions=4, dist=DIST_UNIFORM, zipf_theta_milli=990,
             p_update_ppm=500000, ro_period=0, ro_reads=64, amount_max=100,
             ro_streak=0) -> BankCfg:
    return BankCfg(n_items, n_versions, dist, zipf_theta_milli, p_update_ppm,
                   ro_period, ro_reads, amount_max, ro_streak)


def bank_gen(cfg: BankCfg, seed: int, n_tx: int, tx0: int = 0) -> np.ndarray:
    out = np.zeros(n_tx, dtype=BANK_DESC_DTYPE)
    cdf = zipf_cdf(cfg.n_items, cfg.zipf_theta_milli) if cfg.dist == DIST_ZIPF else None
    rc = lib().or_bank_gen(C.byref(cfg), seed, tx0, n_tx, _ptr(cdf), _ptr(out))
    assert rc == 0, rc
    return out


def bank_check(cfg: BankCfg, init, descs, log, vals=None, max_vals=0, rings=None,
               claims: dict | None = None) -> dict:
    init = np.ascontiguousarray(init, dtype=np.int32)
    descs = np.ascontiguousarray(descs, dtype=BANK_DESC_DTYPE)
    log = np.ascontiguousarray(log, dtype=LOG_DTYPE)
    assert len(log) == len(descs)
    if vals is not None:
        vals = np.ascontiguousarray(vals, dtype=np.uint32)
    if rings is not None:
        rings = np.ascontiguousarray(rings, dtype=np.uint64)
        assert rings.size == cfg.n_items * cfg.n_versions
    cl = None
    if claims is not None:
        cl = Claims(claims["committed_update"], claims["committed_ro"],
                    claims["gts_final"], claims["total_aborts"])
    rep = Report()
    lib().or_bank_check(C.byref(cfg), _ptr(init), len(descs), _ptr(descs), _ptr(log),
                        _ptr(vals), max_vals, _ptr(rings),
                        C.byref(cl) if cl is not None else None, C.byref(rep))
    return rep.as_dict()


def bank_predict(cfg: BankCfg, init, descs, n_lanes=32, max_vals=0):
    init = np.ascontiguousarray(init, dtype=np.int32)
    descs = np.ascontiguousarray(descs, dtype=BANK_DESC_DTYPE)
    n = len(descs)
    log = np.zeros(n, dtype=LOG_DTYPE)
    vals = np.zeros(n * max_vals, dtype=np.uint32) if max_vals else None
    rings = np.zeros(cfg.n_items * cfg.n_versions, dtype=np.uint64)
    st = PredStats()
    rc = lib().or_bank_predict(C.byref(cfg), _ptr(init), n, _ptr(descs), n_lanes,
                               _ptr(log), _ptr(vals), max_vals, _ptr(rings), C.byref(st))
    assert rc == 0, rc
    return log, vals, rings, st.as_dict()


def vbox_bytes(n_items: int, value_bytes: int, k: int) -> int:
    return lib().or_vbox_bytes(n_items, value_bytes, k)


def pack(ts: int, val: int) -> int:
    return (ts << 32) | (val & 0xFFFFFFFF)


def unpack(slot: int):
    ts, v = slot >> 32, slot & 0xFFFFFFFF
    return ts, v - (1 << 32) if v >= (1 << 31) else v


def kv_cfg(n_slots, ways=16, n_keys=None, n_versions=4, dist=DIST_ZIPF, zipf_theta_milli=990,
           p_update_ppm=10_000, ro_streak=0) -> KvCfg:
    return KvCfg(n_slots, ways, n_slots if n_keys is None else n_keys, n_versions, dist,
                 zipf_theta_milli, p_update_ppm, ro_streak)


def key16(k: int) -> np.ndarray:
    out = np.zeros(4, dtype=np.uint32)
    lib().or_kv_key16(k, _ptr(out))
    return out


def kv_set(k: int, n_sets: int) -> int:
    return lib().or_kv_set(k, n_sets)


def kv_gen(cfg: KvCfg, seed: int, n_tx: int, tx0: int = 0) -> np.ndarray:
    out = np.zeros(n_tx, dtype=KV_DESC_DTYPE)
    cdf = zipf_cdf(cfg.n_keys, cfg.zipf_theta_milli) if cfg.dist == DIST_ZIPF else None
    rc = lib().or_kv_gen(C.byref(cfg), seed, tx0, n_tx, _ptr(cdf), _ptr(out))
    assert rc == 0, rc
    return out


def kv_preload(cfg: KvCfg) -> KvStore:
    st = KvStore(cfg.n_slots, cfg.ways)
    cs = st.c()
    rc = lib().or_kv_preload(C.byref(cfg), C.byref(cs))
    assert rc == 0, rc
    return st


def kv_check(cfg: KvCfg, init: KvStore, descs, log, final: KvStore | None = None,
             claims: dict | None = None) -> dict:
    descs = np.ascontiguousarray(descs, dtype=KV_DESC_DTYPE)
    log = np.ascontiguousarray(log, dtype=LOG_DTYPE)
    ci = init.c()
    cf = final.c() if final is not None else None
    cl = None
    if claims is not None:
        cl = Claims(claims["committed_update"], claims["committed_ro"], claims["gts_final"],
                    claims["total_aborts"])
    rep = Report()
    lib().or_kv_check(C.byref(cfg), C.byref(ci), len(descs), _ptr(descs), _ptr(log),
                      C.byref(cf) if cf is not None else None,
                      C.byref(cl) if cl is not None else None, C.byref(rep))
    return rep.as_dict()


def kv_predict(cfg: KvCfg, init: KvStore, descs, n_lanes=32):
    descs = np.ascontiguousarray(descs, dtype=KV_DESC_DTYPE)
    n = len(descs)
    log = np.zeros(n, dtype=LOG_DTYPE)
    out = KvStore(cfg.n_slots, cfg.ways)
    ci, co = init.c(), out.c()
    st = PredStats()
    rc = lib().or_kv_predict(C.byref(cfg), C.byref(ci), n, _ptr(descs), n_lanes, _ptr(log),
                             C.byref(co), C.byref(st))
    assert rc == 0, rc
    return log, out, st.as_dict()
