"""Test-side helpers: an independent Python spelling of the digest of
docs/GENERATOR.md section 5 (pinned to the published splitmix64 vector in
test_generator.py) and history builders used by the oracle pin tests.

Nothing here is imported by the product package or by oracle/.
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15
EMPTY = 0xFFFFFFFF

LOG_DTYPE = np.dtype([("tx", "<u4"), ("snapshot", "<u4"), ("cts", "<u4"),
                      ("attempts", "<u4"), ("read_digest", "<u8"), ("aux", "<u8")])
BANK_DESC_DTYPE = np.dtype([("is_update", "<u4"), ("src", "<u4"), ("dst", "<u4"),
                            ("amt", "<i4"), ("start", "<u4"), ("len", "<u4")])


def mix64(x: int) -> int:
    z = (int(x) + GOLDEN) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def u32(v: int) -> int:
    return v & 0xFFFFFFFF


def s32(v: int) -> int:
    v &= 0xFFFFFFFF
    return v - (1 << 32) if v >= (1 << 31) else v


def dig(items_vals) -> int:
    """Read/write digest: sum of mix64((item << 32) ^ u32(val)) mod 2^64."""
    return sum(mix64((x << 32) ^ u32(v)) for x, v in items_vals) & M64


def pack(ts: int, v: int) -> int:
    return (ts << 32) | u32(v)


def transfer(src, dst, amt):
    return dict(is_update=1, src=src, dst=dst, amt=amt, start=0, len=0)


def rot(start, length):
    return dict(is_update=0, src=0, dst=0, amt=0, start=start, len=length)


def desc_array(descs) -> np.ndarray:
    a = np.zeros(len(descs), dtype=BANK_DESC_DTYPE)
    for i, d in enumerate(descs):
        for k, v in d.items():
            a[i][k] = v
    return a


def log_record(tx, snapshot, cts, attempts, read_digest, aux):
    r = np.zeros(1, dtype=LOG_DTYPE)[0]
    r["tx"], r["snapshot"], r["cts"], r["attempts"] = tx, snapshot, cts, attempts
    r["read_digest"], r["aux"] = read_digest & M64, aux & M64
    return r


def update_record(tx, d, snapshot, cts, attempts, v_src, v_dst):
    rd = dig([(d["src"], v_src), (d["dst"], v_dst)])
    wd = dig([(d["src"], v_src - d["amt"]), (d["dst"], v_dst + d["amt"])])
    return log_record(tx, snapshot, cts, attempts, rd, wd)


def rot_record(tx, d, n_items, snapshot, attempts, values):
    items = [(d["start"] + j) % n_items for j in range(d["len"])]
    rd = dig(zip(items, values))
    return log_record(tx, snapshot, 0, attempts, rd, sum(values) & M64)
