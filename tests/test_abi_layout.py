"""The ctypes mirrors in csmv.py match the structs declared in
include/csmv.h field by field (names, order, sizes): the binding is pure
marshalling and must not drift from the C ABI."""
import ctypes
import os
import re

from paper_conf_ipps_nunesc022_b200 import csmv

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def c_struct_fields(name):
    src = open(os.path.join(ROOT, "include", "csmv.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    body = re.search(r"typedef struct %s \{(.*?)\}" % name, src, flags=re.S).group(1)
    out = []
    for decl in body.split(";"):
        decl = decl.strip()
        if not decl:
            continue
        m = re.match(r"(uint64_t|uint32_t)\s+(.*)", decl)
        typ, rest = m.group(1), m.group(2)
        for v in rest.split(","):
            v = v.strip()
            dims = [int(x) if x.isdigit() else {"CSMV_N_ABORT": 5}[x] for x in re.findall(r"\[(\w+)\]", v)]
            n = 1
            for d in dims:
                n *= d
            out.append((v.split("[")[0].strip(), 8 if typ == "uint64_t" else 4, n))
    return out


def test_workload_mirror():
    c = c_struct_fields("csmv_workload")
    py = [(f, 4, 1) for f, _ in csmv._Workload._fields_]
    assert c == py
    assert [f.name for f in __import__("dataclasses").fields(csmv.Workload)] == [f for f, _, _ in c]


def test_stats_mirror():
    c = c_struct_fields("csmv_stats")
    names = [f for f, _ in csmv._Stats._fields_]
    assert names == [n for n, _, _ in c]
    size = sum(s * n for _, s, n in c)
    assert ctypes.sizeof(csmv._Stats) == size


def test_log_record_is_32_bytes():
    assert csmv.LOG_DTYPE.itemsize == 32
    assert [n for n, _, _ in c_struct_fields("csmv_log_rec")] == list(csmv.LOG_DTYPE.names)


def test_trace_record_mirror():
    c = c_struct_fields("csmv_trace_rec")
    assert [n for n, _, _ in c] == list(csmv.TRACE_DTYPE.names)
    assert sum(s * n for _, s, n in c) == csmv.TRACE_DTYPE.itemsize == 80
