"""Pins of the CPU oracle's MemcachedGPU workload (docs/GENERATOR.md
section 4): the preload against its closed form (FIFO eviction per set),
hand-traced GET / PUT effects with test-side digests, per-set clock
conservation over a run, and mutants of a valid history."""
import numpy as np
import pytest

import oracle
from tests import _ref as R

M64 = R.M64


def key16_ref(k):
    a, b = R.mix64(k), R.mix64(k ^ 0x5555555555555555)
    return [a & 0xFFFFFFFF, a >> 32, b & 0xFFFFFFFF, b >> 32]


def set_ref(k, n_sets):
    return (R.mix64(k ^ 0xA5A5A5A5A5A5A5A5) * n_sets) >> 64


def preload_val_ref(k):
    out = []
    for j in range(4):
        x = R.mix64(((k << 2) | j) ^ 0x3C3C3C3C3C3C3C3C)
        out += [x & 0xFFFFFFFF, x >> 32]
    return out


def dword(item, w, word):
    return R.mix64((int(item) << 35) ^ (int(w) << 32) ^ int(word))


def d32(item, v):
    return R.mix64((int(item) << 32) ^ (int(v) & 0xFFFFFFFF))


def test_key_and_set_functions():
    for k in (0, 1, 12345, 4_194_303):
        assert oracle.key16(k).tolist() == key16_ref(k)
        assert oracle.kv_set(k, 262_144) == set_ref(k, 262_144)


@pytest.mark.parametrize("S,A,n_keys", [(64, 4, 64), (256, 16, 300), (1 << 12, 16, 1 << 12)])
def test_preload_closed_form(S, A, n_keys):
    """With no GET touching LRU, each set's PUTs evict first-in-first-out:
    the q-th key mapped to a set lands in way q mod A, carries LRU stamp
    q + 1, and the set clock ends at the number of keys mapped to it."""
    cfg = oracle.kv_cfg(S, A, n_keys=n_keys)
    st = oracle.kv_preload(cfg)
    T = S // A
    keys = np.zeros((S, 4), dtype=np.uint32)
    vals = np.zeros((S, 8), dtype=np.uint32)
    lru = np.zeros(S, dtype=np.uint32)
    count = [0] * T
    for k in range(n_keys):
        t = set_ref(k, T)
        q = count[t]
        count[t] += 1
        slot = t * A + q % A
        keys[slot] = key16_ref(k)
        vals[slot] = preload_val_ref(k)
        lru[slot] = q + 1
    assert np.array_equal(st.clocks, np.array(count, dtype=np.uint32))
    assert np.array_equal(st.keys, keys) and np.array_equal(st.vals, vals) and np.array_equal(st.lru, lru)


def hand_store():
    """S=4 slots, A=2 ways (2 sets).  Keys 0..3 with their real set mapping,
    placed by hand."""
    cfg = oracle.kv_cfg(4, 2, n_keys=8, n_versions=2)
    st = oracle.KvStore(4, 2)
    return cfg, st


def test_get_hit_miss_and_empty_stop():
    cfg, st = hand_store()
    # find two keys of set 0 and one of set 1
    ks0 = [k for k in range(64) if set_ref(k, 2) == 0][:3]
    ks1 = [k for k in range(64) if set_ref(k, 2) == 1][:1]
    st.keys[0], st.keys[1] = key16_ref(ks0[0]), key16_ref(ks0[1])
    st.vals[1] = list(range(100, 108))
    st.lru[:] = [1, 2, 0, 0]
    st.clocks[:] = [2, 0]
    descs = np.zeros(3, dtype=oracle.KV_DESC_DTYPE)
    descs["key"] = [ks0[1], ks0[2], ks1[0]]
    # GET ks0[1]: reads key slot0 (miss), key slot1 (hit), value slot 1 -> aux 2
    rd_hit = sum(dword(0, w, x) for w, x in enumerate(st.keys[0])) + \
        sum(dword(1, w, x) for w, x in enumerate(st.keys[1])) + \
        sum(dword(4 + 1, w, x) for w, x in enumerate(st.vals[1]))
    # GET ks0[2]: both keys read, no match, set full -> miss
    rd_miss = sum(dword(s, w, x) for s in (0, 1) for w, x in enumerate(st.keys[s]))
    # GET ks1[0]: slot 2 empty -> stop after one read
    rd_empty = sum(dword(2, w, 0) for w in range(4))
    log = np.zeros(3, dtype=R.LOG_DTYPE)
    for t, (rd, aux) in enumerate(((rd_hit, 2), (rd_miss, 0), (rd_empty, 0))):
        log[t] = R.log_record(t, 0, 0, 1, rd & M64, aux)
    assert oracle.kv_check(cfg, st, descs, log)["ok"]
    bad = log.copy()
    bad[0]["aux"] = 1
    assert oracle.kv_check(cfg, st, descs, bad)["code"] == "READ"


def test_put_lru_eviction_and_in_place_update():
    """Set 0 full with keys a (LRU 1) and b (LRU 2).  PUT c evicts the least
    recently updated way (a, way 0); then PUT b updates b in place."""
    cfg, st = hand_store()
    a, b, c = [k for k in range(64) if set_ref(k, 2) == 0][:3]
    st.keys[0], st.keys[1] = key16_ref(a), key16_ref(b)
    st.lru[:] = [1, 2, 0, 0]
    st.clocks[:] = [2, 0]
    descs = np.zeros(2, dtype=oracle.KV_DESC_DTYPE)
    descs[0]["is_update"], descs[0]["key"], descs[0]["val"] = 1, c, list(range(8))
    descs[1]["is_update"], descs[1]["key"], descs[1]["val"] = 1, b, list(range(10, 18))
    S = 4
    # tx0: reads key0, key1 (no match, no empty), lru0, lru1, clock0 -> victim 0
    rd0 = sum(dword(s, w, x) for s in (0, 1) for w, x in enumerate(st.keys[s])) + \
        d32(2 * S + 0, 1) + d32(2 * S + 1, 2) + d32(3 * S + 0, 2)
    wd0 = sum(dword(0, w, x) for w, x in enumerate(key16_ref(c))) + \
        sum(dword(S + 0, w, x) for w, x in enumerate(range(8))) + d32(2 * S + 0, 3) + d32(3 * S + 0, 3)
    # tx1 (after tx0): key0 = c (no), key1 = b (match) -> victim 1, clock 3 -> 4
    rd1 = sum(dword(0, w, x) for w, x in enumerate(key16_ref(c))) + \
        sum(dword(1, w, x) for w, x in enumerate(key16_ref(b))) + d32(3 * S + 0, 3)
    wd1 = sum(dword(1, w, x) for w, x in enumerate(key16_ref(b))) + \
        sum(dword(S + 1, w, x) for w, x in enumerate(range(10, 18))) + d32(2 * S + 1, 4) + d32(3 * S + 0, 4)
    log = np.zeros(2, dtype=R.LOG_DTYPE)
    log[0] = R.log_record(0, 0, 1, 1, rd0 & M64, wd0 & M64)
    log[1] = R.log_record(1, 1, 2, 1, rd1 & M64, wd1 & M64)
    fin = st.copy()
    fin.keys[0] = key16_ref(c)
    fin.vals[0] = list(range(8))
    fin.vals[1] = list(range(10, 18))
    fin.lru[:] = [3, 4, 0, 0]
    fin.clocks[:] = [4, 0]
    rep = oracle.kv_check(cfg, st, descs, log, final=fin,
                          claims=dict(committed_update=2, committed_ro=0, gts_final=2, total_aborts=0))
    assert rep["ok"], rep
    # tx1 with snapshot 0 read stale state: it read key0/clock written by CTS 1
    stale = log.copy()
    stale[1]["snapshot"] = 0
    assert oracle.kv_check(cfg, st, descs, stale)["code"] == "VALIDITY"
    # swapped CTS: tx1 first would read key0 = a, not c
    sw = log.copy()
    sw[0]["cts"], sw[1]["cts"] = 2, 1
    sw[1]["snapshot"] = 0
    assert not oracle.kv_check(cfg, st, descs, sw)["ok"]


def test_predictor_clock_conservation_and_last_writer():
    """Over a zipf run: each set clock = keys preloaded into it + PUTs to it;
    every present key's value is the one its last committed PUT wrote (or
    its preload value); keys within a set stay distinct."""
    S, A = 1 << 10, 8
    cfg = oracle.kv_cfg(S, A, n_keys=S, p_update_ppm=200_000)
    init = oracle.kv_preload(cfg)
    d = oracle.kv_gen(cfg, 5, 6000)
    log, fin, ps = oracle.kv_predict(cfg, init, d)
    T = S // A
    puts = np.bincount([set_ref(int(k), T) for k in d["key"][d["is_update"] == 1]], minlength=T)
    pre = np.bincount([set_ref(k, T) for k in range(S)], minlength=T)
    assert np.array_equal(fin.clocks, (pre + puts).astype(np.uint32))
    order = np.argsort(log["cts"])
    last = {}
    for t in order:
        if d["is_update"][t]:
            last[int(d["key"][t])] = d["val"][t]
    slot_of = {tuple(fin.keys[i]): i for i in range(S) if fin.keys[i].any()}
    for k, v in last.items():
        i = slot_of.get(tuple(key16_ref(k)))
        if i is not None:
            assert fin.vals[i].tolist() == v.tolist()
    for t in range(T):
        ks = [tuple(x) for x in fin.keys[t * A:(t + 1) * A] if x.any()]
        assert len(ks) == len(set(ks))
    claims = dict(committed_update=ps["committed_update"], committed_ro=ps["committed_ro"],
                  gts_final=ps["gts_final"], total_aborts=ps["aborts_preval"])
    assert oracle.kv_check(cfg, init, d, log, final=fin, claims=claims)["ok"]
    assert ps["aborts_preval"] > 0     # PUTs to one set always conflict on its clock


def test_predictor_mutants_rejected():
    S, A = 256, 4
    cfg = oracle.kv_cfg(S, A, n_keys=S, p_update_ppm=300_000)
    init = oracle.kv_preload(cfg)
    d = oracle.kv_gen(cfg, 9, 2000)
    log, fin, _ = oracle.kv_predict(cfg, init, d)
    upd = np.nonzero(d["is_update"] == 1)[0]
    ro = np.nonzero(d["is_update"] == 0)[0]
    for field, t in (("read_digest", upd[3]), ("aux", upd[4]), ("read_digest", ro[5]), ("aux", ro[6])):
        bad = log.copy()
        bad[t][field] = (int(bad[t][field]) + 1) & M64
        assert not oracle.kv_check(cfg, init, d, bad)["ok"]
    bad = fin.copy()
    bad.clocks[0] += 1
    assert oracle.kv_check(cfg, init, d, log, final=bad)["code"] == "RING"
