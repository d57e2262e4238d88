"""Pins of the CPU oracle's bank replaying checker and 1-warp predictor
against things other than itself: the hand-computed worked example E0,
closed forms (transfers commute, conservation), the paper's Table V memory
numbers, and hand-traced pre-validation rounds.  (SURVEY.md 8(c) P1-P8, P12.)
"""
import json
import os

import numpy as np
import pytest

import oracle
from tests import _ref as R


def e0(golden_dir):
    with open(os.path.join(golden_dir, "e0_bank.json")) as f:
        g = json.load(f)
    cfg = oracle.bank_cfg(g["n_items"], g["n_versions"], ro_reads=0)
    descs = R.desc_array(g["descs"])
    return g, cfg, descs


def e0_log(g, descs, overrides=None):
    overrides = overrides or {}
    recs = []
    for h in g["history"]:
        h = dict(h, **overrides.get(h["tx"], {}))
        d = g["descs"][h["tx"]]
        if d["is_update"]:
            recs.append(R.update_record(h["tx"], d, h["snapshot"], h["cts"], h["attempts"], *h["reads"]))
        else:
            recs.append(R.rot_record(h["tx"], d, g["n_items"], h["snapshot"], h["attempts"], h["reads"]))
    return np.array(recs, dtype=R.LOG_DTYPE)


def e0_rings(g):
    return np.array([R.pack(ts, v) for ring in g["final_rings"] for ts, v in ring], dtype=np.uint64)


def test_e0_accepted(golden_dir):
    g, cfg, descs = e0(golden_dir)
    log = e0_log(g, descs)
    vals = np.zeros(3 * 4, dtype=np.uint32)
    for h in g["history"]:
        vals[h["tx"] * 4: h["tx"] * 4 + len(h["reads"])] = [R.u32(v) for v in h["reads"]]
    rep = oracle.bank_check(cfg, g["init"], descs, log, vals=vals, max_vals=4, rings=e0_rings(g),
                            claims=dict(committed_update=2, committed_ro=1, gts_final=2, total_aborts=1))
    assert rep["ok"], rep
    assert sum(g["history"][2]["reads"]) == g["rot_sum"] == 4 * 1000


def test_e0_final_state_matches_closed_form(golden_dir):
    g, _, _ = e0(golden_dir)
    final = np.array(g["init"], dtype=np.int64)
    for d in g["descs"]:
        if d["is_update"]:
            final[d["src"]] -= d["amt"]
            final[d["dst"]] += d["amt"]
    assert final.tolist() == g["final_state"]
    newest = [max((s for s in ring if s[0] != R.EMPTY), key=lambda s: s[0])[1] for ring in g["final_rings"]]
    assert newest == g["final_state"]


@pytest.mark.parametrize("mi", [0, 1])
def test_e0_mutants_rejected(golden_dir, mi):
    g, cfg, descs = e0(golden_dir)
    m = g["mutants"][mi]
    ov = {m["field"]: m["value"]}
    if "reads" in m:
        ov["reads"] = m["reads"]
    log = e0_log(g, descs, {m["tx"]: ov})
    rep = oracle.bank_check(cfg, g["init"], descs, log)
    assert not rep["ok"] and rep["code"] == m["expect"], rep


def test_e0_version_miss_reading(golden_dir):
    """After CTS 2's write-back item 1 holds versions {1, 2}: a ROT with
    snapshot 0 finds no version <= 0 and must abort."""
    g, _, _ = e0(golden_dir)
    ring1 = g["final_rings"][1]
    assert not [ts for ts, _ in ring1 if ts != R.EMPTY and ts <= 0]


def _accept(cfg, init, descs, log, **kw):
    return oracle.bank_check(cfg, init, descs, log, **kw)


def test_other_mutants(golden_dir):
    g, cfg, descs = e0(golden_dir)
    good = e0_log(g, descs)
    init = g["init"]
    assert _accept(cfg, init, descs, good)["ok"]
    bad = good.copy(); bad[0]["read_digest"] ^= 1
    assert _accept(cfg, init, descs, bad)["code"] == "READ"
    bad = good.copy(); bad[0]["aux"] += 1
    assert _accept(cfg, init, descs, bad)["code"] == "WRITE"
    bad = good.copy(); bad[0]["cts"], bad[1]["cts"] = 2, 1
    assert not _accept(cfg, init, descs, bad)["ok"]
    bad = good.copy(); bad[1]["cts"] = 3
    assert _accept(cfg, init, descs, bad)["code"] == "CTS"
    bad = good.copy(); bad[2]["cts"] = 2
    assert _accept(cfg, init, descs, bad)["code"] == "CTS"
    bad = good.copy(); bad[2]["attempts"] = 0
    assert _accept(cfg, init, descs, bad)["code"] == "MISSING"
    bad = good.copy(); bad[1]["tx"] = 0
    assert _accept(cfg, init, descs, bad)["code"] == "MISSING"
    bad = good.copy(); bad[2]["snapshot"] = 0   # state at 0 has item0=1000, item1=1000
    assert _accept(cfg, init, descs, bad)["code"] == "READ"
    bad = good.copy(); bad[0]["snapshot"] = 1   # snapshot must precede CTS
    assert _accept(cfg, init, descs, bad)["code"] == "SNAPSHOT"
    rings = e0_rings(g); rings[2] = R.pack(1, 1005)
    assert _accept(cfg, init, descs, good, rings=rings)["code"] == "RING"
    cl = dict(committed_update=2, committed_ro=1, gts_final=2, total_aborts=0)
    assert _accept(cfg, init, descs, good, claims=cl)["code"] == "STATS"


def test_prevalidation_hand_trace():
    """Three transfers in one 3-lane warp round (SURVEY Q5 greedy rule):
    lane0 0->1 kept; lane1 1->2 shares item 1 with lane0 -> dropped; lane2 2->3
    does not meet the kept lane0 -> kept.  Round 1: CTS 1 (lane0), 2 (lane2);
    round 2: lane1 retries with snapshot 2 and gets CTS 3."""
    cfg = oracle.bank_cfg(4, 4, ro_reads=0)
    descs = R.desc_array([R.transfer(0, 1, 10), R.transfer(1, 2, 20), R.transfer(2, 3, 30)])
    init = [100, 100, 100, 100]
    log, _, rings, st = oracle.bank_predict(cfg, init, descs, n_lanes=3)
    assert [tuple(log[i][["snapshot", "cts", "attempts"]]) for i in range(3)] == [(0, 1, 1), (2, 3, 2), (0, 2, 1)]
    assert st["aborts_preval"] == 1 and st["batches"] == 2 and st["rounds"] == 2 and st["gts_final"] == 3
    # t1 read item1 after t0 (110) and item2 after t2 (70): 110-20=90, 70+20=90
    assert log[1]["read_digest"] == R.dig([(1, 110), (2, 70)])
    assert log[1]["aux"] == R.dig([(1, 90), (2, 90)])
    # rings: item2 got CTS 2 (70) then CTS 3 (90); item0 only CTS 1
    rr = rings.reshape(4, 4)
    assert sorted(int(s) >> 32 for s in rr[2] if int(s) >> 32 != R.EMPTY) == [0, 2, 3]
    assert oracle.bank_check(cfg, init, descs, log, rings=rings)["ok"]


def test_prevalidation_lost_lane_does_not_block():
    """Greedy over *kept* lanes: lane1 loses to lane0 and therefore must not
    block lane2 even though lane1 and lane2 share item 2."""
    cfg = oracle.bank_cfg(5, 4, ro_reads=0)
    descs = R.desc_array([R.transfer(0, 1, 1), R.transfer(1, 2, 1), R.transfer(2, 3, 1)])
    log, _, _, st = oracle.bank_predict(cfg, [0] * 5, descs, n_lanes=3)
    assert log[2]["cts"] == 2 and log[1]["cts"] == 3 and st["aborts_preval"] == 1


def _c1_like(n_items=1024, k=4, n_tx=11111, seed=1, ro_period=10, ro_reads=0, lanes=32, dist=0):
    cfg = oracle.bank_cfg(n_items, k, dist=dist, ro_period=ro_period, ro_reads=ro_reads)
    descs = oracle.bank_gen(cfg, seed, n_tx)
    init = np.full(n_items, 1000, dtype=np.int32)
    log, vals, rings, st = oracle.bank_predict(cfg, init, descs, n_lanes=lanes)
    return cfg, descs, init, log, rings, st


def test_c1_predictor_pins():
    cfg, descs, init, log, rings, st = _c1_like()
    upd = descs["is_update"] == 1
    C = int(upd.sum())
    assert C == 10000 and (~upd).sum() == 1111
    # P3: CTS = {1..C}, final GTS = C
    assert sorted(log["cts"][upd].tolist()) == list(range(1, C + 1))
    assert st["gts_final"] == C and st["committed_update"] == C
    # P2: every total-sum ROT sees N*init (P:177-183 conservation)
    assert np.all(log["aux"][~upd].view(np.int64) == 1024 * 1000)
    # P1: the newest version of every item equals the closed form
    final = init.astype(np.int64).copy()
    np.add.at(final, descs["src"][upd], -descs["amt"][upd].astype(np.int64))
    np.add.at(final, descs["dst"][upd], descs["amt"][upd].astype(np.int64))
    rr = rings.reshape(cfg.n_items, cfg.n_versions)
    ts = (rr >> np.uint64(32)).astype(np.int64)
    ts[ts == R.EMPTY] = -1
    newest = (rr[np.arange(cfg.n_items), ts.argmax(axis=1)] & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
    assert np.array_equal(newest, final.astype(np.int32))
    # P12: ring timestamps = the last K CTS that wrote each item
    writers = [[] for _ in range(cfg.n_items)]
    for t in np.nonzero(upd)[0]:
        writers[descs["src"][t]].append(int(log["cts"][t]))
        writers[descs["dst"][t]].append(int(log["cts"][t]))
    for x in range(cfg.n_items):
        expect = sorted([0] + writers[x])[-cfg.n_versions:]
        got = sorted(int(t) for t in ts[x] if t >= 0)
        assert got == expect, x
    # P4: within a round the batch has one snapshot and contiguous CTS
    for s in np.unique(log["snapshot"][upd]):
        c = np.sort(log["cts"][upd & (log["snapshot"] == s)])
        assert np.array_equal(c, np.arange(s + 1, s + 1 + len(c)))
        # and is conflict-free
        items = np.concatenate([descs["src"][upd & (log["snapshot"] == s)], descs["dst"][upd & (log["snapshot"] == s)]])
        assert len(np.unique(items)) == len(items)
    # attempts-1 summed equals the predicted pre-validation aborts
    assert int((log["attempts"] - 1).sum()) == st["aborts_preval"]
    rep = oracle.bank_check(cfg, init, descs, log, rings=rings,
                            claims=dict(committed_update=C, committed_ro=1111, gts_final=C,
                                        total_aborts=st["aborts_preval"]))
    assert rep["ok"], rep


def test_p5_read_only_workload():
    """p_update = 0: the store never changes, all ROTs read init, GTS stays 0."""
    cfg = oracle.bank_cfg(256, 2, p_update_ppm=0, ro_reads=16)
    descs = oracle.bank_gen(cfg, 7, 500)
    assert descs["is_update"].sum() == 0
    init = np.arange(256, dtype=np.int32) * 3 - 100
    log, _, rings, st = oracle.bank_predict(cfg, init, descs)
    assert st["gts_final"] == 0 and st["aborts_preval"] == 0 and st["batches"] == 0
    for t in range(0, 500, 37):
        items = (descs["start"][t] + np.arange(16)) % 256
        assert log["aux"][t].view(np.int64) == init[items].astype(np.int64).sum()


def test_wraparound_int32():
    """Unconditional transfers wrap like int32."""
    cfg = oracle.bank_cfg(2, 2, ro_reads=0)
    descs = R.desc_array([R.transfer(0, 1, 100)])
    init = [-2**31 + 50, 2**31 - 50]
    log, _, rings, _ = oracle.bank_predict(cfg, init, descs, n_lanes=1)
    rr = rings.reshape(2, 2)
    assert R.s32(int(rr[0][1])) == 2**31 - 50 and R.s32(int(rr[1][1])) == -2**31 + 50
    assert oracle.bank_check(cfg, init, descs, log, rings=rings)["ok"]


def test_table_v_memory(golden_dir):
    """P8: 4 + (sizeof(X)+4)*K bytes per item reproduces Table V's
    'Tx. Data Size' row for 6000 int accounts (column '7v' is 5v)."""
    with open(os.path.join(golden_dir, "table_v.json")) as f:
        g = json.load(f)
    for k, kb in zip(g["versions"], g["tx_data_kb"]):
        got = oracle.vbox_bytes(g["n_items"], 4, k) / 1024
        assert round(got) == kb, (k, got, kb)
    assert abs(g["n_items"] * 4 / 1024 - g["pr_stm_kb"]) < 0.02  # 23.4375 vs printed 23.45


@pytest.mark.parametrize("streak,expect,rounds,batches,preval", [
    # (tx: (snapshot, cts, attempts)) hand-traced, see docstring
    (4, {0: (0, 0, 1), 2: (0, 0, 1), 1: (0, 1, 1), 4: (1, 2, 1), 3: (1, 3, 1), 5: (1, 0, 1)}, 2, 2, 0),
    (0, {0: (0, 0, 1), 1: (0, 1, 1), 2: (1, 0, 1), 3: (1, 2, 1), 4: (2, 3, 1), 5: (2, 0, 1)}, 3, 3, 0),
])
def test_ro_streak_hand_trace(streak, expect, rounds, batches, preval):
    """Two lanes; lane0 runs tx 0,2,4 and lane1 tx 1,3,5 (static assignment).
    tx0, tx2, tx5 are read-only, tx1 = 1->2, tx3 = 2->3, tx4 = 0->1.
    A round reads the pending updates first, then runs read-only
    transactions (with ro_streak > 0 a lane runs ahead of its pending update).
    streak 4: round 1 (s=0) lane1's tx1 commits (CTS 1) while lane0 runs ROTs
    0 and 2 and stops at tx4; round 2 (s=1) tx4 (items 0,1) and tx3 (items
    2,3) are disjoint and commit as one batch (CTS 2, 3) while lane1 runs
    the ROT tx5 ahead of its pending tx3, at s=1.
    streak 0 (one tx per lane per round): rounds (tx0,tx1), (tx2,tx3), (tx4,tx5)."""
    cfg = oracle.bank_cfg(4, 4, ro_reads=2, ro_streak=streak)
    descs = R.desc_array([R.rot(0, 2), R.transfer(1, 2, 5), R.rot(1, 2), R.transfer(2, 3, 5),
                          R.transfer(0, 1, 5), R.rot(2, 2)])
    log, _, rings, st = oracle.bank_predict(cfg, [10, 20, 30, 40], descs, n_lanes=2)
    got = {t: tuple(int(v) for v in log[t][["snapshot", "cts", "attempts"]]) for t in range(6)}
    assert got == expect
    assert (st["rounds"], st["batches"], st["aborts_preval"]) == (rounds, batches, preval)
    assert oracle.bank_check(cfg, [10, 20, 30, 40], descs, log, rings=rings)["ok"]
