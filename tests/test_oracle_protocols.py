"""Brute-force checks of two protocol variants before (or instead of) GPU
code, on a small abstract machine in the style of test_oracle_bruteforce
(every interleaving of atomic steps, states deduplicated):

1. Blind-write elision (NEXT-4): "if one can a priori exclude ...
   the possibility of blind writes, this additional validation step can be
   safely omitted."  With transfers only (every write is preceded by a read
   of the item) and the write-write check dropped, every reachable history
   is accepted by the oracle; with a blind write in the mix the same
   elision reaches histories whose final store contradicts the commit
   order -- the negative control the library's refusal (KV: EINVAL) rests on.

2. Item-partitioned commit over two servers (NEXT-3, DESIGN.md
   11): server A owns the even items, server B the odd ones; a transaction
   PREPAREs at each server owning one of its items (validate its part
   against that server's records after the snapshot and against the other
   in-flight prepares, then mark its items pending), takes its CTS from one
   global counter only once every server voted yes, and RECORDs its
   write-set at each server.  Every interleaving of those steps is accepted
   by the oracle; without the pending marks some history is not.  The
   same holds with the GPU's finer lock-free steps (a claim per item, then
   the check; record, then release) -- and not with release before record.

Test infrastructure only: the machine is test-side Python, the checker is
oracle/ (bank_check) plus an independent commit-order replay.
"""

import numpy as np
import pytest

import oracle
from tests import _ref as R

EMPTY = R.EMPTY


def lookup(ring, s):
    best = None
    for ts, v in ring:
        if ts != EMPTY and ts <= s and (best is None or ts > best[0]):
            best = (ts, v)
    return best


def install(ring, cts, v):
    ring = list(ring)
    victim = next((j for j, (ts, _) in enumerate(ring) if ts == EMPTY), None)
    if victim is None:
        victim = min(range(len(ring)), key=lambda j: ring[j][0])
    ring[victim] = (cts, v)
    return tuple(ring)


def blind(x, v):
    """A blind write: WS = {x} with value v, RS = {} (not a bank transaction)."""
    return dict(kind="blind", x=x, v=v)


def rs_ws(d):
    if d.get("kind") == "blind":
        return (), (d["x"],)
    if d["is_update"]:
        return (d["src"], d["dst"]), (d["src"], d["dst"])
    return tuple((d["start"] + j) % 4 for j in range(d["len"])), ()


class Machine:
    """One agent per transaction.  servers = 1: one commit step validating
    against the list ATR (`ww` = also validate the write-set);
    servers = 2: PREPARE at every owning server, DECIDE (global CTS),
    RECORD at every owning server (`pending` = in-flight prepares block)."""

    def __init__(self, k, init, descs, ww=True, servers=1, pending=True, max_att=2, claims=False):
        self.K, self.init, self.d = k, init, descs
        self.ww, self.S, self.pending, self.max_att = ww, servers, pending, max_att
        self.claims = claims  # the GPU's lock-free PREPARE: per-item CLAIM steps, then CHECK; REC then REL
        self.ops = []
        for t, d in enumerate(descs):
            rs, ws = rs_ws(d)
            ops = [("BEGIN",)] + [("READ", x) for x in rs]
            if ws:
                owners = sorted({x % servers for x in rs + ws})
                if servers == 1:
                    ops.append(("COMMIT",))
                elif claims:
                    for o in owners:
                        ops += [("CLAIM", o, x) for x in self.items_at(t, o)] + [("CHECK", o)]
                    ops += [("DECIDE",)]
                    for o in owners:
                        ops += [("REC", o), ("REL", o)]
                else:
                    ops += [("PREP", o) for o in owners] + [("DECIDE",)] + [("REC", o) for o in owners]
                ops += [("WB", x) for x in ws] + [("PUBLISH",)]
            ops.append(("END",))
            self.ops.append(ops)

    def initial(self):
        rings = tuple(tuple([(0, v)] + [(EMPTY, 0)] * (self.K - 1)) for v in self.init)
        # tx: (pc, status, snapshot, reads, cts, attempts, votes); status run/fail/ok/done
        txs = tuple((0, "run", 0, (), 0, 0, ()) for _ in self.d)
        atr = tuple(() for _ in range(self.S))    # per server: ((cts, items), ...)
        pend = tuple(() for _ in range(self.S))   # per server: ((tx, items), ...)
        return (0, 0, atr, pend, rings, txs)

    def items_at(self, t, srv):
        rs, ws = rs_ws(self.d[t])
        check = set(rs) | (set(ws) if self.ww else set())
        return tuple(sorted(x for x in check if x % self.S == srv))

    def step(self, st, t):
        gts, tail, atr, pend, rings, txs = st
        pc, stat, s, reads, cts, att, votes = txs[t]
        ops = self.ops[t]
        if stat == "done":
            return None
        op = ops[pc]
        d = self.d[t]
        rs, ws = rs_ws(d)
        kind = op[0]
        if kind == "BEGIN":
            s, stat, reads, cts, votes, att = gts, "run", (), 0, (), att + 1
        elif kind == "READ":
            if stat == "run":
                v = lookup(rings[op[1]], s)
                if v is None:
                    stat = "fail"
                else:
                    reads = reads + (v[1],)
        elif kind == "COMMIT":
            if stat == "run":
                mine = set(rs) | (set(ws) if self.ww else set())
                if any(c > s and set(w) & mine for c, w in atr[0]):
                    stat = "fail"
                else:
                    tail += 1
                    cts, stat = tail, "ok"
                    atr = (atr[0] + ((cts, tuple(sorted(ws))),),)
        elif kind == "PREP":
            srv = op[1]
            if stat == "run":
                mine = set(self.items_at(t, srv))
                wsx = tuple(sorted(x for x in ws if x % self.S == srv))
                bad = any(c > s and set(w) & mine for c, w in atr[srv])
                if self.pending:
                    bad = bad or any(set(w) & mine for u, w in pend[srv] if u != t)
                if bad:
                    stat = "fail"
                else:
                    votes = votes + (srv,)
                    pend = pend[:srv] + (pend[srv] + ((t, wsx),),) + pend[srv + 1:]
        elif kind == "CLAIM":  # atomicOr of one pending bit; a taken bit fails the lane here
            srv, x = op[1], op[2]
            if stat == "run":
                if any(x in w for u, w in pend[srv] if u != t):
                    stat = "fail"
                    pend = pend[:srv] + (tuple(e for e in pend[srv] if e[0] != t),) + pend[srv + 1:]
                else:
                    pend = pend[:srv] + (pend[srv] + ((t, (x,)),),) + pend[srv + 1:]
        elif kind == "CHECK":  # after the claims: the records after the snapshot
            srv = op[1]
            if stat == "run":
                mine = set(self.items_at(t, srv))
                if any(c > s and set(w) & mine for c, w in atr[srv]):
                    stat = "fail"
                    pend = pend[:srv] + (tuple(e for e in pend[srv] if e[0] != t),) + pend[srv + 1:]
                else:
                    votes = votes + (srv,)
        elif kind == "REL":
            srv = op[1]
            pend = pend[:srv] + (tuple(e for e in pend[srv] if e[0] != t),) + pend[srv + 1:]
        elif kind == "DECIDE":
            if stat == "run":
                tail += 1
                cts, stat = tail, "ok"
            else:  # abort: release this transaction's prepares
                pend = tuple(tuple(e for e in p if e[0] != t) for p in pend)
        elif kind == "REC":
            srv = op[1]
            if stat == "ok":
                wsx = tuple(sorted(x for x in ws if x % self.S == srv))
                atr = atr[:srv] + (atr[srv] + ((cts, wsx),),) + atr[srv + 1:]
                if not self.claims:  # (claims: released by the REL step after the record)
                    pend = pend[:srv] + (tuple(e for e in pend[srv] if e[0] != t),) + pend[srv + 1:]
        elif kind == "WB":
            if stat == "ok":
                x = op[1]
                if d.get("kind") == "blind":
                    nv = d["v"]
                else:
                    vs, vd = reads
                    nv = R.s32(vs - d["amt"]) if x == d["src"] else R.s32(vd + d["amt"])
                rings = rings[:x] + (install(rings[x], cts, nv),) + rings[x + 1:]
        elif kind == "PUBLISH":
            if stat == "ok":
                if gts != cts - 1:
                    return None  # blocked until every earlier commit is published
                gts = cts
        elif kind == "END":
            if stat == "ok" or (stat == "run" and not ws):
                stat = "done"
            else:
                if att >= self.max_att:
                    return "dead"
                txs = txs[:t] + ((0, "run", s, (), 0, att, ()),) + txs[t + 1:]
                return (gts, tail, atr, pend, rings, txs)
        txs = txs[:t] + ((pc + 1, stat, s, reads, cts, att, votes),) + txs[t + 1:]
        return (gts, tail, atr, pend, rings, txs)

    def explore(self):
        seen, stack, finals = set(), [self.initial()], set()
        while stack:
            st = stack.pop()
            if st in seen:
                continue
            seen.add(st)
            moved = False
            for t in range(len(self.d)):
                nx = self.step(st, t)
                if nx is None or nx == "dead":
                    continue
                moved = True
                stack.append(nx)
            if not moved and all(x[1] == "done" for x in st[5]):
                finals.add(st)
        return finals


def replay_ok(m, st):
    """Independent check: apply the committed transactions in CTS order
    (read-only ones at their snapshot) -- every read must see the replayed
    state and the final newest versions must equal the replayed store."""
    gts, tail, atr, pend, rings, txs = st
    state = list(m.init)
    snaps = {0: tuple(state)}
    order = sorted((t for t in range(len(m.d)) if rs_ws(m.d[t])[1]), key=lambda t: txs[t][4])
    for t in order:
        d = m.d[t]
        rs, ws = rs_ws(d)
        if tuple(state[x] for x in rs) != txs[t][3]:
            return False
        if d.get("kind") == "blind":
            state[d["x"]] = d["v"]
        else:
            state[d["src"]] = R.s32(state[d["src"]] - d["amt"])
            state[d["dst"]] = R.s32(state[d["dst"]] + d["amt"])
        snaps[txs[t][4]] = tuple(state)
    for t in range(len(m.d)):
        rs, ws = rs_ws(m.d[t])
        if not ws and tuple(snaps[txs[t][2]][x] for x in rs) != txs[t][3]:
            return False
    newest = [max((e for e in ring if e[0] != EMPTY), key=lambda e: e[0])[1] for ring in rings]
    return newest == state


def bank_history(m, st):
    gts, tail, atr, pend, rings, txs = st
    recs = []
    for t, (_, _, s, reads, cts, att, _) in enumerate(txs):
        d = m.d[t]
        if d["is_update"]:
            recs.append(R.update_record(t, d, s, cts, att, *reads))
        else:
            recs.append(R.rot_record(t, d, 4, s, att, list(reads)))
    log = np.array(recs, dtype=R.LOG_DTYPE)
    ring_arr = np.array([R.pack(ts, v) for ring in rings for ts, v in ring], dtype=np.uint64)
    return log, ring_arr, gts


def oracle_accepts(m, st):
    log, rings, gts = bank_history(m, st)
    cfg = oracle.bank_cfg(4, m.K, ro_reads=0)
    C = sum(d["is_update"] for d in m.d)
    return oracle.bank_check(cfg, m.init, R.desc_array(m.d), log, rings=rings,
                             claims=dict(committed_update=C, committed_ro=len(m.d) - C, gts_final=gts,
                                         total_aborts=int((log["attempts"] - 1).sum())))["ok"]


TRANSFERS = {
    "chain": [R.transfer(0, 1, 5), R.transfer(1, 2, 7), R.rot(0, 4)],
    "same_pair": [R.transfer(0, 1, 5), R.transfer(1, 0, 3), R.rot(1, 2)],
    "three": [R.transfer(0, 1, 1), R.transfer(1, 2, 2), R.transfer(2, 3, 3)],
}


@pytest.mark.parametrize("k", [1, 2])
@pytest.mark.parametrize("name", sorted(TRANSFERS))
def test_ww_elision_is_safe_without_blind_writes(name, k):
    m = Machine(k, [1000] * 4, TRANSFERS[name], ww=False)
    finals = m.explore()
    assert finals
    for st in finals:
        assert replay_ok(m, st), (name, k)
        assert oracle_accepts(m, st), (name, k)


@pytest.mark.parametrize("k", [1])
def test_ww_elision_with_blind_writes_is_caught(k):
    """Two concurrent blind writers of item 0 (and a transfer reading it):
    with the write-write check they are ordered; without it their
    write-backs can land out of commit order, and the later install of the
    older version recycles the newer one (the one-version ring here; the
    head of the paper's VBox list, in general) -- a reader or the
    final store then sees the older write and the replay rejects the
    history.  (With K >= 2 ts-tagged slots the newest version survives a
    reordered install; what breaks in this build is then the item-indexed
    ATR's lastw, which the clients' plain stores keep exact only because
    two writers of an item are never concurrent -- server.cuh.)"""
    descs = [blind(0, 11), blind(0, 22), R.transfer(0, 1, 5)]
    full = Machine(k, [1000] * 4, descs, ww=True)
    assert all(replay_ok(full, st) for st in full.explore())
    elided = Machine(k, [1000] * 4, descs, ww=False)
    finals = elided.explore()
    assert any(not replay_ok(elided, st) for st in finals)


SPANNING = {
    # transfers 0->1 and 1->2 span both servers (even/odd items)
    "chain": [R.transfer(0, 1, 5), R.transfer(1, 2, 7), R.rot(0, 4)],
    "cross": [R.transfer(0, 1, 5), R.transfer(2, 3, 7), R.transfer(1, 2, 3)],
    "same_pair": [R.transfer(0, 1, 5), R.transfer(1, 0, 3), R.rot(1, 2)],
}


@pytest.mark.parametrize("k", [1, 2])
@pytest.mark.parametrize("name", sorted(SPANNING))
def test_two_server_commit_is_opaque(name, k):
    m = Machine(k, [1000] * 4, SPANNING[name], servers=2)
    finals = m.explore()
    assert finals
    for st in finals:
        assert replay_ok(m, st), (name, k)
        assert oracle_accepts(m, st), (name, k)
    # every update committed exactly once with CTS 1..C (P:130 across servers)
    C = sum(d["is_update"] for d in SPANNING[name])
    for st in finals:
        assert sorted(x[4] for x in st[5] if x[4]) == list(range(1, C + 1))


@pytest.mark.parametrize("k", [1, 2])
@pytest.mark.parametrize("name", sorted(SPANNING))
def test_two_server_lockfree_claims_are_opaque(name, k):
    """The GPU's server_part.cuh prepares without a lock: one atomic claim
    per item (increasing order), then the record check; a decide records
    first and releases after.  Every interleaving of those finer steps is
    accepted too, with CTS 1..C."""
    m = Machine(k, [1000] * 4, SPANNING[name], servers=2, claims=True)
    finals = m.explore()
    assert finals
    C = sum(d["is_update"] for d in SPANNING[name])
    for st in finals:
        assert replay_ok(m, st), (name, k)
        assert oracle_accepts(m, st), (name, k)
        assert sorted(x[4] for x in st[5] if x[4]) == list(range(1, C + 1))


def test_lockfree_release_before_record_is_caught():
    """Negative control for the decide's order: releasing the bits before
    recording the write-set lets a conflicting prepare slip in between."""
    class Early(Machine):
        def __init__(self, *a, **kw):
            super().__init__(*a, **kw)
            for ops in self.ops:  # swap every (REC o, REL o) pair
                for i in range(len(ops) - 1):
                    if ops[i][0] == "REC" and ops[i + 1][0] == "REL":
                        ops[i], ops[i + 1] = ops[i + 1], ops[i]
    bad = False
    for name in ("chain", "same_pair"):
        m = Early(1, [1000] * 4, SPANNING[name], servers=2, claims=True)
        bad = bad or any(not oracle_accepts(m, st) for st in m.explore())
    assert bad


def test_two_server_commit_needs_pending_marks():
    """Negative control: validating each part only against the records
    already there (no pending marks) lets two conflicting transactions both
    prepare and commit -- the oracle rejects some reachable history."""
    for name in ("chain", "same_pair"):
        m = Machine(2, [1000] * 4, SPANNING[name], servers=2, pending=False)
        finals = m.explore()
        assert any(not oracle_accepts(m, st) for st in finals), name
