"""pin the oracle's replaying checker against brute-force
enumeration of every interleaving of a small abstract CSMV machine.

The machine (test-side model of PAPER.md section III) has atomic steps
  BEGIN      s <- GTS
  READ(x)    newest version of x with ts <= s; none => abort
  COMMIT     server: client pre-validation of the batch, validation
             against ATR entries with CTS > s on RS u WS,
             consecutive CTS for the survivors
  WB(x)      install (CTS, value) over the oldest version
  PUBLISH    blocks until GTS == first CTS - 1, then GTS += n
and read-only transactions run BEGIN, READs and finish.
Agents are client warps: a batch of one or two update transactions sharing a
snapshot, or one read-only transaction.  Aborted transactions retry (bounded).

For every reachable terminal history: (a) the oracle accepts it; (b) its CTS
order (ROTs at their snapshots) is among the serial orders found by trying
every permutation; (c) mutated histories are rejected; and the machine with
validation disabled produces at least one history the oracle rejects.
"""
import itertools

import numpy as np
import pytest

import oracle
from tests import _ref as R

MAX_ATTEMPTS = 2


def _lookup(ring, s):
    best = None
    for ts, v in ring:
        if ts != R.EMPTY and ts <= s and (best is None or ts > best[0]):
            best = (ts, v)
    return best


def _install(ring, cts, v):
    ring = list(ring)
    victim = next((j for j, (ts, _) in enumerate(ring) if ts == R.EMPTY), None)
    if victim is None:
        victim = min(range(len(ring)), key=lambda j: ring[j][0])
    ring[victim] = (cts, v)
    return tuple(ring)


class Machine:
    def __init__(self, n_items, k, init, descs, agents, validate=True):
        self.N, self.K, self.init, self.d, self.agents = n_items, k, init, descs, agents
        self.validate = validate
        # ops per agent
        self.ops = []
        for txs in agents:
            ops = [("BEGIN",)]
            for t in txs:
                for x in self.items(t):
                    ops.append(("READ", t, x))
            if self.d[txs[0]]["is_update"]:
                ops.append(("COMMIT",))
                for t in txs:
                    ops += [("WB", t, self.d[t]["src"]), ("WB", t, self.d[t]["dst"])]
                ops.append(("PUBLISH",))
            ops.append(("END",))
            self.ops.append(ops)

    def items(self, t):
        d = self.d[t]
        if d["is_update"]:
            return [d["src"], d["dst"]]
        return [(d["start"] + j) % self.N for j in range(d["len"])]

    def initial(self):
        rings = tuple(tuple([(0, v)] + [(R.EMPTY, 0)] * (self.K - 1)) for v in self.init)
        # per tx: (status, snapshot, reads, cts, attempts); status: idle/run/fail/ok/done
        txs = tuple(("idle", 0, (), 0, 0) for _ in self.d)
        agents = tuple((0, 0, 0) for _ in self.agents)  # (pc, snapshot, cts_base/n packed)
        return (0, 0, (), rings, agents, txs, 0)  # GTS, tail, ATR, rings, agents, txs, misses

    def step(self, st, a):
        gts, tail, atr, rings, agents, txs, misses = st
        pc, s, nb = agents[a]
        ops = self.ops[a]
        if pc >= len(ops):
            return None
        op = ops[pc]
        txs = list(txs)
        mine = self.agents[a]
        live = [t for t in mine if txs[t][0] != "done"]
        if not live:
            return None
        kind = op[0]
        if kind == "BEGIN":
            s = gts
            for t in live:
                _, _, _, _, att = txs[t]
                txs[t] = ("run", s, (), 0, att + 1)
        elif kind == "READ":
            t, x = op[1], op[2]
            if txs[t][0] == "run":
                v = _lookup(rings[x], s)
                if v is None:
                    txs[t] = ("fail",) + txs[t][1:]
                    misses += 1
                else:
                    stt, ss, rd, c, att = txs[t]
                    txs[t] = (stt, ss, rd + (v[1],), c, att)
        elif kind == "COMMIT":
            kept = []
            for t in live:
                if txs[t][0] != "run":
                    continue
                mine_items = set(self.items(t))
                if any(mine_items & set(self.items(u)) for u in kept):   # pre-validation
                    txs[t] = ("fail",) + txs[t][1:]
                    continue
                if self.validate and any(c > s and (set(ws) & mine_items) for c, ws in atr):
                    txs[t] = ("fail",) + txs[t][1:]
                    continue
                kept.append(t)
            for r, t in enumerate(kept):
                stt, ss, rd, _, att = txs[t]
                txs[t] = ("ok", ss, rd, tail + 1 + r, att)
                atr = atr + ((tail + 1 + r, tuple(sorted(set(self.items(t))))),)
            nb = len(kept)
            tail += nb
        elif kind == "WB":
            t, x = op[1], op[2]
            if txs[t][0] == "ok":
                d = self.d[t]
                vs, vd = txs[t][2]
                newv = R.s32(vs - d["amt"]) if x == d["src"] else R.s32(vd + d["amt"])
                rings = list(rings)
                rings[x] = _install(rings[x], txs[t][3], newv)
                rings = tuple(rings)
        elif kind == "PUBLISH":
            if nb:
                base = min(txs[t][3] for t in live if txs[t][0] == "ok")
                if gts != base - 1:
                    return None          # blocked
                gts += nb
        elif kind == "END":
            retry = False
            for t in live:
                stt = txs[t][0]
                if stt in ("ok",) or (stt == "run" and not self.d[t]["is_update"]):
                    txs[t] = ("done",) + txs[t][1:]
                else:                    # failed attempt
                    if txs[t][4] >= MAX_ATTEMPTS:
                        return "dead"
                    retry = True
            nb = 0
            if retry:
                agents = agents[:a] + ((0, s, 0),) + agents[a + 1:]
                return (gts, tail, atr, rings, agents, tuple(txs), misses)
        agents = agents[:a] + ((pc + 1, s, nb),) + agents[a + 1:]
        return (gts, tail, atr, rings, agents, tuple(txs), misses)

    def explore(self):
        seen, stack, finals = set(), [self.initial()], set()
        while stack:
            st = stack.pop()
            if st in seen:
                continue
            seen.add(st)
            moved = False
            for a in range(len(self.agents)):
                nx = self.step(st, a)
                if nx is None:
                    continue
                moved = True
                if nx == "dead":
                    continue
                stack.append(nx)
            if not moved and all(t[0] == "done" for t in st[5]):
                finals.add(st)
        return finals, len(seen)


def history(m, st):
    gts, tail, atr, rings, agents, txs, misses = st
    recs = []
    for t, (stt, s, reads, cts, att) in enumerate(txs):
        d = m.d[t]
        if d["is_update"]:
            recs.append(R.update_record(t, d, s, cts, att, *reads))
        else:
            recs.append(R.rot_record(t, d, m.N, s, att, list(reads)))
    log = np.array(recs, dtype=R.LOG_DTYPE)
    ring_arr = np.array([R.pack(ts, v) for ring in rings for ts, v in ring], dtype=np.uint64)
    return log, ring_arr, gts, misses


def serial_orders_ok(m, txs):
    """Every serial order of the committed updates that reproduces all
    observed reads (ROTs placed at any prefix); return the valid orders."""
    upd = [t for t in range(len(m.d)) if m.d[t]["is_update"]]
    valid = []
    for perm in itertools.permutations(upd):
        state = list(m.init)
        prefixes = [tuple(state)]
        ok = True
        for t in perm:
            d = m.d[t]
            if tuple(txs[t][2]) != (state[d["src"]], state[d["dst"]]):
                ok = False
                break
            state[d["src"]] = R.s32(state[d["src"]] - d["amt"])
            state[d["dst"]] = R.s32(state[d["dst"]] + d["amt"])
            prefixes.append(tuple(state))
        if not ok:
            continue
        for t in range(len(m.d)):
            if not m.d[t]["is_update"]:
                items = m.items(t)
                if not any(tuple(p[x] for x in items) == tuple(txs[t][2]) for p in prefixes):
                    ok = False
        if ok:
            valid.append(perm)
    return valid


SCENARIOS = {
    # name: (n_items, init, descs, agents)
    "conflicting_pair_rot": (4, [1000] * 4, [R.transfer(0, 1, 5), R.transfer(1, 2, 7), R.rot(0, 4)],
                             [[0], [1], [2]]),
    "disjoint_pair_rot": (4, [1000] * 4, [R.transfer(0, 1, 5), R.transfer(2, 3, 7), R.rot(0, 4)],
                          [[0], [1], [2]]),
    "batch_of_two_plus_one": (4, [10, 20, 30, 40],
                              [R.transfer(0, 1, 1), R.transfer(2, 3, 2), R.transfer(1, 2, 3)],
                              [[0, 1], [2]]),
    "batch_internal_conflict": (4, [10, 20, 30, 40],
                                [R.transfer(0, 1, 1), R.transfer(1, 2, 2), R.rot(1, 2)],
                                [[0, 1], [2]]),
    "three_chain": (4, [5, 6, 7, 8], [R.transfer(0, 1, 1), R.transfer(1, 2, 2), R.transfer(2, 3, 3)],
                    [[0], [1], [2]]),
}


@pytest.mark.parametrize("k", [1, 2, 3])
@pytest.mark.parametrize("name", sorted(SCENARIOS))
def test_every_interleaving_accepted(name, k):
    n, init, descs, agents = SCENARIOS[name]
    m = Machine(n, k, init, descs, agents)
    finals, n_states = m.explore()
    assert finals, "no complete history"
    cfg = oracle.bank_cfg(n, k, ro_reads=0)
    darr = R.desc_array(descs)
    max_writes = max(sum(x in (d["src"], d["dst"]) for d in descs if d["is_update"]) for x in range(n))
    for st in finals:
        log, rings, gts, misses = history(m, st)
        C = sum(d["is_update"] for d in descs)
        aborts = int((log["attempts"] - 1).sum())
        rep = oracle.bank_check(cfg, init, darr, log, rings=rings,
                                claims=dict(committed_update=C, committed_ro=len(descs) - C,
                                            gts_final=gts, total_aborts=aborts))
        assert rep["ok"], (name, k, rep)
        # (b) the CTS order is one of the brute-force serial orders
        valid = serial_orders_ok(m, st[5])
        cts_order = tuple(sorted((t for t in range(len(descs)) if descs[t]["is_update"]),
                                 key=lambda t: st[5][t][3]))
        assert cts_order in valid, (name, k, cts_order, valid)
        # P6: enough versions => no version misses
        if k >= 1 + max_writes:
            assert misses == 0
        # (c) mutants: perturb one observed value of each transaction
        for t in range(len(descs)):
            bad = log.copy()
            bad[t]["read_digest"] = (int(bad[t]["read_digest"]) + 1) & R.M64
            assert not oracle.bank_check(cfg, init, darr, bad)["ok"]
        # swapping the CTS of two conflicting updates is rejected
        upd = [t for t in range(len(descs)) if descs[t]["is_update"]]
        for a, b in itertools.combinations(upd, 2):
            if set(m.items(a)) & set(m.items(b)):
                bad = log.copy()
                bad[a]["cts"], bad[b]["cts"] = log[b]["cts"], log[a]["cts"]
                assert not oracle.bank_check(cfg, init, darr, bad)["ok"]


def test_k1_produces_version_misses():
    """With one version per VBox a ROT racing an update can miss."""
    n, init, descs, agents = SCENARIOS["conflicting_pair_rot"]
    finals, _ = Machine(n, 1, init, descs, agents).explore()
    assert any(st[6] > 0 for st in finals)


def test_dropping_validation_is_caught():
    """Negative control: with the server's validation disabled (P:75, P:115
    removed) some reachable history is not opaque and the oracle rejects it."""
    for name in ("conflicting_pair_rot", "three_chain"):
        n, init, descs, agents = SCENARIOS[name]
        m = Machine(n, 3, init, descs, agents, validate=False)
        finals, _ = m.explore()
        cfg = oracle.bank_cfg(n, 3, ro_reads=0)
        darr = R.desc_array(descs)
        rejected = 0
        for st in finals:
            log, rings, gts, _ = history(m, st)
            rep = oracle.bank_check(cfg, init, darr, log, rings=rings)
            if not rep["ok"]:
                rejected += 1
                assert rep["code"] in ("VALIDITY", "READ"), rep
                assert not serial_orders_ok(m, st[5]) or rep["code"] == "VALIDITY"
        assert rejected > 0, name
