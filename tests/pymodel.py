"""Independent pure-Python model of OPS-mode semantics for tiny batches.

Used to pin the C++ oracle (PIN-3 brute force, PIN-6 serial replay).  It
re-derives each txn's read/write/add sets with its own small executor and
decides commits by the *pairwise definition* (SURVEY §8(c) O3):

    commit_r  <=>  for all j < r:  (WS_j | AS_j) & (RS_r | WS_r) == {}
                                   and  WS_j & AS_r == {}
                   and not user_abort_r

-- no minimum marks, no hashing, no per-unit state.  Shares no code with the
oracle or the CUDA path.
"""
from workloads.formats import (SELECT, UPDATE, ADD, INSERT, DELETE, SCAN, COL_COUNT,
                               STATIC, NOT_FOUND, ST_COMMIT, ST_CONFLICT, ST_USER_ABORT)

M = 1 << 64


def wrap(v):
    v %= M
    return v - M if v >= (1 << 63) else v


class Model:
    def __init__(self, descs):
        # descs: table -> (col_group, col_is_add, n_groups)
        self.descs = descs
        self.rows = {t: {} for t in descs}  # t -> key -> list(values)

    def copy(self):
        m = Model(self.descs)
        m.rows = {t: {k: list(v) for k, v in r.items()} for t, r in self.rows.items()}
        return m

    def load(self, t, keys, cols):
        for i, k in enumerate(keys):
            self.rows[t][int(k)] = [int(cols[c][i]) for c in range(len(cols))]

    def exec_op(self, op, arg):
        """Run one op on the current state; return (result, R, W, A, effects, user_abort)."""
        key, kind, t, col, aux = (int(op["key"]), int(op["kind"]), int(op["table"]),
                                  int(op["col"]), int(op["aux"]))
        groups, is_add, ng = self.descs[t]
        rows = self.rows[t]
        R, W, A, eff = set(), set(), set(), []
        ua = False

        def exist(k):
            if ng:
                R.add((t, k, 0))

        if kind == SCAN:
            cnt, s = 0, 0
            for k in range(key, key + aux):
                if k in rows:
                    cnt += 1
                    if col != COL_COUNT:
                        s += rows[k][col]
                    g = groups[col] if (col != COL_COUNT and groups[col] != STATIC) else 0
                    if ng:
                        R.add((t, k, g))
                else:
                    exist(k)
            return (cnt if col == COL_COUNT else wrap(s)), R, W, A, eff, ua
        present = key in rows
        if kind == INSERT:
            if present:
                R.add((t, key, 0))
                return 0, R, W, A, eff, True
            for g in range(ng):
                W.add((t, key, g))
            eff.append(("ins", t, key, [wrap(arg + c) for c in range(len(groups))]))
            return 1, R, W, A, eff, ua
        if not present:
            exist(key)
            return NOT_FOUND, R, W, A, eff, ua
        v = rows[key]
        if kind == SELECT:
            if groups[col] != STATIC:
                R.add((t, key, groups[col]))
            return v[col], R, W, A, eff, ua
        if kind == UPDATE:
            W.add((t, key, groups[col]))
            eff.append(("set", t, key, col, wrap(v[col] + arg)))
            return v[col], R, W, A, eff, ua
        if kind == ADD:
            A.add((t, key, groups[col]))
            eff.append(("add", t, key, col, arg))
            return 0, R, W, A, eff, ua
        if kind == DELETE:
            for g in range(ng):
                W.add((t, key, g))
            eff.append(("del", t, key))
            return 1, R, W, A, eff, ua
        raise ValueError(kind)

    def apply(self, eff):
        for e in eff:
            if e[0] == "set":
                self.rows[e[1]][e[2]][e[3]] = e[4]
            elif e[0] == "add":
                self.rows[e[1]][e[2]][e[3]] = wrap(self.rows[e[1]][e[2]][e[3]] + e[4])
            elif e[0] == "ins":
                self.rows[e[1]][e[2]] = list(e[3])
            elif e[0] == "del":
                del self.rows[e[1]][e[2]]

    def exec_txn(self, batch, r):
        b, e = int(batch["op_begin"][r]), int(batch["op_begin"][r + 1])
        res, R, W, A, eff, ua = [], set(), set(), set(), [], False
        for i in range(b, e):
            x = self.exec_op(batch["ops"][i], int(batch["args"][i]))
            res.append(x[0])
            R |= x[1]
            W |= x[2]
            A |= x[3]
            eff += x[4]
            ua |= x[5]
        return res, R, W, A, eff, ua


def brute_force_batch(model, batch, reorder=False):
    """Pairwise-definition commit decision on snapshot `model`; returns (status, reads, final).

    base rule:   abort iff WAW or RAW against a smaller rank;
    reorder:     abort iff WAW or (RAW and WAR)  (P:237 logical reordering, Aria)."""
    n = len(batch["tid"])
    execs = [model.exec_txn(batch, r) for r in range(n)]  # all against the snapshot
    status = []
    for r in range(n):
        _, Rr, Wr, Ar, _, ua = execs[r]
        waw = raw = war = False
        for j in range(r):
            _, Rj, Wj, Aj, _, _ = execs[j]
            waw |= bool(((Wj | Aj) & Wr) or (Wj & Ar))
            raw |= bool((Wj | Aj) & Rr)
            war |= bool(Rj & (Wr | Ar))
        bad = (waw or (raw and war)) if reorder else (waw or raw)
        status.append(ST_CONFLICT if bad else (ST_USER_ABORT if ua else ST_COMMIT))
    final = model.copy()
    for r in range(n):
        if status[r] == ST_COMMIT:
            final.apply(execs[r][4])
    reads = [x for e in execs for x in e[0]]
    return status, reads, final


def logical_order(model, batch, status):
    """Committed txns in a serial order consistent with snapshot reads: a txn that read a
    unit precedes every committed txn that writes or adds to it (Kahn's algorithm, ties by
    TID).  Raises if the dependency graph has a cycle (the commit rule would be unsound)."""
    import heapq
    com = [r for r in range(len(batch["tid"])) if status[r] == ST_COMMIT]
    sets = {r: model.exec_txn(batch, r) for r in com}
    succ = {r: set() for r in com}
    indeg = {r: 0 for r in com}
    for a in com:
        for b in com:
            if a != b and sets[a][1] & (sets[b][2] | sets[b][3]):  # a reads what b changes
                if b not in succ[a]:
                    succ[a].add(b)
                    indeg[b] += 1
    heap = [r for r in com if indeg[r] == 0]
    heapq.heapify(heap)
    order = []
    while heap:
        r = heapq.heappop(heap)
        order.append(r)
        for b in succ[r]:
            indeg[b] -= 1
            if indeg[b] == 0:
                heapq.heappush(heap, b)
    if len(order) != len(com):
        raise AssertionError("cycle among committed txns")
    return order


def serial_replay(model, batch, status, order=None):
    """Apply committed txns one at a time (TID order, or `order`), each seeing its predecessors."""
    cur = model.copy()
    reads = {}
    if order is None:
        order = [r for r in range(len(batch["tid"])) if status[r] == ST_COMMIT]
    for r in order:
        if status[r] != ST_COMMIT:
            continue
        res, _, _, _, eff, ua = cur.exec_txn(batch, r)
        assert not ua
        reads[r] = res
        cur.apply(eff)
    return reads, cur
