"""Seeded synthetic YCSB workload (inputs only; no method arithmetic).

Shape of the paper's YCSB runs (Zipfian keys, 10 ops per
txn, 10^4..10^7 rows) and of BASELINE.json configs[0] / configs[2]:
  * table ``usertable`` (table id 0): keys 0..N-1, F=10 int64 fields,
    initial value ``splitmix64(key*16+f) & 0xFFFFFFFF``;
  * every txn has ``ops_per_txn`` distinct keys drawn Zipf(theta) by exact
    inverse CDF over popularity ranks, ranks scrambled to keys by
    ``key = (a*rank + b) mod N`` (gcd(a, N) = 1) so hot keys spread over the
    key space;
  * YCSB-A mix: SELECT 50% / UPDATE(+U[1,1000]) 50%, field U[0,F).
"""
import math
import numpy as np

from .formats import OP_DTYPE, SELECT, UPDATE, SCAN, INSERT, KEY_EMPTY

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x):
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


_CDF_CACHE = {}


def zipf_cdf(n, theta):
    key = (n, theta)
    if key not in _CDF_CACHE:
        w = np.arange(1, n + 1, dtype=np.float64) ** (-theta)
        c = np.cumsum(w)
        c /= c[-1]
        _CDF_CACHE.clear()
        _CDF_CACHE[key] = c
    return _CDF_CACHE[key]


def _coprime_multiplier(n, seed):
    a = int(0x9E3779B1 + 2 * seed) % max(n, 1)
    a = max(a, 1)
    while math.gcd(a, n) != 1:
        a += 1
    return a


class YcsbWorkload:
    TABLE = 0

    def __init__(self, n_rows, n_fields=10, theta=0.99, ops_per_txn=10, read_frac=0.5,
                 seed=0x17C0, scan_frac=0.0, insert_frac=0.0, max_scan_len=10, read_latest=False,
                 sparse_keys=False):
        self.n_rows = int(n_rows)
        self.n_fields = int(n_fields)
        self.theta = float(theta)
        self.ops_per_txn = int(ops_per_txn)
        self.read_frac = float(read_frac)
        self.scan_frac = float(scan_frac)
        self.insert_frac = float(insert_frac)
        self.max_scan_len = int(max_scan_len)
        self.seed = int(seed)
        self.a = _coprime_multiplier(self.n_rows, self.seed)
        self.b = (self.seed * 7919) % self.n_rows
        self.next_insert_key = self.n_rows
        self.read_latest = bool(read_latest)
        # sparse_keys: row k is stored under the u64 key splitmix64(k) (a bijection), so keys are
        # scattered over 2^64 and every lookup goes through the PK hash index instead of the
        # dense key -> row arithmetic; point ops only (no SCAN / INSERT)
        self.sparse_keys = bool(sparse_keys)
        assert not (self.sparse_keys and (self.scan_frac or self.insert_frac)), "sparse keys: point ops only"

    # -- table ------------------------------------------------------------------
    def table_desc(self):
        """(col_group, col_is_add, n_groups, has_pk): one conflict unit per row (G=1)."""
        return [0] * self.n_fields, [0] * self.n_fields, 1, True

    def key_of(self, k):
        """Stored key of logical row k (identity, or splitmix64 with sparse_keys)."""
        k = np.asarray(k, dtype=np.uint64)
        if not self.sparse_keys:
            return k
        with np.errstate(over="ignore"):
            return splitmix64(k)

    def initial_table(self):
        keys = np.arange(self.n_rows, dtype=np.uint64)
        cols = np.empty((self.n_fields, self.n_rows), dtype=np.int64)
        for f in range(self.n_fields):
            with np.errstate(over="ignore"):
                v = splitmix64(keys * np.uint64(16) + np.uint64(f)) & np.uint64(0xFFFFFFFF)
            cols[f] = v.astype(np.int64)
        keys = self.key_of(keys)
        assert not (keys == np.uint64(KEY_EMPTY)).any()
        return keys, cols

    # -- batches ------------------------------------------------------------------
    def _rng(self, batch_no):
        return np.random.Generator(np.random.PCG64([self.seed, int(batch_no)]))

    def _keys_from_ranks(self, ranks):
        with np.errstate(over="ignore"):
            k = (np.uint64(self.a) * ranks.astype(np.uint64) + np.uint64(self.b)) % np.uint64(self.n_rows)
        return k

    def _draw_ranks(self, rng, shape):
        cdf = zipf_cdf(self.n_rows, self.theta)
        ranks = np.searchsorted(cdf, rng.random(shape), side="right")
        return np.minimum(ranks, self.n_rows - 1)

    @staticmethod
    def _dedupe_scans(keys, kinds, aux):
        """R10: a txn's SCAN range may not cover a key the txn writes (INSERT/UPDATE) or
        another point key; such SCANs are shortened to length 0 (an empty read)."""
        n, k = keys.shape
        lo = keys.astype(np.uint64)
        for j in range(k):
            sc = kinds[:, j] == SCAN
            if not sc.any():
                continue
            hi = lo[:, j] + aux[:, j].astype(np.uint64)
            clash = np.zeros(n, bool)
            for m in range(k):
                if m == j:
                    continue
                other_hi = lo[:, m] + np.where(kinds[:, m] == SCAN, aux[:, m], 1).astype(np.uint64)
                ov = (lo[:, m] < hi) & (lo[:, j] < other_hi)
                writes = np.isin(kinds[:, m], [UPDATE, INSERT])
                clash |= sc & ov & (writes | (kinds[:, m] != SCAN))
            aux[clash, j] = 0

    def _draw_keys(self, rng, shape):
        cdf = zipf_cdf(self.n_rows, self.theta)
        u = rng.random(shape)
        ranks = np.searchsorted(cdf, u, side="right")
        np.minimum(ranks, self.n_rows - 1, out=ranks)
        return self._keys_from_ranks(ranks)

    def batch(self, n_txns, tid_start, batch_no):
        """Return dict(tid, op_begin, ops, args) for ``n_txns`` fresh txns."""
        rng = self._rng(batch_no)
        k = self.ops_per_txn
        keys = self._draw_keys(rng, (n_txns, k))
        # distinct keys per txn: resample duplicate positions
        upper = np.triu(np.ones((k, k), dtype=bool), 1)[None, :, :]
        s = np.sort(keys, axis=1)
        rows = np.nonzero((s[:, 1:] == s[:, :-1]).any(axis=1))[0]  # txns with a repeated key
        while len(rows):
            sub = keys[rows]
            pos = ((sub[:, :, None] == sub[:, None, :]) & upper).any(axis=1)  # l repeats an earlier j
            sub[pos] = self._draw_keys(rng, int(pos.sum()))
            keys[rows] = sub
            s = np.sort(sub, axis=1)
            rows = rows[(s[:, 1:] == s[:, :-1]).any(axis=1)]
        u = rng.random((n_txns, k))
        kinds = np.where(u < self.read_frac, SELECT, UPDATE).astype(np.uint8)
        aux = np.zeros((n_txns, k), np.uint32)
        if self.scan_frac > 0 or self.insert_frac > 0:
            # YCSB D/E: INSERTs of fresh keys N, N+1, ... (unique across batches) and
            # short SCANs [key, key+len) with len U[1, max_scan_len]
            u2 = rng.random((n_txns, k))
            scan = u2 < self.scan_frac
            ins = (u2 >= self.scan_frac) & (u2 < self.scan_frac + self.insert_frac)
            kinds = np.where(scan, SCAN, np.where(ins, INSERT, kinds)).astype(np.uint8)
            aux = np.where(scan, rng.integers(1, self.max_scan_len + 1, (n_txns, k)), 0).astype(np.uint32)
            n_ins = int(ins.sum())
            latest = self.next_insert_key - 1  # newest key inserted before this batch
            keys[ins] = np.arange(self.next_insert_key, self.next_insert_key + n_ins, dtype=np.uint64)
            self.next_insert_key += n_ins
            if self.read_latest:  # YCSB D: reads skewed toward the most recently inserted keys
                off = self._draw_ranks(rng, (n_txns, k)).astype(np.int64)
                off = np.where(kinds == SELECT, off, 1 << 40)  # non-reads sort last
                order = np.argsort(off, axis=1, kind="stable")
                so = np.take_along_axis(off, order, axis=1)
                idx = np.arange(k)[None, :]
                so = idx + np.maximum.accumulate(so - idx, axis=1)  # distinct offsets per txn (R10)
                np.put_along_axis(off, order, so, axis=1)
                rd = kinds == SELECT
                keys[rd] = (np.uint64(latest) - (off[rd] % (latest + 1)).astype(np.uint64))
            self._dedupe_scans(keys, kinds, aux)
        ops = np.zeros(n_txns * k, dtype=OP_DTYPE)
        ops["key"] = self.key_of(keys.reshape(-1))
        ops["kind"] = kinds.reshape(-1)
        ops["table"] = self.TABLE
        ops["col"] = rng.integers(0, self.n_fields, n_txns * k, dtype=np.uint16)
        ops["aux"] = aux.reshape(-1)
        args = rng.integers(1, 1001, n_txns * k, dtype=np.int64)
        op_begin = (np.arange(n_txns + 1, dtype=np.uint64) * k).astype(np.uint32)
        tid = np.arange(tid_start, tid_start + n_txns, dtype=np.uint64)
        return {"tid": tid, "op_begin": op_begin, "ops": ops, "args": args}


def random_ops_batch(rng, n_txns, n_keys, n_fields=2, max_ops=4, kinds=(SELECT, UPDATE),
                     tid_start=1, table=0, scan_len=3, insert_key_base=None):
    """Tiny random OPS batch (distinct keys per txn) for brute-force / parity tests."""
    op_begin = [0]
    recs, args = [], []
    for _ in range(n_txns):
        k = int(rng.integers(1, max_ops + 1))
        k = min(k, n_keys)
        chosen = rng.choice(n_keys + (4 if insert_key_base is not None else 0), size=k, replace=False)
        for key in chosen:
            kind = int(rng.choice(kinds))
            col = int(rng.integers(0, n_fields))
            aux = 0
            if kind == SCAN:
                aux = int(rng.integers(0, scan_len + 1))
            recs.append((int(key), kind, table, col, aux))
            args.append(int(rng.integers(-50, 51)))
        op_begin.append(len(recs))
    ops = np.zeros(len(recs), dtype=OP_DTYPE)
    for i, r in enumerate(recs):
        ops[i] = r
    return {"tid": np.arange(tid_start, tid_start + n_txns, dtype=np.uint64),
            "op_begin": np.array(op_begin, dtype=np.uint32),
            "ops": ops, "args": np.array(args, dtype=np.int64)}


# YCSB core workloads A-E (Cooper et al. [7]), as op mixes of this OPS model.
# Fractions are of ops: read / (update = RMW) / insert / scan.
YCSB_MIXES = {
    "A": dict(read_frac=0.50),                                        # update heavy
    "B": dict(read_frac=0.95),                                        # read heavy
    "C": dict(read_frac=1.00),                                        # read only
    "D": dict(read_frac=1.00, insert_frac=0.05, read_latest=True),    # read latest
    "E": dict(read_frac=1.00, scan_frac=0.95, insert_frac=0.05),      # short ranges
}


def ycsb_letter(letter, n_rows, theta=2.5, ops_per_txn=10, seed=0x17C0, **kw):
    """YCSB workload `letter` at Zipf theta (the paper's alpha = 2.5)."""
    args = dict(YCSB_MIXES[letter])
    args.update(kw)
    return YcsbWorkload(n_rows, theta=theta, ops_per_txn=ops_per_txn, seed=seed, **args)
