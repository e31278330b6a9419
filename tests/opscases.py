"""Hand-written and random tiny OPS-mode cases shared by oracle pins and GPU parity.

Inputs only (tables, descriptors, batches); no method arithmetic.
"""
import json
import os

import numpy as np

from workloads.formats import (OP_DTYPE, SELECT, UPDATE, ADD, INSERT, DELETE, SCAN, COL_COUNT,
                               STATIC)

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def make_batch(txns, tid_start=1):
    """txns: list of lists of (key, kind, table, col, aux, arg)."""
    op_begin = [0]
    recs, args = [], []
    for t in txns:
        for (key, kind, table, col, aux, arg) in t:
            recs.append((key, kind, table, col, aux))
            args.append(arg)
        op_begin.append(len(recs))
    ops = np.zeros(len(recs), dtype=OP_DTYPE)
    for i, r in enumerate(recs):
        ops[i] = r
    return {"tid": np.arange(tid_start, tid_start + len(txns), dtype=np.uint64),
            "op_begin": np.array(op_begin, dtype=np.uint32), "ops": ops,
            "args": np.array(args, dtype=np.int64)}


def example3(encoding):
    """Example 3 under one of three unit encodings.

    returns (descs, tables, batch) where descs: t -> (col_group, col_is_add, n_groups).
    """
    g = json.load(open(os.path.join(GOLDEN, "example3.json")))
    key = g["table"]["key"]
    init = g["table"]["initial"]
    if encoding in ("row_level_no_optimizations", "row_level_reordering"):
        desc = ([0, 0], [0, 0], 1)
        wkind = UPDATE
    elif encoding == "split_only_write":
        desc = ([0, 1], [0, 0], 2)
        wkind = UPDATE
    elif encoding == "split_and_delayed_update":
        desc = ([0, 1], [0, 1], 2)
        wkind = ADD
    else:
        raise ValueError(encoding)
    txns = []
    for tx in g["txns"]:
        if tx["op"] == "SELECT":
            txns.append([(key, SELECT, 0, 0, 0, 0)])
        else:
            txns.append([(key, wkind, 0, 1, 0, tx["arg"])])
    tables = {0: (np.array([key, 1, 2], dtype=np.uint64),
                  np.array([[init[0], 1, 2], [init[1], 10, 20]], dtype=np.int64))}
    return {0: desc}, tables, make_batch(txns), g


# ---- random tiny batches over two tables exercising every op kind ----------------------
RAND_DESCS = {
    0: ([0, 0, 1], [0, 0, 0], 2),            # two write groups; INSERT/DELETE allowed
    1: ([STATIC, 0, 1], [0, 0, 1], 2),       # static col, write group, ADD group
    2: ([0, 0, 1], [0, 0, 1], 2),            # write group + ADD group; DELETE allowed
}
RAND_LOADED_KEYS = 8   # keys 0..7 present, 8..11 absent (INSERT / NOT_FOUND paths)
RAND_KEY_SPACE = 12


def rand_tables(rng):
    t = {}
    for tab in RAND_DESCS:
        keys = np.arange(RAND_LOADED_KEYS, dtype=np.uint64)
        cols = rng.integers(-100, 100, (3, RAND_LOADED_KEYS)).astype(np.int64)
        t[tab] = (keys, cols)
    return t


def _valid_kinds(tab):
    if tab == 0:
        return [(SELECT, [0, 1, 2]), (UPDATE, [0, 1, 2]), (INSERT, [0]), (DELETE, [0]),
                (SCAN, [0, 2, COL_COUNT])]
    if tab == 1:
        return [(SELECT, [0, 1, 2]), (UPDATE, [1]), (ADD, [2]), (INSERT, [0]),
                (SCAN, [0, 1, 2, COL_COUNT])]
    return [(SELECT, [0, 2]), (UPDATE, [0, 1]), (ADD, [2]), (ADD, [2]), (INSERT, [0]), (DELETE, [0]),
            (SCAN, [1, 2, COL_COUNT])]


def _txn_ok(ops):
    for i in range(len(ops)):
        for j in range(i):
            a, b = ops[i], ops[j]
            if a[2] != b[2]:
                continue
            alo, ahi = a[0], a[0] + (a[4] if a[1] == SCAN else 1)
            blo, bhi = b[0], b[0] + (b[4] if b[1] == SCAN else 1)
            if alo < bhi and blo < ahi:
                if a[1] in (UPDATE, ADD, INSERT, DELETE) or b[1] in (UPDATE, ADD, INSERT, DELETE):
                    return False
                if a[1] != SCAN and b[1] != SCAN:
                    return False
    return True


def rand_batch(rng, n_txns, max_ops=4, kinds=None, tables=(0, 1, 2), tid_start=1, key_space=RAND_KEY_SPACE):
    txns = []
    while len(txns) < n_txns:
        k = int(rng.integers(1, max_ops + 1))
        ops = []
        for _ in range(k):
            tab = int(rng.choice(tables))
            choices = _valid_kinds(tab)
            if kinds is not None:
                choices = [c for c in choices if c[0] in kinds]
            kind, cols = choices[int(rng.integers(0, len(choices)))]
            col = int(cols[int(rng.integers(0, len(cols)))])
            key = int(rng.integers(0, key_space))
            aux = int(rng.integers(0, 4)) if kind == SCAN else 0
            ops.append((key, kind, tab, col, aux, int(rng.integers(-50, 51))))
        if _txn_ok(ops):
            txns.append(ops)
    return make_batch(txns, tid_start)
