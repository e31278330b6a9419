"""Pins of the CPU oracle, OPS mode (YCSB / micro-cases).  CPU only.

PIN-1  Example 3           -- golden fixture tests/golden/example3.json
PIN-2  Example 2 (Fig. 4)        -- WAW keeps the smallest TID; reads never conflict
PIN-3  brute force of the pairwise definition (tests/pymodel.py, independent code)
PIN-6  serial replay of the committed set in TID order
PIN-7  closed forms (read-only, disjoint, single hot key, rank 0 commits)
"""
import numpy as np
import pytest

import oracle
from tests import opscases, pymodel
from workloads.formats import (SELECT, UPDATE, ADD, INSERT, DELETE, SCAN, ST_COMMIT,
                               ST_CONFLICT, ST_USER_ABORT, NOT_FOUND)
from workloads.ycsb import YcsbWorkload


def make_db(descs, tables):
    db = oracle.OracleDB(max(descs) + 1)
    for t, (g, a, ng) in descs.items():
        db.define_table(t, g, a, ng, True)
    for t, (k, c) in tables.items():
        db.load_table(t, k, c)
    return db


@pytest.mark.parametrize("encoding", ["row_level_no_optimizations", "split_only_write",
                                      "split_and_delayed_update", "row_level_reordering"])
def test_example3(encoding):
    descs, tables, batch, g = opscases.example3(encoding)
    db = make_db(descs, tables)
    if encoding == "row_level_reordering":
        db.set_reorder(True)
    rc, status, reads = db.run_ops(batch)
    assert rc == 0
    committed = [i + 1 for i, s in enumerate(status) if s == ST_COMMIT]
    assert committed == g["expected_commits"][encoding]["value"]
    keys, cols = db.dump_table(0)
    assert cols[1][list(keys).index(4)] == g["expected_final_W_YTD"][encoding]
    # W_ZIP reads all return the snapshot value
    assert all(reads[i] == 12345 for i in (0, 2, 4))


def test_example2_fig4():
    # TX2, TX3 write Warehouse 13 (WAW) and read Item 419; the smaller TID
    # updates, the other is marked WAW; reading the same item never conflicts.
    descs = {0: ([0], [0], 1), 1: ([0], [0], 1)}  # 0 = WAREHOUSE, 1 = ITEM
    tables = {0: (np.array([7, 13], np.uint64), np.array([[70, 130]], np.int64)),
              1: (np.array([1, 419], np.uint64), np.array([[10, 4190]], np.int64))}
    db = make_db(descs, tables)
    b = opscases.make_batch([
        [(1, SELECT, 1, 0, 0, 0)],                              # TX1 reads Item 1
        [(13, UPDATE, 0, 0, 0, 5), (419, SELECT, 1, 0, 0, 0)],  # TX2
        [(13, UPDATE, 0, 0, 0, 9), (419, SELECT, 1, 0, 0, 0)],  # TX3
        [(7, SELECT, 0, 0, 0, 0)],                              # TX4 reads Warehouse 7
    ])
    rc, status, reads = db.run_ops(b)
    assert rc == 0
    assert list(status) == [ST_COMMIT, ST_COMMIT, ST_CONFLICT, ST_COMMIT]
    keys, cols = db.dump_table(0)
    assert list(cols[0]) == [70, 135]
    assert list(reads) == [10, 130, 4190, 130, 4190, 70]


def _ycsb_small():
    return YcsbWorkload(200, n_fields=4, theta=0.5, ops_per_txn=4, seed=3)


def test_closed_forms():
    wl = _ycsb_small()
    keys, cols = wl.initial_table()
    descs = {0: ([0] * 4, [0] * 4, 1)}
    # read-only batch: all commit, reads == snapshot
    b = opscases.make_batch([[(k, SELECT, 0, k % 4, 0, 0)] for k in range(50)])
    db = make_db(descs, {0: (keys, cols)})
    rc, st, rd = db.run_ops(b)
    assert rc == 0 and (st == ST_COMMIT).all()
    assert list(rd) == [cols[k % 4][k] for k in range(50)]
    # disjoint keys, all writes: all commit
    b = opscases.make_batch([[(k, UPDATE, 0, 1, 0, 7)] for k in range(60)])
    rc, st, rd = db.run_ops(b)
    assert (st == ST_COMMIT).all()
    _, c2 = db.dump_table(0)
    assert (c2[1][:60] == cols[1][:60] + 7).all() and (c2[1][60:] == cols[1][60:]).all()
    # every txn writes one hot key: exactly rank 0 commits
    b = opscases.make_batch([[(5, UPDATE, 0, 0, 0, 1), (100 + i, SELECT, 0, 0, 0, 0)] for i in range(40)])
    rc, st, rd = db.run_ops(b)
    assert st[0] == ST_COMMIT and (st[1:] == ST_CONFLICT).all()
    # rank 0 commits in any batch without a user abort
    for s in range(20):
        rb = opscases.rand_batch(np.random.default_rng(s), 30, kinds=(SELECT, UPDATE, ADD, DELETE, SCAN))
        db2 = make_db(opscases.RAND_DESCS, opscases.rand_tables(np.random.default_rng(s)))
        rc, st, _ = db2.run_ops(rb)
        assert rc == 0 and st[0] == ST_COMMIT


def test_validation_einval():
    descs = {0: ([0, 0], [0, 0], 1)}
    tables = {0: (np.arange(4, dtype=np.uint64), np.zeros((2, 4), np.int64))}
    db = make_db(descs, tables)
    bad_dup = opscases.make_batch([[(1, UPDATE, 0, 0, 0, 1), (1, SELECT, 0, 1, 0, 0)]])
    assert db.run_ops(bad_dup)[0] == oracle.ORC_EINVAL
    b = opscases.make_batch([[(1, SELECT, 0, 0, 0, 0)], [(2, SELECT, 0, 0, 0, 0)]])
    b["tid"] = np.array([5, 5], np.uint64)
    assert db.run_ops(b)[0] == oracle.ORC_EINVAL
    bad_col = opscases.make_batch([[(1, SELECT, 0, 9, 0, 0)]])
    assert db.run_ops(bad_col)[0] == oracle.ORC_EINVAL
    bad_add = opscases.make_batch([[(1, ADD, 0, 0, 0, 1)]])  # not an ADD column
    assert db.run_ops(bad_add)[0] == oracle.ORC_EINVAL
    scan_over_write = opscases.make_batch([[(0, SCAN, 0, 0, 3, 0), (2, UPDATE, 0, 0, 0, 1)]])
    assert db.run_ops(scan_over_write)[0] == oracle.ORC_EINVAL
    # state untouched by rejected batches
    _, c = db.dump_table(0)
    assert (c == 0).all()


def _model_from(descs, tables):
    m = pymodel.Model(descs)
    for t, (k, c) in tables.items():
        m.load(t, k, c)
    return m


def _dump_model(m, t):
    ks = sorted(m.rows[t])
    return np.array(ks, dtype=np.uint64), np.array([m.rows[t][k] for k in ks], dtype=np.int64).T.reshape(
        len(m.descs[t][0]), len(ks))


@pytest.mark.parametrize("seed", range(40))
def test_brute_force_and_serial_replay(seed):
    rng = np.random.default_rng(1000 + seed)
    tables = opscases.rand_tables(rng)
    n_txns = int(rng.integers(1, 40))
    batch = opscases.rand_batch(rng, n_txns)
    db = make_db(opscases.RAND_DESCS, tables)
    rc, status, reads = db.run_ops(batch)
    assert rc == 0
    model = _model_from(opscases.RAND_DESCS, tables)
    bst, breads, bfinal = pymodel.brute_force_batch(model, batch)
    assert list(status) == bst                       # PIN-3
    assert list(reads) == breads
    for t in opscases.RAND_DESCS:
        k, c = db.dump_table(t)
        mk, mc = _dump_model(bfinal, t)
        assert (k == mk).all() and (c == mc).all()
    # PIN-6: serial replay in TID order reproduces reads of committed txns and S'
    sreads, sfinal = pymodel.serial_replay(model, batch, list(status))
    ob = batch["op_begin"]
    for r, res in sreads.items():
        assert list(reads[ob[r]:ob[r + 1]]) == res, r
    for t in opscases.RAND_DESCS:
        k, c = db.dump_table(t)
        mk, mc = _dump_model(sfinal, t)
        assert (k == mk).all() and (c == mc).all()


def test_multi_batch_retry_loop_small():
    """a9: aborted txns re-run next batch with their original TIDs; state stays serial."""
    wl = YcsbWorkload(50, n_fields=2, theta=0.9, ops_per_txn=3, seed=11)
    keys, cols = wl.initial_table()
    descs = {0: ([0, 0], [0, 0], 1)}
    db = make_db(descs, {0: (keys, cols)})
    model = _model_from(descs, {0: (keys, cols)})
    pending = None
    tid_next = 1
    for b in range(6):
        fresh = wl.batch(40, tid_next, b)
        tid_next += 40
        batch = fresh if pending is None else _concat(pending, fresh)
        rc, st, rd = db.run_ops(batch)
        assert rc == 0 and st[0] == ST_COMMIT
        _, model = pymodel.serial_replay(model, batch, list(st))
        k, c = db.dump_table(0)
        mk, mc = _dump_model(model, 0)
        assert (c == mc).all()
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = _select(batch, ab) if len(ab) else None


def _select(batch, idx):
    ob = batch["op_begin"]
    parts = [np.arange(ob[i], ob[i + 1]) for i in idx]
    sel = np.concatenate(parts) if parts else np.zeros(0, np.int64)
    lens = np.array([ob[i + 1] - ob[i] for i in idx], dtype=np.uint32)
    return {"tid": batch["tid"][idx], "ops": batch["ops"][sel], "args": batch["args"][sel],
            "op_begin": np.concatenate([[0], np.cumsum(lens)]).astype(np.uint32)}


def _concat(a, b):
    return {"tid": np.concatenate([a["tid"], b["tid"]]), "ops": np.concatenate([a["ops"], b["ops"]]),
            "args": np.concatenate([a["args"], b["args"]]),
            "op_begin": np.concatenate([a["op_begin"], b["op_begin"][1:] + a["op_begin"][-1]]).astype(np.uint32)}


def test_example3_reordering_logical_order():
    """with logical reordering the serial order is Tx1, Tx3, Tx5, Tx2."""
    descs, tables, batch, g = opscases.example3("row_level_reordering")
    db = make_db(descs, tables)
    db.set_reorder(True)
    rc, status, reads = db.run_ops(batch)
    model = _model_from(descs, tables)
    order = pymodel.logical_order(model, batch, list(status))
    assert [r + 1 for r in order] == g["expected_logical_order"]["row_level_reordering"]["value"]


@pytest.mark.parametrize("seed", range(40))
def test_brute_force_reordering(seed):
    """NEXT-1: oracle with logical reordering == pairwise definition (WAW or (RAW and WAR)),
    and the committed set replays serially in a reader-before-writer topological order."""
    rng = np.random.default_rng(7000 + seed)
    tables = opscases.rand_tables(rng)
    batch = opscases.rand_batch(rng, int(rng.integers(1, 40)))
    db = make_db(opscases.RAND_DESCS, tables)
    db.set_reorder(True)
    rc, status, reads = db.run_ops(batch)
    assert rc == 0
    model = _model_from(opscases.RAND_DESCS, tables)
    bst, breads, bfinal = pymodel.brute_force_batch(model, batch, reorder=True)
    assert list(status) == bst
    assert list(reads) == breads
    order = pymodel.logical_order(model, batch, list(status))
    sreads, sfinal = pymodel.serial_replay(model, batch, list(status), order)
    ob = batch["op_begin"]
    for r, res in sreads.items():
        assert list(reads[ob[r]:ob[r + 1]]) == res, r
    for t in opscases.RAND_DESCS:
        k, c = db.dump_table(t)
        mk, mc = _dump_model(sfinal, t)
        assert (k == mk).all() and (c == mc).all()
    # reordering never commits fewer txns than the base rule on the same batch
    db2 = make_db(opscases.RAND_DESCS, tables)
    _, st2, _ = db2.run_ops(batch)
    assert (status == ST_COMMIT).sum() >= (st2 == ST_COMMIT).sum()
