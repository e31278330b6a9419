"""Pins of the CPU oracle, PROC mode (TPC-C).  CPU only.

PIN-4  Table VI "no" rows: strict mode, fresh 50/50 batches:
       committed Payments == #warehouses, NewOrder commit rate ~ 63.4/88.3/88.3/96.9%.
PIN-5  TPC-C consistency conditions after every batch (tests/tpcc_cc.py).
PIN-6  serial replay: committed txns re-run one per batch in TID order.
       + hand-computed NewOrder / Payment values on a tiny database.
"""
import numpy as np
import pytest

import oracle
from tests import tpcc_cc
from workloads import tpcc
from workloads.formats import (ST_COMMIT, ST_CONFLICT, ST_USER_ABORT, NEW_ORDER, PAYMENT, ORDER_STATUS,
                               DELIVERY, STOCK_LEVEL, T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_STOCK,
                               T_ITEM, T_ORDER, T_NEW_ORDER, T_ORDER_LINE, T_HISTORY, tpcc_col,
                               NEWORDER_DTYPE, PAYMENT_DTYPE)


def dumps(db):
    return {t: db.dump_table(t) for t in range(9)}


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_cc_initial_and_after_batches(mode):
    wl = tpcc.TpccWorkload(2, seed=5, mode=mode, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    db = oracle.tpcc_db(wl, tables)
    cc = tpcc_cc.check(dumps(db))
    assert all(cc.values()), cc
    tid = 1
    pending = None
    n_commit = np.zeros(5, int)
    for b in range(6):
        fresh = wl.batch(2000, tid, b)
        tid += 2000
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        rc, st, res = db.run_tpcc(batch, clock=2 + b)
        assert rc == 0
        for t in range(5):
            n_commit[t] += int(((batch["type"] == t) & (st == ST_COMMIT)).sum())
        cc = tpcc_cc.check(dumps(db))
        assert all(cc.values()), (b, cc)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    assert (n_commit > 0).all(), n_commit  # every procedure type committed at least once


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_serial_replay(mode):
    """Committed set replayed one txn per batch in TID order gives the same results and S'."""
    wl = tpcc.TpccWorkload(1, seed=9, mode=mode, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    db = oracle.tpcc_db(wl, tables)
    ser = oracle.tpcc_db(wl, tables)
    tid = 1
    for b in range(3):
        batch = wl.batch(600, tid, b)
        tid += 600
        rc, st, res = db.run_tpcc(batch, clock=2 + b)
        assert rc == 0
        for r in np.nonzero(st == ST_COMMIT)[0]:
            one = {k: v[r:r + 1] for k, v in batch.items()}
            rc1, st1, res1 = ser.run_tpcc(one, clock=2 + b)
            assert rc1 == 0 and st1[0] == ST_COMMIT
            assert (res1[0] == res[r]).all(), (r, res1[0], res[r])
        for t in range(9):
            k1, c1 = db.dump_table(t)
            k2, c2 = ser.dump_table(t)
            assert c1.shape == c2.shape and (c1 == c2).all(), t
            if k1 is not None:
                assert (k1 == k2).all()


def _table6_db(W, seed):
    """Only the tables NewOrder/Payment read at execution (others empty)."""
    wl = tpcc.TpccWorkload(W, seed=seed, mode="strict", mix=tpcc.MIX_NO_PAY)
    full = wl.initial_tables()
    db = oracle.OracleDB(9, W)
    for t, (g, a, ng, pk) in wl.table_descs().items():
        db.define_table(t, g, a, ng, pk)
    for t in (T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_ITEM, T_STOCK):
        db.load_table(t, *full[t])
    return wl, db


@pytest.mark.parametrize("W,B,paper_no_rate", [(8, 16384, 63.4), (32, 16384, 88.3),
                                               (8, 4096, 88.3), (32, 4096, 96.9)])
def test_table6_no_rows(W, B, paper_no_rate):
    """P:382-388 Table VI, "Has optimization = no" rows."""
    wl, db = _table6_db(W, seed=0x17C0 + W)
    batch = wl.batch(B, 1, 0)
    rc, st, res = db.run_tpcc(batch, clock=2)
    assert rc == 0
    no = batch["type"] == NEW_ORDER
    pay = batch["type"] == PAYMENT
    n_pay = int((pay & (st == ST_COMMIT)).sum())
    rate = 100.0 * (no & (st == ST_COMMIT)).sum() / no.sum()
    assert n_pay == W                       # paper: 8 and 32 committed Payments
    assert abs(rate - paper_no_rate) <= 2.0, rate


def _tiny_db(mode="strict"):
    wl = tpcc.TpccWorkload(1, seed=21, mode=mode)
    tables = wl.initial_tables()
    return wl, tables, oracle.tpcc_db(wl, tables)


def _col(tables, t, name, key):
    keys, cols = tables[t]
    i = int(np.nonzero(keys == np.uint64(key))[0][0])
    return int(cols[tpcc_col(t, name)][i])


def test_hand_computed_neworder_payment():
    """Values computed here directly from the TPC-C formulas (clauses 2.4.2.2, 2.5.2.2)."""
    wl, tables, db = _tiny_db()
    p = np.zeros(1, dtype=NEWORDER_DTYPE)
    p["w"], p["d"], p["c"], p["n_lines"] = 1, 3, 17, 2
    p["line"]["i"][0, :2] = [5, 77]
    p["line"]["supply_w"][0, :2] = [1, 1]
    p["line"]["qty"][0, :2] = [4, 9]
    q = np.zeros(1, dtype=PAYMENT_DTYPE)
    q["w"], q["d"], q["c_w"], q["c_d"], q["c_id"], q["amount"] = 1, 3, 1, 3, 17, 12345
    params = np.zeros((2, 128), np.uint8)
    params[0] = p.view(np.uint8)
    params[1] = q.view(np.uint8)
    batch = {"tid": np.array([10, 11], np.uint64), "type": np.array([NEW_ORDER, PAYMENT], np.uint8),
             "params": params}
    rc, st, res = db.run_tpcc(batch, clock=7)
    assert rc == 0 and list(st) == [ST_COMMIT, ST_COMMIT]  # disjoint units
    dk = 1 * 10 + 3
    ck = dk * 3000 + 17
    price5, price77 = _col(tables, T_ITEM, "I_PRICE", 5), _col(tables, T_ITEM, "I_PRICE", 77)
    disc = _col(tables, T_CUSTOMER, "C_DISCOUNT", ck)
    wtax, dtax = _col(tables, T_WAREHOUSE, "W_TAX", 1), _col(tables, T_DISTRICT, "D_TAX", dk)
    amt = 4 * price5 + 9 * price77
    assert res[0][0] == 3001                                  # o_id = D_NEXT_O_ID (fresh)
    assert res[0][1] == amt * (10000 - disc) * (10000 + wtax + dtax) // 10 ** 8
    assert res[1][0] == 17 and res[1][1] == -1000             # C_BALANCE pre-image
    d = dumps(db)
    after = {t: (d[t][0], d[t][1]) for t in d}
    for i, qty in ((5, 4), (77, 9)):
        q0 = _col(tables, T_STOCK, "S_QUANTITY", 100000 + i)
        exp = q0 - qty if q0 >= qty + 10 else q0 - qty + 91
        assert _col(after, T_STOCK, "S_QUANTITY", 100000 + i) == exp
        assert _col(after, T_STOCK, "S_YTD", 100000 + i) == qty
        assert _col(after, T_STOCK, "S_ORDER_CNT", 100000 + i) == 1
    ok = (dk << 32) | 3001
    assert _col(after, T_ORDER, "O_C_ID", ok) == 17
    assert _col(after, T_ORDER, "O_OL_CNT", ok) == 2
    assert _col(after, T_ORDER, "O_ENTRY_D", ok) == 7
    assert _col(after, T_ORDER_LINE, "OL_AMOUNT", ok * 16 + 2) == 9 * price77
    assert _col(after, T_NEW_ORDER, "NO_O_ID", ok) == 3001
    assert _col(after, T_DISTRICT, "D_NEXT_O_ID", dk) == 3002
    assert _col(after, T_WAREHOUSE, "W_YTD", 1) == 30_000_000 + 12345
    assert _col(after, T_DISTRICT, "D_YTD", dk) == 3_000_000 + 12345
    assert _col(after, T_CUSTOMER, "C_BALANCE", ck) == -1000 - 12345
    assert _col(after, T_CUSTOMER, "C_PAYMENT_CNT", ck) == 2
    hk, hc = d[T_HISTORY]
    assert hc.shape[1] == tables[T_HISTORY][1].shape[1] + 1
    new = np.nonzero(hc[7] == 11)[0]
    assert len(new) == 1 and list(hc[:, new[0]]) == [17, 3, 1, 3, 1, 7, 12345, 11, 0]


def test_fetch_add_order_ids_in_tid_order():
    """R12 / P:241: committed NewOrders of one district get consecutive o_ids in TID order."""
    wl, tables, db = _tiny_db()
    n = 5
    p = np.zeros(n, dtype=NEWORDER_DTYPE)
    p["w"], p["d"], p["c"], p["n_lines"] = 1, 2, 5, 1
    p["line"]["i"][:, 0] = [11, 12, 13, 12, 14]   # txn 3 collides with txn 1 on stock (1,12)
    p["line"]["supply_w"][:, 0] = 1
    p["line"]["qty"][:, 0] = 1
    batch = {"tid": np.arange(100, 100 + n, dtype=np.uint64), "type": np.zeros(n, np.uint8),
             "params": p.view(np.uint8).reshape(n, 128).copy()}
    rc, st, res = db.run_tpcc(batch, clock=3)
    assert list(st) == [ST_COMMIT, ST_COMMIT, ST_COMMIT, ST_CONFLICT, ST_COMMIT]
    assert list(res[:, 0]) == [3001, 3002, 3003, 0, 3004]


def test_delivery_and_stocklevel_conflict_with_neworder():
    """Delivery on an empty queue and StockLevel RAW-abort behind an earlier NewOrder
    of the same district (they read the D_NEXT_O_ID unit)."""
    wl, tables, db = _tiny_db()
    batch = wl.batch(4, 1, 0, types=[NEW_ORDER, STOCK_LEVEL, DELIVERY, ORDER_STATUS])
    params = batch["params"].copy()
    # make the StockLevel target the NewOrder's district
    params[1, 2] = params[0, 2]
    batch["params"] = params
    rc, st, res = db.run_tpcc(batch, clock=2)
    assert rc == 0
    assert st[0] == ST_COMMIT and st[1] == ST_CONFLICT
    assert st[2] == ST_COMMIT and res[2][0] == 10       # queues non-empty at load
    # StockLevel alone (rank 0) commits and reports its window
    b2 = wl.batch(1, 10, 1, types=[STOCK_LEVEL])
    rc, st, res = db.run_tpcc(b2, clock=3)
    assert st[0] == ST_COMMIT and res[0][1] >= 3001


def test_user_abort_rollback():
    """R11: an unused item id makes NewOrder a user abort (status 2), not retried."""
    wl = tpcc.TpccWorkload(1, seed=4, rollback_frac=1.0)
    db = oracle.tpcc_db(wl)
    b = wl.batch(3, 1, 0, types=[NEW_ORDER, NEW_ORDER, NEW_ORDER])
    rc, st, res = db.run_tpcc(b, clock=2)
    assert rc == 0 and (st == ST_USER_ABORT).all()
    assert (res[:, 0] == 0).all()


def test_proc_validation():
    wl, tables, db = _tiny_db()
    b = wl.batch(3, 1, 0, types=[PAYMENT, PAYMENT, PAYMENT])
    b["params"][1, 0] = 7  # warehouse 7 does not exist (W=1)
    assert db.run_tpcc(b, clock=2)[0] == oracle.ORC_EINVAL
    b = wl.batch(3, 1, 0)
    b["type"][2] = 9
    assert db.run_tpcc(b, clock=2)[0] == oracle.ORC_EINVAL
