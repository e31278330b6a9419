"""Hand-computed pins of the oracle's TPC-C read and result paths.  CPU only.

Every expected value below is derived by hand from the fixture in tests/tpcc_tiny.py (rows
written out literally) and the TPC-C clauses SURVEY §8(c)'s procedure table follows
(integer attributes; range queries over predefined keys):

  StockLevel  (2.8.2.2)  window = orders [D_NEXT_O_ID - 20, D_NEXT_O_ID) of the district;
                         result = number of DISTINCT items of their lines whose stock (home
                         warehouse) has S_QUANTITY < threshold (strict);  res = [low, nx, 0, 0]
  OrderStatus (2.6.2.2)  res = [c_id, C_BALANCE, O_CARRIER_ID, sum of OL_DELIVERY_D] of the
                         customer's predefined order (C_INIT_O_ID, reading R14)
  Delivery    (2.7.4.2)  per district: the order at the cursor if its NEW_ORDER row exists;
                         res = [districts delivered, sum of their OL_AMOUNT, 0, 0]; effects:
                         NEW_ORDER row deleted, O_CARRIER_ID = carrier, OL_DELIVERY_D = clock,
                         C_BALANCE += amount, C_DELIVERY_CNT += 1, cursor + 1
  by name     (2.5.2.2)  customers of (w, d, C_LAST) sorted by C_FIRST (ties: c_id, DESIGN.md
                         reading), the one at position ceil(n / 2), 1-based

tools/mutate_oracle.py applies plausible one-line mistakes to oracle/ltpg_oracle.cpp and shows
that each one turns at least one of these tests red (tests/test_oracle_mutations.py).
"""
import numpy as np
import pytest

import oracle
from tests import tpcc_tiny as tt
from workloads import tpcc
from workloads.formats import (ST_COMMIT, T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY, T_NEW_ORDER, T_ORDER,
                               T_ORDER_LINE)


def oracle_db(mode="strict"):
    wl = tpcc.TpccWorkload(1, mode=mode)  # schema (groups / ADD flags) and W only
    tables = tt.tiny_tables()
    return tables, oracle.tpcc_db(wl, tables)


@pytest.fixture
def make_db():
    """Database factory: the oracle here; tests/test_gpu_tpcc_pins.py runs the same tests on the
    CUDA path through the C-ABI with the same hand-computed expectations."""
    return oracle_db


def _run1(db, batch, clock=9):
    rc, st, res = db.run_tpcc(batch, clock=clock)
    assert rc == 0
    assert (st == ST_COMMIT).all(), st
    return res


@pytest.mark.parametrize("threshold,low", [
    (15, 7),    # q < 15: items 110..114 (q 10..14), 500 (q 5), 929 (q 2); item 115 (q == 15) not
    (10, 2),    # 500, 929 (item 110 has q == 10: not below)
    (11, 3),    # + item 110
    (1, 0),
    (3, 1),     # 929 only (902 is outside the window)
    (29, 21),   # every distinct item of the window: 110..128 (19), 500, 929
    (255, 21),
])
def test_stocklevel_window_threshold_distinct(make_db, threshold, low):
    tables, db = make_db()
    res = _run1(db, tt.stocklevel(1, 1, threshold))
    assert list(res[0]) == [low, 30, 0, 0]


def test_stocklevel_reads_the_stock_of_the_home_warehouse_only_once_per_item(make_db):
    """Item 500 is on 19 orders of the window: counted once (distinct), not 19 times."""
    tables, db = make_db()
    res = _run1(db, tt.stocklevel(1, 1, 6))
    assert res[0][0] == 2  # 500 (q 5) and 929 (q 2)


def test_orderstatus_slots_by_id_and_by_name(make_db):
    tables, db = make_db()
    res = _run1(db, tt.orderstatus(1, 2, c_id=7))
    assert list(res[0]) == [7, -12345, 6, 11 + 0 + 13 + 17]
    # C_LAST 42: (C_FIRST, c) sorted = (100,21) (200,22) (200,23) (300,20); ceil(4/2) = 2 -> c 22
    res = _run1(db, tt.orderstatus(1, 2, c_last=42))
    assert list(res[0]) == [22, 30, 2, 3 + 4]


@pytest.mark.parametrize("c_last,c_id,balance", [
    (42, 22, 30),   # n = 4: position 2 of (21, 22, 23, 20) -- the C_FIRST tie 22/23 broken by c_id
    (43, 30, 50),   # n = 3: (1,32) (5,30) (9,31) -> position 2 -> 30
    (44, 40, 80),   # n = 1
])
def test_payment_by_name_position_ceil_half(make_db, c_last, c_id, balance):
    tables, db = make_db()
    res = _run1(db, tt.payment(1, 2, 1, 2, 250, c_last=c_last))
    assert list(res[0]) == [c_id, balance, 0, 0]
    after = {t: db.dump_table(t) for t in (T_CUSTOMER,)}
    ck = tt.kc(1, 2, c_id)
    assert tt.col(after, T_CUSTOMER, "C_BALANCE", ck) == balance - 250
    assert tt.col(after, T_CUSTOMER, "C_PAYMENT_CNT", ck) == 2


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_delivery_counts_totals_and_effects(make_db, mode):
    tables, db = make_db(mode)
    res = _run1(db, tt.delivery(1, 3), clock=9)
    # district 1: order 5 (100 + 200 + 300), district 3: order 1 (1000 + 2345); the others empty
    assert list(res[0]) == [2, 600 + 3345, 0, 0]
    d = {t: db.dump_table(t) for t in range(9)}
    assert tt.col(d, T_NEW_ORDER, "NO_O_ID", tt.ko(1, 1, 5)) is None       # deleted
    assert tt.col(d, T_NEW_ORDER, "NO_O_ID", tt.ko(1, 3, 1)) is None
    assert len(d[T_NEW_ORDER][0]) == 0
    assert tt.col(d, T_ORDER, "O_CARRIER_ID", tt.ko(1, 1, 5)) == 3
    assert tt.col(d, T_ORDER, "O_CARRIER_ID", tt.ko(1, 3, 1)) == 3
    assert tt.col(d, T_ORDER, "O_CARRIER_ID", tt.ko(1, 2, 3)) == 6          # not queued: untouched
    for o_key, n in ((tt.ko(1, 1, 5), 3), (tt.ko(1, 3, 1), 2)):
        for ol in range(1, n + 1):
            assert tt.col(d, T_ORDER_LINE, "OL_DELIVERY_D", o_key * 16 + ol) == 9
    assert tt.col(d, T_ORDER_LINE, "OL_DELIVERY_D", tt.kol(1, 2, 3, 2)) == 0
    assert tt.col(d, T_CUSTOMER, "C_BALANCE", tt.kc(1, 1, 50)) == -1000 + 600
    assert tt.col(d, T_CUSTOMER, "C_DELIVERY_CNT", tt.kc(1, 1, 50)) == 1
    assert tt.col(d, T_CUSTOMER, "C_BALANCE", tt.kc(1, 3, 60)) == 0 + 3345
    assert tt.col(d, T_CUSTOMER, "C_DELIVERY_CNT", tt.kc(1, 3, 60)) == 1
    assert tt.col(d, T_CUSTOMER, "C_DELIVERY_CNT", tt.kc(1, 2, 7)) == 0
    cursors = [tt.col(d, T_DISTRICT, "D_NEXT_DELIV_O_ID", tt.kd(1, dd)) for dd in range(1, 11)]
    assert cursors == [6, 3, 2] + [1] * 7
    # a second Delivery finds every queue empty
    res = _run1(db, tt.delivery(1, 4, tid=2), clock=10)
    assert list(res[0]) == [0, 0, 0, 0]


def test_delivery_then_orderstatus_sees_the_delivery(make_db):
    """Two batches: OrderStatus of customer 50 after its order 5 was delivered at clock 9."""
    tables, db = make_db()
    _run1(db, tt.delivery(1, 3), clock=9)
    # customer 50's predefined order is order 5 of district 1 (C_INIT_O_ID 5)
    res = _run1(db, tt.orderstatus(1, 1, c_id=50, tid=2), clock=10)
    assert list(res[0]) == [50, -400, 3, 3 * 9]


def test_one_batch_verdicts_on_the_fixture(make_db):
    """StockLevel, OrderStatus, Payment and Delivery in one batch.  Rank 1's Payment on
    customer 7 (strict: WRITE of the customer unit) makes rank 3's OrderStatus of customer 7 a
    RAW abort; rank 2's StockLevel reads no unit a smaller rank writes (Delivery writes
    district 1's cursor, not D_NEXT_O_ID; its queue is non-empty), so it commits."""
    tables, db = make_db()
    b = tt.concat(tt.delivery(1, 3, tid=10), tt.payment(1, 2, 1, 2, 5, c_id=7, tid=11),
                  tt.stocklevel(1, 1, 15, tid=12), tt.orderstatus(1, 2, c_id=7, tid=13))
    rc, st, res = db.run_tpcc(b, clock=9)
    assert rc == 0
    assert list(st) == [1, 1, 1, 0]
    assert list(res[0]) == [2, 3945, 0, 0]
    assert list(res[1]) == [7, -12345, 0, 0]
    assert list(res[2]) == [7, 30, 0, 0]
    h = db.dump_table(T_HISTORY)[1]
    assert h.shape[1] == 1 and list(h[:, 0]) == [7, 2, 1, 2, 1, 9, 5, 11, 0]
    w = db.dump_table(T_WAREHOUSE)
    assert tt.col({0: w}, 0, "W_YTD", 1) == 30_000_005


def test_delivery_on_an_empty_queue_reads_the_order_counter(make_db):
    """SURVEY §8(c) Delivery: an empty queue in S is a READ of the district's D_NEXT_O_ID unit.
    A smaller-rank NewOrder of that district appends the order the Delivery would deliver in
    TID-serial order, so the Delivery must RAW-abort (R1); with the ranks swapped the NewOrder's
    fetch-ADD does not conflict with the earlier read (WAR never aborts) and both commit."""
    tables, db = make_db()
    b = tt.concat(tt.neworder(1, 4, 1, [(700, 1, 2), (701, 1, 3)], tid=20), tt.delivery(1, 3, tid=21))
    rc, st, res = db.run_tpcc(b, clock=9)
    assert rc == 0 and list(st) == [1, 0]
    assert res[0][0] == 2                              # o_id = district 4's D_NEXT_O_ID
    tables, db = make_db()
    b = tt.concat(tt.delivery(1, 3, tid=20), tt.neworder(1, 4, 1, [(700, 1, 2), (701, 1, 3)], tid=21))
    rc, st, res = db.run_tpcc(b, clock=9)
    assert rc == 0 and list(st) == [1, 1]
    assert list(res[0]) == [2, 3945, 0, 0] and res[1][0] == 2
    # the NewOrder total by hand: amount = 2*I_PRICE(700) + 3*I_PRICE(701) = 2*800 + 3*801,
    # total = floor(amount * (10000 - 1000) * (10000 + 500 + 400) / 10^8)   (W_TAX 500, D_TAX 400)
    amount = 2 * 800 + 3 * 801
    assert res[1][2] == amount and res[1][1] == amount * 9000 * 10900 // 10 ** 8
