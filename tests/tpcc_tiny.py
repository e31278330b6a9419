"""A tiny, hand-built TPC-C database (one warehouse) whose read / result paths have values
worked out by hand in the tests (tests/test_oracle_tpcc_pins.py, tests/test_gpu_tpcc_pins.py).

Inputs only: every row below is written out literally (no generator, no method arithmetic), so
the expected results of StockLevel, OrderStatus, Delivery and the by-name customer choice can
be derived with pencil and paper from TPC-C clauses 2.5.2.2 / 2.6.2.2 / 2.7.4.2 / 2.8.2.2 and
SURVEY §8(c)'s procedure table (PAPER.md: integer attributes, predefined range keys).

Layout of the fixture (W = 1):
  district 1  D_NEXT_O_ID = 30 -> StockLevel window o in [10, 30)
              orders 9..29: order o in 10..28 has lines {item 100+o, item 500}; order 29 has
              {item 929}; order 9 (just outside the window) has {901, 902}
              stock: q(100+o) = o, q(500) = 5, q(929) = 2, q(901) = 1, q(902) = 3
              Delivery cursor 5 -> order 5 (customer 50, 3 lines, amounts 100/200/300) is queued
  district 2  customer 7: C_BALANCE -12345, C_INIT_O_ID 3; order 3: carrier 6, 4 lines with
              OL_DELIVERY_D 11, 0, 13, 17 (OrderStatus)
              C_LAST 42: customers 20..23 with C_FIRST 300, 100, 200, 200
              C_LAST 43: customers 30..32 with C_FIRST 5, 9, 1;  C_LAST 44: customer 40
              customer 22: C_INIT_O_ID 4; order 4: carrier 2, 2 lines with OL_DELIVERY_D 3, 4
              Delivery cursor 3, but no NEW_ORDER row for order 3 -> empty queue
  district 3  Delivery cursor 1 -> order 1 (customer 60, 2 lines, amounts 1000/2345) is queued
  district 4  customer 1 (for a NewOrder: discount 1000); no orders, empty queue (cursor 1)
  districts 5..10  no orders, empty queues (cursor 1)
"""
import numpy as np

from workloads.formats import (T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY, T_NEW_ORDER, T_ORDER,
                               T_ORDER_LINE, T_ITEM, T_STOCK, TPCC_COLS)


def kd(w, d):
    return w * 10 + d


def kc(w, d, c):
    return kd(w, d) * 3000 + c


def ko(w, d, o):
    return (kd(w, d) << 32) | o


def kol(w, d, o, ol):
    return ko(w, d, o) * 16 + ol


def ks(w, i):
    return w * 100000 + i


class _Rows:
    def __init__(self, t):
        self.t = t
        self.keys, self.rows = [], []

    def add(self, key, **cols):
        names = TPCC_COLS[self.t]
        assert set(cols) <= set(names), (self.t, set(cols) - set(names))
        self.keys.append(key)
        self.rows.append([int(cols.get(c, 0)) for c in names])

    def arrays(self, keyed=True):
        n = len(self.rows)
        cols = np.array(self.rows, dtype=np.int64).T.reshape(len(TPCC_COLS[self.t]), n)
        keys = np.array(self.keys, dtype=np.uint64) if keyed else None
        return keys, np.ascontiguousarray(cols)


def tiny_tables():
    """dict table -> (keys u64[n] or None, cols int64[n_cols, n]), as TpccWorkload.initial_tables()."""
    W = _Rows(T_WAREHOUSE)
    W.add(1, W_TAX=500, W_YTD=30_000_000)
    D = _Rows(T_DISTRICT)
    nxt = {1: 30, 2: 5}
    deliv = {1: 5, 2: 3}
    for d in range(1, 11):
        D.add(kd(1, d), D_TAX=100 * d, D_YTD=3_000_000, D_NEXT_O_ID=nxt.get(d, 2),
              D_NEXT_DELIV_O_ID=deliv.get(d, 1))
    C = _Rows(T_CUSTOMER)
    cust = [  # (d, c, C_LAST, C_FIRST, C_INIT_O_ID, C_BALANCE)
        (1, 50, 900, 1, 5, -1000),
        (2, 7, 901, 1, 3, -12345),
        (2, 20, 42, 300, 0, 10), (2, 21, 42, 100, 0, 20), (2, 22, 42, 200, 4, 30), (2, 23, 42, 200, 0, 40),
        (2, 30, 43, 5, 0, 50), (2, 31, 43, 9, 0, 60), (2, 32, 43, 1, 0, 70),
        (2, 40, 44, 7, 0, 80),
        (3, 60, 902, 1, 1, 0),
        (4, 1, 903, 1, 0, 0),
    ]
    for d, c, last, first, init_o, bal in cust:
        C.add(kc(1, d, c), C_DISCOUNT=1000, C_CREDIT=0, C_LAST=last, C_FIRST=first, C_INIT_O_ID=init_o,
              C_BALANCE=bal, C_YTD_PAYMENT=1000, C_PAYMENT_CNT=1, C_DELIVERY_CNT=0)
    O, NO, OL = _Rows(T_ORDER), _Rows(T_NEW_ORDER), _Rows(T_ORDER_LINE)
    stock_q = {}

    def order(d, o, c, carrier, lines, queued=False):
        O.add(ko(1, d, o), O_C_ID=c, O_ENTRY_D=1, O_OL_CNT=len(lines), O_ALL_LOCAL=1, O_CARRIER_ID=carrier)
        for ol, (item, amount, dd) in enumerate(lines, start=1):
            OL.add(kol(1, d, o, ol), OL_I_ID=item, OL_SUPPLY_W_ID=1, OL_QUANTITY=5, OL_AMOUNT=amount,
                   OL_DELIVERY_D=dd)
        if queued:
            NO.add(ko(1, d, o), NO_O_ID=o)

    # district 1: StockLevel window and the queued order 5
    order(1, 5, 50, 0, [(700, 100, 0), (701, 200, 0), (702, 300, 0)], queued=True)
    order(1, 9, 50, 1, [(901, 0, 1), (902, 0, 1)])
    for o in range(10, 29):
        order(1, o, 50, 1, [(100 + o, 0, 1), (500, 0, 1)])
        stock_q[100 + o] = o
    order(1, 29, 50, 1, [(929, 0, 1)])
    stock_q.update({500: 5, 929: 2, 901: 1, 902: 3, 700: 50, 701: 50, 702: 50})
    # district 2: OrderStatus orders (order 3 is delivered, not queued)
    order(2, 3, 7, 6, [(703, 0, 11), (704, 0, 0), (705, 0, 13), (706, 0, 17)])
    order(2, 4, 22, 2, [(707, 0, 3), (708, 0, 4)])
    # district 3: the queued order 1
    order(3, 1, 60, 0, [(709, 1000, 0), (710, 2345, 0)], queued=True)
    for i in range(703, 711):
        stock_q.setdefault(i, 50)
    I, S = _Rows(T_ITEM), _Rows(T_STOCK)
    for i in sorted(stock_q):
        I.add(i, I_PRICE=100 + i, I_IM_ID=1)
        S.add(ks(1, i), S_QUANTITY=stock_q[i])
    out = {T_WAREHOUSE: W.arrays(), T_DISTRICT: D.arrays(), T_CUSTOMER: C.arrays(), T_ORDER: O.arrays(),
           T_NEW_ORDER: NO.arrays(), T_ORDER_LINE: OL.arrays(), T_ITEM: I.arrays(), T_STOCK: S.arrays(),
           T_HISTORY: (None, np.zeros((len(TPCC_COLS[T_HISTORY]), 0), np.int64))}
    return out


def one_txn(ptype, fields, tid=1):
    """A one-txn PROC batch: fields = {byte offset: (numpy dtype str, value)}."""
    p = np.zeros((1, 128), np.uint8)
    for off, (dt, v) in fields.items():
        b = np.array([v], dtype=dt).view(np.uint8)
        p[0, off:off + len(b)] = b
    return {"tid": np.array([tid], np.uint64), "type": np.array([ptype], np.uint8), "params": p}


def stocklevel(w, d, threshold, tid=1):
    return one_txn(4, {0: ("<u2", w), 2: ("u1", d), 3: ("u1", threshold)}, tid)


def orderstatus(w, d, c_id=0, c_last=None, tid=1):
    f = {0: ("<u2", w), 2: ("u1", d), 3: ("u1", 0 if c_last is None else 1), 4: ("<u2", c_id)}
    if c_last is not None:
        f[6] = ("<u2", c_last)
    return one_txn(2, f, tid)


def neworder(w, d, c, lines, tid=1):
    """lines: [(item, supply_w, qty)]"""
    f = {0: ("<u2", w), 2: ("u1", d), 3: ("u1", len(lines)), 4: ("<u2", c)}
    for k, (i, sw, q) in enumerate(lines):
        f[8 + 8 * k] = ("<u4", i)
        f[12 + 8 * k] = ("<u2", sw)
        f[14 + 8 * k] = ("u1", q)
    return one_txn(0, f, tid)


def delivery(w, carrier, tid=1):
    return one_txn(3, {0: ("<u2", w), 2: ("u1", carrier)}, tid)


def payment(w, d, c_w, c_d, amount, c_id=0, c_last=None, tid=1):
    f = {0: ("<u2", w), 2: ("u1", d), 3: ("u1", 0 if c_last is None else 1), 4: ("<u2", c_w), 6: ("u1", c_d),
         8: ("<u2", c_id), 16: ("<i8", amount)}
    if c_last is not None:
        f[10] = ("<u2", c_last)
    return one_txn(1, f, tid)


def concat(*batches):
    return {k: np.concatenate([b[k] for b in batches]) for k in ("tid", "type", "params")}


def col(tables_or_dump, t, name, key):
    keys, cols = tables_or_dump[t]
    i = np.nonzero(keys == np.uint64(key))[0]
    if len(i) == 0:
        return None
    return int(cols[TPCC_COLS[t].index(name)][i[0]])
