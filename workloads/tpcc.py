"""Seeded synthetic TPC-C workload, integer-only (inputs only; no method arithmetic).

PAPER.md P:297: "All attributes in tables are set to integer type"; NewOrder +
Payment mixes (Table II/III/VI) and the full mix.  Initial population follows
TPC-C clause 4.3.3 integerised as SURVEY.md §8(c) "TPC-C initial population":
money in int64 cents, rates in 1/10,000, strings dropped or replaced by ints.

Readings used here:
  * R13 -- NewOrder items uniform in [1, 100000] (reproduces Table VI "no").
  * OrderStatus uses a predefined order key ("we can only predefine the
    primary key values of query items for the range queries"): the static
    column C_INIT_O_ID holds the customer's order from the load permutation.
  * Initial O_ENTRY_D / H_DATE / delivered OL_DELIVERY_D are 1; callers pass
    batch clocks >= 2.
"""
import numpy as np

from .formats import (PARAM_BYTES, NEWORDER_DTYPE, PAYMENT_DTYPE, ORDERSTATUS_DTYPE,
                      DELIVERY_DTYPE, STOCKLEVEL_DTYPE, NEW_ORDER, PAYMENT, ORDER_STATUS,
                      DELIVERY, STOCK_LEVEL, T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, T_HISTORY,
                      T_NEW_ORDER, T_ORDER, T_ORDER_LINE, T_ITEM, T_STOCK, TPCC_COLS,
                      TPCC_GROUPS, TPCC_HAS_PK)

N_ITEMS = 100000
DIST_PER_W = 10
CUST_PER_D = 3000
ORD_PER_D = 3000
FIRST_UNDELIVERED = 2101

MIX_NO_PAY = (0.5, 0.5, 0.0, 0.0, 0.0)
MIX_FULL = (0.45, 0.43, 0.04, 0.04, 0.04)


# ---- key encodings (SURVEY §8(c) "Keys") --------------------------------------
def k_w(w):
    return np.asarray(w, dtype=np.uint64)


def k_d(w, d):
    return np.asarray(w, dtype=np.uint64) * np.uint64(10) + np.asarray(d, dtype=np.uint64)


def k_c(w, d, c):
    return k_d(w, d) * np.uint64(3000) + np.asarray(c, dtype=np.uint64)


def k_s(w, i):
    return np.asarray(w, dtype=np.uint64) * np.uint64(100000) + np.asarray(i, dtype=np.uint64)


def k_o(w, d, o):
    return (k_d(w, d) << np.uint64(32)) | np.asarray(o, dtype=np.uint64)


def k_ol(w, d, o, ol):
    return k_o(w, d, o) * np.uint64(16) + np.asarray(ol, dtype=np.uint64)


def nurand(rng, A, x, y, C, size):
    a = rng.integers(0, A + 1, size)
    b = rng.integers(x, y + 1, size)
    return (((a | b) + C) % (y - x + 1)) + x


class TpccWorkload:
    def __init__(self, n_warehouses, seed=0x17C1, mode="strict", mix=MIX_NO_PAY,
                 remote_line_frac=0.01, remote_cust_frac=0.15, by_name_frac=0.60,
                 rollback_frac=0.0):
        self.W = int(n_warehouses)
        self.seed = int(seed)
        self.mode = mode
        self.mix = np.asarray(mix, dtype=np.float64) / np.sum(mix)
        self.remote_line_frac = remote_line_frac
        self.remote_cust_frac = remote_cust_frac
        self.by_name_frac = by_name_frac
        self.rollback_frac = rollback_frac
        r = np.random.Generator(np.random.PCG64([self.seed, 0xC0]))
        self.C_last_load = int(r.integers(0, 256))
        self.C_last_run = int(r.integers(0, 256))
        self.C_cid = int(r.integers(0, 1024))
        self.C_item = int(r.integers(0, 8192))

    # -- schema -------------------------------------------------------------------
    def table_descs(self):
        g = TPCC_GROUPS[self.mode]
        return {t: (list(g[t][0]), list(g[t][1]), g[t][2], TPCC_HAS_PK[t]) for t in range(9)}

    # -- initial population -----------------------------------------------------------
    def initial_tables(self):
        """dict table_id -> (keys u64[n] or None, cols int64[n_cols, n])."""
        W = self.W
        rng = np.random.Generator(np.random.PCG64([self.seed, 0x10AD]))
        out = {}
        ws = np.arange(1, W + 1, dtype=np.int64)
        # ITEM
        i = np.arange(1, N_ITEMS + 1, dtype=np.int64)
        out[T_ITEM] = (i.astype(np.uint64),
                       np.stack([rng.integers(100, 10001, N_ITEMS), rng.integers(1, 10001, N_ITEMS)]).astype(np.int64))
        # WAREHOUSE
        out[T_WAREHOUSE] = (ws.astype(np.uint64),
                            np.stack([rng.integers(0, 2001, W), np.full(W, 30_000_000)]).astype(np.int64))
        # DISTRICT
        dw = np.repeat(ws, DIST_PER_W)
        dd = np.tile(np.arange(1, DIST_PER_W + 1, dtype=np.int64), W)
        nD = W * DIST_PER_W
        out[T_DISTRICT] = (k_d(dw, dd),
                           np.stack([rng.integers(0, 2001, nD), np.full(nD, 3_000_000),
                                     np.full(nD, ORD_PER_D + 1), np.full(nD, FIRST_UNDELIVERED)]).astype(np.int64))
        # ORDER (needs the customer permutation first)
        perm = np.argsort(rng.random((nD, ORD_PER_D)), axis=1).astype(np.int64) + 1  # O_C_ID per (district, o-1)
        inv = np.empty_like(perm)                                                     # C_INIT_O_ID per (district, c-1)
        rows = np.arange(nD)[:, None]
        inv[rows, perm - 1] = np.arange(1, ORD_PER_D + 1, dtype=np.int64)[None, :]
        # CUSTOMER
        nC = nD * CUST_PER_D
        cw = np.repeat(dw, CUST_PER_D)
        cd = np.repeat(dd, CUST_PER_D)
        cc = np.tile(np.arange(1, CUST_PER_D + 1, dtype=np.int64), nD)
        last = nurand(rng, 255, 0, 999, self.C_last_load, nC)
        last = np.where(cc <= 1000, cc - 1, last)
        credit = (rng.random(nC) < 0.10).astype(np.int64)
        out[T_CUSTOMER] = (k_c(cw, cd, cc),
                           np.stack([rng.integers(0, 5001, nC), credit, last,
                                     rng.integers(0, 1 << 31, nC), inv.reshape(-1),
                                     np.full(nC, -1000), np.full(nC, 1000), np.full(nC, 1),
                                     np.zeros(nC)]).astype(np.int64))
        # HISTORY (keyless): one row per customer
        out[T_HISTORY] = (None,
                          np.stack([cc, cd, cw, cd, cw, np.ones(nC), np.full(nC, 1000),
                                    np.zeros(nC), np.arange(nC)]).astype(np.int64))
        # ORDER
        nO = nD * ORD_PER_D
        ow = np.repeat(dw, ORD_PER_D)
        od = np.repeat(dd, ORD_PER_D)
        oo = np.tile(np.arange(1, ORD_PER_D + 1, dtype=np.int64), nD)
        olcnt = rng.integers(5, 16, nO).astype(np.int64)
        delivered = oo < FIRST_UNDELIVERED
        carrier = np.where(delivered, rng.integers(1, 11, nO), 0)
        out[T_ORDER] = (k_o(ow, od, oo),
                        np.stack([perm.reshape(-1), np.ones(nO), olcnt, np.ones(nO), carrier]).astype(np.int64))
        # NEW_ORDER
        nm = ~delivered
        out[T_NEW_ORDER] = (k_o(ow[nm], od[nm], oo[nm]), oo[nm][None, :].astype(np.int64))
        # ORDER_LINE
        nOL = int(olcnt.sum())
        rep = np.repeat(np.arange(nO), olcnt)
        start = np.cumsum(olcnt) - olcnt
        ol = np.arange(nOL, dtype=np.int64) - start[rep] + 1
        ldel = delivered[rep]
        amount = np.where(ldel, 0, rng.integers(1, 1_000_000, nOL))
        out[T_ORDER_LINE] = (k_ol(ow[rep], od[rep], oo[rep], ol),
                             np.stack([rng.integers(1, N_ITEMS + 1, nOL), ow[rep], np.full(nOL, 5),
                                       amount, np.where(ldel, 1, 0)]).astype(np.int64))
        # STOCK
        nS = W * N_ITEMS
        sw = np.repeat(ws, N_ITEMS)
        si = np.tile(np.arange(1, N_ITEMS + 1, dtype=np.int64), W)
        out[T_STOCK] = (k_s(sw, si),
                        np.stack([rng.integers(10, 101, nS), np.zeros(nS), np.zeros(nS),
                                  np.zeros(nS)]).astype(np.int64))
        for t, (k, c) in out.items():
            assert c.shape[0] == len(TPCC_COLS[t]), (t, c.shape)
        return out

    # -- transactions ---------------------------------------------------------------------
    def _other_w(self, rng, w):
        if self.W == 1:
            return w.copy()
        o = rng.integers(1, self.W, len(w))
        return np.where(o >= w, o + 1, o)

    def batch(self, n_txns, tid_start, batch_no, types=None):
        """dict(tid, type u8[n], params u8[n,128])."""
        W = self.W
        rng = np.random.Generator(np.random.PCG64([self.seed, 0xBA7C, int(batch_no)]))
        if types is None:
            types = rng.choice(5, size=n_txns, p=self.mix).astype(np.uint8)
        else:
            types = np.asarray(types, dtype=np.uint8)
        params = np.zeros((n_txns, PARAM_BYTES), dtype=np.uint8)

        idx = np.nonzero(types == NEW_ORDER)[0]
        n = len(idx)
        if n:
            p = np.zeros(n, dtype=NEWORDER_DTYPE)
            w = rng.integers(1, W + 1, n)
            p["w"] = w
            p["d"] = rng.integers(1, 11, n)
            p["c"] = nurand(rng, 1023, 1, 3000, self.C_cid, n)
            nl = rng.integers(5, 16, n)
            p["n_lines"] = nl
            items = rng.integers(1, N_ITEMS + 1, (n, 15))
            while True:  # distinct items within the used lines (R10)
                used = np.arange(15)[None, :] < nl[:, None]
                eq = (items[:, :, None] == items[:, None, :]) & np.triu(np.ones((15, 15), bool), 1)[None]
                eq &= used[:, :, None] & used[:, None, :]
                pos = eq.any(axis=1)
                if not pos.any():
                    break
                items[pos] = rng.integers(1, N_ITEMS + 1, int(pos.sum()))
            remote = rng.random((n, 15)) < self.remote_line_frac
            sw = np.where(remote, self._other_w(rng, np.repeat(w, 15)).reshape(n, 15), w[:, None])
            qty = rng.integers(1, 11, (n, 15))
            used = np.arange(15)[None, :] < nl[:, None]
            if self.rollback_frac > 0:
                rb = rng.random(n) < self.rollback_frac
                p["rbk"] = rb
                last = nl - 1
                items[np.nonzero(rb)[0], last[rb]] = N_ITEMS + 1  # unused item id -> user abort
            p["line"]["i"] = np.where(used, items, 0)
            p["line"]["supply_w"] = np.where(used, sw, 0)
            p["line"]["qty"] = np.where(used, qty, 0)
            params[idx] = p.view(np.uint8).reshape(n, PARAM_BYTES)

        idx = np.nonzero(types == PAYMENT)[0]
        n = len(idx)
        if n:
            p = np.zeros(n, dtype=PAYMENT_DTYPE)
            w = rng.integers(1, W + 1, n)
            d = rng.integers(1, 11, n)
            remote = (rng.random(n) < self.remote_cust_frac) & (W > 1)
            p["w"] = w
            p["d"] = d
            p["c_w"] = np.where(remote, self._other_w(rng, w), w)
            p["c_d"] = np.where(remote, rng.integers(1, 11, n), d)
            p["by_name"] = rng.random(n) < self.by_name_frac
            p["c_id"] = nurand(rng, 1023, 1, 3000, self.C_cid, n)
            p["c_last"] = nurand(rng, 255, 0, 999, self.C_last_run, n)
            p["amount"] = rng.integers(100, 500001, n)
            params[idx] = p.view(np.uint8).reshape(n, PARAM_BYTES)

        idx = np.nonzero(types == ORDER_STATUS)[0]
        n = len(idx)
        if n:
            p = np.zeros(n, dtype=ORDERSTATUS_DTYPE)
            p["w"] = rng.integers(1, W + 1, n)
            p["d"] = rng.integers(1, 11, n)
            p["by_name"] = rng.random(n) < self.by_name_frac
            p["c_id"] = nurand(rng, 1023, 1, 3000, self.C_cid, n)
            p["c_last"] = nurand(rng, 255, 0, 999, self.C_last_run, n)
            params[idx] = p.view(np.uint8).reshape(n, PARAM_BYTES)

        idx = np.nonzero(types == DELIVERY)[0]
        n = len(idx)
        if n:
            p = np.zeros(n, dtype=DELIVERY_DTYPE)
            p["w"] = rng.integers(1, W + 1, n)
            p["carrier"] = rng.integers(1, 11, n)
            params[idx] = p.view(np.uint8).reshape(n, PARAM_BYTES)

        idx = np.nonzero(types == STOCK_LEVEL)[0]
        n = len(idx)
        if n:
            p = np.zeros(n, dtype=STOCKLEVEL_DTYPE)
            p["w"] = rng.integers(1, W + 1, n)
            p["d"] = rng.integers(1, 11, n)
            p["threshold"] = rng.integers(10, 21, n)
            params[idx] = p.view(np.uint8).reshape(n, PARAM_BYTES)

        tid = np.arange(tid_start, tid_start + n_txns, dtype=np.uint64)
        return {"tid": tid, "type": types, "params": params}


def home_warehouse(params):
    """Home warehouse of every PROC txn (first u16 of the block) -- used for routing."""
    return params[:, 0].astype(np.int64) | (params[:, 1].astype(np.int64) << 8)
