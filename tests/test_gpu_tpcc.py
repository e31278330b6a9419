"""GPU parity, TPC-C PROC mode: the CUDA stored procedures through the C-ABI vs
the CPU oracle -- status, 4 result slots per txn and every table's canonical
dump, bit-exact; TPC-C consistency conditions on the GPU's own state."""
import numpy as np
import pytest

import oracle
from tests import tpcc_cc
from workloads import tpcc
from workloads.formats import ST_COMMIT, ST_CONFLICT, NEW_ORDER, PAYMENT, DELIVERY

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


def pair(W, mode, mix, max_txns, batches, seed=5):
    wl = tpcc.TpccWorkload(W, seed=seed, mode=mode, mix=mix)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=max_txns, tables=tables, append_batches=batches + 1)
    o = oracle.tpcc_db(wl, tables)
    return wl, g, o


def compare(g, o, batch, clock):
    rc, ost, ores = o.run_tpcc(batch, clock)
    assert rc == 0
    out = g.run_tpcc(batch, clock)
    bad = np.nonzero(out["status"] != ost)[0]
    assert len(bad) == 0, ("status", bad[:10], batch["type"][bad[:10]], out["status"][bad[:10]], ost[bad[:10]])
    diff = np.nonzero((out["reads"] != ores).any(axis=1))[0]
    assert len(diff) == 0, ("results", diff[:5], batch["type"][diff[:5]], out["reads"][diff[:5]], ores[diff[:5]])
    assert (out["abort_idx"] == np.nonzero(ost == ST_CONFLICT)[0]).all()
    return ost


def compare_tables(g, o):
    dumps = {}
    for t in range(9):
        gk, gc = g.dump_table(t)
        ok, oc = o.dump_table(t)
        assert gc.shape == oc.shape, (t, gc.shape, oc.shape)
        if ok is not None:
            assert (gk == ok).all(), t
        assert (gc == oc).all(), (t, np.nonzero((gc != oc).any(axis=0))[0][:5])
        dumps[t] = (gk, gc)
    return dumps


@pytest.mark.parametrize("mode", ["strict", "delayed"])
@pytest.mark.parametrize("W", [1, 2])
def test_full_mix_closed_loop(W, mode):
    B = 3000
    wl, g, o = pair(W, mode, tpcc.MIX_FULL, B, 6)
    pending = None
    tid = 1
    for bno in range(5):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    dumps = compare_tables(g, o)
    cc = tpcc_cc.check(dumps)
    assert all(cc.values()), cc


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_c2_one_warehouse_16k(mode):
    """BASELINE configs[1]: TPC-C 1 warehouse, NewOrder+Payment, batch 16k."""
    wl, g, o = pair(1, mode, tpcc.MIX_NO_PAY, 16384, 3, seed=0x17C1)
    tid = 1
    for bno in range(2):
        batch = wl.batch(16384, tid, bno)
        tid += 16384
        st = compare(g, o, batch, 2 + bno)
        if mode == "strict":
            assert ((batch["type"] == PAYMENT) & (st == ST_COMMIT)).sum() == 1  # Table VI-style: 1 per warehouse
    compare_tables(g, o)


def test_table6_gpu():
    """Table VI "no" row 8/16,384 reproduced by the GPU path (== oracle)."""
    wl, g, o = pair(8, "strict", tpcc.MIX_NO_PAY, 16384, 1, seed=0x17C0 + 8)
    batch = wl.batch(16384, 1, 0)
    st = compare(g, o, batch, 2)
    no = batch["type"] == NEW_ORDER
    rate = 100.0 * (no & (st == ST_COMMIT)).sum() / no.sum()
    assert ((batch["type"] == PAYMENT) & (st == ST_COMMIT)).sum() == 8
    assert abs(rate - 63.4) <= 2.0


@pytest.mark.parametrize("path", ["single", "multi"])
def test_tpcc_validation_and_capacity(path):
    lib = L()
    wl = tpcc.TpccWorkload(1, seed=3, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=512, tables=tables, append_batches=1,
                          flags=lib.LTPG_FLAG_NO_SINGLE_LAUNCH if path == "multi" else 0)
    b = wl.batch(100, 1, 0)
    b["params"][5, 0] = 9  # warehouse 9 does not exist
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(b, 2)
    assert e.value.rc == lib.LTPG_EINVAL
    bt = wl.batch(100, 1, 0)
    bt["tid"][40] = bt["tid"][39]  # TIDs must be strictly increasing
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(bt, 2)
    assert e.value.rc == lib.LTPG_EINVAL
    # capacity: append region sized for one batch of 512; two full batches of NewOrders overflow
    o = oracle.tpcc_db(wl, tables)
    nb = wl.batch(512, 1000, 1, types=[NEW_ORDER] * 512)
    compare(g, o, nb, 3)
    nb2 = wl.batch(512, 5000, 2, types=[NEW_ORDER] * 512)
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(nb2, 4)
    assert e.value.rc == lib.LTPG_ECAPACITY
    compare_tables(g, o)  # nothing changed by the rejected batch


def test_delivery_heavy():
    """Delivery drains NEW_ORDER queues across batches (cursor, delete, carrier, OL dates, balance)."""
    wl, g, o = pair(1, "strict", (0.3, 0.0, 0.0, 0.7, 0.0), 256, 12)
    tid = 1
    for bno in range(10):
        batch = wl.batch(200, tid, bno)
        tid += 200
        compare(g, o, batch, 2 + bno)
    dumps = compare_tables(g, o)
    assert all(tpcc_cc.check(dumps).values())


def test_packed_params_equal_fixed_blocks():
    """proc_offsets: packed parameter blocks (used prefixes only) give the same results."""
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=17, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=2048, tables=tables, append_batches=4)
    o = oracle.tpcc_db(wl, tables)
    for bno in range(3):
        b = wl.batch(2000, 1 + 2000 * bno, bno)
        packed, offs = lib.pack_params(b["type"], b["params"])
        assert packed.nbytes < b["params"].nbytes * 0.6
        pb = {"tid": b["tid"], "type": b["type"], "params": packed, "offsets": offs}
        out = g.run_tpcc(pb, 2 + bno)
        rc, st, res = o.run_tpcc(b, 2 + bno)
        assert (out["status"] == st).all() and (out["reads"] == res).all()
    compare_tables(g, o)
    bad = dict(pb)
    bad["offsets"] = offs.copy()
    bad["offsets"][1:] += 200  # first block 200+ bytes long
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(bad, 9)
    assert e.value.rc == lib.LTPG_EINVAL


def test_deferred_orderline_index_then_ops_lookup():
    """New ORDER_LINE rows skip the PK-index insert at write-back (reached via ORDER.aux); an
    OPS batch afterwards must still find them by key (the index is caught up first)."""
    from tests.opscases import make_batch
    from workloads.formats import T_ORDER_LINE, SELECT, SCAN, tpcc_col
    lib = L()
    wl = tpcc.TpccWorkload(1, seed=21, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=2048, tables=tables, append_batches=5, max_ops=4096)
    o = oracle.tpcc_db(wl, tables)
    for bno in range(3):
        compare(g, o, wl.batch(2000, 1 + 2000 * bno, bno), 2 + bno)
    keys, _ = o.dump_table(T_ORDER_LINE)
    rng = np.random.default_rng(3)
    pick = np.concatenate([keys[-300:], rng.choice(keys, 200)])  # newest lines + old ones
    amt = tpcc_col(T_ORDER_LINE, "OL_AMOUNT")
    txns = [[(int(k), SELECT, T_ORDER_LINE, amt, 0, 0)] for k in pick]
    txns.append([(int(keys[-1]) + 1, SELECT, T_ORDER_LINE, amt, 0, 0)])  # absent
    txns.append([(int(keys[-20]), SCAN, T_ORDER_LINE, amt, 40, 0)])
    batch = make_batch(txns, tid_start=100000)
    rc, ost, ord_ = o.run_ops(batch)
    out = g.run_ops(batch)
    assert rc == 0 and (out["status"] == ost).all() and (out["reads"] == ord_).all()
    compare(g, o, wl.batch(2000, 200000, 7), 9)
    compare_tables(g, o)


def test_stocklevel_shared_per_district_any_threshold():
    """StockLevel is evaluated once per district (prefix table over S_QUANTITY) and shared by
    the batch's StockLevels of that district: every threshold 0..255, mixed with NewOrders
    that write the stock rows (RAW for larger ranks), equals the oracle."""
    from workloads.formats import STOCK_LEVEL
    wl, g, o = pair(2, "strict", tpcc.MIX_FULL, 4096, 4, seed=31)
    compare(g, o, wl.batch(3000, 1, 0), 2)
    rng = np.random.default_rng(5)
    types = [STOCK_LEVEL] * 1500 + [NEW_ORDER] * 300
    rng.shuffle(types)
    b = wl.batch(1800, 10000, 1, types=types)
    sl = b["type"] == STOCK_LEVEL
    b["params"][sl, 3] = rng.integers(0, 256, sl.sum()).astype(np.uint8)
    st = compare(g, o, b, 3)
    assert (st[sl] == ST_COMMIT).any() and (st[sl] == ST_CONFLICT).any()
    compare(g, o, wl.batch(2000, 20000, 2), 4)
    compare_tables(g, o)


def test_compact_params_equal_fixed_blocks():
    """LTPG_BATCH_COMPACT_PARAMS: compact records (u32 NewOrder lines, remote supply lists,
    u32 Payment amounts) expanded on the GPU give the oracle's results; a record whose length
    contradicts its header is EINVAL with nothing changed."""
    lib = L()
    wl = tpcc.TpccWorkload(3, seed=19, mix=tpcc.MIX_FULL, remote_line_frac=0.25)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=3000, tables=tables, append_batches=4)
    o = oracle.tpcc_db(wl, tables)
    for bno in range(3):
        b = wl.batch(2999, 1 + 3000 * bno, bno)  # ragged: not a multiple of 32
        packed, offs = lib.pack_params_compact(b["type"], b["params"])
        pb = {"tid": b["tid"], "type": b["type"], "params": packed, "offsets": offs, "compact": True}
        out = g.run_tpcc(pb, 2 + bno)
        rc, st, res = o.run_tpcc(b, 2 + bno)
        assert (out["status"] == st).all() and (out["reads"] == res).all()
    compare_tables(g, o)
    no = int(np.nonzero(b["type"] == 0)[0][0])
    bad = dict(pb)
    bad["offsets"] = offs.copy()
    bad["offsets"][no + 1:] -= 2  # NewOrder record 2 bytes short of its header
    bad["params"] = np.delete(packed, offs[no + 1] - 1)[: len(packed) - 1]
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(bad, 9)
    assert e.value.rc == lib.LTPG_EINVAL
    compare_tables(g, o)  # nothing changed


def test_many_districts_tiled_colscan():
    """More than 2048 district keys (210 warehouses) switch the o_id column scan to the tiled
    kernel (k_no_colscan_tiled): verdicts, o_id results and the DISTRICT / ORDER / NEW_ORDER
    state equal the oracle over a closed loop of NewOrder/Payment batches."""
    W, B = 210, 8192
    wl = tpcc.TpccWorkload(W, seed=21, mode="strict", mix=tpcc.MIX_NO_PAY)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=4)
    o = oracle.tpcc_db(wl, tables)
    pending, tid = None, 1
    for bno in range(3):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        assert (st == 1).sum() > B // 16
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    from workloads.formats import T_WAREHOUSE, T_DISTRICT, T_ORDER, T_NEW_ORDER
    for t in (T_WAREHOUSE, T_DISTRICT, T_ORDER, T_NEW_ORDER):
        gk, gc = g.dump_table(t)
        ok, oc = o.dump_table(t)
        assert (gk == ok).all() and gc.shape == oc.shape and (gc == oc).all(), t


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_ten_repeated_runs_identical(mode):
    """PIN-8: the same closed loop run 10 times on fresh databases gives identical verdicts,
    results and canonical state every time (atomics race in a different order on each run;
    min marks, commutative adds and rank-ordered appends make the outcome unique, R20)."""
    W, B = 2, 3000
    wl = tpcc.TpccWorkload(W, seed=13, mode=mode, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    ref = None
    for run in range(10):
        g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=5)
        outs, pending, tid = [], None, 1
        for bno in range(4):
            fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
            tid += len(fresh["tid"])
            batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
            out = g.run_tpcc(batch, 2 + bno)
            outs.append((out["status"].copy(), out["reads"].copy()))
            ab = np.nonzero(out["status"] == ST_CONFLICT)[0]
            pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
        dumps = [g.dump_table(t) for t in range(9)]
        g.close()
        if ref is None:
            ref = (outs, dumps)
            continue
        for (s0, r0), (s1, r1) in zip(ref[0], outs):
            assert (s0 == s1).all() and (r0 == r1).all(), run
        for (k0, c0), (k1, c1) in zip(ref[1], dumps):
            assert (k0 is None or (k0 == k1).all()) and (c0 == c1).all(), run


@pytest.mark.parametrize("what", ["item0", "item_big", "qty0", "qty11", "supply_w", "dup_item", "dup_far"])
@pytest.mark.parametrize("path", ["single", "multi"])
def test_neworder_line_validation_in_execute(what, path):
    """Unpartitioned batches validate NewOrder lines in execute (the grouping kernel reads only
    the 16-byte headers): every malformed line is EINVAL with nothing changed, and the database
    keeps running the next batch == oracle."""
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=23, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=1024, tables=tables, append_batches=3)
    o = oracle.tpcc_db(wl, tables)
    if path == "multi":  # (batches this small run as one cooperative launch unless told otherwise)
        g = lib.tpcc_database(wl, max_txns=1024, tables=tables, append_batches=3, flags=lib.LTPG_FLAG_NO_SINGLE_LAUNCH)
    b = wl.batch(1000, 1, 0)
    no = np.nonzero((b["type"] == NEW_ORDER) & (b["params"][:, 3] >= 14))[0][3]
    p = b["params"][no]
    line = lambda l: p[8 + 8 * l: 16 + 8 * l]  # noqa: E731
    if what == "item0":
        line(2)[:4] = 0
    elif what == "item_big":
        line(13)[:4] = np.array([100002], "<u4").view(np.uint8)
    elif what == "qty0":
        line(0)[6] = 0
    elif what == "qty11":
        line(5)[6] = 11
    elif what == "supply_w":
        line(7)[4:6] = np.array([3], "<u2").view(np.uint8)   # W = 2
    elif what == "dup_item":
        line(1)[:4] = line(2)[:4]                          # same lane (lines 0..3)
    elif what == "dup_far":
        line(13)[:4] = line(0)[:4]                         # lanes 0 and 3
    assert o.run_tpcc(b, 2)[0] == oracle.ORC_EINVAL
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(b, 2)
    assert e.value.rc == lib.LTPG_EINVAL
    compare_tables(g, o)                                   # nothing changed
    compare(g, o, wl.batch(1000, 5000, 1), 3)              # and the db still works
    compare_tables(g, o)


@pytest.mark.parametrize("ptype,off,val", [
    (NEW_ORDER, 0, 3), (NEW_ORDER, 2, 11), (NEW_ORDER, 3, 0), (NEW_ORDER, 3, 16), (NEW_ORDER, 4, 0),
    (PAYMENT, 0, 0), (PAYMENT, 2, 0), (PAYMENT, 3, 2), (PAYMENT, 4, 5), (PAYMENT, 6, 12),
    (2, 0, 7), (2, 2, 0), (2, 3, 3), (DELIVERY, 0, 9), (DELIVERY, 2, 11), (4, 0, 0), (4, 2, 15),
])
@pytest.mark.parametrize("path", ["single", "multi"])
def test_header_validation_every_type(ptype, off, val, path):
    """Each procedure's header checks (grouping for Delivery / StockLevel, execute for the others in
    an unpartitioned batch): a bad field is EINVAL, nothing changes, the db keeps working == oracle."""
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=29, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=1024, tables=tables, append_batches=3)
    o = oracle.tpcc_db(wl, tables)
    if path == "multi":  # (batches this small run as one cooperative launch unless told otherwise)
        g = lib.tpcc_database(wl, max_txns=1024, tables=tables, append_batches=3, flags=lib.LTPG_FLAG_NO_SINGLE_LAUNCH)
    b = wl.batch(1000, 1, 0)
    i = int(np.nonzero(b["type"] == ptype)[0][2])
    b["params"][i, off] = val
    if off in (0, 4) and val < 256:
        b["params"][i, off + 1] = 0
    assert o.run_tpcc(b, 2)[0] == oracle.ORC_EINVAL
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(b, 2)
    assert e.value.rc == lib.LTPG_EINVAL
    compare_tables(g, o)
    compare(g, o, wl.batch(1000, 5000, 1), 3)


def test_l2_persist_marks_result_identical():
    """LTPG_FLAG_L2_PERSIST_MARKS (an L2 persisting window over the largest mark array) is a
    cache hint only: a closed loop with it == oracle."""
    lib = L()
    wl = tpcc.TpccWorkload(2, seed=37, mode="strict", mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=3000, tables=tables, append_batches=4, flags=lib.LTPG_FLAG_L2_PERSIST_MARKS)
    o = oracle.tpcc_db(wl, tables)
    pending, tid = None, 1
    for bno in range(3):
        fresh = wl.batch(3000 - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    compare_tables(g, o)


def test_reads_cap_einval():
    """ltpg_result.reads_cap: a reads buffer smaller than the batch's result slots is EINVAL
    before any state change; the db keeps working == oracle."""
    lib = L()
    wl, g, o = pair(1, "strict", tpcc.MIX_FULL, 512, 3, seed=31)
    b = wl.batch(300, 1, 0)
    out = g._outputs(300, 4 * 300, False)
    out["reads"] = np.empty(4 * 300 - 1, np.int64)
    with pytest.raises(lib.LtpgError) as e:
        g.run_tpcc(b, 2, out=out)
    assert e.value.rc == lib.LTPG_EINVAL
    compare_tables(g, o)
    compare(g, o, b, 2)
    compare_tables(g, o)
