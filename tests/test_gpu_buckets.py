"""NEXT-3 large-sized hash buckets (Example 2 P:225): with LTPG_FLAG_LARGE_BUCKETS a
popular table (E = T/D > 1) records every mark in sub-slot (TID mod s_u) of its unit's bucket,
s_u = ceil(E/32)*32, and the buckets are folded into the unit marks before detection.  The
bucket layout is invisible in the results: GPU == oracle bit-exactly (PIN-8)."""
import numpy as np
import pytest

import oracle
from tests import opscases, tpcc_cc
from tests.test_gpu_ops import check_batch, make_pair
from tests.test_gpu_tpcc import compare, compare_tables
from workloads import tpcc
from workloads.formats import OP_DTYPE, ST_COMMIT, ST_CONFLICT, UPDATE
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


@pytest.mark.parametrize("reorder", [False, True])
@pytest.mark.parametrize("seed", range(6))
def test_random_ops_large_buckets(seed, reorder):
    """Random OPS batches (all op kinds) on 8-key tables: E = 64/8 > 1, every table popular."""
    rng = np.random.default_rng(7300 + seed)
    tables = opscases.rand_tables(rng)
    flags = L().LTPG_FLAG_LARGE_BUCKETS | (L().LTPG_FLAG_REORDER if reorder else 0)
    g = L().Database(3, 64, 256, flags=flags)
    o = oracle.OracleDB(3)
    o.set_reorder(reorder)
    for t, (grp, add, ng) in opscases.RAND_DESCS.items():
        k, c = tables[t]
        g.load_table(t, grp, add, ng, k, c, capacity=c.shape[1] + 4096)
        o.define_table(t, grp, add, ng, True)
        o.load_table(t, k, c)
    for b in range(6):
        check_batch(g, o, opscases.rand_batch(rng, int(rng.integers(1, 64)), tid_start=1 + 100 * b), tables)


def test_one_hot_key_large_bucket():
    """Closed form (PIN-7): 4096 txns all update key 0 of a 16-row table (E = 256, s_u = 256
    sub-slots) -> only rank 0 commits; every other rank is a WAW abort."""
    wl = YcsbWorkload(16, theta=0.5, ops_per_txn=1, seed=3)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    g, o = make_pair(descs, {0: (keys, cols)}, 4096, 4096, flags=L().LTPG_FLAG_LARGE_BUCKETS)
    n = 4096
    ops = np.zeros(n, dtype=OP_DTYPE)
    ops["key"] = 0
    ops["kind"] = UPDATE
    ops["col"] = 1
    batch = {"tid": np.arange(1, n + 1, dtype=np.uint64), "op_begin": np.arange(n + 1, dtype=np.uint32),
             "ops": ops, "args": np.arange(n, dtype=np.int64) + 1}
    st = check_batch(g, o, batch, {0: (keys, cols)})
    assert st[0] == ST_COMMIT and (st[1:] == ST_CONFLICT).all()


def test_epoch_wrap_large_buckets():
    """Sub-slots are epoch-tagged like the mark words and reset at the 255-batch wrap."""
    wl = YcsbWorkload(32, theta=0.9, ops_per_txn=4, seed=78)
    keys, cols = wl.initial_table()
    descs = {0: tuple(wl.table_desc()[:3])}
    g, o = make_pair(descs, {0: (keys, cols)}, 64, 256, flags=L().LTPG_FLAG_LARGE_BUCKETS)
    tid = 1
    for bno in range(520):
        batch = wl.batch(int(1 + bno % 60), tid, bno)
        tid += len(batch["tid"])
        rc, ost, ord_ = o.run_ops(batch)
        out = g.run_ops(batch)
        assert rc == 0 and (out["status"] == ost).all() and (out["reads"] == ord_).all(), bno
    assert (g.dump_table(0)[1] == o.dump_table(0)[1]).all()


@pytest.mark.parametrize("reorder", [False, True])
@pytest.mark.parametrize("mode", ["strict", "delayed"])
@pytest.mark.parametrize("W", [1, 2])
def test_tpcc_large_buckets(W, mode, reorder):
    """TPC-C full mix, closed loop: WAREHOUSE (E = 3000/W) and DISTRICT (E = 300/W) popular."""
    B = 3000
    wl = tpcc.TpccWorkload(W, seed=91, mode=mode, mix=tpcc.MIX_FULL)
    tables = wl.initial_tables()
    flags = L().LTPG_FLAG_LARGE_BUCKETS | (L().LTPG_FLAG_REORDER if reorder else 0)
    g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=5, flags=flags)
    o = oracle.tpcc_db(wl, tables)
    o.set_reorder(reorder)
    pending, tid = None, 1
    for bno in range(4):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    dumps = compare_tables(g, o)
    assert all(tpcc_cc.check(dumps).values())


@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_realtime_popularity_follows_the_batch(mode):
    """P:215 "identify such tables in real-time": E = T/D with T = the batch's txns accessing the
    table.  Batches of 6, 40, 3000, 3400 and 8 txns on one warehouse (D: WAREHOUSE 1 row, DISTRICT
    10 rows) switch WAREHOUSE / DISTRICT between standard and large buckets
    from batch to batch (ltpg_stats.popular_tables); every batch == oracle."""
    lib = L()
    from workloads.formats import T_WAREHOUSE, T_DISTRICT, T_CUSTOMER, NEW_ORDER, PAYMENT
    W, B = 1, 4096
    wl = tpcc.TpccWorkload(W, seed=61, mode=mode, mix=tpcc.MIX_NO_PAY)
    tables = wl.initial_tables()
    g = lib.tpcc_database(wl, max_txns=B, tables=tables, append_batches=3, flags=lib.LTPG_FLAG_LARGE_BUCKETS)
    o = oracle.tpcc_db(wl, tables)
    std, large, su = g.mark_memory(T_WAREHOUSE)
    assert su == 4096 and large > 0                       # allocated for E <= 4096 / 1
    assert g.mark_memory(T_DISTRICT)[2] == 416            # ceil(4096 / 10 / 32) * 32
    assert g.mark_memory(T_CUSTOMER)[2] == 1              # 30,000 rows > 4096: never popular
    tid = 1
    for bno, (n, types) in enumerate([(6, [NEW_ORDER] * 6), (40, None), (3000, [PAYMENT] * 1500 + [NEW_ORDER] * 1500),
                                      (3400, [PAYMENT] * 3100 + [NEW_ORDER] * 300), (8, None)]):
        b = wl.batch(n, tid, bno, types=types)
        tid += n
        rc, ost, ores = o.run_tpcc(b, 2 + bno)
        out = g.run_tpcc(b, 2 + bno, stats=True)
        assert rc == 0 and (out["status"] == ost).all() and (out["reads"] == ores).all()
        pop = out["stats"]["popular_tables"]
        T = n  # every NewOrder / Payment accesses WAREHOUSE, DISTRICT and CUSTOMER
        assert bool(pop >> T_WAREHOUSE & 1) == (T > 1), (n, pop)
        assert bool(pop >> T_DISTRICT & 1) == (T > 10), (n, pop)
        assert not pop >> T_CUSTOMER & 1
    compare_tables(g, o)
