"""SURVEY §8(d) secondary CPU baseline: the oracle with O1-O3 on several threads
(orc_set_threads) gives exactly the single-threaded oracle's outputs and state.  CPU only."""
import numpy as np
import pytest

import oracle
from workloads import tpcc
from workloads.formats import ST_CONFLICT
from workloads.ycsb import YcsbWorkload


def _dumps(db, n):
    return [db.dump_table(t) for t in range(n)]


@pytest.mark.parametrize("reorder", [False, True])
@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_tpcc_threads_equal_single(mode, reorder):
    wl = tpcc.TpccWorkload(2, seed=3, mode=mode, mix=tpcc.MIX_FULL, rollback_frac=0.05)
    tables = wl.initial_tables()
    one, many = oracle.tpcc_db(wl, tables), oracle.tpcc_db(wl, tables)
    many.set_threads(7)
    for db in (one, many):
        db.set_reorder(reorder)
    pending, tid = None, 1
    for b in range(3):
        fresh = wl.batch(3000, tid, b)
        tid += 3000
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        r1, s1, x1 = one.run_tpcc(batch, clock=2 + b)
        r2, s2, x2 = many.run_tpcc(batch, clock=2 + b)
        assert r1 == r2 == 0 and (s1 == s2).all() and (x1 == x2).all()
        ab = np.nonzero(s1 == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()}
    for (k1, c1), (k2, c2) in zip(_dumps(one, 9), _dumps(many, 9)):
        assert (k1 is None or (k1 == k2).all()) and (c1 == c2).all()


@pytest.mark.parametrize("reorder", [False, True])
def test_ycsb_threads_equal_single(reorder):
    wl = YcsbWorkload(2000, theta=0.9, ops_per_txn=6, seed=5)
    one, many = oracle.ycsb_db(wl), oracle.ycsb_db(wl)
    many.set_threads(5)
    for db in (one, many):
        db.set_reorder(reorder)
    for b in range(3):
        batch = wl.batch(1500, 1 + 1500 * b, b)
        r1, s1, x1 = one.run_ops(batch)
        r2, s2, x2 = many.run_ops(batch)
        assert r1 == r2 == 0 and (s1 == s2).all() and (x1 == x2).all()
    (k1, c1), (k2, c2) = one.dump_table(0), many.dump_table(0)
    assert (k1 == k2).all() and (c1 == c2).all()
