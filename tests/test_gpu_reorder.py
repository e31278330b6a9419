"""NEXT-1 logical reordering (Aria): LTPG_FLAG_REORDER keeps per-unit minimum reader
marks and aborts iff WAW or (RAW and WAR).  GPU == oracle (orc_set_reorder) bit-exactly."""
import numpy as np
import pytest

import oracle
from tests import opscases, tpcc_cc
from tests.test_gpu_ops import check_batch
from tests.test_gpu_tpcc import compare, compare_tables
from workloads import tpcc
from workloads.formats import ST_COMMIT, ST_CONFLICT

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


def pair_ops(descs, tables, flags, loopback=1, key_space=0, owner_rule=0, extra=4096):
    g = L().Database(max(descs) + 1, 64, 256, flags=flags, loopback=loopback, key_space=key_space)
    o = oracle.OracleDB(max(descs) + 1)
    o.set_reorder(True)
    for t, (grp, add, ng) in descs.items():
        k, c = tables[t]
        g.load_table(t, grp, add, ng, k, c, capacity=c.shape[1] + extra, owner_rule=owner_rule)
        o.define_table(t, grp, add, ng, True)
        o.load_table(t, k, c)
    return g, o


def test_example3_reordering_gpu():
    descs, tables, batch, gold = opscases.example3("row_level_reordering")
    g, o = pair_ops(descs, tables, L().LTPG_FLAG_REORDER)
    st = check_batch(g, o, batch, tables)
    assert [i + 1 for i, s in enumerate(st) if s == ST_COMMIT] == [1, 2, 3, 5]


@pytest.mark.parametrize("loopback", [1, 3])
@pytest.mark.parametrize("seed", range(10))
def test_random_reordering(seed, loopback):
    rng = np.random.default_rng(4100 + seed)
    tables = opscases.rand_tables(rng)
    g, o = pair_ops(opscases.RAND_DESCS, tables, L().LTPG_FLAG_REORDER, loopback=loopback,
                    key_space=opscases.RAND_KEY_SPACE, owner_rule=2)
    for b in range(5):
        check_batch(g, o, opscases.rand_batch(rng, int(rng.integers(1, 60)), tid_start=1 + 100 * b), tables)


@pytest.mark.parametrize("loopback", [1, 2])
@pytest.mark.parametrize("mode", ["strict", "delayed"])
def test_tpcc_reordering(mode, loopback):
    W, B = 2, 3000
    wl = tpcc.TpccWorkload(W, seed=71, mode=mode, mix=tpcc.MIX_FULL, remote_line_frac=0.1,
                           remote_cust_frac=0.2)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=5, loopback=loopback,
                          flags=L().LTPG_FLAG_REORDER)
    o = oracle.tpcc_db(wl, tables)
    o.set_reorder(True)
    base = oracle.tpcc_db(wl, tables)
    pending, tid, more = None, 1, 0
    for bno in range(4):
        fresh = wl.batch(B - (0 if pending is None else len(pending["tid"])), tid, bno)
        tid += len(fresh["tid"])
        batch = fresh if pending is None else {k: np.concatenate([pending[k], fresh[k]]) for k in fresh}
        st = compare(g, o, batch, 2 + bno)
        if bno == 0:  # reordering commits the read-only StockLevel / OrderStatus txns
            _, st_base, _ = base.run_tpcc(batch, 2)
            more = int((st == ST_COMMIT).sum() - (st_base == ST_COMMIT).sum())
        ab = np.nonzero(st == ST_CONFLICT)[0]
        pending = {k: v[ab] for k, v in batch.items()} if len(ab) else None
    assert more > 0
    dumps = compare_tables(g, o)
    assert all(tpcc_cc.check(dumps).values())
