"""Multi-partition path on one GPU: LTPG_FLAG_LOOPBACK runs P logical
partitions (contiguous key / warehouse ranges) with the same ownership gating,
per-txn verdict exchange (OR of the conflict bits) and result sums as the multi-rank
path; every output must equal the 1-partition run, i.e. the oracle (PIN-8)."""
import numpy as np
import pytest

import oracle
from tests import opscases, tpcc_cc
from tests.test_gpu_ops import check_batch
from tests.test_gpu_tpcc import compare, compare_tables
from workloads import tpcc
from workloads.formats import ST_CONFLICT
from workloads.ycsb import YcsbWorkload

pytestmark = pytest.mark.gpu


def L():
    import paper_conf_icde_wei0l0lzj024_b200 as lib
    return lib


@pytest.mark.parametrize("parts", [2, 3, 4])
@pytest.mark.parametrize("seed", range(6))
def test_ops_loopback_random(parts, seed):
    rng = np.random.default_rng(900 + seed)
    tables = opscases.rand_tables(rng)
    g = L().Database(3, 64, 256, key_space=opscases.RAND_KEY_SPACE, loopback=parts)
    o = oracle.OracleDB(3)
    for t, (grp, add, ng) in opscases.RAND_DESCS.items():
        k, c = tables[t]
        g.load_table(t, grp, add, ng, k, c, capacity=c.shape[1] + 4096, owner_rule=2)
        o.define_table(t, grp, add, ng, True)
        o.load_table(t, k, c)
    for b in range(6):
        batch = opscases.rand_batch(rng, int(rng.integers(1, 60)), tid_start=1 + 100 * b)
        check_batch(g, o, batch, tables)


def test_ycsb_loopback():
    wl = YcsbWorkload(5000, theta=0.8, ops_per_txn=10, seed=12)
    keys, cols = wl.initial_table()
    g = L().ycsb_database(wl, max_txns=2048, max_ops=20480, loopback=4)
    o = oracle.ycsb_db(wl)
    for b in range(3):
        check_batch(g, o, wl.batch(2000, 1 + 2000 * b, b), {0: (keys, cols)})


@pytest.mark.parametrize("mode", ["strict", "delayed"])
@pytest.mark.parametrize("parts", [2, 4])
def test_tpcc_loopback_full_mix(parts, mode):
    W, B = 4, 3000
    wl = tpcc.TpccWorkload(W, seed=33, mode=mode, mix=tpcc.MIX_FULL, remote_line_frac=0.2,
                           remote_cust_frac=0.3)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=5, loopback=parts)
    o = oracle.tpcc_db(wl, tables)
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


def test_tpcc_c5_shape_loopback8():
    """C5 shape (NewOrder/Payment 50/50, 1% remote lines, 15% remote customers) over 8
    warehouse partitions, small scale."""
    W, B = 8, 4096
    wl = tpcc.TpccWorkload(W, seed=0x17C4, mode="strict", mix=tpcc.MIX_NO_PAY)
    tables = wl.initial_tables()
    g = L().tpcc_database(wl, max_txns=B, tables=tables, append_batches=3, loopback=8)
    o = oracle.tpcc_db(wl, tables)
    for bno in range(2):
        compare(g, o, wl.batch(B, 1 + B * bno, bno), 2 + bno)
    compare_tables(g, o)
